"""SURVEY 8(d) "oracle timed beside it": the CPU oracle on BASELINE's configs,
at 1 thread and at all host cores, with the host CPU model.

    python scripts/oracle_table.py > profiles/r02/oracle_table.json

C1: 16^3 CC Poisson, 2 RB pairs (4 sweeps) + residual.  C2: 64^3 VC Helmholtz
V-cycle solve from u = 0 to 1e-10.  C3: one RB pair on the 256^3 VC level.
C4/C5: one F-cycle and one complete solve (F + V to 1e-10) at 512^3 when the
host has the memory.  The oracle's OpenMP build runs every case; with one
thread it is the single-thread arithmetic the parity tests use.
"""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from oracle import oracle as O  # noqa: E402
from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I  # noqa: E402


def lscpu():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        d = {}
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() in ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core",
                             "CPU(s)", "NUMA node(s)", "L3 cache"):
                d[k.strip()] = v.strip()
        return d
    except Exception as e:  # noqa: BLE001
        return {"error": repr(e)}


def timed(fn, reps=1):
    best = None
    for _ in range(reps):
        t0 = time.perf_counter()
        r = fn()
        dt = time.perf_counter() - t0
        best = dt if best is None or dt < best else best
    return best, r


def main():
    O.use_openmp(True)
    lib = O.lib()
    allc = len(os.sched_getaffinity(0))
    res = {"cpu": lscpu(), "affinity_cores": allc, "cases": {}}
    import psutil
    big = psutil.virtual_memory().available > 512**3 * 8 * 40
    for threads in (1, allc):
        used = lib.or_set_threads(threads)
        row = {"threads": used}
        # C1
        n = 16
        h = 1.0 / n
        P = O.Problem(O.Grid(n, n, n, h), 0.0, 1.0, *I.constant_coeffs(n, n, n))
        x, f = I.random_field((n, n, n), 0), I.random_field((n, n, n), 1)
        d = P.dinv()
        t, _ = timed(lambda: P.residual(P.smooth(x, f, 2, dinv=d), f), reps=5)
        row["c1_16_pairs2_residual_ms"] = t * 1e3
        # C2
        n = 64
        h = 1.0 / n
        co = I.hpgmg_coeffs(n, n, n, h)
        _, f = I.manufactured(n, n, n, 1.0, 1.0, h)
        M = O.MG(n, n, n, h, 1.0, 1.0, *co)
        t, (u, hist) = timed(lambda: M.solve(f, fcycle=False, rtol=1e-10), reps=2)
        row["c2_64_vsolve"] = {"ms": t * 1e3, "cycles": len(hist), "dof_s": n**3 / t}
        del M
        # C3
        n = 256
        h = 1.0 / n
        co = I.hpgmg_coeffs(n, n, n, h)
        P = O.Problem(O.Grid(n, n, n, h), 1.0, 1.0, *co)
        x, f = I.random_field((n, n, n), 0), I.random_field((n, n, n), 1)
        d = P.dinv()
        t, _ = timed(lambda: P.smooth(x, f, 1, dinv=d), reps=2)
        row["c3_256_rb_pair"] = {"ms": t * 1e3, "point_updates_s": n**3 / t,
                                 "alg_gbs_64B": 64 * n**3 / t / 1e9}
        del P, co, x, f, d
        # C4 / C5
        if big:
            n = 512
            h = 1.0 / n
            co = I.hpgmg_coeffs(n, n, n, h)
            _, f = I.manufactured(n, n, n, 1.0, 1.0, h)
            M = O.MG(n, n, n, h, 1.0, 1.0, *co)
            del co
            t, _ = timed(lambda: M.fcycle(f))
            row["c4_512_fcycle"] = {"s": t, "dof_s": n**3 / t}
            if threads > 1:
                t, (u, hist) = timed(lambda: M.solve(f, fcycle=True, rtol=1e-10))
                row["c5_512_solve"] = {"s": t, "cycles": len(hist), "dof_s": n**3 / t,
                                       "final_relres": hist[-1]}
            del M, f
        res["cases"][f"threads_{used}"] = row
        print(json.dumps(row), file=sys.stderr, flush=True)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
