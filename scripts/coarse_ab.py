"""Solve time with and without the coarse cluster V-cycle (SF_COARSE_KERNEL),
same session: C2's 64^3 V-solve and F+V solves at 128^3..512^3.
    python scripts/coarse_ab.py [n ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def solve_ms(n, kernel, fcycle, reps):
    os.environ["SF_COARSE_KERNEL"] = kernel
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    z = np.zeros((n, n, n))
    for _ in range(3):
        if not fcycle:
            L.upload(sf.SF_U, z)
        st, cyc, hist = M.solve(fcycle, 1e-10, 50)
    ts = []
    for _ in range(reps):
        if not fcycle:
            L.upload(sf.SF_U, z)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st, cyc, hist = M.solve(fcycle, 1e-10, 50)
        ts.append(time.perf_counter() - t0)
    M.close()
    L.close()
    return min(ts) * 1e3, cyc, hist[-1]


for n in [int(v) for v in sys.argv[1:]] or [64, 128, 256, 512]:
    for fc in ((False, True) if n == 64 else (True,)):
        r = {k: solve_ms(n, k, fc, 20 if n <= 128 else 5) for k in ("0", "1", "0", "1")}
        print(f"n={n} {'F+V' if fc else 'V  '} per-phase launches {r['0'][0]:.3f} ms  cluster kernel "
              f"{r['1'][0]:.3f} ms  ({n**3 / r['1'][0] / 1e6:.3f} GDOF/s)  cycles {r['0'][1]}/{r['1'][1]}"
              f"  relres {r['0'][2]:.2e}/{r['1'][2]:.2e}", flush=True)
