"""P0-fused pair at n^3 with its coarse source e warm in L2 (back-to-back calls)
vs cold (a plain pair on the same level streams ~8 GB through L2 between
calls), in-kernel timed per launch by variant (sf_level_pair_timing).
    python scripts/interp_cold.py [n]"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402,F401

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
Cl = sf.Level(n // 2, n // 2, n // 2, 2.0 / n, stream=L.stream)
plain = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)  # noqa: E731
interp = lambda: sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_U)  # noqa: E731


def run(mode, reps=20):
    for _ in range(3):
        interp()
        plain()
    sf.sf_level_pair_timing(L.handle, 1)
    for _ in range(reps):
        if mode == "cold":
            plain()
        interp()
    sf.sf_level_pair_timing(L.handle, 0)
    ms = (C.c_double * 4)()
    cnt = (C.c_longlong * 4)()
    sf.lib().sf_level_pair_timing_variants(L.handle, ms, cnt)
    return ms[0], ms[3]


for rep in range(2):
    for mode in ("warm", "cold"):
        p, i = run(mode)
        print(f"n={n} {mode}: plain {p:.4f} ms  P0-fused {i:.4f} ms", flush=True)
