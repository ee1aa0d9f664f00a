"""Profiling driver: the P0-fused pair (sf_interpolate_smooth) and the plain
fused pair on the same 512^3 level, same build (32x16 with SF_GSRB_W4=0, the
P0-fused pair's build on big levels).  ncu -k regex:gsrb_pair_tma ...
    python scripts/prof_interp.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("SF_GSRB_W4", "0")
import torch  # noqa: E402,F401

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n, stream=L.stream)
for _ in range(3):   # launches 0-2 plain, 3-5 P0-fused
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
for _ in range(3):
    sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_U)
L.stream.synchronize()
