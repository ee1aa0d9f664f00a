"""Profiling driver: the fused pair + delta-form residual + restriction
(sf_smooth_residual_restrict) at n^3, three calls (ncu -k regex:gsrb_pair_tma
--launch-skip 2 --launch-count 1 captures the third).   python scripts/prof_rrf.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402,F401

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n, stream=L.stream)
for _ in range(3):
    sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F)
L.stream.synchronize()
