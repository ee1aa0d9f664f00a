"""Coarse V-cycle kernel cost vs smoothing pairs and entry size: one eager
V-cycle per (n, pre, post) inside a profiler range (run under ncu with
--profile-from-start off; the coarse kernel's duration is read from its list).
    python scripts/coarse_phase_cost.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

CASES = [(32, 2, 2), (32, 1, 1), (32, 0, 0), (16, 2, 2), (16, 0, 0)]
for n, pre, post in CASES:
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0, pre_pairs=pre, post_pairs=post, use_graph=0)
    M.vcycle(0)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStart()
    M.vcycle(0)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()
    print(n, pre, post, flush=True)
    M.close()
    L.close()
