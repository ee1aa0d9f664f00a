"""One eager V-cycle of an n^3 hierarchy (for ncu launch lists).
    python scripts/vcycle_once_n.py n"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
M.vcycle(0)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
M.vcycle(0)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
