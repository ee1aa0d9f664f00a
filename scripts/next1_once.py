"""One 512^3 smooth (2 RB pairs) of the given smoother kind inside a profiler
range (for ncu --profile-from-start off): 2 = two fused pairs, 4 = NEXT-1.
    python scripts/next1_once.py n kind"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n, kind = int(sys.argv[1]), int(sys.argv[2])
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
