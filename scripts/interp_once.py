"""One P0-fused pair (sf_interpolate_smooth) and one plain pair at n^3 inside a
profiler range (ncu --profile-from-start off).
    python scripts/interp_once.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n, stream=L.stream)
sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_U)
sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_U)
sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
