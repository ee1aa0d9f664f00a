"""One 512^3 solve (F + V to 1e-10) for an ncu launch list of the timed step."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
graph = int(sys.argv[2]) if len(sys.argv) > 2 else 0
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0, use_graph=graph)
st, cyc, hist = M.solve(True, 1e-10, 50)          # warm-up
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
st, cyc, hist = M.solve(True, 1e-10, 50)          # profiled step
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("cycles", cyc, "relres", hist[-1])
