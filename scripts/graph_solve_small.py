import os, sys
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_zhangdmwbf17_b200 import sf
L = sf.Level(32, 32, 32, 1.0 / 32)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, raise_on_error=False)
sf.sf_sync(L.handle)
print("ok graph solve", st, cyc, flush=True)
