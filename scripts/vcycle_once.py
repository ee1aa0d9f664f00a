import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhangdmwbf17_b200 import sf
n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0, use_graph=0)
for _ in range(2):
    sf.sf_vcycle(M.handle, 0)
sf.sf_sync(L.handle)
