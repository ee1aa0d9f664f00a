"""Drive the RESID (solve check) and INTERP (V-cycle post) fused-pair variants at
512^3 without graphs, for ncu captures of each variant (scripts/prof_variants.sh)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhangdmwbf17_b200 import sf
n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
mode = sys.argv[2] if len(sys.argv) > 2 else "vcycle"
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0, use_graph=0)
if mode == "vcycle":
    sf.sf_vcycle(M.handle, 0)
elif mode == "fcycle":
    sf.sf_fcycle(M.handle)
else:
    M.solve(fcycle=False, max_cycles=2, raise_on_error=False)
sf.sf_sync(L.handle)
print("done", mode)
