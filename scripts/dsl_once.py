"""Run the generic engine's A3 and RB pair once at n^3 (for ncu)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhangdmwbf17_b200 import sf, stencil as SD
n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
G = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(G.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(G.handle, 1.0, 1.0)
op = SD.hpgmg_apply_op(1.0, 1.0, 1.0 / n).compile()
pair = SD.hpgmg_gsrb_pair(1.0, 1.0, 1.0 / n).compile()
op(G)
pair(G)
sf.sf_sync(G.handle)
print("ok")
