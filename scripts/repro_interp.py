import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_ipps_zhangdmwbf17_b200 import sf, inputs as I
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32
L = sf.Level(n, n, n, 1.0 / n)
L.set_coeffs(*I.hpgmg_coeffs(n, n, n))
M = sf.MG(L, 1.0, 1.0, use_graph=0)
_, f = I.manufactured(n, n, n, 1.0, 1.0)
L.upload(sf.SF_F, f)
M.vcycle(0)
print("ok", np.abs(L.download(sf.SF_U)).max())
