import os, sys
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
import numpy as np
from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I, sf
from oracle import oracle as O
n = 64; h = 1.0 / n
coeffs = I.hpgmg_coeffs(n, n, n, h)
_, f = I.manufactured(n, n, n, 1.0, 1.0)
for pre, post in ((1, 1), (2, 2)):
    L = sf.Level(n, n, n, h); L.set_coeffs(*coeffs); L.upload(sf.SF_F, f)
    M = sf.MG(L, 1.0, 1.0, pre_pairs=pre, post_pairs=post, use_graph=0)
    st, cyc, hist = M.solve(False, 1e-10, 50, raise_on_error=False)
    Om = O.MG(n, n, n, h, 1.0, 1.0, *coeffs, pre=pre, post=post)
    u_o, hist_o = Om.solve(f, fcycle=False, rtol=1e-10)
    print(os.environ.get("SF_LIB", "shipped"), os.environ.get("SF_COARSE_KERNEL", "-"), pre, post, "gpu", st, cyc, [f"{v:.2e}" for v in hist[:6]], "oracle", len(hist_o), [f"{v:.2e}" for v in hist_o[:6]], flush=True)
    M.close(); L.close()
