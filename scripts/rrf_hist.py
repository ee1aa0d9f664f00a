import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
from paper_conf_ipps_zhangdmwbf17_b200 import sf, inputs as I
for n in (int(a) for a in sys.argv[1:]):
    res = {}
    for on in ("0", "1"):
        os.environ["SF_RRF"] = on
        h = I.level_h(n, n, n)
        L = sf.Level(n, n, n, h)
        L.set_coeffs(*I.hpgmg_coeffs(n, n, n, h))
        L.upload(sf.SF_F, I.manufactured(n, n, n, 1.0, 1.0, h)[1])
        M = sf.MG(L, 1.0, 1.0)
        st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
        res[on] = (cyc, np.array(hist), L.download(sf.SF_U))
        M.close(); L.close()
    h0, h1 = res["0"][1], res["1"][1]
    print(n, "cycles", res["0"][0], res["1"][0])
    for a, b in zip(h0, h1):
        print(f"  {a:.6e} {b:.6e} rel {abs(a-b)/a:.2e} abs {abs(a-b):.2e}")
    u0, u1 = res["0"][2], res["1"][2]
    print("  u rel-L2", np.linalg.norm(u0 - u1) / np.linalg.norm(u0), "max", np.abs(u0 - u1).max())
