"""Where does the fused pair+residual+restriction differ from the plain fused pair?"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I  # noqa: E402
from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

for shape in [(4, 16, 32), (8, 32, 64), (64, 64, 64)]:
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 5)
    Ls = []
    for k in range(2):
        L = sf.Level(nx, ny, nz, h)
        L.set_coeffs(*coeffs)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, I.random_field(shape, 0))
        L.upload(sf.SF_F, I.random_field(shape, 1))
        Ls.append(L)
    C = sf.Level(nx // 2, ny // 2, nz // 2, 2 * h)
    sf.sf_smooth_residual_restrict(Ls[0].handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F)
    sf.sf_smooth_gsrb(Ls[1].handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
    a, b = Ls[0].download(sf.SF_U), Ls[1].download(sf.SF_U)
    d = np.abs(a - b)
    bad = np.argwhere(d > 0)
    print(shape, "mismatches", len(bad), "of", a.size, "max", d.max())
    if len(bad):
        ks = sorted(set(bad[:, 0].tolist()))
        print("  planes", ks[:20])
        for k in ks[:3]:
            m = d[k] > 0
            print("  plane", k, "count", m.sum(), "rows", sorted(set(np.argwhere(m)[:, 0].tolist()))[:20],
                  "cols", sorted(set(np.argwhere(m)[:, 1].tolist()))[:40])
        par = (bad.sum(axis=1) % 2)
        print("  colour (0 red, 1 black) counts", np.bincount(par, minlength=2))
