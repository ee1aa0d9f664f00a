"""Small hierarchies: colour-fused pairs vs colour sweeps on every level (V-solve
from u = 0 to 1e-10, device loop where allowed), same session.
    python scripts/small_level_smoother_ab.py [n ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def solve_ms(n, smoother, reps=20):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0, smoother=smoother)
    z = np.zeros((n, n, n))
    ts = []
    for r in range(reps + 3):
        L.upload(sf.SF_U, z)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st, cyc, hist = M.solve(False, 1e-10, 50)
        if r >= 3:
            ts.append(time.perf_counter() - t0)
    M.close()
    L.close()
    return min(ts) * 1e3, cyc


for n in [int(v) for v in sys.argv[1:]] or [32, 64, 128]:
    a = solve_ms(n, sf.SF_SMOOTH_AUTO)
    c = solve_ms(n, sf.SF_SMOOTH_COLOUR)
    print(f"n={n} V-solve: fused pairs {a[0]:.3f} ms ({a[1]} cycles) | colour sweeps {c[0]:.3f} ms ({c[1]} cycles)",
          flush=True)
