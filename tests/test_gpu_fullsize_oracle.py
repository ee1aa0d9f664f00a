"""The headline configuration cell by cell: the 512^3 HPGMG-FV solve (BASELINE
C5: F-cycle + V-cycles to 1e-10 with the production kernel builds -- 32x8
colour-fused pairs, the 32x16 P0-fused pair, the fused pair + delta-form
residual + restriction on the levels >= 128^3, the z-streamed residual +
restriction below, the coarse cluster V-cycle) against a complete oracle solve of the
same problem.  The oracle runs in a subprocess with its OpenMP build on every
host core (the library build is per process; GSRB colour sweeps and max-norms
are independent of the thread count, so it computes what the single-thread
build computes).  Same cycle count, residual history within 1e-6 relative plus
the residual's absolute rounding floor (1e-12), u within
1e-10 (rel-L2) and 1e-9 of max|u| cell by cell."""
import os
import subprocess
import sys

import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
N = 512

ORACLE_SCRIPT = """
import sys, numpy as np
sys.path.insert(0, {root!r})
from oracle import oracle as O
from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I
import os
O.use_openmp(True)
O.lib().or_set_threads(len(os.sched_getaffinity(0)))
n = {n}
h = I.level_h(n, n, n)
coeffs = I.hpgmg_coeffs(n, n, n, h)
_, f = I.manufactured(n, n, n, 1.0, 1.0, h)
mg = O.MG(n, n, n, h, 1.0, 1.0, *coeffs)
del coeffs
u, hist = mg.solve(f, fcycle=True, rtol=1e-10)
np.save({out!r}, u)
np.save({hist!r}, np.array(hist))
"""


def test_512_solve_matches_oracle(tmp_path):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    try:
        import psutil
        if psutil.virtual_memory().available < 64 * 2**30:
            pytest.skip("the 512^3 oracle hierarchy needs ~45 GB of host memory")
    except ImportError:
        pytest.skip("psutil unavailable")
    from paper_conf_ipps_zhangdmwbf17_b200 import build, sf
    build.build()
    out, hist_p = str(tmp_path / "u_oracle.npy"), str(tmp_path / "hist_oracle.npy")
    # the oracle first (its 45 GB are released before the GPU side allocates)
    r = subprocess.run([sys.executable, "-c", ORACLE_SCRIPT.format(root=ROOT, n=N, out=out,
                                                                   hist=hist_p)],
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    u_o, hist_o = np.load(out), np.load(hist_p)
    # the same host-generated inputs on the GPU
    h = I.level_h(N, N, N)
    L = sf.Level(N, N, N, h)
    L.set_coeffs(*I.hpgmg_coeffs(N, N, N, h))
    L.upload(sf.SF_F, I.manufactured(N, N, N, 1.0, 1.0, h)[1])
    M = sf.MG(L, 1.0, 1.0)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
    u = L.download(sf.SF_U)
    M.close()
    L.close()
    assert cyc == len(hist_o)
    # atol: the max-norm residual's absolute rounding floor at 512^3 (~1e-13,
    # DESIGN.md section 13, R-19); u itself is compared at 1e-10 below
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-12)
    rel = np.linalg.norm((u - u_o).ravel()) / np.linalg.norm(u_o.ravel())
    print(f"512^3 solve vs oracle: cycles {cyc} / {len(hist_o)}, final relres {hist[-1]:.3e} / "
          f"{hist_o[-1]:.3e}, u rel-L2 {rel:.3e}, max-abs {np.abs(u - u_o).max():.3e} "
          f"(max|u| {np.abs(u_o).max():.3e})")
    assert rel < 1e-10
    assert np.abs(u - u_o).max() <= 1e-9 * np.abs(u_o).max()
