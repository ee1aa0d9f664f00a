"""The measurement hooks bench.py reports: the live
per-variant split of the fused-pair timer and the phase times of the
streamed serving path."""
import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sf():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_zhangdmwbf17_b200 import build, sf as S
    build.build()
    S.lib()
    return S


def test_pair_timing_variants_of_a_solve(sf):
    """A solve of F-cycle + c V-cycles books on the finest level: one RESID pair
    (the next cycle's checked first pre-smoothing pair) and one BRES pair (last
    post-smoothing pair) per cycle, one P0-fused pair per cycle, and the
    remaining plain pairs; the variant counts add up to the total and the
    total mean is their weighted mean."""
    n = 64
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    M.solve(fcycle=True, rtol=1e-10)
    sf.sf_level_pair_timing(L.handle, 1)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
    ms, npairs = sf.sf_level_pair_timing(L.handle, 0)
    var = sf.sf_level_pair_timing_variants(L.handle)
    counts = {k: v[1] for k, v in var.items()}
    assert sum(counts.values()) == npairs
    # cycles = 1 F + (cyc - 1) V.  The F-cycle's V(0) smooths with plain, plain,
    # P0-fused, BRES pairs; each later V-cycle with the checked RESID pair, plain,
    # P0-fused, BRES; one more RESID pair checks the last cycle (speculative)
    assert counts["bres"] == cyc and counts["interp"] == cyc
    assert counts["resid"] == (cyc - 1) + 1
    assert counts["plain"] == 2 + (cyc - 1)
    mean = sum(v[0] * v[1] for v in var.values()) / npairs
    assert abs(mean - ms) <= 1e-6 * ms + 1e-9
    assert all(v[0] > 0 for v in var.values())
    M.close()
    L.close()


def test_solve_stream_stats(sf):
    """sf_solve_stream_stats: per right-hand side H2D, solve and D2H device
    times from events, and the host wall time per right-hand side, which the
    overlapped pipeline keeps below the serial sum."""
    import torch
    n = 64
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    hf = torch.empty(L.host_shape(sf.SF_F), dtype=torch.float64, pin_memory=True)
    hu = [torch.empty(L.host_shape(sf.SF_U), dtype=torch.float64, pin_memory=True) for _ in range(2)]
    L.download(sf.SF_F, hf.numpy())
    M.solve_stream([hf] * 4, [hu[k % 2] for k in range(4)])
    h2d, solve, d2h, wall = sf.sf_solve_stream_stats(M.handle)
    assert h2d > 0 and solve > 0 and d2h > 0 and wall > 0
    assert wall < h2d + solve + d2h + 5.0
    M.solve(fcycle=True, rtol=1e-10)
    assert np.array_equal(hu[1].numpy(), L.download(sf.SF_U))
    M.close()
    L.close()
