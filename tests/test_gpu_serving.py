"""Pipelined multi-RHS solve (sf_solve_stream, the serving path): every
right-hand side gives exactly what a standalone sf_solve gives, whatever the
overlap of its copies with the neighbouring solves."""
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


@pytest.mark.parametrize("fcycle", [True, False])
@pytest.mark.parametrize("pinned", [True, False])
def test_stream_equals_individual_solves(sf, fcycle, pinned):
    import torch
    n = 32
    coeffs = I.hpgmg_coeffs(n, n, n)
    L = sf.Level(n, n, n)
    L.set_coeffs(*coeffs)
    M = sf.MG(L, 1.0, 1.0)
    _, fm = I.manufactured(n, n, n, 1.0, 1.0)
    rhs = [fm, 0.5 * fm + 0.1 * I.random_field((n, n, n), 3), I.random_field((n, n, n), 4)]
    ref, cref = [], []
    for f in rhs:
        L.upload(sf.SF_F, f)
        if not fcycle:
            L.upload(sf.SF_U, np.zeros((n, n, n)))
        st, cyc, _ = M.solve(fcycle=fcycle)
        ref.append(L.download(sf.SF_U))
        cref.append(cyc)
    if pinned:
        fs = [torch.from_numpy(np.ascontiguousarray(f)).pin_memory() for f in rhs]
        us = [torch.zeros((n, n, n), dtype=torch.float64).pin_memory() for _ in rhs]
    else:
        fs = [np.ascontiguousarray(f) for f in rhs]
        us = [np.zeros((n, n, n)) for _ in rhs]
    L.upload(sf.SF_U, I.random_field((n, n, n), 9))   # stale state must not leak in
    cyc = M.solve_stream(fs, us, fcycle=fcycle)
    assert cyc == cref
    for k in range(len(rhs)):
        got = us[k].numpy() if pinned else us[k]
        assert np.array_equal(got, ref[k]), k
    M.close()
    L.close()


def test_stream_empty_and_errors(sf):
    n = 16
    L = sf.Level(n, n, n)
    L.set_coeffs(*I.hpgmg_coeffs(n, n, n))
    M = sf.MG(L, 1.0, 1.0)
    assert M.solve_stream([], []) == []
    bad = [np.full((n, n, n), np.nan)]
    with pytest.raises(sf.SfError) as e:
        M.solve_stream(bad, [np.zeros((n, n, n))])
    assert e.value.status == sf.SF_ERR_NUMERIC
    M.close()
    L.close()
