"""NEXT-1: the whole smooth -- two RB pairs -- in one pass of
a temporally blocked kernel (gsrb_twopair.cu, sf_smooth_gsrb kind
SF_SMOOTH_FUSED2).  Every update is the colour-fused pair's, so the result is
bit-identical to two fused pairs, which are pinned to the oracle; here also
checked against the oracle directly (1e-12 relative, max-abs bounded)."""
import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def sf():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_zhangdmwbf17_b200 import build, sf as S
    build.build()
    S.lib()
    return S


def rel(a, b):
    return np.linalg.norm((a - b).ravel()) / np.linalg.norm(b.ravel())


def _smooth(sf, shape, coeffs, x, f, kind, pairs, h):
    nz, ny, nx = shape
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, pairs, kind)
    u = L.download(sf.SF_U)
    L.close()
    return u


@pytest.mark.parametrize("shape", [(24, 16, 64), (37, 32, 96), (64, 64, 64), (9, 16, 32), (3, 16, 32),
                                   (2, 16, 32)])
@pytest.mark.parametrize("depth", [None, "1", "2", "5"])
def test_twopair_bit_identical_to_two_pairs(sf, oracle, shape, depth, monkeypatch):
    if depth:
        monkeypatch.setenv("SF_TWOPAIR_DEPTH", depth)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 21)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    for pairs in (2, 3, 4):
        u2 = _smooth(sf, shape, coeffs, x, f, sf.SF_SMOOTH_FUSED2, pairs, h)
        u1 = _smooth(sf, shape, coeffs, x, f, sf.SF_SMOOTH_FUSED, pairs, h)
        assert np.array_equal(u2, u1), (shape, depth, pairs)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    exp = P.smooth(x, f, 2)
    u2 = _smooth(sf, shape, coeffs, x, f, sf.SF_SMOOTH_FUSED2, 2, h)
    assert rel(u2, exp) < TOL
    assert np.abs(u2 - exp).max() <= 10 * TOL * np.abs(exp).max()


def test_twopair_256_vs_oracle(sf, oracle):
    """BASELINE C3's 256^3 level, one whole smooth (2 pairs) vs the oracle."""
    n = 256
    shape = (n, n, n)
    coeffs = I.hpgmg_coeffs(n, n, n)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    u2 = _smooth(sf, shape, coeffs, x, f, sf.SF_SMOOTH_FUSED2, 2, 1.0 / n)
    u1 = _smooth(sf, shape, coeffs, x, f, sf.SF_SMOOTH_FUSED, 2, 1.0 / n)
    assert np.array_equal(u2, u1)
    P = oracle.Problem(oracle.Grid(n, n, n, 1.0 / n), 1.0, 1.0, *coeffs)
    exp = P.smooth(x, f, 2)
    assert rel(u2, exp) < TOL
    assert np.abs(u2 - exp).max() <= 10 * TOL * np.abs(exp).max()


def test_twopair_rejects_unsupported(sf):
    L = sf.Level(48, 16, 16, 1.0 / 48)       # nx % 32 != 0
    with pytest.raises(sf.SfError) as e:
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, sf.SF_SMOOTH_FUSED2)
    assert e.value.status == sf.SF_ERR_SHAPE
    L.close()
