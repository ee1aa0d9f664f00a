"""GPU parity of the kernel builds and launch shapes the 512^3 headline takes,
exercised where the oracle can compare them cell by cell.

At 512^3 the V-cycle routes the P0-fused first post-smoothing pair (A8 + A5,
PAPER.md:597, 647-653) to the 32x16 / 5-deep build (level.cu, levels above
2^24 cells), and the fused residual + restriction (A6 + A7) walks
many multi-plane z-chunks per persistent CTA.  Small levels would take the
32x8 build and one-plane chunks; the test-only overrides SF_INTERP_T32_CELLS,
SF_RRZS_DEPTH and SF_RRZS_GRID force the headline's paths on sizes the oracle
solves in seconds.  Tolerances: 1e-12 relative per pair / restriction (plus a
max-abs bound relative to the largest value, so one wrong cell cannot hide in
an L2 norm), 1e-11 per V/F-cycle."""
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
    return np.linalg.norm((a - b).ravel()) / max(np.linalg.norm(b.ravel()), 1e-300)


def maxrel(a, b):
    return np.abs(a - b).max() / max(np.abs(b).max(), 1e-300)


HEADLINE_PATHS = {"SF_INTERP_T32_CELLS": "0", "SF_RRZS_DEPTH": "3", "SF_RRZS_GRID": "7"}


@pytest.mark.parametrize("shape", [(16, 32, 64), (24, 48, 96), (64, 64, 64), (40, 16, 128)])
@pytest.mark.parametrize("build", ["default", "t32_interp", "one_cta"])
def test_interpolate_smooth_vs_oracle(sf, oracle, shape, build, monkeypatch):
    """sf_interpolate_smooth (x += P0 e, then one RB pair, fused in one pass) in
    each build of the P0-fused pair vs the oracle's interpolate + smooth."""
    nz, ny, nx = shape
    if build == "t32_interp":
        monkeypatch.setenv("SF_INTERP_T32_CELLS", "0")
    elif build == "one_cta":
        monkeypatch.setenv("SF_GSRB_W4", "0")
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 11)
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    Cl = sf.Level(nx // 2, ny // 2, nz // 2, 2 * h)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    e = I.random_field((nz // 2, ny // 2, nx // 2), 2)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    Cl.upload(sf.SF_U, e)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    d = P.dinv()
    xo = oracle.interpolate(x, e, 1.0, "p0")
    for _ in range(2):   # the second call re-reads the swapped U / TMP mapping
        sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_U)
        if _ == 1:
            xo = oracle.interpolate(xo, e, 1.0, "p0")
        xo = P.smooth(xo, f, 1, dinv=d)
        got = L.download(sf.SF_U)
        assert rel(got, xo) < TOL
        assert maxrel(got, xo) < 10 * TOL
    Cl.close()
    L.close()


def test_interpolate_smooth_builds_bit_identical(sf, monkeypatch):
    """The 32x16 P0-fused build the headline runs and the default 32x8 build
    give the same bits (shared explicit contractions)."""
    nz, ny, nx = (32, 64, 128)
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 12)
    x, f = I.random_field((nz, ny, nx), 0), I.random_field((nz, ny, nx), 1)
    e = I.random_field((nz // 2, ny // 2, nx // 2), 2)
    outs = []
    for cells in (None, "0"):
        if cells:
            monkeypatch.setenv("SF_INTERP_T32_CELLS", cells)
        L = sf.Level(nx, ny, nz, h)
        L.set_coeffs(*coeffs)
        Cl = sf.Level(nx // 2, ny // 2, nz // 2, 2 * h)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        Cl.upload(sf.SF_U, e)
        sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_U)
        outs.append(L.download(sf.SF_U))
        Cl.close()
        L.close()
    assert np.array_equal(outs[0], outs[1])


def _mg(sf, oracle, shape, seed_coeffs=None):
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.hpgmg_coeffs(nx, ny, nz, h)
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    M = sf.MG(L, 1.0, 1.0)
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *coeffs)
    return L, M, O


@pytest.mark.parametrize("shape", [(64, 64, 64), (128, 128, 128), (32, 64, 128)])
def test_vcycle_fcycle_headline_paths_vs_oracle(sf, oracle, shape, monkeypatch):
    """V- and F-cycles with the headline's kernel paths forced (32x16 P0-fused
    pairs on every level that allows them; residual + restriction in 3-plane
    chunks walked by 7 persistent CTAs, ragged last chunk) against the oracle
    cell by cell, and bit-identical to the default paths."""
    nz, ny, nx = shape
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    res = {}
    for mode in ("default", "headline"):
        if mode == "headline":
            for k, v in HEADLINE_PATHS.items():
                monkeypatch.setenv(k, v)
        L, M, O = _mg(sf, oracle, shape)
        L.upload(sf.SF_F, f)
        M.fcycle()
        uf = L.download(sf.SF_U)
        M.vcycle(0)
        uv = L.download(sf.SF_U)
        res[mode] = (uf, uv)
        M.close()
        L.close()
    uo_f = O.fcycle(f)
    uo_v = O.vcycle(uo_f, f)
    for mode in res:
        uf, uv = res[mode]
        assert rel(uf, uo_f) < 1e-11 and maxrel(uf, uo_f) < 1e-10, mode
        assert rel(uv, uo_v) < 1e-11 and maxrel(uv, uo_v) < 1e-10, mode
    assert np.array_equal(res["default"][0], res["headline"][0])
    assert np.array_equal(res["default"][1], res["headline"][1])


@pytest.mark.parametrize("shape", [(64, 64, 64), (128, 128, 128), (32, 64, 128)])
def test_vcycle_fcycle_rrf_vs_oracle(sf, oracle, shape, monkeypatch):
    """V- and F-cycles with the fused pair + delta-form residual + restriction
    (gsrb_rr.cu) forced on every level it supports (the 512^3 headline takes it
    on the levels >= 128^3) against the oracle cell by cell: 1e-11 rel-L2,
    1e-10 max-abs relative (the restricted residual rounds differently from
    rhs - Ax, R-19)."""
    monkeypatch.setenv("SF_RRF_CELLS", "0")
    nz, ny, nx = shape
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L, M, O = _mg(sf, oracle, shape)
    L.upload(sf.SF_F, f)
    sf.sf_level_pair_timing(L.handle, 1)
    M.fcycle()
    uf = L.download(sf.SF_U)
    M.vcycle(0)
    uv = L.download(sf.SF_U)
    sf.sf_level_pair_timing(L.handle, 0)
    assert sf.sf_level_pair_timing_rrf(L.handle)[1] >= 2   # the fused path ran on the finest level
    M.close()
    L.close()
    uo_f = O.fcycle(f)
    uo_v = O.vcycle(uo_f, f)
    assert rel(uf, uo_f) < 1e-11 and maxrel(uf, uo_f) < 1e-10
    assert rel(uv, uo_v) < 1e-11 and maxrel(uv, uo_v) < 1e-10


@pytest.mark.parametrize("fcycle", [False, True])
def test_solve_rrf_vs_oracle(sf, oracle, fcycle, monkeypatch):
    """The device-loop solve with the fused residual + restriction forced: same
    cycle count as the oracle, history within 1e-6 relative plus the residual's
    absolute rounding floor (1e-12 at 512^3, scaled by
    h^-2), u to 1e-10."""
    monkeypatch.setenv("SF_RRF_CELLS", "0")
    shape = (64, 64, 64)
    nz, ny, nx = shape
    L, M, O = _mg(sf, oracle, shape)
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=fcycle, rtol=1e-10)
    u_o, hist_o = O.solve(f, fcycle=fcycle, rtol=1e-10)
    assert cyc == len(hist_o)
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-12 * (nx / 512) ** 2)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10
    M.close()
    L.close()


@pytest.mark.parametrize("fcycle", [False, True])
def test_solve_headline_paths_vs_oracle(sf, oracle, fcycle, monkeypatch):
    """The whole device-loop solve (as bench.py runs it) with the headline's
    paths forced: same cycle count and history as the oracle, u to 1e-10."""
    for k, v in HEADLINE_PATHS.items():
        monkeypatch.setenv(k, v)
    shape = (64, 64, 64)
    nz, ny, nx = shape
    L, M, O = _mg(sf, oracle, shape)
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=fcycle, rtol=1e-10)
    u_o, hist_o = O.solve(f, fcycle=fcycle, rtol=1e-10)
    assert cyc == len(hist_o)
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-14)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10


@pytest.mark.parametrize("depth,grid", [("1", None), ("3", "7"), ("5", "2"), ("64", "1")])
def test_smooth_residual_restrict_chunking(sf, oracle, depth, grid, monkeypatch):
    """sf_smooth_residual_restrict's coarse rhs = R_cell(rhs - A x) of the
    smoothed x, for z-chunkings from one plane per item to one item per CTA
    walking the whole level, vs the oracle (1e-12)."""
    monkeypatch.setenv("SF_RRZS_DEPTH", depth)
    if grid:
        monkeypatch.setenv("SF_RRZS_GRID", grid)
    shape = (26, 32, 64)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 13)
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    Cl = sf.Level(nx // 2, ny // 2, nz // 2, 2 * h)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_F)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    xs = P.smooth(x, f, 1)
    assert rel(L.download(sf.SF_U), xs) < TOL
    exp = oracle.restrict_cell(P.residual(L.download(sf.SF_U), f))
    got = Cl.download(sf.SF_F)
    assert rel(got, exp) < TOL and maxrel(got, exp) < 10 * TOL
    Cl.close()
    L.close()


# --------------------------------------------------------- 512^3, sampled
def _samples(shape, count, seed):
    nz, ny, nx = shape
    rng = np.random.default_rng(seed)
    pts = [rng.integers(0, nx, count), rng.integers(0, ny, count), rng.integers(0, nz, count)]
    extra = [(0, 0, 0), (nx - 1, ny - 1, nz - 1), (0, ny - 1, 0), (nx - 1, 0, nz // 2),
             (31, 15, 1), (32, 16, 2), (33, 17, 255), (480, 496, 511)]
    for e in extra:
        for a in range(3):
            pts[a] = np.r_[pts[a], e[a]]
    return tuple(pts)


def test_512_interpolate_smooth_sampled(sf, oracle):
    """The P0-fused pair at bench's finest level (512^3: the 32x16 build) vs the
    oracle's P0 interpolation and cell-by-cell RB pair at 4000+ cells."""
    n = 512
    h = 1.0 / n
    L = sf.Level(n, n, n, h)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    Cl = sf.Level(n // 2, n // 2, n // 2, 2 * h)
    x = I.random_field((n, n, n), 0)
    e = I.random_field((n // 2, n // 2, n // 2), 2)
    L.upload(sf.SF_U, x)
    Cl.upload(sf.SF_U, e)
    rhs = L.download(sf.SF_F)
    sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_U)
    got = L.download(sf.SF_U)
    Cl.close()
    L.close()
    xp = oracle.interpolate(x, e, 1.0, "p0")
    del x
    coeffs = I.hpgmg_coeffs(n, n, n, h)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *coeffs)
    del coeffs
    pts = _samples((n, n, n), 4000, 3)
    exp = P.gsrb_pair_points(xp, rhs, pts)
    g = got[pts[2], pts[1], pts[0]]
    assert np.abs(g - exp).max() <= 1e-12 * np.abs(exp).max()


def test_512_residual_restrict_sampled(sf, oracle):
    """bench's persistent residual + restriction at 512^3 (multi-plane chunks,
    several items per CTA) vs the oracle's residual at the 8 children of 2000+
    sampled coarse cells, averaged as R_cell."""
    n = 512
    h = 1.0 / n
    L = sf.Level(n, n, n, h)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    Cl = sf.Level(n // 2, n // 2, n // 2, 2 * h)
    L.upload(sf.SF_U, I.random_field((n, n, n), 0))
    sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, Cl.handle, sf.SF_F)
    xs = L.download(sf.SF_U)
    rhs = L.download(sf.SF_F)
    got = Cl.download(sf.SF_F)
    Cl.close()
    L.close()
    coeffs = I.hpgmg_coeffs(n, n, n, h)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *coeffs)
    del coeffs
    cI, cJ, cK = _samples((n // 2, n // 2, n // 2), 2000, 4)
    cI, cJ, cK = cI % (n // 2), cJ % (n // 2), cK % (n // 2)
    ch = [(a, b, c) for c in (0, 1) for b in (0, 1) for a in (0, 1)]
    pts = (np.concatenate([2 * cI + a for a, b, c in ch]),
           np.concatenate([2 * cJ + b for a, b, c in ch]),
           np.concatenate([2 * cK + c for a, b, c in ch]))
    r = P.residual_points(xs, rhs, pts).reshape(8, -1)
    exp = r.sum(axis=0) / 8.0
    g = got[cK, cJ, cI]
    assert np.abs(g - exp).max() <= 1e-12 * np.abs(exp).max()


@pytest.mark.parametrize("use_graph", [0, 1])
def test_solve_after_public_swaps(sf, oracle, use_graph):
    """A public fused smooth between solves swaps the U/TMP ids of the finest
    level (odd count); the cached solve graphs name the old buffers and must be
    re-captured: a V-only solve continues from the smoothed iterate exactly as
    the oracle does, and downloads return the solve's result."""
    shape = (64, 64, 64)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.hpgmg_coeffs(nx, ny, nz, h)
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    M = sf.MG(L, 1.0, 1.0, use_graph=use_graph)
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *coeffs)
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    M.solve(fcycle=True, rtol=1e-6)
    for rep in range(2):
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
        us = L.download(sf.SF_U)
        st, cyc, hist = M.solve(fcycle=False, rtol=1e-10)
        u_o, hist_o = O.solve(f, fcycle=False, rtol=1e-10, u0=us)
        assert cyc == len(hist_o)
        assert rel(L.download(sf.SF_U), u_o) < 1e-10
    M.close()
    L.close()
