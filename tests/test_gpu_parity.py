"""GPU parity: every libsf entry point (through the C ABI) against the CPU
oracle on the same seeded inputs.  Tolerances:
1e-12 relative L2 per call / per RB pair, 1e-10 after a full solve; bit-exact
where both sides perform the identical additions (restriction, P0, BC)."""
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


def make_level(sf, shape, coeffs, parts=1, h=None):
    nz, ny, nx = shape
    comm = sf.Comm.local(parts) if parts > 1 else None
    L = sf.Level(nx, ny, nz, h=h, comm=comm)
    L.set_coeffs(*coeffs)
    L._comm_keep = comm
    return L


SHAPES = [(16, 16, 16), (8, 6, 10), (6, 5, 9), (20, 64, 64), (32, 24, 128), (40, 16, 192)]


@pytest.mark.parametrize("shape", SHAPES)
def test_upload_download_roundtrip(sf, shape):
    nz, ny, nx = shape
    coeffs = I.random_coeffs(nx, ny, nz, 1)
    L = make_level(sf, shape, coeffs)
    for f, arr in zip([sf.SF_ALPHA, sf.SF_BETA_I, sf.SF_BETA_J, sf.SF_BETA_K], coeffs):
        assert np.array_equal(L.download(f), arr)
    x = I.random_field(shape, 3)
    L.upload(sf.SF_U, x)
    assert np.array_equal(L.download(sf.SF_U), x)
    # sf_level_zero clears one field, interior and ghosts (BC fill of zeros is zero)
    sf.sf_apply_bc(L.handle, sf.SF_U)
    sf.sf_level_zero(L.handle, sf.SF_U)
    assert not L.download(sf.SF_U).any()
    assert np.array_equal(L.download(sf.SF_BETA_I), coeffs[1])
    with pytest.raises(sf.SfError):
        sf.sf_level_zero(L.handle, 99)


@pytest.mark.parametrize("shape", [(6, 5, 4), (16, 16, 16), (8, 8, 64)])
def test_apply_bc(sf, oracle, shape):
    nz, ny, nx = shape
    L = make_level(sf, shape, I.random_coeffs(nx, ny, nz, 1))
    x = I.random_field(shape, 0)
    L.upload(sf.SF_U, x)
    sf.sf_apply_bc(L.handle, sf.SF_U)
    got = L.padded(sf.SF_U)
    exp = oracle.apply_bc(oracle.Grid(nx, ny, nz, 1.0), oracle.pad(x))
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("ab", [(0.0, 1.0), (1.0, 1.0), (2.5, 0.75)])
def test_apply_op_and_residual(sf, oracle, shape, ab):
    nz, ny, nx = shape
    a, b = ab
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 2)
    L = make_level(sf, shape, coeffs)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), a, b, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_apply_op(L.handle, sf.SF_R, sf.SF_U, a, b)
    assert rel(L.download(sf.SF_R), P.apply_op(x)) < TOL
    sf.sf_residual(L.handle, sf.SF_R, sf.SF_U, sf.SF_F, a, b)
    assert rel(L.download(sf.SF_R), P.residual(x, f)) < TOL


@pytest.mark.parametrize("shape", SHAPES)
def test_dinv(sf, oracle, shape):
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 4)
    L = make_level(sf, shape, coeffs)
    sf.sf_rebuild_operator(L.handle, 1.5, 0.5)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.5, 0.5, *coeffs)
    assert rel(L.download(sf.SF_DINV), P.dinv()) < 1e-14


@pytest.mark.parametrize("shape", SHAPES + [(64, 64, 64), (24, 8, 64), (12, 16, 32), (8, 16, 96)])
@pytest.mark.parametrize("kind", ["colour", "fused"])
def test_gsrb_per_pair(sf, oracle, shape, kind):
    """Each RB pair (BC, red, BC, black) matches the oracle to 1e-12."""
    nz, ny, nx = shape
    if kind == "fused" and not ((nx % 32 == 0 and ny % 16 == 0) or (nx % 64 == 0 and ny % 8 == 0)):
        pytest.skip("fused kernel needs (nx%32, ny%16) or (nx%64, ny%8) == 0")
    a, b = 1.0, 1.0
    h = I.level_h(nx, ny, nz)
    coeffs = I.hpgmg_coeffs(nx, ny, nz) if nx >= 64 else I.random_coeffs(nx, ny, nz, 5)
    L = make_level(sf, shape, coeffs)
    sf.sf_rebuild_operator(L.handle, a, b)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), a, b, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    k = sf.SF_SMOOTH_FUSED if kind == "fused" else sf.SF_SMOOTH_COLOUR
    d = P.dinv()
    for _ in range(3):
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, a, b, 1, k)
        x = P.smooth(x, f, 1, dinv=d)
        assert rel(L.download(sf.SF_U), x) < TOL


@pytest.mark.parametrize("shape", [(24, 16, 64), (20, 8, 128), (12, 48, 96)])
def test_fused_builds_agree(sf, oracle, shape, monkeypatch):
    """The three builds of the fused pair (32x8 / 3 CTAs per SM, the default;
    32x16 and 64x8 with one CTA, SF_GSRB_W4=0) match the oracle per pair and
    each other bit for bit (explicit contractions shared by all builds)."""
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 5)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    d = P.dinv()
    outs = []
    for mode in ("1", "0"):
        monkeypatch.setenv("SF_GSRB_W4", mode)
        L = make_level(sf, shape, coeffs)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        xo = x
        for _ in range(2):
            sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
            xo = P.smooth(xo, f, 1, dinv=d)
            assert rel(L.download(sf.SF_U), xo) < TOL
        outs.append(L.download(sf.SF_U))
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("parts,overlap", [(1, None), (2, "1"), (2, "0")])
def test_pair_timing_counts_pairs(sf, parts, overlap, monkeypatch):
    """sf_level_pair_timing books one entry per RB pair and part -- also when
    the pair is split into interior and boundary launches around the halo --
    and its mean agrees with CUDA events around back-to-back pairs."""
    import torch
    if overlap is not None:
        monkeypatch.setenv("SF_HALO_OVERLAP", overlap)
    shape = (48 * parts, 32, 64)
    nz, ny, nx = shape
    L = make_level(sf, shape, I.hpgmg_coeffs(nx, ny, nz), parts=parts)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    L.upload(sf.SF_F, I.random_field(shape, 1))
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, sf.SF_SMOOTH_FUSED)   # warm
    sf.sf_level_pair_timing(L.handle, 1)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(L.stream)
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 3, sf.SF_SMOOTH_FUSED)
    b.record(L.stream)
    ms, n = sf.sf_level_pair_timing(L.handle, 0)
    assert n == 3 * parts
    ev = a.elapsed_time(b) / n
    assert 0 < ms <= ev * 1.05 + 0.02
    # disarmed: nothing more is booked
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
    sf.sf_level_pair_timing(L.handle, 1)
    ms2, n2 = sf.sf_level_pair_timing(L.handle, 0)
    assert n2 == 0 and ms2 == 0.0


def test_fused_equals_colour(sf):
    shape = (48, 32, 128)
    nz, ny, nx = shape
    coeffs = I.hpgmg_coeffs(nx, ny, nz)
    outs = []
    for k in (sf.SF_SMOOTH_COLOUR, sf.SF_SMOOTH_FUSED):
        L = make_level(sf, shape, coeffs)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, I.random_field(shape, 0))
        L.upload(sf.SF_F, I.random_field(shape, 1))
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, k)
        outs.append(L.download(sf.SF_U))
    assert rel(outs[1], outs[0]) < 1e-13   # fused sums the fluxes as a tree


def test_c1_config(sf, oracle):
    """BASELINE config 1: 16^3 CC Poisson, 4 GSRB sweeps + residual."""
    n = 16
    shape = (n, n, n)
    h = 1.0 / n
    coeffs = I.constant_coeffs(n, n, n)
    L = make_level(sf, shape, coeffs)
    sf.sf_rebuild_operator(L.handle, 0.0, 1.0)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 0.0, 1.0, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    for _ in range(2):
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 0.0, 1.0, 1)
        x = P.smooth(x, f, 1)
        assert rel(L.download(sf.SF_U), x) < TOL
    sf.sf_residual(L.handle, sf.SF_R, sf.SF_U, sf.SF_F, 0.0, 1.0)
    assert rel(L.download(sf.SF_R), P.residual(x, f)) < TOL


@pytest.mark.parametrize("fine", [(8, 8, 8), (16, 12, 20), (32, 32, 64)])
def test_restrict(sf, oracle, fine):
    nz, ny, nx = fine
    coeffs = I.random_coeffs(nx, ny, nz, 6)
    F = make_level(sf, fine, coeffs)
    C = sf.Level(nx // 2, ny // 2, nz // 2)
    x = I.random_field(fine, 2)
    F.upload(sf.SF_R, x)
    sf.sf_restrict(C.handle, sf.SF_F, F.handle, sf.SF_R, sf.SF_RESTRICT_CELL)
    assert np.array_equal(C.download(sf.SF_F), oracle.restrict_cell(x))
    for kind, fid, arr in [(sf.SF_RESTRICT_FACE_I, sf.SF_BETA_I, coeffs[1]),
                           (sf.SF_RESTRICT_FACE_J, sf.SF_BETA_J, coeffs[2]),
                           (sf.SF_RESTRICT_FACE_K, sf.SF_BETA_K, coeffs[3])]:
        sf.sf_restrict(C.handle, fid, F.handle, fid, kind)
        name = {sf.SF_BETA_I: "beta_i", sf.SF_BETA_J: "beta_j", sf.SF_BETA_K: "beta_k"}[fid]
        assert np.array_equal(C.download(fid), oracle.restrict_face(arr, name))


@pytest.mark.parametrize("fine", [(8, 8, 8), (16, 12, 20), (32, 32, 64)])
@pytest.mark.parametrize("kind", ["p0", "pl"])
@pytest.mark.parametrize("s", [0.0, 1.0, 0.5])
def test_interpolate(sf, oracle, fine, kind, s):
    nz, ny, nx = fine
    F = make_level(sf, fine, I.random_coeffs(nx, ny, nz, 6))
    C = sf.Level(nx // 2, ny // 2, nz // 2)
    y = I.random_field(fine, 1)
    c = I.random_field((nz // 2, ny // 2, nx // 2), 2)
    F.upload(sf.SF_U, y)
    C.upload(sf.SF_U, c)
    k = sf.SF_INTERP_P0 if kind == "p0" else sf.SF_INTERP_PL
    sf.sf_interpolate(F.handle, sf.SF_U, s, C.handle, sf.SF_U, k)
    exp = oracle.interpolate(y, c, s, kind)
    assert rel(F.download(sf.SF_U), exp) < 1e-15


def test_norms(sf, oracle):
    shape = (20, 24, 64)
    nz, ny, nx = shape
    L = make_level(sf, shape, I.random_coeffs(nx, ny, nz, 1))
    x = I.random_field(shape, 9)
    L.upload(sf.SF_R, x)
    assert sf.sf_norm(L.handle, sf.SF_R, sf.SF_NORM_MAX) == oracle.norm(x, "max")
    assert abs(sf.sf_norm(L.handle, sf.SF_R, sf.SF_NORM_L2) / oracle.norm(x, "l2") - 1) < 1e-13
    x[3, 4, 5] = np.nan
    L.upload(sf.SF_R, x)
    assert np.isnan(sf.sf_norm(L.handle, sf.SF_R, sf.SF_NORM_MAX))


def test_init_problem_matches_input_generator(sf):
    for (nz, ny, nx) in [(16, 16, 16), (64, 32, 32)]:
        L = sf.Level(nx, ny, nz)
        sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
        h = I.level_h(nx, ny, nz)
        al, bi, bj, bk = I.hpgmg_coeffs(nx, ny, nz, h)
        _, f = I.manufactured(nx, ny, nz, 1.0, 1.0, h)
        for fid, arr in [(sf.SF_ALPHA, al), (sf.SF_BETA_I, bi), (sf.SF_BETA_J, bj),
                         (sf.SF_BETA_K, bk), (sf.SF_F, f)]:
            assert rel(L.download(fid), arr) < 1e-14


# ------------------------------------------------------------------ multigrid
def mg_pair(sf, oracle, n, shape=None, parts=1, cc=False, **opts):
    shape = shape or (n, n, n)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.constant_coeffs(nx, ny, nz) if cc else I.hpgmg_coeffs(nx, ny, nz, h)
    L = make_level(sf, shape, coeffs, parts=parts, h=h)
    M = sf.MG(L, 1.0, 1.0, **opts)
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *coeffs)
    return L, M, O


@pytest.mark.parametrize("depth", ["1", "2", "3", "5", "8"])
def test_fused_pair_chunk_depths(sf, oracle, depth, monkeypatch):
    """Small z-chunks: many items per CTA, so every item's prologue is issued in
    the previous item's last steps (pipelined item transition); the result
    matches the oracle per pair and is bit-identical to the default chunking."""
    shape = (24, 32, 64)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 8)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    outs = []
    for dep in (None, depth):
        if dep:
            monkeypatch.setenv("SF_GSRB_DEPTH", dep)
        L = make_level(sf, shape, coeffs)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        for _ in range(3):
            sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
        outs.append(L.download(sf.SF_U))
    assert np.array_equal(outs[0], outs[1])
    assert rel(outs[1], P.smooth(x, f, 3, dinv=P.dinv())) < TOL


@pytest.mark.parametrize("depth", ["2", "3"])
def test_vcycle_chunk_depth_invariant(sf, depth, monkeypatch):
    """The V-cycle's fused variants (check-fused, P0-fused, plain) give the same
    bits whatever the z-chunking (items pipelined into each other)."""
    n = 64
    out = []
    for dep in (None, depth):
        if dep:
            monkeypatch.setenv("SF_GSRB_DEPTH", dep)
        L = make_level(sf, (n, n, n), I.hpgmg_coeffs(n, n, n), h=1.0 / n)
        M = sf.MG(L, 1.0, 1.0)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
        out.append((cyc, list(hist), L.download(sf.SF_U)))
    assert out[0][0] == out[1][0] and out[0][1] == out[1][1]
    assert np.array_equal(out[0][2], out[1][2])


RR_SHAPES = [(4, 16, 32), (10, 32, 64), (16, 48, 96), (34, 16, 32), (64, 64, 64), (6, 32, 160)]


@pytest.mark.parametrize("shape", RR_SHAPES)
@pytest.mark.parametrize("depth", [None, "2", "6"])
@pytest.mark.parametrize("ab", [(1.0, 1.0), (2.5, 0.75)])
def test_smooth_residual_restrict(sf, oracle, shape, depth, ab, monkeypatch):
    """A5+A6+A7 fused (sf_smooth_residual_restrict, the pair's delta-form
    residual + restriction, gsrb_rr.cu, forced on every size): the smoothed x
    equals the oracle's RB pair (1e-12) and bit-for-bit the plain fused pair; the
    coarse rhs equals R_cell(rhs - A x) of the oracle (1e-12 rel-L2, 1e-11
    max-abs relative).  Chunk depths 2 and 6 put item (z-chunk) boundaries inside
    the grid, where the partials cross between items."""
    nz, ny, nx = shape
    a, b = ab
    monkeypatch.setenv("SF_RRF_CELLS", "0")
    if depth:
        monkeypatch.setenv("SF_GSRB_DEPTH", depth)
    h = I.level_h(nx, ny, nz)
    coeffs = I.hpgmg_coeffs(nx, ny, nz) if nx >= 64 else I.random_coeffs(nx, ny, nz, 5)
    L = make_level(sf, shape, coeffs)
    L2 = make_level(sf, shape, coeffs)
    C = make_level(sf, (nz // 2, ny // 2, nx // 2), I.random_coeffs(nx // 2, ny // 2, nz // 2, 6))
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), a, b, *coeffs)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    for lv in (L, L2):
        sf.sf_rebuild_operator(lv.handle, a, b)
        lv.upload(sf.SF_U, x)
        lv.upload(sf.SF_F, f)
    sf.sf_level_pair_timing(L.handle, 1)
    sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, a, b, C.handle, sf.SF_F)
    sf.sf_level_pair_timing(L.handle, 0)
    assert sf.sf_level_pair_timing_rrf(L.handle)[1] == 1   # the fused path ran
    sf.sf_smooth_gsrb(L2.handle, sf.SF_U, sf.SF_F, a, b, 1, sf.SF_SMOOTH_FUSED)
    got = L.download(sf.SF_U)
    assert np.array_equal(got, L2.download(sf.SF_U))
    xs = P.smooth(x, f, 1, dinv=P.dinv())
    assert rel(got, xs) < TOL
    exp = oracle.restrict_cell(P.residual(xs, f))
    gotc = C.download(sf.SF_F)
    assert rel(gotc, exp) < TOL
    assert np.abs(gotc - exp).max() <= 10 * TOL * np.abs(exp).max()


def test_smooth_residual_restrict_general(sf, oracle):
    """Shapes the fused kernel does not take (nx % 32 != 0, 2 parts) go through
    pair + residual + restriction with the same result."""
    for shape, parts in [((8, 8, 16), 1), ((16, 16, 32), 2)]:
        nz, ny, nx = shape
        h = I.level_h(nx, ny, nz)
        coeffs = I.random_coeffs(nx, ny, nz, 7)
        L = make_level(sf, shape, coeffs, parts=parts)
        C = make_level(sf, (nz // 2, ny // 2, nx // 2), I.random_coeffs(nx // 2, ny // 2, nz // 2, 6),
                       parts=parts)
        P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
        x, f = I.random_field(shape, 0), I.random_field(shape, 1)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F)
        xs = P.smooth(x, f, 1, dinv=P.dinv())
        assert rel(L.download(sf.SF_U), xs) < TOL
        assert rel(C.download(sf.SF_F), oracle.restrict_cell(P.residual(xs, f))) < TOL
    with pytest.raises(sf.SfError):
        sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, L.handle, sf.SF_F)


@pytest.mark.parametrize("n", [32, 64])
def test_vcycle_rr_matches_separate_residual(sf, monkeypatch, n):
    """The V-cycle with the fused last pre-smoothing pair (the delta-form
    residual + restriction, gsrb_rr.cu, forced on every level) and with the
    separate residual_restrict pass agree to rounding (1e-13)."""
    out = []
    monkeypatch.setenv("SF_RRF_CELLS", "0")
    for on in ("1", "0"):
        monkeypatch.setenv("SF_RRF", on)
        h = 1.0 / n
        coeffs = I.hpgmg_coeffs(n, n, n)
        L = make_level(sf, (n, n, n), coeffs, h=h)
        M = sf.MG(L, 1.0, 1.0)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        for _ in range(3):
            M.vcycle(0)
        out.append(L.download(sf.SF_U))
    assert rel(out[0], out[1]) < 1e-13


@pytest.mark.parametrize("n", [4, 16, 32, 64])
def test_vcycle_parity(sf, oracle, n):
    L, M, O = mg_pair(sf, oracle, n)
    assert M.num_levels == O.levels
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    u = np.zeros((n, n, n))
    L.upload(sf.SF_F, f)
    for _ in range(2):
        M.vcycle(0)
        u = O.vcycle(u, f)
        assert rel(L.download(sf.SF_U), u) < 1e-11


def test_fcycle_parity(sf, oracle):
    n = 32
    L, M, O = mg_pair(sf, oracle, n)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    M.fcycle()
    assert rel(L.download(sf.SF_U), O.fcycle(f)) < 1e-11


@pytest.mark.parametrize("fcycle", [False, True])
def test_c2_solve_parity(sf, oracle, fcycle):
    """BASELINE config 2: 64^3 VC Helmholtz solved to 1e-10; same cycle count
    as the oracle and u within 1e-10 relative L2."""
    n = 64
    L, M, O = mg_pair(sf, oracle, n)
    ue, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=fcycle, rtol=1e-10)
    u_o, hist_o = O.solve(f, fcycle=fcycle, rtol=1e-10)
    u = L.download(sf.SF_U)
    assert cyc == len(hist_o)
    assert hist[-1] < 1e-10
    assert rel(u, u_o) < 1e-10
    assert abs(np.abs(u - ue).max() - 5.19e-7) < 0.05e-6


@pytest.mark.parametrize("pre,post", [(1, 3), (3, 1), (2, 2), (1, 1)])
@pytest.mark.parametrize("use_graph", [0, 1])
def test_fused_check_pair_counts(sf, oracle, pre, post, use_graph):
    """The convergence check fused into the pairs (red part reduced by the next
    cycle's first pair, black part by the last post pair, whose reset rides in
    the P0-fused pair when post >= 2) for several pre/post pair counts: the
    oracle's cycle count and residual history, u within 1e-10.  V(1,1) with P0
    interpolation stalls at relres ~1 on this problem -- in the oracle too --
    so it is compared over 12 cycles (SF_ERR_NOT_CONVERGED on both sides)."""
    n = 64
    h = 1.0 / n
    coeffs = I.hpgmg_coeffs(n, n, n, h)
    L = make_level(sf, (n, n, n), coeffs, h=h)
    M = sf.MG(L, 1.0, 1.0, pre_pairs=pre, post_pairs=post, use_graph=use_graph)
    O = oracle.MG(n, n, n, h, 1.0, 1.0, *coeffs, pre=pre, post=post)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    maxc = 12 if (pre, post) == (1, 1) else 50
    st, cyc, hist = M.solve(fcycle=False, rtol=1e-10, max_cycles=maxc, raise_on_error=False)
    u_o, hist_o = O.solve(f, fcycle=False, rtol=1e-10, maxc=maxc)
    assert cyc == len(hist_o)
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-14)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10
    if (pre, post) == (1, 1):
        assert st == sf.SF_ERR_NOT_CONVERGED and hist[-1] > 0.5
    else:
        assert st == sf.SF_OK and hist[-1] < 1e-10


@pytest.mark.parametrize("shape", [(32, 16, 64), (64, 32, 32), (32, 64, 32)])
@pytest.mark.parametrize("use_graph", [0, 1])
def test_noncube_solve_parity(sf, oracle, shape, use_graph):
    """Non-cube boxes (C5's per-GPU shapes are not cubes): F-cycle + V-cycles to
    1e-10 through the host loop and the device loop, same cycle count as the
    oracle, u within 1e-10.  (Hierarchies whose coarsest box would exceed 64
    cells are rejected with SF_ERR_SHAPE by sf_mg_plan -- reading R-8.)"""
    nz, ny, nx = shape
    L, M, O = mg_pair(sf, oracle, None, shape=shape, use_graph=use_graph)
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
    u_o, hist_o = O.solve(f, fcycle=True, rtol=1e-10)
    assert cyc == len(hist_o)
    assert hist[-1] < 1e-10
    # relres entries agree to rounding of max|f - Au| (~1e-16 of max|f|)
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-14)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10


def test_solve_graph_replay_stable(sf, oracle):
    """Repeated solves through the captured CUDA graphs give identical results."""
    n = 32
    L, M, O = mg_pair(sf, oracle, n)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    res = []
    for _ in range(3):
        L.upload(sf.SF_U, np.zeros((n, n, n)))
        L.upload(sf.SF_F, f)
        st, cyc, hist = M.solve(fcycle=True)
        res.append(L.download(sf.SF_U))
    assert np.array_equal(res[0], res[1]) and np.array_equal(res[1], res[2])


# ------------------------------------------------------- decomposition (loopback)
@pytest.mark.parametrize("parts", [2, 4])
def test_decomposition_invariance_smoother(sf, parts):
    shape = (32, 16, 64)
    nz, ny, nx = shape
    coeffs = I.hpgmg_coeffs(nx, ny, nz)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    out = {}
    for P in (1, parts):
        for kind in (sf.SF_SMOOTH_COLOUR, sf.SF_SMOOTH_FUSED):
            L = make_level(sf, shape, coeffs, parts=P)
            sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
            L.upload(sf.SF_U, x)
            L.upload(sf.SF_F, f)
            sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
            sf.sf_residual(L.handle, sf.SF_R, sf.SF_U, sf.SF_F, 1.0, 1.0)
            out[(P, kind)] = (L.download(sf.SF_U), L.download(sf.SF_R))
    for kind in (sf.SF_SMOOTH_COLOUR, sf.SF_SMOOTH_FUSED):
        assert np.array_equal(out[(1, kind)][0], out[(parts, kind)][0])
        assert np.array_equal(out[(1, kind)][1], out[(parts, kind)][1])


@pytest.mark.parametrize("parts", [2, 4])
@pytest.mark.parametrize("overlap", ["1", "0"])
def test_halo_overlap_bit_identical(sf, oracle, parts, overlap, monkeypatch):
    """>= 24 planes per part: the depth-2 halo runs on a side stream beside the
    interior z-chunks, the boundary chunks after the join (SF_HALO_OVERLAP=1),
    or before one launch (0).  Both equal the undecomposed level bit for bit,
    for the plain, check-fused (solve) and P0-fused (V-cycle) pairs."""
    monkeypatch.setenv("SF_HALO_OVERLAP", overlap)
    shape = (96, 32, 64)
    nz, ny, nx = shape
    coeffs = I.hpgmg_coeffs(nx, ny, nz)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    out = {}
    for P in (1, parts):
        L = make_level(sf, shape, coeffs, parts=P)
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 3, sf.SF_SMOOTH_FUSED)
        out[P] = L.download(sf.SF_U)
    assert np.array_equal(out[1], out[parts])
    P = oracle.Problem(oracle.Grid(nx, ny, nz, I.level_h(nx, ny, nz)), 1.0, 1.0, *coeffs)
    assert rel(out[parts], P.smooth(x, f, 3, dinv=P.dinv())) < TOL
    n = 96
    sol = {}
    for Pn in (1, parts):
        L, M, O = mg_pair(sf, oracle, n, shape=(n, 64, 64), parts=Pn, agglom_min_planes=4)
        _, fm = I.manufactured(64, 64, n, 1.0, 1.0)
        L.upload(sf.SF_F, fm)
        st, cyc, hist = M.solve(fcycle=True)
        sol[Pn] = (L.download(sf.SF_U), cyc)
    assert sol[1][1] == sol[parts][1]
    assert rel(sol[parts][0], sol[1][0]) < 1e-13


@pytest.mark.parametrize("parts", [2, 4])
def test_decomposition_invariance_solve(sf, oracle, parts):
    n = 64
    shape = (n, n, n)
    res = {}
    for P in (1, parts):
        L, M, O = mg_pair(sf, oracle, n, parts=P, agglom_min_planes=4)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        st, cyc, hist = M.solve(fcycle=True)
        res[P] = (L.download(sf.SF_U), cyc)
    assert res[1][1] == res[parts][1]
    assert rel(res[parts][0], res[1][0]) < 1e-13


# ------------------------------------------------------- full-size (BASELINE C3)
def test_c3_full_size_gsrb_pair(sf, oracle):
    """256^3 HPGMG-shaped level, the fused pair bench.py times, element by
    element against the oracle (one pair: a few seconds on the host)."""
    n = 256
    shape = (n, n, n)
    coeffs = I.hpgmg_coeffs(n, n, n)
    L = make_level(sf, shape, coeffs)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
    got = L.download(sf.SF_U)
    P = oracle.Problem(oracle.Grid(n, n, n, 1.0 / n), 1.0, 1.0, *coeffs)
    exp = P.smooth(x, f, 1)
    assert rel(got, exp) < TOL
    # one wrong cell of 2^24 would hide in the relative L2 norm: bound every cell
    assert np.abs(got - exp).max() <= 10 * TOL * np.abs(exp).max()


@pytest.mark.parametrize("fcycle", [False, True])
def test_solve_eager_equals_graph(sf, oracle, fcycle):
    """The fused convergence check (first pre-smoothing pair reduces the input
    residual) gives the same iterate and cycle count with and without CUDA
    graph replay."""
    n = 32
    out = {}
    for g in (0, 1):
        L, M, O = mg_pair(sf, oracle, n, use_graph=g)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        st, cyc, hist = M.solve(fcycle=fcycle, rtol=1e-10)
        out[g] = (L.download(sf.SF_U), cyc, hist)
    assert out[0][1] == out[1][1]
    assert np.array_equal(out[0][0], out[1][0])
    assert np.allclose(out[0][2], out[1][2], rtol=1e-12, atol=0)


@pytest.mark.parametrize("fcycle", [False, True])
@pytest.mark.parametrize("parts", [1, 2])
def test_device_loop_equals_host_loop(sf, oracle, fcycle, parts):
    """With graphs the whole solve is one graph launch whose WHILE node is
    driven by the device-side convergence decision; it must reproduce the host
    loop exactly: iterate, cycle count, every history entry (same IEEE
    division) and the number of kernel launches."""
    n = 32
    out = {}
    for g in (0, 1):
        L, M, O = mg_pair(sf, oracle, n, parts=parts, use_graph=g)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        for rep in range(2):   # second solve: replay of the built loop
            L.upload(sf.SF_U, np.zeros((n, n, n)))
            sf.sf_launch_count(reset=True)
            st, cyc, hist = M.solve(fcycle=fcycle, rtol=1e-10)
            launches = sf.sf_launch_count(reset=True)
        out[g] = (L.download(sf.SF_U), cyc, hist, launches)
    assert out[0][1] == out[1][1] and out[0][2] == out[1][2]
    assert np.array_equal(out[0][0], out[1][0])
    # same kernels; the device loop adds its init + publish kernels and drops
    # the host loop's copy of max|F| to the host
    assert out[1][3] == out[0][3] + 1


def test_device_loop_capture_failure_falls_back(sf, oracle, monkeypatch):
    """A device-loop capture that fails inside the WHILE body leaves the level
    mappings intact and the solve runs the host loop: same iterate and cycles
    as a hierarchy that never tried."""
    n = 32
    out = []
    for fail in (False, True):
        if fail:
            monkeypatch.setenv("SF_TEST_LOOP_FAIL", "1")
        L, M, O = mg_pair(sf, oracle, n)
        _, f = I.manufactured(n, n, n, 1.0, 1.0)
        L.upload(sf.SF_F, f)
        st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
        L.upload(sf.SF_U, np.zeros((n, n, n)))
        st, cyc2, hist2 = M.solve(fcycle=True, rtol=1e-10)   # replay / host loop again
        out.append((L.download(sf.SF_U), cyc, hist, cyc2))
    assert out[0][1] == out[1][1] == out[0][3] == out[1][3]
    assert out[0][2] == out[1][2]
    assert np.array_equal(out[0][0], out[1][0])


@pytest.mark.parametrize("use_graph", [0, 1])
def test_solve_zero_and_nan_rhs(sf, oracle, use_graph):
    """f = 0 gives u = 0 after zero cycles; a NaN in f is reported, not solved."""
    n = 32
    L, M, O = mg_pair(sf, oracle, n, use_graph=use_graph)
    L.upload(sf.SF_U, I.random_field((n, n, n), 3))
    L.upload(sf.SF_F, np.zeros((n, n, n)))
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, raise_on_error=False)
    assert st == sf.SF_OK and cyc == 0
    assert not L.download(sf.SF_U).any()
    f = I.random_field((n, n, n), 1)
    f[3, 4, 5] = np.nan
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, raise_on_error=False)
    assert st == sf.SF_ERR_NUMERIC and cyc == 0


@pytest.mark.parametrize("use_graph", [0, 1])
def test_solve_max_cycles_keeps_last_cycle(sf, oracle, use_graph):
    """Stopping at max_cycles discards the speculative first pair of the next
    cycle: U equals the oracle's iterate after exactly max_cycles cycles."""
    n = 64
    L, M, O = mg_pair(sf, oracle, n, use_graph=use_graph)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, max_cycles=3, raise_on_error=False)
    assert st == sf.SF_ERR_NOT_CONVERGED and cyc == 3
    u = O.fcycle(f)
    for _ in range(2):
        u = O.vcycle(u, f)
    assert rel(L.download(sf.SF_U), u) < 1e-11
    assert abs(hist[-1] / O.relres(u, f) - 1) < 1e-6


# ------------------------------------------------------- NEXT-2 (Fig 7 operators)
@pytest.mark.parametrize("shape", [(16, 16, 16), (8, 6, 10), (20, 64, 64), (33, 12, 40)])
def test_cc_laplacian_and_jacobi(sf, oracle, shape):
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    L = sf.Level(nx, ny, nz, h)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_apply_laplacian(L.handle, sf.SF_R, sf.SF_U)
    assert rel(L.download(sf.SF_R), oracle.laplacian_cc(x, h)) < TOL
    sf.sf_jacobi(L.handle, sf.SF_TMP, sf.SF_U, sf.SF_F, 2.0 / 3.0)
    assert rel(L.download(sf.SF_TMP), oracle.jacobi_cc(x, f, h)) < TOL


def test_cc_decomposition_invariance(sf):
    shape = (32, 16, 32)
    nz, ny, nx = shape
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    outs = []
    for P in (1, 4):
        comm = sf.Comm.local(P) if P > 1 else None
        L = sf.Level(nx, ny, nz, comm=comm)
        L.upload(sf.SF_U, x)
        L.upload(sf.SF_F, f)
        sf.sf_jacobi(L.handle, sf.SF_TMP, sf.SF_U, sf.SF_F, 2.0 / 3.0)
        outs.append(L.download(sf.SF_TMP))
    assert np.array_equal(outs[0], outs[1])


# ------------------------------------------------------- NEXT-3 (Chebyshev smoother)
def start_vector(shape):
    nz, ny, nx = shape
    k, j, i = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    return 1.0 + ((7 * i + 13 * j + 29 * k) % 17) / 17.0


@pytest.mark.parametrize("shape", [(16, 16, 16), (8, 6, 10), (20, 64, 64)])
def test_chebyshev_and_lambda_max(sf, oracle, shape):
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    coeffs = I.random_coeffs(nx, ny, nz, 8)
    L = make_level(sf, shape, coeffs)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    lam = sf.sf_lambda_max(L.handle, sf.SF_U, 1.0, 1.0, 20, True)
    lam_o = P.lambda_max(start_vector(shape), 20)
    assert abs(lam / lam_o - 1) < 1e-12
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    for degree in (1, 4, 5):
        L.upload(sf.SF_U, x)
        sf.sf_smooth_chebyshev(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, degree, 0.1 * lam, 1.05 * lam)
        exp = P.chebyshev(x, f, degree, 0.1 * lam, 1.05 * lam)
        assert rel(L.download(sf.SF_U), exp) < TOL


@pytest.mark.parametrize("graph", [0, 1])
def test_chebyshev_multigrid(sf, oracle, graph):
    n = 32
    L, M, O = mg_pair(sf, oracle, n, smoother=sf.SF_SMOOTH_CHEBY, cheby_degree=2,
                      use_graph=graph)
    O.set_chebyshev(2)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    u = np.zeros((n, n, n))
    for _ in range(2):
        M.vcycle(0)
        u = O.vcycle(u, f)
        assert rel(L.download(sf.SF_U), u) < 1e-11
    L.upload(sf.SF_U, np.zeros((n, n, n)))
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
    u_o, hist_o = O.solve(f, fcycle=True, rtol=1e-10)
    assert cyc == len(hist_o) and rel(L.download(sf.SF_U), u_o) < 1e-10


# ------------------------------------------------------- NEXT-2 / NEXT-3 at the bench size
def test_next2_next3_full_size_256(sf, oracle):
    """The Fig-7 operators at the 256^3 the bench times them on: the CC 7-point
    Laplacian, the CC weighted Jacobi step and one degree-2 Chebyshev
    application on the VC operator, every cell against the oracle (rel-L2 and
    max-abs relative to the largest value)."""
    shape = (256, 256, 256)
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    x, f = I.random_field(shape, 0), I.random_field(shape, 1)
    L = sf.Level(nx, ny, nz, h)
    L.upload(sf.SF_U, x)
    L.upload(sf.SF_F, f)
    sf.sf_apply_laplacian(L.handle, sf.SF_R, sf.SF_U)
    e = oracle.laplacian_cc(x, h)
    out = L.download(sf.SF_R)
    assert rel(out, e) < TOL and np.abs(out - e).max() <= TOL * np.abs(e).max()
    sf.sf_jacobi(L.handle, sf.SF_TMP, sf.SF_U, sf.SF_F, 2.0 / 3.0)
    e = oracle.jacobi_cc(x, f, h)
    out = L.download(sf.SF_TMP)
    assert rel(out, e) < TOL and np.abs(out - e).max() <= TOL * np.abs(e).max()
    coeffs = I.hpgmg_coeffs(nx, ny, nz, h)
    L.set_coeffs(*coeffs)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *coeffs)
    L.upload(sf.SF_U, x)
    sf.sf_smooth_chebyshev(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, 20.0, 900.0)
    e = P.chebyshev(x, f, 2, 20.0, 900.0)
    out = L.download(sf.SF_U)
    assert rel(out, e) < TOL and np.abs(out - e).max() <= 10 * TOL * np.abs(e).max()
    L.close()
