"""GPU parity of the generic stencil engine (NEXT-4): JIT-compiled sm_100a
kernels (NVRTC) through the C ABI against the stencil oracle
(oracle/stencil.py) on the same plain-data specs -- bit for bit, the engine
evaluates each DAG in IEEE order without contraction -- and against the
pinned HPGMG oracle / hand-written kernels for the paper's Fig 4 smoother,
restriction and interpolation."""
import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I
from stencil_specs import (BLACK, RED, at, bc_faces, comp, gsrb_colour, p0_spec,
                           restriction_spec, to_dsl)

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


FIELDS = ["u", "f", "r", "tmp", "alpha", "beta_i", "beta_j", "beta_k", "dinv"]
KIND = {"beta_i": "beta_i", "beta_j": "beta_j", "beta_k": "beta_k"}


def level_with(sf, shape, host, comm=None):
    """Level whose interiors (face arrays incl. their last face) are `host`."""
    nz, ny, nx = shape
    L = sf.Level(nx, ny, nz, h=1.0 / 8, comm=comm)
    L._keep = comm
    for name, arr in host.items():
        L.upload(sf.FIELD_IDS[name], arr)
    return L


def host_fields(shape, seed):
    nz, ny, nx = shape
    alpha, bi, bj, bk = I.random_coeffs(nx, ny, nz, seed)
    out = {"alpha": alpha, "beta_i": bi, "beta_j": bj, "beta_k": bk}
    for k, name in enumerate(["u", "f", "r", "tmp", "dinv"]):
        out[name] = I.random_field(shape, seed + 10 + k)
    return out


def oracle_meshes(oracle, host):
    return {k: oracle.pad(v, KIND.get(k, "cell")) for k, v in host.items()}


def padded_all(sf, L):
    return {k: L.padded(sf.FIELD_IDS[k]) for k in FIELDS}


def _rand_expr(rng, depth=0):
    meshes = ["u", "f", "alpha", "beta_i", "dinv"]
    k = rng.integers(0, 4 if depth < 2 else 2)
    if k == 0:
        return ("const", float(rng.uniform(-2, 2)))
    if k == 1:
        terms, seen = [], set()
        for _ in range(rng.integers(1, 5)):
            off = tuple(int(v) for v in rng.integers(-1, 2, size=3))
            if off in seen:
                continue
            seen.add(off)
            w = [1.0, 0.0, float(rng.uniform(-1, 1))][rng.integers(0, 3)]
            if depth < 1 and rng.random() < 0.3:
                w = _rand_expr(rng, depth + 1)
            terms.append((off, w))
        return comp(meshes[rng.integers(0, len(meshes))], terms)
    op = ["+", "-", "*", "/", "neg"][rng.integers(0, 5)]
    if op == "neg":
        return ("neg", _rand_expr(rng, depth + 1))
    if op == "/":
        return ("/", _rand_expr(rng, depth + 1), ("+", ("const", 3.0), at("alpha")))
    return (op, _rand_expr(rng, depth + 1), _rand_expr(rng, depth + 1))


def _rand_rect(rng):
    lo, hi, st = [], [], []
    for _ in range(3):
        s = int(rng.integers(0, 4))
        lo.append(int(rng.integers(1, 4)))
        hi.append(int(rng.integers(-3, 0)))
        st.append(s)
    return tuple(lo), tuple(hi), tuple(st)


@pytest.mark.parametrize("shape", [(9, 10, 12), (5, 7, 33)])
def test_random_groups_bit_exact(sf, oracle, shape):
    from oracle import stencil as OS
    rng = np.random.default_rng(sum(shape))
    for trial in range(6):
        host = host_fields(shape, trial)
        group = []
        for _ in range(rng.integers(1, 4)):
            out = ["r", "tmp"][rng.integers(0, 2)]
            rects = [_rand_rect(rng) for _ in range(rng.integers(1, 4))]
            group.append({"out": out, "rects": rects, "expr": _rand_expr(rng)})
        L = level_with(sf, shape, host)
        g = to_dsl(group).compile()
        g(L)
        got = padded_all(sf, L)
        exp = OS.apply_group(group, oracle_meshes(oracle, host))
        for k in ("r", "tmp"):
            assert np.array_equal(got[k], exp[k]), (trial, k)
        assert g.phases == g.plan(shape[2], shape[1], shape[0])
        g.close()
        L.close()


@pytest.mark.parametrize("shape", [(8, 8, 8), (6, 10, 14)])
@pytest.mark.parametrize("ab", [(0.0, 1.0), (1.0, 1.0)])
def test_fig4_gsrb_group(sf, oracle, shape, ab):
    """Fig 4 in 3-D (BC faces + red, BC faces + black) on the GPU: bit-exact vs
    the stencil oracle, 1e-12 vs the oracle's RB pair, and it matches the
    hand-written colour-sweep kernels."""
    from oracle import stencil as OS
    nz, ny, nx = shape
    a, b = ab
    h = 1.0 / 8
    host = host_fields(shape, 3)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), a, b, host["alpha"], host["beta_i"],
                       host["beta_j"], host["beta_k"])
    host["dinv"] = P.dinv()
    spec = bc_faces("u") + [gsrb_colour(a, b, h, RED)] + bc_faces("u") + [gsrb_colour(a, b, h, BLACK)]
    L = level_with(sf, shape, host)
    g = to_dsl(spec).compile()
    g(L)
    assert g.phases == 4
    got = L.padded(sf.SF_U)
    exp = OS.apply_group(spec, oracle_meshes(oracle, host))["u"]
    assert np.array_equal(got, exp)
    ref = P.smooth(host["u"], host["f"], 1, host["dinv"])
    gi = oracle.interior(got)
    assert np.linalg.norm(gi - ref) <= 1e-12 * np.linalg.norm(ref)
    # the hand-written colour sweeps on the same data
    L2 = level_with(sf, shape, host)
    sf.sf_rebuild_operator(L2.handle, a, b)
    sf.sf_smooth_gsrb(L2.handle, sf.SF_U, sf.SF_F, a, b, 1, sf.SF_SMOOTH_COLOUR)
    hw = L2.download(sf.SF_U)
    assert np.linalg.norm(gi - hw) <= 1e-13 * np.linalg.norm(hw)
    g.close()


@pytest.mark.parametrize("shape", [(8, 8, 8), (4, 6, 16)])
def test_restriction_p0_cross_level(sf, oracle, shape):
    nz, ny, nx = shape
    fine = I.random_field(shape, 5)
    coarse = I.random_field((nz // 2, ny // 2, nx // 2), 6)
    Lf = level_with(sf, shape, {"r": fine, "u": fine})
    Lc = level_with(sf, (nz // 2, ny // 2, nx // 2), {"u": coarse})
    R = to_dsl([restriction_spec("f", "r")]).compile()
    R(Lc, Lf)
    assert np.array_equal(Lc.download(sf.SF_F), oracle.restrict_cell(fine))
    # and equals the hand-written restriction kernel
    sf.sf_restrict(Lc.handle, sf.SF_TMP, Lf.handle, sf.SF_R, sf.SF_RESTRICT_CELL)
    assert np.array_equal(Lc.download(sf.SF_TMP), Lc.download(sf.SF_F))
    P0 = to_dsl([p0_spec("u", "u")]).compile()
    P0(Lf, Lc)
    assert np.array_equal(Lf.download(sf.SF_U), oracle.interpolate(fine, coarse, 1.0, "p0"))
    R.close()
    P0.close()


@pytest.mark.parametrize("parts", [2, 4])
def test_multipart_equals_single(sf, parts):
    """z-slab parts (loopback): halos of the meshes read across planes are
    exchanged before each launch; the result equals the undecomposed run."""
    shape = (16, 8, 12)
    nz, ny, nx = shape
    h = 1.0 / 16
    host = host_fields(shape, 8)
    spec = bc_faces("u") + [gsrb_colour(1.0, 1.0, h, RED)] + bc_faces("u") + [
        gsrb_colour(1.0, 1.0, h, BLACK)]
    res = {}
    for P in (1, parts):
        comm = sf.Comm.local(P) if P > 1 else None
        L = level_with(sf, shape, host, comm)
        g = to_dsl(spec).compile()
        g(L)
        res[P] = L.download(sf.SF_U)
        g.close()
    assert np.array_equal(res[1], res[parts])


def test_errors(sf):
    shape = (8, 8, 8)
    L = level_with(sf, shape, {"u": I.random_field(shape, 0)})
    from paper_conf_ipps_zhangdmwbf17_b200 import stencil as S
    racy = S.Stencil(S.Component("u", {(1, 0, 0): 1.0, (-1, 0, 0): 1.0}), "u",
                     S.RectDomain((1, 1, 1), (-1, -1, -1))).compile()
    with pytest.raises(sf.SfError) as e:
        racy(L)
    assert e.value.status == sf.SF_ERR_INVALID
    far = S.Stencil(S.Component("u", {(0, 5, 0): 1.0}), "r",
                    S.RectDomain((1, 1, 1), (-1, -1, -1))).compile()
    with pytest.raises(sf.SfError) as e:
        far(L)
    assert e.value.status == sf.SF_ERR_SHAPE
    # reads inside the storage ghost zone (2 layers on every axis) are fine
    ok = S.Stencil(S.Component("u", {(-2, 0, 0): 1.0, (0, 2, 0): 1.0}), "r",
                   S.RectDomain((1, 1, 1), (-1, -1, -1))).compile()
    ok(L)
    sf.sf_sync(L.handle)
    for c in (racy, far, ok):
        c.close()
