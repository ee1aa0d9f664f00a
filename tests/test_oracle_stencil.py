"""Pins of the generic-stencil oracle (oracle/stencil.py, NEXT-4) against what
the paper and the already-pinned HPGMG oracle fix (no GPU):

* Fig 4 in 3-D -- Dirichlet face stencils + the red / black variable-
  coefficient stencils over stride-2 DomainUnions -- equals the oracle's GSRB
  colour sweep (pinned to dense Gauss-Seidel in test_oracle_pins.py);
* restriction as a strided affine stencil equals or_restrict_cell bit for bit;
* P0 interpolation (floor((p+1)/2) affine reads) equals or_interp_p0 bit for bit;
* the constant-coefficient 7-point stencil equals or_laplacian_cc;
* the domain / weight / snapshot semantics against a pure-Python brute force
  written independently here (point by point, dict-of-points domains)."""
import itertools

import numpy as np
import pytest

from oracle import stencil as OS
from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

from stencil_specs import (BLACK, I3, ONE, RED, at, bc_faces, comp, gsrb_colour,  # noqa: E402
                           p0_spec, restriction_spec)


def padded_meshes(shape, coeffs, x, f, dinv):
    from oracle import oracle as O
    alpha, bi, bj, bk = coeffs
    return {"u": O.pad(x), "f": O.pad(f), "dinv": O.pad(dinv), "alpha": O.pad(alpha),
            "beta_i": O.pad(bi, "beta_i"), "beta_j": O.pad(bj, "beta_j"),
            "beta_k": O.pad(bk, "beta_k"), "r": np.zeros(tuple(s + 2 for s in shape)),
            "tmp": np.zeros(tuple(s + 2 for s in shape))}


@pytest.mark.parametrize("shape", [(4, 6, 8), (5, 3, 7)])
@pytest.mark.parametrize("ab", [(0.0, 1.0), (1.3, 0.7)])
def test_fig4_gsrb_equals_oracle_sweep(oracle, shape, ab):
    nz, ny, nx = shape
    a, b = ab
    h = 1.0 / 8
    coeffs = I.random_coeffs(nx, ny, nz, 3)
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), a, b, *coeffs)
    x, f, dinv = I.random_field(shape, 0), I.random_field(shape, 1), P.dinv()
    M = padded_meshes(shape, coeffs, x, f, dinv)
    red = bc_faces("u") + [gsrb_colour(a, b, h, RED)]
    black = bc_faces("u") + [gsrb_colour(a, b, h, BLACK)]
    M1 = OS.apply_group(red, M)
    exp1 = P.gsrb_sweep(x, f, 0, dinv)
    got1 = oracle.interior(M1["u"])
    assert np.abs(got1 - exp1).max() <= 1e-13 * np.abs(exp1).max()
    M2 = OS.apply_group(black, M1)
    exp2 = P.gsrb_sweep(exp1, f, 1, dinv)
    got2 = oracle.interior(M2["u"])
    assert np.abs(got2 - exp2).max() <= 1e-13 * np.abs(exp2).max()
    # the red stencil changed red cells only (black untouched) and the ghosts
    # hold -inside (A2 faces)
    k, j, i = np.meshgrid(range(nz), range(ny), range(nx), indexing="ij")
    black_mask = (i + j + k) % 2 == 1
    assert np.array_equal(got1[black_mask], x[black_mask])
    xp = oracle.pad(x)
    assert np.array_equal(M1["u"][0, 1:-1, 1:-1], -xp[1, 1:-1, 1:-1])
    assert np.array_equal(M1["u"][1:-1, 1:-1, -1], -xp[1:-1, 1:-1, -2])


@pytest.mark.parametrize("shape", [(4, 6, 8), (8, 2, 6)])
def test_restriction_and_p0_bit_exact(oracle, shape):
    nz, ny, nx = shape
    fine = I.random_field(shape, 5)
    coarse = I.random_field((nz // 2, ny // 2, nx // 2), 6)
    Mf = {"r": oracle.pad(fine), "u": oracle.pad(fine)}
    Mc = {"f": np.zeros((nz // 2 + 2, ny // 2 + 2, nx // 2 + 2)), "u": oracle.pad(coarse)}
    got = OS.apply_group([restriction_spec("f", "r")], Mc, Mf)
    assert np.array_equal(oracle.interior(got["f"]), oracle.restrict_cell(fine))
    got = OS.apply_group([p0_spec("u", "u")], Mf, Mc)
    assert np.array_equal(oracle.interior(got["u"]), oracle.interpolate(fine, coarse, 1.0, "p0"))


def test_cc_laplacian(oracle):
    shape = (6, 5, 4)
    nz, ny, nx = shape
    h = 0.25
    x = I.random_field(shape, 2)
    M = {"u": oracle.pad(x), "r": np.zeros((nz + 2, ny + 2, nx + 2))}
    c = -1.0 / (h * h)
    lap = comp("u", [((0, 0, 0), -6.0 * c), ((-1, 0, 0), c), ((1, 0, 0), c), ((0, -1, 0), c),
                     ((0, 1, 0), c), ((0, 0, -1), c), ((0, 0, 1), c)])
    got = OS.apply_group(bc_faces("u") + [{"out": "r", "rects": [(ONE, I3, ONE)], "expr": lap}], M)
    exp = oracle.laplacian_cc(x, h)
    assert np.abs(oracle.interior(got["r"]) - exp).max() <= 1e-13 * np.abs(exp).max()


# --------------------------------------------------------------- brute force
def _bf_points(rect, shape_zyx):
    lo, hi, st = rect
    N = (shape_zyx[2], shape_zyx[1], shape_zyx[0])
    per = []
    for d in range(3):
        a = lo[d] if lo[d] >= 0 else N[d] + lo[d]
        b = hi[d] if hi[d] >= 0 else N[d] + hi[d]
        vals = []
        if st[d] == 0:
            vals = [a]
        else:
            v = a
            while v < b:
                vals.append(v)
                v += st[d]
        per.append(vals)
    return [(x, y, z) for z in per[2] for y in per[1] for x in per[0]]


def _bf_eval(E, p, M):
    if E[0] == "const":
        return E[1]
    if E[0] == "comp":
        _, mesh, terms, src, mul, div, pre = E
        tot, first = 0.0, True
        for off, w in terms:
            if not isinstance(w, tuple) and w == 0.0:
                continue
            q = [(mul[d] * p[d] + pre[d]) // div[d] + off[d] for d in range(3)]
            v = M[mesh][q[2]][q[1]][q[0]]
            t = v if (not isinstance(w, tuple) and w == 1.0) else (
                (_bf_eval(w, p, M) if isinstance(w, tuple) else w) * v)
            tot, first = (t, False) if first else (tot + t, False)
        return tot
    if E[0] == "neg":
        return -_bf_eval(E[1], p, M)
    a, b = _bf_eval(E[1], p, M), _bf_eval(E[2], p, M)
    if E[0] == "+":
        return a + b
    if E[0] == "-":
        return a - b
    return a * b if E[0] == "*" else a / b


def _rand_expr(rng, depth=0):
    meshes = ["u", "f", "alpha"]
    k = rng.integers(0, 4 if depth < 2 else 2)
    if k == 0:
        return ("const", float(rng.uniform(-2, 2)))
    if k == 1:
        terms = []
        for _ in range(rng.integers(1, 4)):
            off = tuple(int(v) for v in rng.integers(-1, 2, size=3))
            w = [1.0, 0.0, float(rng.uniform(-1, 1))][rng.integers(0, 3)]
            if depth < 1 and rng.random() < 0.3:
                w = _rand_expr(rng, depth + 1)
            terms.append((off, w))
        return comp(meshes[rng.integers(0, 3)], terms)
    op = ["+", "-", "*", "neg"][rng.integers(0, 4)]
    if op == "neg":
        return ("neg", _rand_expr(rng, depth + 1))
    return (op, _rand_expr(rng, depth + 1), _rand_expr(rng, depth + 1))


def _rand_rect(rng):
    lo, hi, st = [], [], []
    for _ in range(3):
        s = int(rng.integers(0, 3))
        a = int(rng.integers(1, 3))
        b = int(rng.integers(-2, 0))
        lo.append(a if rng.random() < 0.8 else -2)
        hi.append(b)
        st.append(s)
    return tuple(lo), tuple(hi), tuple(st)


def test_brute_force_random_groups():
    rng = np.random.default_rng(11)
    shape = (5, 6, 7)          # ghost-inclusive (z, y, x)
    for trial in range(40):
        M = {m: rng.uniform(-1, 1, size=shape) for m in ("u", "f", "alpha")}
        group = []
        for _ in range(rng.integers(1, 3)):
            out = ["u", "f"][rng.integers(0, 2)]
            rects = [_rand_rect(rng) for _ in range(rng.integers(1, 3))]
            group.append({"out": out, "rects": rects, "expr": _rand_expr(rng)})
        got = OS.apply_group(group, M)
        # brute force: point by point from a snapshot, stencil by stencil
        cur = {k: v.tolist() for k, v in M.items()}
        for s in group:
            snap = {k: [[list(r) for r in pl] for pl in v] for k, v in cur.items()}
            pts = {}
            for r in s["rects"]:
                for p in _bf_points(r, shape):
                    pts[p] = _bf_eval(s["expr"], p, snap)
            for (x, y, z), v in pts.items():
                cur[s["out"]][z][y][x] = v
        for k in M:
            assert np.array_equal(got[k], np.array(cur[k])), (trial, k)


def test_in_place_reads_the_values_before_the_stencil():
    """Snapshot semantics: an in-place 7-point average over the interior uses
    old neighbours everywhere (closed form with numpy slices)."""
    rng = np.random.default_rng(4)
    u = rng.uniform(-1, 1, size=(6, 7, 8))
    terms = [(o, 1.0) for o in itertools.product((-1, 0, 1), repeat=3) if sum(map(abs, o)) <= 1]
    got = OS.apply_group([{"out": "u", "rects": [(ONE, I3, ONE)], "expr": comp("u", terms)}],
                         {"u": u})["u"]
    exp = u.copy()
    acc = None
    for (ox, oy, oz), _ in terms:
        t = u[1 + oz:u.shape[0] - 1 + oz, 1 + oy:u.shape[1] - 1 + oy, 1 + ox:u.shape[2] - 1 + ox]
        acc = t if acc is None else acc + t
    exp[1:-1, 1:-1, 1:-1] = acc
    assert np.array_equal(got, exp)
