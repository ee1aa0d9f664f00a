"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself:
closed forms, textbook matrices, brute force on tiny grids, invariants and
the values the paper fixes.  CPU only (no GPU marker).

Each test names the oracle function(s) it pins and the passage it checks.
"""
import json
import os

import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def centres(n, h):
    return (np.arange(n) + 0.5) * h


def sine_mode(nx, ny, nz, h, m):
    x, y, z = centres(nx, h), centres(ny, h), centres(nz, h)
    L = (nx * h, ny * h, nz * h)
    return (np.sin(np.pi * m[0] * x / L[0])[None, None, :]
            * np.sin(np.pi * m[1] * y / L[1])[None, :, None]
            * np.sin(np.pi * m[2] * z / L[2])[:, None, None])


def dense_op(P, shape):
    """Dense matrix of the oracle operator (unit-vector columns)."""
    n = int(np.prod(shape))
    A = np.zeros((n, n))
    for c in range(n):
        e = np.zeros(n)
        e[c] = 1.0
        A[:, c] = P.apply_op(e.reshape(shape)).ravel()
    return A


# ----------------------------------------------------------------- A2 (BC)
def test_bc_face_edge_corner_values_vanish(oracle):
    """ghost = -inside makes the boundary value zero.  The
    (bi/tri)linear interpolant of the ghost zone onto every boundary face
    midpoint, edge and corner must therefore be 0 (reading R-5)."""
    nx, ny, nz = 5, 4, 3
    g = oracle.Grid(nx, ny, nz, 1.0)
    x = oracle.pad(I.random_field((nz, ny, nx), 3))
    oracle.apply_bc(g, x)
    # faces: average of ghost and its inside neighbour
    assert np.abs(x[1:-1, 1:-1, 0] + x[1:-1, 1:-1, 1]).max() == 0
    assert np.abs(x[1:-1, 1:-1, -1] + x[1:-1, 1:-1, -2]).max() == 0
    assert np.abs(x[1:-1, 0, 1:-1] + x[1:-1, 1, 1:-1]).max() == 0
    assert np.abs(x[0, 1:-1, 1:-1] + x[1, 1:-1, 1:-1]).max() == 0
    assert np.abs(x[-1, 1:-1, 1:-1] + x[-2, 1:-1, 1:-1]).max() == 0
    # edges: 4 cells around the edge line sum to zero
    e = x[1:-1, 0, 0] + x[1:-1, 1, 0] + x[1:-1, 0, 1] + x[1:-1, 1, 1]
    assert np.abs(e).max() == 0
    e = x[0, 1:-1, -1] + x[1, 1:-1, -1] + x[0, 1:-1, -2] + x[1, 1:-1, -2]
    assert np.abs(e).max() == 0
    # corners: 8 cells around the corner point sum to zero
    for cz in (0, -2):
        for cy in (0, -2):
            for cx in (0, -2):
                blk = x[slice(cz, cz + 2) if cz == 0 else slice(-2, None),
                        slice(cy, cy + 2) if cy == 0 else slice(-2, None),
                        slice(cx, cx + 2) if cx == 0 else slice(-2, None)]
                assert abs(blk.sum()) < 1e-15


# ----------------------------------------------------------------- A3 (op)
@pytest.mark.parametrize("m", [(1, 2, 3), (2, 1, 1), (3, 3, 2)])
@pytest.mark.parametrize("a", [0.0, 2.0])
def test_op_sine_eigenfunction_closed_form(oracle, m, a):
    """Constant-coefficient operator on a sine mode: A u = (a*alpha +
    b*(4/h^2)*sum_d sin^2(pi m_d h/2)) u exactly, boundary cells included
    (the odd reflection of PAPER.md:336-341 is exact for sine modes)."""
    n, h, b, alpha0, beta0 = 8, 1.0 / 8, 1.5, 1.25, 1.0
    u = sine_mode(n, n, n, h, m)
    al, bi, bj, bk = I.constant_coeffs(n, n, n, alpha0, beta0)
    P = oracle.Problem(oracle.Grid(n, n, n, h), a, b, al, bi, bj, bk)
    lam = a * alpha0 + b * beta0 * 4 / h**2 * sum(np.sin(np.pi * mm * h / 2) ** 2 for mm in m)
    Au = P.apply_op(u)
    assert np.abs(Au - lam * u).max() <= 1e-12 * lam


def test_op_quadratic_exact_interior(oracle):
    """-Lap_h(x^2 + 2y^2 - z^2) = -(2+4-2) = -4 exactly (second differences
    are exact on quadratics) on cells whose neighbours are all interior."""
    n, h = 8, 1.0 / 8
    x, y, z = centres(n, h)[None, None, :], centres(n, h)[None, :, None], centres(n, h)[:, None, None]
    u = np.broadcast_to(x**2 + 2 * y**2 - z**2, (n, n, n)).copy()
    P = oracle.Problem(oracle.Grid(n, n, n, h), 0.0, 1.0, *I.constant_coeffs(n, n, n))
    Au = P.apply_op(u)[1:-1, 1:-1, 1:-1]
    assert np.abs(Au + 4.0).max() < 1e-10


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_op_variable_beta_face_convention(oracle, axis):
    """-d/dx((1+x) d/dx x^2) = -(2+4x): exact in the discrete flux form when
    beta is linear and sampled on faces and u is quadratic.  Pins the face
    convention (beta_i(i) = face between cells i-1 and i)."""
    n, h = 8, 1.0 / 8
    c = centres(n, h)
    f = np.arange(n + 1) * h
    shp = [1, 1, 1]
    shp[2 - axis] = n
    u = np.broadcast_to((c**2).reshape(shp), (n, n, n)).copy()
    al, bi, bj, bk = I.constant_coeffs(n, n, n, 1.0, 1.0)
    betas = [bi, bj, bk]
    fshp = [1, 1, 1]
    fshp[2 - axis] = n + 1
    betas[axis] = np.broadcast_to((1 + f).reshape(fshp), betas[axis].shape).copy()
    P = oracle.Problem(oracle.Grid(n, n, n, h), 0.0, 1.0, al, *betas)
    Au = P.apply_op(u)
    expect = np.broadcast_to((-(2 + 4 * c)).reshape(shp), (n, n, n))
    sl = (slice(1, -1),) * 3        # cells with no ghost neighbour in any axis
    assert np.abs(Au[sl] - expect[sl]).max() < 1e-9


def test_op_equals_textbook_kronecker_sum(oracle):
    """a=0, beta=1: the cell-centred Dirichlet Laplacian is the Kronecker sum
    of the 1-D matrix tridiag(-1,2,-1)/h^2 with end diagonals 3/h^2."""
    nx, ny, nz, h = 4, 3, 5, 0.25
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 0.0, 1.0, *I.constant_coeffs(nx, ny, nz))
    A = dense_op(P, (nz, ny, nx))

    def T(n):
        t = (2 * np.eye(n) - np.eye(n, k=1) - np.eye(n, k=-1))
        t[0, 0] = t[-1, -1] = 3
        return t / h**2

    K = (np.kron(np.eye(nz), np.kron(np.eye(ny), T(nx)))
         + np.kron(np.eye(nz), np.kron(T(ny), np.eye(nx)))
         + np.kron(T(nz), np.kron(np.eye(ny), np.eye(nx))))
    assert np.abs(A - K).max() < 1e-12 * np.abs(K).max()


def test_op_symmetric_spd_and_dinv_is_inverse_diagonal(oracle):
    """Random alpha, beta in [1,2): the dense operator is symmetric positive
    definite (so GSRB converges, the bottom solve is Cholesky) and
    Dinv = 1/diag(A) with the BC folded (A4)."""
    n, h = 4, 0.25
    coeffs = I.random_coeffs(n, n, n, seed=11)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.3, 0.7, *coeffs)
    A = dense_op(P, (n, n, n))
    assert np.abs(A - A.T).max() < 1e-12 * np.abs(A).max()
    assert np.linalg.eigvalsh(A).min() > 0
    assert np.allclose(1.0 / np.diag(A), P.dinv().ravel(), rtol=1e-14, atol=0)


# ----------------------------------------------------------------- A5 (GSRB)
def colours(shape):
    nz, ny, nx = shape
    k, j, i = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    return ((i + j + k) % 2).ravel()


@pytest.mark.parametrize("n", [4, 6, 8])
def test_gsrb_equals_dense_red_black_gauss_seidel(oracle, n):
    """Brute force: one red sweep then one black sweep equals block
    Gauss-Seidel in red-black order, x_R = D_R^-1 (f_R - A_RB x_B), then
    x_B = D_B^-1 (f_B - A_BR x_R); the red-red block is exactly diagonal
    (Fig 3a)."""
    h = 1.0 / n
    shape = (n, n, n)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *I.random_coeffs(n, n, n, seed=5))
    A = dense_op(P, shape)
    col = colours(shape)
    R, B = col == 0, col == 1
    offRR = A[np.ix_(R, R)] - np.diag(np.diag(A[np.ix_(R, R)]))
    assert np.abs(offRR).max() == 0
    x0 = I.random_field(shape, 0)
    f = I.random_field(shape, 1)
    x = x0.ravel().copy()
    fr = f.ravel()
    x[R] = (fr[R] - A[np.ix_(R, B)] @ x[B]) / np.diag(A)[R]
    x_red = x.copy()
    x[B] = (fr[B] - A[np.ix_(B, R)] @ x[R]) / np.diag(A)[B]
    got_red = P.gsrb_sweep(x0, f, 0)
    got = P.gsrb_sweep(got_red, f, 1)
    assert np.abs(got_red.ravel() - x_red).max() < 1e-12 * np.abs(x_red).max()
    assert np.abs(got.ravel() - x).max() < 1e-12 * np.abs(x).max()
    assert np.allclose(P.smooth(x0, f, 1), got, rtol=0, atol=0)


def test_gsrb_energy_strictly_decreases(oracle):
    """Gauss-Seidel on an SPD system: J(x) = x'Ax/2 - f'x decreases strictly
    with every colour sweep."""
    n, h = 6, 1.0 / 6
    shape = (n, n, n)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *I.hpgmg_coeffs(n, n, n))
    A = dense_op(P, shape)
    x = I.random_field(shape, 0)
    f = I.random_field(shape, 1)
    J = lambda v: 0.5 * v.ravel() @ A @ v.ravel() - f.ravel() @ v.ravel()
    prev = J(x)
    for s in range(8):
        x = P.gsrb_sweep(x, f, s % 2)
        cur = J(x)
        assert cur < prev
        prev = cur


def test_gsrb_fixed_point_is_solution(oracle):
    """The exact discrete solution is a fixed point of the smoother."""
    n, h = 8, 1.0 / 8
    shape = (n, n, n)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *I.random_coeffs(n, n, n, 2))
    A = dense_op(P, shape)
    f = I.random_field(shape, 4)
    xs = np.linalg.solve(A, f.ravel()).reshape(shape)
    assert np.abs(P.smooth(xs, f, 2) - xs).max() < 1e-10 * np.abs(xs).max()


# ----------------------------------------------------------- A7/A8 transfer
def test_restrict_interp_invariants(oracle):
    nc = (3, 4, 2)  # coarse (nz, ny, nx)
    c = I.random_field(nc, 9)
    fine0 = np.zeros((6, 8, 4))
    p0 = oracle.interpolate(fine0, c, 0.0, "p0")
    assert np.abs(oracle.restrict_cell(p0) - c).max() <= 4e-16 * np.abs(c).max()  # R P0 = I
    f = I.random_field((6, 8, 4), 10)
    assert abs(oracle.restrict_cell(f).sum() - f.sum() / 8) < 1e-13   # mass
    const = np.full(nc, 3.5)
    assert np.all(oracle.interpolate(fine0, const, 0.0, "p0") == 3.5)
    # prescale: fine <- s*fine + P(c)
    g = oracle.interpolate(f, c, 0.5, "p0")
    assert np.allclose(g, 0.5 * f + p0, rtol=0, atol=1e-15)


def test_pl_exact_on_linear_fields(oracle):
    """Trilinear interpolation reproduces a linear field at the fine cell
    centres wherever no ghost value is involved (interior fine cells)."""
    ncx, ncy, ncz = 6, 5, 4
    hc = 1.0
    X = lambda n, hh: (np.arange(n) + 0.5) * hh
    lin = lambda x, y, z: 0.3 + 1.7 * x - 0.9 * y + 0.4 * z
    c = lin(X(ncx, hc)[None, None, :], X(ncy, hc)[None, :, None], X(ncz, hc)[:, None, None])
    c = np.broadcast_to(c, (ncz, ncy, ncx)).copy()
    fine = np.zeros((2 * ncz, 2 * ncy, 2 * ncx))
    got = oracle.interpolate(fine, c, 0.0, "pl")
    hf = hc / 2
    exp = lin(X(2 * ncx, hf)[None, None, :], X(2 * ncy, hf)[None, :, None], X(2 * ncz, hf)[:, None, None])
    exp = np.broadcast_to(exp, fine.shape)
    sl = (slice(1, -1), slice(1, -1), slice(1, -1))
    assert np.abs(got[sl] - exp[sl]).max() < 1e-12


def test_pl_boundary_sine_consistency(oracle):
    """PL of a smooth field vanishing on the boundary converges at O(h^2)
    including boundary cells (ghosts from A2 = linear extrapolation to 0)."""
    errs = []
    for nc in (8, 16, 32):
        c = sine_mode(nc, nc, nc, 1.0 / nc, (1, 1, 1))
        f = oracle.interpolate(np.zeros((2 * nc,) * 3), c, 0.0, "pl")
        e = sine_mode(2 * nc, 2 * nc, 2 * nc, 0.5 / nc, (1, 1, 1))
        errs.append(np.abs(f - e).max())
    r1, r2 = errs[0] / errs[1], errs[1] / errs[2]
    assert 3.5 < r1 < 4.5 and 3.5 < r2 < 4.5


@pytest.mark.parametrize("kind", ["beta_i", "beta_j", "beta_k"])
def test_face_restriction_linear(oracle, kind):
    """Face average of a field linear in the face's tangential coordinates
    equals its value at the coarse face centre (coarse face = union of the 4
    fine faces it covers)."""
    nz, ny, nx, h = 4, 6, 8, 1.0
    d = {"beta_i": 0, "beta_j": 1, "beta_k": 2}[kind]
    n = [nx, ny, nz]

    def coords(nn, hh, face):
        return (np.arange(nn + 1) * hh) if face else (np.arange(nn) + 0.5) * hh

    lin = lambda x, y, z: 2.0 + 0.5 * x + 0.25 * y - 0.125 * z
    fx, fy, fz = (coords(n[a], h, a == d) for a in range(3))
    fine = lin(fx[None, None, :], fy[None, :, None], fz[:, None, None])
    cx, cy, cz = (coords(n[a] // 2, 2 * h, a == d) for a in range(3))
    exp = lin(cx[None, None, :], cy[None, :, None], cz[:, None, None])
    got = oracle.restrict_face(np.ascontiguousarray(fine), kind)
    assert got.shape == exp.shape
    assert np.abs(got - exp).max() < 1e-13


# ----------------------------------------------------------- bottom, norms
def test_bottom_solve_exact(oracle):
    nx, ny, nz, h = 2, 2, 4, 0.5
    P = oracle.Problem(oracle.Grid(nx, ny, nz, h), 1.0, 1.0, *I.random_coeffs(nx, ny, nz, 3))
    A = dense_op(P, (nz, ny, nx))
    f = I.random_field((nz, ny, nx), 8)
    x = P.bottom_solve(f)
    assert np.abs(x.ravel() - np.linalg.solve(A, f.ravel())).max() < 1e-12 * np.abs(x).max()


def test_norms(oracle):
    x = I.random_field((3, 5, 7), 2)
    assert oracle.norm(x, "max") == np.abs(x).max()
    assert abs(oracle.norm(x, "l2") - np.linalg.norm(x.ravel())) < 1e-13


# ----------------------------------------------------------------- A9 (MG)
def _mg(oracle, n, cc=False, a=1.0, b=1.0):
    h = 1.0 / n
    coeffs = I.constant_coeffs(n, n, n) if cc else I.hpgmg_coeffs(n, n, n)
    return oracle.MG(n, n, n, h, a, b, *coeffs)


@pytest.mark.parametrize("n,cycles", [(16, 9), (32, 11)])
def test_vcycle_cycles_to_1e10(oracle, n, cycles):
    """V-cycle (2+2 RB pairs, P0, exact 2^3 bottom) on the
    manufactured HPGMG-shaped problem reaches ||r||inf/||f||inf < 1e-10 in
    the cycle count fixed by the convergence factor (9, 11)."""
    mg = _mg(oracle, n)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    u, hist = mg.solve(f)
    assert len(hist) == cycles and hist[-1] < 1e-10
    # monotone residual decrease, factor <= 0.25 after the first cycle
    rho = [hist[i + 1] / hist[i] for i in range(len(hist) - 1)]
    assert max(rho[1:]) <= 0.25


@pytest.mark.parametrize("n", [16, 32])
def test_vcycle_convergence_factor_random_rhs(oracle, n):
    mg = _mg(oracle, n, cc=True, a=0.0)
    f = I.random_field((n, n, n), 1)
    u = np.zeros_like(f)
    r0 = mg.relres(u, f)
    rhos = []
    for _ in range(6):
        u = mg.vcycle(u, f)
        r1 = mg.relres(u, f)
        rhos.append(r1 / r0)
        r0 = r1
    assert max(rhos[2:]) <= 0.25


def test_discretisation_error_second_order(oracle):
    """||u_h - u||inf against the manufactured solution falls ~4x per
    refinement (second-order FV, HPGMG 2nd order)."""
    errs = []
    for n in (16, 32, 64):
        mg = _mg(oracle, n)
        ue, f = I.manufactured(n, n, n, 1.0, 1.0)
        u, hist = mg.solve(f)
        errs.append(np.abs(u - ue).max())
    assert 3.4 < errs[0] / errs[1] < 4.4 and 3.6 < errs[1] / errs[2] < 4.4
    assert abs(errs[0] - 7.37e-6) < 0.05e-6        # SURVEY 8c verified value


def test_solve_closed_form_discrete_solution(oracle):
    """CC Helmholtz with f = (a + b*lambda_m) * sine mode has the sine mode as
    its exact discrete solution; the solver must reproduce it."""
    n, a, b = 16, 1.0, 1.0
    h = 1.0 / n
    m = (1, 2, 1)
    s = sine_mode(n, n, n, h, m)
    lam = 4 / h**2 * sum(np.sin(np.pi * mm * h / 2) ** 2 for mm in m)
    mg = oracle.MG(n, n, n, h, a, b, *I.constant_coeffs(n, n, n))
    u, hist = mg.solve((a + b * lam) * s)
    assert np.abs(u - s).max() < 1e-9


def test_fcycle_sanity(oracle):
    n = 32
    mg = _mg(oracle, n)
    ue, f = I.manufactured(n, n, n, 1.0, 1.0)
    u = mg.fcycle(f)
    r = mg.relres(u, f)
    assert 1e-3 < r < 5e-2                          # ~1.2e-2
    # F-cycle already reaches discretisation-error accuracy
    assert np.abs(u - ue).max() < 3 * 2.0e-6
    u2, hist = mg.solve(f, fcycle=True)
    assert hist[-1] < 1e-10 and len(hist) <= 11


def test_nonsquare_hierarchy(oracle):
    """C5 shapes (z twice as long): hierarchy coarsens to 2x2x4 and the
    solve converges at the same rate."""
    nx, ny, nz = 16, 16, 32
    h = I.level_h(nx, ny, nz)
    mg = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *I.hpgmg_coeffs(nx, ny, nz, h))
    assert mg.level_dims(mg.levels - 1) == (2, 2, 4)
    ue, f = I.manufactured(nx, ny, nz, 1.0, 1.0, h)
    u, hist = mg.solve(f)
    assert hist[-1] < 1e-10 and len(hist) <= 12


def test_paper_constants_fixture():
    """tests/golden/paper_constants.json holds the numbers the paper prints
     that the measurement code uses."""
    with open(os.path.join(GOLDEN, "paper_constants.json")) as fh:
        g = json.load(fh)
    assert g["compulsory_bytes_per_stencil"]["vc_gsrb"] == 64
    assert g["compulsory_bytes_per_stencil"]["cc_7pt"] == 24
    assert g["compulsory_bytes_per_stencil"]["cc_jacobi"] == 40
    # 64 B = x read + x write + rhs, alpha, beta_i, beta_j, beta_k, lambda (8 B each)
    assert 8 * (2 + 6) == g["compulsory_bytes_per_stencil"]["vc_gsrb"]
    assert g["hpgmg_run"]["smooths_pre_post_sweeps"] == 4


def test_point_evaluations_match_whole_grid(oracle):
    """The sampled (one cell at a time) oracle evaluations used at full size
    equal the whole-grid oracle sweeps they restate."""
    nx, ny, nz = 8, 6, 10
    P = oracle.Problem(oracle.Grid(nx, ny, nz, 0.1), 1.0, 1.0, *I.random_coeffs(nx, ny, nz, 4))
    x = I.random_field((nz, ny, nx), 0)
    f = I.random_field((nz, ny, nx), 1)
    rng = np.random.default_rng(3)
    pts = (rng.integers(0, nx, 40), rng.integers(0, ny, 40), rng.integers(0, nz, 40))
    pts = (np.r_[pts[0], 0, nx - 1, 0], np.r_[pts[1], 0, ny - 1, ny - 1], np.r_[pts[2], 0, nz - 1, 1])
    r = P.residual(x, f)
    assert np.array_equal(P.residual_points(x, f, pts), r[pts[2], pts[1], pts[0]])
    s = P.smooth(x, f, 1)
    assert np.array_equal(P.gsrb_pair_points(x, f, pts), s[pts[2], pts[1], pts[0]])


# ------------------------------------------------------- NEXT-2 (Fig 7 operators)
def _kron_laplacian(nx, ny, nz, h):
    def T(n):
        t = (2 * np.eye(n) - np.eye(n, k=1) - np.eye(n, k=-1))
        t[0, 0] = t[-1, -1] = 3
        return t / h**2
    return (np.kron(np.eye(nz), np.kron(np.eye(ny), T(nx)))
            + np.kron(np.eye(nz), np.kron(T(ny), np.eye(nx)))
            + np.kron(T(nz), np.kron(np.eye(ny), np.eye(nx))))


def test_cc_laplacian_is_textbook_matrix(oracle):
    """The CC 7-point Laplacian with the Dirichlet fold is the Kronecker sum of
    tridiag(-1,2,-1)/h^2 with end diagonals 3/h^2."""
    nz, ny, nx, h = 5, 3, 4, 0.25
    K = _kron_laplacian(nx, ny, nz, h)
    x = I.random_field((nz, ny, nx), 4)
    got = oracle.laplacian_cc(x, h)
    assert np.abs(got.ravel() - K @ x.ravel()).max() < 1e-12 * np.abs(K @ x.ravel()).max()


def test_cc_jacobi_brute_force(oracle):
    """x + (2/3) D^-1 (f - L x) with dense L and D = diag(L) (reading R-11)."""
    nz, ny, nx, h = 4, 5, 6, 0.2
    K = _kron_laplacian(nx, ny, nz, h)
    x, f = I.random_field((nz, ny, nx), 0), I.random_field((nz, ny, nx), 1)
    exp = x.ravel() + (2.0 / 3.0) * (f.ravel() - K @ x.ravel()) / np.diag(K)
    got = oracle.jacobi_cc(x, f, h)
    assert np.abs(got.ravel() - exp).max() < 1e-12 * np.abs(exp).max()
    # the damped Jacobi iteration converges (spectral radius < 1 for SPD L, omega 2/3)
    Jm = np.eye(K.shape[0]) - (2.0 / 3.0) * K / np.diag(K)[:, None]
    assert np.abs(np.linalg.eigvals(Jm)).max() < 1.0


# ------------------------------------------------------- NEXT-3 (Chebyshev smoother)
def test_chebyshev_is_scaled_chebyshev_polynomial(oracle):
    """After m steps the error is P_m(D^-1 A) e_0 with
    P_m(l) = T_m((theta - l)/delta) / T_m(theta/delta) (Saad Alg. 12.1): checked
    through the eigen-decomposition of the dense D^-1 A."""
    n, h = 4, 0.25
    shape = (n, n, n)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *I.random_coeffs(n, n, n, 3))
    A = dense_op(P, shape)
    D = np.diag(A)
    M = A / D[:, None]                       # D^-1 A, similar to the SPD D^-1/2 A D^-1/2
    lam, V = np.linalg.eig(M)
    lam, V = lam.real, V.real
    hi, lo = 1.1 * lam.max(), 0.1 * lam.max()
    theta, delta = (hi + lo) / 2, (hi - lo) / 2
    f = I.random_field(shape, 1)
    xs = np.linalg.solve(A, f.ravel())
    x0 = I.random_field(shape, 0)
    for m in (1, 2, 4):
        Tm = np.polynomial.chebyshev.Chebyshev.basis(m)
        pm = Tm((theta - lam) / delta) / Tm(theta / delta)
        e0 = np.linalg.solve(V, x0.ravel() - xs)
        exp = xs + V @ (pm * e0)
        got = P.chebyshev(x0, f, m, lo, hi)
        assert np.abs(got.ravel() - exp).max() < 1e-10 * np.abs(exp).max()


def test_chebyshev_smooths_and_lambda_max(oracle):
    n, h = 8, 1.0 / 8
    shape = (n, n, n)
    P = oracle.Problem(oracle.Grid(n, n, n, h), 1.0, 1.0, *I.hpgmg_coeffs(n, n, n))
    A = dense_op(P, shape)
    lam_true = np.abs(np.linalg.eigvals(A / np.diag(A)[:, None])).max()
    lam10 = P.lambda_max(I.random_field(shape, 5), 10)
    lam = P.lambda_max(I.random_field(shape, 5), 200)
    assert abs(lam / lam_true - 1) < 5e-3 and abs(lam / lam_true - 1) < abs(lam10 / lam_true - 1)
    # the high-frequency end of the spectrum is damped by at least 1/T_m(sigma)
    f = np.zeros(shape)
    x = I.random_field(shape, 6)
    lo, hi = 0.1 * 1.1 * lam, 1.1 * lam
    y = P.chebyshev(x, f, 4, lo, hi)
    J = lambda v: v.ravel() @ A @ v.ravel()
    assert J(y) < J(x)


def test_chebyshev_vcycle_converges(oracle):
    """V-cycles with Chebyshev smoothing (4 steps pre/post, interval from the
    power-iteration lambda_max) converge with rho <= 0.25 (reading R-16)."""
    n = 16
    mg = _mg(oracle, n)
    mg.set_chebyshev(2)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    u, hist = mg.solve(f)
    assert hist[-1] < 1e-10 and len(hist) <= 12
    rho = [hist[i + 1] / hist[i] for i in range(1, len(hist) - 1)]
    assert max(rho) <= 0.25
