"""Seeded synthetic input generators shared by the oracle tests, the GPU tests
and bench.py.

This module holds NONE of the method's arithmetic (no operator, smoother,
restriction, interpolation or cycle).  It only produces the problem data the
method is applied to: random fields, HPGMG-shaped coefficient fields and a
manufactured right-hand side.  Recipe:

* random fields:   U[lo, hi) from ``numpy.random.default_rng(seed)``;
* random coefficients: alpha, beta_i, beta_j, beta_k ~ U[1, 2) (catches
  indexing bugs, keeps the operator SPD);
* HPGMG-shaped problem (reading R-1; the paper, shows only
  the 2-D constant-``a``-free form): alpha == 1,
  beta = 5.5 + 4.5*tanh(10*(r - 0.25)) with r the distance of the *face
  centre* from the box centre (Bmin = 1, Bmax = 10), evaluated on the unit
  cube coordinates x^ = x / L per axis;
  manufactured u = X(x^) X(y^) X(z^), X(t) = 2t^6 - 6t^5 + 5t^4 - t^2
  (zero on the boundary), and
  f = a*alpha*u - b*(grad(beta).grad(u) + beta*lap(u)) point-sampled at
  cell centres.

Array conventions (x fastest, C order):
  cell fields  shape (nz, ny, nx)
  beta_i       shape (nz, ny, nx+1)   face i lies between cells i-1 and i
  beta_j       shape (nz, ny+1, nx)
  beta_k       shape (nz+1, ny, nx)
"""
from __future__ import annotations

import numpy as np

FACE_SHAPES = {
    "cell": lambda nx, ny, nz: (nz, ny, nx),
    "beta_i": lambda nx, ny, nz: (nz, ny, nx + 1),
    "beta_j": lambda nx, ny, nz: (nz, ny + 1, nx),
    "beta_k": lambda nx, ny, nz: (nz + 1, ny, nx),
}


def random_field(shape, seed, lo=-1.0, hi=1.0):
    rng = np.random.default_rng(seed)
    return rng.uniform(lo, hi, size=shape)


def random_coeffs(nx, ny, nz, seed=7):
    """alpha, beta_i, beta_j, beta_k ~ U[1,2) with face shapes."""
    rng = np.random.default_rng(seed)
    alpha = rng.uniform(1.0, 2.0, size=(nz, ny, nx))
    bi = rng.uniform(1.0, 2.0, size=(nz, ny, nx + 1))
    bj = rng.uniform(1.0, 2.0, size=(nz, ny + 1, nx))
    bk = rng.uniform(1.0, 2.0, size=(nz + 1, ny, nx))
    return alpha, bi, bj, bk


def constant_coeffs(nx, ny, nz, alpha=1.0, beta=1.0):
    return (np.full((nz, ny, nx), alpha), np.full((nz, ny, nx + 1), beta),
            np.full((nz, ny + 1, nx), beta), np.full((nz + 1, ny, nx), beta))


# ---------------------------------------------------------------- HPGMG shape
BMIN, BMAX, BSHARP, BRAD = 1.0, 10.0, 10.0, 0.25


def _beta(xh, yh, zh):
    r = np.sqrt((xh - 0.5) ** 2 + (yh - 0.5) ** 2 + (zh - 0.5) ** 2)
    return 0.5 * (BMAX + BMIN) + 0.5 * (BMAX - BMIN) * np.tanh(BSHARP * (r - BRAD))


def _dbeta(xh, yh, zh):
    """Gradient of beta w.r.t. the unit-cube coordinates."""
    dx, dy, dz = xh - 0.5, yh - 0.5, zh - 0.5
    r = np.sqrt(dx * dx + dy * dy + dz * dz)
    s = 0.5 * (BMAX - BMIN) * BSHARP / np.cosh(BSHARP * (r - BRAD)) ** 2
    # r = 0 only at the centre cell of an all-odd grid: the gradient's direction
    # is undefined there but bounded, so its limit contribution is 0
    ir = np.divide(1.0, r, out=np.zeros_like(r), where=r > 0)
    return s * dx * ir, s * dy * ir, s * dz * ir


def _X(t):
    return 2 * t**6 - 6 * t**5 + 5 * t**4 - t**2


def _dX(t):
    return 12 * t**5 - 30 * t**4 + 20 * t**3 - 2 * t


def _d2X(t):
    return 60 * t**4 - 120 * t**3 + 60 * t**2 - 2


def level_h(nx, ny, nz):
    """Isotropic spacing h = 1/max(n) (unit cube for cubes)."""
    return 1.0 / max(nx, ny, nz)


def hpgmg_coeffs(nx, ny, nz, h=None):
    """alpha == 1 and tanh beta on face centres (HPGMG-shaped, reading R-1)."""
    h = level_h(nx, ny, nz) if h is None else h
    L = (nx * h, ny * h, nz * h)
    xc = (np.arange(nx) + 0.5) * h / L[0]
    yc = (np.arange(ny) + 0.5) * h / L[1]
    zc = (np.arange(nz) + 0.5) * h / L[2]
    xf = np.arange(nx + 1) * h / L[0]
    yf = np.arange(ny + 1) * h / L[1]
    zf = np.arange(nz + 1) * h / L[2]
    alpha = np.ones((nz, ny, nx))
    bi = _beta(xf[None, None, :], yc[None, :, None], zc[:, None, None])
    bj = _beta(xc[None, None, :], yf[None, :, None], zc[:, None, None])
    bk = _beta(xc[None, None, :], yc[None, :, None], zf[:, None, None])
    return alpha, bi, bj, bk


def manufactured(nx, ny, nz, a, b, h=None):
    """(u_exact, f) at cell centres for the HPGMG-shaped problem."""
    h = level_h(nx, ny, nz) if h is None else h
    L = (nx * h, ny * h, nz * h)
    x = ((np.arange(nx) + 0.5) * h / L[0])[None, None, :]
    y = ((np.arange(ny) + 0.5) * h / L[1])[None, :, None]
    z = ((np.arange(nz) + 0.5) * h / L[2])[:, None, None]
    X, Y, Z = _X(x), _X(y), _X(z)
    u = X * Y * Z
    ux = _dX(x) * Y * Z / L[0]
    uy = X * _dX(y) * Z / L[1]
    uz = X * Y * _dX(z) / L[2]
    lap = (_d2X(x) * Y * Z / L[0] ** 2 + X * _d2X(y) * Z / L[1] ** 2
           + X * Y * _d2X(z) / L[2] ** 2)
    beta = _beta(x, y, z)
    bx, by, bz = _dbeta(x, y, z)
    bx, by, bz = bx / L[0], by / L[1], bz / L[2]
    f = a * 1.0 * u - b * (bx * ux + by * uy + bz * uz + beta * lap)
    return np.ascontiguousarray(np.broadcast_to(u, (nz, ny, nx))), np.ascontiguousarray(
        np.broadcast_to(f, (nz, ny, nx)))


def manufactured_at(nx, ny, nz, h, idx):
    """Exact solution u at the cell-centre sub-grid idx = (i_array, j_array,
    k_array); returns shape (len(k), len(j), len(i))."""
    L = (nx * h, ny * h, nz * h)
    x = ((np.asarray(idx[0]) + 0.5) * h / L[0])[None, None, :]
    y = ((np.asarray(idx[1]) + 0.5) * h / L[1])[None, :, None]
    z = ((np.asarray(idx[2]) + 0.5) * h / L[2])[:, None, None]
    return _X(x) * _X(y) * _X(z)


def split_slabs(arr, kind, parts):
    """Split a global array into z-slabs for `parts` parts (layout only).

    Face arrays along z (beta_k) keep the shared interface face in both
    neighbouring slabs (each slab stores its faces 0..lnz)."""
    if kind == "beta_k":
        nz = arr.shape[0] - 1
        l = nz // parts
        return [np.ascontiguousarray(arr[p * l:(p + 1) * l + 1]) for p in range(parts)]
    nz = arr.shape[0]
    l = nz // parts
    return [np.ascontiguousarray(arr[p * l:(p + 1) * l]) for p in range(parts)]
