"""ctypes wrapper around oracle/liboracle.so -- the CPU ORACLE.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  It shares no
code with the CUDA path (paper_conf_ipps_zhangdmwbf17_b200/); the only common
dependency is the seeded input generator module, which holds no arithmetic of
the method.

Arrays cross this wrapper as interior-only numpy float64 arrays
(cell (nz,ny,nx); beta_i (nz,ny,nx+1); beta_j (nz,ny+1,nx); beta_k (nz+1,ny,nx))
and are padded here to the oracle's one-ghost layout (layout only, no math).
Every numerical step is in oracle.c, which cites the paper passage it follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")
GCC_FLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c99"]
# The pins and every parity test use the single-thread build.  The -fopenmp
# build (same source: the plane loops' "omp parallel for" pragmas become live)
# is only for timing the oracle on all host cores (bench.py's cpu_baseline and
# --impl reference legs); select it with use_openmp() before the first call.
_use_omp = False


def use_openmp(on=True):
    global _use_omp
    if _lib is not None and on != _use_omp:
        raise RuntimeError("oracle library already loaded with the other build")
    _use_omp = on


def build(force=False, omp=None):
    """Compile liboracle.so (and liboracle_omp.so) with gcc (plain C, no contraction)."""
    omp = _use_omp if omp is None else omp
    out = _LIB_OMP if omp else _LIB
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(_SRC):
        tmp = out + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *GCC_FLAGS, *(["-fopenmp"] if omp else []), "-o", tmp, _SRC,
                               "-lm"])
        os.replace(tmp, out)
    return out


_lib = None
_P = C.POINTER(C.c_double)
_IP = C.POINTER(C.c_int)


class _Grid(C.Structure):
    _fields_ = [("nx", C.c_int), ("ny", C.c_int), ("nz", C.c_int), ("h", C.c_double)]


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        G = C.POINTER(_Grid)
        d = C.c_double
        sig = {
            "or_set_threads": (C.c_int, [C.c_int]),
            "or_apply_bc": (None, [G, _P]),
            "or_apply_op": (None, [G, d, d, _P, _P, _P, _P, _P, _P]),
            "or_residual": (None, [G, d, d, _P, _P, _P, _P, _P, _P, _P]),
            "or_dinv": (None, [G, d, d, _P, _P, _P, _P, _P]),
            "or_gsrb_sweep": (None, [G, d, d, _P, _P, _P, _P, _P, _P, _P, C.c_int]),
            "or_smooth": (None, [G, d, d, _P, _P, _P, _P, _P, _P, _P, C.c_int]),
            "or_restrict_cell": (None, [G, _P, G, _P]),
            "or_restrict_face": (None, [G, _P, G, _P, C.c_int]),
            "or_interp_p0": (None, [G, _P, d, G, _P]),
            "or_interp_pl": (None, [G, _P, d, G, _P]),
            "or_norm_max": (d, [G, _P]),
            "or_norm_l2": (d, [G, _P]),
            "or_bottom_solve": (C.c_int, [G, d, d, _P, _P, _P, _P, _P, _P]),
            "or_mg_create": (C.c_void_p, [C.c_int, C.c_int, C.c_int, d, d, d, _P, _P, _P, _P,
                                          C.c_int, C.c_int]),
            "or_mg_free": (None, [C.c_void_p]),
            "or_mg_levels": (C.c_int, [C.c_void_p]),
            "or_mg_level_dims": (None, [C.c_void_p, C.c_int, C.POINTER(C.c_int)]),
            "or_mg_vcycle": (C.c_int, [C.c_void_p, _P, _P]),
            "or_mg_set_chebyshev": (None, [C.c_void_p, C.c_int]),
            "or_mg_fcycle": (C.c_int, [C.c_void_p, _P, _P]),
            "or_mg_relres": (d, [C.c_void_p, _P, _P]),
            "or_mg_solve": (C.c_int, [C.c_void_p, _P, _P, C.c_int, d, C.c_int, _P]),
            "or_laplacian_cc": (None, [G, _P, _P]),
            "or_jacobi_cc": (None, [G, d, _P, _P, _P]),
            "or_chebyshev": (None, [G, d, d, _P, _P, _P, _P, _P, _P, _P, C.c_int, d, d, _P, _P]),
            "or_lambda_max": (d, [G, d, d, _P, _P, _P, _P, _P, _P, _P, C.c_int]),
            "or_residual_points": (None, [G, d, d, _P, _P, _P, _P, _P, _P, C.c_int, _IP, _IP, _IP,
                                          _P]),
            "or_gsrb_pair_points": (None, [G, d, d, _P, _P, _P, _P, _P, _P, _P, C.c_int, _IP, _IP,
                                           _IP, _P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


# ------------------------------------------------------------------ layout
def pad(arr, kind="cell"):
    """Interior (face) array -> oracle padded layout (nz+2, ny+2, nx+2)."""
    a = np.asarray(arr, dtype=np.float64)
    if kind == "cell":
        nz, ny, nx = a.shape
    elif kind == "beta_i":
        nz, ny, nx = a.shape[0], a.shape[1], a.shape[2] - 1
    elif kind == "beta_j":
        nz, ny, nx = a.shape[0], a.shape[1] - 1, a.shape[2]
    elif kind == "beta_k":
        nz, ny, nx = a.shape[0] - 1, a.shape[1], a.shape[2]
    else:
        raise ValueError(kind)
    out = np.zeros((nz + 2, ny + 2, nx + 2))
    out[1:1 + a.shape[0], 1:1 + a.shape[1], 1:1 + a.shape[2]] = a
    return out


def interior(p):
    return np.ascontiguousarray(p[1:-1, 1:-1, 1:-1])


def _iptr(a):
    assert a.dtype == np.int32 and a.flags.c_contiguous
    return a.ctypes.data_as(_IP)


def _ptr(a):
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(_P)


class Grid:
    def __init__(self, nx, ny, nz, h):
        self.nx, self.ny, self.nz, self.h = nx, ny, nz, float(h)
        self._g = _Grid(nx, ny, nz, float(h))

    @property
    def ref(self):
        return C.byref(self._g)

    def coarse(self):
        return Grid(self.nx // 2, self.ny // 2, self.nz // 2, 2 * self.h)


class Problem:
    """Operator data (a, b, alpha, beta_i/j/k) on one grid, oracle layout."""

    def __init__(self, grid, a, b, alpha, bi, bj, bk):
        self.g, self.a, self.b = grid, float(a), float(b)
        self.alpha, self.bi = pad(alpha), pad(bi, "beta_i")
        self.bj, self.bk = pad(bj, "beta_j"), pad(bk, "beta_k")

    def _c(self):
        return (self.g.ref, self.a, self.b, _ptr(self.alpha), _ptr(self.bi), _ptr(self.bj),
                _ptr(self.bk))

    def dinv(self):
        d = np.zeros_like(self.alpha)
        lib().or_dinv(*self._c(), _ptr(d))
        return interior(d)

    def apply_op(self, x):
        xp, out = pad(x), np.zeros_like(self.alpha)
        lib().or_apply_op(*self._c(), _ptr(xp), _ptr(out))
        return interior(out)

    def residual(self, x, rhs):
        xp, rp, out = pad(x), pad(rhs), np.zeros_like(self.alpha)
        lib().or_residual(*self._c(), _ptr(xp), _ptr(rp), _ptr(out))
        return interior(out)

    def gsrb_sweep(self, x, rhs, colour, dinv=None):
        dinv = self.dinv() if dinv is None else dinv
        xp, rp, dp = pad(x), pad(rhs), pad(dinv)
        lib().or_gsrb_sweep(*self._c(), _ptr(dp), _ptr(xp), _ptr(rp), int(colour))
        return interior(xp)

    def smooth(self, x, rhs, rb_pairs, dinv=None):
        dinv = self.dinv() if dinv is None else dinv
        xp, rp, dp = pad(x), pad(rhs), pad(dinv)
        lib().or_smooth(*self._c(), _ptr(dp), _ptr(xp), _ptr(rp), int(rb_pairs))
        return interior(xp)

    def residual_points(self, x, rhs, pts):
        """rhs - A x at the cells pts = (i, j, k) index arrays (sampled parity)."""
        ii, jj, kk = (np.ascontiguousarray(p, dtype=np.int32) for p in pts)
        xp, rp, out = pad(x), pad(rhs), np.zeros(len(ii))
        lib().or_residual_points(*self._c(), _ptr(xp), _ptr(rp), len(ii), _iptr(ii), _iptr(jj),
                                 _iptr(kk), _ptr(out))
        return out

    def gsrb_pair_points(self, x, rhs, pts, dinv=None):
        """Values at pts after one RB pair from x, evaluated cell by cell."""
        dinv = self.dinv() if dinv is None else dinv
        ii, jj, kk = (np.ascontiguousarray(p, dtype=np.int32) for p in pts)
        xp, rp, dp, out = pad(x), pad(rhs), pad(dinv), np.zeros(len(ii))
        lib().or_gsrb_pair_points(*self._c(), _ptr(dp), _ptr(xp), _ptr(rp), len(ii), _iptr(ii),
                                  _iptr(jj), _iptr(kk), _ptr(out))
        return out

    def chebyshev(self, x, rhs, degree, lo, hi, dinv=None):
        """NEXT-3: degree Chebyshev steps for D^-1 A eigenvalues in [lo, hi]."""
        dinv = self.dinv() if dinv is None else dinv
        xp, rp, dp = pad(x), pad(rhs), pad(dinv)
        w1, w2 = np.zeros_like(xp), np.zeros_like(xp)
        lib().or_chebyshev(*self._c(), _ptr(dp), _ptr(xp), _ptr(rp), int(degree), float(lo),
                           float(hi), _ptr(w1), _ptr(w2))
        return interior(xp)

    def lambda_max(self, v0, iters, dinv=None):
        dinv = self.dinv() if dinv is None else dinv
        vp, dp, w = pad(v0), pad(dinv), np.zeros_like(self.alpha)
        return lib().or_lambda_max(*self._c(), _ptr(dp), _ptr(vp), _ptr(w), int(iters))

    def bottom_solve(self, rhs):
        xp, rp = np.zeros_like(self.alpha), pad(rhs)
        rc = lib().or_bottom_solve(*self._c(), _ptr(xp), _ptr(rp))
        if rc != 0:
            raise RuntimeError("oracle bottom solve: matrix not SPD")
        return interior(xp)


def apply_bc(grid, x_padded):
    """Fill the ghost zone of a padded array in place (A2)."""
    lib().or_apply_bc(grid.ref, _ptr(x_padded))
    return x_padded


def restrict_cell(fine):
    nz, ny, nx = fine.shape
    gf, gc = Grid(nx, ny, nz, 1.0), Grid(nx // 2, ny // 2, nz // 2, 2.0)
    fp, cp = pad(fine), np.zeros((nz // 2 + 2, ny // 2 + 2, nx // 2 + 2))
    lib().or_restrict_cell(gc.ref, _ptr(cp), gf.ref, _ptr(fp))
    return interior(cp)


def restrict_face(fine, kind):
    """kind in beta_i/beta_j/beta_k; returns the coarse face array."""
    d = {"beta_i": 0, "beta_j": 1, "beta_k": 2}[kind]
    s = list(fine.shape)
    s[2 - d] -= 1
    nz, ny, nx = s
    gf, gc = Grid(nx, ny, nz, 1.0), Grid(nx // 2, ny // 2, nz // 2, 2.0)
    fp, cp = pad(fine, kind), np.zeros((nz // 2 + 2, ny // 2 + 2, nx // 2 + 2))
    lib().or_restrict_face(gc.ref, _ptr(cp), gf.ref, _ptr(fp), d)
    cs = [nz // 2, ny // 2, nx // 2]
    cs[2 - d] += 1
    return np.ascontiguousarray(cp[1:1 + cs[0], 1:1 + cs[1], 1:1 + cs[2]])


def interpolate(fine, coarse, prescale, kind="p0"):
    nz, ny, nx = fine.shape
    gf, gc = Grid(nx, ny, nz, 1.0), Grid(nx // 2, ny // 2, nz // 2, 2.0)
    fp, cp = pad(fine), pad(coarse)
    fn = lib().or_interp_p0 if kind == "p0" else lib().or_interp_pl
    fn(gf.ref, _ptr(fp), float(prescale), gc.ref, _ptr(cp))
    return interior(fp)


def laplacian_cc(x, h):
    """NEXT-2: constant-coefficient 7-point Laplacian (Fig 7)."""
    nz, ny, nx = x.shape
    g = Grid(nx, ny, nz, h)
    xp, out = pad(x), np.zeros((nz + 2, ny + 2, nx + 2))
    lib().or_laplacian_cc(g.ref, _ptr(xp), _ptr(out))
    return interior(out)


def jacobi_cc(x, f, h, omega=2.0 / 3.0):
    """NEXT-2: weighted Jacobi x + omega D^-1 (f - L x) (R-11)."""
    nz, ny, nx = x.shape
    g = Grid(nx, ny, nz, h)
    xp, fp, out = pad(x), pad(f), np.zeros((nz + 2, ny + 2, nx + 2))
    lib().or_jacobi_cc(g.ref, float(omega), _ptr(xp), _ptr(fp), _ptr(out))
    return interior(out)


def norm(x, kind="max"):
    nz, ny, nx = x.shape
    g = Grid(nx, ny, nz, 1.0)
    fn = lib().or_norm_max if kind == "max" else lib().or_norm_l2
    return fn(g.ref, _ptr(pad(x)))


class MG:
    """Oracle multigrid hierarchy (A9).  pre/post = RB pairs per smooth."""

    def __init__(self, nx, ny, nz, h, a, b, alpha, bi, bj, bk, pre=2, post=2):
        self.shape = (nz, ny, nx)
        self._keep = [pad(alpha), pad(bi, "beta_i"), pad(bj, "beta_j"), pad(bk, "beta_k")]
        self.h = lib().or_mg_create(nx, ny, nz, float(h), float(a), float(b),
                                    *[_ptr(x) for x in self._keep], pre, post)

    def __del__(self):
        if getattr(self, "h", None):
            lib().or_mg_free(self.h)
            self.h = None

    def set_chebyshev(self, steps_per_pair=2):
        """NEXT-3: Chebyshev smoothing in every V-cycle (reading R-16)."""
        lib().or_mg_set_chebyshev(self.h, int(steps_per_pair))

    @property
    def levels(self):
        return lib().or_mg_levels(self.h)

    def level_dims(self, l):
        d = (C.c_int * 3)()
        lib().or_mg_level_dims(self.h, l, d)
        return tuple(d)

    def vcycle(self, u, f):
        up, fp = pad(u), pad(f)
        lib().or_mg_vcycle(self.h, _ptr(up), _ptr(fp))
        return interior(up)

    def fcycle(self, f):
        up, fp = np.zeros((self.shape[0] + 2, self.shape[1] + 2, self.shape[2] + 2)), pad(f)
        lib().or_mg_fcycle(self.h, _ptr(up), _ptr(fp))
        return interior(up)

    def relres(self, u, f):
        return lib().or_mg_relres(self.h, _ptr(pad(u)), _ptr(pad(f)))

    def solve(self, f, fcycle=False, rtol=1e-10, maxc=50, u0=None):
        up = pad(np.zeros(self.shape) if u0 is None else u0)
        fp = pad(f)
        hist = np.zeros(maxc + 1)
        n = lib().or_mg_solve(self.h, _ptr(up), _ptr(fp), int(fcycle), float(rtol), int(maxc),
                              _ptr(hist))
        return interior(up), list(hist[:n])
