"""CPU ORACLE of the generic stencil language, plain numpy.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  It shares no
code with the CUDA path (the product's DSL front end, its lowering, its code
generator and its dependence analysis live in paper_conf_ipps_zhangdmwbf17_b200/
and csrc/stencil.cu); tests describe each stencil to it separately, as plain
data:

    stencil := {"out": mesh, "rects": [(lo, hi, stride), ...], "expr": E}
    E       := ("const", v)
             | ("comp", mesh, [(offset, W), ...], src, mul, div, pre)
             | ("+", E, E) | ("-", E, E) | ("*", E, E) | ("/", E, E) | ("neg", E)
    W       := number | E

It follows the paper's definitions (Table I, Fig 4) in the
readings of DESIGN.md R-17/R-18:

  * meshes are the oracle's padded arrays, shape (nz+2, ny+2, nx+2) indexed
    [Z, Y, X]: stencil coordinates are ghost-inclusive with one ghost layer,
    interior 1..n (Fig 4's domains start at 1);
  * a RectDomain (lo, hi, stride) covers lo, lo+s, ... < hi per axis (x, y, z);
    a negative bound b stands for N + b with N = n + 2;
    stride 0 = the single coordinate lo (Fig 4 l.17); a DomainUnion is the
    union of its rects;
  * a Component (mesh, weights) at point p is sum_o w(o) * mesh[q_o(p)] with
    q_o(p) = floor((mul*p + pre)/div) + o per axis, summed left to right in
    the listed order, w == 1 -> the read itself, w == 0 -> no term; a weight
    that is an expression is evaluated at p (variable coefficients,
    PAPER.md:313-316);
  * a Stencil computes every point of its domain from the values BEFORE it
    (its points are independent), then stores them into `out`; the stencils
    of a group apply in order (Table I: "performed consecutively").
"""
from __future__ import annotations

import numpy as np


def _resolve(rect, shape_zyx):
    """(lo, hi, stride) -> per-axis coordinate arrays (x, y, z)."""
    lo, hi, st = rect
    N = (shape_zyx[2], shape_zyx[1], shape_zyx[0])   # ghost-inclusive sizes x, y, z
    axes = []
    for d in range(3):
        a = lo[d] + N[d] if lo[d] < 0 else lo[d]
        b = hi[d] + N[d] if hi[d] < 0 else hi[d]
        if st[d] == 0:
            axes.append(np.array([a]))
        else:
            axes.append(np.arange(a, b, st[d]))
    return axes


def points(rects, shape_zyx):
    """All (X, Y, Z) points of a DomainUnion as flat int arrays (rect order)."""
    xs, ys, zs = [], [], []
    for r in rects:
        ax, ay, az = _resolve(r, shape_zyx)
        Z, Y, X = np.meshgrid(az, ay, ax, indexing="ij")
        xs.append(X.ravel())
        ys.append(Y.ravel())
        zs.append(Z.ravel())
    return np.concatenate(xs), np.concatenate(ys), np.concatenate(zs)


def _affine(p, mul, div, pre, off):
    return np.floor_divide(mul * p + pre, div) + off


def _read(arr, X, Y, Z):
    nz, ny, nx = arr.shape
    if (X.size and (X.min() < 0 or X.max() >= nx or Y.min() < 0 or Y.max() >= ny
                    or Z.min() < 0 or Z.max() >= nz)):
        raise IndexError("stencil read outside the one-ghost mesh")
    return arr[Z, Y, X]


def evaluate(E, P, meshes, src_meshes):
    """Value of expression E at the points P = (X, Y, Z) (float64 arrays)."""
    X, Y, Z = P
    tag = E[0]
    if tag == "const":
        return np.full(X.shape, float(E[1]))
    if tag == "comp":
        _, mesh, terms, src, mul, div, pre = E
        arr = (src_meshes if src else meshes)[mesh]
        acc = None
        for off, w in terms:
            if not isinstance(w, tuple) and float(w) == 0.0:
                continue
            q = [_affine(c, mul[d], div[d], pre[d], off[d]) for d, c in enumerate((X, Y, Z))]
            r = _read(arr, q[0], q[1], q[2])
            if isinstance(w, tuple):
                t = evaluate(w, P, meshes, src_meshes) * r
            elif float(w) == 1.0:
                t = r
            else:
                t = float(w) * r
            acc = t if acc is None else acc + t
        return np.zeros(X.shape) if acc is None else acc
    if tag == "neg":
        return -evaluate(E[1], P, meshes, src_meshes)
    a = evaluate(E[1], P, meshes, src_meshes)
    b = evaluate(E[2], P, meshes, src_meshes)
    if tag == "+":
        return a + b
    if tag == "-":
        return a - b
    if tag == "*":
        return a * b
    if tag == "/":
        return a / b
    raise ValueError(tag)


def apply_group(group, meshes, src_meshes=None):
    """Apply stencils in order; returns a new dict of meshes (inputs untouched)."""
    cur = {k: np.array(v, dtype=np.float64, copy=True) for k, v in meshes.items()}
    src = cur if src_meshes is None else src_meshes
    for s in group:
        out = cur[s["out"]]
        P = points(s["rects"], out.shape)
        snap = {k: v.copy() for k, v in cur.items()}          # values before the stencil
        vals = evaluate(s["expr"], P, snap, snap if src_meshes is None else src)
        out[P[2], P[1], P[0]] = vals
    return cur
