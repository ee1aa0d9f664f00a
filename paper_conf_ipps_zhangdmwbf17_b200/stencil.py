"""Snowflake's stencil language (Table I, Fig 4) on the
libsf generic stencil engine (include/sf.h "generic stencils", NEXT-4).

    WeightArray   nested lists, centre element = offset 0
    SparseArray   {offset: weight} (Table I)
    Component     a weight array applied to a mesh; weights may be numbers or
                  expressions over meshes (variable coefficients)
    RectDomain    start, end, stride; negative bounds relative to the grid size
                  (PAPER.md:272-282);  `+` builds a DomainUnion
    Stencil       expression, output mesh (may be an input: in place), domain
    StencilGroup  stencils applied consecutively (Table I)

``compile()`` lowers the expression trees to the engine's DAG (plain data,
include/sf.h ``sf_sx_node``), which renders one CUDA kernel per group and
JIT-compiles it for sm_100a on first use -- the B200 micro-compiler of
PAPER.md:497-522.  The returned callable runs on a ``sf.Level`` (and an
optional source level for restriction / interpolation).

Readings (R-17, R-18):
  * coordinates are (x, y, z), ghost-inclusive with one ghost layer
    (interior 1..n, Dirichlet ghost 0 and n+1), as in Fig 4; a negative
    bound b means N + b with N = n + 2, so ``RectDomain((1,1,1), (-1,-1,-1))``
    is the interior; hi is exclusive; stride 0 makes an axis the single
    coordinate lo (Fig 4 l.17's boundary domain);
  * a WeightArray's outermost list runs along x (Fig 4: ``beta_x`` weights
    vary in the outer index, ``beta_y`` in the inner one);
  * weight expressions are evaluated at the stencil's output point;
  * a Component's value is the left-to-right sum of its terms in weight order,
    a term being ``w * mesh[q]`` (just ``mesh[q]`` for w == 1; w == 0 skipped);
  * cross-level reads: ``Component(mesh, weights, src=1, mul=2)`` reads the
    source level at ``floor((mul*p + pre)/div) + offset`` per axis.
"""
from __future__ import annotations

import numbers

from . import sf

MESHES = dict(sf.FIELD_IDS)


def _mesh_id(m):
    if isinstance(m, str):
        if m not in MESHES:
            raise ValueError(f"unknown mesh {m!r}; one of {sorted(MESHES)}")
        return MESHES[m]
    return int(m)


def _vec3(v, fill):
    if isinstance(v, numbers.Integral):
        return (int(v),) * 3
    v = tuple(int(x) for x in v)
    if not 1 <= len(v) <= 3:
        raise ValueError("1- to 3-component vector expected")
    return v + (fill,) * (3 - len(v))


# ------------------------------------------------------------------ expressions
class Expr:
    def __add__(self, o):
        return BinOp("+", self, as_expr(o))

    def __radd__(self, o):
        return BinOp("+", as_expr(o), self)

    def __sub__(self, o):
        return BinOp("-", self, as_expr(o))

    def __rsub__(self, o):
        return BinOp("-", as_expr(o), self)

    def __mul__(self, o):
        return BinOp("*", self, as_expr(o))

    def __rmul__(self, o):
        return BinOp("*", as_expr(o), self)

    def __truediv__(self, o):
        return BinOp("/", self, as_expr(o))

    def __rtruediv__(self, o):
        return BinOp("/", as_expr(o), self)

    def __neg__(self):
        return Neg(self)


class Const(Expr):
    def __init__(self, value):
        self.value = float(value)


class BinOp(Expr):
    def __init__(self, op, a, b):
        self.op, self.a, self.b = op, a, b


class Neg(Expr):
    def __init__(self, a):
        self.a = a


def as_expr(v):
    if isinstance(v, Expr):
        return v
    if isinstance(v, numbers.Real):
        return Const(v)
    raise TypeError(f"cannot use {type(v).__name__} in a stencil expression")


# ------------------------------------------------------------------ weights
class WeightArray:
    """N-deep nested lists (N = 1..3), odd length per level; element [a][b][c]
    has offset (a - ca, b - cb, c - cc) in (x, y, z)."""

    def __init__(self, nested):
        self.nested = nested

    def items(self):
        out = []

        def walk(node, idx, depth_lens):
            if isinstance(node, (list, tuple)):
                if len(node) % 2 == 0:
                    raise ValueError("weight array levels need odd lengths (a centre element)")
                for i, e in enumerate(node):
                    walk(e, idx + (i - len(node) // 2,), depth_lens)
            else:
                out.append((_vec3(idx, 0), node))
        walk(self.nested, (), None)
        return out


class SparseArray:
    """{offset: weight} with offsets as 1- to 3-tuples (x, y, z); insertion order."""

    def __init__(self, mapping):
        self.mapping = dict(mapping)

    def items(self):
        return [(_vec3(k, 0), w) for k, w in self.mapping.items()]


def _weights(w):
    if isinstance(w, (WeightArray, SparseArray)):
        return w
    if isinstance(w, dict):
        return SparseArray(w)
    if isinstance(w, (list, tuple)):
        return WeightArray(w)
    raise TypeError("weights: WeightArray, SparseArray, nested list or dict")


class Component(Expr):
    """Weights applied to a mesh (Table I).  src = 1 reads the source level;
    mul/div/pre give the affine index map floor((mul*p + pre)/div) + offset."""

    def __init__(self, mesh, weights, src=0, mul=1, div=1, pre=0):
        self.mesh = _mesh_id(mesh)
        self.weights = _weights(weights)
        self.src = int(src)
        self.mul, self.div, self.pre = _vec3(mul, 1), _vec3(div, 1), _vec3(pre, 0)


# ------------------------------------------------------------------ domains
class RectDomain:
    def __init__(self, lo, hi, stride=1):
        self.lo, self.hi, self.stride = _vec3(lo, 0), _vec3(hi, -1), _vec3(stride, 1)
        if min(self.stride) < 0:
            raise ValueError("strides must be >= 0 (0: single coordinate lo)")
        if len(tuple(lo)) != 3 or len(tuple(hi)) != 3:
            raise ValueError("3-D RectDomain bounds expected (x, y, z)")

    @property
    def rects(self):
        return [self]

    def __add__(self, o):
        return DomainUnion(self.rects + o.rects)


RectangularDomain = RectDomain


class DomainUnion:
    def __init__(self, rects):
        self._rects = list(rects)

    @property
    def rects(self):
        return list(self._rects)

    def __add__(self, o):
        return DomainUnion(self._rects + o.rects)


# ------------------------------------------------------------------ lowering
class _Lower:
    def __init__(self):
        self.nodes, self.memo = [], {}

    def add(self, key, node):
        if key in self.memo:
            return self.memo[key]
        self.nodes.append(node)
        self.memo[key] = len(self.nodes) - 1
        return self.memo[key]

    def const(self, v):
        v = float(v)
        return self.add(("c", v.hex()), {"op": sf.SF_SX_CONST, "value": v})

    def read(self, c, off):
        key = ("r", c.mesh, c.src, off, c.mul, c.div, c.pre)
        return self.add(key, {"op": sf.SF_SX_READ, "mesh": c.mesh, "src": c.src, "off": off,
                              "mul": c.mul, "div": c.div, "pre": c.pre})

    def op(self, code, a, b=0):
        return self.add(("o", code, a, b), {"op": code, "a": a, "b": b})

    def expr(self, e):
        if isinstance(e, Const):
            return self.const(e.value)
        if isinstance(e, Component):
            acc = None
            for off, w in e.weights.items():
                if isinstance(w, numbers.Real) and float(w) == 0.0:
                    continue
                r = self.read(e, off)
                if isinstance(w, numbers.Real) and float(w) == 1.0:
                    t = r
                else:
                    t = self.op(sf.SF_SX_MUL, self.expr(as_expr(w)), r)
                acc = t if acc is None else self.op(sf.SF_SX_ADD, acc, t)
            return self.const(0.0) if acc is None else acc
        if isinstance(e, BinOp):
            code = {"+": sf.SF_SX_ADD, "-": sf.SF_SX_SUB, "*": sf.SF_SX_MUL,
                    "/": sf.SF_SX_DIV}[e.op]
            a = self.expr(e.a)
            b = self.expr(e.b)
            return self.op(code, a, b)
        if isinstance(e, Neg):
            return self.op(sf.SF_SX_NEG, self.expr(e.a))
        raise TypeError(f"not a stencil expression: {e!r}")


class Stencil:
    """Stencil(expression, output mesh, domain) (Fig 4 l.13)."""

    def __init__(self, expr, output, domain):
        self.expr = as_expr(expr)
        self.output = _mesh_id(output)
        self.domain = domain

    def lower(self):
        lw = _Lower()
        root = lw.expr(self.expr)
        rects = [(r.lo, r.hi, r.stride) for r in self.domain.rects]
        return lw.nodes, root, self.output, rects

    def compile(self):
        return StencilGroup([self]).compile()


class StencilGroup:
    """Stencils run consecutively (Table I); one rendered kernel for the group."""

    def __init__(self, stencils):
        self.stencils = list(stencils)

    def compile(self):
        return Compiled([s.lower() for s in self.stencils])


class Compiled:
    """The callable ``compile()`` returns."""

    def __init__(self, lowered):
        self.lowered = lowered
        self.handle = sf.sf_stencil_compile(lowered)

    @property
    def source(self):
        return sf.sf_stencil_source(self.handle)

    def plan(self, nx, ny, nz, src_is_output=True):
        """Launches (dependence phases) on an nx x ny x nz grid (host only)."""
        return sf.sf_stencil_plan(self.handle, nx, ny, nz, src_is_output)

    @property
    def phases(self):
        return sf.sf_stencil_phases(self.handle)

    def __call__(self, level, src=None):
        sf.sf_stencil_apply(self.handle, level.handle, None if src is None else src.handle)

    def close(self):
        if getattr(self, "handle", None):
            sf.sf_stencil_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------------------------ HPGMG library
def red_black_domains():
    """3-D red / black DomainUnions (reading R-2 in stencil coordinates: red =
    (X+Y+Z) odd, i.e. 0-based interior (i+j+k) even), each 4 stride-2 rects."""
    I, E = -1, (2, 2, 2)
    red = (RectDomain((1, 1, 1), (I, I, I), E) + RectDomain((2, 2, 1), (I, I, I), E)
           + RectDomain((2, 1, 2), (I, I, I), E) + RectDomain((1, 2, 2), (I, I, I), E))
    black = (RectDomain((2, 1, 1), (I, I, I), E) + RectDomain((1, 2, 1), (I, I, I), E)
             + RectDomain((1, 1, 2), (I, I, I), E) + RectDomain((2, 2, 2), (I, I, I), E))
    return red, black


def dirichlet_faces(mesh):
    """The six face ghost stencils ghost = -inside (Fig 4 l.15-18 in 3-D).  The
    ghost layer is a degenerate axis: stride 0 = the single coordinate lo
    (reading R-17 of Fig 4 l.17), lo = 0 (low face) or -1 (= n+1, high face)."""
    out = []
    for d in range(3):
        for lo_d, off_d in ((0, 1), (-1, -1)):
            lo, hi, st, off = [1, 1, 1], [-1, -1, -1], [1, 1, 1], [0, 0, 0]
            lo[d], hi[d], st[d], off[d] = lo_d, lo_d, 0, off_d
            out.append(Stencil(Component(mesh, SparseArray({tuple(off): -1.0})), mesh,
                               RectDomain(tuple(lo), tuple(hi), tuple(st))))
    return out


def helmholtz_ax(a, b, h, x="u"):
    """A x = a alpha x - b h^-2 sum_f beta_f (x_nbr - x) (A3) as a Component
    with variable-coefficient weights (Fig 4 l.1-5 in 3-D)."""
    bw = Component("beta_i", SparseArray({(0, 0, 0): 1.0}))
    be = Component("beta_i", SparseArray({(1, 0, 0): 1.0}))
    bs = Component("beta_j", SparseArray({(0, 0, 0): 1.0}))
    bn = Component("beta_j", SparseArray({(0, 1, 0): 1.0}))
    bb = Component("beta_k", SparseArray({(0, 0, 0): 1.0}))
    bt = Component("beta_k", SparseArray({(0, 0, 1): 1.0}))
    alpha = Component("alpha", SparseArray({(0, 0, 0): 1.0}))
    c = -b / (h * h)
    centre = a * alpha - c * (((((bw + be) + bs) + bn) + bb) + bt)
    return Component(x, SparseArray({(0, 0, 0): centre, (-1, 0, 0): c * bw, (1, 0, 0): c * be,
                                     (0, -1, 0): c * bs, (0, 1, 0): c * bn,
                                     (0, 0, -1): c * bb, (0, 0, 1): c * bt}))


def gsrb_update(a, b, h, x="u", rhs="f"):
    """x + lambda (rhs - A x) (Fig 4 l.6-10; lambda = Dinv, reading R-4)."""
    return (Component(x, {(0, 0, 0): 1.0}) + Component("dinv", {(0, 0, 0): 1.0})
            * (Component(rhs, {(0, 0, 0): 1.0}) - helmholtz_ax(a, b, h, x)))


def hpgmg_gsrb_pair(a, b, h, x="u", rhs="f"):
    """One RB pair as the paper writes it: [BC, red, BC, black]."""
    red, black = red_black_domains()
    return StencilGroup(dirichlet_faces(x) + [Stencil(gsrb_update(a, b, h, x, rhs), x, red)]
                        + dirichlet_faces(x) + [Stencil(gsrb_update(a, b, h, x, rhs), x, black)])


def hpgmg_apply_op(a, b, h, out="r", x="u"):
    """[BC, out = A x] over the interior (A2 + A3)."""
    return StencilGroup(dirichlet_faces(x) + [
        Stencil(helmholtz_ax(a, b, h, x), out, RectDomain((1, 1, 1), (-1, -1, -1)))])
