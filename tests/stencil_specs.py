"""Plain-data stencil specs shared by the stencil tests (test code only): the
oracle (oracle/stencil.py) takes them as they are; ``to_dsl`` builds the same
stencil with the product's DSL (paper_conf_ipps_zhangdmwbf17_b200/stencil.py)
so the two sides evaluate one description without sharing code."""

I3 = (-1, -1, -1)
ONE = (1, 1, 1)


def comp(mesh, terms, src=0, mul=ONE, div=ONE, pre=(0, 0, 0)):
    return ("comp", mesh, terms, src, mul, div, pre)


def at(mesh, off=(0, 0, 0), src=0):
    return comp(mesh, [(off, 1.0)], src)


RED = [((1, 1, 1), I3, (2, 2, 2)), ((2, 2, 1), I3, (2, 2, 2)),
       ((2, 1, 2), I3, (2, 2, 2)), ((1, 2, 2), I3, (2, 2, 2))]
BLACK = [((2, 1, 1), I3, (2, 2, 2)), ((1, 2, 1), I3, (2, 2, 2)),
         ((1, 1, 2), I3, (2, 2, 2)), ((2, 2, 2), I3, (2, 2, 2))]


def bc_faces(mesh):
    out = []
    for d in range(3):
        for lo_d, off_d in ((0, 1), (-1, -1)):
            lo, hi, st, off = [1, 1, 1], [-1, -1, -1], [1, 1, 1], [0, 0, 0]
            lo[d], hi[d], st[d], off[d] = lo_d, lo_d, 0, off_d
            out.append({"out": mesh, "rects": [(tuple(lo), tuple(hi), tuple(st))],
                        "expr": comp(mesh, [(tuple(off), -1.0)])})
    return out


def helmholtz_ax(a, b, h, x="u"):
    """A3 as a Component with variable-coefficient weights (Fig 4 l.1-5, 3-D)."""
    bw, be = at("beta_i"), at("beta_i", (1, 0, 0))
    bs, bn = at("beta_j"), at("beta_j", (0, 1, 0))
    bb, bt = at("beta_k"), at("beta_k", (0, 0, 1))
    c = -b / (h * h)
    ssum = ("+", ("+", ("+", ("+", ("+", bw, be), bs), bn), bb), bt)
    centre = ("-", ("*", ("const", a), at("alpha")), ("*", ("const", c), ssum))
    cw = lambda e: ("*", ("const", c), e)   # noqa: E731
    return comp(x, [((0, 0, 0), centre), ((-1, 0, 0), cw(bw)), ((1, 0, 0), cw(be)),
                    ((0, -1, 0), cw(bs)), ((0, 1, 0), cw(bn)),
                    ((0, 0, -1), cw(bb)), ((0, 0, 1), cw(bt))])


def gsrb_colour(a, b, h, rects):
    """x + lambda (rhs - A x) on a colour's DomainUnion (Fig 4 l.6-14)."""
    e = ("+", at("u"), ("*", at("dinv"), ("-", at("f"), helmholtz_ax(a, b, h))))
    return {"out": "u", "rects": rects, "expr": e}


def restriction_spec(mesh_c, mesh_f):
    terms = [((aa - 1, bb - 1, d - 1), 1.0) for d in (0, 1) for bb in (0, 1) for aa in (0, 1)]
    return {"out": mesh_c, "rects": [(ONE, I3, ONE)],
            "expr": ("/", comp(mesh_f, terms, src=1, mul=(2, 2, 2)), ("const", 8.0))}


def p0_spec(mesh_f, mesh_c):
    e = ("+", at(mesh_f), comp(mesh_c, [((0, 0, 0), 1.0)], src=1, div=(2, 2, 2), pre=(1, 1, 1)))
    return {"out": mesh_f, "rects": [(ONE, I3, ONE)], "expr": e}




def to_dsl(spec_group):
    """Plain specs -> product StencilGroup (mirrors each expression node)."""
    from paper_conf_ipps_zhangdmwbf17_b200 import stencil as S

    def ex(E):
        t = E[0]
        if t == "const":
            return S.Const(E[1])
        if t == "comp":
            _, mesh, terms, src, mul, div, pre = E
            w = {}
            for off, wt in terms:
                w[tuple(off)] = ex(wt) if isinstance(wt, tuple) else wt
            if len(w) != len(terms):
                raise ValueError("duplicate offsets in a component")
            return S.Component(mesh, S.SparseArray(w), src=src, mul=mul, div=div, pre=pre)
        if t == "neg":
            return -ex(E[1])
        a, b = ex(E[1]), ex(E[2])
        return {"+": lambda: a + b, "-": lambda: a - b, "*": lambda: a * b,
                "/": lambda: a / b}[t]()

    out = []
    for s in spec_group:
        dom = None
        for lo, hi, st in s["rects"]:
            r = S.RectDomain(lo, hi, st)
            dom = r if dom is None else dom + r
        out.append(S.Stencil(ex(s["expr"]), s["out"], dom))
    return S.StencilGroup(out)
