"""Host side of the generic stencil engine (NEXT-4), no GPU: the DSL front end
lowers and renders, and the Diophantine dependence analysis (sf_stencil_plan)
agrees with brute-force point-set intersection on random strided domains."""
import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import sf
from paper_conf_ipps_zhangdmwbf17_b200 import stencil as S


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_ipps_zhangdmwbf17_b200 import build
    build.build()
    sf.lib()


def u_at(off):
    return S.Component("u", S.SparseArray({off: 1.0}))


INTERIOR = S.RectDomain((1, 1, 1), (-1, -1, -1))


def gsrb_group(a=1.0, b=1.0, h=0.125):
    red, black = S.red_black_domains()
    upd = lambda: (S.Component("u", {(0, 0, 0): 1.0})   # noqa: E731
                   + S.Component("dinv", {(0, 0, 0): 1.0})
                   * (S.Component("f", {(0, 0, 0): 1.0}) - S.helmholtz_ax(a, b, h)))
    return S.StencilGroup(S.dirichlet_faces("u") + [S.Stencil(upd(), "u", red)]
                          + S.dirichlet_faces("u") + [S.Stencil(upd(), "u", black)])


def test_render_and_source():
    c = gsrb_group().compile()
    src = c.source
    assert 'extern "C" __global__' in src and "sf_stencil_group" in src
    assert src.count("case ") == 14          # 12 boundary stencils + red + black
    # the weight-array lowering reads each (mesh, offset) once per stencil
    red_ev = src.split("sf_ev6(")[1].split("sf_ev7(")[0]
    assert red_ev.count("a.f[0][0][") == 7          # u at its 7 offsets, each once
    c.close()


def test_weight_array_offsets():
    """Nested lists: outermost = x, centre element = offset 0 (reading R-18)."""
    wa = S.WeightArray([[[0, 1, 0]], [[2, 3, 4]], [[0, 5, 0]]])
    items = dict(wa.items())
    assert items[(0, 0, 0)] == 3 and items[(0, 0, -1)] == 2 and items[(0, 0, 1)] == 4
    assert items[(-1, 0, 0)] == 1 and items[(1, 0, 0)] == 5
    assert dict(S.WeightArray([7, 8, 9]).items())[(1, 0, 0)] == 9
    with pytest.raises(ValueError):
        S.WeightArray([1, 2]).items()


def test_gsrb_group_phases():
    """BC faces are mutually independent (1 launch); red reads the ghosts they
    wrote (RAW); the next BC reads cells red wrote; black reads those ghosts."""
    c = gsrb_group().compile()
    assert c.plan(16, 16, 16) == 4
    c.close()


def test_racy_in_place_rejected():
    jac = S.Stencil(u_at((-1, 0, 0)) + u_at((1, 0, 0)), "u", INTERIOR).compile()
    with pytest.raises(sf.SfError) as e:
        jac.plan(8, 8, 8)
    assert e.value.status == sf.SF_ERR_INVALID
    # out of place is fine; colour-restricted in place is fine
    ok = S.Stencil(u_at((-1, 0, 0)) + u_at((1, 0, 0)), "tmp", INTERIOR).compile()
    assert ok.plan(8, 8, 8) == 1
    red, _ = S.red_black_domains()
    ok2 = S.Stencil(u_at((-1, 0, 0)) + u_at((0, 0, 1)), "u", red).compile()
    assert ok2.plan(8, 8, 8) == 1
    # red+black in one in-place stencil reads what it writes
    red, black = S.red_black_domains()
    bad = S.Stencil(u_at((1, 0, 0)), "u", red + black).compile()
    with pytest.raises(sf.SfError):
        bad.plan(8, 8, 8)
    # overlapping rects of one stencil that reads its own point race too
    dup = S.Stencil(u_at((0, 0, 0)) + 1.0, "u", INTERIOR + INTERIOR).compile()
    with pytest.raises(sf.SfError):
        dup.plan(8, 8, 8)
    for c in (jac, ok, ok2, bad, dup):
        c.close()


def _lattice(lo, hi, st, n):
    N = n + 2
    a = lo + N if lo < 0 else lo
    b = hi + N if hi < 0 else hi
    if st == 0:
        return {a}
    return set(range(a, b, st))


def test_diophantine_matches_brute_force():
    """Stencil A writes u over rect RA; stencil B reads u at offset o over RB and
    writes tmp.  One launch iff no point of RB+o lies in RA (per-axis lattice
    intersection, extended Euclid) -- checked against explicit point sets."""
    rng = np.random.default_rng(5)
    n = 13
    agree = {True: 0, False: 0}
    for _ in range(300):
        ra = [(int(rng.integers(0, 4)), int(rng.integers(-3, 0)), int(rng.integers(0, 5)))
              for _ in range(3)]
        rb = [(int(rng.integers(0, 4)), int(rng.integers(-3, 0)), int(rng.integers(0, 5)))
              for _ in range(3)]
        off = tuple(int(v) for v in rng.integers(-2, 3, size=3))
        A = S.Stencil(S.Component("f", {(0, 0, 0): 2.0}), "u",
                      S.RectDomain(*[tuple(r[k] for r in ra) for k in range(3)]))
        B = S.Stencil(u_at(off), "tmp", S.RectDomain(*[tuple(r[k] for r in rb) for k in range(3)]))
        c = S.StencilGroup([A, B]).compile()
        phases = c.plan(n, n, n)
        c.close()
        hit = all(bool({x + off[d] for x in _lattice(*rb[d], n)} & _lattice(*ra[d], n))
                  for d in range(3))
        assert phases == (2 if hit else 1), (ra, rb, off)
        agree[hit] += 1
    assert agree[True] > 20 and agree[False] > 20


def test_waw_and_war():
    red, black = S.red_black_domains()
    # WAW on disjoint colours of the same mesh: independent
    g = S.StencilGroup([S.Stencil(S.Component("f", {(0, 0, 0): 1.0}), "u", red),
                        S.Stencil(S.Component("f", {(0, 0, 0): 2.0}), "u", black)]).compile()
    assert g.plan(8, 8, 8) == 1
    # WAR: the second writes f where the first reads it
    g2 = S.StencilGroup([S.Stencil(S.Component("f", {(0, 0, 0): 1.0}), "u", INTERIOR),
                         S.Stencil(u_at((0, 0, 0)), "f", INTERIOR)]).compile()
    assert g2.plan(8, 8, 8) == 2
    g.close()
    g2.close()


def test_compile_rejects_malformed():
    with pytest.raises(sf.SfError):
        sf.sf_stencil_compile([([{"op": sf.SF_SX_ADD, "a": 0, "b": 0}], 0, 0,
                                [((1, 1, 1), (-1, -1, -1), (1, 1, 1))])])
    with pytest.raises(sf.SfError):
        sf.sf_stencil_compile([([{"op": sf.SF_SX_CONST, "value": float("nan")}], 0, 0,
                                [((1, 1, 1), (-1, -1, -1), (1, 1, 1))])])
    with pytest.raises(sf.SfError):
        sf.sf_stencil_compile([([{"op": sf.SF_SX_READ, "mesh": 42}], 0, 0,
                                [((1, 1, 1), (-1, -1, -1), (1, 1, 1))])])
