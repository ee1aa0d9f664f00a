"""The coarse-level V-cycle as one thread-block-cluster launch (coarse.cu:
nz/2 CTAs of one 2-plane layer each, iterates in registers / shared memory,
DSMEM z-neighbours, the coarsest levels gathered on CTA 0) from the first
single-part level of <= 32^3 cells down to the bottom and back: every colour
sweep, residual + restriction, P0 interpolation and the exact bottom solve run
in one kernel.  Compared with the oracle (1e-11 per cycle, same cycle counts
per solve) and with the per-phase launches it replaces (SF_COARSE_KERNEL=0),
for cluster caps 16 / 8 / 4 (SF_COARSE_MAX_CS: entry levels 32^3 / 16^3 / 8^3)."""
import numpy as np
import pytest

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

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


def rel(a, b):
    return np.linalg.norm((a - b).ravel()) / np.linalg.norm(b.ravel())


def _run(sf, shape, kernel, monkeypatch, cycles=2, fcycle=False, **opts):
    monkeypatch.setenv("SF_COARSE_KERNEL", "1" if kernel else "0")
    nz, ny, nx = shape
    h = I.level_h(nx, ny, nz)
    L = sf.Level(nx, ny, nz, h)
    L.set_coeffs(*I.hpgmg_coeffs(nx, ny, nz, h))
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    M = sf.MG(L, 1.0, 1.0, **opts)
    out = []
    if fcycle:
        M.fcycle()
        out.append(L.download(sf.SF_U))
    for _ in range(cycles):
        M.vcycle(0)
        out.append(L.download(sf.SF_U))
    M.close()
    L.close()
    return out, f


@pytest.mark.parametrize("shape", [(64, 64, 64), (32, 32, 32), (32, 64, 128), (64, 32, 32),
                                   (16, 16, 64)])
def test_coarse_kernel_cycles_vs_oracle(sf, oracle, shape, monkeypatch):
    nz, ny, nx = shape
    on, f = _run(sf, shape, True, monkeypatch, fcycle=True)
    off, _ = _run(sf, shape, False, monkeypatch, fcycle=True)
    h = I.level_h(nx, ny, nz)
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *I.hpgmg_coeffs(nx, ny, nz, h))
    u = O.fcycle(f)
    exp = [u]
    for _ in range(2):
        u = O.vcycle(u, f)
        exp.append(u)
    for a, b, e in zip(on, off, exp):
        assert rel(a, e) < 1e-11
        assert rel(a, b) < 1e-12


@pytest.mark.parametrize("cap", ["8", "4"])
@pytest.mark.parametrize("shape", [(64, 64, 64), (32, 64, 128)])
def test_coarse_kernel_cluster_caps(sf, oracle, shape, cap, monkeypatch):
    """Smaller clusters (entry 16^3 / 8^3 on the cube): same results."""
    monkeypatch.setenv("SF_COARSE_MAX_CS", cap)
    nz, ny, nx = shape
    on, f = _run(sf, shape, True, monkeypatch, fcycle=True)
    off, _ = _run(sf, shape, False, monkeypatch, fcycle=True)
    h = I.level_h(nx, ny, nz)
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *I.hpgmg_coeffs(nx, ny, nz, h))
    u = O.fcycle(f)
    exp = [u]
    for _ in range(2):
        u = O.vcycle(u, f)
        exp.append(u)
    for a, b, e in zip(on, off, exp):
        assert rel(a, e) < 1e-11
        assert rel(a, b) < 1e-12


@pytest.mark.parametrize("opts", [{"pre_pairs": 1, "post_pairs": 3},
                                  {"pre_pairs": 0, "post_pairs": 2},   # no folded red sweep
                                  {"pre_pairs": 2, "post_pairs": 0},
                                  {"smoother": 1},   # SF_SMOOTH_COLOUR
                                  {"pre_pairs": 3, "post_pairs": 1, "use_graph": 0}])
def test_coarse_kernel_options(sf, oracle, opts, monkeypatch):
    shape = (64, 64, 64)
    on, f = _run(sf, shape, True, monkeypatch, **opts)
    off, _ = _run(sf, shape, False, monkeypatch, **opts)
    for a, b in zip(on, off):
        assert rel(a, b) < 1e-12
    if "smoother" not in opts:   # the oracle's smoother is GSRB with the same pair counts
        n = shape[0]
        h = I.level_h(n, n, n)
        O = oracle.MG(n, n, n, h, 1.0, 1.0, *I.hpgmg_coeffs(n, n, n, h),
                      pre=opts["pre_pairs"], post=opts["post_pairs"])
        u = np.zeros_like(f)
        for a in on:
            u = O.vcycle(u, f)
            assert rel(a, u) < 1e-11


@pytest.mark.parametrize("n", [32, 64, 128])
def test_coarse_kernel_solve(sf, oracle, n, monkeypatch):
    """Solve to 1e-10 (device loop): same cycle count and history as the
    oracle (1e-6 relative plus the residual's rounding floor), u within 1e-10."""
    monkeypatch.setenv("SF_COARSE_KERNEL", "1")
    h = 1.0 / n
    coeffs = I.hpgmg_coeffs(n, n, n, h)
    L = sf.Level(n, n, n, h)
    L.set_coeffs(*coeffs)
    ue, f = I.manufactured(n, n, n, 1.0, 1.0)
    L.upload(sf.SF_F, f)
    M = sf.MG(L, 1.0, 1.0)
    st, cyc, hist = M.solve(fcycle=False, rtol=1e-10)
    O = oracle.MG(n, n, n, h, 1.0, 1.0, *coeffs)
    u_o, hist_o = O.solve(f, fcycle=False, rtol=1e-10)
    assert cyc == len(hist_o)
    # atol: the max-norm residual's absolute rounding floor, ~1e-13 at 512^3
    # scaled by h^-2 (R-19); the 128^3 level takes the
    # delta-form restricted residual, which rounds differently from rhs - Ax
    assert np.allclose(hist, hist_o, rtol=1e-6, atol=1e-12 * (n / 512) ** 2)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10
    M.close()
    L.close()


def test_coarse_kernel_decomposed_fine_levels(sf, monkeypatch):
    """Distributed fine levels (4 loopback parts) above replicated coarse
    levels run by the cluster kernel: equal to one part."""
    monkeypatch.setenv("SF_COARSE_KERNEL", "1")
    n = 64
    coeffs = I.hpgmg_coeffs(n, n, n)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    out = []
    for parts in (1, 4):
        comm = sf.Comm.local(parts) if parts > 1 else None
        L = sf.Level(n, n, n, comm=comm)
        L.set_coeffs(*coeffs)
        L.upload(sf.SF_F, f)
        M = sf.MG(L, 1.0, 1.0, agglom_min_planes=4)
        st, cyc, hist = M.solve(fcycle=True)
        out.append((L.download(sf.SF_U), cyc))
        M.close()
        L.close()
    assert out[0][1] == out[1][1]
    assert rel(out[1][0], out[0][0]) < 1e-13
