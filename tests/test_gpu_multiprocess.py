"""Per-rank z-slab path in SEPARATE processes.

The driver's GPU boxes have one B200 and NCCL refuses two ranks on one
device, so the NCCL transport cannot run here.  These tests run the same
per-rank code (one part per process: slab offsets, depth-1/2 halos before
every operator/pair, all-reduced norms and lambda_max, agglomeration of the
coarse planes onto every rank, replicated coarse levels) with the hostipc
transport (world_size processes on cuda:0, peer buffers opened through CUDA
IPC, host synchronisation over gloo) and with the p2p transport (the same
peer buffers, but halos / agglomeration / all-reduces are kernels that read
the peers' memory and synchronise through device flags, CUDA graphs on).  The result must equal the in-process
loopback decomposition (itself pinned to the undecomposed run and to the
oracle in test_gpu_parity.py)."""
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I

pytestmark = pytest.mark.gpu

SMOOTH_SHAPE = (96, 16, 64)   # >= 24 planes per rank: halo overlapped with the interior chunks
N_SOLVE = 64


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _slab_coeffs(coeffs, world, rank):
    kinds = ["cell", "beta_i", "beta_j", "beta_k"]
    return [I.split_slabs(c, k, world)[rank] for c, k in zip(coeffs, kinds)]


def _run(sf, comm, world, rank, out_key, out):
    """The same sequence on a hostipc (comm given) or loopback (rank None) level."""
    part = (lambda a: I.split_slabs(a, "cell", world)[rank]) if rank is not None else (lambda a: a)
    cpart = (lambda c: _slab_coeffs(c, world, rank)) if rank is not None else (lambda c: c)
    res = {}
    # fused and colour GSRB pairs + residual (halo depth 2 / 1 every pair)
    nz, ny, nx = SMOOTH_SHAPE
    coeffs = I.hpgmg_coeffs(nx, ny, nz)
    x, f = I.random_field(SMOOTH_SHAPE, 0), I.random_field(SMOOTH_SHAPE, 1)
    for kind in (sf.SF_SMOOTH_COLOUR, sf.SF_SMOOTH_FUSED):
        L = sf.Level(nx, ny, nz, comm=comm)
        L.set_coeffs(*cpart(coeffs))
        sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
        L.upload(sf.SF_U, part(x))
        L.upload(sf.SF_F, part(f))
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
        sf.sf_residual(L.handle, sf.SF_R, sf.SF_U, sf.SF_F, 1.0, 1.0)
        nrm = sf.sf_norm(L.handle, sf.SF_R, 0)
        res[("smooth", kind)] = (L.download(sf.SF_U), L.download(sf.SF_R), nrm)
        L.close()
    # full solves: GSRB F-cycle and Chebyshev V-cycle (all-reduced lambda_max)
    n = N_SOLVE
    coeffs = I.hpgmg_coeffs(n, n, n)
    _, fs = I.manufactured(n, n, n, 1.0, 1.0)
    for name, opts, fcyc in (("gsrb_f", {}, True),
                             ("cheby_v", {"smoother": sf.SF_SMOOTH_CHEBY}, False)):
        L = sf.Level(n, n, n, comm=comm)
        L.set_coeffs(*cpart(coeffs))
        L.upload(sf.SF_F, part(fs))
        M = sf.MG(L, 1.0, 1.0, agglom_min_planes=4, **opts)
        st, cyc, hist = M.solve(fcycle=fcyc)
        res[name] = (L.download(sf.SF_U), cyc, hist, M.num_levels)
        M.close()
        L.close()
    out[out_key] = res


def _worker(rank, world, port, out, transport):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        comm = sf.Comm.hostipc() if transport == "hostipc" else sf.Comm.p2p()
        _run(sf, comm, world, rank, rank, out)
        dist.barrier()
        comm.close()
    finally:
        dist.destroy_process_group()


@pytest.fixture(scope="module")
def sf():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_zhangdmwbf17_b200 import build, sf as S
    build.build()
    S.lib()
    return S


@pytest.mark.parametrize("transport", ["hostipc", "p2p"])
@pytest.mark.parametrize("world", [2, 4])
def test_per_rank_matches_loopback(sf, world, transport):
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_worker, args=(world, _free_port(), out, transport), nprocs=world, join=True)
        ranks = {r: out[r] for r in range(world)}
    ref = {}
    comm = sf.Comm.local(world)
    _run(sf, comm, world, None, "ref", ref)
    ref = ref["ref"]
    # smoother + residual: identical arithmetic on identical data -> bit-exact
    for kind in (sf.SF_SMOOTH_COLOUR, sf.SF_SMOOTH_FUSED):
        u = np.concatenate([ranks[r][("smooth", kind)][0] for r in range(world)])
        rr = np.concatenate([ranks[r][("smooth", kind)][1] for r in range(world)])
        assert np.array_equal(u, ref[("smooth", kind)][0])
        assert np.array_equal(rr, ref[("smooth", kind)][1])
        for r in range(world):  # all-reduced max norm is the same on every rank
            assert ranks[r][("smooth", kind)][2] == ref[("smooth", kind)][2]
    for name in ("gsrb_f", "cheby_v"):
        u = np.concatenate([ranks[r][name][0] for r in range(world)])
        uref, cref, href, lref = ref[name]
        for r in range(world):
            assert ranks[r][name][1] == cref and ranks[r][name][3] == lref
            # relres history: the same up to the rounding of the distributed sums
            # (Chebyshev's lambda_max is an all-reduced sum of partial dots)
            np.testing.assert_allclose(ranks[r][name][2], href, rtol=1e-9, atol=1e-13 * href[0])
        rel = np.linalg.norm((u - uref).ravel()) / np.linalg.norm(uref.ravel())
        assert rel < 1e-13, (name, rel)


def _fail_worker(rank, world, port, out):
    import os

    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    os.environ["SF_TEST_IPC_FAIL_RANK"] = "1"
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        comm = sf.Comm.p2p()
        try:
            sf.Level(32, 32, 48, comm=comm)
            out[rank] = "created"
        except sf.SfError as e:
            out[rank] = str(e)
        dist.barrier()
        comm.close()
    finally:
        dist.destroy_process_group()


def test_p2p_registration_fails_on_every_rank(sf):
    """One rank cannot map its peers' buffers: every rank gets the same error
    (no rank is left waiting in a barrier), so callers can fall back together
    (bench.py switches to NCCL)."""
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_fail_worker, args=(3, _free_port(), out), nprocs=3, join=True)
        res = dict(out)
    assert len(res) == 3
    assert all("rank 1 could not export or open" in v for v in res.values()), res
