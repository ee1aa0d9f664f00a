"""The N = 8 configuration and the failure paths of the multi-GPU transports,
exercised on the one GPU the test boxes have.

* 8-part loopback decomposition of a (64, 64, 256) level with the default
  agglomeration threshold (16 planes): two distributed levels, then
  agglomerated ones -- the same level pattern as bench.py's 1024^3 plan at
  N = 8 -- equal to one part (1e-13) and to the oracle (1e-10).
* 8 processes on one device with the device-initiated p2p transport: the
  per-rank code equals the loopback decomposition.
* A one-rank NCCL communicator: sf_comm_check runs ncclAllReduce (max, sum),
  ncclBroadcast and ncclAllGather; levels and a solve on that communicator
  (host-polled waits, ncclCommGetAsyncError).
* A dead or hung peer makes a p2p wait time out: the survivor gets
  SF_ERR_CUDA naming the timed-out flag within the bound instead of hanging.
"""
import os
import socket
import time

import numpy as np
import pytest
import torch.multiprocessing as mp

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


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def rel(a, b):
    return np.linalg.norm((a - b).ravel()) / np.linalg.norm(b.ravel())


def test_eight_part_decomposition_solve(sf, oracle):
    nx, ny, nz = 64, 64, 256
    h = I.level_h(nx, ny, nz)
    coeffs = I.hpgmg_coeffs(nx, ny, nz, h)
    _, f = I.manufactured(nx, ny, nz, 1.0, 1.0)
    out = {}
    for parts in (1, 8):
        comm = sf.Comm.local(parts) if parts > 1 else None
        L = sf.Level(nx, ny, nz, h, comm=comm)
        L.set_coeffs(*coeffs)
        L.upload(sf.SF_F, f)
        M = sf.MG(L, 1.0, 1.0)      # default agglom_min_planes = 16
        st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
        out[parts] = (L.download(sf.SF_U), cyc, hist, M.num_levels)
        M.close()
        L.close()
        if comm:
            comm.close()
    O = oracle.MG(nx, ny, nz, h, 1.0, 1.0, *coeffs)
    u_o, hist_o = O.solve(f, fcycle=True, rtol=1e-10)
    assert out[8][1] == out[1][1] == len(hist_o)
    assert out[8][3] == out[1][3]
    assert rel(out[8][0], out[1][0]) < 1e-13
    assert rel(out[8][0], u_o) < 1e-10 and rel(out[1][0], u_o) < 1e-10


# --------------------------------------------------------------- 8 processes
SMOOTH_SHAPE = (96, 16, 64)
N_SOLVE = 64


def _run8(sf, comm, world, rank):
    part = (lambda a: I.split_slabs(a, "cell", world)[rank]) if rank is not None else (lambda a: a)
    kinds = ["cell", "beta_i", "beta_j", "beta_k"]
    cpart = ((lambda c: [I.split_slabs(a, k, world)[rank] for a, k in zip(c, kinds)])
             if rank is not None else (lambda c: c))
    res = {}
    nz, ny, nx = SMOOTH_SHAPE
    coeffs = I.hpgmg_coeffs(nx, ny, nz)
    x, f = I.random_field(SMOOTH_SHAPE, 0), I.random_field(SMOOTH_SHAPE, 1)
    L = sf.Level(nx, ny, nz, comm=comm)
    L.set_coeffs(*cpart(coeffs))
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    L.upload(sf.SF_U, part(x))
    L.upload(sf.SF_F, part(f))
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, sf.SF_SMOOTH_FUSED)
    res["smooth"] = (L.download(sf.SF_U), sf.sf_norm(L.handle, sf.SF_U, 0))
    L.close()
    n = N_SOLVE
    coeffs = I.hpgmg_coeffs(n, n, n)
    _, fs = I.manufactured(n, n, n, 1.0, 1.0)
    L = sf.Level(n, n, n, comm=comm)
    L.set_coeffs(*cpart(coeffs))
    L.upload(sf.SF_F, part(fs))
    M = sf.MG(L, 1.0, 1.0, agglom_min_planes=4)
    st, cyc, hist = M.solve(fcycle=True)
    res["solve"] = (L.download(sf.SF_U), cyc, hist, M.num_levels)
    M.close()
    L.close()
    return res


def _worker8(rank, world, port, out):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        comm = sf.Comm.p2p()
        out[rank] = _run8(sf, comm, world, rank)
        dist.barrier()
        comm.close()
    finally:
        dist.destroy_process_group()


def test_eight_processes_p2p_match_loopback(sf):
    world = 8
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_worker8, args=(world, _free_port(), out), nprocs=world, join=True)
        ranks = {r: out[r] for r in range(world)}
    comm = sf.Comm.local(world)
    ref = _run8(sf, comm, world, None)
    u = np.concatenate([ranks[r]["smooth"][0] for r in range(world)])
    assert np.array_equal(u, ref["smooth"][0])
    for r in range(world):
        assert ranks[r]["smooth"][1] == ref["smooth"][1]
    u = np.concatenate([ranks[r]["solve"][0] for r in range(world)])
    for r in range(world):
        assert ranks[r]["solve"][1] == ref["solve"][1] and ranks[r]["solve"][3] == ref["solve"][3]
    assert rel(u, ref["solve"][0]) < 1e-13


# --------------------------------------------------------------- NCCL, 1 rank
def test_nccl_one_rank_smoke(sf, oracle):
    """ncclCommInitRank + every collective of the slab path (sf_comm_check),
    then a level and a full solve on the NCCL communicator (host loop with
    ncclCommGetAsyncError polling at every synchronisation)."""
    import torch
    uid = sf.sf_get_unique_id()
    h = sf.sf_comm_create_nccl(uid, 1, 0)
    comm = sf.Comm(h, 1, 1, 0)
    s = torch.cuda.Stream()
    sf.sf_comm_check(comm.h, s.cuda_stream)
    n = 64
    coeffs = I.hpgmg_coeffs(n, n, n)
    _, f = I.manufactured(n, n, n, 1.0, 1.0)
    L = sf.Level(n, n, n, comm=comm)
    L.set_coeffs(*coeffs)
    L.upload(sf.SF_F, f)
    assert sf.sf_norm(L.handle, sf.SF_F, 0) == np.abs(f).max()
    M = sf.MG(L, 1.0, 1.0)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
    O = oracle.MG(n, n, n, 1.0 / n, 1.0, 1.0, *coeffs)
    u_o, hist_o = O.solve(f, fcycle=True, rtol=1e-10)
    assert cyc == len(hist_o)
    assert rel(L.download(sf.SF_U), u_o) < 1e-10
    M.close()
    L.close()
    comm.close()


# ------------------------------------------------- dead / hung peer (p2p)
def _peer_fail_worker(rank, world, port, out, mode):
    os.environ["SF_P2P_TIMEOUT_S"] = "3"
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    comm = sf.Comm.p2p()
    L = sf.Level(64, 32, 64, comm=comm)
    L.upload(sf.SF_U, np.ones((32, 32, 64)))
    dist.barrier()
    if rank == 1:
        # never takes part in the next exchange
        if mode == "exit":
            os._exit(0)
        time.sleep(25)
        out[rank] = "slept"
        os._exit(0)
    t0 = time.time()
    try:
        sf.sf_norm(L.handle, sf.SF_U, 0)      # all-reduce over peer memory
        out[rank] = ("ok", time.time() - t0)
    except sf.SfError as e:
        out[rank] = (str(e), time.time() - t0, e.status)
    os._exit(0)   # the CUDA context is unusable after the trap


@pytest.mark.parametrize("mode", ["hung", "exit"])
def test_dead_peer_returns_error(sf, mode):
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_peer_fail_worker, args=(2, _free_port(), out, mode), nprocs=2, join=True)
        res = dict(out)
    msg, dt, status = res[0]
    assert status == sf.SF_ERR_CUDA, msg
    assert dt < 20.0, dt
    if mode == "hung":
        assert "p2p peer wait timed out" in msg, msg
