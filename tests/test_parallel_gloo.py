"""Multi-process (world_size 2, gloo, CPU) tests of the host side of the
z-slab path: NCCL-id bootstrap through torch.distributed, slab ownership, the
agglomeration plan every rank must agree on, and max-over-ranks timing."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    import torch.distributed as dist

    from paper_conf_ipps_zhangdmwbf17_b200 import parallel, sf
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        uid, r, w = parallel.broadcast_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        gnx, gny, gnz = parallel.weak_dims(512, world)
        plan = sf.sf_mg_plan(gnx, gny, gnz, world, 16)
        plans = [None] * world
        dist.all_gather_object(plans, plan)
        slabs = [None] * world
        dist.all_gather_object(slabs, parallel.slab(gnz, world, rank))
        tmax = parallel.max_over_ranks(1.0 + rank)
        tsum = parallel.sum_over_ranks(1.0 + rank)
        out[rank] = dict(ids=ids, plans=plans, slabs=slabs, tmax=tmax, tsum=tsum, r=r, w=w,
                         dims=(gnx, gny, gnz))
    finally:
        dist.destroy_process_group()


@pytest.fixture(scope="module")
def gloo_results():
    from paper_conf_ipps_zhangdmwbf17_b200 import build
    build.build()
    world = 2
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
        return dict(out)


def test_unique_id_broadcast(gloo_results):
    for r, res in gloo_results.items():
        assert res["r"] == r and res["w"] == 2
        assert len(set(res["ids"])) == 1 and len(res["ids"][0]) == 128


def test_plan_agreement_and_agglomeration(gloo_results):
    plans = [p for res in gloo_results.values() for p in res["plans"]]
    assert all(p == plans[0] for p in plans)
    plan = plans[0]
    assert plan[0] == ((512, 512, 1024), True)          # BASELINE C5 at N = 2
    assert plan[-1][1] is False                           # bottom replicated
    flags = [d for _, d in plan]
    k = flags.index(False)
    assert all(flags[:k]) and not any(flags[k:])          # agglomerate once, stay replicated
    for (dims, dist) in plan:
        if dist:
            assert (dims[2] // 2) >= 16 and (dims[2] // 2) % 2 == 0 or dims == plan[0][0]


def test_slabs_partition_domain(gloo_results):
    res = gloo_results[0]
    slabs = sorted(res["slabs"])
    gnz = res["dims"][2]
    assert slabs[0][0] == 0 and slabs[-1][1] == gnz
    assert all(a[1] == b[0] for a, b in zip(slabs, slabs[1:]))


def test_max_over_ranks(gloo_results):
    for res in gloo_results.values():
        assert res["tmax"] == 2.0 and res["tsum"] == 3.0


def test_plan_rejects_bad_shapes():
    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    with pytest.raises(sf.SfError):
        sf.sf_mg_plan(512, 512, 1000, 8, 16)      # 1000 % 8 != 0 ... 125 planes: odd
    with pytest.raises(sf.SfError):
        sf.sf_mg_plan(512, 512, 30, 2, 16)        # 15 planes per slab cannot halve
    assert len(sf.sf_mg_plan(16, 16, 16)) == 4


def test_mg_plan_matches_bench_n8():
    """bench.py at N = 8: 1024^3 in 8 slabs of 128 planes stays distributed
    down to 128^3 (16 planes per rank) and is agglomerated from 64^3 on; the
    64x64x256 8-part GPU test (test_gpu_multigpu_readiness.py) has the same
    pattern: distributed levels, then agglomerated ones down to the bottom."""
    from paper_conf_ipps_zhangdmwbf17_b200 import sf
    d8 = [d for _, d in sf.sf_mg_plan(1024, 1024, 1024, 8, 16)]
    dt = [d for _, d in sf.sf_mg_plan(64, 64, 256, 8, 16)]
    assert d8 == [True] * 4 + [False] * 6
    assert dt == [True] * 2 + [False] * 4
