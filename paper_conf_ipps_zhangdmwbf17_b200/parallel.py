"""Host-side plumbing of the z-slab decomposition.

One process per GPU; torch.distributed carries only bootstrap and timing
scalars (NCCL on GPU boxes, gloo for the CPU tests): the NCCL unique id that
libsf's communicator is built from, the slab each rank owns, and the
max-over-ranks of a device time.  Halos, norms and agglomeration run inside
libsf (NCCL over NVLink), never here.
"""
from __future__ import annotations

import os

# BASELINE config 5: 2^27 cells per GPU, global shapes per world size (x, y, z)
WEAK_SHAPES = {1: (512, 512, 512), 2: (512, 512, 1024), 4: (512, 1024, 1024),
               8: (1024, 1024, 1024)}


def env_rank():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def weak_dims(n, world):
    """Global (nx, ny, nz) for n^3 cells per GPU on `world` GPUs (z-slabs)."""
    if n == 512 and world in WEAK_SHAPES:
        return WEAK_SHAPES[world]
    return (n, n, n * world)


def slab(gnz, world, rank):
    """[z0, z1) of rank's slab (sf.h: part p owns [p*lnz, (p+1)*lnz))."""
    if gnz % world:
        raise ValueError(f"gnz={gnz} not divisible by {world}")
    l = gnz // world
    return rank * l, (rank + 1) * l


def broadcast_unique_id(group=None, make_id=None):
    """Rank 0 creates the NCCL unique id (libsf), every rank receives it.
    Returns (id_bytes, rank, world)."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    if make_id is None:
        from . import sf
        make_id = sf.sf_get_unique_id
    box = [make_id() if rank == 0 else None]
    dist.broadcast_object_list(box, src=0, group=group)
    uid = box[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise RuntimeError("bad NCCL unique id")
    return bytes(uid), rank, world


def max_over_ranks(x, device=None, group=None):
    """Max of a host float over ranks (device timing rule: max over ranks)."""
    import torch
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def sum_over_ranks(x, device=None, group=None):
    import torch
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return float(t.item())
