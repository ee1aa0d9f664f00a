"""Two ranks on ONE GPU through the real NCCL path (if NCCL allows it here):
z-slab decomposed solve vs a single-process solve of the same problem."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import torch.distributed as dist

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I, sf

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo")
n = int(os.environ.get("N", "64"))
comm = sf.Comm.nccl()
L = sf.Level(n, n, n, 1.0 / n, comm=comm)
al, bi, bj, bk = I.hpgmg_coeffs(n, n, n)
l = n // world
sl = slice(rank * l, (rank + 1) * l)
L.set_coeffs(al[sl], bi[sl], bj[sl], bk[rank * l:(rank + 1) * l + 1])
_, f = I.manufactured(n, n, n, 1.0, 1.0)
L.upload(sf.SF_F, f[sl])
M = sf.MG(L, 1.0, 1.0, agglom_min_planes=int(os.environ.get("AGG", "8")))
st, cyc, hist = M.solve(fcycle=True, rtol=1e-10)
u = L.download(sf.SF_U)
parts = [None] * world
dist.all_gather_object(parts, u)
if rank == 0:
    uu = np.concatenate(parts, axis=0)
    L1 = sf.Level(n, n, n, 1.0 / n)
    L1.set_coeffs(al, bi, bj, bk)
    L1.upload(sf.SF_F, f)
    M1 = sf.MG(L1, 1.0, 1.0)
    st1, cyc1, hist1 = M1.solve(fcycle=True, rtol=1e-10)
    u1 = L1.download(sf.SF_U)
    err = np.linalg.norm(uu - u1) / np.linalg.norm(u1)
    print(f"NCCL {world} ranks: cycles {cyc} vs {cyc1}, rel diff {err:.3e}, levels {M.num_levels}", flush=True)
    assert cyc == cyc1 and err < 1e-12
M.close(); L.close(); comm.close()
dist.destroy_process_group()
