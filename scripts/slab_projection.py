"""Per-rank cost of bench.py's N-GPU weak-scaling slabs, measured on ONE GPU:
the global problem of N ranks is built as an N-part loopback level on one
device (every part is exactly a rank's slab: same kernels, same launch shapes,
same split-phase fused pairs beside the halo copies), so solve time / N is the
per-rank work of the N-GPU run without its inter-GPU exchanges.  Compared with
the 512^3 single-part solve this projects the weak-scaling efficiency that the
slab shape alone allows.     python scripts/slab_projection.py [N ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402
from paper_conf_ipps_zhangdmwbf17_b200.parallel import weak_dims  # noqa: E402


def solve_ms(nx, ny, nz, parts, reps=3):
    comm = sf.Comm.local(parts) if parts > 1 else None
    L = sf.Level(nx, ny, nz, 1.0 / max(nx, ny, nz), comm=comm)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    s = L.stream
    st, cyc, hist = M.solve(True, 1e-10, 50)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.synchronize()
    a.record(s)
    for _ in range(reps):
        st, cyc, hist = M.solve(True, 1e-10, 50)
    b.record(s)
    s.synchronize()
    ms = a.elapsed_time(b) / reps
    M.close()
    L.close()
    if comm:
        comm.close()
    torch.cuda.empty_cache()
    return ms, cyc, hist[-1]


base, cyc1, r1 = solve_ms(512, 512, 512, 1)
print(f"N=1 512x512x512 single part: {base:.1f} ms/solve, {cyc1} cycles, relres {r1:.2e}")
for n in [int(v) for v in sys.argv[1:]] or [2]:
    nx, ny, nz = weak_dims(512, n)
    ms, cyc, r = solve_ms(nx, ny, nz, n, reps=2)
    per = ms / n
    print(f"N={n} global {nx}x{ny}x{nz} as {n} loopback parts: {ms:.1f} ms/solve on one GPU "
          f"-> {per:.1f} ms per rank-slab, {cyc} cycles, relres {r:.2e}; "
          f"slab-shape efficiency {base / per:.3f} (halos as on-device copies; no inter-GPU link)")
