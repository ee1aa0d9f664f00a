"""C4 strong scaling projected on ONE GPU: the global 512^3 F-cycle (HPGMG FOM)
split into N z-slab loopback parts on one device.  Every distributed part is
exactly a rank's slab (same kernels and launch shapes); the parts run one after
another here, while the agglomerated coarse levels run once here but on EVERY
rank there.  Per-rank time = (T_N - T_rep) / N + T_rep, with T_rep the time of
the replicated levels (an F-cycle of the agglomeration level's hierarchy on
one part).  Inter-GPU exchanges are not included (on-device copies instead).
    python scripts/strong_projection.py [N ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def fcycle_ms(n, parts, reps=5):
    comm = sf.Comm.local(parts) if parts > 1 else None
    L = sf.Level(n, n, n, 1.0 / n, comm=comm)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    s = L.stream
    for _ in range(2):
        M.fcycle()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.synchronize()
    a.record(s)
    for _ in range(reps):
        M.fcycle()
    b.record(s)
    s.synchronize()
    ms = a.elapsed_time(b) / reps
    plan = sf.sf_mg_plan(n, n, n, parts, 16)
    M.close()
    L.close()
    if comm:
        comm.close()
    torch.cuda.empty_cache()
    return ms, plan


n = 512
t1, _ = fcycle_ms(n, 1)
print(f"N=1 {n}^3 F-cycle: {t1:.3f} ms ({n**3 / t1 / 1e6:.3f} GDOF/s)", flush=True)
for N in [int(v) for v in sys.argv[1:]] or [2, 4, 8]:
    tN, plan = fcycle_ms(n, N)
    rep = [d for d, dist in plan if not dist]
    t_rep = fcycle_ms(rep[0][0], 1)[0] if rep else 0.0
    per = (tN - t_rep) / N + t_rep
    print(f"N={N}: {N} parts of {n}x{n}x{n // N}: {tN:.3f} ms on one GPU, replicated levels from "
          f"{rep[0] if rep else None} {t_rep:.3f} ms -> {per:.3f} ms per rank; speedup {t1 / per:.2f} "
          f"(efficiency {t1 / per / N:.3f}; exchanges excluded)", flush=True)
