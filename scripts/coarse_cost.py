"""Per-V-cycle time of small hierarchies (graph replay through sf_solve with a
fixed cycle count): the coarse-level share of the 512^3 V-cycle.
    python scripts/coarse_cost.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

for n in (8, 16, 32, 64, 128, 256):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    s = L.stream
    for _ in range(3):
        M.vcycle(0)
    # eager V-cycles (host enqueue) and graph-replayed solves with a forced cycle count
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.synchronize()
    a.record(s)
    for _ in range(20):
        M.vcycle(0)
    b.record(s)
    s.synchronize()
    eager = a.elapsed_time(b) / 20
    M.solve(fcycle=False, rtol=1e-300, max_cycles=10, raise_on_error=False)
    s.synchronize()
    a.record(s)
    st, cyc, hist = M.solve(fcycle=False, rtol=1e-300, max_cycles=20, raise_on_error=False)
    b.record(s)
    s.synchronize()
    g = a.elapsed_time(b) / max(cyc, 1)
    print(f"n={n:4d} levels={M.num_levels} eager V {eager * 1e3:8.1f} us   graph solve per cycle {g * 1e3:8.1f} us")
    del M, L
