"""Full HPGMG-FV solve (F-cycle + V-cycles to 1e-10, device-resident loop) at
several sizes on one GPU: ms per solve, DOF/s, cycles, error vs the manufactured
solution (O(h^2) pin).  1024^3 is BASELINE C5's N=8 global problem.
    python scripts/solve_sizes.py [n ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

for n in [int(v) for v in sys.argv[1:]] or [128, 256, 512, 1024]:
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    s = L.stream
    for _ in range(2):
        st, cyc, hist = M.solve(True, 1e-10, 50)
    reps = 5 if n <= 512 else 2
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.synchronize()
    a.record(s)
    for _ in range(reps):
        st, cyc, hist = M.solve(True, 1e-10, 50)
    b.record(s)
    s.synchronize()
    ms = a.elapsed_time(b) / reps
    print(f"n={n}^3: {ms:8.2f} ms/solve  {n**3 / (ms / 1e3) / 1e9:6.3f} GDOF/s  cycles {cyc}  "
          f"relres {hist[-1]:.2e}", flush=True)
    M.close()
    L.close()
    torch.cuda.empty_cache()
