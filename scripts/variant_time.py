"""Event-time the fused pair variants at n^3: plain, INTERP (P0-fused), RESID (check-fused)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhangdmwbf17_b200 import sf
n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
s = L.stream
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def t(fn, reps=10):
    for _ in range(3): fn()
    s.synchronize(); a.record(s)
    for _ in range(reps): fn()
    b.record(s); s.synchronize()
    return a.elapsed_time(b) / reps
print(f"n={n} plain pair {t(lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)):.4f} ms")
v = t(lambda: sf.sf_vcycle(M.handle, 0), 5)
print(f"n={n} V-cycle (eager) {v:.3f} ms")
st, cyc, hist = M.solve(True, 1e-10, 50)
print(f"n={n} solve {t(lambda: M.solve(True, 1e-10, 50), 3):.2f} ms cycles {cyc}")
