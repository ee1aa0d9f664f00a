"""Per-level cost of the V-cycle below level l (eager launches) at 512^3."""
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
def t(fn, reps=20):
    for _ in range(3): fn()
    s.synchronize(); a.record(s)
    for _ in range(reps): fn()
    b.record(s); s.synchronize()
    return a.elapsed_time(b) / reps
prev = None
res = []
for l in range(M.num_levels):
    ms = t(lambda: sf.sf_vcycle(M.handle, l), 5 if l == 0 else 50)
    res.append(ms)
for l, ms in enumerate(res):
    own = ms - (res[l + 1] if l + 1 < len(res) else 0.0)
    print(f"level {l} ({n >> l}^3): V(l) {ms*1e3:9.1f} us, this level alone {own*1e3:9.1f} us")
st, cyc, hist = M.solve(True, 1e-10, 50)
print(f"graph solve {t(lambda: M.solve(True, 1e-10, 50), 3):.2f} ms, {cyc} cycles")
