import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhangdmwbf17_b200 import sf
n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
G = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(G.handle, 1, 1.0, 1.0, 1)
s = G.stream
def t(fn, reps=50):
    for _ in range(5): fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps): fn()
    b.record(s); s.synchronize()
    return a.elapsed_time(b) / reps
c = n**3
m1 = t(lambda: sf.sf_apply_laplacian(G.handle, sf.SF_R, sf.SF_U))
m2 = t(lambda: sf.sf_jacobi(G.handle, sf.SF_R, sf.SF_U, sf.SF_F, 2 / 3))
print(f"n={n} lap {m1:.4f} ms {16*c/m1/1e6:.0f} GB/s | jacobi {m2:.4f} ms {24*c/m2/1e6:.0f} GB/s")
