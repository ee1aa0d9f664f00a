"""Probe the e2e pieces at 512^3: H2D/D2H of one field, pack/unpack, solve, stream."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhangdmwbf17_b200 import sf
n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
hf = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
hu = [torch.empty((n, n, n), dtype=torch.float64, pin_memory=True) for _ in range(2)]
L.download(sf.SF_F, hf.numpy())
def wall(fn, reps=3):
    fn(); torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) / reps * 1e3
print("upload f  ms", wall(lambda: (sf.sf_level_upload(L.handle, sf.SF_F, hf.data_ptr()), sf.sf_sync(L.handle))))
print("download u ms", wall(lambda: sf.sf_level_download(L.handle, sf.SF_U, hu[0].data_ptr())))
print("solve ms", wall(lambda: M.solve(True, 1e-10, 50)))
print("stream x5 ms/step", wall(lambda: M.solve_stream([hf] * 5, [hu[k % 2] for k in range(5)]), 1) / 5)
