"""bench.py's e2e sequence at 512^3 with the phase times of sf_solve_stream:
odd public smooths first (remaps U/TMP under the cached graphs), then the
streamed solve (2 warm-up, 5 timed right-hand sides) and the serial
upload-solve-download, each u checked against a standalone solve.

    python scripts/e2e_phases.py [n]
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
for _ in range(3):
    M.solve(True, 1e-10, 50)
for _ in range(23):
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
hf = torch.empty(L.host_shape(sf.SF_F), dtype=torch.float64, pin_memory=True)
hu = [torch.empty(L.host_shape(sf.SF_U), dtype=torch.float64, pin_memory=True) for _ in range(2)]
L.download(sf.SF_F, hf.numpy())
M.solve(True, 1e-10, 50)
uref = L.download(sf.SF_U)
M.solve_stream([hf] * 2, hu)
print("warm-up stats", sf.sf_solve_stream_stats(M.handle), flush=True)
torch.cuda.synchronize()
t0 = time.perf_counter()
M.solve_stream([hf] * 5, [hu[k % 2] for k in range(5)])
te = (time.perf_counter() - t0) / 5
print(f"streamed ms/rhs {te * 1e3:.2f}; stats (h2d, solve, d2h, wall) "
      f"{tuple(round(v, 2) for v in sf.sf_solve_stream_stats(M.handle))}", flush=True)
print("streamed u == standalone u:", bool(np.array_equal(hu[0].numpy(), uref)), flush=True)
t1 = time.perf_counter()
for _ in range(2):
    sf.sf_level_upload(L.handle, sf.SF_F, hf.data_ptr())
    sf.sf_solve(M.handle, True, 1e-10, 50)
    sf.sf_level_download(L.handle, sf.SF_U, hu[0].data_ptr())
ts = (time.perf_counter() - t1) / 2
print(f"serial ms/rhs {ts * 1e3:.2f}", flush=True)
