"""The fused pair under sustained load (the power-capped regime of the solve):
n^3 plain pairs back to back for ~2 s, the last 300 event-timed, SM clock
sampled with NVML during them.  usage: python scripts/pair_sustained.py [n]"""
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
s = L.stream
f = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)  # noqa: E731
clk = []
stop = False


def sampler():
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
    while not stop:
        clk.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
        time.sleep(0.02)


for _ in range(1200):
    f()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
th = threading.Thread(target=sampler)
a.record(s)
for _ in range(300):
    f()
b.record(s)
th.start()
s.synchronize()
stop = True
th.join()
ms = a.elapsed_time(b) / 300
clk.sort()
print(f"n={n} sustained plain pair {ms:.4f} ms ({56 * n**3 / ms / 1e6:.0f} GB/s on 56 B, "
      f"{64 * n**3 / ms / 1e6:.0f} on 64 B)  SM clock median {clk[len(clk) // 2] if clk else 'n/a'} MHz",
      flush=True)
