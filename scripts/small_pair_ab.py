"""Fused pair time per launch at small levels (50 pairs per call, CUDA events)
and the 64^3 V-solve / 128^3 F+V solve, in this process's environment (run it
once per SF_GSRB_* setting to compare builds / chunk depths).
    python scripts/small_pair_ab.py [label]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

label = sys.argv[1] if len(sys.argv) > 1 else ""
out = []
for n in (64, 128):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    s = L.stream
    for _ in range(2):
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 50, sf.SF_SMOOTH_FUSED)
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(4):
        sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 50, sf.SF_SMOOTH_FUSED)
    b.record(s)
    s.synchronize()
    out.append(f"pair {n}^3 {a.elapsed_time(b) / 200 * 1e3:.2f} us")
    L.close()
for n, fc in ((64, False), (128, True)):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    z = np.zeros((n, n, n))
    ts = []
    for r in range(23):
        L.upload(sf.SF_U, z)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st, cyc, hist = M.solve(fc, 1e-10, 50)
        if r >= 3:
            ts.append(time.perf_counter() - t0)
    out.append(f"solve {n}^3 {'F+V' if fc else 'V'} {min(ts) * 1e3:.3f} ms ({cyc} cycles, "
               f"{n**3 / min(ts) / 1e9:.3f} GDOF/s)")
    M.close()
    L.close()
print(label, "|", "; ".join(out), flush=True)
