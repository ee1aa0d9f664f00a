"""Profiling driver: fused / colour GSRB pairs (and residual) on one level.
    python scripts/prof_gsrb.py [n] [pairs] [kind: fused|colour]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
pairs = int(sys.argv[2]) if len(sys.argv) > 2 else 4
kind = sf.SF_SMOOTH_FUSED if (sys.argv[3] if len(sys.argv) > 3 else "fused") == "fused" else sf.SF_SMOOTH_COLOUR
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
for _ in range(pairs):
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, kind)
sf.sf_residual(L.handle, sf.SF_R, sf.SF_U, sf.SF_F, 1.0, 1.0)
L.stream.synchronize()
s = L.stream
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(s)
for _ in range(10):
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, kind)
b.record(s)
s.synchronize()
ms = a.elapsed_time(b) / 10
print(f"n={n} kind={kind} ms/pair={ms:.4f} alg GB/s={64 * n**3 / ms / 1e6:.1f}")
