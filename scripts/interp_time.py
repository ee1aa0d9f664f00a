"""P0-fused pair (sf_interpolate_smooth) vs the plain fused pair at n^3, both
builds of the P0-fused variant (SF_INTERP_T32=1: 32x16 / 5-deep, =0: 32x8 /
3 CTAs per SM), event-timed back to back.
    python scripts/interp_time.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
L = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n, stream=L.stream)
s = L.stream


def t(fn, reps=20):
    for _ in range(3):
        fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


plain = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)  # noqa: E731
interp = lambda: sf.sf_interpolate_smooth(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_U)  # noqa: E731
res = {}
for rep in range(2):
    res["plain"] = t(plain)
    for b in ("1", "0"):
        os.environ["SF_INTERP_T32"] = b
        res[f"interp_t32={b}"] = t(interp)
print(f"n={n} " + "  ".join(f"{k} {v:.4f} ms" for k, v in res.items()), flush=True)
