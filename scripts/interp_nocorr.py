"""P0-fused pair on the 32x16 build vs plain pairs at n^3 (event-timed back to
back); run with SF_LIB=<measurement build> to compare builds.
    python scripts/interp_nocorr.py [n]"""
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
out = []
for rep in range(2):
    os.environ.pop("SF_GSRB_W4", None)
    out.append(f"plain(32x8/3) {t(plain):.4f}")
    os.environ["SF_GSRB_W4"] = "0"
    out.append(f"plain(32x16) {t(plain):.4f}")
    os.environ.pop("SF_GSRB_W4", None)
    out.append(f"interp(32x16) {t(interp):.4f}")
print(os.environ.get("SF_LIB", "shipped"), f"n={n}", " ".join(out), flush=True)
