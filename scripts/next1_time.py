"""NEXT-1 timing: one whole smooth (2 RB pairs) as one temporally blocked pass
(SF_SMOOTH_FUSED2) vs two colour-fused pairs, same level, same session.
    python scripts/next1_time.py [n ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def ms(L, kind, reps=20):
    s = L.stream
    f = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)  # noqa: E731
    for _ in range(3):
        f()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        f()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


for n in [int(v) for v in sys.argv[1:]] or [128, 256, 512]:
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    r = {k: ms(L, k) for k in (sf.SF_SMOOTH_FUSED, sf.SF_SMOOTH_FUSED2, sf.SF_SMOOTH_FUSED,
                              sf.SF_SMOOTH_FUSED2)}
    t1, t2 = r[sf.SF_SMOOTH_FUSED], r[sf.SF_SMOOTH_FUSED2]
    c = n**3
    print(f"n={n} smooth (2 pairs): two fused pairs {t1:.4f} ms | one two-pair pass {t2:.4f} ms "
          f"(x{t1 / t2:.2f}); two-pair pass on the 56 B one-pass basis {56 * c / t2 / 1e6:.0f} GB/s, "
          f"on the 2 x 56 B two-pass basis {112 * c / t2 / 1e6:.0f} GB/s", flush=True)
    L.close()
