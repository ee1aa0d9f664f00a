"""Time the fused pair + delta-form residual + restriction (gsrb_rr.cu) against the plain fused
pair, and a V-cycle with and without it.   python scripts/rr_time.py [n ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def timed(s, fn, reps):
    fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


for n in [int(v) for v in sys.argv[1:]] or [256, 512]:
    L = sf.Level(n, n, n, 1.0 / n)
    C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    s = L.stream
    reps = 20 if n <= 256 else 10
    t_pair = timed(s, lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED), reps)
    os.environ["SF_RRF_CELLS"] = "0"
    t_rr = timed(s, lambda: sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F), reps)
    print(f"n={n} pair {t_pair:.4f} ms  pair+res+restrict {t_rr:.4f} ms  extra {t_rr - t_pair:.4f} ms "
          f"(alg 64 B/cell: pair {64 * n**3 / t_pair / 1e6:.0f} GB/s)")
    del C, L
    torch.cuda.empty_cache()
    for off in ("1", ""):
        os.environ["SF_RRF"] = "0" if off else "1"
        L = sf.Level(n, n, n, 1.0 / n)
        sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
        M = sf.MG(L, 1.0, 1.0)
        t_v = timed(L.stream, lambda: M.vcycle(0), 3 if n >= 512 else 10)
        print(f"n={n} V-cycle ({'separate residual_restrict' if off else 'fused rr'}): {t_v:.3f} ms")
        del M, L
        torch.cuda.empty_cache()
os.environ.pop("SF_RRF", None); os.environ.pop("SF_RRF_CELLS", None)
