"""A/B of the residual_restrict kernels (SF_RR_ZS=0: one pass per launch-chunk,
1/2/3: persistent z-streamed with 4/6/8 min CTAs per SM).  Prints the time of
pair + residual_restrict minus the plain pair, a V-cycle and the solve, and a
hash of the restricted coarse field (bit-identity across variants).
    SF_RR_ZS=<v> python scripts/rr_zs_ab.py [n ...]"""
import hashlib
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def timed(s, fn, reps):
    for _ in range(2):
        fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


v = os.environ.get("SF_RR_ZS", "1")
for n in [int(a) for a in sys.argv[1:]] or [256, 512]:
    L = sf.Level(n, n, n, 1.0 / n)
    C = sf.Level(n // 2, n // 2, n // 2, 2.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    s = L.stream
    reps = 20 if n <= 256 else 10
    t_pair = timed(s, lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED), reps)
    t_both = timed(s, lambda: sf.sf_smooth_residual_restrict(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F), reps)
    host = C.download(sf.SF_F)
    h = hashlib.sha1(host.tobytes()).hexdigest()[:12]
    rr = t_both - t_pair
    print(f"SF_RR_ZS={v} n={n} pair {t_pair:.4f} ms  residual_restrict {rr:.4f} ms "
          f"({49 * n**3 / rr / 1e6:.0f} GB/s on 49 B/cell)  coarse hash {h}", flush=True)
    del C, L
    torch.cuda.empty_cache()
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0)
    t_v = timed(L.stream, lambda: M.vcycle(0), 5 if n >= 512 else 10)
    st, cyc, hist = M.solve(True, 1e-10, 50)
    t_s = timed(L.stream, lambda: M.solve(True, 1e-10, 50), 3)
    print(f"SF_RR_ZS={v} n={n} V-cycle {t_v:.3f} ms  solve {t_s:.2f} ms cycles {cyc} relres {hist[-1]:.3e}",
          flush=True)
    del M, L
    torch.cuda.empty_cache()
