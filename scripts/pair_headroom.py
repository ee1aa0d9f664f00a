"""SM-side headroom of the colour-fused RB pair: the same launch with every
operand plane aliased into 4 L2-resident planes (SF_DBG_ZMASK=3; values
meaningless) against the normal HBM-streaming launch.

    python scripts/pair_headroom.py [n ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import sf  # noqa: E402


def pair_ms(L, reps=30):
    s = L.stream
    f = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)  # noqa: E731
    for _ in range(5):
        f()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        f()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


for n in [int(v) for v in sys.argv[1:]] or [256, 512]:
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    res = {}
    for mask in ("0", "3"):
        os.environ["SF_DBG_ZMASK"] = mask
        res[mask] = pair_ms(L)
    os.environ["SF_DBG_ZMASK"] = "0"
    cells = n**3
    print(f"n={n} hbm {res['0']:.4f} ms ({56 * cells / res['0'] / 1e6:.0f} GB/s on 56 B)  "
          f"l2-resident {res['3']:.4f} ms  headroom x{res['0'] / res['3']:.2f}", flush=True)
    L.close()
