import os, sys
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_ipps_zhangdmwbf17_b200 import sf
for n in (64, 128):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    s = L.stream
    res = {}
    for name, kind in (("fused x2", sf.SF_SMOOTH_FUSED), ("twopair", sf.SF_SMOOTH_FUSED2)):
        for _ in range(3):
            sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
        s.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        for _ in range(100):
            sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, kind)
        b.record(s)
        s.synchronize()
        res[name] = a.elapsed_time(b) / 100 * 1e3
    print(n, {k: round(v, 2) for k, v in res.items()}, "us per 2 pairs", flush=True)
    L.close()
