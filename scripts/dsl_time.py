"""Time the generic stencil engine's JIT kernels at n^3 vs the hand-written ones."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhangdmwbf17_b200 import sf, stencil as SD
n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
G = sf.Level(n, n, n, 1.0 / n)
sf.sf_init_problem(G.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(G.handle, 1.0, 1.0)
s = G.stream
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def per_call(fn, reps=30):
    for _ in range(3):
        fn()
    s.synchronize(); a.record(s)
    for _ in range(reps):
        fn()
    b.record(s); s.synchronize()
    return a.elapsed_time(b) / reps
pair = SD.hpgmg_gsrb_pair(1.0, 1.0, 1.0 / n).compile()
op = SD.hpgmg_apply_op(1.0, 1.0, 1.0 / n).compile()
red, black = SD.red_black_domains()
only_red = SD.Stencil(SD.gsrb_update(1.0, 1.0, 1.0 / n), "u", red).compile()
bc = SD.StencilGroup(SD.dirichlet_faces("u")).compile()
t = {"dsl_pair": per_call(lambda: pair(G)), "dsl_apply_op": per_call(lambda: op(G)),
     "dsl_red_only": per_call(lambda: only_red(G)), "dsl_bc6": per_call(lambda: bc(G)),
     "hw_colour_pair": per_call(lambda: sf.sf_smooth_gsrb(G.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_COLOUR)),
     "hw_apply_op": per_call(lambda: sf.sf_apply_op(G.handle, sf.SF_R, sf.SF_U, 1.0, 1.0))}
for k, v in t.items():
    print(f"{k:16s} {v*1e3:8.1f} us")
