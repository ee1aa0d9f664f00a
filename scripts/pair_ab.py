"""The fused pair alone at 256^3 / 512^3 with the library under test and a
second build (SF_LIB_B), alternating in separate processes.
    SF_LIB_B=path python scripts/pair_ab.py"""
import os
import subprocess
import sys

code = r'''
import os, sys, torch
sys.path.insert(0, ".")
from paper_conf_ipps_zhangdmwbf17_b200 import sf
for n in (256, 512):
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    s = L.stream
    f = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)
    for _ in range(5): f()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(30): f()
    b.record(s); s.synchronize()
    print(n, round(a.elapsed_time(b) / 30, 4), end="  ")
    L.close()
print()
'''
for rep in range(2):
    for lib in ("", os.environ.get("SF_LIB_B", "")):
        env = dict(os.environ)
        if lib:
            env["SF_LIB"] = lib
        else:
            env.pop("SF_LIB", None)
        r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env)
        print(lib or "default", r.stdout.strip(), r.stderr[-300:] if r.returncode else "", flush=True)
