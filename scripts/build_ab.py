"""Fused-pair builds A/B (SF_GSRB_BUILD): the pair alone at 256^3 / 512^3 and
bit-identity of the results against the default build.
    python scripts/build_ab.py build [build ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I, sf  # noqa: E402


def run(build, n, reps=20):
    if build:
        os.environ["SF_GSRB_BUILD"] = build
    else:
        os.environ.pop("SF_GSRB_BUILD", None)
    L = sf.Level(n, n, n, 1.0 / n)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    s = L.stream
    f = lambda: sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_FUSED)  # noqa: E731
    for _ in range(3):
        f()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        f()
    b.record(s)
    s.synchronize()
    ms = a.elapsed_time(b) / reps
    L.close()
    return ms


def bits(build):
    if build:
        os.environ["SF_GSRB_BUILD"] = build
    else:
        os.environ.pop("SF_GSRB_BUILD", None)
    shape = (40, 32, 64)
    nz, ny, nx = shape
    L = sf.Level(nx, ny, nz, 1.0 / 64)
    L.set_coeffs(*I.random_coeffs(nx, ny, nz, 3))
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    L.upload(sf.SF_U, I.random_field(shape, 0))
    L.upload(sf.SF_F, I.random_field(shape, 1))
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 3, sf.SF_SMOOTH_FUSED)
    u = L.download(sf.SF_U)
    L.close()
    return u


ref = bits(None)
for bld in sys.argv[1:]:
    print(f"{bld}: bit-identical to default: {np.array_equal(bits(bld), ref)}", flush=True)
for n in (256, 512):
    r = {b: run(b, n) for b in [None] + sys.argv[1:] + [None] + sys.argv[1:]}
    print(f"n={n} " + "  ".join(f"{b or 'default'} {v:.4f} ms" for b, v in r.items()), flush=True)
