"""Small end-to-end workload for compute-sanitizer: fused pair variants (plain,
check-fused, P0-fused), colour sweeps, residual/restriction, CC kernels, and a
32^3 / 64^3 solve (graphs off so every launch is visible)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhangdmwbf17_b200 import inputs as I, sf  # noqa: E402

for n, parts in ((32, 1), (64, 1), (64, 2)):
    comm = sf.Comm.local(parts) if parts > 1 else None
    L = sf.Level(n, n, n, 1.0 / n, comm=comm)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    M = sf.MG(L, 1.0, 1.0, use_graph=0, agglom_min_planes=4)
    st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, max_cycles=3, raise_on_error=False)
    sf.sf_apply_laplacian(L.handle, sf.SF_R, sf.SF_U)
    sf.sf_jacobi(L.handle, sf.SF_TMP, sf.SF_U, sf.SF_F)
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 1, sf.SF_SMOOTH_COLOUR)
    sf.sf_apply_bc(L.handle, sf.SF_U)
    sf.sf_sync(L.handle)
    print("ok", n, parts, cyc, flush=True)
    M.close(); L.close()
    if comm:
        comm.close()

# halo exchange beside the interior chunks (2 parts x 24 planes), the pair +
# residual + restriction (delta form, SF_RRF_CELLS=0 forces it) and the 32x16 build (SF_GSRB_W4=0)
os.environ["SF_HALO_OVERLAP"] = "1"   # force the split (2-plane boundary chunks)
comm = sf.Comm.local(2)
L = sf.Level(64, 32, 48, 1.0 / 64, comm=comm)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 2, sf.SF_SMOOTH_FUSED)
sf.sf_sync(L.handle)
print("ok overlap", flush=True)
L.close()
comm.close()
os.environ["SF_RRF_CELLS"] = "0"
F = sf.Level(64, 32, 12, 1.0 / 64)
C = sf.Level(32, 16, 6, 2.0 / 64)
sf.sf_init_problem(F.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(F.handle, 1.0, 1.0)
sf.sf_smooth_residual_restrict(F.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F)
sf.sf_sync(F.handle)
print("ok rr", flush=True)
F.close(); C.close()

# graphs on: the device-resident solve loop (WHILE node) and PDL launches
os.environ.pop("SF_RRF_CELLS", None)
L = sf.Level(32, 32, 32, 1.0 / 32)
sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
M = sf.MG(L, 1.0, 1.0)
st, cyc, hist = M.solve(fcycle=True, rtol=1e-10, raise_on_error=False)
sf.sf_sync(L.handle)
print("ok graph solve", cyc, flush=True)
M.close(); L.close()

# r02 kernels: NEXT-1 two-pair smoother (4 chunk depths incl. ragged ones),
# sf_interpolate_smooth on the 32x16 P0-fused build, the persistent residual +
# restriction with forced multi-item chunking; the coarse cluster V-cycle
# runs inside every solve above (levels <= 16^3)
for dep in ("0", "1", "3", "7"):
    if dep != "0":
        os.environ["SF_TWOPAIR_DEPTH"] = dep
    L = sf.Level(64, 32, 20, 1.0 / 64)
    sf.sf_init_problem(L.handle, 1, 1.0, 1.0, 1)
    sf.sf_rebuild_operator(L.handle, 1.0, 1.0)
    sf.sf_smooth_gsrb(L.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, 3, sf.SF_SMOOTH_FUSED2)
    sf.sf_sync(L.handle)
    L.close()
os.environ.pop("SF_TWOPAIR_DEPTH", None)
print("ok twopair", flush=True)
os.environ["SF_INTERP_T32_CELLS"] = "0"
os.environ["SF_RRZS_DEPTH"] = "3"
os.environ["SF_RRZS_GRID"] = "5"
F = sf.Level(64, 32, 24, 1.0 / 64)
C = sf.Level(32, 16, 12, 2.0 / 64)
sf.sf_init_problem(F.handle, 1, 1.0, 1.0, 1)
sf.sf_rebuild_operator(F.handle, 1.0, 1.0)
sf.sf_interpolate_smooth(F.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_U)
sf.sf_smooth_residual_restrict(F.handle, sf.SF_U, sf.SF_F, 1.0, 1.0, C.handle, sf.SF_F)
sf.sf_sync(F.handle)
print("ok interp t32 / rr chunks", flush=True)
F.close(); C.close()
