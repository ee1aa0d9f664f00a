"""Thin ctypes binding of libsf (include/sf.h).  Argument marshalling only.

Every function named ``sf_*`` here calls the C entry point of the same name;
the small classes (Comm, Level, MG) only hold handles, the torch-owned device
buffer and stream, and convert numpy host arrays.  All arithmetic of the
method runs in libsf's CUDA kernels.  There is no CPU fallback: if libsf.so is
missing or no sm_100 device is present, the calls raise.

PyTorch is used for device memory (one uint8 tensor per level, passed to
sf_level_create as the caller-owned buffer) and streams
(``torch.cuda.Stream``), and torch.distributed broadcasts the NCCL id.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SF_LIB: A/B timing of another build of the same library (scripts/ab_lib.sh)
LIB_PATH = os.environ.get("SF_LIB") or os.path.join(_HERE, "libsf.so")

# enums (include/sf.h)
SF_OK, SF_ERR_INVALID, SF_ERR_SHAPE, SF_ERR_OOM, SF_ERR_CUDA, SF_ERR_NCCL = range(6)
SF_ERR_NOT_CONVERGED, SF_ERR_NUMERIC = 6, 7
(SF_U, SF_F, SF_R, SF_TMP, SF_ALPHA, SF_BETA_I, SF_BETA_J, SF_BETA_K, SF_DINV) = range(9)
SF_NFIELDS = 9
SF_RESTRICT_CELL, SF_RESTRICT_FACE_I, SF_RESTRICT_FACE_J, SF_RESTRICT_FACE_K = range(4)
SF_INTERP_P0, SF_INTERP_PL = 0, 1
SF_NORM_MAX, SF_NORM_L2 = 0, 1
SF_SMOOTH_AUTO, SF_SMOOTH_COLOUR, SF_SMOOTH_FUSED, SF_SMOOTH_CHEBY, SF_SMOOTH_FUSED2 = 0, 1, 2, 3, 4

FIELD_IDS = {"u": SF_U, "f": SF_F, "r": SF_R, "tmp": SF_TMP, "alpha": SF_ALPHA,
             "beta_i": SF_BETA_I, "beta_j": SF_BETA_J, "beta_k": SF_BETA_K, "dinv": SF_DINV}

EXPORTS = [
    "sf_mg_opts_default", "sf_last_error", "sf_version", "sf_comm_create_local",
    "sf_get_unique_id", "sf_comm_create_nccl", "sf_comm_destroy", "sf_comm_info",
    "sf_level_bytes_needed", "sf_level_create", "sf_level_destroy", "sf_level_upload",
    "sf_level_download", "sf_level_zero", "sf_level_field_ptr", "sf_init_problem", "sf_rebuild_operator",
    "sf_apply_bc", "sf_apply_op", "sf_smooth_gsrb", "sf_residual", "sf_restrict",
    "sf_interpolate", "sf_norm", "sf_sync", "sf_mg_create", "sf_mg_num_levels", "sf_mg_level",
    "sf_vcycle", "sf_fcycle", "sf_solve", "sf_mg_destroy", "sf_launch_count", "sf_mg_plan",
    "sf_apply_laplacian", "sf_jacobi", "sf_smooth_chebyshev", "sf_lambda_max",
    "sf_comm_create_hostipc", "sf_stencil_compile", "sf_stencil_source", "sf_stencil_apply",
    "sf_stencil_plan", "sf_stencil_phases", "sf_stencil_destroy", "sf_solve_stream",
    "sf_comm_create_p2p", "sf_smooth_residual_restrict", "sf_level_pair_timing",
    "sf_interpolate_smooth", "sf_comm_check", "sf_solve_stream_stats",
    "sf_level_pair_timing_variants", "sf_level_pair_timing_rrf",
]


class SfError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"libsf status {status}: {msg}")
        self.status = status


class MgOpts(C.Structure):
    _fields_ = [("pre_pairs", C.c_int), ("post_pairs", C.c_int), ("vcycle_interp", C.c_int),
                ("fcycle_interp", C.c_int), ("agglom_min_planes", C.c_int),
                ("max_cycles", C.c_int), ("use_graph", C.c_int), ("smoother", C.c_int),
                ("rtol", C.c_double), ("cheby_degree", C.c_int)]


_lib = None
_vp, _d, _i = C.c_void_p, C.c_double, C.c_int
_P = C.POINTER(C.c_double)
# generic stencil IR (include/sf.h, NEXT-4)
SF_SX_CONST, SF_SX_READ, SF_SX_ADD, SF_SX_SUB, SF_SX_MUL, SF_SX_DIV, SF_SX_NEG = range(7)


class SxNode(C.Structure):
    _fields_ = [("op", C.c_int), ("a", C.c_int), ("b", C.c_int), ("mesh", C.c_int),
                ("src", C.c_int), ("off", C.c_int * 3), ("mul", C.c_int * 3),
                ("div", C.c_int * 3), ("pre", C.c_int * 3), ("value", C.c_double)]


class SfRect(C.Structure):
    _fields_ = [("lo", C.c_int * 3), ("hi", C.c_int * 3), ("stride", C.c_int * 3)]


class StencilDesc(C.Structure):
    _fields_ = [("n_nodes", C.c_int), ("nodes", C.POINTER(SxNode)), ("root", C.c_int),
                ("out_mesh", C.c_int), ("n_rects", C.c_int), ("rects", C.POINTER(SfRect))]


# int (*)(const void* send, size_t nbytes, void* recv, void* user)
HOST_ALLGATHER = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)


def lib():
    """Load libsf.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                           "`python -m paper_conf_ipps_zhangdmwbf17_b200.build` (no CPU fallback)")
    L = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
    sig = {
        "sf_mg_opts_default": (None, [C.POINTER(MgOpts)]),
        "sf_last_error": (C.c_char_p, []),
        "sf_version": (C.c_char_p, []),
        "sf_comm_create_local": (_i, [C.POINTER(_vp), _i]),
        "sf_get_unique_id": (_i, [C.c_char_p]),
        "sf_comm_create_nccl": (_i, [C.POINTER(_vp), C.c_char_p, _i, _i]),
        "sf_comm_create_hostipc": (_i, [C.POINTER(_vp), _i, _i, HOST_ALLGATHER, _vp]),
        "sf_comm_create_p2p": (_i, [C.POINTER(_vp), _i, _i, HOST_ALLGATHER, _vp]),
        "sf_comm_destroy": (_i, [_vp]),
        "sf_stencil_compile": (_i, [C.POINTER(_vp), C.POINTER(StencilDesc), _i]),
        "sf_stencil_source": (_i, [_vp, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]),
        "sf_stencil_apply": (_i, [_vp, _vp, _vp]),
        "sf_stencil_plan": (_i, [_vp, _i, _i, _i, _i, C.POINTER(_i)]),
        "sf_stencil_phases": (_i, [_vp, C.POINTER(_i)]),
        "sf_stencil_destroy": (_i, [_vp]),
        "sf_comm_info": (_i, [_vp, C.POINTER(_i), C.POINTER(_i), C.POINTER(_i)]),
        "sf_level_bytes_needed": (_i, [_i, _i, _i, _vp, C.POINTER(C.c_size_t)]),
        "sf_level_create": (_i, [C.POINTER(_vp), _i, _i, _i, _d, _vp, _vp, _vp, C.c_size_t]),
        "sf_level_destroy": (_i, [_vp]),
        "sf_level_upload": (_i, [_vp, _i, _vp]),
        "sf_level_download": (_i, [_vp, _i, _vp]),
        "sf_level_zero": (_i, [_vp, _i]),
        "sf_level_field_ptr": (_i, [_vp, _i, _i, C.POINTER(_P), C.POINTER(C.c_long)]),
        "sf_init_problem": (_i, [_vp, _i, _d, _d, _i]),
        "sf_rebuild_operator": (_i, [_vp, _d, _d]),
        "sf_apply_bc": (_i, [_vp, _i]),
        "sf_apply_op": (_i, [_vp, _i, _i, _d, _d]),
        "sf_smooth_gsrb": (_i, [_vp, _i, _i, _d, _d, _i, _i]),
        "sf_residual": (_i, [_vp, _i, _i, _i, _d, _d]),
        "sf_smooth_residual_restrict": (_i, [_vp, _i, _i, _d, _d, _vp, _i]),
        "sf_interpolate_smooth": (_i, [_vp, _i, _i, _d, _d, _vp, _i]),
        "sf_comm_check": (_i, [_vp, _vp]),
        "sf_level_pair_timing_variants": (_i, [_vp, C.POINTER(C.c_double), C.POINTER(C.c_longlong)]),
        "sf_level_pair_timing_rrf": (_i, [_vp, C.POINTER(C.c_double), C.POINTER(C.c_longlong)]),
        "sf_solve_stream_stats": (_i, [_vp, C.POINTER(C.c_double)]),
        "sf_apply_laplacian": (_i, [_vp, _i, _i]),
        "sf_jacobi": (_i, [_vp, _i, _i, _i, _d]),
        "sf_smooth_chebyshev": (_i, [_vp, _i, _i, _d, _d, _i, _d, _d]),
        "sf_lambda_max": (_i, [_vp, _i, _d, _d, _i, _i, _P]),
        "sf_restrict": (_i, [_vp, _i, _vp, _i, _i]),
        "sf_interpolate": (_i, [_vp, _i, _d, _vp, _i, _i]),
        "sf_norm": (_i, [_vp, _i, _i, _P]),
        "sf_sync": (_i, [_vp]),
        "sf_level_pair_timing": (_i, [_vp, _i, _P, C.POINTER(C.c_longlong)]),
        "sf_mg_create": (_i, [C.POINTER(_vp), _vp, _d, _d, C.POINTER(MgOpts)]),
        "sf_mg_num_levels": (_i, [_vp, C.POINTER(_i)]),
        "sf_mg_level": (_i, [_vp, _i, C.POINTER(_vp)]),
        "sf_vcycle": (_i, [_vp, _i]),
        "sf_fcycle": (_i, [_vp]),
        "sf_solve": (_i, [_vp, _i, _d, _i, C.POINTER(_i), _P]),
        "sf_mg_destroy": (_i, [_vp]),
        "sf_solve_stream": (_i, [_vp, _i, _d, _i, _i, C.POINTER(_vp), C.POINTER(_vp),
                                 C.POINTER(_i)]),
        "sf_launch_count": (_i, [C.POINTER(C.c_longlong), _i]),
        "sf_mg_plan": (_i, [_i, _i, _i, _i, _i, _i, C.POINTER(_i), C.POINTER(_i), C.POINTER(_i)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype, f.argtypes = res, args
    _lib = L
    return L


def _check(status):
    if status != SF_OK:
        raise SfError(status, lib().sf_last_error().decode(errors="replace"))
    return status


# ------------------------------------------------------------ C-ABI mirrors
def sf_version():
    return lib().sf_version().decode()


def sf_mg_opts_default():
    o = MgOpts()
    lib().sf_mg_opts_default(C.byref(o))
    return o


def sf_comm_create_local(nparts):
    h = _vp()
    _check(lib().sf_comm_create_local(C.byref(h), int(nparts)))
    return h


def sf_get_unique_id():
    buf = C.create_string_buffer(128)
    _check(lib().sf_get_unique_id(buf))
    return buf.raw


def sf_comm_create_nccl(uid, nranks, rank):
    h = _vp()
    _check(lib().sf_comm_create_nccl(C.byref(h), uid, int(nranks), int(rank)))
    return h


def sf_comm_create_hostipc(nranks, rank, allgather_cb):
    """allgather_cb must be a HOST_ALLGATHER the caller keeps alive."""
    h = _vp()
    _check(lib().sf_comm_create_hostipc(C.byref(h), int(nranks), int(rank), allgather_cb, None))
    return h


def sf_stencil_compile(stencils):
    """stencils: list of (nodes, root, out_mesh, rects); nodes = list of dicts with
    SxNode fields, rects = list of (lo, hi, stride) 3-tuples (x, y, z)."""
    descs = (StencilDesc * len(stencils))()
    keep = []
    for d, (nodes, root, out, rects) in zip(descs, stencils):
        na = (SxNode * len(nodes))()
        for x, n in zip(na, nodes):
            x.op = n["op"]
            x.a, x.b = n.get("a", 0), n.get("b", 0)
            x.mesh, x.src = n.get("mesh", 0), n.get("src", 0)
            for k, dflt in (("off", 0), ("mul", 1), ("div", 1), ("pre", 0)):
                getattr(x, k)[:] = list(n.get(k, (dflt,) * 3))
            x.value = float(n.get("value", 0.0))
        ra = (SfRect * len(rects))()
        for x, (lo, hi, st) in zip(ra, rects):
            x.lo[:], x.hi[:], x.stride[:] = list(lo), list(hi), list(st)
        keep += [na, ra]
        d.n_nodes, d.nodes, d.root, d.out_mesh = len(nodes), na, int(root), int(out)
        d.n_rects, d.rects = len(rects), ra
    h = _vp()
    _check(lib().sf_stencil_compile(C.byref(h), descs, len(stencils)))
    return h


def sf_stencil_source(h):
    n = C.c_size_t()
    _check(lib().sf_stencil_source(h, None, 0, C.byref(n)))
    buf = C.create_string_buffer(n.value + 1)
    _check(lib().sf_stencil_source(h, buf, n.value + 1, None))
    return buf.value.decode()


def sf_stencil_apply(h, level, src=None):
    _check(lib().sf_stencil_apply(h, level, src))


def sf_stencil_plan(h, gnx, gny, gnz, src_is_output=True):
    n = _i()
    _check(lib().sf_stencil_plan(h, int(gnx), int(gny), int(gnz), int(bool(src_is_output)),
                                 C.byref(n)))
    return n.value


def sf_stencil_phases(h):
    n = _i()
    _check(lib().sf_stencil_phases(h, C.byref(n)))
    return n.value


def sf_stencil_destroy(h):
    _check(lib().sf_stencil_destroy(h))


def sf_comm_create_p2p(nranks, rank, allgather_cb):
    """allgather_cb must be a HOST_ALLGATHER the caller keeps alive."""
    h = _vp()
    _check(lib().sf_comm_create_p2p(C.byref(h), int(nranks), int(rank), allgather_cb, None))
    return h


def sf_comm_destroy(h):
    _check(lib().sf_comm_destroy(h))


def sf_level_bytes_needed(gnx, gny, gnz, comm=None):
    n = C.c_size_t()
    _check(lib().sf_level_bytes_needed(gnx, gny, gnz, comm, C.byref(n)))
    return n.value


def sf_level_create(gnx, gny, gnz, h, comm=None, stream=None, dev_buf=None, buf_bytes=0):
    out = _vp()
    _check(lib().sf_level_create(C.byref(out), gnx, gny, gnz, float(h), comm, stream, dev_buf,
                                 buf_bytes))
    return out


def sf_level_destroy(level):
    _check(lib().sf_level_destroy(level))


def sf_level_upload(level, field, host):
    _check(lib().sf_level_upload(level, field, host))


def sf_level_zero(level, field):
    _check(lib().sf_level_zero(level, field))


def sf_level_download(level, field, host):
    _check(lib().sf_level_download(level, field, host))


def sf_level_field_ptr(level, part, field):
    p = _P()
    st = (C.c_long * 3)()
    _check(lib().sf_level_field_ptr(level, part, field, C.byref(p), st))
    return C.cast(p, C.c_void_p).value, tuple(st)


def sf_init_problem(level, problem, a, b, want_rhs=1):
    _check(lib().sf_init_problem(level, problem, float(a), float(b), int(want_rhs)))


def sf_rebuild_operator(level, a, b):
    _check(lib().sf_rebuild_operator(level, float(a), float(b)))


def sf_apply_bc(level, field):
    _check(lib().sf_apply_bc(level, field))


def sf_apply_op(level, out, x, a, b):
    _check(lib().sf_apply_op(level, out, x, float(a), float(b)))


def sf_smooth_gsrb(level, x, rhs, a, b, rb_pairs, kind=SF_SMOOTH_AUTO):
    _check(lib().sf_smooth_gsrb(level, x, rhs, float(a), float(b), int(rb_pairs), int(kind)))


def sf_smooth_residual_restrict(fine, x, rhs, a, b, coarse, c_field):
    _check(lib().sf_smooth_residual_restrict(fine, x, rhs, float(a), float(b), coarse, c_field))


def sf_comm_check(comm, stream=None):
    _check(lib().sf_comm_check(comm, stream))


def sf_interpolate_smooth(fine, x, rhs, a, b, coarse, c_field):
    _check(lib().sf_interpolate_smooth(fine, x, rhs, float(a), float(b), coarse, c_field))


def sf_apply_laplacian(level, out, x):
    _check(lib().sf_apply_laplacian(level, out, x))


def sf_jacobi(level, out, x, f, omega=2.0 / 3.0):
    _check(lib().sf_jacobi(level, out, x, f, float(omega)))


def sf_smooth_chebyshev(level, x, rhs, a, b, degree, lo, hi):
    _check(lib().sf_smooth_chebyshev(level, x, rhs, float(a), float(b), int(degree), float(lo),
                                     float(hi)))


def sf_lambda_max(level, v, a, b, iters=30, start=True):
    out = C.c_double()
    _check(lib().sf_lambda_max(level, v, float(a), float(b), int(iters), int(start), C.byref(out)))
    return out.value


def sf_residual(level, res, x, rhs, a, b):
    _check(lib().sf_residual(level, res, x, rhs, float(a), float(b)))


def sf_restrict(coarse, c_field, fine, f_field, kind=SF_RESTRICT_CELL):
    _check(lib().sf_restrict(coarse, c_field, fine, f_field, kind))


def sf_interpolate(fine, f_field, prescale, coarse, c_field, kind=SF_INTERP_P0):
    _check(lib().sf_interpolate(fine, f_field, float(prescale), coarse, c_field, kind))


def sf_norm(level, field, kind=SF_NORM_MAX):
    out = C.c_double()
    _check(lib().sf_norm(level, field, kind, C.byref(out)))
    return out.value


def sf_sync(level):
    _check(lib().sf_sync(level))


def sf_level_pair_timing_rrf(level):
    """(mean ms, launches) of the fused pair + residual + restriction since the
    last sf_level_pair_timing(op 0) read-out."""
    ms, n = C.c_double(), C.c_longlong()
    _check(lib().sf_level_pair_timing_rrf(level, C.byref(ms), C.byref(n)))
    return ms.value, n.value


def sf_level_pair_timing(level, op):
    """op 1: arm the in-kernel timer of the colour-fused pair on this level;
    op 0: disarm, returns (mean ms per launch, launches since arming)."""
    ms, n = C.c_double(), C.c_longlong()
    _check(lib().sf_level_pair_timing(level, int(op), C.byref(ms), C.byref(n)))
    return ms.value, n.value


def sf_mg_create(level, a, b, opts=None):
    out = _vp()
    _check(lib().sf_mg_create(C.byref(out), level, float(a), float(b),
                              C.byref(opts) if opts is not None else None))
    return out


def sf_mg_num_levels(mg):
    n = _i()
    _check(lib().sf_mg_num_levels(mg, C.byref(n)))
    return n.value


def sf_mg_level(mg, l):
    out = _vp()
    _check(lib().sf_mg_level(mg, l, C.byref(out)))
    return out


def sf_vcycle(mg, l=0):
    _check(lib().sf_vcycle(mg, l))


def sf_fcycle(mg):
    _check(lib().sf_fcycle(mg))


def sf_solve(mg, fcycle=True, rtol=1e-10, max_cycles=50, raise_on_error=True):
    """Returns (status, cycles, history)."""
    cyc = _i()
    hist = (C.c_double * (max_cycles + 1))()
    st = lib().sf_solve(mg, int(fcycle), float(rtol), int(max_cycles), C.byref(cyc), hist)
    if raise_on_error:
        _check(st)
    return st, cyc.value, list(hist[:cyc.value])


def sf_solve_stream(mg, host_f_ptrs, host_u_ptrs, fcycle=True, rtol=1e-10, max_cycles=50):
    """Pipelined multi-RHS solve; pointers are ints (pinned host or device
    addresses).  Returns the cycle count of each solve."""
    n = len(host_f_ptrs)
    if len(host_u_ptrs) != n:
        raise ValueError("one output per right-hand side")
    fa = (_vp * max(n, 1))(*host_f_ptrs)
    ua = (_vp * max(n, 1))(*host_u_ptrs)
    cyc = (_i * max(n, 1))()
    _check(lib().sf_solve_stream(mg, int(fcycle), float(rtol), int(max_cycles), n, fa, ua, cyc))
    return list(cyc[:n])


def sf_mg_destroy(mg):
    _check(lib().sf_mg_destroy(mg))


def sf_level_pair_timing_variants(level):
    """{variant: (mean_ms, pairs)} of the last sf_level_pair_timing read-out."""
    ms = (C.c_double * 4)()
    n = (C.c_longlong * 4)()
    _check(lib().sf_level_pair_timing_variants(level, ms, n))
    return {name: (ms[i], n[i]) for i, name in enumerate(("plain", "resid", "bres", "interp"))}


def sf_solve_stream_stats(mg):
    """(h2d_ms, solve_ms, d2h_ms, wall_ms) per right-hand side of the last
    sf_solve_stream call."""
    out = (C.c_double * 4)()
    _check(lib().sf_solve_stream_stats(mg, out))
    return tuple(out)


def sf_mg_plan(gnx, gny, gnz, nparts=1, agglom_min_planes=8, max_levels=32):
    """Host-only hierarchy plan: [((nx, ny, nz), distributed), ...] finest first."""
    n = _i()
    dims = (_i * (3 * max_levels))()
    dist = (_i * max_levels)()
    _check(lib().sf_mg_plan(gnx, gny, gnz, nparts, agglom_min_planes, max_levels, C.byref(n),
                            dims, dist))
    return [((dims[3 * l], dims[3 * l + 1], dims[3 * l + 2]), bool(dist[l]))
            for l in range(min(n.value, max_levels))]


def sf_launch_count(reset=False):
    n = C.c_longlong()
    _check(lib().sf_launch_count(C.byref(n), int(reset)))
    return n.value


# ------------------------------------------------------------ convenience layer
def host_shape(field, nx, ny, nz):
    return {SF_BETA_I: (nz, ny, nx + 1), SF_BETA_J: (nz, ny + 1, nx),
            SF_BETA_K: (nz + 1, ny, nx)}.get(field, (nz, ny, nx))


class Comm:
    """Loopback (``Comm.local(P)``: P slabs in this process) or NCCL comm."""

    def __init__(self, handle, nparts, nlocal, first):
        self.h, self.nparts, self.nlocal, self.first = handle, nparts, nlocal, first

    @classmethod
    def local(cls, nparts):
        return cls(sf_comm_create_local(nparts), nparts, nparts, 0)

    @classmethod
    def nccl(cls, group=None):
        """One part per rank of the default (or given) torch.distributed group."""
        from . import parallel
        uid, rank, world = parallel.broadcast_unique_id(group)
        return cls(sf_comm_create_nccl(uid, world, rank), world, 1, rank)

    @classmethod
    def p2p(cls, group=None):
        """Device-initiated transport: one part per rank, halos / agglomeration /
        all-reduces by kernels reading the peers' memory (CUDA IPC, NVLink P2P
        across GPUs); ``group`` (e.g. gloo) only exchanges the IPC handles when
        levels are created (include/sf.h, sf_comm_create_p2p)."""
        return cls._ipc(group, sf_comm_create_p2p)

    @classmethod
    def hostipc(cls, group=None):
        """Test transport: one part per rank of a (gloo) torch.distributed group,
        all ranks on the SAME GPU; peer buffers through CUDA IPC, host
        synchronisation through ``group`` (include/sf.h, sf_comm_create_hostipc)."""
        return cls._ipc(group, sf_comm_create_hostipc)

    @classmethod
    def _ipc(cls, group, create):
        import torch
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)

        def allgather(send, n, recv, _user):
            try:
                src = torch.frombuffer(bytearray(C.string_at(send, n)), dtype=torch.uint8) if n else \
                    torch.empty(0, dtype=torch.uint8)
                outs = [torch.empty(n, dtype=torch.uint8) for _ in range(world)]
                dist.all_gather(outs, src.clone(), group=group)
                C.memmove(recv, torch.cat(outs).numpy().tobytes(), n * world)
                return 0
            except Exception as e:  # noqa: BLE001 -- reported through the C status
                print(f"hostipc all-gather failed: {e!r}")
                return 1

        cb = HOST_ALLGATHER(allgather)
        c = cls(create(world, rank, cb), world, 1, rank)
        c._cb = cb          # keep the trampoline alive as long as the comm
        return c

    def close(self):
        if self.h:
            sf_comm_destroy(self.h)
            self.h = None


class Level:
    """One level: device buffer from torch, stream from torch, handle from libsf."""

    def __init__(self, nx, ny, nz, h=None, comm=None, stream=None, device=None):
        import torch
        self.gnx, self.gny, self.gnz = nx, ny, nz
        self.h = (1.0 / max(nx, ny, nz)) if h is None else float(h)
        self.comm = comm
        chandle = comm.h if comm is not None else None
        self.nparts = comm.nparts if comm is not None else 1
        self.nlocal = comm.nlocal if comm is not None else 1
        self.lnz = nz // self.nparts
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else device
        self.stream = stream if stream is not None else torch.cuda.Stream(device=dev)
        nbytes = sf_level_bytes_needed(nx, ny, nz, chandle)
        self.buf = torch.empty(nbytes + 256, dtype=torch.uint8, device=dev)
        base = self.buf.data_ptr()
        base = (base + 255) // 256 * 256
        self.handle = sf_level_create(nx, ny, nz, self.h, chandle, self.stream.cuda_stream, base,
                                      nbytes)

    def host_shape(self, field):
        return host_shape(field, self.gnx, self.gny, self.lnz * self.nlocal)

    def upload(self, field, arr):
        a = np.ascontiguousarray(arr, dtype=np.float64)
        if a.shape != self.host_shape(field):
            raise ValueError(f"field {field}: shape {a.shape} != {self.host_shape(field)}")
        sf_level_upload(self.handle, field, a.ctypes.data)
        sf_sync(self.handle)          # pageable host memory: keep `a` alive until done

    def upload_async(self, field, pinned_ptr):
        sf_level_upload(self.handle, field, pinned_ptr)

    def download(self, field, out=None):
        out = np.empty(self.host_shape(field)) if out is None else out
        sf_level_download(self.handle, field, out.ctypes.data)
        return out

    def padded(self, field, part=0, ghost=1):
        """Device copy of (lnz+2g, ny+2g, nx+2g) incl. ghost zone -> numpy (tests)."""
        import torch
        self.stream.synchronize()
        ptr, (s0, s1, s2) = sf_level_field_ptr(self.handle, part, field)
        base = self.buf.data_ptr()
        off = (ptr - base) // 8
        assert (ptr - base) % 8 == 0
        nbytes = self.buf.numel() - (self.buf.numel() % 8)
        d = self.buf[:nbytes].view(torch.float64)
        g = ghost
        out = np.empty((self.lnz + 2 * g, self.gny + 2 * g, self.gnx + 2 * g))
        for k in range(-g, self.lnz + g):
            start = off + k * s2 - g * s1 - g
            rows = d[start: start + (self.gny + 2 * g) * s1].view(self.gny + 2 * g, s1)
            out[k + g] = rows[:, : self.gnx + 2 * g].cpu().numpy()
        return out

    def set_coeffs(self, alpha, bi, bj, bk):
        self.upload(SF_ALPHA, alpha)
        self.upload(SF_BETA_I, bi)
        self.upload(SF_BETA_J, bj)
        self.upload(SF_BETA_K, bk)

    def close(self):
        if getattr(self, "handle", None):
            sf_level_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class MG:
    def __init__(self, level, a, b, **opts):
        o = sf_mg_opts_default()
        for k, v in opts.items():
            setattr(o, k, v)
        self.level, self.a, self.b = level, a, b
        self.handle = sf_mg_create(level.handle, a, b, o)

    @property
    def num_levels(self):
        return sf_mg_num_levels(self.handle)

    def solve(self, fcycle=True, rtol=1e-10, max_cycles=50, raise_on_error=True):
        return sf_solve(self.handle, fcycle, rtol, max_cycles, raise_on_error)

    def solve_stream(self, fs, us, fcycle=True, rtol=1e-10, max_cycles=50):
        """Solve for each host rhs in `fs` (arrays of the level's host shape,
        pinned torch tensors for overlap) into the matching `us`; the copies of
        neighbouring right-hand sides overlap each solve (sf_solve_stream)."""
        def ptr(a):
            if hasattr(a, "data_ptr"):
                return a.data_ptr()
            if not a.flags.c_contiguous or a.dtype != np.float64:
                raise ValueError("C-contiguous float64 arrays expected")
            return a.ctypes.data
        return sf_solve_stream(self.handle, [ptr(f) for f in fs], [ptr(u) for u in us], fcycle,
                               rtol, max_cycles)

    def vcycle(self, l=0):
        sf_vcycle(self.handle, l)

    def fcycle(self):
        sf_fcycle(self.handle)

    def close(self):
        if getattr(self, "handle", None):
            sf_mg_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
