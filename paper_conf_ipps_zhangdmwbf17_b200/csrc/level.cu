// Level / box layout (A1), C-ABI entry points of the per-level operators,
// error reporting and launch accounting.
#include <cstdarg>
#include <cstring>

#include <cstdlib>

#include "sf_internal.h"

// ----------------------------------------------------------------- errors
static thread_local char g_err[1024] = "";
static std::atomic<long long> g_launches{0};

sf_status sf_fail(sf_status s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

void sf_count_launch(long long n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

sf_status sf_check_launch(const char* what) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        char w[160];
        snprintf(w, sizeof(w), "launch of %s", what);
        return sf_cuda_failure(e, w);
    }
    return SF_OK;
}

extern "C" const char* sf_last_error(void) { return g_err; }

extern "C" const char* sf_version(void) {
    return "libsf 0.1 (sm_100a, fp64; HPGMG-FV hot path of Snowflake, IPDPSW 2017)";
}

extern "C" sf_status sf_launch_count(long long* count, int reset) {
    if (!count) return sf_fail(SF_ERR_INVALID, "count is NULL");
    *count = reset ? g_launches.exchange(0) : g_launches.load();
    return SF_OK;
}

// ----------------------------------------------------------------- device check
static sf_status check_device() {
    int dev = -1;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return sf_fail(SF_ERR_CUDA, "no CUDA device: %s", cudaGetErrorString(e));
    cudaDeviceProp pr;
    SF_CUDA(cudaGetDeviceProperties(&pr, dev));
    if (pr.major != 10 || pr.minor != 0)
        return sf_fail(SF_ERR_CUDA, "libsf is built for sm_100a; device %d is sm_%d%d (%s)", dev,
                       pr.major, pr.minor, pr.name);
    return SF_OK;
}

// ----------------------------------------------------------------- layout
static void layout(int gnx, int gny, int lnz, long* js, long* ks, size_t* felems) {
    long j = SF_OX + gnx + 2;
    j = (j + 15) / 16 * 16;  // 128-byte rows
    *js = j;
    *ks = j * (gny + 2 * SF_GY);
    *felems = (size_t)(*ks) * (lnz + 2 * SF_GZ);
}

static size_t field_bytes_aligned(size_t felems) { return (felems * sizeof(double) + 255) / 256 * 256; }

static sf_status decomposition(int gnz, const sf_comm* comm, int* nparts, int* nlocal, int* first) {
    if (!comm) {
        *nparts = 1; *nlocal = 1; *first = 0;
        return SF_OK;
    }
    *nparts = comm->nparts; *nlocal = comm->nlocal; *first = comm->first;
    if (gnz % comm->nparts != 0)
        return sf_fail(SF_ERR_SHAPE, "gnz=%d not divisible by %d parts", gnz, comm->nparts);
    return SF_OK;
}

extern "C" sf_status sf_level_bytes_needed(int gnx, int gny, int gnz, const sf_comm* comm,
                                           size_t* bytes) {
    if (!bytes) return sf_fail(SF_ERR_INVALID, "bytes is NULL");
    if (gnx < 2 || gny < 2 || gnz < 2) return sf_fail(SF_ERR_SHAPE, "dims must be >= 2");
    int np, nl, fi;
    SF_TRY(decomposition(gnz, comm, &np, &nl, &fi));
    long js, ks;
    size_t fe;
    layout(gnx, gny, gnz / np, &js, &ks, &fe);
    *bytes = (size_t)nl * SF_NF_ALL * field_bytes_aligned(fe) + SF_SCRATCH_BYTES;
    return SF_OK;
}

extern "C" sf_status sf_level_create(sf_level** out, int gnx, int gny, int gnz, double h,
                                     const sf_comm* comm, void* stream, void* dev_buf,
                                     size_t buf_bytes) {
    if (!out) return sf_fail(SF_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (!(h > 0)) return sf_fail(SF_ERR_INVALID, "h must be > 0");
    SF_TRY(check_device());
    size_t need;
    SF_TRY(sf_level_bytes_needed(gnx, gny, gnz, comm, &need));
    sf_level* L = new sf_level();
    L->gnx = gnx; L->gny = gny; L->gnz = gnz; L->h = h;
    SF_TRY(decomposition(gnz, comm, &L->nparts, &L->nlocal, &L->first));
    L->comm = comm;
    L->nx = gnx; L->ny = gny; L->lnz = gnz / L->nparts;
    layout(gnx, gny, L->lnz, &L->js, &L->ks, &L->felems);
    L->stream = (cudaStream_t)stream;
    if (dev_buf) {
        if (buf_bytes < need) {
            delete L;
            return sf_fail(SF_ERR_OOM, "caller buffer %zu bytes < %zu needed", buf_bytes, need);
        }
        if (((uintptr_t)dev_buf) & 255) {
            delete L;
            return sf_fail(SF_ERR_INVALID, "caller buffer must be 256-byte aligned");
        }
        L->buf = dev_buf;
        L->owns = false;
    } else {
        cudaError_t e = cudaMalloc(&L->buf, need);
        if (e != cudaSuccess) {
            delete L;
            cudaGetLastError();
            return sf_fail(SF_ERR_OOM, "cudaMalloc(%zu): %s", need, cudaGetErrorString(e));
        }
        L->owns = true;
    }
    char* p = (char*)L->buf;
    size_t fb = field_bytes_aligned(L->felems);
    L->parts.resize(L->nlocal);
    for (int q = 0; q < L->nlocal; q++) {
        SfPart& P = L->parts[q];
        P.index = L->first + q;
        P.z0 = P.index * L->lnz;
        for (int f = 0; f < SF_NF_ALL; f++) {
            P.f[f] = (double*)p;
            p += fb;
        }
    }
    L->dscratch = (double*)p;  // 32 device scalars, then the P2P sync words
    L->dsync = (unsigned long long*)(L->dscratch + 32);
    cudaError_t e = cudaHostAlloc(&L->hscratch, 256, cudaHostAllocMapped);
    if (e == cudaSuccess) e = cudaHostGetDevicePointer(&L->hscratch_dev, L->hscratch, 0);
    if (e != cudaSuccess) {
        if (L->owns) cudaFree(L->buf);
        delete L;
        return sf_fail(SF_ERR_CUDA, "cudaMallocHost: %s", cudaGetErrorString(e));
    }
    e = cudaMemsetAsync(L->buf, 0, need, L->stream);
    if (e != cudaSuccess) return sf_fail(SF_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
    if (comm && (comm->kind == 2 || comm->kind == 3)) {
        sf_status s = sf_ipc_register(L, comm);
        if (s != SF_OK) {
            sf_level_destroy(L);
            return s;
        }
    }
    *out = L;
    return SF_OK;
}

extern "C" sf_status sf_level_destroy(sf_level* L) {
    if (!L) return SF_OK;
    cudaStreamSynchronize(L->stream);
    if (L->side) {
        cudaStreamSynchronize(L->side);
        cudaStreamDestroy(L->side);
    }
    if (L->ev_fork) cudaEventDestroy(L->ev_fork);
    if (L->ev_join) cudaEventDestroy(L->ev_join);
    sf_ipc_close(L);
    if (L->rrf_buf) cudaFree(L->rrf_buf);
    if (L->owns) cudaFree(L->buf);
    cudaFreeHost(L->hscratch);
    delete L;
    return SF_OK;
}

PV sf_view(const sf_level* L, int p) {
    PV v;
    for (int f = 0; f < SF_NF_ALL; f++) v.f[f] = L->parts[p].f[f];
    v.nx = L->nx; v.ny = L->ny; v.nz = L->lnz;
    v.z0 = L->parts[p].z0; v.gnz = L->gnz;
    v.js = L->js; v.ks = L->ks;
    return v;
}

static sf_status check_field(int f) {
    if (f < 0 || f >= SF_NFIELDS) return sf_fail(SF_ERR_INVALID, "bad field id %d", f);
    return SF_OK;
}

// host extent of a field per part: (nzh planes, nyh rows, nxh columns)
static void host_extent(const sf_level* L, int field, int* nxh, int* nyh, int* nzh) {
    *nxh = L->nx + (field == SF_BETA_I);
    *nyh = L->ny + (field == SF_BETA_J);
    *nzh = L->lnz + (field == SF_BETA_K);
}

// copy a field's interior between the level and a packed host-layout buffer
// (host memory or device memory: cudaMemcpyDefault) on `stream`
sf_status sf_copy_field(sf_level* L, int field, double* host, bool up, cudaStream_t stream) {
    int nxh, nyh, nzh;
    host_extent(L, field, &nxh, &nyh, &nzh);
    for (int q = 0; q < L->nlocal; q++) {
        cudaMemcpy3DParms m = {};
        double* dev = L->parts[q].f[field] + (long)SF_GZ * L->ks + (long)SF_GY * L->js + SF_OX;
        double* hp = host + (size_t)q * L->lnz * nyh * nxh;  // parts share the interface face
        cudaPitchedPtr dp = make_cudaPitchedPtr(dev, L->js * sizeof(double), nxh * sizeof(double),
                                                L->ny + 2 * SF_GY);
        cudaPitchedPtr hpp = make_cudaPitchedPtr(hp, nxh * sizeof(double), nxh * sizeof(double), nyh);
        m.extent = make_cudaExtent(nxh * sizeof(double), nyh, nzh);
        if (up) {
            m.srcPtr = hpp; m.dstPtr = dp;
        } else {
            m.srcPtr = dp; m.dstPtr = hpp;
        }
        m.kind = cudaMemcpyDefault;
        SF_CUDA(cudaMemcpy3DAsync(&m, stream));
    }
    return SF_OK;
}

static sf_status copy3d(sf_level* L, int field, double* host, bool up) {
    return sf_copy_field(L, field, host, up, L->stream);
}

extern "C" sf_status sf_level_zero(sf_level* L, int field) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(field));
    return k_zero(L, field);
}

extern "C" sf_status sf_level_upload(sf_level* L, int field, const double* host) {
    if (!L || !host) return sf_fail(SF_ERR_INVALID, "NULL argument");
    SF_TRY(check_field(field));
    return copy3d(L, field, const_cast<double*>(host), true);
}

extern "C" sf_status sf_level_download(sf_level* L, int field, double* host) {
    if (!L || !host) return sf_fail(SF_ERR_INVALID, "NULL argument");
    SF_TRY(check_field(field));
    SF_TRY(copy3d(L, field, host, false));
    SF_TRY(sf_stream_sync(L));
    return SF_OK;
}

extern "C" sf_status sf_level_field_ptr(sf_level* L, int part, int field, double** dev,
                                        long strides[3]) {
    if (!L || !dev) return sf_fail(SF_ERR_INVALID, "NULL argument");
    SF_TRY(check_field(field));
    if (part < 0 || part >= L->nlocal) return sf_fail(SF_ERR_INVALID, "bad local part %d", part);
    *dev = L->parts[part].f[field] + (long)SF_GZ * L->ks + (long)SF_GY * L->js + SF_OX;
    if (strides) {
        strides[0] = 1; strides[1] = L->js; strides[2] = L->ks;
    }
    return SF_OK;
}

extern "C" sf_status sf_sync(sf_level* L) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(sf_stream_sync(L));
    SF_CUDA(cudaGetLastError());
    return SF_OK;
}

// ----------------------------------------------------------------- operators
extern "C" sf_status sf_init_problem(sf_level* L, int problem, double a, double b, int want_rhs) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    if (problem != 0 && problem != 1) return sf_fail(SF_ERR_INVALID, "problem must be 0 or 1");
    if (want_rhs) SF_TRY(k_zero(L, SF_U));
    return k_init_problem(L, problem, a, b, want_rhs);
}

extern "C" sf_status sf_rebuild_operator(sf_level* L, double a, double b) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    // coefficient halos for the colour-fused smoother's redundant ring work
    for (int f : {SF_ALPHA, SF_BETA_I, SF_BETA_J, SF_BETA_K}) SF_TRY(sf_halo(L, f, 2));
    SF_TRY(k_dinv(L, a, b));
    SF_TRY(k_beta0(L));   // boundary-zeroed faces of the colour-fused pair (halos included)
    return sf_halo(L, SF_DINV, 2);
}

extern "C" sf_status sf_apply_bc(sf_level* L, int field) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(field));
    return k_bc(L, field);
}

extern "C" sf_status sf_apply_op(sf_level* L, int out, int x, double a, double b) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(out));
    SF_TRY(check_field(x));
    if (out == x) return sf_fail(SF_ERR_INVALID, "out must differ from x");
    return k_apply_op(L, out, x, a, b);
}

extern "C" sf_status sf_apply_laplacian(sf_level* L, int out, int x) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(out));
    SF_TRY(check_field(x));
    if (out == x) return sf_fail(SF_ERR_INVALID, "out must differ from x");
    return k_cc(L, out, x, -1, 0.0, false);
}

extern "C" sf_status sf_jacobi(sf_level* L, int out, int x, int f, double omega) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(out));
    SF_TRY(check_field(x));
    SF_TRY(check_field(f));
    if (out == x || out == f) return sf_fail(SF_ERR_INVALID, "out must differ from x and f");
    return k_cc(L, out, x, f, omega, true);
}

// NEXT-3: Chebyshev smoother (reading R-16; Saad Alg. 12.1, Jacobi-preconditioned).
// Ids rotate over {x, TMP, R}; the final iterate ends under the id x.
sf_status sf_chebyshev_impl(sf_level* L, int x, int rhs, double a, double b, int degree, double lo,
                            double hi) {
    const double theta = 0.5 * (hi + lo), delta = 0.5 * (hi - lo), sigma = theta / delta;
    double rho_prev = 1.0 / sigma, rho = rho_prev;
    int cur = x, prv = SF_TMP, nxt = SF_R;
    for (int it = 0; it < degree; it++) {
        double c1, c2;
        if (it == 0) {
            c1 = 0.0;
            c2 = 1.0 / theta;
        } else {
            rho = 1.0 / (2.0 * sigma - rho_prev);
            c1 = rho * rho_prev;
            c2 = 2.0 * rho / delta;
        }
        SF_TRY(k_cheby_step(L, nxt, cur, it == 0 ? cur : prv, rhs, c1, c2, a, b));
        const int t = prv;
        prv = cur;
        cur = nxt;
        nxt = t;
        if (it > 0) rho_prev = rho;
    }
    // the result lives in the buffer named `cur`: make `x` name it
    if (cur != x) sf_swap_fields(L, x, cur);
    return SF_OK;
}

extern "C" sf_status sf_smooth_chebyshev(sf_level* L, int x, int rhs, double a, double b,
                                         int degree, double lo, double hi) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(x));
    SF_TRY(check_field(rhs));
    if (x == SF_TMP || x == SF_R || rhs == SF_TMP || rhs == SF_R || x == rhs)
        return sf_fail(SF_ERR_INVALID, "x and rhs must be distinct and not TMP/R (scratch)");
    if (degree < 0 || !(hi > lo) || !(lo > 0)) return sf_fail(SF_ERR_INVALID, "bad degree/interval");
    return sf_chebyshev_impl(L, x, rhs, a, b, degree, lo, hi);
}

sf_status sf_lambda_max_impl(sf_level* L, int v, double a, double b, int iters, bool start,
                             double* out) {
    if (start) SF_TRY(k_start_vector(L, v));
    double* sumsq = L->dscratch + 1;
    for (int it = 0; it < iters; it++) SF_TRY(k_power_step(L, v, SF_R, a, b, sumsq));
    // last ratio ||D^-1 A v|| / ||v|| with ||v|| = 1 after normalisation
    SF_TRY(sf_scalar_to_host(L, sumsq, 1));
    SF_TRY(sf_stream_sync(L));
    *out = sqrt(L->hscratch[1]);
    return SF_OK;
}

extern "C" sf_status sf_lambda_max(sf_level* L, int v, double a, double b, int iters, int start,
                                   double* out) {
    if (!L || !out) return sf_fail(SF_ERR_INVALID, "NULL argument");
    SF_TRY(check_field(v));
    if (v == SF_R || iters < 1) return sf_fail(SF_ERR_INVALID, "v must not be R; iters >= 1");
    return sf_lambda_max_impl(L, v, a, b, iters, start != 0, out);
}

extern "C" sf_status sf_residual(sf_level* L, int res, int x, int rhs, double a, double b) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(res));
    SF_TRY(check_field(x));
    SF_TRY(check_field(rhs));
    if (res == x) return sf_fail(SF_ERR_INVALID, "res must differ from x");
    return k_residual(L, res, x, rhs, a, b);
}

static bool coarse_of(const sf_level* C, const sf_level* F);

extern "C" sf_status sf_smooth_residual_restrict(sf_level* F, int x, int rhs, double a, double b,
                                                 sf_level* C, int cf) {
    if (!F || !C) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(x));
    SF_TRY(check_field(rhs));
    SF_TRY(check_field(cf));
    if (x == rhs || x == SF_DINV || rhs == SF_DINV || x == SF_R || rhs == SF_R || cf == SF_DINV)
        return sf_fail(SF_ERR_INVALID, "x, rhs, R and DINV must be distinct fields");
    if (!coarse_of(C, F)) return sf_fail(SF_ERR_SHAPE, "coarse dims must be fine dims / 2");
    // (inside a graph capture the fused path needs its partial arrays from an
    // earlier eager call or sf_mg_create; otherwise the composite path runs)
    if (x == SF_U && rhs != SF_TMP && gsrb_fused_supported(F) && gsrb_rr_supported(F, C) &&
        sf_rrf_usable(F, C)) {
        const int other = (x == SF_U) ? SF_TMP : SF_U;
        SF_TRY(sf_halo(F, rhs, 1));
        SF_TRY(sf_halo(F, x, 2));
        SF_TRY(k_gsrb_pair_rr(F, x, other, rhs, a, b, C, cf));
        sf_swap_fields(F, x, other);
        return SF_OK;
    }
    SF_TRY(sf_smooth_gsrb(F, x, rhs, a, b, 1, SF_SMOOTH_AUTO));
    if (pair_ok(F))   // residual never stored (A6 + A7, 49 B/cell)
        return k_residual_restrict(F, x, rhs, a, b, C, cf);
    SF_TRY(k_residual(F, SF_R, x, rhs, a, b));
    return k_restrict(C, cf, F, SF_R, SF_RESTRICT_CELL);
}

extern "C" sf_status sf_interpolate_smooth(sf_level* F, int x, int rhs, double a, double b,
                                           sf_level* C, int cf) {
    if (!F || !C) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(x));
    SF_TRY(check_field(rhs));
    SF_TRY(check_field(cf));
    if (x == rhs || x == SF_DINV || rhs == SF_DINV)
        return sf_fail(SF_ERR_INVALID, "x, rhs and DINV must be distinct fields");
    if (!coarse_of(C, F)) return sf_fail(SF_ERR_SHAPE, "coarse dims must be fine dims / 2");
    if (x == SF_U && rhs != SF_TMP && gsrb_fused_supported(F)) {
        // e_l += P0 e_{l+1} applied to each x plane in shared memory inside the
        // colour-fused pair (the V-cycle's first post-smoothing pair, mg.cu)
        SF_TRY(sf_halo(C, cf, 1));
        SF_TRY(sf_halo(F, rhs, 1));
        SF_TRY(k_gsrb_pair_halo(F, SF_U, SF_TMP, rhs, a, b, nullptr, C, cf, SF_RM_NONE));
        sf_swap_fields(F, SF_U, SF_TMP);
        return SF_OK;
    }
    SF_TRY(k_interp(F, x, 1.0, C, cf, SF_INTERP_P0));
    return sf_smooth_gsrb(F, x, rhs, a, b, 1, SF_SMOOTH_AUTO);
}

bool gsrb_fused_supported(const sf_level* L) {
    return gsrb_fused_supported_t32(L) || gsrb_fused_supported_t64(L);
}

sf_status k_gsrb_pair_fused(sf_level* L, int xin, int xout, int rhs, double a, double b,
                            double* rmax, sf_level* C, int cf, int phase, int reserve, int rmode) {
    // 32x8 tiles with three CTAs per SM: 7.5 % faster than 32x16 with one at
    // 256^3, equal at 512^3 timed alone and 2 % faster inside the power-capped
    // solve (profiles/r01/ab_256_ctas_per_sm.txt, ab_w4_512.txt,
    // ab_w4_instep.txt): the default wherever the shape allows.  SF_GSRB_W4=0
    // selects the 32x16 / 64x8 one-CTA builds (read per call: tests switch it)
    const char* ew = getenv("SF_GSRB_W4");
    int w4 = ew ? atoi(ew) : -1;
    // the P0-fused variant keeps 5-deep prefetch on big levels (its end-of-step
    // correction waits one bundle ahead): 32x16 build there, 0.25 % faster
    // solve (r01/ab_interp_t32.txt); SF_INTERP_T32=0 disables
    const char* ei = getenv("SF_INTERP_T32");
    // SF_INTERP_T32_CELLS: the level size above which it applies (tests lower it
    // to compare that build with the oracle cell by cell on small levels)
    const char* ec = getenv("SF_INTERP_T32_CELLS");
    const long t32_cells = ec ? atol(ec) : (1L << 24);
    if (C && !(ei && atoi(ei) == 0) && w4 < 0 && (long)L->nx * L->ny * L->lnz > t32_cells &&
        gsrb_fused_supported_t32(L))
        w4 = 0;
    if (w4 != 0 && gsrb_fused_supported_t32w4(L))
        return k_gsrb_pair_fused_t32w4(L, xin, xout, rhs, a, b, rmax, C, cf, phase, reserve, rmode);
    if (gsrb_fused_supported_t32(L))
        return k_gsrb_pair_fused_t32(L, xin, xout, rhs, a, b, rmax, C, cf, phase, reserve, rmode);
    return k_gsrb_pair_fused_t64(L, xin, xout, rhs, a, b, rmax, C, cf, phase, reserve, rmode);
}

void sf_swap_fields(sf_level* L, int f1, int f2) {
    for (auto& P : L->parts) std::swap(P.f[f1], P.f[f2]);
}

extern "C" sf_status sf_smooth_gsrb(sf_level* L, int x, int rhs, double a, double b, int rb_pairs,
                                    int kind) {
    if (!L) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(x));
    SF_TRY(check_field(rhs));
    if (rb_pairs < 0) return sf_fail(SF_ERR_INVALID, "rb_pairs < 0");
    if (x == rhs || x == SF_DINV || rhs == SF_DINV)
        return sf_fail(SF_ERR_INVALID, "x, rhs and DINV must be distinct fields");
    bool fused_ok = gsrb_fused_supported(L) && (x == SF_U || x == SF_TMP) && rhs != SF_TMP &&
                    rhs != SF_U;
    if (kind == SF_SMOOTH_FUSED2) {   // NEXT-1: two pairs per pass
        if (!fused_ok || !gsrb_twopair_supported(L))
            return sf_fail(SF_ERR_SHAPE, "two-pair smoother unsupported for this level/fields");
        if (rb_pairs == 0) return SF_OK;
        int other = (x == SF_U) ? SF_TMP : SF_U;
        SF_TRY(sf_halo(L, rhs, 1));
        for (int p = 0; p + 1 < rb_pairs; p += 2) {
            SF_TRY(k_gsrb_twopair(L, x, other, rhs, a, b));
            sf_swap_fields(L, x, other);
        }
        if (rb_pairs & 1) {
            SF_TRY(k_gsrb_pair_halo(L, x, other, rhs, a, b));
            sf_swap_fields(L, x, other);
        }
        return SF_OK;
    }
    if (kind == SF_SMOOTH_FUSED && !fused_ok)
        return sf_fail(SF_ERR_SHAPE, "fused smoother unsupported for this level/fields");
    // the fused pair ping-pongs x through the other of U / TMP; AUTO only takes
    // it when that other field is the scratch TMP (x = U), so a solution in U is
    // never clobbered by a call that did not ask for the fused kernel
    bool fused = (kind == SF_SMOOTH_FUSED) || (kind == SF_SMOOTH_AUTO && fused_ok && x == SF_U);
    if (rb_pairs == 0) return SF_OK;
    if (fused) {
        int other = (x == SF_U) ? SF_TMP : SF_U;
        SF_TRY(sf_halo(L, rhs, 1));
        for (int p = 0; p < rb_pairs; p++) {
            SF_TRY(k_gsrb_pair_halo(L, x, other, rhs, a, b));
            sf_swap_fields(L, x, other);  // result now lives under the id `x`
        }
        return SF_OK;
    }
    for (int p = 0; p < rb_pairs; p++) {
        SF_TRY(k_gsrb_colour(L, x, rhs, a, b, 0));
        SF_TRY(k_gsrb_colour(L, x, rhs, a, b, 1));
    }
    return SF_OK;
}

static bool coarse_of(const sf_level* C, const sf_level* F) {
    return C->gnx * 2 == F->gnx && C->gny * 2 == F->gny && C->gnz * 2 == F->gnz &&
           (C->nparts == F->nparts || C->nparts == 1) && (F->lnz % 2 == 0);
}

extern "C" sf_status sf_restrict(sf_level* C, int cf, sf_level* F, int ff, int kind) {
    if (!C || !F) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(cf));
    SF_TRY(check_field(ff));
    if (!coarse_of(C, F)) return sf_fail(SF_ERR_SHAPE, "coarse dims must be fine dims / 2");
    if (kind < SF_RESTRICT_CELL || kind > SF_RESTRICT_FACE_K)
        return sf_fail(SF_ERR_INVALID, "bad restriction kind");
    return k_restrict(C, cf, F, ff, kind);
}

extern "C" sf_status sf_interpolate(sf_level* F, int ff, double prescale, sf_level* C, int cf,
                                    int kind) {
    if (!C || !F) return sf_fail(SF_ERR_INVALID, "NULL level");
    SF_TRY(check_field(cf));
    SF_TRY(check_field(ff));
    if (!coarse_of(C, F)) return sf_fail(SF_ERR_SHAPE, "coarse dims must be fine dims / 2");
    if (kind != SF_INTERP_P0 && kind != SF_INTERP_PL)
        return sf_fail(SF_ERR_INVALID, "bad interpolation kind");
    return k_interp(F, ff, prescale, C, cf, kind);
}

sf_status sf_norm_async(sf_level* L, int field, int kind, double* dst) {
    SF_TRY(k_norm(L, field, kind, dst));
    if (L->comm && L->comm->kind != 0 && L->nparts > 1)
        SF_TRY(sf_allreduce_scalar(L, L->comm, dst, kind == SF_NORM_MAX ? 0 : 1));
    return SF_OK;
}

// A device scalar -> hscratch[slot] through mapped pinned memory, written by a
// one-thread kernel: no copy-engine transfer, so the per-cycle convergence
// scalar never queues behind bulk PCIe copies (sf_solve_stream).
static __global__ void scalar_to_host_kernel(const double* src, double* dst) { pdl_wait(); *dst = *src; }

sf_status sf_scalar_to_host(sf_level* L, const double* src, int slot) {
    sf_launch(scalar_to_host_kernel, 1, 1, 0, L->stream, src, L->hscratch_dev + slot);
    SF_LAUNCHED();
    return sf_check_launch("scalar_to_host");
}

extern "C" sf_status sf_norm(sf_level* L, int field, int kind, double* out) {
    if (!L || !out) return sf_fail(SF_ERR_INVALID, "NULL argument");
    SF_TRY(check_field(field));
    if (kind != SF_NORM_MAX && kind != SF_NORM_L2) return sf_fail(SF_ERR_INVALID, "bad norm kind");
    SF_TRY(sf_norm_async(L, field, kind, L->dscratch));
    SF_TRY(sf_scalar_to_host(L, L->dscratch, 0));
    SF_TRY(sf_stream_sync(L));
    double v = L->hscratch[0];
    *out = (kind == SF_NORM_L2) ? sqrt(v) : v;
    return SF_OK;
}

// programmatic stream serialisation on every launch unless SF_PDL=0 (sf_internal.h)
bool sf_pdl_on() {
    static const int v = getenv("SF_PDL") ? atoi(getenv("SF_PDL")) : 1;
    return v != 0;
}

// Live duration of the colour-fused pair kernel on this level (SF_TS_OFF slots
// of the level's device scratch; gsrb_fused.cu stamps them when armed).
extern "C" sf_status sf_level_pair_timing(sf_level* L, int op, double* mean_ms, long long* count) {
    if (!L || (op != 0 && op != 1)) return sf_fail(SF_ERR_INVALID, "NULL level or bad op");
    unsigned long long* ts = (unsigned long long*)(L->dscratch + SF_TS_OFF);
    if (op == 1) {
        static const unsigned long long arm[16] = {1ull, ~0ull, 0ull, 0ull, 0ull, 0ull, 0ull, 0ull,
                                                   0ull, 0ull, 0ull, 0ull, 0ull, 0ull, 0ull, 0ull};
        SF_CUDA(cudaMemcpyAsync(ts, arm, sizeof(arm), cudaMemcpyHostToDevice, L->stream));
        SF_TRY(sf_stream_sync(L));
        return SF_OK;
    }
    unsigned long long h[16];
    SF_CUDA(cudaMemcpyAsync(h, ts, sizeof(h), cudaMemcpyDeviceToHost, L->stream));
    SF_TRY(sf_stream_sync(L));
    static const unsigned long long off = 0ull;
    SF_CUDA(cudaMemcpyAsync(ts, &off, sizeof(off), cudaMemcpyHostToDevice, L->stream));
    SF_TRY(sf_stream_sync(L));
    if (count) *count = (long long)h[4];
    if (mean_ms) *mean_ms = h[4] ? (double)h[5] / (double)h[4] * 1e-6 : 0.0;
    for (int v = 0; v < 5; v++) L->ts_var[v][0] = (double)h[6 + 2 * v], L->ts_var[v][1] = (double)h[7 + 2 * v];
    return SF_OK;
}

extern "C" sf_status sf_level_pair_timing_rrf(const sf_level* L, double* mean_ms, long long* count) {
    if (!L || !mean_ms || !count) return sf_fail(SF_ERR_INVALID, "NULL argument");
    *count = (long long)L->ts_var[4][0];
    *mean_ms = *count ? L->ts_var[4][1] / L->ts_var[4][0] * 1e-6 : 0.0;
    return SF_OK;
}

extern "C" sf_status sf_level_pair_timing_variants(const sf_level* L, double mean_ms[4],
                                                   long long counts[4]) {
    if (!L || !mean_ms || !counts) return sf_fail(SF_ERR_INVALID, "NULL argument");
    for (int v = 0; v < 4; v++) {
        counts[v] = (long long)L->ts_var[v][0];
        mean_ms[v] = counts[v] ? L->ts_var[v][1] / L->ts_var[v][0] * 1e-6 : 0.0;
    }
    return SF_OK;
}
