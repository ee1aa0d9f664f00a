// Coarse-level V-cycle in ONE launch of ONE CTA (A9 on the smallest levels).
//
// Levels of 16^3 cells and fewer are pure latency: every colour sweep,
// residual + restriction, P0 interpolation and the bottom solve of V(l)
// (A5-A9) is well under a microsecond of
// work behind a launch of its own -- ~30 launches per V-cycle below 32^3.
// Here one 512-thread CTA runs the whole V(l0) .. bottom .. V(l0) recursion
// with every operand in SHARED MEMORY OR REGISTERS, phases separated by
// __syncthreads: after one staging pass at the start, no phase touches global
// memory (the previous design read alpha / beta through L1/L2 in every phase,
// ~1.2 us per phase; profiles/r02/coarse_smem_staging.txt).
//
// Shared memory, compact per level (nx*ny*nz cells, x fastest):
//   U                              every level
//   F, Dinv, alpha                 every level below the entry level
//   beta_i (nx+1 faces per row), beta_j (ny+1 rows per plane),
//   beta_k (nz+1 planes)           every level above the bottom
// The entry level's F, Dinv and alpha (3 x 32 KB at 16^3 would not fit next to
// its faces) live in REGISTERS: thread t owns the 2x2x2 block of entry cells
// whose parent is coarse cell t (at most 512 blocks = 4096 cells), so its
// colour sweeps, its residual + restriction into parent t and the P0
// correction from parent t touch only its own F / Dinv / alpha.  Levels below
// the entry run one thread per cell with everything in shared memory.
//
// Arithmetic: op_sh is op_at's expression (cell_ops.cuh: same terms, order and
// Dirichlet fold); the colour sweep is gsrb_colour_kernel's update
// x += Dinv (rhs - A x); the residual + restriction sums rhs - A x over the 8
// children in restrict_cell's order and divides by 8; P0 adds the parent; the
// bottom applies the exact inverse in bottom_solve_kernel's order.
#include <cstdlib>

#include "sf_internal.h"

namespace {

constexpr int CMAXL = 8;                    // levels per launch
constexpr int CNT = 512;                    // threads = entry-level 2x2x2 blocks at most
constexpr long CMAX_CELLS = 8L * CNT;       // entry level at most 4096 cells (16^3)
constexpr int CSMEM_MAX = 227 * 1024;       // opt-in shared memory per CTA

struct CLevel {
    PV v;                 // global view: coefficients, the entry level's U / F / Dinv
    double bh2;
    int lx, ly, lz;       // log2 of nx, ny, nz (power-of-two levels: cell indices by shifts)
    int u, f, d, al;      // shared offsets (doubles) of U, F, Dinv, alpha (f/d/al: below entry)
    int bi, bj, bk;       // shared offsets of the face coefficients (above the bottom)
};

struct CoarseArgs {
    CLevel lv[CMAXL];
    int nlev;             // lv[0] = V's entry level, lv[nlev-1] = bottom
    int pre, post;        // RB pairs
    double a;
    const double* ainv;   // exact inverse of the bottom operator (n x n)
};

// A3 at (i,j,k) of a level held in shared memory; xc = x(i,j,k), al = alpha(i,j,k).
// op_at's expression term by term.
__device__ __forceinline__ double op_sh(const CLevel& L, const double* sm, int i, int j, int k,
                                        double xc, double al, double a) {
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int sy = nx, sz = nx << L.ly;
    const int c = i + (j << L.lx) + (k << (L.lx + L.ly));
    const double* x = sm + L.u;
    const double xw = (i == 0) ? -xc : x[c - 1];
    const double xe = (i == nx - 1) ? -xc : x[c + 1];
    const double xs = (j == 0) ? -xc : x[c - sy];
    const double xn = (j == ny - 1) ? -xc : x[c + sy];
    const double xb = (k == 0) ? -xc : x[c - sz];
    const double xt = (k == nz - 1) ? -xc : x[c + sz];
    const double* bi = sm + L.bi + i + (nx + 1) * (j + (k << L.ly));
    const double* bj = sm + L.bj + i + ((j + (ny + 1) * k) << L.lx);
    const double* bk = sm + L.bk + c;
    double flux = bi[1] * (xe - xc);
    flux += bi[0] * (xw - xc);
    flux += bj[sy] * (xn - xc);
    flux += bj[0] * (xs - xc);
    flux += bk[sz] * (xt - xc);
    flux += bk[0] * (xb - xc);
    return a * al * xc - L.bh2 * flux;
}

// The entry level's 2x2x2 block owned by this thread: origin (2I, 2J, 2K),
// sub-cell s = di + 2 dj + 4 dk; F / Dinv / alpha in registers.
struct Block {
    int i0, j0, k0;
    bool own;
    double F[8], D[8], A[8];
};

__device__ __forceinline__ int cell_of(const CLevel& L, int i, int j, int k) {
    return i + (j << L.lx) + (k << (L.lx + L.ly));
}

// one colour sweep of the entry level: the thread's 4 cells of colour `colour`
__device__ __forceinline__ void sweep_entry(const CLevel& L, double* sm, const Block& B, double a,
                                            int colour) {
    if (B.own) {
        double* x = sm + L.u;
#pragma unroll
        for (int s = 0; s < 8; s++) {
            const int di = s & 1, dj = (s >> 1) & 1, dk = s >> 2;
            if (((di + dj + dk) & 1) != colour) continue;   // block origin is even
            const int i = B.i0 + di, j = B.j0 + dj, k = B.k0 + dk;
            const int c = cell_of(L, i, j, k);
            const double xc = x[c];
            const double ax = op_sh(L, sm, i, j, k, xc, B.A[s], a);
            x[c] = xc + B.D[s] * (B.F[s] - ax);
        }
    }
    __syncthreads();
}

// one colour sweep of a level below the entry: one thread per cell of the colour
__device__ __forceinline__ void sweep_cells(const CLevel& L, double* sm, double a, int colour) {
    const int lh = L.lx - 1;                    // nx >= 2 on every level that is smoothed
    const int n = 1 << (lh + L.ly + L.lz);      // cells of one colour
    double* x = sm + L.u;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int th = t & ((1 << lh) - 1), r = t >> lh;
        const int j = r & ((1 << L.ly) - 1), k = r >> L.ly;
        const int i = 2 * th + ((j + k + colour) & 1);
        const int c = cell_of(L, i, j, k);
        const double xc = x[c];
        const double ax = op_sh(L, sm, i, j, k, xc, sm[L.al + c], a);
        x[c] = xc + sm[L.d + c] * (sm[L.f + c] - ax);
    }
    __syncthreads();
}

__device__ __forceinline__ void smooth(const CLevel& L, double* sm, const Block* B, double a,
                                       int pairs) {
    for (int p = 0; p < pairs; p++) {
        if (B) {
            sweep_entry(L, sm, *B, a, 0);
            sweep_entry(L, sm, *B, a, 1);
        } else {
            sweep_cells(L, sm, a, 0);
            sweep_cells(L, sm, a, 1);
        }
    }
}

// A6 + A7 from the entry level: C.F[t] = R_cell(F - A U) over block t; C.U = 0
__device__ __forceinline__ void residual_restrict_entry(const CLevel& F, const CLevel& C, double* sm,
                                                        const Block& B, double a) {
    if (B.own) {
        const double* x = sm + F.u;
        double acc = 0.0;
#pragma unroll
        for (int s = 0; s < 8; s++) {
            const int i = B.i0 + (s & 1), j = B.j0 + ((s >> 1) & 1), k = B.k0 + (s >> 2);
            const double xc = x[cell_of(F, i, j, k)];
            acc += B.F[s] - op_sh(F, sm, i, j, k, xc, B.A[s], a);
        }
        sm[C.f + threadIdx.x] = acc / 8.0;
        sm[C.u + threadIdx.x] = 0.0;
    }
    __syncthreads();
}

// A6 + A7 below the entry level: one thread per coarse cell
__device__ __forceinline__ void residual_restrict_cells(const CLevel& F, const CLevel& C, double* sm,
                                                        double a) {
    const int n = 1 << (C.lx + C.ly + C.lz);
    const double* x = sm + F.u;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int I = t & ((1 << C.lx) - 1), r = t >> C.lx;
        const int J = r & ((1 << C.ly) - 1), K = r >> C.ly;
        double acc = 0.0;
#pragma unroll
        for (int s = 0; s < 8; s++) {
            const int i = 2 * I + (s & 1), j = 2 * J + ((s >> 1) & 1), k = 2 * K + (s >> 2);
            const int c = cell_of(F, i, j, k);
            acc += sm[F.f + c] - op_sh(F, sm, i, j, k, x[c], sm[F.al + c], a);
        }
        sm[C.f + t] = acc / 8.0;
        sm[C.u + t] = 0.0;
    }
    __syncthreads();
}

// A8 P0 into the entry level: the block's 8 cells += parent t
__device__ __forceinline__ void interp_entry(const CLevel& F, const CLevel& C, double* sm,
                                             const Block& B) {
    if (B.own) {
        double* y = sm + F.u;
        const double e = sm[C.u + threadIdx.x];
#pragma unroll
        for (int s = 0; s < 8; s++) {
            const int c = cell_of(F, B.i0 + (s & 1), B.j0 + ((s >> 1) & 1), B.k0 + (s >> 2));
            y[c] = y[c] + e;
        }
    }
    __syncthreads();
}

// A8 P0 below the entry level: one thread per fine cell
__device__ __forceinline__ void interp_cells(const CLevel& F, const CLevel& C, double* sm) {
    const int n = 1 << (F.lx + F.ly + F.lz);
    double* y = sm + F.u;
    const double* e = sm + C.u;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int i = t & ((1 << F.lx) - 1), r = t >> F.lx;
        const int j = r & ((1 << F.ly) - 1), k = r >> F.ly;
        y[t] = y[t] + e[cell_of(C, i >> 1, j >> 1, k >> 1)];
    }
    __syncthreads();
}

// R-8: U = A^-1 F on the bottom level (<= 64 cells)
__device__ __forceinline__ void bottom(const CLevel& B, double* sm, const double* __restrict__ ainv) {
    const int n = 1 << (B.lx + B.ly + B.lz);
    const int r = threadIdx.x;
    if (r < n) {
        double acc = 0.0;
        for (int c = 0; c < n; c++) acc += __ldg(ainv + r * n + c) * sm[B.f + c];
        sm[B.u + r] = acc;
    }
    __syncthreads();
}

// padded global -> compact shared, one 8-byte cp.async per value (no thread
// waits on a load; one cp.async.wait_all before the first phase).  The box is
// 2^lw values x 2^lrj rows x rk planes starting at (ioff, joff, 0); shared
// element (i, j, k) at i + sw (j + srj k).
__device__ __forceinline__ void stage_box(double* dst, const double* __restrict__ src, int lw, int lrj,
                                          int rk, int ioff, int joff, int sw, int srj, long js,
                                          long ks) {
    const unsigned d0 = (unsigned)__cvta_generic_to_shared(dst);
    const int n = rk << (lw + lrj);
    for (int e = threadIdx.x; e < n; e += CNT) {
        const int i = (e & ((1 << lw) - 1)) + ioff, r = e >> lw;
        const int j = (r & ((1 << lrj) - 1)) + joff, k = r >> lrj;
        const double* g = src + (long)(k + SF_GZ) * ks + (long)(j + SF_GY) * js + SF_OX + i;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d0 + 8u * (i + sw * (j + srj * k))),
                     "l"(g)
                     : "memory");
    }
}

// a cell-centred field of level L (nx x ny x nz)
__device__ __forceinline__ void stage_cells(double* dst, const double* src, const CLevel& L) {
    stage_box(dst, src, L.lx, L.ly, 1 << L.lz, 0, 0, 1 << L.lx, 1 << L.ly, L.v.js, L.v.ks);
}

__global__ void __launch_bounds__(CNT, 1) coarse_vcycle_kernel(const __grid_constant__ CoarseArgs A) {
    extern __shared__ double sm[];
    pdl_wait();
    const int nl = A.nlev;
    // ---- staging: faces of every smoothed level, Dinv / alpha below the
    // entry, the entry's U (shared) and its F / Dinv / alpha (registers)
    for (int l = 0; l + 1 < nl; l++) {
        const CLevel& L = A.lv[l];
        const PV& v = L.v;
        const int nx = v.nx, ny = v.ny, nz = v.nz;
        // beta_i: faces 0..nx-1 of every row, then face nx
        stage_box(sm + L.bi, v.f[SF_BETA_I], L.lx, L.ly, nz, 0, 0, nx + 1, ny, v.js, v.ks);
        stage_box(sm + L.bi, v.f[SF_BETA_I], 0, L.ly, nz, nx, 0, nx + 1, ny, v.js, v.ks);
        // beta_j: rows 0..ny-1 of every plane, then row ny
        stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, L.ly, nz, 0, 0, nx, ny + 1, v.js, v.ks);
        stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, 0, nz, 0, ny, nx, ny + 1, v.js, v.ks);
        // beta_k: planes 0..nz
        stage_box(sm + L.bk, v.f[SF_BETA_K], L.lx, L.ly, nz + 1, 0, 0, nx, ny, v.js, v.ks);
        if (l > 0) {
            stage_cells(sm + L.d, v.f[SF_DINV], L);
            stage_cells(sm + L.al, v.f[SF_ALPHA], L);
        }
    }
    const CLevel& E = A.lv[0];
    stage_cells(sm + E.u, E.v.f[SF_U], E);
    asm volatile("cp.async.commit_group;" ::: "memory");
    Block B;
    {
        const int t = threadIdx.x;
        const int lhx = E.lx - 1, lhy = E.ly - 1, lhz = E.lz - 1;
        B.own = t < (1 << (lhx + lhy + lhz));
        B.i0 = 2 * (t & ((1 << lhx) - 1));
        B.j0 = 2 * ((t >> lhx) & ((1 << lhy) - 1));
        B.k0 = 2 * (t >> (lhx + lhy));
#pragma unroll
        for (int s = 0; s < 8; s++) {
            B.F[s] = B.D[s] = B.A[s] = 0.0;
            if (B.own) {
                const long q = sf_ix(E.v, B.i0 + (s & 1), B.j0 + ((s >> 1) & 1), B.k0 + (s >> 2));
                B.F[s] = __ldg(E.v.f[SF_F] + q);
                B.D[s] = __ldg(E.v.f[SF_DINV] + q);
                B.A[s] = __ldg(E.v.f[SF_ALPHA] + q);
            }
        }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncthreads();
    // ---- V(l0) down to the bottom and back
    smooth(E, sm, &B, A.a, A.pre);
    residual_restrict_entry(E, A.lv[1], sm, B, A.a);
    for (int l = 1; l + 1 < nl; l++) {
        smooth(A.lv[l], sm, nullptr, A.a, A.pre);
        residual_restrict_cells(A.lv[l], A.lv[l + 1], sm, A.a);
    }
    bottom(A.lv[nl - 1], sm, A.ainv);
    for (int l = nl - 2; l >= 1; l--) {
        interp_cells(A.lv[l], A.lv[l + 1], sm);
        smooth(A.lv[l], sm, nullptr, A.a, A.post);
    }
    interp_entry(E, A.lv[1], sm, B);
    smooth(E, sm, &B, A.a, A.post);
    // ---- the entry level's U back to global memory
    const PV& v = E.v;
    const int n = v.nx * v.ny * v.nz;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int i = t & (v.nx - 1), r = t >> E.lx;
        v.f[SF_U][sf_ix(v, i, r & (v.ny - 1), r >> E.ly)] = sm[E.u + t];
    }
}

// shared-memory plan of a V(lv[0]) over n levels: offsets into lv[], total doubles
long plan_smem(sf_level* const* lv, int n, CLevel* out) {
    long off = 0;
    for (int l = 0; l < n; l++) {
        const long nx = lv[l]->nx, ny = lv[l]->ny, nz = lv[l]->lnz, c = nx * ny * nz;
        CLevel L = {};
        L.u = (int)off;
        off += c;
        L.f = L.d = L.al = L.bi = L.bj = L.bk = -1;
        if (l > 0) {
            L.f = (int)off;
            off += c;
        }
        if (l > 0 && l + 1 < n) {
            L.d = (int)off;
            off += c;
            L.al = (int)off;
            off += c;
        }
        if (l + 1 < n) {
            L.bi = (int)off;
            off += (nx + 1) * ny * nz;
            L.bj = (int)off;
            off += nx * (ny + 1) * nz;
            L.bk = (int)off;
            off += nx * ny * (nz + 1);
        }
        if (out) out[l] = L;
    }
    return off;
}

}  // namespace

int coarse_vcycle_max_levels() { return CMAXL; }

// a V-cycle from lv[0] over n levels fits the kernel: single-part power-of-two
// levels, the entry at most 4096 cells, every operand within shared memory
bool coarse_vcycle_fits(sf_level* const* lv, int n) {
    if (n < 2 || n > CMAXL) return false;
    auto pow2 = [](int v) { return v >= 1 && (v & (v - 1)) == 0; };
    for (int l = 0; l < n; l++) {
        if (lv[l]->nparts != 1 || lv[l]->nlocal != 1) return false;
        if (!pow2(lv[l]->nx) || !pow2(lv[l]->ny) || !pow2(lv[l]->lnz)) return false;
        // every smoothed level halves into the next in all three directions
        if (l + 1 < n && (lv[l]->nx < 2 || lv[l]->ny < 2 || lv[l]->lnz < 2 ||
                          lv[l + 1]->nx * 2 != lv[l]->nx || lv[l + 1]->ny * 2 != lv[l]->ny ||
                          lv[l + 1]->lnz * 2 != lv[l]->lnz))
            return false;
    }
    const long bot = (long)lv[n - 1]->nx * lv[n - 1]->ny * lv[n - 1]->lnz;
    return (long)lv[0]->nx * lv[0]->ny * lv[0]->lnz <= CMAX_CELLS && bot <= CNT &&
           plan_smem(lv, n, nullptr) * (long)sizeof(double) <= CSMEM_MAX;
}

// V(lv[0]) down to the bottom lv[n-1] and back, one single-CTA launch
sf_status k_coarse_vcycle(sf_level* const* lv, int n, double a, double b, const double* ainv,
                          int pre, int post) {
    if (!coarse_vcycle_fits(lv, n)) return sf_fail(SF_ERR_SHAPE, "coarse V-cycle levels do not fit");
    static bool attr = false;
    if (!attr) {
        SF_CUDA(cudaFuncSetAttribute(coarse_vcycle_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     CSMEM_MAX));
        attr = true;
    }
    CoarseArgs A = {};
    const long doubles = plan_smem(lv, n, A.lv);
    for (int l = 0; l < n; l++) {
        A.lv[l].v = sf_view(lv[l], 0);
        A.lv[l].bh2 = b / (lv[l]->h * lv[l]->h);
        A.lv[l].lx = __builtin_ctz(lv[l]->nx);
        A.lv[l].ly = __builtin_ctz(lv[l]->ny);
        A.lv[l].lz = __builtin_ctz(lv[l]->lnz);
    }
    A.nlev = n;
    A.pre = pre;
    A.post = post;
    A.a = a;
    A.ainv = ainv;
    SF_CUDA(sf_launch(coarse_vcycle_kernel, 1, CNT, (size_t)doubles * sizeof(double), lv[0]->stream, A));
    SF_LAUNCHED();
    return sf_check_launch("coarse_vcycle");
}
