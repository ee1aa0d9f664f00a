// Coarse-level V-cycle in ONE launch of ONE CTA (A9 on the smallest levels).
//
// Levels of 16^3 cells and fewer are pure latency: every colour sweep,
// residual + restriction, P0 interpolation and the bottom solve of V(l)
// (A5-A9) is well under a microsecond of
// work behind a launch of its own -- ~30 launches per V-cycle below 32^3.
// Here one 1024-thread CTA runs the whole V(l0) .. bottom .. V(l0) recursion
// with the iterates of every level in SHARED memory (U, F and Dinv, compact
// nx*ny*nz layout: 16^3 + 8^3 + 4^3 + 2^3 cells = 110 KB), phases separated by
// __syncthreads instead of kernel boundaries; the read-only coefficients
// (alpha, beta) come through the read-only data cache.  Only F and U of the
// entry level are read from global memory (the level above restricted F; U is
// 0 in a V-cycle or the PL interpolant in an F-cycle) and only its U is
// written back.
//
// Arithmetic: op_acc is op_at's expression (cell_ops.cuh: same terms, order
// and Dirichlet fold); the colour sweep is gsrb_colour_kernel's update
// x += Dinv (rhs - A x); the residual + restriction sums rhs - A x over the 8
// children in restrict_cell's order; P0 adds the parent; the bottom applies the
// exact inverse in bottom_solve_kernel's order.
#include <cstdlib>

#include "sf_internal.h"

namespace {

constexpr int CMAXL = 8;          // levels per launch
constexpr int CNT = 1024;         // threads
constexpr long CMAX_CELLS = 4096; // entry level at most 16^3
constexpr int CSMEM_CELLS = 4096 + 512 + 64 + 8 + 64;   // room for a 16^3 .. 2^3 chain (+ slack)

struct CLevel {
    PV v;             // global view: coefficients (alpha, beta), entry level's U / F
    double bh2;
    int off;          // first cell of this level in the shared arrays
    int lx, ly, lz;   // log2 of nx, ny, nz (the kernel takes power-of-two levels:
                      // cell indices by shifts, no integer division in the phases)
};

struct CoarseArgs {
    CLevel lv[CMAXL];
    int nlev;         // lv[0] = V's entry level, lv[nlev-1] = bottom
    int pre, post;    // RB pairs
    double a;
    const double* ainv;   // exact inverse of the bottom operator (n x n)
};

// A3 at (i,j,k) of a level whose x lives compactly in shared memory (cell
// index c); coefficients at global index q.  op_at's expression term by term.
__device__ __forceinline__ double op_acc(const PV& v, const double* __restrict__ x, int c, int i,
                                         int j, int k, double a, double bh2) {
    const long q = sf_ix(v, i, j, k);
    const int sy = v.nx, sz = v.nx * v.ny;
    const double xc = x[c];
    const double xw = (i == 0) ? -xc : x[c - 1];
    const double xe = (i == v.nx - 1) ? -xc : x[c + 1];
    const double xs = (j == 0) ? -xc : x[c - sy];
    const double xn = (j == v.ny - 1) ? -xc : x[c + sy];
    const double xb = (k == 0) ? -xc : x[c - sz];
    const double xt = (k == v.nz - 1) ? -xc : x[c + sz];
    const double* bi = v.f[SF_BETA_I];
    const double* bj = v.f[SF_BETA_J];
    const double* bk = v.f[SF_BETA_K];
    double flux = __ldg(bi + q + 1) * (xe - xc);
    flux += __ldg(bi + q) * (xw - xc);
    flux += __ldg(bj + q + v.js) * (xn - xc);
    flux += __ldg(bj + q) * (xs - xc);
    flux += __ldg(bk + q + v.ks) * (xt - xc);
    flux += __ldg(bk + q) * (xb - xc);
    return a * __ldg(v.f[SF_ALPHA] + q) * xc - bh2 * flux;
}

struct Sh {
    double* U;
    double* F;
    double* D;
};

__device__ __forceinline__ void sweep(const CLevel& L, const Sh& s, double a, int colour) {
    const PV& v = L.v;
    const int hx = v.nx >> 1;
    const int n = hx * v.ny * v.nz;
    double* x = s.U + L.off;
    const double* rhs = s.F + L.off;
    const double* dv = s.D + L.off;
    const int lh = L.lx - 1;   // nx >= 2: hx = nx / 2
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int th = t & (hx - 1), r = t >> lh;
        const int j = r & (v.ny - 1), k = r >> L.ly;
        const int i = 2 * th + ((j + k + colour) & 1);
        const int c = (((k << L.ly) + j) << L.lx) + i;
        const double ax = op_acc(v, x, c, i, j, k, a, L.bh2);
        x[c] = x[c] + dv[c] * (rhs[c] - ax);
    }
    __syncthreads();
}

__device__ __forceinline__ void smooth(const CLevel& L, const Sh& s, double a, int pairs) {
    for (int p = 0; p < pairs; p++) {
        sweep(L, s, a, 0);
        sweep(L, s, a, 1);
    }
}

// A6 + A7: C.F = R_cell(F - A U); C.U = 0 (the next V's start)
__device__ __forceinline__ void residual_restrict(const CLevel& F, const CLevel& C, const Sh& s, double a) {
    const PV& f = F.v;
    const PV& c = C.v;
    const int n = c.nx * c.ny * c.nz;
    const double* x = s.U + F.off;
    const double* rhs = s.F + F.off;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int I = t & (c.nx - 1), r = t >> C.lx;
        const int J = r & (c.ny - 1), K = r >> C.ly;
        double acc = 0.0;
#pragma unroll 1
        for (int d = 0; d < 2; d++)
#pragma unroll 1
            for (int bb = 0; bb < 2; bb++)
#pragma unroll
                for (int aa = 0; aa < 2; aa++) {
                    const int i = 2 * I + aa, j = 2 * J + bb, k = 2 * K + d;
                    const int cf = (((k << F.ly) + j) << F.lx) + i;
                    acc += rhs[cf] - op_acc(f, x, cf, i, j, k, a, F.bh2);
                }
        s.F[C.off + t] = acc / 8.0;
        s.U[C.off + t] = 0.0;
    }
    __syncthreads();
}

// A8 P0: f.U += C.U(parent)
__device__ __forceinline__ void interp_p0(const CLevel& F, const CLevel& C, const Sh& s) {
    const PV& f = F.v;
    const PV& c = C.v;
    const int n = f.nx * f.ny * f.nz;
    double* y = s.U + F.off;
    const double* e = s.U + C.off;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int i = t & (f.nx - 1), r = t >> F.lx;
        const int j = r & (f.ny - 1), k = r >> F.ly;
        y[t] = y[t] + e[((((k >> 1) << C.ly) + (j >> 1)) << C.lx) + (i >> 1)];
    }
    __syncthreads();
}

// R-8: U = A^-1 F on the bottom level (<= 64 cells)
__device__ __forceinline__ void bottom(const CLevel& B, const Sh& s, const double* __restrict__ ainv) {
    const int n = B.v.nx * B.v.ny * B.v.nz;
    const int r = threadIdx.x;
    if (r < n) {
        double acc = 0.0;
        for (int c = 0; c < n; c++) acc += __ldg(ainv + r * n + c) * s.F[B.off + c];
        s.U[B.off + r] = acc;
    }
    __syncthreads();
}

// compact shared <-> padded global copies of one field of a level
__device__ __forceinline__ void load_field(const CLevel& L, const double* __restrict__ g, double* sh) {
    const PV& v = L.v;
    const int n = v.nx * v.ny * v.nz;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int i = t & (v.nx - 1), r = t >> L.lx;
        sh[t] = g[sf_ix(v, i, r & (v.ny - 1), r >> L.ly)];
    }
}

__global__ void __launch_bounds__(CNT, 1) coarse_vcycle_kernel(const __grid_constant__ CoarseArgs A) {
    extern __shared__ double csm[];
    Sh s{csm, csm + CSMEM_CELLS, csm + 2 * CSMEM_CELLS};
    pdl_wait();
    const int nl = A.nlev;
    for (int l = 0; l < nl; l++) load_field(A.lv[l], A.lv[l].v.f[SF_DINV], s.D + A.lv[l].off);
    load_field(A.lv[0], A.lv[0].v.f[SF_F], s.F + A.lv[0].off);
    load_field(A.lv[0], A.lv[0].v.f[SF_U], s.U + A.lv[0].off);
    __syncthreads();
    for (int l = 0; l + 1 < nl; l++) {
        smooth(A.lv[l], s, A.a, A.pre);
        residual_restrict(A.lv[l], A.lv[l + 1], s, A.a);
    }
    bottom(A.lv[nl - 1], s, A.ainv);
    for (int l = nl - 2; l >= 0; l--) {
        interp_p0(A.lv[l], A.lv[l + 1], s);
        smooth(A.lv[l], s, A.a, A.post);
    }
    const PV& v = A.lv[0].v;
    const int n = v.nx * v.ny * v.nz;
    for (int t = threadIdx.x; t < n; t += CNT) {
        const int i = t & (v.nx - 1), r = t >> A.lv[0].lx;
        v.f[SF_U][sf_ix(v, i, r & (v.ny - 1), r >> A.lv[0].ly)] = s.U[A.lv[0].off + t];
    }
}

constexpr size_t CSMEM = 3 * CSMEM_CELLS * sizeof(double);

}  // namespace

int coarse_vcycle_max_levels() { return CMAXL; }

// a V-cycle from lv[0] over n levels fits the kernel's shared arrays
bool coarse_vcycle_fits(sf_level* const* lv, int n) {
    if (n < 2 || n > CMAXL) return false;
    long cells = 0;
    auto pow2 = [](int v) { return v >= 1 && (v & (v - 1)) == 0; };
    for (int l = 0; l < n; l++) {
        if (lv[l]->nparts != 1 || lv[l]->nlocal != 1) return false;
        if (!pow2(lv[l]->nx) || !pow2(lv[l]->ny) || !pow2(lv[l]->lnz) || lv[l]->nx < 2) return false;
        cells += (long)lv[l]->nx * lv[l]->ny * lv[l]->lnz;
    }
    return (long)lv[0]->nx * lv[0]->ny * lv[0]->lnz <= CMAX_CELLS && cells <= CSMEM_CELLS;
}

// V(lv[0]) down to the bottom lv[n-1] and back, one single-CTA launch
sf_status k_coarse_vcycle(sf_level* const* lv, int n, double a, double b, const double* ainv,
                          int pre, int post) {
    if (!coarse_vcycle_fits(lv, n)) return sf_fail(SF_ERR_SHAPE, "coarse V-cycle levels do not fit");
    static bool attr = false;
    if (!attr) {
        SF_CUDA(cudaFuncSetAttribute(coarse_vcycle_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)CSMEM));
        attr = true;
    }
    CoarseArgs A = {};
    int off = 0;
    for (int l = 0; l < n; l++) {
        A.lv[l].v = sf_view(lv[l], 0);
        A.lv[l].bh2 = b / (lv[l]->h * lv[l]->h);
        A.lv[l].off = off;
        A.lv[l].lx = __builtin_ctz(lv[l]->nx);
        A.lv[l].ly = __builtin_ctz(lv[l]->ny);
        A.lv[l].lz = __builtin_ctz(lv[l]->lnz);
        off += lv[l]->nx * lv[l]->ny * lv[l]->lnz;
    }
    A.nlev = n;
    A.pre = pre;
    A.post = post;
    A.a = a;
    A.ainv = ainv;
    SF_CUDA(sf_launch(coarse_vcycle_kernel, 1, CNT, CSMEM, lv[0]->stream, A));
    SF_LAUNCHED();
    return sf_check_launch("coarse_vcycle");
}
