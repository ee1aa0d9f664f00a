// Coarse-level V-cycle in ONE launch (A9 below the bandwidth-bound levels).
//
// Levels of 32^3 cells and fewer are latency-bound: every colour sweep,
// residual + restriction, P0 interpolation and the bottom solve of V(l)
// (A5-A9) is a few microseconds of work
// behind a launch and a drain of its own -- ~40 launches per V-cycle below
// 64^3.  Here one thread-block CLUSTER (16 CTAs x 512 threads on 16 SMs, 8 if
// the device refuses 16) runs the whole V(l0) .. bottom .. V(l0) recursion:
// each phase spreads the cells of its level over all threads of the cluster,
// and phases are separated by the hardware cluster barrier
// (barrier.cluster.arrive.release / wait.acquire) instead of kernel
// boundaries.  The levels stay in L2 (a 32^3 level is ~0.5 MB per field);
// values written in one phase and read in a later one go through L2 (.cg
// loads / stores), the static coefficients (alpha, beta, Dinv) may be cached
// in L1.
//
// Arithmetic: the colour sweep is gsrb_colour_kernel's update
// x += Dinv (rhs - A x) with op_at (cell_ops.cuh, the same definition), the
// residual + restriction sums rhs - A x over the 8 children in restrict_cell's
// order, P0 adds the parent, the bottom applies the exact inverse as
// bottom_solve_kernel does.  Single-part levels only (replicated coarse levels
// of a slab decomposition run redundantly on every rank, as before).
#include <cstdlib>

#include "sf_internal.h"

namespace {

#include "cell_ops.cuh"

constexpr int CMAXL = 12;    // levels per launch (32^3 .. 2^3 is 5)
constexpr int CNT = 512;     // threads per CTA

struct CoarseArgs {
    PV lv[CMAXL];
    double bh2[CMAXL];
    int nlev;                // lv[0] = V's entry level, lv[nlev-1] = bottom
    int pre, post;           // RB pairs
    double a;
    const double* ainv;      // exact inverse of the bottom operator (n x n)
};

__device__ __forceinline__ void cluster_barrier() {
    asm volatile(
        "barrier.cluster.arrive.release.aligned;\n\t"
        "barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ unsigned cl_rank() {
    unsigned r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ unsigned cl_size() {
    unsigned r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}

// one colour sweep of A5 on a single-part level (z0 = 0)
__device__ __forceinline__ void sweep(const PV& v, double a, double bh2, int colour, int g, int G) {
    const int hx = (v.nx + 1) >> 1;
    const int n = hx * v.ny * v.nz;
    double* x = v.f[SF_U];
    const double* rhs = v.f[SF_F];
    for (int t = g; t < n; t += G) {
        const int th = t % hx, r = t / hx;
        const int j = r % v.ny, k = r / v.ny;
        const int i = 2 * th + ((j + k + colour) & 1);
        if (i >= v.nx) continue;
        const long c = sf_ix(v, i, j, k);
        const double ax = op_at<true>(v, x, i, j, k, a, bh2);
        __stcg(x + c, __ldcg(x + c) + v.f[SF_DINV][c] * (__ldcg(rhs + c) - ax));
    }
}

__device__ __forceinline__ void smooth(const PV& v, double a, double bh2, int pairs, int g, int G) {
    for (int p = 0; p < pairs; p++) {
        sweep(v, a, bh2, 0, g, G);
        cluster_barrier();
        sweep(v, a, bh2, 1, g, G);
        cluster_barrier();
    }
}

// A6 + A7: C.F = R_cell(F - A U) of the fine level, and C.U = 0 (next V's start)
__device__ __forceinline__ void residual_restrict(const PV& f, const PV& c, double a, double bh2,
                                                  int g, int G) {
    const int n = c.nx * c.ny * c.nz;
    const double* x = f.f[SF_U];
    const double* rhs = f.f[SF_F];
    for (int t = g; t < n; t += G) {
        const int I = t % c.nx, r = t / c.nx;
        const int J = r % c.ny, K = r / c.ny;
        double s = 0.0;
#pragma unroll
        for (int d = 0; d < 2; d++)
#pragma unroll
            for (int bb = 0; bb < 2; bb++)
#pragma unroll
                for (int aa = 0; aa < 2; aa++) {
                    const int i = 2 * I + aa, j = 2 * J + bb, k = 2 * K + d;
                    s += __ldcg(rhs + sf_ix(f, i, j, k)) - op_at<true>(f, x, i, j, k, a, bh2);
                }
        const long q = sf_ix(c, I, J, K);
        __stcg(c.f[SF_F] + q, s / 8.0);
        __stcg(c.f[SF_U] + q, 0.0);
    }
}

// A8 P0: f.U += C.U(parent)
__device__ __forceinline__ void interp_p0(const PV& f, const PV& c, int g, int G) {
    const int n = f.nx * f.ny * f.nz;
    double* y = f.f[SF_U];
    for (int t = g; t < n; t += G) {
        const int i = t % f.nx, r = t / f.nx;
        const int j = r % f.ny, k = r / f.ny;
        const long q = sf_ix(f, i, j, k);
        const double p = __ldcg(c.f[SF_U] + sf_ix(c, i >> 1, j >> 1, k >> 1));
        __stcg(y + q, __ldcg(y + q) + p);
    }
}

// R-8: U = A^-1 F on the bottom level (<= 64 cells), first CTA of the cluster
__device__ __forceinline__ void bottom(const PV& v, const double* __restrict__ ainv) {
    const int n = v.nx * v.ny * v.nz;
    const int r = threadIdx.x;
    if (cl_rank() != 0 || r >= n) return;
    double s = 0.0;
    for (int c = 0; c < n; c++) {
        const int i = c % v.nx, j = (c / v.nx) % v.ny, k = c / (v.nx * v.ny);
        s += ainv[r * n + c] * __ldcg(v.f[SF_F] + sf_ix(v, i, j, k));
    }
    const int i = r % v.nx, j = (r / v.nx) % v.ny, k = r / (v.nx * v.ny);
    __stcg(v.f[SF_U] + sf_ix(v, i, j, k), s);
}

__global__ void __launch_bounds__(CNT, 1) coarse_vcycle_kernel(const __grid_constant__ CoarseArgs A) {
    pdl_wait();
    const int g = (int)(cl_rank() * blockDim.x + threadIdx.x);
    const int G = (int)(cl_size() * blockDim.x);
    const int nl = A.nlev;
    for (int l = 0; l + 1 < nl; l++) {
        smooth(A.lv[l], A.a, A.bh2[l], A.pre, g, G);
        residual_restrict(A.lv[l], A.lv[l + 1], A.a, A.bh2[l], g, G);
        cluster_barrier();
    }
    bottom(A.lv[nl - 1], A.ainv);
    cluster_barrier();
    for (int l = nl - 2; l >= 0; l--) {
        interp_p0(A.lv[l], A.lv[l + 1], g, G);
        cluster_barrier();
        smooth(A.lv[l], A.a, A.bh2[l], A.post, g, G);
    }
}

int g_cluster = 0;   // CTAs per cluster the device accepts (16, else 8); -1: none

int cluster_ctas() {
    if (g_cluster) return g_cluster;
    const char* e = getenv("SF_COARSE_CLUSTER");
    for (int want : {16, 8}) {
        if (e && atoi(e) > 0 && atoi(e) != want) continue;
        if (want > 8 && cudaFuncSetAttribute(coarse_vcycle_kernel,
                                             cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess) {
            cudaGetLastError();
            continue;
        }
        cudaLaunchConfig_t c = {};
        c.gridDim = dim3(want);
        c.blockDim = dim3(CNT);
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = want;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        c.attrs = at;
        c.numAttrs = 1;
        int n = 0;
        if (cudaOccupancyMaxActiveClusters(&n, coarse_vcycle_kernel, &c) == cudaSuccess && n >= 1) {
            g_cluster = want;
            return g_cluster;
        }
        cudaGetLastError();
    }
    g_cluster = -1;
    return g_cluster;
}

}  // namespace

bool coarse_vcycle_available() { return cluster_ctas() > 0; }

int coarse_vcycle_max_levels() { return CMAXL; }

// V(lv[0]) down to the bottom lv[n-1] and back, one cluster launch on stream s
sf_status k_coarse_vcycle(sf_level* const* lv, int n, double a, double b, const double* ainv,
                          int pre, int post) {
    if (n < 1 || n > CMAXL) return sf_fail(SF_ERR_INVALID, "coarse V-cycle over %d levels", n);
    const int cl = cluster_ctas();
    if (cl <= 0) return sf_fail(SF_ERR_CUDA, "thread-block clusters unavailable");
    CoarseArgs A = {};
    for (int l = 0; l < n; l++) {
        if (lv[l]->nparts != 1 || lv[l]->nlocal != 1)
            return sf_fail(SF_ERR_SHAPE, "coarse V-cycle needs single-part levels");
        A.lv[l] = sf_view(lv[l], 0);
        A.bh2[l] = b / (lv[l]->h * lv[l]->h);
    }
    A.nlev = n;
    A.pre = pre;
    A.post = post;
    A.a = a;
    A.ainv = ainv;
    cudaLaunchConfig_t c = {};
    c.gridDim = dim3(cl);
    c.blockDim = dim3(CNT);
    c.stream = lv[0]->stream;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cl;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = 1;
    c.attrs = at;
    c.numAttrs = sf_pdl_on() ? 2 : 1;
    SF_CUDA(cudaLaunchKernelEx(&c, coarse_vcycle_kernel, A));
    SF_LAUNCHED();
    return sf_check_launch("coarse_vcycle");
}
