// Coarse-level V-cycle in ONE launch of ONE thread-block cluster (A9 on the
// smallest levels).
//
// Levels of 32^3 cells and fewer are pure latency: every colour sweep,
// residual + restriction, P0 interpolation and the bottom solve of V(l)
// (A5-A9) is a few microseconds of work
// behind a launch of its own -- ~40 launches per V-cycle below 64^3.  Here one
// cluster of C = nz/2 CTAs (entry level nz <= 32: up to 16 CTAs, one per SM,
// the non-portable cluster size where the device schedules it) runs the whole
// V(l0) .. bottom .. V(l0) recursion with every operand in REGISTERS or SHARED
// MEMORY; phases are separated by cluster barriers and the z-neighbours that
// live in the next CTA are read through distributed shared memory (DSMEM).
// After one staging pass no phase touches global memory.
//
// Ownership: on every distributed level CTA c owns the 2-plane layer of 2x2x2
// blocks whose parents form coarse plane c (planes 2c, 2c+1), so the
// restriction of a block and the P0 correction of its cells involve only the
// block's CTA and the owner of the parent plane (CTA c/2 on the next
// distributed level).  The coarsest levels (<= 512 cells, and the bottom) are
// GATHERED whole on CTA 0, which runs their part of the cycle alone with
// __syncthreads (a cluster barrier per phase would cost more than their work).
//
// Entry level: thread t of CTA c owns block t of the layer and keeps its
// 8 x values, F, Dinv, alpha and the 36 face coefficients of the block in
// registers; its x values are mirrored in shared memory for the neighbours'
// reads.  Levels below: one thread per cell, U / F / Dinv / alpha and the
// faces in shared memory.
//
// Arithmetic: the colour sweep is the fused pairs' lambda-form update
// x = Dinv (F + b h^-2 S) (sum6 / gs_upd of tma_common.cuh),
// a restatement of x += Dinv (F - A x) equal up to rounding; the residual of
// the restriction is op_at's expression (cell_ops.cuh: same terms, order and
// Dirichlet fold), summed over the 8 children in restrict_cell's order and
// divided by 8; P0 adds the parent; the bottom applies the exact inverse in
// bottom_solve_kernel's order.  The first red sweep of every level below the
// entry rides in the restriction that produced its F (from U = 0 it is
// x = Dinv F exactly).
#include <cooperative_groups.h>
#include <cuda.h>

#include <algorithm>
#include <cstdlib>

#include "sf_internal.h"

namespace cg = cooperative_groups;

namespace {

#include "tma_common.cuh"   // sum6 / gs_upd: the lambda-form update of the fused pairs

constexpr int CMAXL = 8;                 // levels per launch
constexpr int NT = 256;                  // threads per CTA (entry blocks per layer at most)
constexpr int CS_MAX = 16;               // CTAs per cluster (non-portable above 8)
constexpr int BOT_MAX = 64;              // bottom cells (plan_levels: <= 64)
constexpr int GMAX = 2 * NT;             // levels of at most this many cells are gathered on CTA 0
constexpr int CSMEM_MAX = 225 * 1024;    // opt-in shared memory per CTA (2 KB for static use)

struct KLevel {
    PV v;                 // global view: coefficients; the entry level's U / F / Dinv
    double bh2;
    int lx, ly, lz;       // log2 of nx, ny, nz (power-of-two levels)
    int u, f, d, al;      // shared offsets (doubles) of U, F, Dinv, alpha: the CTA's two planes
    int bi, bj, bk;       // (gathered: every plane, on CTA 0; bottom: U and F only); faces
    int g;                // gathered on CTA 0 (the coarsest levels, <= GMAX cells)
};

struct KArgs {
    KLevel lv[CMAXL];
    int nlev;             // lv[0] = entry, lv[nlev-1] = bottom
    int pre, post;        // RB pairs
    double a;
    int ainv;             // shared offset of the bottom inverse (CTA 0)
    int rscr;             // shared offset of the residual scratch (GMAX doubles)
    int uzero;            // the entry level's U is zero (V-cycle): not read
    int trig;             // let the next launch start early (it reads only our U of the entry)
    const double* ainv_g; // n x n, row major
};

// A3 at one cell from its value, its six neighbours (Dirichlet ghosts already
// folded in as -xc) and its six faces: op_at's expression term by term.
__device__ __forceinline__ double op7(double xc, double xw, double xe, double xs, double xn,
                                     double xb, double xt, double bw, double be, double bs,
                                     double bn, double bb, double bt, double al, double a,
                                     double bh2) {
    double flux = be * (xe - xc);
    flux += bw * (xw - xc);
    flux += bn * (xn - xc);
    flux += bs * (xs - xc);
    flux += bt * (xt - xc);
    flux += bb * (xb - xc);
    return a * al * xc - bh2 * flux;
}

// shared memory of this CTA and of its z-neighbours (DSMEM, generic pointers)
struct Mem {
    double* sm;
    double* lo;   // CTA rank-1 (planes below), nullptr at rank 0
    double* hi;   // CTA rank+1
    int rank, csize;
    // shared memory of the CTA that owns plane p of the next level (gathered: CTA 0)
    __device__ __forceinline__ double* owner(cg::cluster_group& cl, int p, bool gathered) const {
        const int r = gathered ? 0 : p >> 1;
        return r == rank ? sm : cl.map_shared_rank(sm, r);
    }
};

#ifdef SF_COARSE_TRACE   // phase clock trace (measurement builds only)
__shared__ long long trace_t[128];
__shared__ int trace_n;
#define TRACE()                                                     \
    do {                                                            \
        if (threadIdx.x == 0 && trace_n < 128) trace_t[trace_n++] = clock64(); \
    } while (0)
#else
#define TRACE() \
    do {        \
    } while (0)
#endif

__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::
                     : "memory");
    TRACE();
}

// ------------------------------------------------------------ entry level
struct Block {
    bool own;
    int i0, j0;                 // block origin (k0 = 2 * rank)
    double X[8], F[8], D[8], A[8];
    double BI[3][2][2];         // beta_i faces i0..i0+2 at (dj, dk)
    double BJ[3][2][2];         // beta_j faces j0..j0+2 at (di, dk)
    double BK[3][2][2];         // beta_k faces k0..k0+2 at (di, dj)
};

// GS update of sub-cell s in lambda form, x = Dinv (F + b h^-2 S) with S the
// beta-weighted sum of the neighbours (a Dirichlet ghost contributes 0: its
// -x(c) is part of the diagonal) -- the fused pairs' update (sum6 / gs_upd)
__device__ __forceinline__ double upd_block(const KLevel& L, const Mem& M, const Block& B, int s) {
    const int di = s & 1, dj = (s >> 1) & 1, dk = s >> 2;
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int i = B.i0 + di, j = B.j0 + dj, k = 2 * M.rank + dk;
    const double* U = M.sm + L.u;
    const int cp = i + (j << L.lx);
    const int c = cp + (dk << (L.lx + L.ly));
    double xw, xe, xs, xn, xb, xt;
    if (di) { xw = B.X[s - 1]; xe = (i == nx - 1) ? 0.0 : U[c + 1]; }
    else    { xe = B.X[s + 1]; xw = (i == 0) ? 0.0 : U[c - 1]; }
    if (dj) { xs = B.X[s - 2]; xn = (j == ny - 1) ? 0.0 : U[c + nx]; }
    else    { xn = B.X[s + 2]; xs = (j == 0) ? 0.0 : U[c - nx]; }
    if (dk) { xb = B.X[s - 4]; xt = (k == nz - 1) ? 0.0 : (M.hi + L.u)[cp]; }
    else    { xt = B.X[s + 4]; xb = (k == 0) ? 0.0 : (M.lo + L.u)[cp + (1 << (L.lx + L.ly))]; }
    return gs_upd(B.D[s], B.F[s], L.bh2,
                  sum6(xw, xe, xs, xn, xb, xt, B.BI[di][dj][dk], B.BI[di + 1][dj][dk], B.BJ[dj][di][dk],
                       B.BJ[dj + 1][di][dk], B.BK[dk][di][dj], B.BK[dk + 1][di][dj]));
}

// A x at sub-cell s = di + 2 dj + 4 dk of the block, with the block's current x
__device__ __forceinline__ double op_block(const KLevel& L, const Mem& M, const Block& B, int s,
                                           double a) {
    const int di = s & 1, dj = (s >> 1) & 1, dk = s >> 2;
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int i = B.i0 + di, j = B.j0 + dj, k = 2 * M.rank + dk;
    const double xc = B.X[s];
    const double* U = M.sm + L.u;
    const int cp = i + (j << L.lx);                   // in-plane offset
    const int c = cp + (dk << (L.lx + L.ly));         // local cell (plane dk of the CTA)
    double xw, xe, xs, xn, xb, xt;
    if (di) { xw = B.X[s - 1]; xe = (i == nx - 1) ? -xc : U[c + 1]; }
    else    { xe = B.X[s + 1]; xw = (i == 0) ? -xc : U[c - 1]; }
    if (dj) { xs = B.X[s - 2]; xn = (j == ny - 1) ? -xc : U[c + nx]; }
    else    { xn = B.X[s + 2]; xs = (j == 0) ? -xc : U[c - nx]; }
    if (dk) { xb = B.X[s - 4]; xt = (k == nz - 1) ? -xc : (M.hi + L.u)[cp]; }
    else    { xt = B.X[s + 4]; xb = (k == 0) ? -xc : (M.lo + L.u)[cp + (1 << (L.lx + L.ly))]; }
    return op7(xc, xw, xe, xs, xn, xb, xt, B.BI[di][dj][dk], B.BI[di + 1][dj][dk], B.BJ[dj][di][dk],
               B.BJ[dj + 1][di][dk], B.BK[dk][di][dj], B.BK[dk + 1][di][dj], B.A[s], a, L.bh2);
}

__device__ __forceinline__ void sweep_entry(const KLevel& L, const Mem& M, Block& B, double a,
                                            int colour) {
    if (B.own) {
        double* U = M.sm + L.u;
        // every operator value first (the colour's cells read only the other
        // colour), then the updates: the neighbour loads -- one of them from the
        // next CTA -- are all in flight together
        double xnew[8];
#pragma unroll
        for (int s = 0; s < 8; s++)
            if ((((s & 1) + ((s >> 1) & 1) + (s >> 2)) & 1) == colour) xnew[s] = upd_block(L, M, B, s);
#pragma unroll
        for (int s = 0; s < 8; s++) {
            const int di = s & 1, dj = (s >> 1) & 1, dk = s >> 2;
            if (((di + dj + dk) & 1) != colour) continue;   // block origin is even
            B.X[s] = xnew[s];
            U[B.i0 + di + ((B.j0 + dj + (dk << L.ly)) << L.lx)] = B.X[s];
        }
    }
    cluster_sync();
}

// ------------------------------------------------------------ levels below
// A x at (i, j, plane kl of this CTA) of a non-entry level in shared memory
__device__ __forceinline__ double op_cell(const KLevel& L, const Mem& M, int i, int j, int kl,
                                          double xc, double a) {
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int k = 2 * M.rank + kl;
    const double* U = M.sm + L.u;
    const int pl = 1 << (L.lx + L.ly);
    const int cp = i + (j << L.lx), c = cp + kl * pl;
    const double xw = (i == 0) ? -xc : U[c - 1];
    const double xe = (i == nx - 1) ? -xc : U[c + 1];
    const double xs = (j == 0) ? -xc : U[c - nx];
    const double xn = (j == ny - 1) ? -xc : U[c + nx];
    double xb, xt;
    if (kl) { xb = U[cp]; xt = (k == nz - 1) ? -xc : (M.hi + L.u)[cp]; }
    else    { xt = U[cp + pl]; xb = (k == 0) ? -xc : (M.lo + L.u)[cp + pl]; }
    const double* bi = M.sm + L.bi + i + (nx + 1) * (j + (kl << L.ly));
    const double* bj = M.sm + L.bj + i + ((j + (ny + 1) * kl) << L.lx);
    const double* bk = M.sm + L.bk + c;
    return op7(xc, xw, xe, xs, xn, xb, xt, bi[0], bi[1], bj[0], bj[nx], bk[0], bk[pl],
               M.sm[L.al + c], a, L.bh2);
}

// lambda-form GS update at (i, j, plane kl of this CTA) of a non-entry level
__device__ __forceinline__ double upd_cell(const KLevel& L, const Mem& M, int i, int j, int kl) {
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int k = 2 * M.rank + kl;
    const double* U = M.sm + L.u;
    const int pl = 1 << (L.lx + L.ly);
    const int cp = i + (j << L.lx), c = cp + kl * pl;
    const double xw = (i == 0) ? 0.0 : U[c - 1];
    const double xe = (i == nx - 1) ? 0.0 : U[c + 1];
    const double xs = (j == 0) ? 0.0 : U[c - nx];
    const double xn = (j == ny - 1) ? 0.0 : U[c + nx];
    double xb, xt;
    if (kl) { xb = U[cp]; xt = (k == nz - 1) ? 0.0 : (M.hi + L.u)[cp]; }
    else    { xt = U[cp + pl]; xb = (k == 0) ? 0.0 : (M.lo + L.u)[cp + pl]; }
    const double* bi = M.sm + L.bi + i + (nx + 1) * (j + (kl << L.ly));
    const double* bj = M.sm + L.bj + i + ((j + (ny + 1) * kl) << L.lx);
    const double* bk = M.sm + L.bk + c;
    return gs_upd(M.sm[L.d + c], M.sm[L.f + c], L.bh2,
                  sum6(xw, xe, xs, xn, xb, xt, bi[0], bi[1], bj[0], bj[nx], bk[0], bk[pl]));
}

// one colour sweep: thread t updates the t-th cell of the colour in the CTA's two planes
__device__ __forceinline__ void sweep_cells(const KLevel& L, const Mem& M, double a, int colour) {
    if (M.rank < (1 << (L.lz - 1))) {
        const int lh = L.lx - 1;
        const int n = 1 << (lh + L.ly + 1);   // cells of one colour in two planes
        double* U = M.sm + L.u;
        for (int t = threadIdx.x; t < n; t += NT) {
            const int th = t & ((1 << lh) - 1), r = t >> lh;
            const int j = r & ((1 << L.ly) - 1), kl = r >> L.ly;
            const int i = 2 * th + ((j + kl + colour) & 1);   // plane 2*rank+kl: parity of kl
            U[i + ((j + (kl << L.ly)) << L.lx)] = upd_cell(L, M, i, j, kl);
        }
    }
    cluster_sync();
}

// skip_red: the first red sweep was folded into the restriction that produced
// this level's F (from U = 0 it is x = Dinv F exactly, see residual_restrict)
__device__ __forceinline__ void smooth(const KLevel& L, const Mem& M, Block* B, double a, int pairs,
                                       bool skip_red = false) {
    for (int p = 0; p < pairs; p++) {
        if (B) {
            sweep_entry(L, M, *B, a, 0);
            sweep_entry(L, M, *B, a, 1);
        } else {
            if (p > 0 || !skip_red) sweep_cells(L, M, a, 0);
            sweep_cells(L, M, a, 1);
        }
    }
}

// U of a coarse cell after the restriction: 0, or with `fold` the first red
// sweep of its pre-smoothing from U = 0: a red cell's neighbours are all 0, so
// the lambda-form update is gs_upd(Dinv, F, b h^-2, 0) = Dinv F exactly and a
// black cell stays 0 -- one phase less per level
__device__ __forceinline__ double u_after_restrict(bool fold, bool red, double dinv, double f,
                                                   double bh2) {
    return (fold && red) ? gs_upd(dinv, f, bh2, 0.0) : 0.0;
}

// coarse cell (I, J) of plane `rank` of level C: its slot in the owner's shared memory
__device__ __forceinline__ int coarse_slot(const KLevel& C, const Mem& M, int I, int J, bool cgat) {
    const int kl = cgat ? M.rank : (M.rank & 1);
    return I + ((J + (kl << C.ly)) << C.lx);
}

// A6 + A7: C.F = R_cell(F - A U) for the CTA's layer of blocks (coarse plane
// `rank`), C.U = 0; written into the owner of that coarse plane
__device__ __forceinline__ void residual_restrict(cg::cluster_group& cl, const KLevel& F,
                                                  const KLevel& C, const Mem& M, const Block* B,
                                                  double a, bool cgat, int rscr, bool fold) {
    if (M.rank < (1 << (F.lz - 1))) {
        double* dst = M.owner(cl, M.rank, cgat);
        if (B) {
            if (B->own) {
                double r[8];   // the 8 residuals are independent: evaluated together
#pragma unroll
                for (int s = 0; s < 8; s++) r[s] = B->F[s] - op_block(F, M, *B, s, a);
                double acc = 0.0;
#pragma unroll
                for (int s = 0; s < 8; s++) acc += r[s];
                const int q = coarse_slot(C, M, B->i0 >> 1, B->j0 >> 1, cgat);
                const double fc = acc / 8.0;
                const bool red = (((B->i0 + B->j0) >> 1) + M.rank & 1) == 0;
                dst[C.f + q] = fc;
                dst[C.u + q] = u_after_restrict(fold, red, fold ? dst[C.d + q] : 0.0, fc, C.bh2);
            }
        } else {
            // residual of every cell of the two planes (one thread per cell),
            // then the ordered sums of 8 children (one thread per block)
            double* R = M.sm + rscr;
            const int nc = 1 << (F.lx + F.ly + 1);
            for (int t = threadIdx.x; t < nc; t += NT) {
                const int i = t & ((1 << F.lx) - 1), j = (t >> F.lx) & ((1 << F.ly) - 1);
                const int kl = t >> (F.lx + F.ly);
                R[t] = M.sm[F.f + t] - op_cell(F, M, i, j, kl, M.sm[F.u + t], a);
            }
            __syncthreads();
            const int n = 1 << (F.lx + F.ly - 2);   // blocks of the layer
            for (int t = threadIdx.x; t < n; t += NT) {
                const int I = t & ((1 << (F.lx - 1)) - 1), J = t >> (F.lx - 1);
                double acc = 0.0;
#pragma unroll
                for (int s = 0; s < 8; s++)
                    acc += R[2 * I + (s & 1) + ((2 * J + ((s >> 1) & 1) + ((s >> 2) << F.ly)) << F.lx)];
                const int q = coarse_slot(C, M, I, J, cgat);
                const double fc = acc / 8.0;
                dst[C.f + q] = fc;
                dst[C.u + q] = u_after_restrict(fold, ((I + J + M.rank) & 1) == 0,
                                                fold ? dst[C.d + q] : 0.0, fc, C.bh2);
            }
        }
    }
    cluster_sync();
}

// A8 P0: the CTA's cells += their parent (coarse plane `rank`, in its owner)
__device__ __forceinline__ void interp(cg::cluster_group& cl, const KLevel& F, const KLevel& C,
                                       const Mem& M, Block* B, bool cgat) {
    if (M.rank < (1 << (F.lz - 1))) {
        const double* e = M.owner(cl, M.rank, cgat) + C.u;
        if (B) {
            if (B->own) {
                const double ec = e[coarse_slot(C, M, B->i0 >> 1, B->j0 >> 1, cgat)];
                double* U = M.sm + F.u;
#pragma unroll
                for (int s = 0; s < 8; s++) {
                    B->X[s] = B->X[s] + ec;
                    U[B->i0 + (s & 1) + ((B->j0 + ((s >> 1) & 1) + ((s >> 2) << F.ly)) << F.lx)] = B->X[s];
                }
            }
        } else {
            const int n = 1 << (F.lx + F.ly + 1);   // cells of the two planes
            double* U = M.sm + F.u;
            for (int t = threadIdx.x; t < n; t += NT) {
                const int i = t & ((1 << F.lx) - 1), j = (t >> F.lx) & ((1 << F.ly) - 1);
                U[t] = U[t] + e[coarse_slot(C, M, i >> 1, j >> 1, cgat)];
            }
        }
    }
    cluster_sync();
}

// ------------------------------------------------------------ gathered levels
// The coarsest levels (<= GMAX cells) live whole on CTA 0, which runs their
// part of the V-cycle alone with __syncthreads between phases (a cluster
// barrier per phase would cost more than their work); the other CTAs wait at
// the next cluster barrier.  One thread per cell of a colour / coarse cell.

// A x at (i, j, k) of a gathered level
__device__ __forceinline__ double op_g(const KLevel& L, const double* sm, int i, int j, int k,
                                       double xc, double a) {
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int pl = 1 << (L.lx + L.ly);
    const int c = i + ((j + (k << L.ly)) << L.lx);
    const double* U = sm + L.u;
    const double xw = (i == 0) ? -xc : U[c - 1];
    const double xe = (i == nx - 1) ? -xc : U[c + 1];
    const double xs = (j == 0) ? -xc : U[c - nx];
    const double xn = (j == ny - 1) ? -xc : U[c + nx];
    const double xb = (k == 0) ? -xc : U[c - pl];
    const double xt = (k == nz - 1) ? -xc : U[c + pl];
    const double* bi = sm + L.bi + i + (nx + 1) * (j + (k << L.ly));
    const double* bj = sm + L.bj + i + ((j + (ny + 1) * k) << L.lx);
    const double* bk = sm + L.bk + c;
    return op7(xc, xw, xe, xs, xn, xb, xt, bi[0], bi[1], bj[0], bj[nx], bk[0], bk[pl],
               sm[L.al + c], a, L.bh2);
}

// lambda-form GS update at (i, j, k) of a gathered level
__device__ __forceinline__ double upd_g(const KLevel& L, const double* sm, int i, int j, int k) {
    const int nx = 1 << L.lx, ny = 1 << L.ly, nz = 1 << L.lz;
    const int pl = 1 << (L.lx + L.ly);
    const int c = i + ((j + (k << L.ly)) << L.lx);
    const double* U = sm + L.u;
    const double xw = (i == 0) ? 0.0 : U[c - 1];
    const double xe = (i == nx - 1) ? 0.0 : U[c + 1];
    const double xs = (j == 0) ? 0.0 : U[c - nx];
    const double xn = (j == ny - 1) ? 0.0 : U[c + nx];
    const double xb = (k == 0) ? 0.0 : U[c - pl];
    const double xt = (k == nz - 1) ? 0.0 : U[c + pl];
    const double* bi = sm + L.bi + i + (nx + 1) * (j + (k << L.ly));
    const double* bj = sm + L.bj + i + ((j + (ny + 1) * k) << L.lx);
    const double* bk = sm + L.bk + c;
    return gs_upd(sm[L.d + c], sm[L.f + c], L.bh2,
                  sum6(xw, xe, xs, xn, xb, xt, bi[0], bi[1], bj[0], bj[nx], bk[0], bk[pl]));
}

__device__ __forceinline__ void sweep_g(const KLevel& L, double* sm, double a, int colour) {
    const int lh = L.lx - 1;
    const int n = 1 << (lh + L.ly + L.lz);   // cells of one colour
    double* U = sm + L.u;
    for (int t = threadIdx.x; t < n; t += NT) {
        const int th = t & ((1 << lh) - 1), r = t >> lh;
        const int j = r & ((1 << L.ly) - 1), k = r >> L.ly;
        const int i = 2 * th + ((j + k + colour) & 1);
        U[i + ((j + (k << L.ly)) << L.lx)] = upd_g(L, sm, i, j, k);
    }
    __syncthreads();
    TRACE();
}

// C.F = R_cell(F - A U), C.U = 0: one thread per coarse cell
// (residual of every fine cell into the scratch R first, one thread per cell)
__device__ __forceinline__ void restrict_g(const KLevel& F, const KLevel& C, double* sm, double a,
                                           double* R, bool fold) {
    const int nf = 1 << (F.lx + F.ly + F.lz);
    for (int t = threadIdx.x; t < nf; t += NT) {
        const int i = t & ((1 << F.lx) - 1), r = t >> F.lx;
        const int j = r & ((1 << F.ly) - 1), k = r >> F.ly;
        R[t] = sm[F.f + t] - op_g(F, sm, i, j, k, sm[F.u + t], a);
    }
    __syncthreads();
    const int n = 1 << (C.lx + C.ly + C.lz);
    for (int t = threadIdx.x; t < n; t += NT) {
        const int I = t & ((1 << C.lx) - 1), r = t >> C.lx;
        const int J = r & ((1 << C.ly) - 1), K = r >> C.ly;
        double acc = 0.0;
#pragma unroll
        for (int s = 0; s < 8; s++)
            acc += R[2 * I + (s & 1) + ((2 * J + ((s >> 1) & 1) + ((2 * K + (s >> 2)) << F.ly)) << F.lx)];
        const double fc = acc / 8.0;
        sm[C.f + t] = fc;
        sm[C.u + t] = u_after_restrict(fold, ((I + J + K) & 1) == 0, fold ? sm[C.d + t] : 0.0, fc, C.bh2);
    }
    __syncthreads();
    TRACE();
}

// F.U += P0(C.U): one thread per fine cell
__device__ __forceinline__ void interp_g(const KLevel& F, const KLevel& C, double* sm) {
    const int n = 1 << (F.lx + F.ly + F.lz);
    double* U = sm + F.u;
    for (int t = threadIdx.x; t < n; t += NT) {
        const int i = t & ((1 << F.lx) - 1), r = t >> F.lx;
        const int j = r & ((1 << F.ly) - 1), k = r >> F.ly;
        U[t] = U[t] + sm[C.u + (i >> 1) + (((j >> 1) + ((k >> 1) << C.ly)) << C.lx)];
    }
    __syncthreads();
    TRACE();
}

// R-8: U = A^-1 F on the bottom level
__device__ __forceinline__ void bottom_g(const KLevel& Bt, double* sm, int ainv) {
    const int n = 1 << (Bt.lx + Bt.ly + Bt.lz);
    const int r = threadIdx.x;
    if (r < n) {
        double acc = 0.0;
        for (int c = 0; c < n; c++) acc += sm[ainv + r * n + c] * sm[Bt.f + c];
        sm[Bt.u + r] = acc;
    }
    __syncthreads();
    TRACE();
}

// V(l0) .. bottom .. V(l0) over the gathered levels l0..nl-1 (CTA 0 only)
__device__ __forceinline__ void gathered_cycle(const KArgs& A, double* sm, int l0) {
    const int nl = A.nlev;
    const bool fold = A.pre >= 1;   // every level's first red sweep came with its F
    for (int l = l0; l + 1 < nl; l++) {
        for (int p = 0; p < A.pre; p++) {
            if (p > 0 || !fold) sweep_g(A.lv[l], sm, A.a, 0);
            sweep_g(A.lv[l], sm, A.a, 1);
        }
        restrict_g(A.lv[l], A.lv[l + 1], sm, A.a, sm + A.rscr, fold && l + 2 < nl);
    }
    bottom_g(A.lv[nl - 1], sm, A.ainv);
    for (int l = nl - 2; l >= l0; l--) {
        interp_g(A.lv[l], A.lv[l + 1], sm);
        for (int p = 0; p < A.post; p++) {
            sweep_g(A.lv[l], sm, A.a, 0);
            sweep_g(A.lv[l], sm, A.a, 1);
        }
    }
}

// padded global -> compact shared, one 8-byte cp.async per value: 2^lw values
// x 2^lrj rows x rk planes starting at (ioff, joff, koff); shared element
// (i, j, k) at i + sw (j + srj (k - koff)).
__device__ __forceinline__ void stage_box(double* dst, const double* __restrict__ src, int lw, int lrj,
                                          int rk, int ioff, int joff, int koff, int sw, int srj,
                                          long js, long ks) {
    const unsigned d0 = (unsigned)__cvta_generic_to_shared(dst);
    const int n = rk << (lw + lrj);
    for (int e = threadIdx.x; e < n; e += NT) {
        const int i = (e & ((1 << lw) - 1)) + ioff, r = e >> lw;
        const int j = (r & ((1 << lrj) - 1)) + joff, kr = r >> lrj;
        const double* g = src + (long)(kr + koff + SF_GZ) * ks + (long)(j + SF_GY) * js + SF_OX + i;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d0 + 8u * (i + sw * (j + srj * kr))),
                     "l"(g)
                     : "memory");
    }
}

__global__ void __launch_bounds__(NT, 1) coarse_vcycle_kernel(const __grid_constant__ KArgs A) {
    extern __shared__ double sm[];
    cg::cluster_group cl = cg::this_cluster();
    Mem M;
    M.sm = sm;
    M.rank = (int)cl.block_rank();
    M.csize = (int)cl.num_blocks();
    M.lo = M.rank > 0 ? cl.map_shared_rank(sm, M.rank - 1) : nullptr;
    M.hi = M.rank + 1 < M.csize ? cl.map_shared_rank(sm, M.rank + 1) : nullptr;
#ifdef SF_COARSE_NOREMOTE   // timing experiment only: z-neighbours read locally (wrong results)
    M.lo = M.hi = sm;
#endif
#ifdef SF_COARSE_TRACE
    if (threadIdx.x == 0) trace_n = 0;
    __syncthreads();
#endif
    TRACE();
    const int nl = A.nlev;
    const int k0 = 2 * M.rank;
    // Constant operands first -- before griddepcontrol.wait, so with an early
    // trigger in the previous kernel (k_residual_restrict) they load while it
    // still runs; only F and U of the entry are that kernel's output.
    // ---- staging (async): D / alpha / faces of the CTA's planes of every
    // level below the entry, the bottom inverse on CTA 0
    for (int l = 1; l + 1 < nl; l++) {
        const KLevel& L = A.lv[l];
        const PV& v = L.v;
        const int nx = v.nx, ny = v.ny;
        if (L.g) {   // every plane, on CTA 0
            if (M.rank != 0) continue;
            const int nz = v.nz;
            stage_box(sm + L.d, v.f[SF_DINV], L.lx, L.ly, nz, 0, 0, 0, nx, ny, v.js, v.ks);
            stage_box(sm + L.al, v.f[SF_ALPHA], L.lx, L.ly, nz, 0, 0, 0, nx, ny, v.js, v.ks);
            stage_box(sm + L.bi, v.f[SF_BETA_I], L.lx, L.ly, nz, 0, 0, 0, nx + 1, ny, v.js, v.ks);
            stage_box(sm + L.bi, v.f[SF_BETA_I], 0, L.ly, nz, nx, 0, 0, nx + 1, ny, v.js, v.ks);
            stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, L.ly, nz, 0, 0, 0, nx, ny + 1, v.js, v.ks);
            stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, 0, nz, 0, ny, 0, nx, ny + 1, v.js, v.ks);
            stage_box(sm + L.bk, v.f[SF_BETA_K], L.lx, L.ly, nz + 1, 0, 0, 0, nx, ny, v.js, v.ks);
            continue;
        }
        if (M.rank >= (1 << (L.lz - 1))) continue;
        stage_box(sm + L.d, v.f[SF_DINV], L.lx, L.ly, 2, 0, 0, k0, nx, ny, v.js, v.ks);
        stage_box(sm + L.al, v.f[SF_ALPHA], L.lx, L.ly, 2, 0, 0, k0, nx, ny, v.js, v.ks);
        stage_box(sm + L.bi, v.f[SF_BETA_I], L.lx, L.ly, 2, 0, 0, k0, nx + 1, ny, v.js, v.ks);
        stage_box(sm + L.bi, v.f[SF_BETA_I], 0, L.ly, 2, nx, 0, k0, nx + 1, ny, v.js, v.ks);
        stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, L.ly, 2, 0, 0, k0, nx, ny + 1, v.js, v.ks);
        stage_box(sm + L.bj, v.f[SF_BETA_J], L.lx, 0, 2, 0, ny, k0, nx, ny + 1, v.js, v.ks);
        stage_box(sm + L.bk, v.f[SF_BETA_K], L.lx, L.ly, 3, 0, 0, k0, nx, ny, v.js, v.ks);
    }
    if (M.rank == 0) {
        const KLevel& Bt = A.lv[nl - 1];
        const int n = 1 << (Bt.lx + Bt.ly + Bt.lz);
        const unsigned d0 = (unsigned)__cvta_generic_to_shared(sm + A.ainv);
        for (int e = threadIdx.x; e < n * n; e += NT)
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d0 + 8u * e), "l"(A.ainv_g + e)
                         : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    // ---- the entry block of this thread into registers: Dinv, alpha, faces
    const KLevel& E = A.lv[0];
    const PV& ev = E.v;
    Block B;
    B.own = threadIdx.x < (1 << (E.lx - 1 + E.ly - 1));
    B.i0 = 2 * (threadIdx.x & ((1 << (E.lx - 1)) - 1));
    B.j0 = 2 * (threadIdx.x >> (E.lx - 1));
    const long q0 = sf_ix(ev, B.i0, B.j0, k0);
    // 16-byte loads of x-adjacent pairs (i0 even, rows 32-byte aligned): a warp
    // reads whole contiguous row segments
    auto ld2 = [&](int f, long q) {
        return B.own ? __ldg((const double2*)(ev.f[f] + q)) : make_double2(0.0, 0.0);
    };
    auto ld1 = [&](int f, long q) { return B.own ? __ldg(ev.f[f] + q) : 0.0; };
#pragma unroll
    for (int r = 0; r < 4; r++) {   // rows (dj, dk) = (r & 1, r >> 1): sub-cells 2r, 2r+1
        const long q = q0 + (r & 1) * ev.js + (r >> 1) * ev.ks;
        double2 t2 = ld2(SF_DINV, q);
        B.D[2 * r] = t2.x; B.D[2 * r + 1] = t2.y;
        t2 = ld2(SF_ALPHA, q);
        B.A[2 * r] = t2.x; B.A[2 * r + 1] = t2.y;
        // beta_i faces i0, i0+1 (pair) and i0+2 at (dj, dk) = (r & 1, r >> 1)
        t2 = ld2(SF_BETA_I, q);
        B.BI[0][r & 1][r >> 1] = t2.x; B.BI[1][r & 1][r >> 1] = t2.y;
        B.BI[2][r & 1][r >> 1] = ld1(SF_BETA_I, q + 2);
    }
#pragma unroll
    for (int f = 0; f < 3; f++)
#pragma unroll
        for (int r = 0; r < 2; r++) {
            // beta_j face j0+f at dk = r, beta_k face k0+f at dj = r: di = 0, 1 as a pair
            double2 t2 = ld2(SF_BETA_J, q0 + f * ev.js + r * ev.ks);
            B.BJ[f][0][r] = t2.x; B.BJ[f][1][r] = t2.y;
            t2 = ld2(SF_BETA_K, q0 + r * ev.js + f * ev.ks);
            B.BK[f][0][r] = t2.x; B.BK[f][1][r] = t2.y;
        }
    pdl_wait();   // the previous kernel's output from here on
    if (A.trig) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    TRACE();
    // ---- the entry's F and U (registers; U mirrored in shared memory)
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const long q = q0 + (r & 1) * ev.js + (r >> 1) * ev.ks;
        double2 t2 = A.uzero ? make_double2(0.0, 0.0) : ld2(SF_U, q);
        B.X[2 * r] = t2.x; B.X[2 * r + 1] = t2.y;
        t2 = ld2(SF_F, q);
        B.F[2 * r] = t2.x; B.F[2 * r + 1] = t2.y;
    }
    if (B.own) {
        double* U = sm + E.u;
#pragma unroll
        for (int s = 0; s < 8; s++)
            U[B.i0 + (s & 1) + ((B.j0 + ((s >> 1) & 1) + ((s >> 2) << E.ly)) << E.lx)] = B.X[s];
    }
    cluster_sync();
    // ---- V(l0) down to the bottom and back
    smooth(E, M, &B, A.a, A.pre);
    asm volatile("cp.async.wait_all;" ::: "memory");   // staged levels visible after the next barrier
    const bool fold = A.pre >= 1;   // first red sweep of each coarser level folded into its restriction
    residual_restrict(cl, E, A.lv[1], M, &B, A.a, A.lv[1].g, A.rscr, fold && nl > 2);
    int lg = 1;   // first gathered level
    for (; !A.lv[lg].g; lg++) {
        smooth(A.lv[lg], M, nullptr, A.a, A.pre, fold);
        residual_restrict(cl, A.lv[lg], A.lv[lg + 1], M, nullptr, A.a, A.lv[lg + 1].g, A.rscr,
                          fold && lg + 2 < nl);
    }
    if (M.rank == 0) gathered_cycle(A, sm, lg);
    TRACE();
    cluster_sync();
    for (int l = lg - 1; l >= 1; l--) {
        interp(cl, A.lv[l], A.lv[l + 1], M, nullptr, A.lv[l + 1].g);
        smooth(A.lv[l], M, nullptr, A.a, A.post);
    }
    interp(cl, E, A.lv[1], M, &B, A.lv[1].g);
    smooth(E, M, &B, A.a, A.post);
    // ---- the entry block's x back to global memory
    if (B.own) {
        const PV& v = E.v;
        const long q0 = sf_ix(v, B.i0, B.j0, k0);
#pragma unroll
        for (int s = 0; s < 8; s++)
            v.f[SF_U][q0 + (s & 1) + ((s >> 1) & 1) * v.js + (s >> 2) * v.ks] = B.X[s];
    }
#ifdef SF_COARSE_TRACE
    TRACE();
    if (threadIdx.x == 0 && M.rank <= 1) {
        for (int i = 1; i < trace_n; i++)
            printf("trace rank %d phase %d: %lld\n", M.rank, i, trace_t[i] - trace_t[i - 1]);
    }
#endif
}

// shared-memory plan (doubles per CTA): offsets into out[], total returned
long plan_smem(sf_level* const* lv, int n, KLevel* out, int* ainv, int* rscr) {
    long off = 0;
    if (rscr) *rscr = 0;   // residual scratch: two planes of a distributed level / a gathered level
    off += GMAX;
    for (int l = 0; l < n; l++) {
        const long nx = lv[l]->nx, ny = lv[l]->ny, pl = nx * ny;
        KLevel L = {};
        L.u = L.f = L.d = L.al = L.bi = L.bj = L.bk = -1;
        const long c = pl * lv[l]->lnz;
        L.g = l > 0 && c <= GMAX;
        if (l == 0) {
            L.u = (int)off;
            off += 2 * pl;
        } else if (l + 1 < n && L.g) {   // every plane, on CTA 0
            L.u = (int)off;  off += c;
            L.f = (int)off;  off += c;
            L.d = (int)off;  off += c;
            L.al = (int)off; off += c;
            L.bi = (int)off; off += (nx + 1) * ny * lv[l]->lnz;
            L.bj = (int)off; off += nx * (ny + 1) * lv[l]->lnz;
            L.bk = (int)off; off += pl * (lv[l]->lnz + 1);
        } else if (l + 1 < n) {
            L.u = (int)off;  off += 2 * pl;
            L.f = (int)off;  off += 2 * pl;
            L.d = (int)off;  off += 2 * pl;
            L.al = (int)off; off += 2 * pl;
            L.bi = (int)off; off += 2 * ny * (nx + 1);
            L.bj = (int)off; off += 2 * (ny + 1) * nx;
            L.bk = (int)off; off += 3 * pl;
        } else {   // bottom: every plane (CTA 0)
            L.g = 1;
            L.u = (int)off; off += c;
            L.f = (int)off; off += c;
            if (ainv) *ainv = (int)off;
            off += c * c;
        }
        if (out) out[l] = L;
    }
    return off;
}

// largest cluster the kernel may use: 16 CTAs if a 16-CTA cluster of it is
// schedulable (non-portable size), else 8; SF_COARSE_MAX_CS caps it (A/B, tests)
int max_cluster() {
    static int probed = 0;
    if (!probed) {
        probed = 8;
        if (cudaFuncSetAttribute(coarse_vcycle_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) ==
                cudaSuccess &&
            cudaFuncSetAttribute(coarse_vcycle_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 CSMEM_MAX) == cudaSuccess) {
            cudaLaunchConfig_t c = {};
            c.gridDim = dim3(CS_MAX);
            c.blockDim = dim3(NT);
            c.dynamicSmemBytes = 96 * 1024;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = CS_MAX;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            c.attrs = at;
            c.numAttrs = 1;
            int nc = 0;
            if (cudaOccupancyMaxActiveClusters(&nc, coarse_vcycle_kernel, &c) == cudaSuccess && nc >= 1)
                probed = CS_MAX;
        }
        cudaGetLastError();
    }
    const char* e = getenv("SF_COARSE_MAX_CS");
    return e ? std::max(1, std::min(probed, atoi(e))) : probed;
}

}  // namespace

int coarse_vcycle_max_levels() { return CMAXL; }

// a V-cycle from lv[0] over n levels fits the kernel: single-part power-of-two
// levels halving into each other, entry nz/2 <= the cluster limit and at most
// NT blocks per layer, the bottom within BOT_MAX cells, shared memory within 227 KB
bool coarse_vcycle_fits(sf_level* const* lv, int n) {
    if (n < 2 || n > CMAXL) return false;
    auto pow2 = [](int v) { return v >= 1 && (v & (v - 1)) == 0; };
    for (int l = 0; l < n; l++) {
        if (lv[l]->nparts != 1 || lv[l]->nlocal != 1) return false;
        if (!pow2(lv[l]->nx) || !pow2(lv[l]->ny) || !pow2(lv[l]->lnz)) return false;
        if (l + 1 < n && (lv[l]->nx < 2 || lv[l]->ny < 2 || lv[l]->lnz < 2 ||
                          lv[l + 1]->nx * 2 != lv[l]->nx || lv[l + 1]->ny * 2 != lv[l]->ny ||
                          lv[l + 1]->lnz * 2 != lv[l]->lnz))
            return false;
    }
    const long bot = (long)lv[n - 1]->nx * lv[n - 1]->ny * lv[n - 1]->lnz;
    return lv[0]->lnz / 2 <= max_cluster() && (long)lv[0]->nx * lv[0]->ny / 4 <= NT &&
           bot <= BOT_MAX && plan_smem(lv, n, nullptr, nullptr, nullptr) * (long)sizeof(double) <= CSMEM_MAX;
}

// V(lv[0]) down to the bottom lv[n-1] and back: one launch of one cluster
sf_status k_coarse_vcycle(sf_level* const* lv, int n, double a, double b, const double* ainv,
                          int pre, int post, bool u_zero, bool trigger_next) {
    if (!coarse_vcycle_fits(lv, n)) return sf_fail(SF_ERR_SHAPE, "coarse V-cycle levels do not fit");
    KArgs A = {};
    const long doubles = plan_smem(lv, n, A.lv, &A.ainv, &A.rscr);
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
    A.ainv_g = ainv;
    A.uzero = u_zero ? 1 : 0;
    A.trig = trigger_next ? 1 : 0;
    const int C = lv[0]->lnz / 2;
#ifdef SF_COARSE_TRACE
    for (int l = 0; l < n; l++)
        printf("plan l=%d %dx%dx%d g=%d u=%d f=%d d=%d bi=%d total=%ld C=%d\n", l, lv[l]->nx, lv[l]->ny,
               lv[l]->lnz, A.lv[l].g, A.lv[l].u, A.lv[l].f, A.lv[l].d, A.lv[l].bi, doubles, C);
#endif
    cudaLaunchConfig_t c = {};
    c.gridDim = dim3(C);
    c.blockDim = dim3(NT);
    c.dynamicSmemBytes = (size_t)doubles * sizeof(double);
    c.stream = lv[0]->stream;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = C;
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
