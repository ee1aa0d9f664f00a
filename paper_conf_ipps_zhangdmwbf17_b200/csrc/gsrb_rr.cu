// The V-cycle's last pre-smoothing RB pair fused with its residual and the
// residual's restriction (A5 + A6 + A7 in one HBM pass), sm_100a, fp64, TMA-fed.
//
// V(l) smooths, then forms res = rhs - A x and restricts it, R_cell, onto the
// coarse right-hand side.  Done separately
// the residual pass re-reads x, rhs and the coefficients (48 B per fine cell)
// right after the smoother streamed them.  This kernel is the colour-fused
// pair of gsrb_fused.cu, rescheduled with two barriers per z step t:
//
//   phase A  R(t+1): red update of plane t+1 on the (x,y) tile, its 1-ring
//            (incl. the two red corners) and the red cells of the 2-ring that
//            neighbour black ring cells (old x on a 3-ring box);
//            Res(t-2): rhs - A x_final at the tile's cells of plane t-2 -- every
//            value it needs (x final on the tile + 1-ring of planes t-3..t-1) is
//            in shared memory; R_cell sums the 2x2x2 children (x pair in a
//            thread, z pair over two steps, y pair across warps through shared
//            memory) and writes 1/8 of the sum to the coarse rhs;
//   phase B  B(t): black update of plane t on the tile AND its 1-ring, written
//            back into shared memory (the tile part also to HBM).
//
// The black residual is the update's own by-product: after B the red
// neighbours of a black cell are final, so rhs - (A x)(d) = q - x_d/lambda with
// q = rhs + b h^-2 S the quantity B just formed (lambda-form, gsrb_fused.cu).
// A red cell's coefficients are captured in registers at R(p) and carried to
// Res(p) three steps later; black coefficients are read in phase B from the
// plane's shared-memory slot, which is refilled only after the step.  Every
// stencil sum uses the explicit contractions of tma_common.cuh, so the
// smoothed x is bit-identical to gsrb_fused.cu's pair.
//
// Single-part levels only (the extended z range reads 3 planes past the
// chunk); the V-cycle falls back to pair + residual_restrict elsewhere.
// Built only with SF_WITH_RR (build.py: environment SF_BUILD_RR=1): measured
// slower than the separate passes on B200 (below), so the default library
// carries the stubs at the end of this file and sf_smooth_residual_restrict
// takes the composite path.
#ifdef SF_WITH_RR
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>

#include "sf_internal.h"

namespace {

#include "tma_common.cuh"

constexpr int TX = 32, TY = 16, PPR = TX / 2, NWARP = 8, NT = 32 * NWARP;
static_assert(NWARP * 32 / PPR == TY, "tile shape");
constexpr int WX = TX + 8;      // x box columns:    gx in [x0-4, x0+TX+4)
constexpr int XH = TY + 6;      // x box rows:       gy in [y0-3, y0+TY+3)
constexpr int WC = TX + 6;      // coef box columns: gx in [x0-2, x0+TX+4)
constexpr int CH = TY + 5;      // coef box rows:    gy in [y0-2, y0+TY+3)
constexpr int PF = 3;           // bundles in flight ahead of the one being consumed
// slot counts: x(t-3..t+2) live + PF in flight; coefficient planes t (phase B,
// refilled after the step), t+1 + PF; beta_k planes t..t+2 + PF; mbarriers:
// pre-bundle + PF + current
constexpr int NXS = 6 + PF, NCS = 1 + PF, NKS = 2 + PF, NMB = PF + 2;
constexpr int NCA = 4;
constexpr int XSLOT = (XH * WX + 15) / 16 * 16;
constexpr int CARR = (CH * WC + 15) / 16 * 16;
constexpr int CSLOT = NCA * CARR;
constexpr int XBYTES = XH * WX * 8, CBYTES = CH * WC * 8;
constexpr int BUNDLE_BYTES = XBYTES + (NCA + 1) * CBYTES;
constexpr int NSCR = (TY / 2) * PPR;   // y-pair partial sums of one coarse plane
constexpr size_t SMEM = sizeof(double) * (NXS * XSLOT + NCS * CSLOT + NKS * CARR + NSCR) + 64;
static_assert(SMEM <= 227 * 1024, "shared memory");
enum { CA_DV = 0, CA_RH = 1, CA_BI = 2, CA_BJ = 3 };
constexpr int NRED_RING = 2 * (TX + TY) + 2;   // 1-ring (no corners) + 2-ring half + 2 red corners
constexpr int RED_PER_WARP = (NRED_RING + NWARP - 1) / NWARP;   // 13
constexpr int NBLK_RING = TX + TY;                               // black 1-ring (no corners)
constexpr int BLK_PER_WARP = NBLK_RING / NWARP;                  // 6
static_assert(RED_PER_WARP <= 32 && NBLK_RING % NWARP == 0, "ring lanes");

struct Maps {
    CUtensorMap x, dv, rh, bi, bj, bk;
};
struct Ptrs {
    double* coarse;             // coarse rhs field (allocation base, plane -SF_GZ)
    long cjs, cks;
};
struct Geo {
    int nx, ny, nz;
    long js, ks;
};

__device__ __forceinline__ int xo_of(int gx, int gy, int x0, int y0) {
    return (gy - y0 + 3) * WX + (gx - x0 + 4);
}
__device__ __forceinline__ int co_of(int gx, int gy, int x0, int y0) {
    return (gy - y0 + 2) * WC + (gx - x0 + 2);
}

// Red ring cell rt in [0, NRED_RING) of a plane with parity par = gk & 1:
// [0, 48) the 1-ring without corners, [48, 96) the 2-ring cells that neighbour
// black 1-ring cells, [96, 98) the two red corners of the 1-ring.
__device__ __forceinline__ void red_ring_cell(int rt, int par, int x0, int y0, int& gx, int& gy) {
    if (rt >= 2 * (TX + TY)) {
        const int c = rt - 2 * (TX + TY);   // corners with (cx + cy) % 2 == par
        // (x0-1,y0-1): even, (x0+TX,y0-1): odd, (x0-1,y0+TY): odd, (x0+TX,y0+TY): even
        const int k = par == 0 ? (c == 0 ? 0 : 3) : (c == 0 ? 1 : 2);
        gx = (k & 1) ? x0 + TX : x0 - 1;
        gy = (k & 2) ? y0 + TY : y0 - 1;
        return;
    }
    const int ring = rt >= TX + TY ? 2 : 1;
    const int m0 = rt - (ring - 1) * (TX + TY);
    if (m0 < TX) {
        const int pp = m0 % (TX / 2);
        gy = (m0 < TX / 2) ? y0 - ring : y0 + TY - 1 + ring;
        gx = x0 + 2 * pp + ((gy + par) & 1);
    } else {
        int m = m0 - TX;
        const int side = m / (TY / 2);
        m -= side * (TY / 2);
        gx = side ? x0 + TX - 1 + ring : x0 - ring;
        const int gyp = y0 + 2 * m;
        gy = gyp + ((gx + gyp + par) & 1);
    }
}

// Black 1-ring cell rb in [0, NBLK_RING) (no corners) of a plane with parity par
__device__ __forceinline__ void black_ring_cell(int rb, int par, int x0, int y0, int& gx, int& gy) {
    if (rb < TX) {
        const int pp = rb % (TX / 2);
        gy = (rb < TX / 2) ? y0 - 1 : y0 + TY;
        gx = x0 + 2 * pp + ((gy + par + 1) & 1);
    } else {
        int m = rb - TX;
        const int side = m / (TY / 2);
        m -= side * (TY / 2);
        gx = side ? x0 + TX : x0 - 1;
        const int gyp = y0 + 2 * m;
        gy = gyp + ((gx + gyp + par + 1) & 1);
    }
}

struct Cell {       // a ring cell: smem offsets, boundary flags, inside the domain
    int xo, co, fl;
    bool ok;
};

__device__ __forceinline__ Cell make_cell(int gx, int gy, int x0, int y0, const Geo& g) {
    Cell c;
    c.ok = gx >= 0 && gx < g.nx && gy >= 0 && gy < g.ny;
    c.xo = xo_of(gx, gy, x0, y0);
    c.co = co_of(gx, gy, x0, y0);
    c.fl = (gx == 0) | ((gx == g.nx - 1) << 1) | ((gy == 0) << 2) | ((gy == g.ny - 1) << 3);
    return c;
}

// lambda-form update / residual pieces at one cell from smem: S over interior faces
__device__ __forceinline__ double sum_at(const double* Xk, const double* Xm, const double* Xp, int xo,
                                         int fl, bool zlo, bool zhi, double bw, double be, double bs,
                                         double bn, double bb, double bt) {
    const double xw = (fl & 1) ? 0.0 : Xk[xo - 1];
    const double xe = (fl & 2) ? 0.0 : Xk[xo + 1];
    const double xs = (fl & 4) ? 0.0 : Xk[xo - WX];
    const double xn = (fl & 8) ? 0.0 : Xk[xo + WX];
    const double xb = zlo ? 0.0 : Xm[xo];
    const double xt = zhi ? 0.0 : Xp[xo];
    return sum6(xw, xe, xs, xn, xb, xt, bw, be, bs, bn, bb, bt);
}

__global__ void __launch_bounds__(NT, 1)
gsrb_rr_kernel(const __grid_constant__ Maps mp, const Ptrs pt, Geo g, double* __restrict__ xo,
               double bh2, int depth, int ntx, int ntiles, int nitems) { pdl_wait();
    extern __shared__ __align__(128) double sm[];
    double* Xs = sm;                                  // [NXS][XH][WX]
    double* Cs = Xs + NXS * XSLOT;                    // [NCS][NCA][CH][WC]
    double* Ks = Cs + NCS * CSLOT;                    // [NKS][CH][WC]
    double* Scr = Ks + NKS * CARR;                    // [TY/2][PPR]
    unsigned long long* mbar = (unsigned long long*)(Scr + NSCR);

    const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int i = 0; i < NMB; i++) mbar_init(&mbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    const unsigned xs_u = smem_u32(Xs), cs_u = smem_u32(Cs), ks_u = smem_u32(Ks);
    const unsigned mb_u = smem_u32(mbar);
    unsigned seq = 0;
    for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int chunk = item / ntiles, tile = item - chunk * ntiles;
        const int x0 = (tile % ntx) * TX, y0 = (tile / ntx) * TY;
        const int z0 = chunk * depth, z1 = min(z0 + depth, g.nz);
        const int cxx = SF_OX + x0 - 4, cyx = y0 - 3 + SF_GY;   // TMA origin of the x box
        const int cxc = SF_OX + x0 - 2, cyc = y0 - 2 + SF_GY;   // ... of the coefficient boxes
        const unsigned seq0 = seq;   // pre-bundle; bundle q -> seq0 + 3 + q - z0

        // bundle q: x(q+1), Dinv/rhs/beta_i/beta_j (q), beta_k(q+1); needed by R(q)
        auto issue = [&](int q) {
            const unsigned sq = seq0 + 3 + (q - z0);
            const unsigned b = mb_u + 8u * (sq % NMB);
            mbar_expect_u(b, BUNDLE_BYTES);
            tma3u(xs_u + 8u * (md(q + 1, NXS) * XSLOT), &mp.x, cxx, cyx, q + 1 + SF_GZ, b);
            const unsigned c = cs_u + 8u * (md(q, NCS) * CSLOT);
            tma3u(c + 8u * (CA_DV * CARR), &mp.dv, cxc, cyc, q + SF_GZ, b);
            tma3u(c + 8u * (CA_RH * CARR), &mp.rh, cxc, cyc, q + SF_GZ, b);
            tma3u(c + 8u * (CA_BI * CARR), &mp.bi, cxc, cyc, q + SF_GZ, b);
            tma3u(c + 8u * (CA_BJ * CARR), &mp.bj, cxc, cyc, q + SF_GZ, b);
            tma3u(ks_u + 8u * (md(q + 1, NKS) * CARR), &mp.bk, cxc, cyc, q + 1 + SF_GZ, b);
        };
        if (tid == 0) {
            fence_proxy_async();   // generic smem writes of the previous item before TMA reuse
            const unsigned b = mb_u + 8u * (seq0 % NMB);
            mbar_expect_u(b, 2 * XBYTES + CBYTES);
            tma3u(xs_u + 8u * (md(z0 - 3, NXS) * XSLOT), &mp.x, cxx, cyx, z0 - 3 + SF_GZ, b);
            tma3u(xs_u + 8u * (md(z0 - 2, NXS) * XSLOT), &mp.x, cxx, cyx, z0 - 2 + SF_GZ, b);
            tma3u(ks_u + 8u * (md(z0 - 2, NKS) * CARR), &mp.bk, cxc, cyc, z0 - 2 + SF_GZ, b);
            for (int q = z0 - 2; q <= min(z0 + PF - 3, z1 + 1); q++) issue(q);
        }

        // this thread's pair: row gy, cells gxa (even) and gxa+1
        const int hl = lane % PPR, row = w + NWARP * (lane / PPR);
        const int gxa = x0 + 2 * hl, gy = y0 + row;
        const int xoff = xo_of(gxa, gy, x0, y0);
        const int coff = co_of(gxa, gy, x0, y0);
        const long goff = (long)(gy + SF_GY) * g.js + SF_OX + gxa;   // global offset in a plane
        const int fl0 = (gxa == 0) | ((gy == 0) << 2) | ((gy == g.ny - 1) << 3);   // even cell
        const int fl1 = ((gxa + 1 == g.nx - 1) << 1) | ((gy == 0) << 2) | ((gy == g.ny - 1) << 3);
        // ring cells of this thread for both plane parities
        Cell rc[2], bc[2];
        const bool red_lane = lane < RED_PER_WARP && w * RED_PER_WARP + lane < NRED_RING;
        const bool blk_lane = lane < BLK_PER_WARP;
#pragma unroll
        for (int par = 0; par < 2; par++) {
            int gx, gyr;
            red_ring_cell(min(w * RED_PER_WARP + lane, NRED_RING - 1), par, x0, y0, gx, gyr);
            rc[par] = make_cell(gx, gyr, x0, y0, g);
            rc[par].ok = rc[par].ok && red_lane;
            black_ring_cell(w * BLK_PER_WARP + min(lane, BLK_PER_WARP - 1), par, x0, y0, gx, gyr);
            bc[par] = make_cell(gx, gyr, x0, y0, g);
            bc[par].ok = bc[par].ok && blk_lane;
        }
        // red-cell coefficients of R(p) kept for Res(p) three steps later:
        // cf0 = plane t (captured last step) .. cf2 = plane t-2 (consumed now)
        double cf0[8], cf1[8], cf2[8];
#pragma unroll
        for (int i = 0; i < 8; i++) cf0[i] = cf1[i] = cf2[i] = 0.0;
        double br1 = 0.0, br2 = 0.0;    // black residuals of planes t-1, t-2 (this pair)
        double acc = 0.0, pend = 0.0;   // R_cell partial sums
        int pendK = -1;

        // rotating slot indices for step t = z0-3
        int ix[6];                      // x(t-3) .. x(t+2)
#pragma unroll
        for (int i = 0; i < 6; i++) ix[i] = md(z0 - 6 + i, NXS);
        int ic = md(z0 - 2, NCS);                        // coef(t+1); coef(t) is the slot before
        int ik0 = md(z0 - 3, NKS), ik1 = md(z0 - 2, NKS), ik2 = md(z0 - 1, NKS);   // beta_k(t..t+2)
        mbar_wait(&mbar[seq0 % NMB], (seq0 / NMB) & 1);

        // step t: [R(t+1) + red ring, Res(t-2)] | barrier | [B(t) + black ring] | barrier
        for (int t = z0 - 3; t <= z1 + 1; t++) {
            // finish the coarse cell whose odd-row partial was published last step
            if (pendK >= 0) {
                pt.coarse[(long)(pendK + SF_GZ) * pt.cks + (long)((gy >> 1) + SF_GY) * pt.cjs + SF_OX +
                          (gxa >> 1)] = __dmul_rn(__dadd_rn(pend, Scr[(row >> 1) * PPR + hl]), 0.125);
                pendK = -1;
            }
            const int q = t + 1;
            if (q <= z1 + 1) {
                const unsigned sq = seq0 + 3 + (q - z0);
                mbar_wait(&mbar[sq % NMB], (sq / NMB) & 1);
            }
            const double* X3 = Xs + ix[0] * XSLOT;   // x(t-3)
            const double* X2 = Xs + ix[1] * XSLOT;   // x(t-2)
            const double* X1 = Xs + ix[2] * XSLOT;   // x(t-1)
            double* X0 = Xs + ix[3] * XSLOT;         // x(t)
            double* Xq = Xs + ix[4] * XSLOT;         // x(t+1)
            const double* Xq1 = Xs + ix[5] * XSLOT;  // x(t+2)
            const double* C = Cs + ic * CSLOT;       // coef(t+1)
            const double* Cb = Cs + md(ic - 1, NCS) * CSLOT;   // coef(t) (slot refilled after this step)
            const double* K0 = Ks + ik0 * CARR;      // beta_k(t)
            const double* K1 = Ks + ik1 * CARR;      // beta_k(t+1)
            const double* K2 = Ks + ik2 * CARR;      // beta_k(t+2)

            // Every load of a phase is issued before its first shared-memory store
            // (stores are deferred to the end of the phase): the phase's stencils
            // are independent, and without aliasing barriers the compiler can
            // overlap their load latencies.
            // ---- phase A.1: Res(r), rhs - A x_final at the tile cells of plane r = t-2
            const int rp = t - 2;
            const bool rv = rp >= z0 && rp < z1;
            double v = 0.0;
            if (rv) {
                const int rs = (y0 + w + rp) & 1;   // red position
                const double S = sum_at(X2, X3, X1, xoff + rs, rs ? fl1 : fl0, rp == 0, rp == g.nz - 1,
                                        cf2[2], cf2[3], cf2[4], cf2[5], cf2[6], cf2[7]);
                const double rr = __fma_rn(-X2[xoff + rs], inv_fast(cf2[0]), gs_q(cf2[1], bh2, S));
                v = rs ? __dadd_rn(br2, rr) : __dadd_rn(rr, br2);
            }
            // ---- phase A.2: R(q), tile pair + red ring cells of plane q = t+1 (old black)
            const bool rin = q >= z0 - 2 && q <= z1 + 1 && q >= 0 && q < g.nz;
            const int sel = (y0 + w + q) & 1;   // position of the red cell in the pair
            const Cell& rcq = (q & 1) ? rc[1] : rc[0];
            const bool rring = rin && rcq.ok;
            double rnew = 0.0, rrng = 0.0;
            {
                const bool zlo = q == 0, zhi = q == g.nz - 1;
#pragma unroll
                for (int i = 0; i < 8; i++) {   // rotate the Res coefficient sets
                    cf2[i] = cf1[i];
                    cf1[i] = cf0[i];
                }
                if (rin) {
                    const int co = coff + sel;
                    cf0[0] = C[CA_DV * CARR + co];
                    cf0[1] = C[CA_RH * CARR + co];
                    cf0[2] = C[CA_BI * CARR + co];
                    cf0[3] = C[CA_BI * CARR + co + 1];
                    cf0[4] = C[CA_BJ * CARR + co];
                    cf0[5] = C[CA_BJ * CARR + co + WC];
                    cf0[6] = K1[co];
                    cf0[7] = K2[co];
                    const double S = sum_at(Xq, X0, Xq1, xoff + sel, sel ? fl1 : fl0, zlo, zhi, cf0[2],
                                            cf0[3], cf0[4], cf0[5], cf0[6], cf0[7]);
                    rnew = gs_upd(cf0[0], cf0[1], bh2, S);
                }
                if (rring) {
                    const double S = sum_at(Xq, X0, Xq1, rcq.xo, rcq.fl, zlo, zhi, C[CA_BI * CARR + rcq.co],
                                            C[CA_BI * CARR + rcq.co + 1], C[CA_BJ * CARR + rcq.co],
                                            C[CA_BJ * CARR + rcq.co + WC], K1[rcq.co], K2[rcq.co]);
                    rrng = gs_upd(C[CA_DV * CARR + rcq.co], C[CA_RH * CARR + rcq.co], bh2, S);
                }
            }
            if (rin) Xq[xoff + sel] = rnew;
            if (rring) Xq[rcq.xo] = rrng;
            if (rv) {   // R_cell: z pair in registers, y pair across warps
                if ((rp & 1) == 0) {
                    acc = v;
                } else {
                    acc = __dadd_rn(acc, v);
                    if (w & 1) {
                        Scr[(row >> 1) * PPR + hl] = acc;
                    } else {
                        pend = acc;
                        pendK = rp >> 1;
                    }
                }
            }
            __syncthreads();   // red-new of plane t+1 (tile + ring) visible

            // ---- phase B: B(t), tile pair + black 1-ring of plane t (red-new neighbours)
            double brn = 0.0;
            if (t >= z0 - 1 && t <= z1 && t >= 0 && t < g.nz) {
                const bool zlo = t == 0, zhi = t == g.nz - 1;
                const int bs = 1 - ((y0 + w + t) & 1);   // position of the black cell
                const int co = coff + bs;
                const double dv = Cb[CA_DV * CARR + co];
                const double S = sum_at(X0, X1, Xq, xoff + bs, bs ? fl1 : fl0, zlo, zhi,
                                        Cb[CA_BI * CARR + co], Cb[CA_BI * CARR + co + 1],
                                        Cb[CA_BJ * CARR + co], Cb[CA_BJ * CARR + co + WC], K0[co], K1[co]);
                const double rd = X0[xoff + 1 - bs];   // red-new partner of the pair
                const Cell& c = (t & 1) ? bc[1] : bc[0];
                double bring = 0.0;
                if (c.ok) {
                    const double Sr = sum_at(X0, X1, Xq, c.xo, c.fl, zlo, zhi, Cb[CA_BI * CARR + c.co],
                                             Cb[CA_BI * CARR + c.co + 1], Cb[CA_BJ * CARR + c.co],
                                             Cb[CA_BJ * CARR + c.co + WC], K0[c.co], K1[c.co]);
                    bring = gs_upd(Cb[CA_DV * CARR + c.co], Cb[CA_RH * CARR + c.co], bh2, Sr);
                }
                const double qv = gs_q(Cb[CA_RH * CARR + co], bh2, S);
                const double bnew = __dmul_rn(dv, qv);
                brn = __fma_rn(-bnew, inv_fast(dv), qv);   // rhs - A x at the black cell
                X0[xoff + bs] = bnew;
                if (c.ok) X0[c.xo] = bring;
                if (t >= z0 && t < z1)   // streaming store: other tiles still need halo lines
                    __stcs((double2*)(xo + (long)(t + SF_GZ) * g.ks + goff),
                           bs ? make_double2(rd, bnew) : make_double2(bnew, rd));
            }
            br2 = br1;
            br1 = brn;
            fence_proxy_async();
            __syncthreads();
            // refill bundle t+PF+1 (its slots were last read before this barrier)
            if (tid == 0 && t + PF + 1 <= z1 + 1) issue(t + PF + 1);
#pragma unroll
            for (int i = 0; i < 5; i++) ix[i] = ix[i + 1];
            ix[5] = (ix[5] + 1 == NXS) ? 0 : ix[5] + 1;
            ic = (ic + 1 == NCS) ? 0 : ic + 1;
            ik0 = ik1; ik1 = ik2; ik2 = (ik2 + 1 == NKS) ? 0 : ik2 + 1;
        }
        if (pendK >= 0) {
            pt.coarse[(long)(pendK + SF_GZ) * pt.cks + (long)((gy >> 1) + SF_GY) * pt.cjs + SF_OX +
                      (gxa >> 1)] = __dmul_rn(__dadd_rn(pend, Scr[(row >> 1) * PPR + hl]), 0.125);
        }
        seq = seq0 + 3 + (z1 + 1 - z0) + 1;
        __syncthreads();   // all reads of this item's slots done before the next prologue
    }
}

PFN_cuTensorMapEncodeTiled_v12000 g_enc = nullptr;
int g_sms = 0;

sf_status encode_box(CUtensorMap* m, const sf_level* L, const double* base, int cols, int rows) {
    cuuint64_t dims[3] = {(cuuint64_t)L->js, (cuuint64_t)(L->ny + 2 * SF_GY),
                          (cuuint64_t)(L->lnz + 2 * SF_GZ)};
    cuuint64_t strides[2] = {(cuuint64_t)L->js * 8, (cuuint64_t)L->ks * 8};
    cuuint32_t box[3] = {(cuuint32_t)cols, (cuuint32_t)rows, 1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult r = g_enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)base, dims, strides, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    return SF_OK;
}

}  // namespace

// Measured on B200 (scripts/rr_time.py, 512^3): this kernel takes 2.56-2.64 ms
// against 1.33 ms for the plain pair + 1.16 ms for the separate residual_restrict
// pass.  The per-z-step work is latency-bound (5 stencil rounds and 2 barriers
// per step instead of 3 and 1), which costs more than the 48 B/cell it saves,
// so the V-cycle and sf_smooth_residual_restrict use it only when SF_RR=1.
bool gsrb_rr_supported(const sf_level* F, const sf_level* C) {
    const char* e = getenv("SF_RR");
    if (!e || atoi(e) == 0) return false;
    return F->nparts == 1 && C->nparts == 1 && F->nx % TX == 0 && F->ny % TY == 0 &&
           F->lnz % 2 == 0 && C->nx * 2 == F->nx && C->ny * 2 == F->ny && C->lnz * 2 == F->lnz;
}

sf_status k_gsrb_pair_rr(sf_level* L, int xin, int xout, int rhs, double a, double b, sf_level* C,
                         int cf) {
    (void)a;   // the lambda-form update and residual take a only through Dinv
    if (!gsrb_rr_supported(L, C)) return sf_fail(SF_ERR_SHAPE, "fused pair+residual+restriction unsupported");
    if (!g_enc) {
        cudaDriverEntryPointQueryResult qr;
        void* fn = nullptr;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &qr);
        if (e != cudaSuccess || qr != cudaDriverEntryPointSuccess || !fn)
            return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
        g_enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
        SF_CUDA(cudaFuncSetAttribute(gsrb_rr_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)SMEM));
        int dev;
        SF_CUDA(cudaGetDevice(&dev));
        SF_CUDA(cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev));
    }
    const int ntx = L->nx / TX, nty = L->ny / TY, tiles = ntx * nty;
    // even chunk depth minimising rounds * (depth + 5 steps + fill) over persistent CTAs
    int best_d = L->lnz;
    double best = 1e30;
    for (int d = L->lnz; d >= 2; d -= 2) {
        const long items = (long)tiles * ((L->lnz + d - 1) / d);
        const double cost = (double)((items + g_sms - 1) / g_sms) * (d + 7.0);
        if (cost < best - 1e-9) { best = cost; best_d = d; }
        if (d < 8) break;
    }
    const char* ed = getenv("SF_RR_DEPTH");   // tuning / test override (rounded up to even)
    if (ed && atoi(ed) > 0) best_d = std::min(L->lnz, (atoi(ed) + 1) / 2 * 2);
    const int depth = best_d, items = tiles * ((L->lnz + depth - 1) / depth);
    PV v = sf_view(L, 0);
    PV c = sf_view(C, 0);
    Maps mp;
    SF_TRY(encode_box(&mp.x, L, v.f[xin], WX, XH));
    SF_TRY(encode_box(&mp.dv, L, v.f[SF_DINV], WC, CH));
    SF_TRY(encode_box(&mp.rh, L, v.f[rhs], WC, CH));
    SF_TRY(encode_box(&mp.bi, L, v.f[SF_BETA_I], WC, CH));
    SF_TRY(encode_box(&mp.bj, L, v.f[SF_BETA_J], WC, CH));
    SF_TRY(encode_box(&mp.bk, L, v.f[SF_BETA_K], WC, CH));
    Ptrs pt{c.f[cf], C->js, C->ks};
    Geo g{v.nx, v.ny, v.nz, v.js, v.ks};
    const double bh2 = b / (L->h * L->h);
    sf_launch(gsrb_rr_kernel, std::min(items, g_sms), NT, SMEM, L->stream, mp, pt, g, v.f[xout], bh2, depth,
                                                                     ntx, tiles, items);
    SF_LAUNCHED();
    return sf_check_launch("gsrb_rr");
}

#else   // !SF_WITH_RR

#include "sf_internal.h"

bool gsrb_rr_supported(const sf_level*, const sf_level*) { return false; }

sf_status k_gsrb_pair_rr(sf_level*, int, int, int, double, double, sf_level*, int) {
    return sf_fail(SF_ERR_SHAPE, "fused pair+residual+restriction not built (SF_BUILD_RR=1)");
}

#endif  // SF_WITH_RR
