// Colour-fused Gauss-Seidel red-black pair (A5) for sm_100a, fp64, TMA-fed.
//
// One kernel pass performs a whole RB pair -- [BC, red, BC, black] of
// PAPER.md:641-644 with x += lambda*(rhs - Ax) (Fig 4) --
// so the 64 B/cell compulsory traffic of PAPER.md:669-672 is paid once per
// pair instead of once per colour sweep.  It is the B200 counterpart of the
// paper's "multicolor reordering" and OpenCL "tall-skinny blocking" (2-D tiles
// rolled up through the remaining dimension):
//
//   (x,y) tile (32 x 16 cells; 32 x 8 in the two-CTA-per-SM build) streamed
//   along z by one CTA; step t runs
//   R(t+1)  red cells of plane t+1 on the tile AND on a one-cell ring around
//           it (the ring belongs to neighbouring tiles; recomputing it here,
//           bit-identically, means the black update needs no other CTA), and
//   B(t-1)  black cells of plane t-1 on the tile, which read red-new values of
//           planes t-2, t-1 (incl. ring) and t --
//   two independent dependency chains between consecutive barriers.  The
//   update is evaluated in lambda-form (below), so alpha is never read.
//
// Out of place (xin -> xout): the 2-ring reads of xin must see OLD values
// whatever neighbouring CTAs have written, so the pair writes a second buffer
// and the level swaps U <-> TMP.
//
// Data movement (Blackwell): every operand plane -- x (tile + 2-ring), Dinv,
// rhs, beta_i, beta_j (tile + 1-ring) and beta_k -- arrives by TMA
// (cp.async.bulk.tensor.3d) into shared memory, completion tracked by an
// mbarrier per plane "bundle", PF bundles ahead of use (5 in the 32x16 build,
// ~170 KB in flight per SM).  One elected thread issues; all warps compute
// from shared memory (16-byte pair loads); the output pair is stored with
// coalesced 16-byte streaming stores.  Persistent CTAs walk (tile, z-chunk)
// items in chunk-major order so neighbouring tiles stream the same planes at
// the same time (ring/halo reads hit L2).
//
// Variants (template flags): RESID reduces the red part of max|rhs - A x| of
// the input, BRES the black part of the output's (the split convergence check,
// mg.cu), INTERP applies x_in += P0(e_coarse) to each x plane in shared memory
// one step before its first read (A8 of the V-cycle fused into the first
// post-smoothing pair).  Launches can be restricted to the interior or the
// boundary z-chunks of a part (halo exchange overlapped, comm.cu).
//
// Dirichlet BC is folded in: a neighbour across a global face contributes 0 to
// the lambda-form sum (its -x(c) ghost term is part of the diagonal,
// PAPER.md:336-341).  Part (slab) interfaces read exchanged halo planes
// (x depth 2, coefficients depth 2, rhs depth 1).
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdlib>

#include "sf_internal.h"

namespace {

// One red/black pair per thread.  32x16 (8 warps) carries ~22% less halo per
// cell than 64x8 and 48 instead of 72 redundant ring cells.  Compiled three
// times by build.py: 32x16 with 5-deep prefetch (_t32), 64x8 with 4-deep
// (_t64, when ny % 16 != 0) and 32x8 / 4 warps / 2-deep with three CTAs per
// SM (_t32w4, levels up to 256^3: three independent z-step chains per SM hide
// each other's per-item pipeline fill; 6 % faster than two CTAs with 3-deep
// prefetch at 256^3, profiles/r01/ab_256_ctas_per_sm.txt).
#ifndef SF_GSRB_TX
#define SF_GSRB_TX 32
#endif
#ifndef SF_GSRB_PF
#define SF_GSRB_PF 5
#endif
#ifndef SF_GSRB_SUFFIX
#define SF_GSRB_SUFFIX _t32
#endif
#define SF_CAT2(a, b) a##b
#define SF_CAT(a, b) SF_CAT2(a, b)
constexpr int TX = SF_GSRB_TX;         // tile width (cells)
constexpr int PPR = TX / 2;            // pairs per row = lanes per row segment
#ifndef SF_GSRB_NWARP
#define SF_GSRB_NWARP 8
#endif
#ifndef SF_GSRB_MINB   // resident CTAs per SM the variant is built for
#define SF_GSRB_MINB 1
#endif
constexpr int NWARP = SF_GSRB_NWARP;
constexpr int MINB = SF_GSRB_MINB;
static_assert(NWARP % 2 == 0, "rows w and w + NWARP must have the same parity");
constexpr int TY = NWARP * 32 / PPR;   // tile height (rows): 16 for TX = 32
constexpr int NT = 32 * NWARP;         // 256 threads
constexpr int W = TX + 4;              // smem row: gx in [x0-2, x0+TX+2)
constexpr int XH = TY + 4;             // x rows:   gy in [y0-2, y0+TY+2)
constexpr int CHH = TY + 3;            // coef rows: gy in [y0-1, y0+TY+2)
constexpr int PF = SF_GSRB_PF;         // bundles in flight ahead of the one being consumed
constexpr int NXS = 5 + PF, NCS = 1 + PF, NKS = 2 + PF, NMB = PF + 2;  // slot counts
constexpr int NCA = 4;                 // staged coefficient arrays per plane (beta_k separate)
constexpr int XSLOT = (XH * W + 15) / 16 * 16;   // doubles, 128-byte multiple
constexpr int CARR = (CHH * W + 15) / 16 * 16;
constexpr int CSLOT = NCA * CARR;
// Only beta_j (north faces of the ring's top row) needs the last coefficient
// row; Dinv, rhs, beta_i and beta_k boxes stop one row short (CHS rows; the
// slot's last row is never read).  SF_TRIM_ROWS=0 restores full boxes.
#ifndef SF_TRIM_ROWS
#define SF_TRIM_ROWS 1
#endif
constexpr int CHS = CHH - SF_TRIM_ROWS;
constexpr int XBYTES = XH * W * 8, CBYTES = CHH * W * 8, CBYTES_S = CHS * W * 8;
static_assert(XSLOT >= TY * PPR, "RRF y shares fit one x slot");
constexpr int BUNDLE_BYTES = XBYTES + (NCA - 1) * CBYTES_S + CBYTES + CBYTES_S;
constexpr size_t SMEM = sizeof(double) * (NXS * XSLOT + NCS * CSLOT + NKS * CARR) + 64;
static_assert(MINB * (SMEM + 1024) <= 228 * 1024, "MINB CTAs per SM must fit in shared memory");
// fused P0 interpolation (INTERP): each x-box pair (2 cells, one parent) is
// corrected in smem; a thread owns pairs tid and tid+NT of the box
constexpr int XPAIRS = XH * (W / 2);
static_assert(XPAIRS <= 2 * NT, "two correction pairs per thread");
static_assert(TX % 2 == 0 && 32 % PPR == 0, "tile shape");
enum { CA_DV = 0, CA_RH = 1, CA_BI = 2, CA_BJ = 3 };
constexpr int NRING = TX + TY;         // red ring cells per plane (half of the 1-ring)

// Dirichlet faces: the pair reads the boundary-zeroed face coefficients
// (SF_BI0/BJ0/BK0, sf_internal.h), so a boundary neighbour's term is
// 0 * (finite ghost) and no select is needed (13 % fewer instructions; the
// pair 1.4 % faster under the power cap, profiles/r02/ab_nobc_selects.txt).
// SF_PAIR_SELECTS=1 builds keep the selects (A/B; same results).
#ifndef SF_PAIR_SELECTS
#define SF_PAIR_SELECTS 0
#endif
#if SF_PAIR_SELECTS
#define BCZ(c) (c)
#else
#define BCZ(c) false
#endif

struct Maps {
    CUtensorMap x, dv, rh, bi, bj, bk;
};

// INTERP: coarse correction field e_c (read through L2, it is 1/8 of the fine level)
struct CoarseView {
    const double* e;
    long js, ks;
    int zoff;   // coarse plane of fine plane 0 inside a replicated coarse part
};

#include "tma_common.cuh"

struct Geo {
    int nx, ny, nz, z0, gnz;
    long js, ks;
    int zmask;   // measurement knob (SF_DBG_ZMASK): planes aliased to q & zmask, 0 = off
};

// storage plane (TMA coordinate / store row) of plane q; with the measurement
// knob every plane aliases one of zmask+1 planes, so the whole working set is
// L2-resident and the kernel's SM-side throughput is measured (results are
// meaningless then)
__device__ __forceinline__ int zplane(const Geo& g, int q) { return (g.zmask ? (q & g.zmask) : q) + SF_GZ; }

// Per-step state shared by the templated step bodies.
struct StepCtx {
    const double* Xk;   // x(p)      (written: red-new of plane p)
    const double* Xm;   // x(p-1)
    const double* Xp;   // x(p+1)
    const double* Xmm;  // x(p-2)
    const double* C;    // coefficients of plane p
    const double* Klo;  // beta_k(p)
    const double* Khi;  // beta_k(p+1)
};

// R(p) for the pair at smem offsets (xo_: x box, co_: coef box).  SEL = 1 if
// the odd cell of the pair is red at this plane (warp-uniform).  Returns the
// red-new value; leaves the black cell's coefficients of plane p in nb.
// R for the pair at smem offsets (xo_: x box, co_: coef box).  SEL = 1 if
// the odd cell of the pair is red at this plane (warp-uniform).  Returns the
// red-new value; leaves the black cell's coefficients of the plane in nb
// (bw, be, bs, bn, bb, bt, dinv, rhs).  RESID: rres = rhs - A x_in at the red
// cell (A x = x(c)/dinv - b h^-2 S): the red part of the INPUT's residual.
// The thread's own pair at planes q-1, q, q+1 (pb, xp2, pt) comes from
// registers: each step loads only the pair of the newest plane.
template <int SEL, bool RESID>
__device__ __forceinline__ double red_pair(const StepCtx& s, int xo_, int co_, int lane, int gx,
                                           int gy, const Geo& g, bool zlo, bool zhi, double bh2,
                                           double* nb, double& rres, double2 pb, double2 xp2,
                                           double2 pt, double2 bkl, double2& bkh) {
    const double2 dv2 = *(const double2*)&s.C[CA_DV * CARR + co_];
    const double2 rh2 = *(const double2*)&s.C[CA_RH * CARR + co_];
    const double2 bi2 = *(const double2*)&s.C[CA_BI * CARR + co_];
    const double2 bjl = *(const double2*)&s.C[CA_BJ * CARR + co_];
    const double2 bjh = *(const double2*)&s.C[CA_BJ * CARR + co_ + W];
    bkh = *(const double2*)&s.Khi[co_];   // beta_k(q+1); beta_k(q) was the last step's
    const double bie = s.C[CA_BI * CARR + co_ + 2];   // east face of the odd cell
    const int col = xo_ + SEL;
    double xw, xe;
    if (SEL == 0) {
        xw = s.Xk[xo_ - 1]; xe = xp2.y;
    } else {
        xw = xp2.x; xe = s.Xk[xo_ + 2];
    }
    [[maybe_unused]] const int gxr = gx + SEL;
    if (BCZ(gxr == 0)) xw = 0.0;
    if (BCZ(gxr == g.nx - 1)) xe = 0.0;
    const double xs = BCZ(gy == 0) ? 0.0 : s.Xk[col - W];
    const double xn = BCZ(gy == g.ny - 1) ? 0.0 : s.Xk[col + W];
    const double xb = BCZ(zlo) ? 0.0 : (SEL ? pb.y : pb.x);
    const double xt = BCZ(zhi) ? 0.0 : (SEL ? pt.y : pt.x);
    double r, S;
    if (SEL == 0) {
        S = sum6(xw, xe, xs, xn, xb, xt, bi2.x, bi2.y, bjl.x, bjh.x, bkl.x, bkh.x);
        const double q = gs_q(rh2.x, bh2, S);
        r = __dmul_rn(dv2.x, q);
        if (RESID) rres = q - xp2.x * inv_fast(dv2.x);
        nb[0] = bi2.y; nb[1] = bie; nb[2] = bjl.y; nb[3] = bjh.y; nb[4] = bkl.y; nb[5] = bkh.y;
        nb[6] = dv2.y; nb[7] = rh2.y;
    } else {
        S = sum6(xw, xe, xs, xn, xb, xt, bi2.y, bie, bjl.y, bjh.y, bkl.y, bkh.y);
        const double q = gs_q(rh2.y, bh2, S);
        r = __dmul_rn(dv2.y, q);
        if (RESID) rres = q - xp2.y * inv_fast(dv2.y);
        nb[0] = bi2.x; nb[1] = bi2.y; nb[2] = bjl.x; nb[3] = bjh.x; nb[4] = bkl.x; nb[5] = bkh.x;
        nb[6] = dv2.x; nb[7] = rh2.x;
    }
    return r;
}

// B for the pair; SEL = position (0: even x, 1: odd x) of the black cell in
// the pair.  Returns the output pair (red-new, black-new in place).  BRES: bres
// = rhs - A x at the black cell AFTER its update, q - x_new/dinv with q the
// quantity the update just formed (its red neighbours are final: this is the
// black part of the residual of the pair's output).
// The black cell's in-pair partner and its neighbours below / above are the
// red cells this thread updated itself in the last three steps (rn_same,
// rn_below, rn_above: the values it stored to shared memory), so they come
// from registers.
template <int SEL, bool BRES>
__device__ __forceinline__ double2 black_pair(const StepCtx& s, int xo_, int gx, int gy,
                                              const Geo& g, int gkm, double bh2, const double* rb,
                                              double& bres, double rn_below, double rn_same,
                                              double rn_above) {
    double xw, xe;
    if (SEL == 0) {
        xw = s.Xm[xo_ - 1]; xe = rn_same;
    } else {
        xw = rn_same; xe = s.Xm[xo_ + 2];
    }
    [[maybe_unused]] const int gxb = gx + SEL;
    if (BCZ(gxb == 0)) xw = 0.0;
    if (BCZ(gxb == g.nx - 1)) xe = 0.0;
    const int col = xo_ + SEL;
    const double xs = BCZ(gy == 0) ? 0.0 : s.Xm[col - W];
    const double xn = BCZ(gy == g.ny - 1) ? 0.0 : s.Xm[col + W];
    const double xb = BCZ(gkm == 0) ? 0.0 : rn_below;
    const double xt = BCZ(gkm == g.gnz - 1) ? 0.0 : rn_above;
    const double q = gs_q(rb[7], bh2, sum6(xw, xe, xs, xn, xb, xt, rb[0], rb[1], rb[2], rb[3], rb[4], rb[5]));
    const double bnew = __dmul_rn(rb[6], q);
    if (BRES) bres = __fma_rn(-bnew, inv_fast(rb[6]), q);
    return SEL ? make_double2(rn_same, bnew) : make_double2(bnew, rn_same);
}

// Ring red cell at smem offsets (xo_, co_) (scalar loads; bounds in flags)
__device__ __forceinline__ double red_ring(const StepCtx& s, int xo_, int co_, int flags, double bh2,
                                           bool zlo, bool zhi) {
    const double xw = BCZ(flags & 1) ? 0.0 : s.Xk[xo_ - 1];
    const double xe = BCZ(flags & 2) ? 0.0 : s.Xk[xo_ + 1];
    const double xs = BCZ(flags & 4) ? 0.0 : s.Xk[xo_ - W];
    const double xn = BCZ(flags & 8) ? 0.0 : s.Xk[xo_ + W];
    const double xb = BCZ(zlo) ? 0.0 : s.Xm[xo_];
    const double xt = BCZ(zhi) ? 0.0 : s.Xp[xo_];
    const double S = sum6(xw, xe, xs, xn, xb, xt, s.C[CA_BI * CARR + co_],
                          s.C[CA_BI * CARR + co_ + 1], s.C[CA_BJ * CARR + co_],
                          s.C[CA_BJ * CARR + co_ + W], s.Klo[co_], s.Khi[co_]);
    return gs_upd(s.C[CA_DV * CARR + co_], s.C[CA_RH * CARR + co_], bh2, S);
}

// RESID: max |rhs - A x| over the red cells of the INPUT (the black part of
// that residual was reduced by the BRES pair that produced the input).
// BRES: max |rhs - A x| over the black cells of the OUTPUT.  Both into *rmax.
// RRF (pair + residual + restriction, gsrb_rr.cu; single-part levels, even
// z-chunks): the residual of the pair's output in delta form.  A red cell's
// residual vanished at its own update (lambda = 1/diag(A)) and the black sweep
// then changed only its six black neighbours, so r(c) = b h^-2 sum_f beta_f
// delta(n_f) with delta = x_new - x_old of a black cell; a black cell's own
// residual vanishes likewise (both up to rounding).  Each black cell scatters
// beta_f * b h^-2 * delta over its faces: three into its own 2x2x2 block, one
// per axis into the neighbouring block.  x shares go to the next pair column by
// a lane shuffle, z shares stay in the thread's registers (carried to the next /
// previous coarse plane), so a thread writes two partials per coarse cell: its
// block's (P) and the y share (other warps); only shares crossing a tile or
// z-chunk edge go to the edge arrays.  Each array entry has exactly one writer
// (SfRRF); the fix-up pass sums them in a fixed order (x 1/8).
template <bool RESID, bool INTERP, bool BRES, bool RRF = false>
__global__ void __launch_bounds__(NT, MINB)
gsrb_pair_tma_kernel(const __grid_constant__ Maps mp, Geo g, double* __restrict__ xo, double a,
                     double bh2, int depth, int ntx, int ntiles, int nitems, double* rmax,
                     CoarseView cv, int c0, int cstride, unsigned long long* ts, int bd,
                     int nch, int tcount, int zero_rmax, int early, const __grid_constant__ SfRRF rv) {
    static_assert(!(RRF && (RESID || INTERP || BRES)), "RRF is a plain pair");
    // early: the launch before this one triggered early and wrote nothing this
    // pair reads but the P0 source -- the first item's TMA prologue is issued
    // before griddepcontrol.wait (it overlaps that launch)
    bool waited = !early;
    auto after_wait = [&]() {
        // SF_RM_ZERO: reset the BRES scalar of a later pair (no separate launch)
        if (zero_rmax && blockIdx.x == 0 && threadIdx.x == 0) *rmax = 0.0;
    };
    if (!early) {
        pdl_wait();
        after_wait();
    }
    // live timing (sf_level_pair_timing): thread 0 of every CTA stamps its start
    // and end on the global timer; the last CTA to finish books end - start
    bool timing = false;
    if (threadIdx.x == 0 && *(volatile unsigned long long*)ts != 0ull) {
        timing = true;
        atomicMin(&ts[1], gtimer());
    }
    constexpr int RING_PER_WARP = (NRING + NWARP - 1) / NWARP;   // 6 (32x16) / 9 (64x8)
    extern __shared__ __align__(128) double sm[];
    double* Xs = sm;                                  // [NXS][XH][W]
    double* Cs = Xs + NXS * XSLOT;                    // [NCS][NCA][CHH][W]
    double* Ks = Cs + NCS * CSLOT;                    // [NKS][CHH][W]
    unsigned long long* mbar = (unsigned long long*)(Ks + NKS * CARR);

    const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int i = 0; i < NMB; i++) mbar_init(&mbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    unsigned long long rbits = 0ull;  // RESID / BRES: max |rhs - A x| of this thread's cells
    unsigned seq = 0;  // bundles issued by this CTA so far (all threads track it)
    for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int ci = item / ntiles, tile = item - ci * ntiles;
        const int chunk = c0 + ci * cstride;  // z-chunks of this launch (all / interior / boundary)
        const int x0 = (tile % ntx) * TX, y0 = (tile / ntx) * TY;
        // bd = 0: uniform chunks of `depth` planes.  bd > 0 (split launches beside
        // a halo exchange): chunks 0 and nch-1 are the bd planes at either end
        // (the only ones whose stencils read ghost planes), the interior chunks
        // cover the rest in `depth`-plane pieces
        int z0, z1;
        if (bd == 0) {
            z0 = chunk * depth;
            z1 = min(z0 + depth, g.nz);
        } else if (chunk == 0) {
            z0 = 0;
            z1 = bd;
        } else if (chunk == nch - 1) {
            z0 = g.nz - bd;
            z1 = g.nz;
        } else {
            z0 = bd + (chunk - 1) * depth;
            z1 = min(z0 + depth, g.nz - bd);
        }
        const int cx = SF_OX + x0 - 2;        // TMA x coordinate of the box
        const int cyx = y0, cyc = y0 + 1;     // TMA y coordinates (x box, coef box)
        const unsigned seq0 = seq;            // pre-bundle; bundle q -> seq0 + 2 + q - z0

        // bundle q: x(q+1), Dinv/rhs/beta_i/beta_j (q), beta_k(q+1); needed by R(q).
        // Part k of the bundle (0: arrive.expect_tx + x, 1..4: coefficient
        // arrays, 5: beta_k), all issued by thread 0 after the step's barrier
        // (spreading the parts over the warps' lane 0 measured slower, c1a7abc).
        const unsigned xs_u = smem_u32(Xs), cs_u = smem_u32(Cs), ks_u = smem_u32(Ks);
        const unsigned mb_u = smem_u32(mbar);
        auto issue_part = [&](int q, int part) {
            const unsigned sq = seq0 + 2 + (q - z0);
            const unsigned b = mb_u + 8u * (sq % NMB);
            if (part == 0) {
                mbar_expect_u(b, BUNDLE_BYTES);
                tma3u(xs_u + 8u * (md(q + 1, NXS) * XSLOT), &mp.x, cx, cyx, zplane(g, q + 1), b);
            } else if (part == 5) {
                tma3u(ks_u + 8u * (md(q + 1, NKS) * CARR), &mp.bk, cx, cyc, zplane(g, q + 1), b);
            } else {
                const unsigned c = cs_u + 8u * (md(q, NCS) * CSLOT + (part - 1) * CARR);
                const CUtensorMap* m = part == 1 ? &mp.dv : part == 2 ? &mp.rh : part == 3 ? &mp.bi : &mp.bj;
                tma3u(c, m, cx, cyc, zplane(g, q), b);
            }
        };
        auto issue = [&](int q) {
            for (int k = 0; k < 6; k++) issue_part(q, k);
        };
        if (tid == 0) {
            fence_proxy_async();  // generic smem writes of the previous item before TMA reuse
            unsigned long long* b = &mbar[seq0 % NMB];
            mbar_expect(b, 2 * XBYTES + CBYTES_S);
            tma3(Xs + md(z0 - 2, NXS) * XSLOT, &mp.x, cx, cyx, zplane(g, z0 - 2), b);
            tma3(Xs + md(z0 - 1, NXS) * XSLOT, &mp.x, cx, cyx, zplane(g, z0 - 1), b);
            tma3(Ks + md(z0 - 1, NKS) * CARR, &mp.bk, cx, cyc, zplane(g, z0 - 1), b);
            for (int q = z0 - 1; q <= min(z0 + PF - 2, z1); q++) issue(q);  // step t: t+PF+1
        }
        if (!waited) {
            pdl_wait();
            after_wait();
            waited = true;
        }

        // this thread's pair: row gy, cells gxa (even) and gxa+1
        // lanes [seg*PPR, (seg+1)*PPR) of warp w own row w + NWARP*seg (same parity)
        const int hl = lane % PPR, row = w + NWARP * (lane / PPR);
        const int gxa = x0 + 2 * hl, gy = y0 + row;
        const int xoff = (row + 2) * W + 2 * hl + 2;
        const int coff = (row + 1) * W + 2 * hl + 2;
        // ring cell of this thread for both parities of the plane (offsets + BC flags)
        int rxo[2], rco[2], rfl[2];
        bool rok[2];
        {
            const int rt = w * RING_PER_WARP + lane;
#pragma unroll
            for (int par = 0; par < 2; par++) {
                int rgx = 0, rgy = 0;
                bool ok = lane < RING_PER_WARP && rt < NRING;
                if (rt < TX) {
                    int pp = rt % (TX / 2);
                    rgy = (rt < TX / 2) ? y0 - 1 : y0 + TY;
                    rgx = x0 + 2 * pp + ((rgy + par) & 1);
                } else {
                    int m = rt - TX, side = m / (TY / 2);
                    m -= side * (TY / 2);
                    rgx = side ? x0 + TX : x0 - 1;
                    int gyp = y0 + 2 * m;
                    rgy = gyp + ((rgx + gyp + par) & 1);
                }
                ok = ok && rgx >= 0 && rgx < g.nx && rgy >= 0 && rgy < g.ny;
                rok[par] = ok;
                rxo[par] = (rgy - y0 + 2) * W + rgx - x0 + 2;
                rco[par] = (rgy - y0 + 1) * W + rgx - x0 + 2;
                rfl[par] = (rgx == 0) | ((rgx == g.nx - 1) << 1) | ((rgy == 0) << 2) |
                           ((rgy == g.ny - 1) << 3);
            }
        }
        double stA[8], stB[8];
#pragma unroll
        for (int i = 0; i < 8; i++) stA[i] = stB[i] = 0.0;

        // rotating slot indices for step t = z0-2: R(z0-1) / B(z0-3)
        // x slots: x(t-2) .. x(t+2)
        int ix_m2 = md(z0 - 4, NXS), ix_m1 = md(z0 - 3, NXS), ix_0 = md(z0 - 2, NXS),
            ix_p1 = md(z0 - 1, NXS), ix_p2 = md(z0, NXS);
        int ic = md(z0 - 1, NCS);                       // coef(t+1)
        int ik1 = md(z0 - 1, NKS), ik2 = md(z0, NKS);   // beta_k(t+1), beta_k(t+2)
        mbar_wait(&mbar[seq0 % NMB], (seq0 / NMB) & 1);
        // INTERP (A8 P0 fused): x(p) += e_c(parent) in smem, once per plane, one
        // step before its first read; the two parents a thread needs for plane
        // p are loaded (L2) one step earlier still.
        const int ep0 = tid, ep1 = tid + NT;   // x-box pairs of this thread
        // in-plane offsets of their coarse parents (fixed per item): only the
        // coarse plane (p >> 1) changes from step to step
        // (32-bit offsets: a coarse part holds < 2^31 doubles; the step code
        // then costs two integer ops per load instead of 64-bit address math)
        auto e_inplane = [&](int pr) -> int {
            const int r = pr / (W / 2), c2 = pr - r * (W / 2);
            const int I = x0 / 2 - 1 + c2, J = y0 / 2 - 1 + (r >> 1);
            return (J + SF_GY) * (int)cv.js + SF_OX + I;
        };
        const int eo0 = INTERP ? e_inplane(ep0) : 0;
        const int eo1 = (INTERP && ep1 < XPAIRS) ? e_inplane(ep1) : eo0;
        const double* ebase = cv.e + (long)(cv.zoff + SF_GZ) * cv.ks;   // coarse plane 0
        const int cks = (int)cv.ks;
        auto load_e = [&](int p, double& e0, double& e1) {
            const int o = (p >> 1) * cks;
            e0 = __ldg(ebase + (o + eo0));
            e1 = __ldg(ebase + (o + eo1));
        };
        auto correct_slot = [&](int slot, double e0, double e1) {
            double* X = Xs + slot * XSLOT;
            double2 v = *(double2*)&X[2 * ep0];
            v.x = v.x + e0;
            v.y = v.y + e0;
            *(double2*)&X[2 * ep0] = v;
            if (ep1 < XPAIRS) {
                double2 u = *(double2*)&X[2 * ep1];
                u.x = u.x + e1;
                u.y = u.y + e1;
                *(double2*)&X[2 * ep1] = u;
            }
        };
        auto correct = [&](int p, double e0, double e1) { correct_slot(md(p, NXS), e0, e1); };
        // parents of the plane a step corrects, loaded two steps ahead (the
        // coarse field may come from DRAM, slower than one z step) into one of
        // two register sets that alternate with the steps (A: steps z0-2, z0, ..;
        // B: z0-1, z0+1, ..): each set is refilled right after its use, so no
        // register copy waits on a load in flight
        double eA0 = 0.0, eA1 = 0.0, eB0 = 0.0, eB1 = 0.0;
        if (INTERP) {
            mbar_wait(&mbar[(seq0 + 1) % NMB], ((seq0 + 1) / NMB) & 1);   // bundle z0-1: x(z0)
            for (int p = z0 - 2; p <= z0; p++) {
                double e0, e1;
                load_e(p, e0, e1);
                correct(p, e0, e1);
            }
            if (z0 + 1 <= z1 + 1) load_e(z0 + 1, eA0, eA1);
            if (z0 + 2 <= z1 + 1) load_e(z0 + 2, eB0, eB1);
            __syncthreads();
        }

        double rn0 = 0.0, rn1 = 0.0, rn2 = 0.0;   // red-new of planes t, t-1, t-2 at step t
        // RRF: y shares crossing to the neighbouring block row (other warps) go
        // through the x slot of plane t-2 at an odd-plane step t: its last
        // reader was B(t-2) at step t-1 and its TMA refill is issued after step
        // t+1, when the shares have been read (no extra shared memory: three
        // CTAs per SM stay resident)
        int yslot = 0;
        // RRF partials of the thread's pair column: the coarse plane being summed,
        // the previous one (waiting for its share of the next plane), the next
        // one's share carried from an odd plane, and the y share
        double rAcc = 0.0, rPend = 0.0, rCarry = 0.0, rY = 0.0;
        // own pair of planes t and t+1 at step t (INTERP: after their correction)
        double2 pq0 = *(const double2*)&Xs[ix_0 * XSLOT + xoff];
        double2 pq1 = *(const double2*)&Xs[ix_p1 * XSLOT + xoff];
        double2 bkc = *(const double2*)&Ks[ik1 * CARR + coff];   // beta_k(t+1) at step t
        auto step = [&](int t, double* stash, double& ce0, double& ce1) {
            // --- wait for bundle t+1 (R(t+1) operands)
            const int q = t + 1;
            if (!INTERP && q <= z1) {
                const unsigned sq = seq0 + 2 + (q - z0);
                mbar_wait(&mbar[sq % NMB], (sq / NMB) & 1);
            }

            const int gkr = g.z0 + q;                    // plane of R
            const bool rin = q <= z1 && gkr >= 0 && gkr < g.gnz;
            const bool bin = t - 1 >= z0;                // B(t-1) on the tile
            const int sel = (y0 + w + gkr) & 1;          // same for both row segments
            StepCtx s;                                   // centred on plane q = t+1 for R
            s.Xk = Xs + ix_p1 * XSLOT;
            s.Xm = Xs + ix_0 * XSLOT;
            s.Xp = Xs + ix_p2 * XSLOT;
            s.C = Cs + ic * CSLOT;
            s.Klo = Ks + ik1 * CARR;
            s.Khi = Ks + ik2 * CARR;
            StepCtx sb;                                  // centred on plane t-1 for B
            sb.Xk = Xs + ix_0 * XSLOT;                   // x(t)   (top neighbour)
            sb.Xm = Xs + ix_m1 * XSLOT;                  // x(t-1) (the plane)
            sb.Xmm = Xs + ix_m2 * XSLOT;                 // x(t-2) (bottom neighbour)
            double nb[8];
            double rn = 0.0;
            double2 o = make_double2(0.0, 0.0);
            const bool zlo = gkr == 0, zhi = gkr == g.gnz - 1;
            const int gkm = g.z0 + t - 1;
            // planes t+1 and t-1 have the same parity: the black cell of
            // plane t-1 is the pair's other cell (position 1-sel)
            double rres = 0.0, bres = 0.0;
            const double2 pn = *(const double2*)&s.Xp[xoff];   // own pair, plane t+2
            double2 bkn = make_double2(0.0, 0.0);   // beta_k(t+2) at the own pair (R loads it)
            if (sel == 0) {
                if (rin) rn = red_pair<0, RESID>(s, xoff, coff, hl, gxa, gy, g, zlo, zhi, bh2, nb, rres, pq0, pq1, pn, bkc, bkn);
                if (bin) o = black_pair<1, BRES>(sb, xoff, gxa, gy, g, gkm, bh2, stash, bres, rn2, rn1, rn0);
            } else {
                if (rin) rn = red_pair<1, RESID>(s, xoff, coff, hl, gxa, gy, g, zlo, zhi, bh2, nb, rres, pq0, pq1, pn, bkc, bkn);
                if (bin) o = black_pair<0, BRES>(sb, xoff, gxa, gy, g, gkm, bh2, stash, bres, rn2, rn1, rn0);
            }
            if (RRF && bin) {   // delta-form residual + restriction partials (see the kernel head)
                const int bs = 1 - sel;                        // black cell's position in the pair (warp-uniform)
                const double bnew = bs ? o.y : o.x;
                const double bold = sb.Xm[xoff + bs];          // still the input value
                const double u = __dmul_rn(bh2, bnew - bold);
                const int p = t - 1;                           // its plane (single part: global)
                const bool pe = (p & 1) == 0, ye = (gy & 1) == 0;
                // stash: w, e, s, n, b, t faces of this black cell (boundary-zeroed betas)
                double own = __dmul_rn(bs ? stash[0] : stash[1], u);
                own = __fma_rn(ye ? stash[3] : stash[2], u, own);
                own = __fma_rn(pe ? stash[5] : stash[4], u, own);
                const double xo2 = __dmul_rn(bs ? stash[1] : stash[0], u);
                const double yo2 = __dmul_rn(ye ? stash[2] : stash[3], u);
                const double zo2 = __dmul_rn(pe ? stash[4] : stash[5], u);
                const int I = gxa >> 1, J = gy >> 1, K = p >> 1, rp = gy & 1;
                auto at = [&](int i, int j, int k) {
                    return (long)(k + SF_GZ) * rv.cks + (long)(j + SF_GY) * rv.cjs + SF_OX + i;
                };
                // x: the neighbouring pair column of this row is lane hl -+ 1 of the
                // 16-lane row segment; across the tile edge -> edge array (XW / XE)
                double xr = bs ? __shfl_up_sync(0xffffffffu, xo2, 1, PPR)
                               : __shfl_down_sync(0xffffffffu, xo2, 1, PPR);
                if (bs ? hl == 0 : hl == PPR - 1) xr = 0.0;
                if (!bs && hl == 0 && I > 0) (rp ? rv.a[3] : rv.a[2])[at(I - 1, J, K)] = xo2;
                if (bs && hl == PPR - 1 && I + 1 < rv.ncx) (rp ? rv.a[5] : rv.a[4])[at(I + 1, J, K)] = xo2;
                const double c2 = own + xr;
                if (pe) {
                    // z: down into block K-1 -- the pending partial when K-1 is this
                    // item's (written now, complete), else the ZB edge array;
                    // the y share of K-1 from the neighbouring row of the other
                    // block row arrived in shared memory at the last step
                    if (p > z0) {
                        rPend = rPend + zo2;
                        if (rp ? row + 1 < TY : row > 0) rPend = rPend + Xs[yslot * XSLOT + row * PPR + hl];
                        (rp ? rv.a[1] : rv.a[0])[at(I, J, K - 1)] = rPend;
                    } else if (K > 0) {
                        (rp ? rv.a[9] : rv.a[8])[at(I, J, K - 1)] = zo2;
                    }
                    rAcc = c2 + rCarry;   // rCarry: block K's share of plane 2K-1 (0 at the item start)
                    rCarry = 0.0;
                    rY = yo2;
                } else {
                    rAcc = rAcc + c2;
                    rY = rY + yo2;
                    // y: into the neighbouring row of the next block row (another
                    // warp) through shared memory -- read there next step, before
                    // its partial is written; across the tile edge, or on the
                    // item's last block (no next step), into the YS / YN arrays
                    const int trow = rp ? row + 1 : row - 1;
                    yslot = ix_m2;
                    if (p + 1 < z1 && trow >= 0 && trow < TY) Xs[ix_m2 * XSLOT + trow * PPR + hl] = rY;
                    else if (!rp && J > 0) rv.a[6][at(I, J - 1, K)] = rY;
                    else if (rp && J + 1 < rv.ncy) rv.a[7][at(I, J + 1, K)] = rY;
                    if (p + 1 < z1) {     // block K+1 is this item's: carry, K waits for its ZB share
                        rCarry = zo2;
                        rPend = rAcc;
                    } else {              // last block of the item: ZT edge, partial now
                        if (K + 1 < rv.ncz) (rp ? rv.a[11] : rv.a[10])[at(I, J, K + 1)] = zo2;
                        (rp ? rv.a[1] : rv.a[0])[at(I, J, K)] = rAcc;
                    }
                }
            }
            if (RESID && rin && q >= z0 && q < z1) {   // this item's planes only
                const unsigned long long m2 = abits(rres);
                rbits = m2 > rbits ? m2 : rbits;
            }
            if (BRES && bin) {
                const unsigned long long m2 = abits(bres);
                rbits = m2 > rbits ? m2 : rbits;
            }
            const int par = gkr & 1;
            const bool ring = rin && (par ? rok[1] : rok[0]);
            const int ro = par ? rxo[1] : rxo[0];
            double rr = 0.0;
            if (ring) rr = red_ring(s, ro, par ? rco[1] : rco[0], par ? rfl[1] : rfl[0], bh2, zlo, zhi);
            {
                double* Xw = Xs + ix_p1 * XSLOT;
                if (rin) Xw[xoff + sel] = rn;
                if (ring) Xw[ro] = rr;
            }
            rn2 = rn1;   // this thread's red-new values of planes t-1, t, t+1
            rn1 = rn0;
            rn0 = rn;
            pq0 = pq1;   // own pair (old values) of planes t+1, t+2 for the next step
            pq1 = pn;
            bkc = rin ? bkn : *(const double2*)&s.Khi[coff];   // beta_k(t+2): next step's bottom face
            if (bin)   // streaming store: do not evict halo lines other tiles still need
                __stcs((double2*)(xo + (long)zplane(g, t - 1) * g.ks + (long)(gy + SF_GY) * g.js +
                                  SF_OX + gxa), o);
#pragma unroll
            for (int i = 0; i < 8; i++) stash[i] = nb[i];
            // INTERP: correct x(t+3) (bundle t+2) at the END of the step: no one
            // reads that plane before step t+1, and the TMA had the whole step
            // (correcting at the start of the step instead measured slower:
            // the wait for bundle t+2 then stalls the step's stencils)
            if (INTERP && q + 1 <= z1) {
                const unsigned sq = seq0 + 2 + (q + 1 - z0);
                mbar_wait(&mbar[sq % NMB], (sq / NMB) & 1);
                correct_slot(ix_p2 + 1 == NXS ? 0 : ix_p2 + 1, ce0, ce1);   // x(t+3)
                if (t + 5 <= z1 + 1) load_e(t + 5, ce0, ce1);                // this set's next plane
            }
            fence_proxy_async();
            __syncthreads();
            // refill bundle t+PF+1 (its slots were last read before this barrier)
            if (tid == 0 && t + PF + 1 <= z1) issue(t + PF + 1);
            // rotate slots
            ix_m2 = ix_m1; ix_m1 = ix_0; ix_0 = ix_p1; ix_p1 = ix_p2;
            ix_p2 = (ix_p2 + 1 == NXS) ? 0 : ix_p2 + 1;
            ic = (ic + 1 == NCS) ? 0 : ic + 1;
            ik1 = ik2; ik2 = (ik2 + 1 == NKS) ? 0 : ik2 + 1;
        };
        // steps t = z0-2 .. z1; B(t-1) consumes the stash R(t-1) filled at step t-2
        for (int t = z0 - 2; t <= z1; t += 2) {
            step(t, stA, eA0, eA1);
            if (t + 1 <= z1) step(t + 1, stB, eB0, eB1);
        }
        seq = seq0 + 2 + (z1 - z0) + 1;
        __syncthreads();  // all reads of this item's slots done before the next prologue
    }
    if (timing) {
        atomicMax(&ts[2], gtimer());
        __threadfence();
        if (atomicAdd(&ts[3], 1ull) == gridDim.x - 1) {   // every CTA has stamped
            __threadfence();
            const unsigned long long t0 = atomicAdd(&ts[1], 0ull), t1 = atomicAdd(&ts[2], 0ull);
            if (!RRF) {   // the pair roofline covers the four pair variants
                ts[5] += t1 - t0;
                ts[4] += tcount;   // a split pair (interior + boundary launch) counts once
            }
            // per variant: 0 plain, 1 RESID, 2 BRES, 3 INTERP (with or without BRES), 4 RRF
            constexpr int var = RRF ? 4 : INTERP ? 3 : RESID ? 1 : BRES ? 2 : 0;
            ts[6 + 2 * var] += tcount;
            ts[7 + 2 * var] += t1 - t0;
            ts[1] = ~0ull;
            ts[2] = 0ull;
            ts[3] = 0ull;
        }
    }
    if (RESID || BRES) {   // CTA max -> one atomic (bit order = numeric order for |r|; NaN wins)
        __shared__ unsigned long long wmax[NWARP];
        for (int o2 = 16; o2 > 0; o2 >>= 1) {
            unsigned long long v = __shfl_xor_sync(0xffffffffu, rbits, o2);
            rbits = v > rbits ? v : rbits;
        }
        if (lane == 0) wmax[w] = rbits;
        __syncthreads();
        if (tid == 0) {
            for (int i = 1; i < NWARP; i++) rbits = wmax[i] > rbits ? wmax[i] : rbits;
            atomicMax((unsigned long long*)rmax, rbits);
        }
    }
}

// ---------------------------------------------------------------- host side
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

sf_status get_encoder() {
    if (g_encode) return SF_OK;
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    g_encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    return SF_OK;
}

// 3-D map over one field allocation: dims (js, ny+2GY, lnz+2GZ), box (W, rows, 1)
sf_status encode(CUtensorMap* m, const sf_level* L, const double* base, int rows) {
    cuuint64_t dims[3] = {(cuuint64_t)L->js, (cuuint64_t)(L->ny + 2 * SF_GY),
                          (cuuint64_t)(L->lnz + 2 * SF_GZ)};
    cuuint64_t strides[2] = {(cuuint64_t)L->js * 8, (cuuint64_t)L->ks * 8};
    cuuint32_t box[3] = {(cuuint32_t)W, (cuuint32_t)rows, 1};
    cuuint32_t es[3] = {1, 1, 1};
    // L2 fill granularity of the box loads (SF_TMA_PROMO = 0/64/128/256 for A/B runs)
    CUtensorMapL2promotion promo = CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    if (const char* e = getenv("SF_TMA_PROMO")) {
        const int v = atoi(e);
        promo = v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                : v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                : v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    }
    CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)base, dims, strides, box, es,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, promo,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    return SF_OK;
}

int g_num_sms = 0;

}  // namespace

bool SF_CAT(gsrb_fused_supported, SF_GSRB_SUFFIX)(const sf_level* L) {
    return L->nx % TX == 0 && L->ny % TY == 0 && L->lnz >= 1;
}

static __global__ void zero_bits(double* p) { pdl_wait(); *p = 0.0; }

template <bool R, bool I, bool B, bool F = false>
static sf_status set_attrs() {
    SF_CUDA(cudaFuncSetAttribute(gsrb_pair_tma_kernel<R, I, B, F>,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM));
    if (MINB > 1)   // room for MINB CTAs per SM
        SF_CUDA(cudaFuncSetAttribute(gsrb_pair_tma_kernel<R, I, B, F>,
                                     cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    return SF_OK;
}

// rmode SF_RM_INPUT_RED: reduce max |rhs - A x| over the red cells of the
// INPUT into *rmax (no reset: the BRES pair that produced the input holds the
// black part there).  SF_RM_OUTPUT_BLACK: reset *rmax, reduce the black cells
// of the OUTPUT.  The caller all-reduces *rmax across ranks.
// C != NULL: fuse fine.xin += P0(C.cf) (A8, V-cycle) into the pair (INTERP).
// phase 0: every z-chunk; 1: the interior chunks [1, nch-1) with `reserve` SMs
// left free (the halo exchange runs beside it); 2: the boundary chunks 0 and
// nch-1, which read the exchanged ghost planes.  Phases 1 and 2 use at least
// 3 chunks per part.
sf_status SF_CAT(k_gsrb_pair_fused, SF_GSRB_SUFFIX)(sf_level* L, int xin, int xout, int rhs, double a,
                                                    double b, double* rmax, sf_level* C, int cf,
                                                    int phase, int reserve, int rmode, SfRRF* rrf) {
    if (rrf && (phase != 0 || C || rmode != SF_RM_NONE || L->nlocal != 1 || L->nparts != 1 || (L->lnz & 1)))
        return sf_fail(SF_ERR_INVALID, "RRF pair: single-part level, even nz, plain pair only");
    if (!SF_CAT(gsrb_fused_supported, SF_GSRB_SUFFIX)(L)) return sf_fail(SF_ERR_SHAPE, "fused GSRB needs nx%%%d==0, ny%%%d==0", TX, TY);
    if (rmode != SF_RM_NONE && !rmax) return sf_fail(SF_ERR_INVALID, "residual mode needs a scalar");
    if (rmode == SF_RM_INPUT_RED && C) return sf_fail(SF_ERR_INVALID, "input residual with P0 fusion");
    SF_TRY(get_encoder());
    static bool attr = false;
    if (!attr) {
        SF_TRY((set_attrs<false, false, false>()));
        SF_TRY((set_attrs<true, false, false>()));
        SF_TRY((set_attrs<false, true, false>()));
        SF_TRY((set_attrs<false, false, true>()));
        SF_TRY((set_attrs<false, true, true>()));
        SF_TRY((set_attrs<false, false, false, true>()));
        int dev;
        SF_CUDA(cudaGetDevice(&dev));
        SF_CUDA(cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev));
        attr = true;
    }
    const int ntx = L->nx / TX, nty = L->ny / TY, tiles = ntx * nty;
    // chunk depth: minimise rounds * (depth + prologue) over persistent CTAs
    const int G = g_num_sms * MINB;   // resident CTAs
    int best_d = L->lnz;
    double best = 1e30;
    const int min_nch = phase ? 3 : 1;
    if (L->lnz < min_nch) return sf_fail(SF_ERR_SHAPE, "split fused pair needs >= 3 planes per part");
    // shallowest chunk considered (SF_GSRB_MIND, A/B knob; 8 before r02): small
    // levels whose items fit one round of resident CTAs want shallow chunks
    // (fewer serial z steps per CTA); big levels pick deep ones anyway
    static const int mind = getenv("SF_GSRB_MIND") ? std::max(1, atoi(getenv("SF_GSRB_MIND"))) : 1;
    for (int nch = min_nch; nch <= L->lnz; nch++) {
        int d = (L->lnz + nch - 1) / nch;
        if (d < mind && nch > min_nch) break;
        if ((L->lnz + d - 1) / d < min_nch) continue;
        int n = (L->lnz + d - 1) / d;
        long items = (long)tiles * n;
        double rounds = (double)((items + G - 1) / G);
        double cost = rounds * (d + 3.0);
        if (cost < best - 1e-9) { best = cost; best_d = d; }
    }
    const char* ed = getenv("SF_GSRB_DEPTH");   // tuning override
    if (ed && atoi(ed) > 0) best_d = std::min(L->lnz, atoi(ed));
    const int Gl = phase == 1 ? std::max(1, g_num_sms - reserve) * MINB : G;
    // split launches (phase 1 interior beside the halo exchange, phase 2 the two
    // boundary chunks after it): thin boundary chunks of bd planes, so the part
    // that waits for the halo is small; the interior depth from the same cost
    // model over the resident CTAs phase 1 gets
    int bd = 0;
    if (phase) {
        const char* eb = getenv("SF_SPLIT_BD");
        bd = std::max(2, std::min(eb && atoi(eb) > 0 ? atoi(eb) : 2, L->lnz / 3));
        const int P = L->lnz - 2 * bd;
        best = 1e30;
        best_d = P;
        for (int nc = 1; nc <= P; nc++) {
            const int d = (P + nc - 1) / nc;
            if (d < 8 && nc > 1) break;
            const long it = (long)tiles * ((P + d - 1) / d);
            const double cost = (double)((it + Gl - 1) / Gl) * (d + 3.0);
            if (cost < best - 1e-9) { best = cost; best_d = d; }
        }
        if (ed && atoi(ed) > 0) best_d = std::min(P, atoi(ed));
    }
    // RRF: every item holds whole coarse planes (even chunk depth)
    if (rrf && (best_d & 1)) best_d = std::min(L->lnz, best_d + 1);
    if (rrf) rrf->zdepth = best_d;   // the fix-up reads the z-edge arrays at chunk edges
    const int depth = best_d;
    const int nch = phase ? 2 + (L->lnz - 2 * bd + depth - 1) / depth : (L->lnz + depth - 1) / depth;
    const int c0 = phase == 1 ? 1 : 0;
    const int cstride = phase == 2 ? nch - 1 : 1;
    const int items = tiles * (phase == 0 ? nch : phase == 1 ? nch - 2 : 2);
    const double bh2 = b / (L->h * L->h);
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        Maps mp;
        SF_TRY(encode(&mp.x, L, v.f[xin], XH));
        SF_TRY(encode(&mp.dv, L, v.f[SF_DINV], CHS));
        SF_TRY(encode(&mp.rh, L, v.f[rhs], CHS));
        SF_TRY(encode(&mp.bi, L, v.f[SF_BI0], CHS));
        SF_TRY(encode(&mp.bj, L, v.f[SF_BJ0], CHH));
        SF_TRY(encode(&mp.bk, L, v.f[SF_BK0], CHS));
        Geo g{v.nx, v.ny, v.nz, v.z0, v.gnz, v.js, v.ks, 0};
        if (const char* ez = getenv("SF_DBG_ZMASK"))   // measurement only (see zplane)
            if (atoi(ez) > 0 && v.nz > atoi(ez)) g.zmask = atoi(ez);
        int grid = std::min(items, Gl);
        CoarseView cvw{nullptr, 0, 0, 0};
        if (C) {
            const bool rep = C->nparts == 1 && L->nparts > 1;
            PV c = sf_view(C, rep ? 0 : p);
            cvw = CoarseView{c.f[cf], C->js, C->ks, rep ? v.z0 / 2 : 0};
        }
        if (rmode == SF_RM_OUTPUT_BLACK && p == 0 && phase != 2) {
            sf_launch(zero_bits, 1, 1, 0, L->stream, rmax);
            SF_LAUNCHED();
        }
        // (after a zero_bits launch the pair cannot start early)
        const int early = L->pdl_early && phase == 0 && L->nlocal == 1 && rmode != SF_RM_OUTPUT_BLACK &&
                          sf_pdl_on();
        const int zr = rmode == SF_RM_ZERO && p == 0 && phase != 2;
        const bool bres = rmode == SF_RM_OUTPUT_BLACK || rmode == SF_RM_OUTPUT_BLACK_ZEROED;
        double* xo = v.f[xout];
        const SfRRF rv = rrf ? *rrf : SfRRF{};
#define SF_LAUNCH_PAIR(R, I, B, ...)                                                                \
    sf_launch(gsrb_pair_tma_kernel<R, I, B, ##__VA_ARGS__>, grid, NT, SMEM, L->stream, mp, g, xo, a, bh2, depth, ntx, tiles, \
                                                                items, rmax, cvw, c0, cstride, \
              (unsigned long long*)(L->dscratch + SF_TS_OFF), bd, nch, phase == 1 ? 0 : 1, zr, early, rv)
        if (rrf) SF_LAUNCH_PAIR(false, false, false, true);
        else if (rmode == SF_RM_INPUT_RED) SF_LAUNCH_PAIR(true, false, false);
        else if (bres && C) SF_LAUNCH_PAIR(false, true, true);
        else if (bres) SF_LAUNCH_PAIR(false, false, true);
        else if (C) SF_LAUNCH_PAIR(false, true, false);
        else SF_LAUNCH_PAIR(false, false, false);
#undef SF_LAUNCH_PAIR
        SF_LAUNCHED();
    }
    L->pdl_early = 0;
    return sf_check_launch("gsrb_pair_tma");
}
