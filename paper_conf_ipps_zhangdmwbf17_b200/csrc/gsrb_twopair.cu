// NEXT-1: temporal blocking of a whole smooth -- TWO red-black pairs (4 GS
// sweeps) in ONE pass over HBM (the
// multicolour reordering / tiling of PAPER.md:565-577 carried one step further
// than the colour-fused pair of gsrb_fused.cu).
//
// A CTA owns a 32x8 (x,y) tile and streams it along z.  Four stages run as a
// wavefront, each on its own plane of the same z step t:
//   R1(t)    red cells of pair 1 on the tile + a 3-cell ring     (x0 -> x1 red)
//   B1(t-2)  black cells of pair 1 on the tile + a 2-cell ring   (x0 -> x1 black)
//   R2(t-4)  red cells of pair 2 on the tile + a 1-cell ring     (x1 -> x2 red)
//   B2(t-6)  black cells of pair 2 on the tile                   (x1 -> x2 black)
// The rings are recomputed bit-identically by every CTA whose tile they
// border, so no stage ever needs another CTA's results: each stage reads only
// values the previous stages of this CTA wrote in earlier steps.  x0 arrives
// by TMA (cp.async.bulk.tensor.3d, one box of the tile + a 4-cell ring per
// plane, mbarrier per plane, PF planes ahead) into shared memory, where the
// first three stages update it in place (a plane's slot lives from its load
// until B2 of the plane above has read its pair-2 reds: 9 + PF slots); B2
// writes the smoothed tile (both colours) to the output field.  HBM sees x
// once in and once out per SMOOTH instead of per pair; the coefficients
// (lambda, rhs, beta) are read per stage through L1 / L2 (the four stages touch
// each plane within 7 steps of one another), so from HBM about once.
//
// Every update is the colour-fused pair's lambda-form update with the same
// explicit contractions (tma_common.cuh: sum6, gs_q), so the result is
// bit-identical to two sf_smooth_gsrb(FUSED) pairs.  Single-part levels
// (the x box needs planes 4 beyond the item, which slab halos do not carry);
// opt-in (SF_SMOOTH_FUSED2): on B200 the colour-fused pair is SM-bound in the
// solve, so trading SM work for HBM traffic loses.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdlib>

#include "sf_internal.h"

namespace {

#include "tma_common.cuh"

constexpr int TX = 32, TY = 8;        // tile (cells)
constexpr int RG = 4;                 // ring of the x box
constexpr int XW = TX + 2 * RG;       // 40
constexpr int XH = TY + 2 * RG;       // 16
constexpr int XSLOT = XW * XH;        // 640 doubles
constexpr int NT = 256;               // threads
constexpr int PF = 2;                 // planes loaded ahead of R1's newest plane
constexpr int NXS = 9 + PF;           // x slots: planes t-7 .. t+1 live, + PF in flight
constexpr int MINB = 2;
constexpr size_t SMEM = sizeof(double) * NXS * XSLOT + 8 * NXS + 64;
static_assert(MINB * (SMEM + 1024) <= 228 * 1024, "two CTAs per SM");

struct Geo {
    int nx, ny, nz;
    long js, ks;
    const double* dv;   // lambda = Dinv
    const double* rh;   // rhs
    const double* bi;
    const double* bj;
    const double* bk;
};

// lambda-form GS update of cell (gx, gy, gz) whose x lives at smem offset o of
// the plane slots Xc (its plane), Xm (below), Xp (above): the fused pair's
// red_pair / black_pair / red_ring expression term for term
__device__ __forceinline__ double upd(const Geo& g, const double* Xc, const double* Xm,
                                      const double* Xp, int o, int gx, int gy, int gz, double bh2) {
    const long q = (long)(gz + SF_GZ) * g.ks + (long)(gy + SF_GY) * g.js + SF_OX + gx;
    const double xw = gx == 0 ? 0.0 : Xc[o - 1];
    const double xe = gx == g.nx - 1 ? 0.0 : Xc[o + 1];
    const double xs = gy == 0 ? 0.0 : Xc[o - XW];
    const double xn = gy == g.ny - 1 ? 0.0 : Xc[o + XW];
    const double xb = gz == 0 ? 0.0 : Xm[o];
    const double xt = gz == g.nz - 1 ? 0.0 : Xp[o];
    const double S = sum6(xw, xe, xs, xn, xb, xt, __ldg(g.bi + q), __ldg(g.bi + q + 1), __ldg(g.bj + q),
                          __ldg(g.bj + q + g.js), __ldg(g.bk + q), __ldg(g.bk + q + g.ks));
    return __dmul_rn(__ldg(g.dv + q), gs_q(__ldg(g.rh + q), bh2, S));
}

// one colour of plane p on the tile + an r-cell ring, in place in slot Xc
template <int R>
__device__ __forceinline__ void stage(const Geo& g, double* Xc, const double* Xm, const double* Xp,
                                      int x0, int y0, int p, int colour, double bh2) {
    constexpr int W = TX + 2 * R, H = TY + 2 * R, NP = (W / 2) * H;   // cell pairs of the region
    for (int w = threadIdx.x; w < NP; w += NT) {
        const int ry = w / (W / 2), rx = 2 * (w - ry * (W / 2));
        const int gy = y0 - R + ry;
        int gx = x0 - R + rx;
        gx += (gx + gy + p + colour) & 1;          // the pair's cell of this colour
        if (gx < 0 || gx >= g.nx || gy < 0 || gy >= g.ny) continue;
        const int o = (gy - y0 + RG) * XW + (gx - x0 + RG);
        Xc[o] = upd(g, Xc, Xm, Xp, o, gx, gy, p, bh2);
    }
}

// B2 on the tile: black cells of plane p; the pair (red from the slot, black
// computed) goes to the output field with a 16-byte streaming store
__device__ __forceinline__ void stage_out(const Geo& g, const double* Xc, const double* Xm,
                                          const double* Xp, double* __restrict__ out, int x0, int y0,
                                          int p, double bh2) {
    constexpr int NP = (TX / 2) * TY;
    for (int w = threadIdx.x; w < NP; w += NT) {
        const int ry = w / (TX / 2), rx = 2 * (w - ry * (TX / 2));
        const int gy = y0 + ry, gxa = x0 + rx;
        const int sel = (gxa + gy + p + 1) & 1;    // position of the black cell in the pair
        const int gx = gxa + sel;
        const int o = (gy - y0 + RG) * XW + (gx - x0 + RG);
        const double bnew = upd(g, Xc, Xm, Xp, o, gx, gy, p, bh2);
        const double red = Xc[o - (sel ? 1 : -1)];
        __stcs((double2*)(out + (long)(p + SF_GZ) * g.ks + (long)(gy + SF_GY) * g.js + SF_OX + gxa),
               sel ? make_double2(red, bnew) : make_double2(bnew, red));
    }
}

__global__ void __launch_bounds__(NT, MINB)
gsrb_twopair_kernel(const __grid_constant__ CUtensorMap mx, Geo g, double* __restrict__ out, double bh2,
                    int depth, int ntx, int ntiles, int nitems) {
    pdl_wait();
    extern __shared__ __align__(128) double sm[];
    double* Xs = sm;
    unsigned long long* mbar = (unsigned long long*)(Xs + NXS * XSLOT);
    if (threadIdx.x == 0) {
        for (int i = 0; i < NXS; i++) mbar_init(&mbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    // planes are loaded in a CTA-wide sequence: load n goes to slot n % NXS and
    // completes phase (n / NXS) & 1 of that slot's barrier
    unsigned seq = 0;
    for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int ci = item / ntiles, tile = item - ci * ntiles;
        const int x0 = (tile % ntx) * TX, y0 = (tile / ntx) * TY;
        const int z0 = ci * depth, z1 = min(z0 + depth, g.nz);
        // x0 planes z0-4 .. z1+3 (R1 covers z0-3 .. z1+2); plane q is load base + q
        const unsigned base = seq - (unsigned)(z0 - 4);
        auto slot = [&](int q) { return Xs + ((base + (unsigned)q) % NXS) * XSLOT; };
        auto issue = [&](int q) {
            const unsigned n = base + (unsigned)q, sl = n % NXS;
            mbar_expect(&mbar[sl], XSLOT * 8);
            tma3(Xs + sl * XSLOT, &mx, SF_OX + x0 - RG, SF_GY + y0 - RG, q + SF_GZ, &mbar[sl]);
        };
        auto wait = [&](int q) {
            const unsigned n = base + (unsigned)q;
            mbar_wait(&mbar[n % NXS], (n / NXS) & 1);
        };
        if (threadIdx.x == 0) {
            fence_proxy_async();   // generic writes of the previous item before TMA reuse
            for (int q = z0 - 4; q <= min(z0 - 2 + PF, z1 + 3); q++) issue(q);
        }
        wait(z0 - 4);
        wait(z0 - 3);
        for (int t = z0 - 3; t <= z1 + 5; t++) {
            if (t + 1 <= z1 + 3) wait(t + 1);   // R1(t) needs x0(t+1)
            if (t <= z1 + 2 && t >= 0 && t < g.nz)
                stage<3>(g, slot(t), slot(t - 1), slot(t + 1), x0, y0, t, 0, bh2);
            const int p1 = t - 2;
            if (p1 >= z0 - 2 && p1 <= z1 + 1 && p1 >= 0 && p1 < g.nz)
                stage<2>(g, slot(p1), slot(p1 - 1), slot(p1 + 1), x0, y0, p1, 1, bh2);
            const int p2 = t - 4;
            if (p2 >= z0 - 1 && p2 <= z1 && p2 >= 0 && p2 < g.nz)
                stage<1>(g, slot(p2), slot(p2 - 1), slot(p2 + 1), x0, y0, p2, 0, bh2);
            const int p3 = t - 6;
            if (p3 >= z0 && p3 < z1) stage_out(g, slot(p3), slot(p3 - 1), slot(p3 + 1), out, x0, y0, p3, bh2);
            fence_proxy_async();
            __syncthreads();
            // plane t+2+PF reuses the slot of plane t-7, last read by B2(t-6) above
            if (threadIdx.x == 0 && t + 2 + PF <= z1 + 3) issue(t + 2 + PF);
        }
        seq = base + (unsigned)(z1 + 4);
        __syncthreads();
    }
}

PFN_cuTensorMapEncodeTiled_v12000 g_enc2 = nullptr;
int g_sms2 = 0;

}  // namespace

bool gsrb_twopair_supported(const sf_level* L) {
    return L->nparts == 1 && L->nlocal == 1 && L->nx % TX == 0 && L->ny % TY == 0 && L->lnz >= 1;
}

// xout = two RB pairs of xin (NEXT-1); out of place like the fused pair
sf_status k_gsrb_twopair(sf_level* L, int xin, int xout, int rhs, double a, double b) {
    (void)a;   // lambda form: a enters through Dinv only
    if (!gsrb_twopair_supported(L))
        return sf_fail(SF_ERR_SHAPE, "two-pair smoother needs a single-part level, nx%%32 == 0, ny%%8 == 0");
    if (!g_enc2) {
        cudaDriverEntryPointQueryResult qr;
        void* fn = nullptr;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &qr);
        if (e != cudaSuccess || qr != cudaDriverEntryPointSuccess || !fn)
            return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
        g_enc2 = (PFN_cuTensorMapEncodeTiled_v12000)fn;
        SF_CUDA(cudaFuncSetAttribute(gsrb_twopair_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)SMEM));
        SF_CUDA(cudaFuncSetAttribute(gsrb_twopair_kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     100));
        int dev;
        SF_CUDA(cudaGetDevice(&dev));
        SF_CUDA(cudaDeviceGetAttribute(&g_sms2, cudaDevAttrMultiProcessorCount, dev));
    }
    PV v = sf_view(L, 0);
    CUtensorMap mx;
    {
        cuuint64_t dims[3] = {(cuuint64_t)L->js, (cuuint64_t)(L->ny + 2 * SF_GY),
                              (cuuint64_t)(L->lnz + 2 * SF_GZ)};
        cuuint64_t strides[2] = {(cuuint64_t)L->js * 8, (cuuint64_t)L->ks * 8};
        cuuint32_t box[3] = {(cuuint32_t)XW, (cuuint32_t)XH, 1};
        cuuint32_t es[3] = {1, 1, 1};
        // boxes reaching past the storage (rows / planes beyond the ghost zone,
        // all outside the domain) are zero-filled and never used
        CUresult r = g_enc2(&mx, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)v.f[xin], dims, strides, box, es,
                            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    }
    Geo g{v.nx, v.ny, v.nz, v.js, v.ks, v.f[SF_DINV], v.f[rhs], v.f[SF_BETA_I], v.f[SF_BETA_J],
          v.f[SF_BETA_K]};
    const int ntx = L->nx / TX, tiles = ntx * (L->ny / TY);
    // chunk depth: minimise rounds * (depth + 9 prologue / drain steps)
    static int per_sm = 0;
    if (!per_sm) {
        SF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gsrb_twopair_kernel, NT, SMEM));
        per_sm = std::max(per_sm, 1);
    }
    const int G = g_sms2 * per_sm;
    int best_d = L->lnz;
    double best = 1e30;
    for (int nch = 1; nch <= L->lnz; nch++) {
        const int d = (L->lnz + nch - 1) / nch;
        const long items = (long)tiles * ((L->lnz + d - 1) / d);
        const double cost = (double)((items + G - 1) / G) * (d + 9.0);
        if (cost < best - 1e-9) { best = cost; best_d = d; }
    }
    if (const char* e = getenv("SF_TWOPAIR_DEPTH"))
        if (atoi(e) > 0) best_d = std::min(L->lnz, atoi(e));
    const int items = tiles * ((L->lnz + best_d - 1) / best_d);
    const double bh2 = b / (L->h * L->h);
    sf_launch(gsrb_twopair_kernel, std::min(items, G), NT, SMEM, L->stream, mx, g, v.f[xout], bh2, best_d,
              ntx, tiles, items);
    SF_LAUNCHED();
    return sf_check_launch("gsrb_twopair");
}
