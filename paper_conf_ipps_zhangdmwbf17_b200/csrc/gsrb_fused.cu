// Colour-fused Gauss-Seidel red-black pair (A5) for sm_100a, fp64, TMA-fed.
//
// One kernel pass performs a whole RB pair -- [BC, red, BC, black] of
// PAPER.md:641-644 with x += lambda*(rhs - Ax) (Fig 4) --
// so the 64 B/cell compulsory traffic of PAPER.md:669-672 is paid once per
// pair instead of once per colour sweep.  It is the B200 counterpart of the
// paper's "multicolor reordering" and OpenCL "tall-skinny blocking" (2-D tiles
// rolled up through the remaining dimension):
//
//   (x,y) tile of 64 x 8 cells, streamed along z by one CTA; step p runs
//   R(p)    red cells of plane p on the tile AND on a one-cell ring around it
//           (the ring belongs to neighbouring tiles; recomputing it here,
//           bit-identically, means the black update needs no other CTA), then
//   B(p-1)  black cells of plane p-1 on the tile, which read red-new values of
//           planes p-2, p-1 (incl. ring) and p.
//
// Out of place (xin -> xout): the 2-ring reads of xin must see OLD values
// whatever neighbouring CTAs have written, so the pair writes a second buffer
// and the level swaps U <-> TMP.
//
// Data movement (Blackwell): every operand plane -- x (tile + 2-ring), alpha,
// Dinv, rhs, beta_i, beta_j (tile + 1-ring) and beta_k -- arrives by TMA
// (cp.async.bulk.tensor.3d) into shared memory, completion tracked by an
// mbarrier per plane "bundle", two planes ahead of use (~85 KB in flight per
// SM).  One elected thread issues; all 8 warps compute from shared memory
// (16-byte pair loads + warp shuffles for the x-neighbours); the output pair
// is stored with coalesced 16-byte stores.  Persistent CTAs (one per SM, 190
// KB smem) walk (tile, z-chunk) items in chunk-major order so neighbouring
// tiles stream the same planes at the same time (ring/halo reads hit L2).
//
// Dirichlet BC is folded in: a neighbour across a global face reads -x(c)
// (PAPER.md:336-341).  Part (slab) interfaces read exchanged halo planes
// (x depth 2, coefficients depth 2, rhs depth 1).
#include <cuda.h>
#include <cudaTypedefs.h>

#include "sf_internal.h"

namespace {

constexpr int TX = 64;                 // tile width  = 32 lanes x 2 cells
constexpr int TY = 8;                  // tile height = 8 warps
constexpr int NT = 32 * TY;            // 256 threads
constexpr int W = TX + 4;              // smem row: gx in [x0-2, x0+TX+2)
constexpr int XH = TY + 4;             // x rows:   gy in [y0-2, y0+TY+2)
constexpr int CHH = TY + 3;            // coef rows: gy in [y0-1, y0+TY+2)
constexpr int NXS = 6, NCS = 4, NKS = 5, NMB = 4;  // slot counts
constexpr int NCA = 5;                 // staged coefficient arrays per plane (beta_k separate)
constexpr int XSLOT = XH * W;          // doubles (6528 B = 51 x 128)
constexpr int CARR = 752;              // 11*68 = 748 doubles padded to 128 B
constexpr int CSLOT = NCA * CARR;
constexpr int XBYTES = XH * W * 8, CBYTES = CHH * W * 8;
constexpr int BUNDLE_BYTES = XBYTES + (NCA + 1) * CBYTES;
constexpr size_t SMEM = sizeof(double) * (NXS * XSLOT + NCS * CSLOT + NKS * CARR) + 64;
enum { CA_AL = 0, CA_DV = 1, CA_RH = 2, CA_BI = 3, CA_BJ = 4 };
constexpr int NRING = TX + TX + TY / 2 + TY / 2;   // red ring cells per plane (72)

struct Maps {
    CUtensorMap x, al, dv, rh, bi, bj, bk;
};

__device__ __forceinline__ unsigned smem_u32(const void* p) {
    return (unsigned)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long* b, unsigned n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n));
}
__device__ __forceinline__ void mbar_expect(unsigned long long* b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n"
        "W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra W;\n}" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma3(void* dst, const CUtensorMap* m, int c0, int c1, int c2,
                                     unsigned long long* bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(dst)),
        "l"((unsigned long long)m), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ int md(int k, int m) { return ((k % m) + m) % m; }

// x <- x + Dinv (rhs - Ax); operator in the term order of op_at (kernels.cu)
__device__ __forceinline__ double gs_update(double xc, double xw, double xe, double xs, double xn,
                                            double xb, double xt, double bw, double be, double bs,
                                            double bn, double bb, double bt, double al, double dv,
                                            double rh, double a, double bh2) {
    double flux = be * (xe - xc);
    flux += bw * (xw - xc);
    flux += bn * (xn - xc);
    flux += bs * (xs - xc);
    flux += bt * (xt - xc);
    flux += bb * (xb - xc);
    double ax = a * al * xc - bh2 * flux;
    return xc + dv * (rh - ax);
}

struct Geo {
    int nx, ny, nz, z0, gnz;
    long js, ks;
};

__global__ void __launch_bounds__(NT, 1)
gsrb_pair_tma_kernel(const __grid_constant__ Maps mp, Geo g, double* __restrict__ xo, double a,
                     double bh2, int depth, int ntx, int ntiles, int nitems) {
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

    unsigned seq = 0;  // bundles issued by this CTA so far (all threads track it)
    for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int chunk = item / ntiles, tile = item - chunk * ntiles;
        const int x0 = (tile % ntx) * TX, y0 = (tile / ntx) * TY;
        const int z0 = chunk * depth, z1 = min(z0 + depth, g.nz);
        const int cx = SF_OX + x0 - 2;        // TMA x coordinate of the box
        const int cyx = y0, cyc = y0 + 1;     // TMA y coordinates (x box, coef box)
        const unsigned seq0 = seq;            // pre-bundle; bundle p -> seq0 + 2 + p - z0

        // bundle p: x(p+1), alpha/Dinv/rhs/beta_i/beta_j (p), beta_k(p+1)
        auto issue = [&](int p) {
            unsigned s = seq0 + 2 + (p - z0);
            unsigned long long* b = &mbar[s % NMB];
            mbar_expect(b, BUNDLE_BYTES);
            tma3(Xs + md(p + 1, NXS) * XSLOT, &mp.x, cx, cyx, p + 1 + SF_GZ, b);
            double* c = Cs + md(p, NCS) * CSLOT;
            tma3(c + CA_AL * CARR, &mp.al, cx, cyc, p + SF_GZ, b);
            tma3(c + CA_DV * CARR, &mp.dv, cx, cyc, p + SF_GZ, b);
            tma3(c + CA_RH * CARR, &mp.rh, cx, cyc, p + SF_GZ, b);
            tma3(c + CA_BI * CARR, &mp.bi, cx, cyc, p + SF_GZ, b);
            tma3(c + CA_BJ * CARR, &mp.bj, cx, cyc, p + SF_GZ, b);
            tma3(Ks + md(p + 1, NKS) * CARR, &mp.bk, cx, cyc, p + 1 + SF_GZ, b);
        };
        if (tid == 0) {
            fence_proxy_async();  // generic smem writes of the previous item before TMA reuse
            unsigned long long* b = &mbar[seq0 % NMB];
            mbar_expect(b, 2 * XBYTES + CBYTES);
            tma3(Xs + md(z0 - 2, NXS) * XSLOT, &mp.x, cx, cyx, z0 - 2 + SF_GZ, b);
            tma3(Xs + md(z0 - 1, NXS) * XSLOT, &mp.x, cx, cyx, z0 - 1 + SF_GZ, b);
            tma3(Ks + md(z0 - 1, NKS) * CARR, &mp.bk, cx, cyc, z0 - 1 + SF_GZ, b);
            issue(z0 - 1);
            if (z0 <= z1) issue(z0);
        }
        mbar_wait(&mbar[seq0 % NMB], (seq0 / NMB) & 1);

        // this thread's pair: row gy, cells gxa (x even) and gxa+1
        const int gy = y0 + w, gxa = x0 + 2 * lane;
        const int xr = w + 2, cr = w + 1, c0 = 2 * lane + 2;
        double rb[9];  // black-cell coefficients of the previous plane (for B)
#pragma unroll
        for (int i = 0; i < 9; i++) rb[i] = 0.0;

        for (int p = z0 - 1; p <= z1; p++) {
            const unsigned s = seq0 + 2 + (p - z0);
            mbar_wait(&mbar[s % NMB], (s / NMB) & 1);
            const int gk = g.z0 + p;
            const bool kin = gk >= 0 && gk < g.gnz;
            const bool zlo = gk == 0, zhi = gk == g.gnz - 1;
            const double* Xk = Xs + md(p, NXS) * XSLOT;
            const double* Xm = Xs + md(p - 1, NXS) * XSLOT;
            const double* Xp = Xs + md(p + 1, NXS) * XSLOT;
            const double* C = Cs + md(p, NCS) * CSLOT;
            const double* Klo = Ks + md(p, NKS) * CARR;
            const double* Khi = Ks + md(p + 1, NKS) * CARR;

            // ------------------------------------------------ R(p): tile
            const int sel = (gy + gk) & 1;  // 1: the red cell is the odd one (b)
            double2 xp2 = *(const double2*)&Xk[xr * W + c0];
            double xl = __shfl_up_sync(0xffffffffu, xp2.y, 1);
            double xr_ = __shfl_down_sync(0xffffffffu, xp2.x, 1);
            if (lane == 0) xl = Xk[xr * W + 1];
            if (lane == 31) xr_ = Xk[xr * W + TX + 2];
            double2 al2 = *(const double2*)&C[CA_AL * CARR + cr * W + c0];
            double2 dv2 = *(const double2*)&C[CA_DV * CARR + cr * W + c0];
            double2 rh2 = *(const double2*)&C[CA_RH * CARR + cr * W + c0];
            double2 bi2 = *(const double2*)&C[CA_BI * CARR + cr * W + c0];
            double bie = __shfl_down_sync(0xffffffffu, bi2.x, 1);
            if (lane == 31) bie = C[CA_BI * CARR + cr * W + TX + 2];
            double2 bjl = *(const double2*)&C[CA_BJ * CARR + cr * W + c0];
            double2 bjh = *(const double2*)&C[CA_BJ * CARR + (cr + 1) * W + c0];
            double2 bkl = *(const double2*)&Klo[cr * W + c0];
            double2 bkh = *(const double2*)&Khi[cr * W + c0];
            double rnew = 0.0;
            if (kin) {
                const int gx = gxa + sel, col = c0 + sel;
                double xc = sel ? xp2.y : xp2.x;
                double xw = sel ? xp2.x : xl;
                double xe = sel ? xr_ : xp2.y;
                if (gx == 0) xw = -xc;
                if (gx == g.nx - 1) xe = -xc;
                double xs = (gy == 0) ? -xc : Xk[(xr - 1) * W + col];
                double xn = (gy == g.ny - 1) ? -xc : Xk[(xr + 1) * W + col];
                double xb = zlo ? -xc : Xm[xr * W + col];
                double xt = zhi ? -xc : Xp[xr * W + col];
                rnew = gs_update(xc, xw, xe, xs, xn, xb, xt, sel ? bi2.y : bi2.x,
                                 sel ? bie : bi2.y, sel ? bjl.y : bjl.x, sel ? bjh.y : bjh.x,
                                 sel ? bkl.y : bkl.x, sel ? bkh.y : bkh.x, sel ? al2.y : al2.x,
                                 sel ? dv2.y : dv2.x, sel ? rh2.y : rh2.x, a, bh2);
            }
            // black cell of this plane = the other one; keep its coefficients
            double nb[9] = {sel ? bi2.x : bi2.y, sel ? bi2.y : bie, sel ? bjl.x : bjl.y,
                            sel ? bjh.x : bjh.y, sel ? bkl.x : bkl.y, sel ? bkh.x : bkh.y,
                            sel ? al2.x : al2.y, sel ? dv2.x : dv2.y, sel ? rh2.x : rh2.y};

            // ------------------------------------------------ R(p): ring (9 per warp)
            int rt = w * 9 + lane;
            bool ring = kin && lane < 9 && rt < NRING;
            int rgx = 0, rgy = 0, rxr = 0, rcol = 0;
            if (ring) {
                if (rt < TX) {
                    int pp = rt % (TX / 2);
                    rgy = (rt < TX / 2) ? y0 - 1 : y0 + TY;
                    int s2 = (rgy + gk) & 1;
                    rgx = x0 + 2 * pp + s2;
                } else {
                    int m = rt - TX, side = m / (TY / 2);
                    m -= side * (TY / 2);
                    rgx = side ? x0 + TX : x0 - 1;
                    int gyp = y0 + 2 * m;
                    rgy = gyp + ((rgx + gyp + gk) & 1);
                }
                ring = rgx >= 0 && rgx < g.nx && rgy >= 0 && rgy < g.ny;
                rxr = rgy - y0 + 2;
                rcol = rgx - x0 + 2;
            }
            double ringnew = 0.0;
            if (ring) {
                const int rcr = rxr - 1;
                double xc = Xk[rxr * W + rcol];
                double xw = (rgx == 0) ? -xc : Xk[rxr * W + rcol - 1];
                double xe = (rgx == g.nx - 1) ? -xc : Xk[rxr * W + rcol + 1];
                double xs = (rgy == 0) ? -xc : Xk[(rxr - 1) * W + rcol];
                double xn = (rgy == g.ny - 1) ? -xc : Xk[(rxr + 1) * W + rcol];
                double xb = zlo ? -xc : Xm[rxr * W + rcol];
                double xt = zhi ? -xc : Xp[rxr * W + rcol];
                ringnew = gs_update(xc, xw, xe, xs, xn, xb, xt, C[CA_BI * CARR + rcr * W + rcol],
                                    C[CA_BI * CARR + rcr * W + rcol + 1],
                                    C[CA_BJ * CARR + rcr * W + rcol],
                                    C[CA_BJ * CARR + (rcr + 1) * W + rcol], Klo[rcr * W + rcol],
                                    Khi[rcr * W + rcol], C[CA_AL * CARR + rcr * W + rcol],
                                    C[CA_DV * CARR + rcr * W + rcol],
                                    C[CA_RH * CARR + rcr * W + rcol], a, bh2);
            }
            // R(p) reads only black cells of plane p (and planes p+-1 at
            // positions that are black there), so writing red cells now is safe.
            double* Xkw = Xs + md(p, NXS) * XSLOT;
            if (kin) Xkw[xr * W + c0 + sel] = rnew;
            if (ring) Xkw[rxr * W + rcol] = ringnew;
            fence_proxy_async();
            __syncthreads();

            // refill: bundle p+2 (its slots were last read by B(p-2), before this barrier)
            if (tid == 0 && p + 2 <= z1) issue(p + 2);

            // ------------------------------------------------ B(p-1): tile
            if (p - 1 >= z0) {
                const int gkm = gk - 1;
                const double* Xmm = Xs + md(p - 2, NXS) * XSLOT;
                const int bsel = 1 - ((gy + gkm) & 1);  // black cell of plane p-1
                double2 q2 = *(const double2*)&Xm[xr * W + c0];  // (red-new, black-old) pair
                double ql = __shfl_up_sync(0xffffffffu, q2.y, 1);
                double qr = __shfl_down_sync(0xffffffffu, q2.x, 1);
                if (lane == 0) ql = Xm[xr * W + 1];
                if (lane == 31) qr = Xm[xr * W + TX + 2];
                const int gx = gxa + bsel, col = c0 + bsel;
                double xc = bsel ? q2.y : q2.x;
                double xw = bsel ? q2.x : ql;
                double xe = bsel ? qr : q2.y;
                if (gx == 0) xw = -xc;
                if (gx == g.nx - 1) xe = -xc;
                double xs = (gy == 0) ? -xc : Xm[(xr - 1) * W + col];
                double xn = (gy == g.ny - 1) ? -xc : Xm[(xr + 1) * W + col];
                double xb = (gkm == 0) ? -xc : Xmm[xr * W + col];
                double xt = (gkm == g.gnz - 1) ? -xc : Xk[xr * W + col];
                double bnew = gs_update(xc, xw, xe, xs, xn, xb, xt, rb[0], rb[1], rb[2], rb[3],
                                        rb[4], rb[5], rb[6], rb[7], rb[8], a, bh2);
                double2 o = bsel ? make_double2(q2.x, bnew) : make_double2(bnew, q2.y);
                *(double2*)(xo + (long)(p - 1 + SF_GZ) * g.ks + (long)(gy + SF_GY) * g.js +
                            SF_OX + gxa) = o;
            }
#pragma unroll
            for (int i = 0; i < 9; i++) rb[i] = nb[i];
        }
        seq = seq0 + 2 + (z1 - z0) + 1;
        __syncthreads();  // all reads of this item's slots done before the next prologue
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
    CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)base, dims, strides, box, es,
                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return sf_fail(SF_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    return SF_OK;
}

int g_num_sms = 0;

}  // namespace

bool gsrb_fused_supported(const sf_level* L) {
    return L->nx % TX == 0 && L->ny % TY == 0 && L->lnz >= 1;
}

sf_status k_gsrb_pair_fused(sf_level* L, int xin, int xout, int rhs, double a, double b) {
    if (!gsrb_fused_supported(L)) return sf_fail(SF_ERR_SHAPE, "fused GSRB needs nx%%64==0, ny%%8==0");
    SF_TRY(get_encoder());
    static bool attr = false;
    if (!attr) {
        SF_CUDA(cudaFuncSetAttribute(gsrb_pair_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)SMEM));
        int dev;
        SF_CUDA(cudaGetDevice(&dev));
        SF_CUDA(cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev));
        attr = true;
    }
    const int ntx = L->nx / TX, nty = L->ny / TY, tiles = ntx * nty;
    // chunk depth: minimise rounds * (depth + prologue) over persistent CTAs
    const int G = g_num_sms;
    int best_d = L->lnz;
    double best = 1e30;
    for (int nch = 1; nch <= L->lnz; nch++) {
        int d = (L->lnz + nch - 1) / nch;
        if (d < 8 && nch > 1) break;
        int n = (L->lnz + d - 1) / d;
        long items = (long)tiles * n;
        double rounds = (double)((items + G - 1) / G);
        double cost = rounds * (d + 3.0);
        if (cost < best - 1e-9) { best = cost; best_d = d; }
    }
    const int depth = best_d, nch = (L->lnz + depth - 1) / depth;
    const int items = tiles * nch;
    const double bh2 = b / (L->h * L->h);
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        Maps mp;
        SF_TRY(encode(&mp.x, L, v.f[xin], XH));
        SF_TRY(encode(&mp.al, L, v.f[SF_ALPHA], CHH));
        SF_TRY(encode(&mp.dv, L, v.f[SF_DINV], CHH));
        SF_TRY(encode(&mp.rh, L, v.f[rhs], CHH));
        SF_TRY(encode(&mp.bi, L, v.f[SF_BETA_I], CHH));
        SF_TRY(encode(&mp.bj, L, v.f[SF_BETA_J], CHH));
        SF_TRY(encode(&mp.bk, L, v.f[SF_BETA_K], CHH));
        Geo g{v.nx, v.ny, v.nz, v.z0, v.gnz, v.js, v.ks};
        int grid = std::min(items, G);
        gsrb_pair_tma_kernel<<<grid, NT, SMEM, L->stream>>>(mp, g, v.f[xout], a, bh2, depth, ntx,
                                                            tiles, items);
        SF_LAUNCHED();
    }
    return sf_check_launch("gsrb_pair_tma");
}
