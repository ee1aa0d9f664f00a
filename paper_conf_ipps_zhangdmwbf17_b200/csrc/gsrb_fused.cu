// Colour-fused Gauss-Seidel red-black pair (A5) for sm_100a, fp64.
//
// One kernel pass performs a whole RB pair -- [BC, red, BC, black] of
// PAPER.md:641-644 with x += lambda*(rhs - Ax) (Fig 4) --
// so the 64 B/cell compulsory traffic of PAPER.md:669-672 is paid once per
// pair instead of once per colour sweep.  This is the B200 analogue of the
// paper's "multicolor reordering" + "tall-skinny blocking":
// 2-D (x,y) tiles streamed along z, with a wavefront that runs the red update
// of plane k and the black update of plane k-1 in the same step.
//
//   step k:  R(k)   red cells of plane k on the tile AND a one-cell ring
//                   around it (redundant: the ring belongs to the neighbouring
//                   tiles, recomputed here bit-identically so the black update
//                   never needs another CTA's result);
//            B(k-1) black cells of plane k-1 on the tile, reading red-new
//                   values of planes k-2, k-1 (incl. ring) and k.
//
// Out of place (xin -> xout): a CTA's 2-ring reads of xin must see OLD values
// whatever its neighbours have already written, so the pair writes a second
// buffer and the level swaps U <-> TMP afterwards.
//
// Data movement: x planes (tile + 2-ring) are staged in shared memory with
// 16-byte cp.async (LDGSTS, L1-bypassing), prefetched 1 plane ahead in a
// 5-plane ring; the tile's coefficients (alpha, Dinv, rhs, beta_i/j/k) are
// streamed into registers one plane ahead with 16-byte loads (each thread owns
// one red/black cell pair of a row); ring coefficients are L2 hits from the
// neighbouring tiles, which run concurrently at the same z (grid order).
//
// Dirichlet BC is folded in: a neighbour across a global face reads -x(c)
// (PAPER.md:336-341).  Part (slab) interfaces read exchanged halo planes:
// x needs depth 2 (R of plane -1 reads plane -2), coefficients depth 1-2.
#include "sf_internal.h"

namespace {

constexpr int TX = 64;           // tile width (cells) = one warp x 2 cells
constexpr int TY = 8;            // tile height = warps per CTA
constexpr int NT = 32 * TY;      // 256 threads
constexpr int XW = TX + 4;       // smem row: gx in [x0-2, x0+TX+2)
constexpr int XH = TY + 4;       // smem rows: gy in [y0-2, y0+TY+2)
constexpr int NXS = 5;           // x plane slots (k-2 .. k+2)
constexpr int NRING = TX + TX + TY / 2 + TY / 2;  // red ring cells per plane (72)

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::); }

__device__ __forceinline__ double2 ld2(const double* p) { return __ldg((const double2*)p); }

__device__ __forceinline__ int slot(int k) { return (k + 10) % NXS; }

struct Coef {           // one thread's cell pair (a = even x, b = odd x) of one plane
    double2 al, dv, rh, bi, bj, bjn, bkn;  // bkn = beta_k(k+1) (top faces)
    double bie;                            // beta_i(x_a + 2) (east face of b)
};

__device__ __forceinline__ Coef load_coef(const PV& v, const double* __restrict__ rhs, long c) {
    Coef q;
    q.al = ld2(v.f[SF_ALPHA] + c);
    q.dv = ld2(v.f[SF_DINV] + c);
    q.rh = ld2(rhs + c);
    q.bi = ld2(v.f[SF_BETA_I] + c);
    q.bie = __ldg(v.f[SF_BETA_I] + c + 2);
    q.bj = ld2(v.f[SF_BETA_J] + c);
    q.bjn = ld2(v.f[SF_BETA_J] + c + v.js);
    q.bkn = ld2(v.f[SF_BETA_K] + c + v.ks);
    return q;
}

// x <- x + Dinv (rhs - Ax), operator in the same term order as op_at in
// kernels.cu (A3).
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

__global__ void __launch_bounds__(NT, 2)
gsrb_pair_kernel(PV v, const double* __restrict__ xi, double* __restrict__ xo,
                 const double* __restrict__ rhs, double a, double bh2, int depth, int ntx) {
    __shared__ __align__(16) double X[NXS][XH][XW];

    const int tile = blockIdx.x;
    const int x0 = (tile % ntx) * TX, y0 = (tile / ntx) * TY;
    const int z0 = blockIdx.y * depth;
    const int z1 = min(z0 + depth, v.nz);
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gy = y0 + w, gxa = x0 + 2 * lane;
    const int row = w + 2, cola = 2 * lane + 2;
    const long js = v.js, ks = v.ks;
    const long cbase = (long)(gy + SF_GY) * js + SF_OX + gxa;  // + (k+GZ)*ks
    const double* xsrc = xi + (long)(y0 - 2 + SF_GY) * js + SF_OX + x0 - 2;

    auto issue_x = [&](int k) {
        double* dst = &X[slot(k)][0][0];
        const double* src = xsrc + (long)(k + SF_GZ) * ks;
        for (int t = threadIdx.x; t < XH * (XW / 2); t += NT) {
            int r = t / (XW / 2), c2 = t - r * (XW / 2);
            cp_async16(dst + r * XW + 2 * c2, src + r * js + 2 * c2);
        }
    };

    // prologue: x planes z0-2 .. z0 ; coefficients of plane z0-1
    issue_x(z0 - 2);
    issue_x(z0 - 1);
    issue_x(z0);
    cp_async_commit();
    Coef cur = load_coef(v, rhs, cbase + (long)(z0 - 1 + SF_GZ) * ks);
    double2 bklo = ld2(v.f[SF_BETA_K] + cbase + (long)(z0 - 1 + SF_GZ) * ks);
    Coef prev = cur;
    double2 bklo_prev = bklo;
    double rnew_prev = 0.0;  // this thread's red value of plane k-1

    for (int k = z0 - 1; k <= z1; k++) {
        const int gk = v.z0 + k;
        Coef nxt = cur;
        if (k + 1 <= z1) nxt = load_coef(v, rhs, cbase + (long)(k + 1 + SF_GZ) * ks);

        cp_async_wait_all();
        __syncthreads();  // x(k+1) landed; B(k-2) of the previous step is done
        if (k + 2 <= z1 + 1) issue_x(k + 2);
        cp_async_commit();

        double (*Xk)[XW] = X[slot(k)];
        double (*Xm)[XW] = X[slot(k - 1)];
        double (*Xp)[XW] = X[slot(k + 1)];
        const bool kin = (gk >= 0 && gk < v.gnz);
        const bool zlo = (gk == 0), zhi = (gk == v.gnz - 1);

        // ---------------------------------------------------- R(k): tile
        double rnew = 0.0;
        if (kin) {
            const int sel = (gxa + gy + gk) & 1;  // 0: cell a is red
            const int gx = gxa + sel, col = cola + sel;
            double xc = Xk[row][col];
            double xw = (gx == 0) ? -xc : Xk[row][col - 1];
            double xe = (gx == v.nx - 1) ? -xc : Xk[row][col + 1];
            double xs = (gy == 0) ? -xc : Xk[row - 1][col];
            double xn = (gy == v.ny - 1) ? -xc : Xk[row + 1][col];
            double xb = zlo ? -xc : Xm[row][col];
            double xt = zhi ? -xc : Xp[row][col];
            rnew = gs_update(xc, xw, xe, xs, xn, xb, xt, sel ? cur.bi.y : cur.bi.x,
                             sel ? cur.bie : cur.bi.y, sel ? cur.bj.y : cur.bj.x,
                             sel ? cur.bjn.y : cur.bjn.x, sel ? bklo.y : bklo.x,
                             sel ? cur.bkn.y : cur.bkn.x, sel ? cur.al.y : cur.al.x,
                             sel ? cur.dv.y : cur.dv.x, sel ? cur.rh.y : cur.rh.x, a, bh2);
        }
        // ---------------------------------------------------- R(k): ring
        int rrow = -1, rcol = -1, rgx = -1, rgy = -1;
        if (kin && threadIdx.x < NRING) {
            int t = threadIdx.x;
            if (t < TX) {                      // rows y0-1 and y0+TY
                int p = t % (TX / 2);
                rgy = (t < TX / 2) ? y0 - 1 : y0 + TY;
                int gxp = x0 + 2 * p;
                int s = (gxp + rgy + gk) & 1;
                rgx = gxp + s;
                rrow = rgy - y0 + 2;
                rcol = 2 * p + 2 + s;
            } else {                           // columns x0-1 and x0+TX
                int m = t - TX;
                int side = m / (TY / 2);
                m -= side * (TY / 2);
                rgx = side ? x0 + TX : x0 - 1;
                int gyp = y0 + 2 * m;
                int s = (rgx + gyp + gk) & 1;
                rgy = gyp + s;
                rrow = rgy - y0 + 2;
                rcol = rgx - x0 + 2;
            }
            if (rgx < 0 || rgx >= v.nx || rgy < 0 || rgy >= v.ny) rrow = -1;
        }
        double ringnew = 0.0;
        if (rrow >= 0) {
            long q = (long)(k + SF_GZ) * ks + (long)(rgy + SF_GY) * js + SF_OX + rgx;
            const double* bi = v.f[SF_BETA_I];
            const double* bj = v.f[SF_BETA_J];
            const double* bk = v.f[SF_BETA_K];
            double xc = Xk[rrow][rcol];
            double xw = (rgx == 0) ? -xc : Xk[rrow][rcol - 1];
            double xe = (rgx == v.nx - 1) ? -xc : Xk[rrow][rcol + 1];
            double xs = (rgy == 0) ? -xc : Xk[rrow - 1][rcol];
            double xn = (rgy == v.ny - 1) ? -xc : Xk[rrow + 1][rcol];
            double xb = zlo ? -xc : Xm[rrow][rcol];
            double xt = zhi ? -xc : Xp[rrow][rcol];
            ringnew = gs_update(xc, xw, xe, xs, xn, xb, xt, __ldg(bi + q), __ldg(bi + q + 1),
                                __ldg(bj + q), __ldg(bj + q + js), __ldg(bk + q),
                                __ldg(bk + q + ks), __ldg(v.f[SF_ALPHA] + q),
                                __ldg(v.f[SF_DINV] + q), __ldg(rhs + q), a, bh2);
        }
        // all reads of plane k (old black/red) are done before any red write?
        // Red writes touch only red cells; R(k) reads only black cells of
        // plane k and planes k+-1 -> no intra-step hazard.
        if (kin) Xk[row][cola + ((gxa + gy + gk) & 1)] = rnew;
        if (rrow >= 0) Xk[rrow][rcol] = ringnew;
        __syncthreads();

        // ---------------------------------------------------- B(k-1): tile
        if (k - 1 >= z0) {
            const int gkm = gk - 1;
            double (*Xmm)[XW] = X[slot(k - 2)];
            const int sel = 1 - ((gxa + gy + gkm) & 1);  // black cell of the pair
            const int gx = gxa + sel, col = cola + sel;
            double xc = Xm[row][col];
            double xw = (gx == 0) ? -xc : Xm[row][col - 1];
            double xe = (gx == v.nx - 1) ? -xc : Xm[row][col + 1];
            double xs = (gy == 0) ? -xc : Xm[row - 1][col];
            double xn = (gy == v.ny - 1) ? -xc : Xm[row + 1][col];
            double xb = (gkm == 0) ? -xc : Xmm[row][col];
            double xt = (gkm == v.gnz - 1) ? -xc : Xk[row][col];
            double bnew = gs_update(xc, xw, xe, xs, xn, xb, xt, sel ? prev.bi.y : prev.bi.x,
                                    sel ? prev.bie : prev.bi.y, sel ? prev.bj.y : prev.bj.x,
                                    sel ? prev.bjn.y : prev.bjn.x,
                                    sel ? bklo_prev.y : bklo_prev.x,
                                    sel ? prev.bkn.y : prev.bkn.x, sel ? prev.al.y : prev.al.x,
                                    sel ? prev.dv.y : prev.dv.x, sel ? prev.rh.y : prev.rh.x, a,
                                    bh2);
            double2 o = sel ? make_double2(rnew_prev, bnew) : make_double2(bnew, rnew_prev);
            *(double2*)(xo + cbase + (long)(k - 1 + SF_GZ) * ks) = o;
        }
        prev = cur;
        bklo_prev = bklo;
        bklo = cur.bkn;
        cur = nxt;
        rnew_prev = rnew;
    }
    cp_async_wait_all();
}

}  // namespace

bool gsrb_fused_supported(const sf_level* L) {
    return L->nx % TX == 0 && L->ny % TY == 0 && L->lnz >= 1;
}

sf_status k_gsrb_pair_fused(sf_level* L, int xin, int xout, int rhs, double a, double b) {
    if (!gsrb_fused_supported(L)) return sf_fail(SF_ERR_SHAPE, "fused GSRB needs nx%%64==0, ny%%8==0");
    const int ntx = L->nx / TX, nty = L->ny / TY;
    const int tiles = ntx * nty;
    // z-chunks: enough CTAs for ~4 resident waves (2 CTAs/SM x 148 SMs), but
    // chunks of >= 16 planes so the redundant prologue stays small.
    int want = (4 * 296 + tiles - 1) / tiles;
    int maxc = std::max(1, L->lnz / 16);
    int nch = std::max(1, std::min(want, maxc));
    int depth = (L->lnz + nch - 1) / nch;
    nch = (L->lnz + depth - 1) / depth;
    const double bh2 = b / (L->h * L->h);
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        gsrb_pair_kernel<<<dim3(tiles, nch), NT, 0, L->stream>>>(v, v.f[xin], v.f[xout], v.f[rhs],
                                                                 a, bh2, depth, ntx);
        SF_LAUNCHED();
    }
    return sf_check_launch("gsrb_pair_fused");
}
