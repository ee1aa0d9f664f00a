// Bandwidth-shaped per-level kernels (sm_100a, fp64): each thread owns a PAIR
// of x-adjacent cells (16-byte loads/stores along the unit-stride axis) and
// streams a chunk of z-planes, so a block issues one atomic per launch-chunk
// instead of one per cell.  Rows A6 (+A10, +A7) and A8 of DESIGN.md.
//
//   residual_pair<WRITE, NORM>  res = rhs - A x; optionally
//                               writes res and/or reduces max|res| (A10, the
//                               convergence check of reading R-9) in the same
//                               pass (48 B/cell when only the norm is needed)
//   residual_restrict           coarse rhs = R_cell(rhs - A x) (A6 + A7 fused,
//                               49 B per fine cell): the V-cycle's residual
//                               never goes to HBM
//   interp_p0_pair              fine += P0(coarse) (A8, V-cycle)
//   norm_pair                   max|x| / sum x^2 of a field (A10)
//
// The operator is evaluated in exactly the term order of op_at (kernels.cu)
// and the oracle; the Dirichlet fold reads -x(c) across global faces.
#include <algorithm>
#include <cstdlib>

#include "sf_internal.h"

namespace {

constexpr int PX = 32, PY = 4;  // threads per block: 32 pairs (64 cells) x 4 rows

__device__ __forceinline__ double2 ld2(const double* p) { return *(const double2*)p; }

// A x at the pair (i, i+1) of row j, plane k; c = sf_ix(i, j, k), i even.
__device__ __forceinline__ void op_pair(const PV& v, const double* __restrict__ x, int i, int j,
                                        int gk, long c, double a, double bh2, double& axa,
                                        double& axb) {
    const double2 xc = ld2(x + c);
    double xw = (i == 0) ? -xc.x : x[c - 1];
    double xe = (i + 1 == v.nx - 1) ? -xc.y : x[c + 2];
    double2 xs = ld2(x + c - v.js), xn = ld2(x + c + v.js);
    double2 xb = ld2(x + c - v.ks), xt = ld2(x + c + v.ks);
    if (j == 0) xs = make_double2(-xc.x, -xc.y);
    if (j == v.ny - 1) xn = make_double2(-xc.x, -xc.y);
    if (gk == 0) xb = make_double2(-xc.x, -xc.y);
    if (gk == v.gnz - 1) xt = make_double2(-xc.x, -xc.y);
    const double2 bi = ld2(v.f[SF_BETA_I] + c);
    const double bie = v.f[SF_BETA_I][c + 2];
    const double2 bjs = ld2(v.f[SF_BETA_J] + c), bjn = ld2(v.f[SF_BETA_J] + c + v.js);
    const double2 bkb = ld2(v.f[SF_BETA_K] + c), bkt = ld2(v.f[SF_BETA_K] + c + v.ks);
    const double2 al = ld2(v.f[SF_ALPHA] + c);
    double fa = bi.y * (xc.y - xc.x);
    fa += bi.x * (xw - xc.x);
    fa += bjn.x * (xn.x - xc.x);
    fa += bjs.x * (xs.x - xc.x);
    fa += bkt.x * (xt.x - xc.x);
    fa += bkb.x * (xb.x - xc.x);
    double fb = bie * (xe - xc.y);
    fb += bi.y * (xc.x - xc.y);
    fb += bjn.y * (xn.y - xc.y);
    fb += bjs.y * (xs.y - xc.y);
    fb += bkt.y * (xt.y - xc.y);
    fb += bkb.y * (xb.y - xc.y);
    axa = a * al.x * xc.x - bh2 * fa;
    axb = a * al.y * xc.y - bh2 * fb;
}

__device__ __forceinline__ unsigned long long umax64(unsigned long long a, unsigned long long b) {
    return a > b ? a : b;
}

// block-wide max of non-negative doubles via their bit patterns (NaN wins)
__device__ __forceinline__ void block_max_atomic(unsigned long long m, double* out) {
    __shared__ unsigned long long red[PX * PY / 32];
    for (int o = 16; o > 0; o >>= 1) m = umax64(m, __shfl_xor_sync(0xffffffffu, m, o));
    const int t = threadIdx.y * PX + threadIdx.x;
    if ((t & 31) == 0) red[t >> 5] = m;
    __syncthreads();
    if (t == 0) {
        for (int wq = 1; wq < PX * PY / 32; wq++) m = umax64(m, red[wq]);
        atomicMax((unsigned long long*)out, m);
    }
}

__device__ __forceinline__ unsigned long long abits(double v) {
    return (unsigned long long)__double_as_longlong(fabs(v));
}

template <bool WRITE, bool NORM>
__global__ void __launch_bounds__(PX* PY) residual_pair_kernel(PV v, double* __restrict__ res,
                                                                const double* __restrict__ x,
                                                                const double* __restrict__ rhs,
                                                                double a, double bh2, int depth,
                                                                double* nout) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    unsigned long long m = 0ull;
    if (i < v.nx && j < v.ny) {
        for (int k = k0; k < k1; k++) {
            const long c = sf_ix(v, i, j, k);
            double axa, axb;
            op_pair(v, x, i, j, v.z0 + k, c, a, bh2, axa, axb);
            const double2 f = ld2(rhs + c);
            const double ra = f.x - axa, rb = f.y - axb;
            if (WRITE) *(double2*)(res + c) = make_double2(ra, rb);
            if (NORM) m = umax64(m, umax64(abits(ra), abits(rb)));
        }
    }
    if (NORM) block_max_atomic(m, nout);
}

// coarse(I,J,K) = 1/8 sum over the 8 children of (rhs - A x); thread per (I,J)
__global__ void __launch_bounds__(PX* PY) residual_restrict_kernel(PV f, const double* __restrict__ x,
                                                                    const double* __restrict__ rhs,
                                                                    double a, double bh2, PV c,
                                                                    double* __restrict__ cx,
                                                                    int zoff, int depth) { pdl_wait();
    const int I = blockIdx.x * PX + threadIdx.x, J = blockIdx.y * PY + threadIdx.y;
    const int K0 = blockIdx.z * depth, K1 = min(K0 + depth, f.nz / 2);
    if (2 * I >= f.nx || 2 * J >= f.ny) return;
    for (int K = K0; K < K1; K++) {
        double s = 0.0;
#pragma unroll
        for (int d = 0; d < 2; d++)
#pragma unroll
            for (int bb = 0; bb < 2; bb++) {
                const int j = 2 * J + bb, k = 2 * K + d;
                const long q = sf_ix(f, 2 * I, j, k);
                double axa, axb;
                op_pair(f, x, 2 * I, j, f.z0 + k, q, a, bh2, axa, axb);
                const double2 r = ld2(rhs + q);
                s += r.x - axa;
                s += r.y - axb;
            }
        cx[sf_ix(c, I, J, K + zoff)] = s / 8.0;
    }
}

// A x at the pair of row j from operands already in registers (op_pair's term
// order and roundings; xs/xn/xb/xt carry the row's y/z neighbours, BC folded by
// the caller's flags).
__device__ __forceinline__ void op_pair_r(const PV& v, const double* __restrict__ x, int i, long c,
                                          double2 xc, double2 xs, double2 xn, double2 xb,
                                          double2 xt, double2 bjs, double2 bjn, double2 bkb,
                                          double2 bkt, double a, double bh2, double& axa,
                                          double& axb) {
    const double xw = (i == 0) ? -xc.x : x[c - 1];
    const double xe = (i + 1 == v.nx - 1) ? -xc.y : x[c + 2];
    const double2 bi = ld2(v.f[SF_BETA_I] + c);
    const double bie = v.f[SF_BETA_I][c + 2];
    const double2 al = ld2(v.f[SF_ALPHA] + c);
    double fa = bi.y * (xc.y - xc.x);
    fa += bi.x * (xw - xc.x);
    fa += bjn.x * (xn.x - xc.x);
    fa += bjs.x * (xs.x - xc.x);
    fa += bkt.x * (xt.x - xc.x);
    fa += bkb.x * (xb.x - xc.x);
    double fb = bie * (xe - xc.y);
    fb += bi.y * (xc.x - xc.y);
    fb += bjn.y * (xn.y - xc.y);
    fb += bjs.y * (xs.y - xc.y);
    fb += bkt.y * (xt.y - xc.y);
    fb += bkb.y * (xb.y - xc.y);
    axa = a * al.x * xc.x - bh2 * fa;
    axb = a * al.y * xc.y - bh2 * fb;
}

__device__ __forceinline__ double2 neg2(double2 u) { return make_double2(-u.x, -u.y); }

// residual_restrict, persistent and z-streamed: items = (32x4 coarse columns
// tile, chunk of `depth` coarse planes), walked by an occupancy-sized grid; a
// thread keeps the x planes 2K-1 .. 2K+2 and beta_k planes 2K .. 2K+2 of its
// 2x2 fine columns in registers, so each coarse step loads two new x planes
// and two beta_k planes (42 loads per 8 fine cells instead of 60).  Same
// arithmetic, term order and roundings as residual_restrict_kernel.
template <int MINB>
__global__ void __launch_bounds__(PX* PY, MINB) residual_restrict_zs_kernel(
    PV f, const double* __restrict__ x, const double* __restrict__ rhs, double a, double bh2, PV c,
    double* __restrict__ cx, int zoff, int depth, int tgx, int ntiles, int nitems, int trig) { pdl_wait();
    // trig: the next launch (the coarse cluster V-cycle) may start now -- it
    // stages its constant coefficients while this kernel runs and waits for
    // this kernel's output (the coarse rhs) in griddepcontrol.wait
    if (trig) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int nK = f.nz / 2;
    const double* bj = f.f[SF_BETA_J];
    const double* bk = f.f[SF_BETA_K];
    for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int ch = item / ntiles, tile = item - ch * ntiles;
        const int I = (tile % tgx) * PX + threadIdx.x, J = (tile / tgx) * PY + threadIdx.y;
        if (2 * I >= f.nx || 2 * J >= f.ny) continue;
        const int K0 = ch * depth, K1 = min(K0 + depth, nK);
        const int i = 2 * I, j0 = 2 * J, j1 = j0 + 1;
        const long js = f.js, ks = f.ks;
        long q0 = sf_ix(f, i, j0, 2 * K0);   // row j0 of plane 2K
        // carried: x(2K-1), x(2K) and beta_k(2K) of rows j0, j1
        double2 xa0 = ld2(x + q0 - ks), xa1 = ld2(x + q0 - ks + js);
        double2 xb0 = ld2(x + q0), xb1 = ld2(x + q0 + js);
        double2 k00 = ld2(bk + q0), k01 = ld2(bk + q0 + js);
        for (int K = K0; K < K1; K++, q0 += 2 * ks) {
            const long q1 = q0 + ks;   // plane 2K+1
            const double2 xc0 = ld2(x + q1), xc1 = ld2(x + q1 + js);
            const double2 xd0 = ld2(x + q1 + ks), xd1 = ld2(x + q1 + ks + js);
            const double2 k10 = ld2(bk + q1), k11 = ld2(bk + q1 + js);
            const double2 k20 = ld2(bk + q1 + ks), k21 = ld2(bk + q1 + ks + js);
            double s = 0.0;
#pragma unroll
            for (int d = 0; d < 2; d++) {
                const long q = d ? q1 : q0;
                const int gk = f.z0 + 2 * K + d;
                const double2 c0 = d ? xc0 : xb0, c1 = d ? xc1 : xb1;
                double2 b0 = d ? xb0 : xa0, b1 = d ? xb1 : xa1;
                double2 t0 = d ? xd0 : xc0, t1 = d ? xd1 : xc1;
                const double2 kb0 = d ? k10 : k00, kb1 = d ? k11 : k01;
                const double2 kt0 = d ? k20 : k10, kt1 = d ? k21 : k11;
                if (gk == 0) { b0 = neg2(c0); b1 = neg2(c1); }
                if (gk == f.gnz - 1) { t0 = neg2(c0); t1 = neg2(c1); }
                double2 ys = ld2(x + q - js), yn = ld2(x + q + 2 * js);
                if (j0 == 0) ys = neg2(c0);
                if (j1 == f.ny - 1) yn = neg2(c1);
                const double2 bj0 = ld2(bj + q), bj1 = ld2(bj + q + js), bj2 = ld2(bj + q + 2 * js);
                double axa, axb;
                // row j0: north neighbour row j1 (an interior row: j0 + 1 < ny)
                op_pair_r(f, x, i, q, c0, ys, c1, b0, t0, bj0, bj1, kb0, kt0, a, bh2, axa, axb);
                double2 r = ld2(rhs + q);
                s += r.x - axa;
                s += r.y - axb;
                op_pair_r(f, x, i, q + js, c1, c0, yn, b1, t1, bj1, bj2, kb1, kt1, a, bh2, axa, axb);
                r = ld2(rhs + q + js);
                s += r.x - axa;
                s += r.y - axb;
            }
            cx[sf_ix(c, I, J, K + zoff)] = s / 8.0;
            xa0 = xc0; xa1 = xc1; xb0 = xd0; xb1 = xd1; k00 = k20; k01 = k21;
        }
    }
}

// fine pair (2I', 2I'+1) shares its coarse parent
__global__ void __launch_bounds__(PX* PY) interp_p0_pair_kernel(PV f, double* __restrict__ y, double s,
                                                                 PV c, const double* __restrict__ x,
                                                                 int zoff, int depth) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, f.nz);
    if (i >= f.nx || j >= f.ny) return;
    for (int k = k0; k < k1; k++) {
        const long q = sf_ix(f, i, j, k);
        const double p = x[sf_ix(c, i >> 1, j >> 1, (k >> 1) + zoff)];
        double2 u = ld2(y + q);
        if (s == 0.0) {
            u.x = p;
            u.y = p;
        } else {
            u.x = s * u.x + p;
            u.y = s * u.y + p;
        }
        *(double2*)(y + q) = u;
    }
}

__global__ void __launch_bounds__(PX* PY) norm_pair_kernel(PV v, const double* __restrict__ x,
                                                            int kind, int depth, double* out) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    unsigned long long m = 0ull;
    double acc = 0.0;
    if (i < v.nx && j < v.ny)
        for (int k = k0; k < k1; k++) {
            const double2 u = ld2(x + sf_ix(v, i, j, k));
            m = umax64(m, umax64(abits(u.x), abits(u.y)));
            acc += u.x * u.x;
            acc += u.y * u.y;
        }
    if (kind == SF_NORM_MAX) {
        block_max_atomic(m, out);
    } else {
        __shared__ double rs[PX * PY / 32];
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        const int t = threadIdx.y * PX + threadIdx.x;
        if ((t & 31) == 0) rs[t >> 5] = acc;
        __syncthreads();
        if (t == 0) {
            for (int wq = 1; wq < PX * PY / 32; wq++) acc += rs[wq];
            atomicAdd(out, acc);
        }
    }
}

// NEXT-2 (Fig 7): constant-coefficient 7-point Laplacian
// L x = h^-2 sum_n (x_c - x_n) (Dirichlet fold: a boundary neighbour is -x_c),
// and weighted Jacobi out = x + w D^-1 (f - L x), D^-1 = h^2 / (6 + boundary
// faces) computed on the fly.  Streams x only (Laplacian: 16 B/cell) or x, f
// (Jacobi: 24 B/cell); no coefficient arrays.
template <bool JACOBI>
__global__ void __launch_bounds__(PX* PY) cc_pair_kernel(PV v, double* __restrict__ out,
                                                          const double* __restrict__ x,
                                                          const double* __restrict__ f,
                                                          double hm2, double h2w, int depth) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    if (i >= v.nx || j >= v.ny) return;
    const double h2w6 = h2w / 6.0;
    // register streaming along z: the column's planes k-1, k, k+1 ride in registers
    long c = sf_ix(v, i, j, k0);
    double2 xb = ld2(x + c - v.ks), xc = ld2(x + c);
    for (int k = k0; k < k1; k++, c += v.ks) {
        const int gk = v.z0 + k;
        const double2 xtr = ld2(x + c + v.ks);
        double xw = (i == 0) ? -xc.x : x[c - 1];
        double xe = (i + 1 == v.nx - 1) ? -xc.y : x[c + 2];
        double2 xs = ld2(x + c - v.js), xn = ld2(x + c + v.js);
        double2 xbb = xb, xt = xtr;
        if (j == 0) xs = make_double2(-xc.x, -xc.y);
        if (j == v.ny - 1) xn = make_double2(-xc.x, -xc.y);
        if (gk == 0) xbb = make_double2(-xc.x, -xc.y);
        if (gk == v.gnz - 1) xt = make_double2(-xc.x, -xc.y);
        double sa = xc.x - xc.y;
        sa += xc.x - xw;
        sa += xc.x - xn.x;
        sa += xc.x - xs.x;
        sa += xc.x - xt.x;
        sa += xc.x - xbb.x;
        double sb = xc.y - xe;
        sb += xc.y - xc.x;
        sb += xc.y - xn.y;
        sb += xc.y - xs.y;
        sb += xc.y - xt.y;
        sb += xc.y - xbb.y;
        double2 o;
        if (JACOBI) {
            // D^-1 = h^2 / (6 + boundary faces): one shared factor for interior cells
            const int nyz = (j == 0) + (j == v.ny - 1) + (gk == 0) + (gk == v.gnz - 1);
            const int na = nyz + (i == 0), nb = nyz + (i + 1 == v.nx - 1);
            const double2 fv = ld2(f + c);
            const double wa = na ? h2w / (6.0 + na) : h2w6, wb = nb ? h2w / (6.0 + nb) : h2w6;
            o.x = xc.x + wa * (fv.x - hm2 * sa);
            o.y = xc.y + wb * (fv.y - hm2 * sb);
        } else {
            o.x = hm2 * sa;
            o.y = hm2 * sb;
        }
        __stcs((double2*)(out + c), o);
        xb = xc;
        xc = xtr;
    }
}

// NEXT-3 Chebyshev step (reading R-16): out = x + c1 (x - xp) + c2 Dinv (rhs - A x),
// A in op_at's term order.  72 B/cell (x, xp, rhs, alpha, beta x3, Dinv, out).
__global__ void __launch_bounds__(PX* PY) cheby_pair_kernel(PV v, double* __restrict__ out,
                                                             const double* __restrict__ x,
                                                             const double* __restrict__ xp,
                                                             const double* __restrict__ rhs,
                                                             double c1, double c2, double a,
                                                             double bh2, int depth) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    if (i >= v.nx || j >= v.ny) return;
    for (int k = k0; k < k1; k++) {
        const long c = sf_ix(v, i, j, k);
        double axa, axb;
        op_pair(v, x, i, j, v.z0 + k, c, a, bh2, axa, axb);
        const double2 f = ld2(rhs + c), xc = ld2(x + c), xq = ld2(xp + c),
                      dv = ld2(v.f[SF_DINV] + c);
        double2 o;
        o.x = xc.x + c1 * (xc.x - xq.x) + c2 * dv.x * (f.x - axa);
        o.y = xc.y + c1 * (xc.y - xq.y) + c2 * dv.y * (f.y - axb);
        *(double2*)(out + c) = o;
    }
}

// power-iteration helpers for lambda_max(D^-1 A): w *= Dinv with sum w^2 (atomic),
// and v = w * scale[0]
__global__ void __launch_bounds__(PX* PY) dinv_scale_pair_kernel(PV v, double* __restrict__ w,
                                                                  int depth, double* sumsq) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    double acc = 0.0;
    if (i < v.nx && j < v.ny)
        for (int k = k0; k < k1; k++) {
            const long c = sf_ix(v, i, j, k);
            double2 u = ld2(w + c);
            const double2 dv = ld2(v.f[SF_DINV] + c);
            u.x = dv.x * u.x;
            u.y = dv.y * u.y;
            *(double2*)(w + c) = u;
            acc += u.x * u.x;
            acc += u.y * u.y;
        }
    __shared__ double rs[PX * PY / 32];
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    const int t = threadIdx.y * PX + threadIdx.x;
    if ((t & 31) == 0) rs[t >> 5] = acc;
    __syncthreads();
    if (t == 0) {
        for (int wq = 1; wq < PX * PY / 32; wq++) acc += rs[wq];
        atomicAdd(sumsq, acc);
    }
}

// deterministic positive start vector for the power iteration (the oracle
// test builds the same formula independently):
// v(i,j,k) = 1 + ((7 gi + 13 gj + 29 gk) mod 17) / 17
__global__ void __launch_bounds__(PX* PY) start_vector_kernel(PV v, double* __restrict__ y,
                                                               int depth) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    if (i >= v.nx || j >= v.ny) return;
    for (int k = k0; k < k1; k++) {
        const long gk = v.z0 + k;
        double2 o;
        o.x = 1.0 + (double)((7L * i + 13L * j + 29L * gk) % 17) / 17.0;
        o.y = 1.0 + (double)((7L * (i + 1) + 13L * j + 29L * gk) % 17) / 17.0;
        *(double2*)(y + sf_ix(v, i, j, k)) = o;
    }
}

__global__ void __launch_bounds__(PX* PY) scale_pair_kernel(PV v, double* __restrict__ y,
                                                             const double* __restrict__ src,
                                                             const double* sumsq, int depth) { pdl_wait();
    const int i = 2 * (blockIdx.x * PX + threadIdx.x), j = blockIdx.y * PY + threadIdx.y;
    const int k0 = blockIdx.z * depth, k1 = min(k0 + depth, v.nz);
    if (i >= v.nx || j >= v.ny) return;
    const double sc = 1.0 / sqrt(*sumsq);
    for (int k = k0; k < k1; k++) {
        const long c = sf_ix(v, i, j, k);
        double2 u = ld2(src + c);
        u.x = u.x * sc;
        u.y = u.y * sc;
        *(double2*)(y + c) = u;
    }
}

__global__ void zero_scalar(double* p) { pdl_wait(); *p = 0.0; }

// grid over pairs: (ceil(nx/64), ceil(ny/4), z-chunks) with ~16 blocks per SM
inline dim3 pair_grid(int nx, int ny, int nz, int* depth, long per_sm = 16) {
    const int gx = (nx / 2 + PX - 1) / PX, gy = (ny + PY - 1) / PY;
    const long want = 148L * per_sm;
    int zc = (int)std::max(1L, std::min((long)nz, (want + (long)gx * gy - 1) / ((long)gx * gy)));
    *depth = (nz + zc - 1) / zc;
    zc = (nz + *depth - 1) / *depth;
    return dim3(gx, gy, zc);
}

// SF_RR_ZS = 0 selects the one-pass-per-launch residual_restrict (A/B runs)
int rr_zs() {
    static const int v = getenv("SF_RR_ZS") ? atoi(getenv("SF_RR_ZS")) : 1;
    return v;
}

// resident CTAs of the z-streamed residual_restrict on this device
int rr_zs_resident() {
    static int g = 0;
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (rr_zs() == 2)
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, residual_restrict_zs_kernel<6>, PX * PY, 0);
        else if (rr_zs() == 3)
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, residual_restrict_zs_kernel<8>, PX * PY, 0);
        else
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, residual_restrict_zs_kernel<4>, PX * PY, 0);
        g = sms * std::max(per, 1);
    }
    return g;
}

}  // namespace

bool pair_ok(const sf_level* L) { return L->nx % 2 == 0; }

sf_status k_residual_pair(sf_level* L, int res, int x, int rhs, double a, double b, double* nout) {
    const double bh2 = b / (L->h * L->h);
    SF_TRY(sf_halo(L, x, 1));
    if (nout) {
        sf_launch(zero_scalar, 1, 1, 0, L->stream, nout);
        SF_LAUNCHED();
    }
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        double* r = res >= 0 ? v.f[res] : nullptr;
        if (r && nout)
            sf_launch(residual_pair_kernel<true, true>, g, dim3(PX, PY), 0, L->stream, v, r, v.f[x], v.f[rhs], a, bh2, depth, nout);
        else if (r)
            sf_launch(residual_pair_kernel<true, false>, g, dim3(PX, PY), 0, L->stream, v, r, v.f[x], v.f[rhs], a, bh2, depth, nout);
        else
            sf_launch(residual_pair_kernel<false, true>, g, dim3(PX, PY), 0, L->stream, v, r, v.f[x], v.f[rhs], a, bh2, depth, nout);
        SF_LAUNCHED();
    }
    return sf_check_launch("residual_pair");
}

sf_status k_residual_restrict(sf_level* F, int x, int rhs, double a, double b, sf_level* C, int cf,
                              bool trigger_next) {
    const double bh2 = b / (F->h * F->h);
    const bool rep = C->nparts == 1 && F->nparts > 1;
    SF_TRY(sf_halo(F, x, 1));
    for (int p = 0; p < F->nlocal; p++) {
        PV f = sf_view(F, p);
        PV c = sf_view(C, rep ? 0 : p);
        if (rr_zs()) {
            // persistent z-streamed kernel: chunk depth D minimising rounds * (D + 1)
            // (one plane of prologue) over the resident CTAs
            const int tgx = (f.nx / 2 + PX - 1) / PX, tgy = (f.ny / 2 + PY - 1) / PY;
            const int tiles = tgx * tgy, nK = f.nz / 2, G = rr_zs_resident();
            int best_d = nK;
            double best = 1e30;
            for (int d = nK; d >= 1; d--) {
                const long items = (long)tiles * ((nK + d - 1) / d);
                const double cost = (double)((items + G - 1) / G) * (d + 1.0);
                if (cost < best - 1e-9) { best = cost; best_d = d; }
            }
            // test / tuning overrides: chunk depth (coarse planes) and grid size,
            // so small levels take the multi-plane, multi-item paths of 512^3
            if (const char* e = getenv("SF_RRZS_DEPTH"))
                if (atoi(e) > 0) best_d = std::min(nK, atoi(e));
            const int items = tiles * ((nK + best_d - 1) / best_d);
            int grid = std::min(items, G);
            if (const char* e = getenv("SF_RRZS_GRID"))
                if (atoi(e) > 0) grid = std::min(items, atoi(e));
#define SF_RRZS(MB)                                                                              \
    sf_launch(residual_restrict_zs_kernel<MB>, grid, dim3(PX, PY), 0, F->stream,                         \
        f, f.f[x], f.f[rhs], a, bh2, c, c.f[cf], rep ? f.z0 / 2 : 0, best_d, tgx, tiles, items, \
        trigger_next && !rep ? 1 : 0)
            if (rr_zs() == 2) SF_RRZS(6);
            else if (rr_zs() == 3) SF_RRZS(8);
            else SF_RRZS(4);
#undef SF_RRZS
        } else {
            int depth;
            dim3 g = pair_grid(f.nx, f.ny / 2, f.nz / 2, &depth);  // thread per coarse (I,J)
            sf_launch(residual_restrict_kernel, g, dim3(PX, PY), 0, F->stream, f, f.f[x], f.f[rhs], a, bh2,
                                                                        c, c.f[cf],
                                                                        rep ? f.z0 / 2 : 0, depth);
        }
        SF_LAUNCHED();
    }
    SF_TRY(sf_check_launch("residual_restrict"));
    if (rep) SF_TRY(sf_agglomerate(C, cf, F->nparts, F->lnz / 2));
    return SF_OK;
}

sf_status k_interp_p0_pair(sf_level* F, int ff, double s, sf_level* C, int cf) {
    const bool rep = C->nparts == 1 && F->nparts > 1;
    for (int p = 0; p < F->nlocal; p++) {
        PV f = sf_view(F, p);
        PV c = sf_view(C, rep ? 0 : p);
        int depth;
        dim3 g = pair_grid(f.nx, f.ny, f.nz, &depth);
        sf_launch(interp_p0_pair_kernel, g, dim3(PX, PY), 0, F->stream, f, f.f[ff], s, c, c.f[cf],
                                                                 rep ? f.z0 / 2 : 0, depth);
        SF_LAUNCHED();
    }
    return sf_check_launch("interp_p0_pair");
}

sf_status k_cc(sf_level* L, int out, int x, int f, double omega, bool jacobi) {
    if (!pair_ok(L)) return sf_fail(SF_ERR_SHAPE, "CC kernels need an even nx");
    SF_TRY(sf_halo(L, x, 1));
    const double hm2 = 1.0 / (L->h * L->h), h2w = omega * L->h * L->h;
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        // shallower z runs per thread (64 blocks per SM of work): 256^3 Laplacian
        // 0.0555 -> 0.0502 ms, 512^3 0.388 -> 0.372 ms (profiles/r02/ab_cc_per_sm.txt)
        static const long per_sm = getenv("SF_CC_PER_SM") ? atol(getenv("SF_CC_PER_SM")) : 64;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth, per_sm);
        if (jacobi)
            sf_launch(cc_pair_kernel<true>, g, dim3(PX, PY), 0, L->stream, v, v.f[out], v.f[x], v.f[f], hm2,
                                                                     h2w, depth);
        else
            sf_launch(cc_pair_kernel<false>, g, dim3(PX, PY), 0, L->stream, v, v.f[out], v.f[x], nullptr,
                                                                      hm2, h2w, depth);
        SF_LAUNCHED();
    }
    return sf_check_launch("cc_pair");
}

sf_status k_cheby_step(sf_level* L, int out, int x, int xp, int rhs, double c1, double c2, double a,
                       double b) {
    if (!pair_ok(L)) return sf_fail(SF_ERR_SHAPE, "Chebyshev smoother needs an even nx");
    SF_TRY(sf_halo(L, x, 1));
    const double bh2 = b / (L->h * L->h);
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        sf_launch(cheby_pair_kernel, g, dim3(PX, PY), 0, L->stream, v, v.f[out], v.f[x], v.f[xp], v.f[rhs],
                                                             c1, c2, a, bh2, depth);
        SF_LAUNCHED();
    }
    return sf_check_launch("cheby_pair");
}

sf_status k_start_vector(sf_level* L, int field) {
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        sf_launch(start_vector_kernel, g, dim3(PX, PY), 0, L->stream, v, v.f[field], depth);
        SF_LAUNCHED();
    }
    return sf_check_launch("start_vector");
}

// one power-iteration step: w = Dinv (A v) (into `w`), ||w||^2 -> *sumsq, v = w / ||w||
sf_status k_power_step(sf_level* L, int v_id, int w_id, double a, double b, double* sumsq) {
    if (!pair_ok(L)) return sf_fail(SF_ERR_SHAPE, "power iteration needs an even nx");
    SF_TRY(k_apply_op(L, w_id, v_id, a, b));
    sf_launch(zero_scalar, 1, 1, 0, L->stream, sumsq);
    SF_LAUNCHED();
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        sf_launch(dinv_scale_pair_kernel, g, dim3(PX, PY), 0, L->stream, v, v.f[w_id], depth, sumsq);
        SF_LAUNCHED();
    }
    if (L->comm && L->comm->kind != 0 && L->nparts > 1)
        SF_TRY(sf_allreduce_scalar(L, L->comm, sumsq, 1));
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        sf_launch(scale_pair_kernel, g, dim3(PX, PY), 0, L->stream, v, v.f[v_id], v.f[w_id], sumsq, depth);
        SF_LAUNCHED();
    }
    return sf_check_launch("power_step");
}

sf_status k_norm_pair(sf_level* L, int field, int kind, double* dst) {
    sf_launch(zero_scalar, 1, 1, 0, L->stream, dst);
    SF_LAUNCHED();
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        int depth;
        dim3 g = pair_grid(v.nx, v.ny, v.nz, &depth);
        sf_launch(norm_pair_kernel, g, dim3(PX, PY), 0, L->stream, v, v.f[field], kind, depth, dst);
        SF_LAUNCHED();
    }
    return sf_check_launch("norm_pair");
}
