// Per-cell stencil kernels of the HPGMG-FV hot path (sm_100a, fp64, CUDA cores).
//
// These are the straightforward, one-thread-per-cell forms of rows A2-A8 and
// A10 of DESIGN.md.  They run every level of the hierarchy; the finest-level
// smoother additionally has a colour-fused z-streaming kernel
// (gsrb_fused.cu).  HBM-bound: no tensor cores (not a contraction).
//
// The Dirichlet condition (ghost = -inside) is folded into
// every stencil: a neighbour across a global boundary face reads -x(c).  Slab
// halos (z ghost planes at part interfaces) are read from memory.
#include <cfloat>
#include <cmath>

#include <algorithm>

#include "sf_internal.h"

namespace {

constexpr int BX = 32, BY = 4;

inline dim3 cell_grid(const PV& v) {
    return dim3((v.nx + BX - 1) / BX, (v.ny + BY - 1) / BY, v.nz);
}

#include "cell_ops.cuh"

__global__ void __launch_bounds__(BX* BY) apply_op_kernel(PV v, double* __restrict__ out,
                                                           const double* __restrict__ x, double a,
                                                           double bh2) { pdl_wait();
    int i = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    if (i >= v.nx || j >= v.ny) return;
    out[sf_ix(v, i, j, k)] = op_at(v, x, i, j, k, a, bh2);
}

__global__ void __launch_bounds__(BX* BY) residual_kernel(PV v, double* __restrict__ res,
                                                           const double* __restrict__ x,
                                                           const double* __restrict__ rhs,
                                                           double a, double bh2) { pdl_wait();
    int i = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    if (i >= v.nx || j >= v.ny) return;
    long c = sf_ix(v, i, j, k);
    res[c] = rhs[c] - op_at(v, x, i, j, k, a, bh2);
}

// One colour sweep of A5: x(c) += Dinv(c) * (rhs(c) - Ax(c)) on cells with
// (gi+gj+gk) % 2 == colour (reading R-2).  One thread per cell of the colour.
__global__ void __launch_bounds__(BX* BY) gsrb_colour_kernel(PV v, double* __restrict__ x,
                                                              const double* __restrict__ rhs,
                                                              double a, double bh2, int colour) { pdl_wait();
    int t = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    int i = 2 * t + ((j + v.z0 + k + colour) & 1);
    if (i >= v.nx || j >= v.ny) return;
    long c = sf_ix(v, i, j, k);
    double ax = op_at(v, x, i, j, k, a, bh2);
    x[c] = x[c] + v.f[SF_DINV][c] * (rhs[c] - ax);
}

// A4: exact inverse diagonal with the Dirichlet fold.
__global__ void __launch_bounds__(BX* BY) dinv_kernel(PV v, double a, double bh2) { pdl_wait();
    int i = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    if (i >= v.nx || j >= v.ny) return;
    long c = sf_ix(v, i, j, k);
    int gk = v.z0 + k;
    const double* bi = v.f[SF_BETA_I];
    const double* bj = v.f[SF_BETA_J];
    const double* bk = v.f[SF_BETA_K];
    double s = bi[c] * (i == 0 ? 2.0 : 1.0);
    s += bi[c + 1] * (i == v.nx - 1 ? 2.0 : 1.0);
    s += bj[c] * (j == 0 ? 2.0 : 1.0);
    s += bj[c + v.js] * (j == v.ny - 1 ? 2.0 : 1.0);
    s += bk[c] * (gk == 0 ? 2.0 : 1.0);
    s += bk[c + v.ks] * (gk == v.gnz - 1 ? 2.0 : 1.0);
    v.f[SF_DINV][c] = 1.0 / (a * v.f[SF_ALPHA][c] + bh2 * s);
}

// A2: ghost fill over the one-cell shell [-1,nx] x [-1,ny] x [-1,nz].  Axes
// where the cell is outside a GLOBAL boundary are reflected (odd reflection,
// sign (-1)^m); z ghost planes at part interfaces are halos and are left as
// exchanged (their x/y ghosts are still reflected).
__global__ void bc_kernel(PV v, double* __restrict__ x) { pdl_wait();
    int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
    int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
    int k = blockIdx.z - 1;
    if (i > v.nx || j > v.ny) return;
    bool ox = (i < 0 || i >= v.nx), oy = (j < 0 || j >= v.ny);
    int gk = v.z0 + k;
    bool oz = (gk < 0 || gk >= v.gnz);
    if (!(ox || oy || oz)) return;
    int mi = i < 0 ? 0 : (i >= v.nx ? v.nx - 1 : i);
    int mj = j < 0 ? 0 : (j >= v.ny ? v.ny - 1 : j);
    int mk = k;
    if (gk < 0) mk = -v.z0;
    if (gk >= v.gnz) mk = v.gnz - 1 - v.z0;
    int m = (int)ox + (int)oy + (int)oz;
    double val = x[sf_ix(v, mi, mj, mk)];
    x[sf_ix(v, i, j, k)] = (m & 1) ? -val : val;
}

// A7 cell: coarse(I,J,K) = 1/8 sum of the 8 children.  c/f share part index
// (fine planes [2*zc0, ...)); zoff = plane offset of this fine part inside a
// replicated coarse part (agglomeration), else 0.
__global__ void __launch_bounds__(BX* BY) restrict_cell_kernel(PV c, double* __restrict__ cx,
                                                                PV f, const double* __restrict__ x,
                                                                int zoff) { pdl_wait();
    int I = blockIdx.x * BX + threadIdx.x, J = blockIdx.y * BY + threadIdx.y, K = blockIdx.z;
    if (I >= f.nx / 2 || J >= f.ny / 2) return;
    double s = 0.0;
#pragma unroll
    for (int d = 0; d < 2; d++)
#pragma unroll
        for (int bb = 0; bb < 2; bb++)
#pragma unroll
            for (int aa = 0; aa < 2; aa++) s += x[sf_ix(f, 2 * I + aa, 2 * J + bb, 2 * K + d)];
    cx[sf_ix(c, I, J, K + zoff)] = s / 8.0;
}

// A7 face (dir 0/1/2 = beta_i/j/k): average of the 4 fine faces covering the
// coarse face.  Face index along dir runs to n (inclusive).
__global__ void restrict_face_kernel(PV c, double* __restrict__ cx, PV f,
                                     const double* __restrict__ x, int dir, int zoff, int ncz) { pdl_wait();
    int I = blockIdx.x * blockDim.x + threadIdx.x, J = blockIdx.y * blockDim.y + threadIdx.y;
    int K = blockIdx.z;
    int ncx = f.nx / 2 + (dir == 0), ncy = f.ny / 2 + (dir == 1);
    if (I >= ncx || J >= ncy || K >= ncz) return;
    double s = 0.0;
#pragma unroll
    for (int p = 0; p < 2; p++)
#pragma unroll
        for (int q = 0; q < 2; q++) {
            int i = 2 * I, j = 2 * J, k = 2 * K;
            if (dir == 0) { j += p; k += q; }
            if (dir == 1) { i += p; k += q; }
            if (dir == 2) { i += p; j += q; }
            s += x[sf_ix(f, i, j, k)];
        }
    cx[sf_ix(c, I, J, K + zoff)] = s / 4.0;
}

// A8 P0: fine = s*fine + coarse(parent).  zoff: the fine part's first coarse
// plane inside the coarse part (replicated coarse levels), else 0.
__global__ void __launch_bounds__(BX* BY) interp_p0_kernel(PV f, double* __restrict__ y, double s,
                                                            PV c, const double* __restrict__ x,
                                                            int zoff) { pdl_wait();
    int i = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    if (i >= f.nx || j >= f.ny) return;
    long q = sf_ix(f, i, j, k);
    double p = x[sf_ix(c, i >> 1, j >> 1, (k >> 1) + zoff)];
    y[q] = (s == 0.0) ? p : s * y[q] + p;
}

// A8 PL: trilinear on cell centres; weights 27/64, 9/64, 3/64, 1/64 (products
// of the 1-D 3/4, 1/4).  Coarse ghosts (faces, edges, corners; halos) must be
// valid.  Summation order matches the oracle (children in x, y, z order).
__global__ void __launch_bounds__(BX* BY) interp_pl_kernel(PV f, double* __restrict__ y, double s,
                                                            PV c, const double* __restrict__ x,
                                                            int zoff) { pdl_wait();
    int i = blockIdx.x * BX + threadIdx.x, j = blockIdx.y * BY + threadIdx.y, k = blockIdx.z;
    if (i >= f.nx || j >= f.ny) return;
    int gkf = f.z0 + k;                    // global fine plane -> parity of the child
    int I = i >> 1, J = j >> 1, K = (k >> 1) + zoff;
    int di = (i & 1) ? 1 : -1, dj = (j & 1) ? 1 : -1, dk = (gkf & 1) ? 1 : -1;
    double p = 0.0;
#pragma unroll
    for (int cc = 0; cc < 2; cc++)
#pragma unroll
        for (int bb = 0; bb < 2; bb++)
#pragma unroll
            for (int aa = 0; aa < 2; aa++) {
                double w = (aa ? 0.25 : 0.75) * (bb ? 0.25 : 0.75) * (cc ? 0.25 : 0.75);
                p += w * x[sf_ix(c, I + aa * di, J + bb * dj, K + cc * dk)];
            }
    long q = sf_ix(f, i, j, k);
    y[q] = (s == 0.0) ? p : s * y[q] + p;
}

// A8 PL, one thread per coarse cell: its 8 children from the 3x3x3 coarse
// neighbourhood (27 loads for 8 cells instead of 8 per cell), stored as x
// pairs.  Each child's sum is the same ordered FMA chain as interp_pl_kernel.
__global__ void __launch_bounds__(BX* BY) interp_pl_block_kernel(PV f, double* __restrict__ y, double s,
                                                                  PV c, const double* __restrict__ x,
                                                                  int zoff) { pdl_wait();
    const int I = blockIdx.x * BX + threadIdx.x, J = blockIdx.y * BY + threadIdx.y, Kl = blockIdx.z;
    if (2 * I >= f.nx || 2 * J >= f.ny) return;
    const int K = Kl + zoff;
    double v[3][3][3];
#pragma unroll
    for (int dz = 0; dz < 3; dz++)
#pragma unroll
        for (int dy = 0; dy < 3; dy++)
#pragma unroll
            for (int dx = 0; dx < 3; dx++) v[dz][dy][dx] = x[sf_ix(c, I + dx - 1, J + dy - 1, K + dz - 1)];
#pragma unroll
    for (int c3 = 0; c3 < 2; c3++) {
        const int k = 2 * Kl + c3;
        const int dk = ((f.z0 + k) & 1) ? 1 : -1;
#pragma unroll
        for (int b3 = 0; b3 < 2; b3++) {
            const int j = 2 * J + b3, dj = b3 ? 1 : -1;
            double pr[2];
#pragma unroll
            for (int a3 = 0; a3 < 2; a3++) {
                const int di = a3 ? 1 : -1;
                double p = 0.0;
#pragma unroll
                for (int cc = 0; cc < 2; cc++)
#pragma unroll
                    for (int bb = 0; bb < 2; bb++)
#pragma unroll
                        for (int aa = 0; aa < 2; aa++) {
                            const double w = (aa ? 0.25 : 0.75) * (bb ? 0.25 : 0.75) * (cc ? 0.25 : 0.75);
                            p = __fma_rn(w, v[1 + cc * dk][1 + bb * dj][1 + aa * di], p);
                        }
                pr[a3] = p;
            }
            double2* q = (double2*)(y + sf_ix(f, 2 * I, j, k));
            if (s == 0.0) {
                *q = make_double2(pr[0], pr[1]);
            } else {
                const double2 o = *q;
                *q = make_double2(__fma_rn(s, o.x, pr[0]), __fma_rn(s, o.y, pr[1]));
            }
        }
    }
}

// A10: max |x| or sum x^2.  The max is reduced on the bit patterns of |x|:
// for non-negative doubles the unsigned order of the bits is the numeric
// order, and a (positive) NaN compares above +Inf, so NaN propagates.
__global__ void __launch_bounds__(256) norm_kernel(PV v, const double* __restrict__ x, int kind,
                                                   double* out) { pdl_wait();
    __shared__ unsigned long long rmax[256];
    __shared__ double rsum[256];
    unsigned long long m = 0ull;
    double acc = 0.0;
    long n = (long)v.nx * v.ny * v.nz;
    for (long t = blockIdx.x * 256L + threadIdx.x; t < n; t += (long)gridDim.x * 256) {
        int i = (int)(t % v.nx);
        int j = (int)((t / v.nx) % v.ny);
        int k = (int)(t / ((long)v.nx * v.ny));
        double val = x[sf_ix(v, i, j, k)];
        unsigned long long bits = (unsigned long long)__double_as_longlong(fabs(val));
        m = bits > m ? bits : m;
        acc += val * val;
    }
    rmax[threadIdx.x] = m;
    rsum[threadIdx.x] = acc;
    __syncthreads();
    for (int w = 128; w > 0; w >>= 1) {
        if (threadIdx.x < w) {
            unsigned long long o = rmax[threadIdx.x + w];
            if (o > rmax[threadIdx.x]) rmax[threadIdx.x] = o;
            rsum[threadIdx.x] += rsum[threadIdx.x + w];
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        if (kind == SF_NORM_MAX)
            atomicMax((unsigned long long*)out, rmax[0]);
        else
            atomicAdd(out, rsum[0]);
    }
}

__global__ void zero_scalar_kernel(double* p) { pdl_wait(); *p = 0.0; }

// ----------------------------------------------------------------- problem init
// HPGMG-shaped problem (the same recipe as
// inputs.py, evaluated on the device for the large configs).
constexpr double BMIN = 1.0, BMAX = 10.0, BSHARP = 10.0, BRAD = 0.25;

__device__ double beta_at(double x, double y, double z) {
    double r = sqrt((x - 0.5) * (x - 0.5) + (y - 0.5) * (y - 0.5) + (z - 0.5) * (z - 0.5));
    return 0.5 * (BMAX + BMIN) + 0.5 * (BMAX - BMIN) * tanh(BSHARP * (r - BRAD));
}
__device__ double Xf(double t) { return 2 * pow(t, 6) - 6 * pow(t, 5) + 5 * pow(t, 4) - t * t; }
__device__ double dXf(double t) { return 12 * pow(t, 5) - 30 * pow(t, 4) + 20 * pow(t, 3) - 2 * t; }
__device__ double d2Xf(double t) { return 60 * pow(t, 4) - 120 * pow(t, 3) + 60 * t * t - 2; }

__global__ void init_problem_kernel(PV v, int gnx, int gny, double h, int problem, double a,
                                    double b, int want_rhs) { pdl_wait();
    int i = blockIdx.x * blockDim.x + threadIdx.x, j = blockIdx.y * blockDim.y + threadIdx.y;
    int k = blockIdx.z;  // 0..nz  (face planes run to nz)
    if (i > v.nx || j > v.ny || k > v.nz) return;
    double Lx = gnx * h, Ly = gny * h, Lz = v.gnz * h;
    int gk = v.z0 + k;
    long q = sf_ix(v, i, j, k);
    double xc = (i + 0.5) * h / Lx, yc = (j + 0.5) * h / Ly, zc = (gk + 0.5) * h / Lz;
    double xf = i * h / Lx, yf = j * h / Ly, zf = gk * h / Lz;
    bool cx = i < v.nx, cy = j < v.ny, cz = k < v.nz;
    if (problem == 0) {
        if (cx && cy && cz) v.f[SF_ALPHA][q] = 1.0;
        if (cy && cz) v.f[SF_BETA_I][q] = 1.0;
        if (cx && cz) v.f[SF_BETA_J][q] = 1.0;
        if (cx && cy) v.f[SF_BETA_K][q] = 1.0;
    } else {
        if (cx && cy && cz) v.f[SF_ALPHA][q] = 1.0;
        if (cy && cz) v.f[SF_BETA_I][q] = beta_at(xf, yc, zc);
        if (cx && cz) v.f[SF_BETA_J][q] = beta_at(xc, yf, zc);
        if (cx && cy) v.f[SF_BETA_K][q] = beta_at(xc, yc, zf);
    }
    if (want_rhs && cx && cy && cz) {
        double X = Xf(xc), Y = Xf(yc), Z = Xf(zc);
        double u = X * Y * Z;
        double ux = dXf(xc) * Y * Z / Lx, uy = X * dXf(yc) * Z / Ly, uz = X * Y * dXf(zc) / Lz;
        double lap = d2Xf(xc) * Y * Z / (Lx * Lx) + X * d2Xf(yc) * Z / (Ly * Ly) +
                     X * Y * d2Xf(zc) / (Lz * Lz);
        double beta = 1.0, bx = 0.0, by = 0.0, bz = 0.0;
        if (problem != 0) {
            double dx = xc - 0.5, dy = yc - 0.5, dz = zc - 0.5;
            double r = sqrt(dx * dx + dy * dy + dz * dz);
            double ch = cosh(BSHARP * (r - BRAD));
            double sc = 0.5 * (BMAX - BMIN) * BSHARP / (ch * ch);
            beta = beta_at(xc, yc, zc);
            // grad beta = beta'(r) (dx, dy, dz) / r; at r = 0 (the centre cell of
            // an all-odd grid) the direction is undefined but bounded and beta'
            // is finite: the limit of the flux term's gradient part is 0
            const double ir = r > 0.0 ? 1.0 / r : 0.0;
            bx = sc * dx * ir / Lx;
            by = sc * dy * ir / Ly;
            bz = sc * dz * ir / Lz;
        }
        v.f[SF_F][q] = a * 1.0 * u - b * (bx * ux + by * uy + bz * uz + beta * lap);
    }
}

// ----------------------------------------------------------------- bottom solve
// Exact solve on the coarsest level (reading R-8).  Setup: build the dense
// operator (row r = A3 with the Dirichlet fold), invert it by Gauss-Jordan in
// shared memory (SPD: no pivoting needed), store A^-1.  Solve: x = A^-1 rhs.
constexpr int BOT_MAX = 64;

constexpr int BOT_LD = 2 * BOT_MAX + 1;
constexpr size_t BOT_SMEM = sizeof(double) * BOT_MAX * BOT_LD;

__global__ void bottom_setup_kernel(PV v, double a, double bh2, double* ainv) { pdl_wait();
    extern __shared__ double Msh[];
    double(*M)[BOT_LD] = reinterpret_cast<double(*)[BOT_LD]>(Msh);
    int n = v.nx * v.ny * v.nz;
    int r = threadIdx.x;
    if (r < n) {
        int i = r % v.nx, j = (r / v.nx) % v.ny, k = r / (v.nx * v.ny);
        for (int c = 0; c < 2 * n; c++) M[r][c] = 0.0;
        long q = sf_ix(v, i, j, k);
        const double* bi = v.f[SF_BETA_I];
        const double* bj = v.f[SF_BETA_J];
        const double* bk = v.f[SF_BETA_K];
        double bw = bi[q], be = bi[q + 1], bs = bj[q], bn = bj[q + v.js], bb = bk[q],
               bt = bk[q + v.ks];
        double d = a * v.f[SF_ALPHA][q];
        double s = 0.0;
        // diagonal: sum_f beta_f (1 + [boundary face])
        s += bw * (i == 0 ? 2.0 : 1.0);
        s += be * (i == v.nx - 1 ? 2.0 : 1.0);
        s += bs * (j == 0 ? 2.0 : 1.0);
        s += bn * (j == v.ny - 1 ? 2.0 : 1.0);
        s += bb * (k == 0 ? 2.0 : 1.0);
        s += bt * (k == v.nz - 1 ? 2.0 : 1.0);
        M[r][r] = d + bh2 * s;
        if (i > 0) M[r][r - 1] = -bh2 * bw;
        if (i < v.nx - 1) M[r][r + 1] = -bh2 * be;
        if (j > 0) M[r][r - v.nx] = -bh2 * bs;
        if (j < v.ny - 1) M[r][r + v.nx] = -bh2 * bn;
        if (k > 0) M[r][r - v.nx * v.ny] = -bh2 * bb;
        if (k < v.nz - 1) M[r][r + v.nx * v.ny] = -bh2 * bt;
        M[r][n + r] = 1.0;
    }
    __syncthreads();
    for (int p = 0; p < n; p++) {
        double piv = M[p][p];
        double fac = (r < n && r != p) ? M[r][p] / piv : 0.0;
        __syncthreads();
        if (r < n && r != p)
            for (int c = 0; c < 2 * n; c++) M[r][c] -= fac * M[p][c];
        __syncthreads();
        if (r == p)
            for (int c = 0; c < 2 * n; c++) M[p][c] /= piv;
        __syncthreads();
    }
    if (r < n)
        for (int c = 0; c < n; c++) ainv[r * n + c] = M[r][n + c];
}

__global__ void bottom_solve_kernel(PV v, double* __restrict__ x, const double* __restrict__ rhs,
                                    const double* __restrict__ ainv) { pdl_wait();
    __shared__ double rr[BOT_MAX];
    int n = v.nx * v.ny * v.nz;
    int r = threadIdx.x;
    if (r < n) {
        int i = r % v.nx, j = (r / v.nx) % v.ny, k = r / (v.nx * v.ny);
        rr[r] = rhs[sf_ix(v, i, j, k)];
    }
    __syncthreads();
    if (r < n) {
        double s = 0.0;
        for (int c = 0; c < n; c++) s += ainv[r * n + c] * rr[c];
        int i = r % v.nx, j = (r / v.nx) % v.ny, k = r / (v.nx * v.ny);
        x[sf_ix(v, i, j, k)] = s;
    }
}

}  // namespace

// ======================================================================== host
sf_status k_apply_op(sf_level* L, int out, int x, double a, double b) {
    double bh2 = b / (L->h * L->h);
    SF_TRY(sf_halo(L, x, 1));
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        sf_launch(apply_op_kernel, cell_grid(v), dim3(BX, BY), 0, L->stream, v, v.f[out], v.f[x], a, bh2);
        SF_LAUNCHED();
    }
    return sf_check_launch("apply_op");
}

sf_status k_residual(sf_level* L, int res, int x, int rhs, double a, double b) {
    if (pair_ok(L)) return k_residual_pair(L, res, x, rhs, a, b, nullptr);
    double bh2 = b / (L->h * L->h);
    SF_TRY(sf_halo(L, x, 1));
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        sf_launch(residual_kernel, cell_grid(v), dim3(BX, BY), 0, L->stream, v, v.f[res], v.f[x], v.f[rhs],
                                                                      a, bh2);
        SF_LAUNCHED();
    }
    return sf_check_launch("residual");
}

sf_status k_gsrb_colour(sf_level* L, int x, int rhs, double a, double b, int colour) {
    double bh2 = b / (L->h * L->h);
    SF_TRY(sf_halo(L, x, 1));
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        dim3 g(((v.nx + 1) / 2 + BX - 1) / BX, (v.ny + BY - 1) / BY, v.nz);
        sf_launch(gsrb_colour_kernel, g, dim3(BX, BY), 0, L->stream, v, v.f[x], v.f[rhs], a, bh2, colour);
        SF_LAUNCHED();
    }
    return sf_check_launch("gsrb_colour");
}

// Boundary-zeroed face coefficients (SF_BI0/BJ0/BK0, sf_internal.h): a copy of
// each beta array, ghosts and halo planes included, with the global Dirichlet
// faces (i = 0, nx; j = 0, ny; global k = 0, gnz) set to 0.
__global__ void beta0_kernel(PV v, long n) { pdl_wait();
    const long stride = (long)gridDim.x * blockDim.x;
    for (long e = (long)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += stride) {
        const long kk = e / v.ks, r = e - kk * v.ks, jj = r / v.js;
        const int i = (int)(r - jj * v.js) - SF_OX, j = (int)jj - SF_GY, gk = v.z0 + (int)kk - SF_GZ;
        v.f[SF_BI0][e] = (i == 0 || i == v.nx) ? 0.0 : v.f[SF_BETA_I][e];
        v.f[SF_BJ0][e] = (j == 0 || j == v.ny) ? 0.0 : v.f[SF_BETA_J][e];
        v.f[SF_BK0][e] = (gk == 0 || gk == v.gnz) ? 0.0 : v.f[SF_BETA_K][e];
    }
}

sf_status k_beta0(sf_level* L) {
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        const long n = (long)L->felems;
        const int blocks = (int)std::min<long>((n + 255) / 256, 148L * 16);
        sf_launch(beta0_kernel, blocks, 256, 0, L->stream, v, n);
        SF_LAUNCHED();
    }
    return sf_check_launch("beta0");
}

sf_status k_dinv(sf_level* L, double a, double b) {
    double bh2 = b / (L->h * L->h);
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        sf_launch(dinv_kernel, cell_grid(v), dim3(BX, BY), 0, L->stream, v, a, bh2);
        SF_LAUNCHED();
    }
    return sf_check_launch("dinv");
}

sf_status k_bc(sf_level* L, int field) {
    SF_TRY(sf_halo(L, field, 1));
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        dim3 g((v.nx + 2 + BX - 1) / BX, (v.ny + 2 + BY - 1) / BY, v.nz + 2);
        sf_launch(bc_kernel, g, dim3(BX, BY), 0, L->stream, v, v.f[field]);
        SF_LAUNCHED();
    }
    return sf_check_launch("bc");
}

// Coarse level C is either decomposed like F (same parts, half the planes) or
// replicated (single part holding the whole level on every process).
static inline bool replicated_below(const sf_level* C, const sf_level* F) {
    return C->nparts == 1 && F->nparts > 1;
}

sf_status k_restrict(sf_level* C, int cf, sf_level* F, int ff, int kind) {
    bool rep = replicated_below(C, F);
    for (int p = 0; p < F->nlocal; p++) {
        PV f = sf_view(F, p);
        PV c = sf_view(C, rep ? 0 : p);
        int zoff = rep ? f.z0 / 2 : 0;
        if (kind == SF_RESTRICT_CELL) {
            dim3 g((f.nx / 2 + BX - 1) / BX, (f.ny / 2 + BY - 1) / BY, f.nz / 2);
            sf_launch(restrict_cell_kernel, g, dim3(BX, BY), 0, F->stream, c, c.f[cf], f, f.f[ff], zoff);
        } else {
            int dir = kind - SF_RESTRICT_FACE_I;
            // beta_k: the top face of a part (index lnz/2) is written by every
            // part (it duplicates the next part's face 0, as uploaded).
            int ncz = f.nz / 2 + (dir == 2);
            dim3 g((f.nx / 2 + 1 + BX - 1) / BX, (f.ny / 2 + 1 + BY - 1) / BY, ncz);
            sf_launch(restrict_face_kernel, g, dim3(BX, BY), 0, F->stream, c, c.f[cf], f, f.f[ff], dir, zoff,
                                                                    ncz);
        }
        SF_LAUNCHED();
    }
    SF_TRY(sf_check_launch("restrict"));
    if (rep) SF_TRY(sf_agglomerate(C, cf, F->nparts, F->lnz / 2));
    return SF_OK;
}

sf_status k_interp(sf_level* F, int ff, double s, sf_level* C, int cf, int kind) {
    if (kind == SF_INTERP_P0 && pair_ok(F)) return k_interp_p0_pair(F, ff, s, C, cf);
    bool rep = replicated_below(C, F);
    if (kind == SF_INTERP_PL) SF_TRY(k_bc(C, cf));
    for (int p = 0; p < F->nlocal; p++) {
        PV f = sf_view(F, p);
        PV c = sf_view(C, rep ? 0 : p);
        int zoff = rep ? f.z0 / 2 : 0;
        if (kind == SF_INTERP_P0)
            sf_launch(interp_p0_kernel, cell_grid(f), dim3(BX, BY), 0, F->stream, f, f.f[ff], s, c, c.f[cf],
                                                                           zoff);
        else if (f.nx % 2 == 0 && f.ny % 2 == 0 && f.nz % 2 == 0)
            sf_launch(interp_pl_block_kernel, dim3((f.nx / 2 + BX - 1) / BX, (f.ny / 2 + BY - 1) / BY, f.nz / 2), dim3(BX, BY), 0, F->stream, f, f.f[ff], s, c, c.f[cf], zoff);
        else
            sf_launch(interp_pl_kernel, cell_grid(f), dim3(BX, BY), 0, F->stream, f, f.f[ff], s, c, c.f[cf],
                                                                           zoff);
        SF_LAUNCHED();
    }
    return sf_check_launch("interp");
}

sf_status k_norm(sf_level* L, int field, int kind, double* dst) {
    if (pair_ok(L)) return k_norm_pair(L, field, kind, dst);
    sf_launch(zero_scalar_kernel, 1, 1, 0, L->stream, dst);
    SF_LAUNCHED();
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        long n = (long)v.nx * v.ny * v.nz;
        int blocks = (int)std::min<long>((n + 255) / 256, 148L * 8);
        sf_launch(norm_kernel, blocks, 256, 0, L->stream, v, v.f[field], kind, dst);
        SF_LAUNCHED();
    }
    return sf_check_launch("norm");
}

// packed host-layout buffer (nzh, nyh, nxh) <-> strided field interior of one part
__global__ void __launch_bounds__(256) pack_kernel(double* __restrict__ field, long js, long ks,
                                                   double* __restrict__ buf, int nxh, int nyh,
                                                   int nzh, int up) { pdl_wait();
    const long rows = (long)nyh * nzh;
    for (long r = blockIdx.x; r < rows; r += gridDim.x) {
        const int j = (int)(r % nyh), k = (int)(r / nyh);
        double* f = field + (long)(k + SF_GZ) * ks + (long)(j + SF_GY) * js + SF_OX;
        double* b = buf + r * nxh;
        for (int i = threadIdx.x; i < nxh; i += blockDim.x) {
            if (up)
                f[i] = __ldcs(b + i);
            else
                __stcs(b + i, f[i]);
        }
    }
}

// SM copy between a field and a packed device buffer (the staging buffers of
// sf_solve_stream): a strided 3-D cudaMemcpy D2D runs on a copy engine at a
// fraction of HBM speed and would contend with the PCIe copies
sf_status k_pack(sf_level* L, int field, double* buf, bool up) {
    const int nxh = L->nx + (field == SF_BETA_I), nyh = L->ny + (field == SF_BETA_J);
    const int nzh = L->lnz + (field == SF_BETA_K);
    for (int q = 0; q < L->nlocal; q++) {
        double* b = buf + (size_t)q * L->lnz * nyh * nxh;
        const long rows = (long)nyh * nzh;
        const int grid = (int)std::min<long>(rows, 148L * 16);
        sf_launch(pack_kernel, grid, 256, 0, L->stream, L->parts[q].f[field], L->js, L->ks, b, nxh, nyh,
                                                 nzh, up ? 1 : 0);
        SF_LAUNCHED();
    }
    return sf_check_launch("pack");
}

sf_status k_zero(sf_level* L, int field) {
    for (int p = 0; p < L->nlocal; p++)
        SF_CUDA(cudaMemsetAsync(L->parts[p].f[field], 0, L->felems * sizeof(double), L->stream));
    return SF_OK;
}

sf_status k_init_problem(sf_level* L, int problem, double a, double b, int want_rhs) {
    for (int p = 0; p < L->nlocal; p++) {
        PV v = sf_view(L, p);
        dim3 g((v.nx + 1 + BX - 1) / BX, (v.ny + 1 + BY - 1) / BY, v.nz + 1);
        sf_launch(init_problem_kernel, g, dim3(BX, BY), 0, L->stream, v, L->gnx, L->gny, L->h, problem,
                                                               a, b, want_rhs);
        SF_LAUNCHED();
    }
    return sf_check_launch("init_problem");
}

sf_status k_bottom_setup(sf_level* L, double a, double b, double* ainv) {
    if (L->nlocal != 1 || L->nparts != 1) return sf_fail(SF_ERR_SHAPE, "bottom level must be replicated");
    PV v = sf_view(L, 0);
    int n = v.nx * v.ny * v.nz;
    if (n > BOT_MAX) return sf_fail(SF_ERR_SHAPE, "bottom level has %d cells (> %d)", n, BOT_MAX);
    SF_CUDA(cudaFuncSetAttribute(bottom_setup_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)BOT_SMEM));
    sf_launch(bottom_setup_kernel, 1, BOT_MAX, BOT_SMEM, L->stream, v, a, b / (L->h * L->h), ainv);
    SF_LAUNCHED();
    return sf_check_launch("bottom_setup");
}

sf_status k_bottom_solve(sf_level* L, int x, int rhs, const double* ainv) {
    PV v = sf_view(L, 0);
    sf_launch(bottom_solve_kernel, 1, BOT_MAX, 0, L->stream, v, v.f[x], v.f[rhs], ainv);
    SF_LAUNCHED();
    return sf_check_launch("bottom_solve");
}
