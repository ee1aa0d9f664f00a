/*
 * oracle/oracle.c -- plain, slow, obviously-correct CPU ORACLE for the
 * HPGMG-FV hot path that Snowflake generates (Zhang et al., IPDPSW 2017).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ipps_zhangdmwbf17_b200/, libsf.so) never
 * links, imports or calls it, and this file shares no code, header, table or
 * constant with the CUDA path.
 *
 * Built with  gcc -O2 -ffp-contract=off  (no FMA contraction), IEEE fp64,
 * single thread.  Triple loops, one ghost layer, separate arrays.  The
 * "omp parallel for" pragmas over the outer plane loop are inert in that
 * build; bench.py's cpu_baseline / --impl reference legs time a second build
 * with -fopenmp on the host's cores: every
 * parallel loop writes disjoint cells (colour sweeps are order-independent),
 * so only the L2 norm's summation order differs between the two builds.
 *
 * Citations are PAPER.md line numbers (/root/reference/PAPER.md, text of the
 * paper) plus the DESIGN.md reading (R-n) where the paper is silent.
 *
 * Storage: every field is a (nz+2)*(ny+2)*(nx+2) array, x fastest, with one
 * ghost cell on each side ("ghost zone or halo").
 * Cell (i,j,k), 0 <= i < nx, lives at OIDX(i,j,k).  Face arrays use the same
 * shape: beta_i(i,j,k) is the face between cells i-1 and i (0 <= i <= nx), so
 * the face i = nx lives in the high ghost slot (reading R-3).
 *
 * Pins (tests/test_oracle_pins.py): every function below is pinned to
 * closed forms / brute force / invariants -- see DESIGN.md section "Oracle pins".
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct {
    int nx, ny, nz;
    double h;
} or_grid;

#define SX(g) ((size_t)(g)->nx + 2)
#define SY(g) ((size_t)(g)->ny + 2)
#define OIDX(g, i, j, k) \
    ((((size_t)((k) + 1)) * SY(g) + (size_t)((j) + 1)) * SX(g) + (size_t)((i) + 1))

/* threads of the timing build (1 in the single-thread build) */
int or_set_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
    return omp_get_max_threads();
#else
    (void)n;
    return 1;
#endif
}

size_t or_size(int nx, int ny, int nz) {
    return ((size_t)nx + 2) * ((size_t)ny + 2) * ((size_t)nz + 2);
}

/* ------------------------------------------------------------------------ */
/* A2: homogeneous Dirichlet ghost fill.                                     */
/* PAPER.md:333-341 (Sec. II.B): "the ghost value immediately outside a      */
/* boundary cell is set to the negative of the value immediately inside";    */
/* Fig 4 lines 15-18.  Edges and corners (not shown in    */
/* the paper) follow reading R-5: odd reflection in every axis the cell is   */
/* outside of, i.e. value = (-1)^m * x(mirror).                              */
/* ------------------------------------------------------------------------ */
void or_apply_bc(const or_grid* g, double* x) {
#pragma omp parallel for schedule(static)
    for (int k = -1; k <= g->nz; k++)
        for (int j = -1; j <= g->ny; j++)
            for (int i = -1; i <= g->nx; i++) {
                int m = 0, mi = i, mj = j, mk = k;
                if (i < 0) { mi = 0; m++; }
                if (i >= g->nx) { mi = g->nx - 1; m++; }
                if (j < 0) { mj = 0; m++; }
                if (j >= g->ny) { mj = g->ny - 1; m++; }
                if (k < 0) { mk = 0; m++; }
                if (k >= g->nz) { mk = g->nz - 1; m++; }
                if (m == 0) continue;
                double v = x[OIDX(g, mi, mj, mk)];
                x[OIDX(g, i, j, k)] = (m % 2 == 1) ? -v : v;
            }
}

/* ------------------------------------------------------------------------ */
/* A3: variable-coefficient 7-point Helmholtz operator                       */
/*   Ax(c) = a*alpha(c)*x(c) - b*h^-2 * sum_{6 faces f} beta_f*(x(nbr_f)-x(c))*/
/* PAPER.md:361-367 (Fig 4 lines 1-5, the 2-D beta_x/beta_y 5-point Ax),     */
/* PAPER.md:383-385 ("solving -div(beta grad x) = b")      */
/* ("variable-coefficient 7-point Laplacian"); a, alpha, h per reading R-1.  */
/* Ghost values are read from x, so the caller applies A2 first.             */
/* ------------------------------------------------------------------------ */
static double op_at(const or_grid* g, double a, double b, const double* alpha,
                    const double* bi, const double* bj, const double* bk,
                    const double* x, int i, int j, int k) {
    double hm2 = 1.0 / (g->h * g->h);
    double xc = x[OIDX(g, i, j, k)];
    double flux = 0.0;
    flux += bi[OIDX(g, i + 1, j, k)] * (x[OIDX(g, i + 1, j, k)] - xc);
    flux += bi[OIDX(g, i, j, k)] * (x[OIDX(g, i - 1, j, k)] - xc);
    flux += bj[OIDX(g, i, j + 1, k)] * (x[OIDX(g, i, j + 1, k)] - xc);
    flux += bj[OIDX(g, i, j, k)] * (x[OIDX(g, i, j - 1, k)] - xc);
    flux += bk[OIDX(g, i, j, k + 1)] * (x[OIDX(g, i, j, k + 1)] - xc);
    flux += bk[OIDX(g, i, j, k)] * (x[OIDX(g, i, j, k - 1)] - xc);
    return a * alpha[OIDX(g, i, j, k)] * xc - b * hm2 * flux;
}

/* out = A x  (applies A2 to x first; only interior of out is written) */
void or_apply_op(const or_grid* g, double a, double b, const double* alpha,
                 const double* bi, const double* bj, const double* bk,
                 double* x, double* out) {
    or_apply_bc(g, x);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++)
                out[OIDX(g, i, j, k)] = op_at(g, a, b, alpha, bi, bj, bk, x, i, j, k);
}

/* A6: residual res = rhs - A x  ("residual"; 799-800) */
void or_residual(const or_grid* g, double a, double b, const double* alpha,
                 const double* bi, const double* bj, const double* bk,
                 double* x, const double* rhs, double* res) {
    or_apply_bc(g, x);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++)
                res[OIDX(g, i, j, k)] =
                    rhs[OIDX(g, i, j, k)] - op_at(g, a, b, alpha, bi, bj, bk, x, i, j, k);
}

/* ------------------------------------------------------------------------ */
/* A4: lambda = Dinv = 1/diag(A) with A2 folded in (reading R-4):            */
/* a face on the global Dirichlet boundary has ghost = -x(c), so its term    */
/* beta_f*(-x(c) - x(c)) contributes 2*beta_f to the diagonal.               */
/* PAPER.md:371-373 (Fig 4 line 9 "lambda"), 396-399 ("a factor lambda").    */
/* ------------------------------------------------------------------------ */
void or_dinv(const or_grid* g, double a, double b, const double* alpha,
             const double* bi, const double* bj, const double* bk, double* dinv) {
    double hm2 = 1.0 / (g->h * g->h);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) {
                double s = 0.0;
                s += bi[OIDX(g, i, j, k)] * (i == 0 ? 2.0 : 1.0);
                s += bi[OIDX(g, i + 1, j, k)] * (i == g->nx - 1 ? 2.0 : 1.0);
                s += bj[OIDX(g, i, j, k)] * (j == 0 ? 2.0 : 1.0);
                s += bj[OIDX(g, i, j + 1, k)] * (j == g->ny - 1 ? 2.0 : 1.0);
                s += bk[OIDX(g, i, j, k)] * (k == 0 ? 2.0 : 1.0);
                s += bk[OIDX(g, i, j, k + 1)] * (k == g->nz - 1 ? 2.0 : 1.0);
                dinv[OIDX(g, i, j, k)] = 1.0 / (a * alpha[OIDX(g, i, j, k)] + b * hm2 * s);
            }
}

/* ------------------------------------------------------------------------ */
/* A5: one GSRB colour sweep, in place.                                      */
/* Fig 4 lines 6-14: difference = rhs - Ax;               */
/*   final = original + lambda*difference, over the red (then black) domain. */
/* in place, red reads black and vice versa.               */
/* boundary / red / boundary / black.                      */
/* Colour (reading R-2): red = (i+j+k) even in 0-based interior indices.     */
/* Within one colour no updated cell is read by another update of the same  */
/* colour (7-point stencil), so this loop order is immaterial.               */
/* ------------------------------------------------------------------------ */
void or_gsrb_sweep(const or_grid* g, double a, double b, const double* alpha,
                   const double* bi, const double* bj, const double* bk,
                   const double* dinv, double* x, const double* rhs, int colour) {
    or_apply_bc(g, x);                                   /* "boundary" stencils */
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) {
                if (((i + j + k) & 1) != colour) continue;
                double ax = op_at(g, a, b, alpha, bi, bj, bk, x, i, j, k);
                size_t c = OIDX(g, i, j, k);
                x[c] = x[c] + dinv[c] * (rhs[c] - ax);
            }
}

/* rb_pairs x (BC, red, BC, black); HPGMG "smooth" = 2 pairs */
void or_smooth(const or_grid* g, double a, double b, const double* alpha,
               const double* bi, const double* bj, const double* bk,
               const double* dinv, double* x, const double* rhs, int rb_pairs) {
    for (int p = 0; p < rb_pairs; p++) {
        or_gsrb_sweep(g, a, b, alpha, bi, bj, bk, dinv, x, rhs, 0);
        or_gsrb_sweep(g, a, b, alpha, bi, bj, bk, dinv, x, rhs, 1);
    }
}

/* ------------------------------------------------------------------------ */
/* A7: 2:1 restriction (PAPER.md:293-297 striding; 466-468 affine index      */
/* maps "2i+..."; 597, 652).  Reading R-7: cell average for cell fields,     */
/* face average (4 fine faces on the coarse face) for beta.                  */
/* ------------------------------------------------------------------------ */
void or_restrict_cell(const or_grid* gc, double* coarse, const or_grid* gf,
                      const double* fine) {
#pragma omp parallel for schedule(static)
    for (int K = 0; K < gc->nz; K++)
        for (int J = 0; J < gc->ny; J++)
            for (int I = 0; I < gc->nx; I++) {
                double s = 0.0;
                for (int d = 0; d < 2; d++)
                    for (int bb = 0; bb < 2; bb++)
                        for (int aa = 0; aa < 2; aa++)
                            s += fine[OIDX(gf, 2 * I + aa, 2 * J + bb, 2 * K + d)];
                coarse[OIDX(gc, I, J, K)] = s / 8.0;
            }
}

/* dir 0: beta_i faces (I in [0,nx_c]); 1: beta_j; 2: beta_k */
void or_restrict_face(const or_grid* gc, double* coarse, const or_grid* gf,
                      const double* fine, int dir) {
    int ex = dir == 0, ey = dir == 1, ez = dir == 2;
#pragma omp parallel for schedule(static)
    for (int K = 0; K < gc->nz + ez; K++)
        for (int J = 0; J < gc->ny + ey; J++)
            for (int I = 0; I < gc->nx + ex; I++) {
                double s = 0.0;
                for (int p = 0; p < 2; p++)
                    for (int q = 0; q < 2; q++) {
                        int i = 2 * I, j = 2 * J, k = 2 * K;
                        if (dir == 0) { j += p; k += q; }
                        if (dir == 1) { i += p; k += q; }
                        if (dir == 2) { i += p; j += q; }
                        s += fine[OIDX(gf, i, j, k)];
                    }
                coarse[OIDX(gc, I, J, K)] = s / 4.0;
            }
}

/* ------------------------------------------------------------------------ */
/* A8: 2:1 interpolation with prescale s:  fine <- s*fine + P(coarse).       */
/* P0 (piecewise constant, used in the V-cycle) and PL (trilinear on cell    */
/* centres, used in the F-cycle) -- reading R-7.         */
/* ------------------------------------------------------------------------ */
void or_interp_p0(const or_grid* gf, double* fine, double prescale,
                  const or_grid* gc, const double* coarse) {
#pragma omp parallel for schedule(static)
    for (int k = 0; k < gf->nz; k++)
        for (int j = 0; j < gf->ny; j++)
            for (int i = 0; i < gf->nx; i++) {
                size_t c = OIDX(gf, i, j, k);
                fine[c] = prescale * fine[c] + coarse[OIDX(gc, i / 2, j / 2, k / 2)];
            }
}

/* Trilinear: a fine centre sits h_c/4 from its parent centre toward the     */
/* child side in each axis, so the 1-D weights are 3/4 (parent) and 1/4     */
/* (neighbour on the child side); the 3-D weights are their products.        */
/* Coarse ghosts (faces, edges, corners) come from A2 on the coarse field.   */
void or_interp_pl(const or_grid* gf, double* fine, double prescale,
                  const or_grid* gc, double* coarse) {
    or_apply_bc(gc, coarse);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < gf->nz; k++)
        for (int j = 0; j < gf->ny; j++)
            for (int i = 0; i < gf->nx; i++) {
                int I = i / 2, J = j / 2, K = k / 2;
                int di = (i % 2 == 1) ? 1 : -1;
                int dj = (j % 2 == 1) ? 1 : -1;
                int dk = (k % 2 == 1) ? 1 : -1;
                double p = 0.0;
                for (int c = 0; c < 2; c++)
                    for (int bb = 0; bb < 2; bb++)
                        for (int aa = 0; aa < 2; aa++) {
                            double w = (aa ? 0.25 : 0.75) * (bb ? 0.25 : 0.75) * (c ? 0.25 : 0.75);
                            p += w * coarse[OIDX(gc, I + aa * di, J + bb * dj, K + c * dk)];
                        }
                size_t f = OIDX(gf, i, j, k);
                fine[f] = prescale * fine[f] + p;
            }
}

/* A10: norms over the interior */
double or_norm_max(const or_grid* g, const double* x) {
    double m = 0.0;
#pragma omp parallel for reduction(max : m) schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) {
                double v = fabs(x[OIDX(g, i, j, k)]);
                if (v > m) m = v;
            }
    return m;
}

double or_norm_l2(const or_grid* g, const double* x) {
    double s = 0.0;
#pragma omp parallel for reduction(+ : s) schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) {
                double v = x[OIDX(g, i, j, k)];
                s += v * v;
            }
    return sqrt(s);
}

/* ------------------------------------------------------------------------ */
/* Bottom solve (reading R-8): exact.  Build the dense operator column by    */
/* column by applying A3 (with A2) to unit vectors, then Cholesky (the       */
/* operator is SPD), then forward/back substitution.                         */
/* ------------------------------------------------------------------------ */
int or_bottom_solve(const or_grid* g, double a, double b, const double* alpha,
                    const double* bi, const double* bj, const double* bk,
                    double* x, const double* rhs) {
    int n = g->nx * g->ny * g->nz;
    size_t sz = or_size(g->nx, g->ny, g->nz);
    double* A = calloc((size_t)n * n, sizeof(double));
    double* e = calloc(sz, sizeof(double));
    double* ae = calloc(sz, sizeof(double));
    double* y = calloc((size_t)n, sizeof(double));
    int rc = 0;
    for (int col = 0; col < n; col++) {
        memset(e, 0, sz * sizeof(double));
        int ci = col % g->nx, cj = (col / g->nx) % g->ny, ck = col / (g->nx * g->ny);
        e[OIDX(g, ci, cj, ck)] = 1.0;
        or_apply_op(g, a, b, alpha, bi, bj, bk, e, ae);
        for (int row = 0; row < n; row++) {
            int ri = row % g->nx, rj = (row / g->nx) % g->ny, rk = row / (g->nx * g->ny);
            A[(size_t)row * n + col] = ae[OIDX(g, ri, rj, rk)];
        }
    }
    /* Cholesky A = L L^T, L stored in the lower triangle of A */
    for (int j = 0; j < n; j++) {
        double d = A[(size_t)j * n + j];
        for (int p = 0; p < j; p++) d -= A[(size_t)j * n + p] * A[(size_t)j * n + p];
        if (!(d > 0.0)) { rc = -1; goto done; }
        d = sqrt(d);
        A[(size_t)j * n + j] = d;
        for (int i = j + 1; i < n; i++) {
            double s = A[(size_t)i * n + j];
            for (int p = 0; p < j; p++) s -= A[(size_t)i * n + p] * A[(size_t)j * n + p];
            A[(size_t)i * n + j] = s / d;
        }
    }
    for (int i = 0; i < n; i++) {            /* L y = rhs */
        int ri = i % g->nx, rj = (i / g->nx) % g->ny, rk = i / (g->nx * g->ny);
        double s = rhs[OIDX(g, ri, rj, rk)];
        for (int p = 0; p < i; p++) s -= A[(size_t)i * n + p] * y[p];
        y[i] = s / A[(size_t)i * n + i];
    }
    for (int i = n - 1; i >= 0; i--) {       /* L^T x = y */
        double s = y[i];
        for (int p = i + 1; p < n; p++) s -= A[(size_t)p * n + i] * y[p];
        y[i] = s / A[(size_t)i * n + i];
    }
    for (int i = 0; i < n; i++) {
        int ri = i % g->nx, rj = (i / g->nx) % g->ny, rk = i / (g->nx * g->ny);
        x[OIDX(g, ri, rj, rk)] = y[i];
    }
done:
    free(A); free(e); free(ae); free(y);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* A9: multigrid hierarchy, V-cycle, F-cycle, solve.                         */
/* PAPER.md:595-599 ("restriction, smoothing, and interpolation"),           */
/* 627-629 (10 V-cycles, two GSRB smooths = 4 sweeps pre and post),          */
/* 647-653 (smoother, residual, restriction, interpolation, BC).             */
/* Coarse operators are re-discretised from restricted alpha/beta with       */
/* h_c = 2h (reading R-7); bottom at min dim 2 (reading R-8).                */
/* ------------------------------------------------------------------------ */
#define OR_MAXL 24
void or_chebyshev(const or_grid* g, double a, double b, const double* alpha, const double* bi,
                  const double* bj, const double* bk, const double* dinv, double* x,
                  const double* f, int degree, double lo, double hi, double* xprev,
                  double* xnext);
double or_lambda_max(const or_grid* g, double a, double b, const double* alpha, const double* bi,
                     const double* bj, const double* bk, const double* dinv, double* v,
                     double* w, int iters);
typedef struct {
    int nl;
    double a, b;
    int pre, post;
    int cheby_steps;                  /* NEXT-3: Chebyshev steps per "pair" (0 = GSRB) */
    double lmax[OR_MAXL];
    or_grid g[OR_MAXL];
    double *alpha[OR_MAXL], *bi[OR_MAXL], *bj[OR_MAXL], *bk[OR_MAXL], *dinv[OR_MAXL];
    double *e[OR_MAXL], *r[OR_MAXL], *res[OR_MAXL];
} or_mg;

static double* zalloc(const or_grid* g) {
    return calloc(or_size(g->nx, g->ny, g->nz), sizeof(double));
}

/* alpha/bi/bj/bk: finest-level arrays in oracle layout (copied) */
or_mg* or_mg_create(int nx, int ny, int nz, double h, double a, double b,
                    const double* alpha, const double* bi, const double* bj,
                    const double* bk, int pre, int post) {
    or_mg* m = calloc(1, sizeof(or_mg));
    m->a = a; m->b = b; m->pre = pre; m->post = post;
    or_grid g = {nx, ny, nz, h};
    int l = 0;
    for (;;) {
        m->g[l] = g;
        size_t sz = or_size(g.nx, g.ny, g.nz) * sizeof(double);
        m->alpha[l] = zalloc(&g); m->bi[l] = zalloc(&g); m->bj[l] = zalloc(&g);
        m->bk[l] = zalloc(&g); m->dinv[l] = zalloc(&g);
        m->e[l] = zalloc(&g); m->r[l] = zalloc(&g); m->res[l] = zalloc(&g);
        if (l == 0) {
            memcpy(m->alpha[0], alpha, sz); memcpy(m->bi[0], bi, sz);
            memcpy(m->bj[0], bj, sz); memcpy(m->bk[0], bk, sz);
        } else {
            or_restrict_cell(&m->g[l], m->alpha[l], &m->g[l - 1], m->alpha[l - 1]);
            or_restrict_face(&m->g[l], m->bi[l], &m->g[l - 1], m->bi[l - 1], 0);
            or_restrict_face(&m->g[l], m->bj[l], &m->g[l - 1], m->bj[l - 1], 1);
            or_restrict_face(&m->g[l], m->bk[l], &m->g[l - 1], m->bk[l - 1], 2);
        }
        or_dinv(&m->g[l], a, b, m->alpha[l], m->bi[l], m->bj[l], m->bk[l], m->dinv[l]);
        int mn = g.nx < g.ny ? g.nx : g.ny;
        mn = mn < g.nz ? mn : g.nz;
        if (mn <= 2 || (g.nx | g.ny | g.nz) & 1 || l + 1 == OR_MAXL) break;
        g.nx /= 2; g.ny /= 2; g.nz /= 2; g.h *= 2.0;
        l++;
    }
    m->nl = l + 1;
    return m;
}

void or_mg_free(or_mg* m) {
    if (!m) return;
    for (int l = 0; l < m->nl; l++) {
        free(m->alpha[l]); free(m->bi[l]); free(m->bj[l]); free(m->bk[l]);
        free(m->dinv[l]); free(m->e[l]); free(m->r[l]); free(m->res[l]);
    }
    free(m);
}

int or_mg_levels(const or_mg* m) { return m->nl; }
void or_mg_level_dims(const or_mg* m, int l, int* d) {
    d[0] = m->g[l].nx; d[1] = m->g[l].ny; d[2] = m->g[l].nz;
}

#define LV(m, l) &(m)->g[l], (m)->a, (m)->b, (m)->alpha[l], (m)->bi[l], (m)->bj[l], (m)->bk[l]

/* smoother of V(l): GSRB pairs or, after or_mg_set_chebyshev,
 * Chebyshev with 'pairs * cheby_steps' steps on [hi/8, hi], hi = 1.05 lambda_max
 * (reading R-16) */
static void mg_smooth(or_mg* m, int l, int pairs) {
    if (!m->cheby_steps) {
        or_smooth(LV(m, l), m->dinv[l], m->e[l], m->r[l], pairs);
        return;
    }
    if (pairs == 0) return;
    size_t sz = or_size(m->g[l].nx, m->g[l].ny, m->g[l].nz) * sizeof(double);
    double* w1 = malloc(sz);
    double* w2 = malloc(sz);
    double hi = 1.05 * m->lmax[l], lo = hi / 8.0;
    or_chebyshev(LV(m, l), m->dinv[l], m->e[l], m->r[l], pairs * m->cheby_steps, lo, hi, w1, w2);
    free(w1);
    free(w2);
}

/* NEXT-3: switch the hierarchy to Chebyshev smoothing; lambda_max(D^-1 A) per
 * level by 30 power-iteration steps from v = 1 + ((7i + 13j + 29k) mod 17)/17 */
void or_mg_set_chebyshev(or_mg* m, int steps_per_pair) {
    m->cheby_steps = steps_per_pair;
    for (int l = 0; l + 1 < m->nl; l++) {
        or_grid* g = &m->g[l];
        size_t sz = or_size(g->nx, g->ny, g->nz);
        double* v = calloc(sz, sizeof(double));
        double* w = calloc(sz, sizeof(double));
        for (int k = 0; k < g->nz; k++)
            for (int j = 0; j < g->ny; j++)
                for (int i = 0; i < g->nx; i++)
                    v[OIDX(g, i, j, k)] = 1.0 + (double)((7L * i + 13L * j + 29L * k) % 17) / 17.0;
        m->lmax[l] = or_lambda_max(LV(m, l), m->dinv[l], v, w, 30);
        free(v);
        free(w);
    }
}

/* V(l) on (e[l], r[l]); see SURVEY/DESIGN A9 */
static int vcycle(or_mg* m, int l) {
    if (l == m->nl - 1) return or_bottom_solve(LV(m, l), m->e[l], m->r[l]);
    mg_smooth(m, l, m->pre);
    or_residual(LV(m, l), m->e[l], m->r[l], m->res[l]);
    or_restrict_cell(&m->g[l + 1], m->r[l + 1], &m->g[l], m->res[l]);
    memset(m->e[l + 1], 0,
           or_size(m->g[l + 1].nx, m->g[l + 1].ny, m->g[l + 1].nz) * sizeof(double));
    int rc = vcycle(m, l + 1);
    or_interp_p0(&m->g[l], m->e[l], 1.0, &m->g[l + 1], m->e[l + 1]);
    mg_smooth(m, l, m->post);
    return rc;
}

/* u, f: finest-level arrays in oracle layout; one V-cycle in place on u */
int or_mg_vcycle(or_mg* m, double* u, const double* f) {
    size_t sz = or_size(m->g[0].nx, m->g[0].ny, m->g[0].nz) * sizeof(double);
    memcpy(m->e[0], u, sz); memcpy(m->r[0], f, sz);
    int rc = vcycle(m, 0);
    memcpy(u, m->e[0], sz);
    return rc;
}

/* One F-cycle from scratch: restrict f to all levels, bottom solve, then for */
/* each level from coarse to fine: e_l = PL(e_{l+1}) (prescale 0), V(l).      */
int or_mg_fcycle(or_mg* m, double* u, const double* f) {
    size_t sz = or_size(m->g[0].nx, m->g[0].ny, m->g[0].nz) * sizeof(double);
    memcpy(m->r[0], f, sz);
    for (int l = 1; l < m->nl; l++)
        or_restrict_cell(&m->g[l], m->r[l], &m->g[l - 1], m->r[l - 1]);
    int L = m->nl - 1;
    memset(m->e[L], 0, or_size(m->g[L].nx, m->g[L].ny, m->g[L].nz) * sizeof(double));
    int rc = or_bottom_solve(LV(m, L), m->e[L], m->r[L]);
    for (int l = L - 1; l >= 0; l--) {
        or_interp_pl(&m->g[l], m->e[l], 0.0, &m->g[l + 1], m->e[l + 1]);
        rc |= vcycle(m, l);
    }
    memcpy(u, m->e[0], sz);
    return rc;
}

/* ||f - A u||_inf / ||f||_inf on the finest level */
double or_mg_relres(or_mg* m, double* u, const double* f) {
    or_residual(LV(m, 0), u, f, m->res[0]);
    return or_norm_max(&m->g[0], m->res[0]) / or_norm_max(&m->g[0], f);
}

/* Solve: optional F-cycle first, then V-cycles until relres < rtol or       */
/* maxc cycles in total.  hist[c] = relres after cycle c.  Returns cycles.   */
int or_mg_solve(or_mg* m, double* u, const double* f, int fcycle, double rtol,
                int maxc, double* hist) {
    int c = 0;
    if (fcycle) {
        or_mg_fcycle(m, u, f);
        hist[c++] = or_mg_relres(m, u, f);
        if (hist[c - 1] < rtol) return c;
    }
    while (c < maxc) {
        or_mg_vcycle(m, u, f);
        hist[c++] = or_mg_relres(m, u, f);
        if (hist[c - 1] < rtol) break;
    }
    return c;
}

/* ------------------------------------------------------------------------ */
/* Sampled evaluation at full size (tests at BASELINE sizes): the same A3/A5 */
/* definitions as above, evaluated one cell at a time.                       */
/* ------------------------------------------------------------------------ */
/* res[s] = rhs - A x at cells (ii[s], jj[s], kk[s]).  Applies A2 to x. */
void or_residual_points(const or_grid* g, double a, double b, const double* alpha,
                        const double* bi, const double* bj, const double* bk, double* x,
                        const double* rhs, int n, const int* ii, const int* jj, const int* kk,
                        double* res) {
    or_apply_bc(g, x);
    for (int s = 0; s < n; s++)
        res[s] = rhs[OIDX(g, ii[s], jj[s], kk[s])] -
                 op_at(g, a, b, alpha, bi, bj, bk, x, ii[s], jj[s], kk[s]);
}

/* Value of cell (i,j,k) after ONE RB pair (BC, red, BC, black) started from */
/* x, without sweeping the grid: a red cell needs only its own red update;   */
/* a black cell needs the red updates of its in-domain neighbours first.     */
/* x must have A2 applied (or_apply_bc) and is restored before returning.    */
static double red_update_at(const or_grid* g, double a, double b, const double* alpha,
                            const double* bi, const double* bj, const double* bk,
                            const double* dinv, const double* x, const double* rhs, int i, int j,
                            int k) {
    size_t c = OIDX(g, i, j, k);
    return x[c] + dinv[c] * (rhs[c] - op_at(g, a, b, alpha, bi, bj, bk, x, i, j, k));
}

void or_gsrb_pair_points(const or_grid* g, double a, double b, const double* alpha,
                         const double* bi, const double* bj, const double* bk, const double* dinv,
                         double* x, const double* rhs, int n, const int* ii, const int* jj,
                         const int* kk, double* out) {
    or_apply_bc(g, x);
    static const int off[6][3] = {{1, 0, 0}, {-1, 0, 0}, {0, 1, 0}, {0, -1, 0}, {0, 0, 1}, {0, 0, -1}};
    for (int s = 0; s < n; s++) {
        int i = ii[s], j = jj[s], k = kk[s];
        if (((i + j + k) & 1) == 0) {
            out[s] = red_update_at(g, a, b, alpha, bi, bj, bk, dinv, x, rhs, i, j, k);
            continue;
        }
        double nv[6], ov[6];
        size_t at[6];
        int in[6];
        for (int d = 0; d < 6; d++) {
            int p = i + off[d][0], q = j + off[d][1], r = k + off[d][2];
            in[d] = p >= 0 && p < g->nx && q >= 0 && q < g->ny && r >= 0 && r < g->nz;
            at[d] = OIDX(g, p, q, r);
            if (in[d]) nv[d] = red_update_at(g, a, b, alpha, bi, bj, bk, dinv, x, rhs, p, q, r);
        }
        for (int d = 0; d < 6; d++)
            if (in[d]) { ov[d] = x[at[d]]; x[at[d]] = nv[d]; }
        /* ghosts adjacent to the black cell mirror the black cell itself,  */
        /* which the red sweep did not change: no BC refresh is needed.     */
        out[s] = red_update_at(g, a, b, alpha, bi, bj, bk, dinv, x, rhs, i, j, k);
        for (int d = 0; d < 6; d++)
            if (in[d]) x[at[d]] = ov[d];
    }
}

/* ------------------------------------------------------------------------ */
/* NEXT-2 (Fig 7's other two operators, Sec. V.A):         */
/* the canonical 7-point constant-coefficient Laplacian                      */
/*   L x(c) = h^-2 * sum_{6 neighbours n} (x(c) - x(n))                      */
/* (A3 with a = 0, b = 1, beta = 1; ghosts from A2), and the weighted Jacobi */
/* smoother x <- x + (2/3) D^-1 (f - L x) (garbled "2/3 D^-1", reading R-11),*/
/* D = diag(L) with the Dirichlet fold (a boundary face adds 2/h^2).         */
/* ------------------------------------------------------------------------ */
static double lap_at(const or_grid* g, const double* x, int i, int j, int k) {
    double hm2 = 1.0 / (g->h * g->h);
    double xc = x[OIDX(g, i, j, k)];
    double s = 0.0;
    s += xc - x[OIDX(g, i + 1, j, k)];
    s += xc - x[OIDX(g, i - 1, j, k)];
    s += xc - x[OIDX(g, i, j + 1, k)];
    s += xc - x[OIDX(g, i, j - 1, k)];
    s += xc - x[OIDX(g, i, j, k + 1)];
    s += xc - x[OIDX(g, i, j, k - 1)];
    return hm2 * s;
}

void or_laplacian_cc(const or_grid* g, double* x, double* out) {
    or_apply_bc(g, x);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) out[OIDX(g, i, j, k)] = lap_at(g, x, i, j, k);
}

void or_jacobi_cc(const or_grid* g, double omega, double* x, const double* f, double* out) {
    double hm2 = 1.0 / (g->h * g->h);
    or_apply_bc(g, x);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < g->nz; k++)
        for (int j = 0; j < g->ny; j++)
            for (int i = 0; i < g->nx; i++) {
                int nb = (i == 0) + (i == g->nx - 1) + (j == 0) + (j == g->ny - 1) + (k == 0) +
                         (k == g->nz - 1);
                double d = hm2 * (6.0 + nb);
                size_t c = OIDX(g, i, j, k);
                out[c] = x[c] + omega * (f[c] - lap_at(g, x, i, j, k)) / d;
            }
}

/* ------------------------------------------------------------------------ */
/* NEXT-3: Chebyshev polynomial smoother (PAPER.md:306-308 names "Chebyshev  */
/* smoothing" as an in-place technique; the paper gives no formula -- reading */
/* R-16).  Chebyshev acceleration of the Jacobi-preconditioned iteration     */
/* (Saad, Iterative Methods, Alg. 12.1) for eigenvalues of D^-1 A in         */
/* [lo, hi]: theta = (hi+lo)/2, delta = (hi-lo)/2, sigma = theta/delta,      */
/*   x1 = x0 + (1/theta) D^-1 (f - A x0),                                    */
/*   x_{k+1} = x_k + rho_k rho_{k-1} (x_k - x_{k-1})                         */
/*                 + (2 rho_k / delta) D^-1 (f - A x_k),                    */
/*   rho_0 = 1/sigma, rho_k = 1/(2 sigma - rho_{k-1}).                       */
/* x is overwritten with x_degree; work holds two scratch arrays.            */
/* ------------------------------------------------------------------------ */
void or_chebyshev(const or_grid* g, double a, double b, const double* alpha, const double* bi,
                  const double* bj, const double* bk, const double* dinv, double* x,
                  const double* f, int degree, double lo, double hi, double* xprev,
                  double* xnext) {
    size_t sz = or_size(g->nx, g->ny, g->nz);
    double theta = 0.5 * (hi + lo), delta = 0.5 * (hi - lo), sigma = theta / delta;
    double rho_prev = 1.0 / sigma, rho = rho_prev;
    memcpy(xprev, x, sz * sizeof(double));
    for (int it = 0; it < degree; it++) {
        double c1, c2;
        if (it == 0) {
            c1 = 0.0;
            c2 = 1.0 / theta;
        } else {
            rho = 1.0 / (2.0 * sigma - rho_prev);
            c1 = rho * rho_prev;
            c2 = 2.0 * rho / delta;
        }
        or_apply_bc(g, x);
        for (int k = 0; k < g->nz; k++)
            for (int j = 0; j < g->ny; j++)
                for (int i = 0; i < g->nx; i++) {
                    size_t c = OIDX(g, i, j, k);
                    double r = f[c] - op_at(g, a, b, alpha, bi, bj, bk, x, i, j, k);
                    xnext[c] = x[c] + c1 * (x[c] - xprev[c]) + c2 * dinv[c] * r;
                }
        memcpy(xprev, x, sz * sizeof(double));
        memcpy(x, xnext, sz * sizeof(double));
        if (it > 0) rho_prev = rho;
    }
}

/* Largest eigenvalue of D^-1 A by power iteration (setup of the Chebyshev   */
/* interval, reading R-16): v <- D^-1 A v / ||D^-1 A v||_2, iters times from */
/* the given start; returns the last ||D^-1 A v||_2 / ||v||_2.              */
double or_lambda_max(const or_grid* g, double a, double b, const double* alpha, const double* bi,
                     const double* bj, const double* bk, const double* dinv, double* v,
                     double* w, int iters) {
    double lam = 0.0;
    for (int it = 0; it < iters; it++) {
        double nv = or_norm_l2(g, v);
        or_apply_op(g, a, b, alpha, bi, bj, bk, v, w);
        for (int k = 0; k < g->nz; k++)
            for (int j = 0; j < g->ny; j++)
                for (int i = 0; i < g->nx; i++) {
                    size_t c = OIDX(g, i, j, k);
                    w[c] = dinv[c] * w[c];
                }
        double nw = or_norm_l2(g, w);
        lam = nw / nv;
        for (int k = 0; k < g->nz; k++)
            for (int j = 0; j < g->ny; j++)
                for (int i = 0; i < g->nx; i++) {
                    size_t c = OIDX(g, i, j, k);
                    v[c] = w[c] / nw;
                }
    }
    return lam;
}
