// Multigrid driver (A9): hierarchy construction, V-cycle, F-cycle, solve.
//
// PAPER.md:595-599 (restriction, smoothing, interpolation over grid spacings),
// 627-629 (two GSRB smooths = 4 sweeps pre and post), 647-653 (smoother,
// residual, restriction, interpolation, boundary stencils).  Coarse operators
// are re-discretised from restricted alpha / beta with h_c = 2h (reading R-7);
// bottom = exact solve at min dim 2 (reading R-8).
//
// Every cycle only ENQUEUES work on the finest level's stream (no host sync),
// so a whole V-cycle (+ its convergence residual and norm) is captured once as
// a CUDA graph and replayed: levels <= 64^3 are launch-latency bound.
#include <chrono>
#include <cmath>
#include <cstdlib>

#include <nvtx3/nvToolsExt.h>

#include "sf_internal.h"

// NVTX ranges per cycle and level (Nsight timelines; inert without a tool)
struct NvtxRange {
    explicit NvtxRange(const char* fmt, int a = 0, int b = 0, int c = 0, int d = 0) {
        char name[96];
        snprintf(name, sizeof(name), fmt, a, b, c, d);
        nvtxRangePushA(name);
    }
    ~NvtxRange() { nvtxRangePop(); }
};

// Device-resident solve loop (sf_solve with graphs): termination is decided on
// the device and drives a CUDA-graph WHILE node, so a whole solve is one graph
// launch and one host synchronisation.
#define SF_LOOP_HIST 256
struct LoopCtl {    // device memory
    double fn, rtol;
    int max_cycles, done, status, nbody;
    double hist[SF_LOOP_HIST];
};
struct LoopHost {   // mapped pinned memory: rtol / max_cycles in, results out
    double rtol;
    int max_cycles, done, status, nbody;
    double hist[SF_LOOP_HIST];
};
enum { LS_RUN = 0, LS_CONVERGED = 1, LS_NUMERIC = 2, LS_NOT_CONVERGED = 3, LS_ZERO = 4, LS_RHS_NAN = 5 };

struct sf_mg {
    std::vector<sf_level*> lv;
    std::vector<bool> own;
    double a, b;
    sf_mg_opts o;
    double* ainv = nullptr;
    cudaGraphExec_t gexec[5] = {};  // V+check, F+check, F, first pair+check, rest of V
    long long gnodes[5] = {};
    bool graph_failed = false;
    cudaGraphExec_t gloop[2] = {};  // device-resident solve, V-only / F first
    long long loop_nodes[2][2] = {};   // launches in prologue+epilogue / in one loop body
    bool loop_failed = false;
    LoopCtl* lctl = nullptr;
    LoopHost* lhost = nullptr;
    LoopHost* lhost_dev = nullptr;
    std::vector<double> lmax;   // SF_SMOOTH_CHEBY: lambda_max(D^-1 A) per level
    int coarse_l0 = -1;         // first level whose V-cycle runs as one cluster launch (-1: none)
    // Field -> buffer mapping of every level when the cached graphs were
    // captured: a graph names device pointers, so a public call that swaps
    // U/TMP (sf_smooth_gsrb, sf_smooth_chebyshev, ...) between solves makes
    // every cached graph stale; they are then destroyed and re-captured.
    std::vector<double*> gsig;
    // sf_solve_stream: staging buffers, copy streams and events kept across
    // calls (a per-call 2 x 1 GiB cudaMalloc/cudaFree cost more than it hid)
    double *stf = nullptr, *stu = nullptr;
    size_t st_bytes = 0;
    cudaStream_t sin = nullptr, sout = nullptr;
    cudaEvent_t sev[4] = {};      // f_ready, f_free, u_ready, u_free
    double stats[4] = {};         // last call: mean H2D, solve, D2H ms; wall ms per rhs
};

static std::vector<double*> field_map(const sf_mg* m) {
    std::vector<double*> v;
    for (const sf_level* l : m->lv)
        for (const SfPart& P : l->parts) v.insert(v.end(), P.f, P.f + SF_NFIELDS);
    return v;
}

// Drop every cached graph whose device pointers no longer match the levels'
// field mapping; remember the mapping the next captures will see.
static void refresh_graph_map(sf_mg* m) {
    std::vector<double*> cur = field_map(m);
    if (cur == m->gsig) return;
    if (!m->lv.empty()) cudaStreamSynchronize(m->lv[0]->stream);
    for (auto& g : m->gexec)
        if (g) {
            cudaGraphExecDestroy(g);
            g = nullptr;
        }
    for (auto& g : m->gloop)
        if (g) {
            cudaGraphExecDestroy(g);
            g = nullptr;
        }
    m->gsig.swap(cur);
}

// NEXT-3 reading R-16: Chebyshev interval [hi/8, hi], hi = 1.05 lambda_max(D^-1 A)
// (power iteration, 30 steps from the fixed start vector, at setup)
static const int CHEBY_POWER_ITERS = 30;
static void cheby_interval(double lmax, double* lo, double* hi) {
    *hi = 1.05 * lmax;
    *lo = *hi / 8.0;
}

extern "C" void sf_mg_opts_default(sf_mg_opts* o) {
    if (!o) return;
    o->pre_pairs = 2;
    o->post_pairs = 2;
    o->vcycle_interp = SF_INTERP_P0;
    o->fcycle_interp = SF_INTERP_PL;
    o->agglom_min_planes = 16;
    o->max_cycles = 50;
    o->use_graph = 1;
    o->smoother = SF_SMOOTH_AUTO;
    o->rtol = 1e-10;
    o->cheby_degree = 2;
}

static sf_status destroy_levels(sf_mg* m) {
    for (size_t l = 0; l < m->lv.size(); l++)
        if (m->own[l]) sf_level_destroy(m->lv[l]);
    m->lv.clear();
    return SF_OK;
}

extern "C" sf_status sf_mg_destroy(sf_mg* m) {
    if (!m) return SF_OK;
    if (!m->lv.empty()) cudaStreamSynchronize(m->lv[0]->stream);
    for (auto& g : m->gexec)
        if (g) cudaGraphExecDestroy(g);
    for (auto& g : m->gloop)
        if (g) cudaGraphExecDestroy(g);
    if (m->lctl) cudaFree(m->lctl);
    if (m->lhost) cudaFreeHost(m->lhost);
    if (m->sin) cudaStreamSynchronize(m->sin);
    if (m->sout) cudaStreamSynchronize(m->sout);
    for (cudaEvent_t e : m->sev)
        if (e) cudaEventDestroy(e);
    if (m->sin) cudaStreamDestroy(m->sin);
    if (m->sout) cudaStreamDestroy(m->sout);
    cudaFree(m->stf);
    cudaFree(m->stu);
    if (m->ainv) cudaFree(m->ainv);
    destroy_levels(m);
    delete m;
    return SF_OK;
}

// Hierarchy plan shared by sf_mg_create and the host-side tests.
struct LevelPlan {
    int nx, ny, nz;
    bool distributed;
};

static sf_status plan_levels(int gnx, int gny, int gnz, int nparts, int amin,
                             std::vector<LevelPlan>& out) {
    out.clear();
    if (gnx < 2 || gny < 2 || gnz < 2 || nparts < 1 || amin < 2)
        return sf_fail(SF_ERR_INVALID, "bad plan arguments");
    if (gnz % nparts) return sf_fail(SF_ERR_SHAPE, "gnz=%d not divisible by %d parts", gnz, nparts);
    out.push_back({gnx, gny, gnz, nparts > 1});
    for (;;) {
        const LevelPlan F = out.back();
        int mn = std::min(F.nx, std::min(F.ny, F.nz));
        if (mn <= 2 || (F.nx | F.ny | F.nz) & 1) break;
        int cx = F.nx / 2, cy = F.ny / 2, cz = F.nz / 2;
        if (F.distributed && (F.nz / nparts) % 2 != 0)
            return sf_fail(SF_ERR_SHAPE, "odd planes per part (%d) cannot coarsen", F.nz / nparts);
        bool last = std::min(cx, std::min(cy, cz)) <= 2 || ((cx | cy | cz) & 1);
        bool dist = F.distributed && !last && (F.nz / nparts) / 2 >= amin;
        out.push_back({cx, cy, cz, dist});
    }
    const LevelPlan B = out.back();
    if (B.distributed || (long)B.nx * B.ny * B.nz > 64)
        return sf_fail(SF_ERR_SHAPE, "coarsest level %dx%dx%d is not a <=64-cell replicated box",
                       B.nx, B.ny, B.nz);
    return SF_OK;
}

extern "C" sf_status sf_mg_plan(int gnx, int gny, int gnz, int nparts, int amin, int max_levels,
                                int* nlevels, int* dims, int* distributed) {
    std::vector<LevelPlan> P;
    SF_TRY(plan_levels(gnx, gny, gnz, nparts, amin, P));
    if (nlevels) *nlevels = (int)P.size();
    for (int l = 0; l < (int)P.size() && l < max_levels; l++) {
        if (dims) {
            dims[3 * l] = P[l].nx; dims[3 * l + 1] = P[l].ny; dims[3 * l + 2] = P[l].nz;
        }
        if (distributed) distributed[l] = P[l].distributed ? 1 : 0;
    }
    return SF_OK;
}

// First level l >= 1 from which V(l) runs as ONE single-CTA launch with the
// iterates in shared memory (coarse.cu): every level from l down is
// single-part, l has at most 16^3 cells and the chain fits the kernel's
// arrays; GSRB smoothers with P0 in the V-cycle only (what the kernel
// implements).  SF_COARSE_KERNEL=0 keeps the per-phase launches.
static int plan_coarse(sf_mg* m) {
    const char* e = getenv("SF_COARSE_KERNEL");
    if (e && atoi(e) == 0) return -1;
    if (m->o.smoother == SF_SMOOTH_CHEBY || m->o.vcycle_interp != SF_INTERP_P0) return -1;
    const int nl = (int)m->lv.size();
    for (int l = 1; l < nl - 1; l++)
        if (coarse_vcycle_fits(&m->lv[l], nl - l)) return l;
    return -1;
}

extern "C" sf_status sf_mg_create(sf_mg** out, sf_level* fine, double a, double b,
                                  const sf_mg_opts* opts) {
    if (!out || !fine) return sf_fail(SF_ERR_INVALID, "NULL argument");
    *out = nullptr;
    sf_mg* m = new sf_mg();
    m->a = a; m->b = b;
    if (opts) m->o = *opts; else sf_mg_opts_default(&m->o);
    if (m->o.pre_pairs < 0 || m->o.post_pairs < 0 || m->o.max_cycles < 1 ||
        m->o.agglom_min_planes < 2 ||
        (m->o.smoother == SF_SMOOTH_CHEBY && (m->o.cheby_degree < 1 || (fine->gnx & 1)))) {
        delete m;
        return sf_fail(SF_ERR_INVALID, "bad mg options");
    }
    std::vector<LevelPlan> plan;
    {
        sf_status ps = plan_levels(fine->gnx, fine->gny, fine->gnz, fine->nparts,
                                   m->o.agglom_min_planes, plan);
        if (ps != SF_OK) {
            delete m;
            return ps;
        }
    }
    m->lv.push_back(fine);
    m->own.push_back(false);
    for (size_t l = 1; l < plan.size(); l++) {
        sf_level* F = m->lv.back();
        const LevelPlan& P = plan[l];
        sf_level* C = nullptr;
        sf_status s = sf_level_create(&C, P.nx, P.ny, P.nz, 2.0 * F->h,
                                      P.distributed ? F->comm : nullptr, F->stream, nullptr, 0);
        if (s != SF_OK) {
            sf_mg_destroy(m);
            return s;
        }
        if (!P.distributed) {
            C->rep_comm = F->comm ? F->comm : F->rep_comm;
            s = sf_ipc_register(C, C->rep_comm);   // kind-2/3 comm: collective
            if (s != SF_OK) {
                m->lv.push_back(C);
                m->own.push_back(true);
                sf_mg_destroy(m);
                return s;
            }
        }
        m->lv.push_back(C);
        m->own.push_back(true);
    }
    sf_level* B = m->lv.back();
    // operator on every level: restrict coefficients (A7), rebuild Dinv (A4)
    sf_status s = sf_rebuild_operator(fine, a, b);
    for (size_t l = 1; l < m->lv.size() && s == SF_OK; l++) {
        sf_level* F = m->lv[l - 1];
        sf_level* C = m->lv[l];
        s = k_restrict(C, SF_ALPHA, F, SF_ALPHA, SF_RESTRICT_CELL);
        if (s == SF_OK) s = k_restrict(C, SF_BETA_I, F, SF_BETA_I, SF_RESTRICT_FACE_I);
        if (s == SF_OK) s = k_restrict(C, SF_BETA_J, F, SF_BETA_J, SF_RESTRICT_FACE_J);
        if (s == SF_OK) s = k_restrict(C, SF_BETA_K, F, SF_BETA_K, SF_RESTRICT_FACE_K);
        if (s == SF_OK) s = sf_rebuild_operator(C, a, b);
    }
    if (s == SF_OK) {
        int n = B->gnx * B->gny * B->gnz;
        cudaError_t e = cudaMalloc(&m->ainv, (size_t)n * n * sizeof(double));
        if (e != cudaSuccess) s = sf_fail(SF_ERR_OOM, "bottom inverse: %s", cudaGetErrorString(e));
    }
    if (s == SF_OK) s = k_bottom_setup(B, a, b, m->ainv);
    if (s == SF_OK && m->o.smoother == SF_SMOOTH_CHEBY) {
        for (size_t l = 0; l + 1 < m->lv.size() && s == SF_OK; l++) {
            double lm = 0.0;
            s = sf_lambda_max_impl(m->lv[l], SF_TMP, a, b, CHEBY_POWER_ITERS, true, &lm);
            m->lmax.push_back(lm);
        }
        if (s == SF_OK) s = k_zero(fine, SF_TMP);
    }
    if (s == SF_OK) {
        cudaError_t e = cudaStreamSynchronize(fine->stream);
        if (e != cudaSuccess) s = sf_fail(SF_ERR_CUDA, "mg setup: %s", cudaGetErrorString(e));
    }
    if (s == SF_OK) m->coarse_l0 = plan_coarse(m);
    // partial arrays of the fused pair + residual + restriction, allocated here
    // (outside any graph capture) for every level pair that will use it
    for (size_t l = 0; s == SF_OK && l + 1 < m->lv.size(); l++)
        if ((m->coarse_l0 < 1 || (int)l < m->coarse_l0) && gsrb_rr_supported(m->lv[l], m->lv[l + 1]))
            s = sf_rrf_prepare(m->lv[l], m->lv[l + 1]);
    if (s != SF_OK) {
        sf_mg_destroy(m);
        return s;
    }
    *out = m;
    return SF_OK;
}

extern "C" sf_status sf_mg_num_levels(const sf_mg* m, int* n) {
    if (!m || !n) return sf_fail(SF_ERR_INVALID, "NULL argument");
    *n = (int)m->lv.size();
    return SF_OK;
}

extern "C" sf_status sf_mg_level(sf_mg* m, int l, sf_level** out) {
    if (!m || !out) return sf_fail(SF_ERR_INVALID, "NULL argument");
    if (l < 0 || l >= (int)m->lv.size()) return sf_fail(SF_ERR_INVALID, "bad level %d", l);
    *out = m->lv[l];
    return SF_OK;
}

static sf_status smooth(sf_mg* m, sf_level* L, int pairs) {
    if (m->o.smoother == SF_SMOOTH_CHEBY) {
        if (pairs == 0) return SF_OK;
        size_t l = 0;
        while (m->lv[l] != L) l++;
        double lo, hi;
        cheby_interval(m->lmax[l], &lo, &hi);
        return sf_chebyshev_impl(L, SF_U, SF_F, m->a, m->b, pairs * m->o.cheby_degree, lo, hi);
    }
    return sf_smooth_gsrb(L, SF_U, SF_F, m->a, m->b, pairs, m->o.smoother);
}

static bool fused_check_ok(const sf_mg* m);

// The finest level's last post-smoothing pair of a cycle also reduces the black
// part of max|F - A U| of its output into dscratch (BRES); the next cycle's
// first pair adds the red part of the same iterate (fused check, below).
// zeroed: an earlier pair of the cycle already reset dscratch[0] (SF_RM_ZERO).
static sf_status bres_pair(sf_mg* m, sf_level* L, bool zeroed = false) {
    SF_TRY(sf_halo(L, SF_F, 1));
    SF_TRY(k_gsrb_pair_halo(L, SF_U, SF_TMP, SF_F, m->a, m->b, L->dscratch, nullptr, 0,
                            zeroed ? SF_RM_OUTPUT_BLACK_ZEROED : SF_RM_OUTPUT_BLACK));
    sf_swap_fields(L, SF_U, SF_TMP);
    return SF_OK;
}

// V(l): smooth, residual, restrict, zero e_{l+1}, V(l+1), e_l += P0 e_{l+1}, smooth.
// skip_first: the first pre-smoothing pair was already run (fused check, below).
// u_zero: U of level l is zero on entry (the V-cycle recursion zeroed it, or
// leaves that to the coarse-level launch, which then does not read it)
// trig: the launch after this V(l) may start early (the P0-fused pair above a
// coarse cluster V-cycle)
static sf_status vcyc(sf_mg* m, int l, bool skip_first = false, bool u_zero = false,
                      bool trig = false) {
    const bool bres = l == 0 && fused_check_ok(m);   // last post pair reduces the black residual
    sf_level* L = m->lv[l];
    NvtxRange nv("sf V(l=%d) %dx%dx%d", l, L->gnx, L->gny, L->gnz);
    if (l == (int)m->lv.size() - 1) return k_bottom_solve(L, SF_U, SF_F, m->ainv);
    if (m->coarse_l0 >= 1 && l >= m->coarse_l0)   // the whole V(l) in one launch
        return k_coarse_vcycle(&m->lv[l], (int)m->lv.size() - l, m->a, m->b, m->ainv,
                               m->o.pre_pairs, m->o.post_pairs, u_zero, trig);
    sf_level* C = m->lv[l + 1];
    const int pre = m->o.pre_pairs - (skip_first ? 1 : 0);
    if (pre >= 1 && (m->o.smoother == SF_SMOOTH_AUTO || m->o.smoother == SF_SMOOTH_FUSED) &&
        gsrb_fused_supported(L) && gsrb_rr_supported(L, C) && sf_rrf_usable(L, C)) {
        // the last pre-smoothing pair also forms the residual and restricts it
        // (A5 + A6 + A7 in one pass; gsrb_rr.cu)
        SF_TRY(smooth(m, L, pre - 1));
        // the coarse cluster V-cycle follows directly: it may launch early
        const bool next_coarse = m->coarse_l0 >= 1 && l + 1 == m->coarse_l0 &&
                                 l + 1 < (int)m->lv.size() - 1;
        SF_TRY(k_gsrb_pair_rr(L, SF_U, SF_TMP, SF_F, m->a, m->b, C, SF_F, next_coarse));
        sf_swap_fields(L, SF_U, SF_TMP);
    } else {
        SF_TRY(smooth(m, L, pre));
        if (pair_ok(L)) {  // residual never stored: A6 + A7 in one pass
            // the coarse cluster V-cycle follows directly: it may launch early
            const bool next_coarse = m->coarse_l0 >= 1 && l + 1 == m->coarse_l0 &&
                                     l + 1 < (int)m->lv.size() - 1;
            SF_TRY(k_residual_restrict(L, SF_U, SF_F, m->a, m->b, C, SF_F, next_coarse));
        } else {
            SF_TRY(k_residual(L, SF_R, SF_U, SF_F, m->a, m->b));
            SF_TRY(k_restrict(C, SF_F, L, SF_R, SF_RESTRICT_CELL));
        }
    }
    const bool cz = m->coarse_l0 >= 1 && l + 1 >= m->coarse_l0 && l + 1 < (int)m->lv.size() - 1;
    if (!cz) SF_TRY(k_zero(C, SF_U));   // the coarse-level launch starts from zero itself
    // P0-fused pair right after a coarse cluster V-cycle: it may start under it
    // (its TMA prologue reads only operands older than that launch)
    const bool p0_pair = m->o.vcycle_interp == SF_INTERP_P0 && m->o.post_pairs >= 1 &&
                         (m->o.smoother == SF_SMOOTH_AUTO || m->o.smoother == SF_SMOOTH_FUSED) &&
                         gsrb_fused_supported(L);
    const bool early = p0_pair && cz && L->nparts == 1 && C->nparts == 1 &&
                       !(bres && m->o.post_pairs == 1);
    SF_TRY(vcyc(m, l + 1, false, cz, early));
    if (p0_pair) {
        // e_l += P0 e_{l+1} fused into the first post-smoothing pair (A8 + A5)
        SF_TRY(sf_halo(C, SF_U, 1));
        SF_TRY(sf_halo(L, SF_F, 1));
        // (a later BRES pair: this one resets its scalar, saving a launch)
        const bool last = bres && m->o.post_pairs == 1;
        L->pdl_early = early ? 1 : 0;
        SF_TRY(k_gsrb_pair_halo(L, SF_U, SF_TMP, SF_F, m->a, m->b, bres ? L->dscratch : nullptr, C,
                                SF_U, last ? SF_RM_OUTPUT_BLACK : bres ? SF_RM_ZERO : SF_RM_NONE));
        sf_swap_fields(L, SF_U, SF_TMP);
        if (bres && m->o.post_pairs >= 2) {
            SF_TRY(smooth(m, L, m->o.post_pairs - 2));
            return bres_pair(m, L, true);
        }
        SF_TRY(smooth(m, L, m->o.post_pairs - 1));
        return SF_OK;
    }
    SF_TRY(k_interp(L, SF_U, 1.0, C, SF_U, m->o.vcycle_interp));
    if (bres) {
        SF_TRY(smooth(m, L, m->o.post_pairs - 1));
        return bres_pair(m, L);
    }
    SF_TRY(smooth(m, L, m->o.post_pairs));
    return SF_OK;
}

static sf_status fcyc(sf_mg* m) {
    int nl = (int)m->lv.size();
    NvtxRange nv("sf F-cycle %d levels", nl);
    for (int l = 1; l < nl; l++)
        SF_TRY(k_restrict(m->lv[l], SF_F, m->lv[l - 1], SF_F, SF_RESTRICT_CELL));
    SF_TRY(k_bottom_solve(m->lv[nl - 1], SF_U, SF_F, m->ainv));
    for (int l = nl - 2; l >= 0; l--) {
        SF_TRY(k_interp(m->lv[l], SF_U, 0.0, m->lv[l + 1], SF_U, m->o.fcycle_interp));
        SF_TRY(vcyc(m, l));
    }
    return SF_OK;
}

static sf_status to_host(sf_level* L) { return sf_scalar_to_host(L, L->dscratch, 0); }

// separate convergence check: max|F - A U| of the finest level (A6 + A10)
static sf_status check(sf_mg* m) {
    sf_level* L = m->lv[0];
    if (pair_ok(L)) {  // max|f - Au| reduced in the residual pass, nothing stored
        SF_TRY(k_residual_pair(L, -1, SF_U, SF_F, m->a, m->b, L->dscratch));
        if (L->comm && L->comm->kind != 0 && L->nparts > 1)
            SF_TRY(sf_allreduce_scalar(L, L->comm, L->dscratch, 0));
    } else {
        SF_TRY(k_residual(L, SF_R, SF_U, SF_F, m->a, m->b));
        SF_TRY(sf_norm_async(L, SF_R, SF_NORM_MAX, L->dscratch));
    }
    return to_host(L);
}

// The convergence check rides in the colour-fused pairs that stream every
// operand anyway: max|F - A U| of the iterate after a cycle is the max of its
// black part, reduced by the cycle's last post-smoothing pair right after each
// black update (BRES: the red neighbours are final then), and its red part,
// reduced by the next cycle's first pre-smoothing pair from its INPUT while it
// writes the smoothed iterate to TMP.  If that says "converged", U (the
// previous cycle's result) is untouched.
static bool fused_check_ok(const sf_mg* m) {
    return m->lv.size() > 1 && m->o.pre_pairs >= 1 && m->o.post_pairs >= 1 &&
           (m->o.smoother == SF_SMOOTH_AUTO || m->o.smoother == SF_SMOOTH_FUSED) &&
           gsrb_fused_supported(m->lv[0]) && (m->o.pre_pairs + m->o.post_pairs) % 2 == 0;
}

static sf_status first_pair_check(sf_mg* m) {
    sf_level* L = m->lv[0];
    SF_TRY(sf_halo(L, SF_F, 1));
    SF_TRY(k_gsrb_pair_halo(L, SF_U, SF_TMP, SF_F, m->a, m->b, L->dscratch, nullptr, 0,
                            SF_RM_INPUT_RED));
    sf_swap_fields(L, SF_U, SF_TMP);
    if (L->comm && L->comm->kind != 0 && L->nparts > 1)
        SF_TRY(sf_allreduce_scalar(L, L->comm, L->dscratch, 0));
    return to_host(L);
}

static bool graphs_allowed(const sf_mg* m) {
    if (!m->o.use_graph || m->graph_failed) return false;
    if (m->lv[0]->stream == nullptr) return false;  // legacy stream cannot be captured
    if (m->lv[0]->comm && m->lv[0]->comm->kind == 2) return false;  // host-synchronised halos
    for (const sf_level* l : m->lv)   // agglomeration through the host (kind 2) likewise
        if (l->rep_comm && l->rep_comm->kind == 2) return false;
    // the fused smoother swaps U/TMP per pair; only an even count per captured
    // sequence leaves the host-side mapping unchanged for replays
    if (m->o.smoother == SF_SMOOTH_CHEBY)   // an n-step application ends with swap(U, [U,R,TMP][n%3]):
        return (m->o.pre_pairs * m->o.cheby_degree) % 3 ==   // equal pre/post transpositions cancel
               (m->o.post_pairs * m->o.cheby_degree) % 3;
    return (m->o.pre_pairs % 2 == 0 && m->o.post_pairs % 2 == 0) ||
           m->o.smoother == SF_SMOOTH_COLOUR;
}

enum { G_VCHECK = 0, G_FCHECK = 1, G_F = 2, G_FIRST = 3, G_REST = 4 };

static sf_status body_of(sf_mg* m, int kind) {
    switch (kind) {
        case G_VCHECK: SF_TRY(vcyc(m, 0)); return check(m);
        case G_FCHECK: SF_TRY(fcyc(m)); return check(m);
        case G_F: return fcyc(m);
        case G_FIRST: return first_pair_check(m);
        default: return vcyc(m, 0, true);
    }
}

// Capture cycle piece `kind` into a graph.  Any failure during capture (e.g. a
// collective that refuses capture) leaves graphs off for this hierarchy and
// restores every level's field mapping, so the caller falls back to eager
// enqueueing; only errors of the eager path are reported.
static sf_status capture(sf_mg* m, int kind) {
    sf_level* L = m->lv[0];
    std::vector<std::vector<SfPart>> saved;
    for (sf_level* lv : m->lv) saved.push_back(lv->parts);
    long long before, after;
    sf_launch_count(&before, 0);
    auto give_up = [&]() {
        cudaGetLastError();
        for (size_t i = 0; i < m->lv.size(); i++) m->lv[i]->parts = saved[i];
        m->graph_failed = true;
        for (auto& g : m->gexec)
            if (g) {
                cudaGraphExecDestroy(g);
                g = nullptr;
            }
    };
    if (cudaStreamBeginCapture(L->stream, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
        give_up();
        return SF_OK;
    }
    sf_status s = body_of(m, kind);
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(L->stream, &g);
    sf_launch_count(&after, 0);
    sf_count_launch(-(after - before));  // captured, not launched
    if (s != SF_OK || e != cudaSuccess || !g) {
        if (g) cudaGraphDestroy(g);
        give_up();
        return SF_OK;
    }
    e = cudaGraphInstantiate(&m->gexec[kind], g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        m->gexec[kind] = nullptr;
        give_up();
        return SF_OK;
    }
    m->gnodes[kind] = after - before;
    return SF_OK;
}

// enqueue cycle piece `kind` (graph replay when possible)
static sf_status run(sf_mg* m, int kind) {
    sf_level* L = m->lv[0];
    if (graphs_allowed(m)) refresh_graph_map(m);
    if (graphs_allowed(m) && !m->gexec[kind]) {
        if (kind == G_FIRST || kind == G_REST) {
            // capture both halves back to back: together they hold an even
            // number of U/TMP swaps, so the host mapping is restored
            std::vector<std::vector<SfPart>> saved;
            for (sf_level* lv : m->lv) saved.push_back(lv->parts);
            SF_TRY(capture(m, G_FIRST));
            if (!m->graph_failed) SF_TRY(capture(m, G_REST));
            if (m->graph_failed)
                for (size_t i = 0; i < m->lv.size(); i++) m->lv[i]->parts = saved[i];
        } else {
            SF_TRY(capture(m, kind));
        }
    }
    if (graphs_allowed(m) && m->gexec[kind]) {
        SF_CUDA(cudaGraphLaunch(m->gexec[kind], L->stream));
        sf_count_launch(m->gnodes[kind]);
        return SF_OK;
    }
    return body_of(m, kind);
}

// ---------------------------------------------------------------- device loop
static __global__ void loop_init_kernel(LoopCtl* c, const LoopHost* h, const double* fn, int done0) { pdl_wait();
    c->rtol = h->rtol;
    c->max_cycles = h->max_cycles;
    c->fn = *fn;
    c->done = done0;
    c->status = LS_RUN;
    c->nbody = 0;
}

// After a first pair's fused check: rmax = max|F - A U| of the iterate after
// `done` cycles (the same decision as sf_solve's host loop, made on the device).
static __global__ void loop_check_kernel(LoopCtl* c, const double* rmax, cudaGraphConditionalHandle h) { pdl_wait();
    const int d = c->done;
    unsigned cont = 1;
    const double fn = c->fn;
    if (!(fn == fn) || isinf(fn)) {
        c->status = LS_RHS_NAN;
        cont = 0;
    } else if (fn == 0.0) {
        c->status = LS_ZERO;
        cont = 0;
    } else if (d >= 1) {
        const double rel = *rmax / fn;
        if (d <= SF_LOOP_HIST) c->hist[d - 1] = rel;
        if (!(rel == rel) || isinf(rel)) {
            c->status = LS_NUMERIC;
            cont = 0;
        } else if (rel < c->rtol) {
            c->status = LS_CONVERGED;
            cont = 0;
        } else if (d >= c->max_cycles) {
            c->status = LS_NOT_CONVERGED;
            cont = 0;
        }
    }
    if (cont) {   // the loop body completes cycle d + 1
        c->done = d + 1;
        c->nbody++;
    }
    cudaGraphSetConditional(h, cont);
}

// results -> mapped host memory (posted writes: nothing queues behind bulk copies)
static __global__ void loop_publish_kernel(const LoopCtl* c, LoopHost* h) { pdl_wait();
    const int n = min(c->done, SF_LOOP_HIST);
    for (int i = threadIdx.x; i < n; i += blockDim.x) h->hist[i] = c->hist[i];
    if (threadIdx.x == 0) {
        h->done = c->done;
        h->status = c->status;
        h->nbody = c->nbody;
    }
}

static sf_status first_pair(sf_mg* m) {   // first_pair_check without the host copy
    sf_level* L = m->lv[0];
    SF_TRY(sf_halo(L, SF_F, 1));
    SF_TRY(k_gsrb_pair_halo(L, SF_U, SF_TMP, SF_F, m->a, m->b, L->dscratch, nullptr, 0,
                            SF_RM_INPUT_RED));
    sf_swap_fields(L, SF_U, SF_TMP);
    if (L->comm && L->comm->kind != 0 && L->nparts > 1)
        SF_TRY(sf_allreduce_scalar(L, L->comm, L->dscratch, 0));
    return SF_OK;
}

// Kernel nodes inside a graph with conditional nodes are invisible to Nsight
// Compute ("not supported for profiling"), and compute-sanitizer's racecheck /
// synccheck abort the conditional graph ("unspecified launch failure"; memcheck
// and initcheck run it clean), so under a profiler's or sanitizer's injection
// (the variables those tools set in the target process) the solve uses the
// host loop: the same kernels in the same order, one graph per cycle half.
// SF_DEVICE_LOOP=0 forces the host loop, =1 the device loop even under a tool.
static bool device_loop_env() {
    static const bool on = [] {
        const char* e = getenv("SF_DEVICE_LOOP");
        if (e) return atoi(e) != 0;
        return !getenv("CUDA_INJECTION64_PATH") && !getenv("NV_COMPUTE_PROFILER_PERFWORKS_DIR") &&
               !getenv("NV_NSIGHT_INJECTION_TRANSPORT_TYPE") &&
               !getenv("NV_SANITIZER_INJECTION_TRANSPORT_TYPE");
    }();
    return on;
}

static bool loop_allowed(const sf_mg* m) {
    return device_loop_env() && !m->loop_failed && graphs_allowed(m) && fused_check_ok(m) &&
           !(m->lv[0]->comm && m->lv[0]->comm->kind == 1);   // NCCL: host-side proxies
}

// Build the solve graph:
//   [max|F| -> fn] [init] [F-cycle]? [first pair + check] WHILE(cont) { [rest of the
//   V-cycle] [first pair of the next + check] } [publish]
// The loop body holds 4 U/TMP swaps on the finest level (even on every level),
// so every iteration reads the buffers the capture saw; the iterate a stop
// leaves behind is the input of the last first pair, i.e. the buffer U named
// before the solve.  Any failure leaves the device loop off for this hierarchy.
static sf_status build_loop(sf_mg* m, int fc) {
    sf_level* L = m->lv[0];
    cudaStream_t st = L->stream;
    std::vector<std::vector<SfPart>> saved;
    for (sf_level* lv : m->lv) saved.push_back(lv->parts);
    long long c0, c1, c2, c3;
    cudaGraph_t g = nullptr, body = nullptr;   // body: owned by the WHILE node
    cudaGraphExec_t ge = nullptr;
    bool ok = true;
    auto fail = [&]() {
        cudaStreamCaptureStatus cs;
        if (cudaStreamIsCapturing(st, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone) {
            cudaGraph_t junk = nullptr;
            cudaStreamEndCapture(st, &junk);
            if (junk && junk != g && junk != body) cudaGraphDestroy(junk);
        }
        cudaGetLastError();
        ok = false;
    };
    if (!m->lctl) {
        if (cudaMalloc(&m->lctl, sizeof(LoopCtl)) != cudaSuccess ||
            cudaHostAlloc(&m->lhost, sizeof(LoopHost), cudaHostAllocMapped) != cudaSuccess ||
            cudaHostGetDevicePointer(&m->lhost_dev, m->lhost, 0) != cudaSuccess) {
            cudaGetLastError();
            m->loop_failed = true;
            return SF_OK;
        }
    }
    sf_launch_count(&c0, 0);
    cudaGraphConditionalHandle h = 0;
    cudaGraphNode_t last = nullptr, wnode = nullptr;
    if (cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal) != cudaSuccess) fail();
    if (ok && sf_norm_async(L, SF_F, SF_NORM_MAX, L->dscratch + 2) != SF_OK) fail();
    if (ok) {
        sf_launch(loop_init_kernel, 1, 1, 0, st, m->lctl, m->lhost_dev, L->dscratch + 2, fc ? 1 : 0);
        SF_LAUNCHED();
    }
    if (ok && fc && fcyc(m) != SF_OK) fail();
    if (ok && first_pair(m) != SF_OK) fail();
    if (ok) {
        cudaStreamCaptureStatus cs;
        cudaGraph_t cg = nullptr;
        if (cudaStreamGetCaptureInfo(st, &cs, nullptr, &cg, nullptr, nullptr) != cudaSuccess ||
            cs != cudaStreamCaptureStatusActive ||
            cudaGraphConditionalHandleCreate(&h, cg, 0, cudaGraphCondAssignDefault) != cudaSuccess)
            fail();
    }
    if (ok) {
        sf_launch(loop_check_kernel, 1, 1, 0, st, m->lctl, L->dscratch, h);
        SF_LAUNCHED();
        cudaStreamCaptureStatus cs;
        const cudaGraphNode_t* deps = nullptr;
        size_t nd = 0;
        if (cudaStreamGetCaptureInfo(st, &cs, nullptr, nullptr, &deps, &nd) != cudaSuccess || nd != 1)
            fail();
        else
            last = deps[0];
    }
    if (ok && cudaStreamEndCapture(st, &g) != cudaSuccess) fail();
    sf_launch_count(&c1, 0);
    if (ok) {
        cudaGraphNodeParams p = {};
        p.type = cudaGraphNodeTypeConditional;
        p.conditional.handle = h;
        p.conditional.type = cudaGraphCondTypeWhile;
        p.conditional.size = 1;
        if (cudaGraphAddNode(&wnode, g, &last, 1, &p) != cudaSuccess) fail();
        else body = p.conditional.phGraph_out[0];
    }
    if (ok && cudaStreamBeginCaptureToGraph(st, body, nullptr, nullptr, 0,
                                            cudaStreamCaptureModeThreadLocal) != cudaSuccess)
        fail();
    if (ok && getenv("SF_TEST_LOOP_FAIL")) fail();   // tests: a capture failing mid-body
    if (ok && vcyc(m, 0, true) != SF_OK) fail();
    if (ok && first_pair(m) != SF_OK) fail();
    if (ok) {
        sf_launch(loop_check_kernel, 1, 1, 0, st, m->lctl, L->dscratch, h);
        SF_LAUNCHED();
        cudaGraph_t bo = nullptr;
        if (cudaStreamEndCapture(st, &bo) != cudaSuccess) fail();
    }
    sf_launch_count(&c2, 0);
    if (ok && cudaStreamBeginCaptureToGraph(st, g, &wnode, nullptr, 1,
                                            cudaStreamCaptureModeThreadLocal) != cudaSuccess)
        fail();
    if (ok) {
        sf_launch(loop_publish_kernel, 1, 32, 0, st, m->lctl, m->lhost_dev);
        SF_LAUNCHED();
        cudaGraph_t go = nullptr;
        if (cudaStreamEndCapture(st, &go) != cudaSuccess) fail();
    }
    sf_launch_count(&c3, 0);
    sf_count_launch(-(c3 - c0));   // captured, not launched
    for (size_t i = 0; i < m->lv.size(); i++) m->lv[i]->parts = saved[i];
    if (ok && cudaGraphInstantiate(&ge, g, 0) != cudaSuccess) fail();
    if (g) cudaGraphDestroy(g);
    if (!ok) {
        if (ge) cudaGraphExecDestroy(ge);
        m->loop_failed = true;
        return SF_OK;
    }
    m->gloop[fc] = ge;
    m->loop_nodes[fc][0] = (c1 - c0) + (c3 - c2);
    m->loop_nodes[fc][1] = c2 - c1;
    return SF_OK;
}

// One solve through the device loop.  *handled = false: not available, use the
// host loop.
static sf_status solve_loop(sf_mg* m, int fc, double rtol, int max_cycles, int* cycles,
                            double* hist, bool* handled) {
    *handled = false;
    if (max_cycles > SF_LOOP_HIST || !loop_allowed(m)) return SF_OK;
    refresh_graph_map(m);
    if (!m->gloop[fc]) SF_TRY(build_loop(m, fc));
    if (!m->gloop[fc]) return SF_OK;
    sf_level* L = m->lv[0];
    m->lhost->rtol = rtol;
    m->lhost->max_cycles = max_cycles;
    m->lhost->done = -1;
    SF_CUDA(cudaGraphLaunch(m->gloop[fc], L->stream));
    SF_TRY(sf_stream_sync(L));
    *handled = true;
    const LoopHost& r = *m->lhost;
    if (r.done < 0) return sf_fail(SF_ERR_CUDA, "device solve loop did not publish");
    sf_count_launch(m->loop_nodes[fc][0] + m->loop_nodes[fc][1] * r.nbody);
    const int n = std::min(r.done, SF_LOOP_HIST);
    if (r.status == LS_RHS_NAN) {
        if (cycles) *cycles = 0;
        return sf_fail(SF_ERR_NUMERIC, "rhs has NaN/Inf");
    }
    if (r.status == LS_ZERO) {
        if (cycles) *cycles = 0;
        SF_TRY(k_zero(L, SF_U));
        return sf_sync(L);
    }
    if (cycles) *cycles = r.done;
    if (hist)
        for (int i = 0; i < n; i++) hist[i] = r.hist[i];
    if (r.status == LS_NUMERIC) return sf_fail(SF_ERR_NUMERIC, "residual is NaN/Inf");
    if (r.status == LS_NOT_CONVERGED)
        return sf_fail(SF_ERR_NOT_CONVERGED, "no convergence to %g in %d cycles", rtol, max_cycles);
    return SF_OK;
}

extern "C" sf_status sf_vcycle(sf_mg* m, int l) {
    if (!m) return sf_fail(SF_ERR_INVALID, "NULL mg");
    if (l < 0 || l >= (int)m->lv.size()) return sf_fail(SF_ERR_INVALID, "bad level %d", l);
    return vcyc(m, l);
}

extern "C" sf_status sf_fcycle(sf_mg* m) {
    if (!m) return sf_fail(SF_ERR_INVALID, "NULL mg");
    return fcyc(m);
}

extern "C" sf_status sf_solve(sf_mg* m, int fcycle, double rtol, int max_cycles, int* cycles,
                              double* hist) {
    if (!m) return sf_fail(SF_ERR_INVALID, "NULL mg");
    NvtxRange nv("sf solve fcycle=%d max_cycles=%d", fcycle, max_cycles);
    // hist holds max_cycles entries (sf.h): a silent default cap would overrun it
    if (max_cycles < 1) return sf_fail(SF_ERR_INVALID, "max_cycles must be >= 1");
    if (!(rtol > 0)) rtol = m->o.rtol;
    sf_level* L = m->lv[0];
    {
        bool handled = false;
        sf_status r = solve_loop(m, fcycle ? 1 : 0, rtol, max_cycles, cycles, hist, &handled);
        if (handled || r != SF_OK) return r;
    }
    double fn;
    SF_TRY(sf_norm(L, SF_F, SF_NORM_MAX, &fn));
    if (cycles) *cycles = 0;
    if (!(fn == fn) || std::isinf(fn)) return sf_fail(SF_ERR_NUMERIC, "rhs has NaN/Inf");
    if (fn == 0.0) {
        SF_TRY(k_zero(L, SF_U));
        return sf_sync(L);
    }
    const bool fused = fused_check_ok(m);
    auto fin = [&](double rel, int c) -> int {  // 0 continue, 1 converged, -1 numeric error
        if (hist) hist[c - 1] = rel;
        if (cycles) *cycles = c;
        if (!(rel == rel) || std::isinf(rel)) return -1;
        return rel < rtol ? 1 : 0;
    };
    if (!fused) {
        for (int c = 1; c <= max_cycles; c++) {
            SF_TRY(run(m, (fcycle && c == 1) ? G_FCHECK : G_VCHECK));
            SF_TRY(sf_stream_sync(L));
            int r = fin(L->hscratch[0] / fn, c);
            if (r < 0) return sf_fail(SF_ERR_NUMERIC, "residual is NaN/Inf");
            if (r > 0) return SF_OK;
        }
        return sf_fail(SF_ERR_NOT_CONVERGED, "no convergence to %g in %d cycles", rtol, max_cycles);
    }
    int done = 0;
    if (fcycle) {
        SF_TRY(run(m, G_F));
        done = 1;
    }
    for (;;) {
        // first pair of the next V-cycle + max|F - A U| of the iterate after `done` cycles
        const double* u0 = L->parts[0].f[SF_U];
        SF_TRY(run(m, G_FIRST));
        SF_TRY(sf_stream_sync(L));
        if (done >= 1) {
            int r = fin(L->hscratch[0] / fn, done);
            if (r != 0 || done >= max_cycles) {
                // discard the speculative pair: the iterate of cycle `done` is
                // the buffer U named before it (a graph replay leaves the
                // host-side mapping as it was; an eager run swapped it)
                if (L->parts[0].f[SF_U] != u0) sf_swap_fields(L, SF_U, SF_TMP);
                if (r < 0) return sf_fail(SF_ERR_NUMERIC, "residual is NaN/Inf");
                if (r > 0) return SF_OK;
                return sf_fail(SF_ERR_NOT_CONVERGED, "no convergence to %g in %d cycles", rtol,
                               max_cycles);
            }
        }
        SF_TRY(run(m, G_REST));
        done++;
    }
}

// Pipelined multi-RHS solve (include/sf.h): copies of f_{k+1} (H2D) and
// u_{k-1} (D2H) run on their own streams under solve k; two packed staging
// buffers (kept by the hierarchy) decouple them from the level's F and U.
// Per-phase device times of the call are kept for sf_solve_stream_stats.
extern "C" sf_status sf_solve_stream(sf_mg* m, int fcycle, double rtol, int max_cycles, int n,
                                     const double* const* host_f, double* const* host_u,
                                     int* cycles) {
    if (!m || n < 0 || (n > 0 && (!host_f || !host_u))) return sf_fail(SF_ERR_INVALID, "bad arguments");
    if (n == 0) return SF_OK;
    sf_level* L = m->lv[0];
    const size_t bytes = (size_t)L->nlocal * L->lnz * L->ny * L->nx * sizeof(double);
    if (m->st_bytes != bytes) {
        cudaFree(m->stf);
        cudaFree(m->stu);
        m->stf = m->stu = nullptr;
        m->st_bytes = 0;
        SF_CUDA(cudaMalloc(&m->stf, bytes));
        SF_CUDA(cudaMalloc(&m->stu, bytes));
        m->st_bytes = bytes;
    }
    if (!m->sin) {
        SF_CUDA(cudaStreamCreateWithFlags(&m->sin, cudaStreamNonBlocking));
        SF_CUDA(cudaStreamCreateWithFlags(&m->sout, cudaStreamNonBlocking));
        for (int i = 0; i < 4; i++) SF_CUDA(cudaEventCreateWithFlags(&m->sev[i], cudaEventDisableTiming));
    }
    double *stf = m->stf, *stu = m->stu;
    cudaStream_t sin = m->sin, sout = m->sout;
    cudaEvent_t* ev = m->sev;
    // phase timing: [k][0..5] = H2D start/end, solve start/end, D2H start/end
    std::vector<cudaEvent_t> te(6 * (size_t)n, nullptr);
    for (auto& e : te) SF_CUDA(cudaEventCreate(&e));
    auto tev = [&](int k, int i) { return te[6 * (size_t)k + i]; };
    sf_status st = SF_OK;
    auto cu = [&](cudaError_t e, const char* what) {
        if (e != cudaSuccess && st == SF_OK) st = sf_fail(SF_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
        return st == SF_OK;
    };
    const auto w0 = std::chrono::steady_clock::now();
    int solved = 0;
    // the u staging buffer is free at the start (no D2H pending)
    cu(cudaEventRecord(ev[3], sout), "record");
    if (cu(cudaEventRecord(tev(0, 0), sin), "record") &&
        cu(cudaMemcpyAsync(stf, host_f[0], bytes, cudaMemcpyDefault, sin), "H2D f") &&
        cu(cudaEventRecord(tev(0, 1), sin), "record") && cu(cudaEventRecord(ev[0], sin), "record")) {
        for (int k = 0; k < n && st == SF_OK; k++) {
            if (!cu(cudaStreamWaitEvent(L->stream, ev[0], 0), "wait")) break;
            if (!cu(cudaEventRecord(tev(k, 2), L->stream), "record")) break;
            if ((st = k_pack(L, SF_F, stf, true)) != SF_OK) break;
            if (!cu(cudaEventRecord(ev[1], L->stream), "record")) break;
            if (k + 1 < n && !(cu(cudaStreamWaitEvent(sin, ev[1], 0), "wait") &&
                               cu(cudaEventRecord(tev(k + 1, 0), sin), "record") &&
                               cu(cudaMemcpyAsync(stf, host_f[k + 1], bytes, cudaMemcpyDefault, sin), "H2D f") &&
                               cu(cudaEventRecord(tev(k + 1, 1), sin), "record") &&
                               cu(cudaEventRecord(ev[0], sin), "record")))
                break;
            if (!fcycle && (st = k_zero(L, SF_U)) != SF_OK) break;
            int c = 0;
            st = sf_solve(m, fcycle, rtol, max_cycles, &c, nullptr);
            if (cycles) cycles[k] = c;
            if (st != SF_OK) break;
            if (!cu(cudaStreamWaitEvent(L->stream, ev[3], 0), "wait")) break;
            if ((st = k_pack(L, SF_U, stu, false)) != SF_OK) break;
            if (!(cu(cudaEventRecord(tev(k, 3), L->stream), "record") &&
                  cu(cudaEventRecord(ev[2], L->stream), "record") &&
                  cu(cudaStreamWaitEvent(sout, ev[2], 0), "wait") &&
                  cu(cudaEventRecord(tev(k, 4), sout), "record") &&
                  cu(cudaMemcpyAsync(host_u[k], stu, bytes, cudaMemcpyDefault, sout), "D2H u") &&
                  cu(cudaEventRecord(tev(k, 5), sout), "record") &&
                  cu(cudaEventRecord(ev[3], sout), "record")))
                break;
            solved = k + 1;
        }
    }
    sf_status keep = st;
    cudaStreamSynchronize(sin);
    cudaStreamSynchronize(sout);
    cudaStreamSynchronize(L->stream);
    const double wall = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - w0).count();
    double acc[3] = {0, 0, 0};
    for (int k = 0; k < solved; k++)
        for (int p = 0; p < 3; p++) {
            float ms = 0.f;
            if (cudaEventElapsedTime(&ms, tev(k, 2 * p), tev(k, 2 * p + 1)) == cudaSuccess) acc[p] += ms;
        }
    cudaGetLastError();
    for (auto& e : te) cudaEventDestroy(e);
    for (int p = 0; p < 3; p++) m->stats[p] = solved ? acc[p] / solved : 0.0;
    m->stats[3] = solved ? wall / solved : 0.0;
    return keep;
}

extern "C" sf_status sf_solve_stream_stats(const sf_mg* m, double stats[4]) {
    if (!m || !stats) return sf_fail(SF_ERR_INVALID, "NULL argument");
    for (int i = 0; i < 4; i++) stats[i] = m->stats[i];
    return SF_OK;
}
