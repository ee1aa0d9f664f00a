// Internal definitions of libsf (CUDA C++ for sm_100a).  Not part of the ABI.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdio>
#include <string>
#include <vector>

#include "sf.h"

// ------------------------------------------------------------------ layout (A1)
// Per part and field: (lnz + 2*SF_GZ) planes x (ny + 2*SF_GY) rows x js doubles.
// Element (i,j,k) at (k+SF_GZ)*ks + (j+SF_GY)*js + SF_OX + i, i in [-2, nx+1].
// SF_OX = 2 puts i = -2 on a 128-byte row start (js is a multiple of 16
// doubles, every field base 256-byte aligned) and i = 0 on a 16-byte boundary:
// the colour-fused pair's TMA boxes (x0-2 .. x0+TX+1, 36 doubles) then cover
// 9 instead of 10 32-byte sectors per row (-10 % L2 -> SM bytes; 512^3 pair
// -3.4 % under the power cap, profiles/r02/ab_ox2.txt), and double2 loads of
// interior pairs stay aligned.  (OX = 4 put i = 0 on a 32-byte boundary.)  Two ghost planes in z (depth-2 slab halos of
// the colour-fused smoother) and two ghost rows in y (its 2-ring tile loads).
#ifndef SF_OX
#define SF_OX 2
#endif
#define SF_GY 2
#define SF_GZ 2
// per-level device scratch after the fields: 32 doubles + the P2P sync block
// (comm kind 3): u64 [0] ready, [1] consumed, [2] op sequence, [3] CTA count,
// [8, 8 + SF_P2P_MAX_RANKS) all-reduce slots (doubles)
#define SF_P2P_MAX_RANKS 64
#define SF_SCRATCH_BYTES (256 + 8 * (8 + SF_P2P_MAX_RANKS))
// dscratch slots: [0] fused-check max residual, [1] power-iteration sum, [2] max|F|
// of the device solve loop, [8..21] live timing of the colour-fused pair
// (u64: armed, min start, max end, finished CTAs, launches, sum of ns, then
// (launches, sum of ns) per variant: plain, RESID, BRES, INTERP)
#define SF_TS_OFF 8

struct sf_comm {
    int kind;          // 0 = local (all parts in this process), 1 = NCCL, 2 = host+IPC (tests),
                       // 3 = device-initiated P2P (peer memory over NVLink, CUDA IPC)
    int nparts;        // parts in the whole job
    int nlocal;        // parts held by this process
    int first;         // global index of the first local part
    int rank, nranks;
    void* nccl;        // ncclComm_t
    sf_host_allgather_fn hostfn;  // kind 2
    void* hostuser;
};

// Internal fields after the public ones (not addressable through the C ABI):
// the face coefficients with every global Dirichlet face set to 0, read only by
// the colour-fused pair.  With them a boundary neighbour's term beta_f * x_ghost
// vanishes by itself (the ghost is finite: buffers are zeroed at creation), so
// the pair needs no boundary selects; the face's -x(c) ghost term lives in
// Dinv as before.  Rebuilt with Dinv by sf_rebuild_operator.
#define SF_BI0 (SF_NFIELDS + 0)
#define SF_BJ0 (SF_NFIELDS + 1)
#define SF_BK0 (SF_NFIELDS + 2)
#define SF_NF_ALL (SF_NFIELDS + 3)

struct SfPart {
    int index;                 // global part index
    int z0;                    // global z of local plane 0
    double* f[SF_NF_ALL];      // base of each field's allocation (plane -SF_GZ)
};

struct sf_level {
    int gnx, gny, gnz;         // global cells
    int nx, ny, lnz;           // per-part interior dims
    double h;
    long js, ks;               // strides (doubles)
    size_t felems;             // doubles per field per part
    int nparts, nlocal, first; // decomposition (nparts == 1: single / replicated)
    const sf_comm* comm;       // NULL for a single / replicated level
    const sf_comm* rep_comm;   // replicated (agglomerated) level: the job's comm
    std::vector<SfPart> parts; // local parts
    cudaStream_t stream;
    cudaStream_t side = nullptr;       // halo exchange beside the interior sweep (lazy)
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    void* buf;
    bool owns;
    double* dscratch;          // device scalars (norms)
    unsigned long long* dsync; // P2P sync block (inside buf: peers reach it through IPC)
    double* hscratch;          // pinned, mapped host scalars
    double* hscratch_dev;      // their device alias
    double ts_var[5][2] = {};  // last sf_level_pair_timing read-out per variant: launches, ns
                               // (plain, RESID, BRES, INTERP, pair + residual + restriction)
    double* rrf_buf = nullptr; // SfRRF partial arrays for the coarse level below (gsrb_rr.cu)
    size_t rrf_felems = 0;
    // the next fused pair may start under the launch before it (that launch
    // triggers early and writes nothing the pair reads except the P0 source;
    // set by the V-cycle, consumed by the pair launch)
    int pdl_early = 0;
    std::vector<char*> peer;   // kind-2 comm: peer ranks' level buffers (CUDA IPC), by rank
    std::vector<void*> ipc_opened;
};

// Part view passed to kernels by value.  Kernels must only index f[] with
// compile-time constants (a runtime index spills the struct to local memory);
// fields chosen at run time are passed as separate pointers.
struct PV {
    double* f[SF_NF_ALL];
    int nx, ny, nz;            // local interior dims
    int z0, gnz;               // global z offset / extent (Dirichlet faces at 0, gnz)
    long js, ks;
};

__host__ __device__ __forceinline__ long sf_ix(const PV& v, int i, int j, int k) {
    return (long)(k + SF_GZ) * v.ks + (long)(j + SF_GY) * v.js + SF_OX + i;
}

PV sf_view(const sf_level* L, int p);
void sf_swap_fields(sf_level* L, int f1, int f2);   // host-side id <-> buffer mapping

sf_status sf_norm_async(sf_level* L, int field, int kind, double* dst);
sf_status sf_scalar_to_host(sf_level* L, const double* src, int slot);
sf_status sf_copy_field(sf_level* L, int field, double* host, bool up, cudaStream_t stream);

// ------------------------------------------------------------------ errors
sf_status sf_fail(sf_status s, const char* fmt, ...);
// SF_ERR_CUDA for e; names a timed-out p2p peer wait if that caused it (comm.cu)
sf_status sf_cuda_failure(cudaError_t e, const char* what);
#define SF_CUDA(call)                                                                  \
    do {                                                                               \
        cudaError_t e_ = (call);                                                       \
        if (e_ != cudaSuccess) return sf_cuda_failure(e_, #call);                      \
    } while (0)
#define SF_TRY(call)                                \
    do {                                            \
        sf_status s_ = (call);                      \
        if (s_ != SF_OK) return s_;                 \
    } while (0)
#define SF_LAUNCHED() sf_count_launch()

// ------------------------------------------------------------------ launches
// Every kernel is launched with programmatic stream serialisation (PDL): the
// next kernel of the stream may be scheduled onto SMs the previous one has
// left while that one drains, and runs its prologue up to pdl_wait(), which
// blocks until the previous grid has completed and its writes are visible.
// Every kernel calls pdl_wait() before touching global memory, so stream
// order semantics are unchanged; only launch latency is hidden.  SF_PDL=0
// launches without the attribute (A/B).
__device__ __forceinline__ void pdl_wait() {
#if defined(__CUDA_ARCH__) && __CUDA_ARCH__ >= 900
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}
bool sf_pdl_on();
template <typename... K, typename... A>
inline cudaError_t sf_launch(void (*k)(K...), dim3 g, dim3 b, size_t smem, cudaStream_t s,
                             A&&... args) {
    cudaLaunchConfig_t c = {};
    c.gridDim = g;
    c.blockDim = b;
    c.dynamicSmemBytes = smem;
    c.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    c.attrs = at;
    c.numAttrs = sf_pdl_on() ? 1 : 0;
    return cudaLaunchKernelEx(&c, k, static_cast<A&&>(args)...);
}
void sf_count_launch(long long n = 1);
sf_status sf_check_launch(const char* what);

// residual reductions riding in a fused pair (rmax = device scalar)
// SF_RM_ZERO: the pair only zeroes *rmax (for a BRES pair later in the stream,
// which then skips its own reset launch: SF_RM_OUTPUT_BLACK_ZEROED)
enum { SF_RM_NONE = 0, SF_RM_INPUT_RED = 1, SF_RM_OUTPUT_BLACK = 2, SF_RM_ZERO = 3,
       SF_RM_OUTPUT_BLACK_ZEROED = 4 };

// ------------------------------------------------------------------ kernels (kernels.cu)
sf_status k_apply_op(sf_level* L, int out, int x, double a, double b);
sf_status k_residual(sf_level* L, int res, int x, int rhs, double a, double b);
sf_status k_gsrb_colour(sf_level* L, int x, int rhs, double a, double b, int colour);
sf_status k_dinv(sf_level* L, double a, double b);
sf_status k_beta0(sf_level* L);
sf_status k_bc(sf_level* L, int field);
sf_status k_restrict(sf_level* C, int cf, sf_level* F, int ff, int kind);
sf_status k_interp(sf_level* F, int ff, double s, sf_level* C, int cf, int kind);
sf_status k_norm(sf_level* L, int field, int kind, double* dst_dev);
sf_status k_zero(sf_level* L, int field);
sf_status k_pack(sf_level* L, int field, double* buf, bool up);
sf_status k_init_problem(sf_level* L, int problem, double a, double b, int want_rhs);
sf_status k_bottom_setup(sf_level* L, double a, double b, double* ainv);
sf_status k_bottom_solve(sf_level* L, int x, int rhs, const double* ainv);

// pair-per-thread bandwidth kernels (kernels_pair.cu); need even nx
bool pair_ok(const sf_level* L);
sf_status k_residual_pair(sf_level* L, int res /* -1: do not write */, int x, int rhs, double a,
                          double b, double* max_out /* NULL: no norm */);
// trigger_next: let the next launch start early (PDL trigger; it must only
// read this kernel's output after griddepcontrol.wait -- the coarse cluster V-cycle)
sf_status k_residual_restrict(sf_level* F, int x, int rhs, double a, double b, sf_level* C, int cf,
                              bool trigger_next = false);
sf_status k_interp_p0_pair(sf_level* F, int ff, double s, sf_level* C, int cf);
sf_status k_norm_pair(sf_level* L, int field, int kind, double* dst);
sf_status k_cc(sf_level* L, int out, int x, int f, double omega, bool jacobi);  // NEXT-2
// NEXT-3 Chebyshev smoother pieces
sf_status k_cheby_step(sf_level* L, int out, int x, int xp, int rhs, double c1, double c2, double a,
                       double b);
sf_status k_start_vector(sf_level* L, int field);
sf_status k_power_step(sf_level* L, int v_id, int w_id, double a, double b, double* sumsq);
sf_status sf_chebyshev_impl(sf_level* L, int x, int rhs, double a, double b, int degree, double lo,
                            double hi);
sf_status sf_lambda_max_impl(sf_level* L, int v, double a, double b, int iters, bool start,
                             double* out);

// Restriction partials of the pair + residual + restriction (gsrb_rr.cu): twelve
// coarse-shaped arrays (coarse layout, allocation bases), each entry written by
// at most one thread of the fused pair's RRF launch; the fix-up pass sums them
// into the coarse rhs.  Order: P (the block's own, x and z shares) even / odd
// fine row; XW, XE (shares from the east / west tile's edge column) even / odd;
// YS, YN (from the block row north / south); ZB, ZT (from the z-chunk above /
// below, edge planes only) even / odd.  zdepth: the launch's z-chunk depth
// (set by the pair launch; the fix-up reads the z edges there).
struct SfRRF {
    double* a[12];
    int cjs, cks, ncx, ncy, ncz, zdepth;
};

// fused colour pair (gsrb_fused.cu, built as 32x16 "_t32" and 64x8 "_t64"; dispatch in level.cu)
bool gsrb_fused_supported_t32(const sf_level* L);
bool gsrb_fused_supported_t64(const sf_level* L);
sf_status k_gsrb_pair_fused_t32(sf_level* L, int xin, int xout, int rhs, double a, double b,
                                double* rmax, sf_level* C, int cf, int phase = 0, int reserve = 0,
                                int rmode = 0, SfRRF* rrf = nullptr);
sf_status k_gsrb_pair_fused_t64(sf_level* L, int xin, int xout, int rhs, double a, double b,
                                double* rmax, sf_level* C, int cf, int phase = 0, int reserve = 0,
                                int rmode = 0, SfRRF* rrf = nullptr);
// 32x8 tiles, 4 warps, 3 CTAs per SM (three independent z-step chains per SM)
bool gsrb_fused_supported_t32w4(const sf_level* L);
sf_status k_gsrb_pair_fused_t32w4(sf_level* L, int xin, int xout, int rhs, double a, double b,
                                  double* rmax, sf_level* C, int cf, int phase = 0, int reserve = 0,
                                int rmode = 0, SfRRF* rrf = nullptr);
bool gsrb_fused_supported(const sf_level* L);
// rmax != NULL: the pair also reduces max|rhs - A x_in| of its input into *rmax;
// C != NULL: the pair first applies x_in += P0(C.cf) (V-cycle interpolation)
sf_status k_gsrb_pair_fused(sf_level* L, int xin, int xout, int rhs, double a, double b,
                            double* rmax = nullptr, sf_level* C = nullptr, int cf = 0,
                            int phase = 0, int reserve = 0, int rmode = SF_RM_NONE);
// the depth-2 x halo exchange + fused pair, overlapped on multi-part levels:
// the halo runs on a side stream while the interior z-chunks are smoothed, then
// the boundary chunks (comm.cu)
sf_status k_gsrb_pair_halo(sf_level* L, int xin, int xout, int rhs, double a, double b,
                           double* rmax = nullptr, sf_level* C = nullptr, int cf = 0,
                           int rmode = SF_RM_NONE);
// halo exchange enqueued on stream s instead of the level's stream (kinds 0, 1, 3)
sf_status sf_halo_on(sf_level* L, int field, int depth, cudaStream_t s);
// NEXT-1: two RB pairs in one pass (gsrb_twopair.cu): xout = pair(pair(xin));
// single-part levels, nx % 32 == 0, ny % 8 == 0
bool gsrb_twopair_supported(const sf_level* L);
sf_status k_gsrb_twopair(sf_level* L, int xin, int xout, int rhs, double a, double b);
// last pre-smoothing pair fused with residual + restriction (gsrb_rr.cu):
// xout = pair(xin); C.cf = R_cell(rhs - A xout).  Single-part levels, 32x16 tiles.
bool gsrb_rr_supported(const sf_level* F, const sf_level* C);
sf_status k_gsrb_pair_rr(sf_level* L, int xin, int xout, int rhs, double a, double b, sf_level* C,
                         int cf, bool trigger_next = false);
// allocate the fine level's RRF partial arrays for coarse level C (before any capture)
sf_status sf_rrf_prepare(sf_level* F, const sf_level* C);
bool sf_rrf_usable(const sf_level* F, const sf_level* C);

// coarse-level V-cycle in one thread-block-cluster launch, iterates in registers and
// shared memory (coarse.cu)
bool coarse_vcycle_fits(sf_level* const* lv, int n);
int coarse_vcycle_max_levels();
// u_zero: lv[0]'s U is zero on entry (V-cycle recursion): not read, not zeroed first
// trigger_next: the launch after it may start early (griddepcontrol.launch_dependents)
sf_status k_coarse_vcycle(sf_level* const* lv, int n, double a, double b, const double* ainv,
                          int pre, int post, bool u_zero, bool trigger_next = false);

// ------------------------------------------------------------------ comm (comm.cu)
// Exchange `depth` z-halo planes of `field` between neighbouring parts.
sf_status sf_halo(sf_level* L, int field, int depth);
// Replicated coarse level C receives, on every process, the planes each part
// of the distributed fine level F wrote into it (in-place all-gather).
sf_status sf_agglomerate(sf_level* C, int field, int parts, int lnz_per_part);
// kind-2 comm: open the peers' buffers of level L (collective)
sf_status sf_ipc_register(sf_level* L, const sf_comm* c);
void sf_ipc_close(sf_level* L);
// Host synchronisation of the level's stream: NCCL async errors polled, a
// timed-out p2p peer wait reported by name (comm.cu).
sf_status sf_stream_sync(sf_level* L);
// Reduce a device scalar over ranks (op 0 = max, 1 = sum); in place.
sf_status sf_allreduce_scalar(sf_level* L, const sf_comm* comm, double* dev, int op);
