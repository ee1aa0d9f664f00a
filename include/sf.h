/*
 * include/sf.h -- C ABI of libsf, the B200-native (sm_100a, fp64) HPGMG-FV
 * hot path that Snowflake's micro-compilers generate (Zhang, Driscoll, Fox,
 * Markley, Williams, Basu: "Snowflake: A Lightweight Portable Stencil DSL",
 * IPDPSW 2017).  "PAPER.md:n" cites a line of the paper's text; "R-n" cites a
 * reading listed in DESIGN.md where the paper is silent or garbled.
 *
 * Plain C types only: ints, doubles, host pointers and device pointers
 * (void*), no torch types.  Every call returns sf_status (SF_OK == 0); the
 * message of the last failure on the calling thread is sf_last_error().
 *
 * GENERAL CONVENTIONS
 *  - Precision: IEEE fp64 everywhere; indices int32/int64.
 *  - Grids: a level is a box of gnx x gny x gnz cells of spacing h (cell
 *    centres at (i+1/2)h), homogeneous Dirichlet boundary on all six faces
 *    (PAPER.md:333-341).  It is split into z-slabs ("parts"); part p owns
 *    global planes [p*lnz, (p+1)*lnz), lnz = gnz/nparts.  A process holds
 *    either all parts (loopback comm, one device) or one part (NCCL comm,
 *    one part per rank / GPU).
 *  - Host arrays are C-order (x fastest), interior only, covering the z-range
 *    of ALL parts local to the caller:
 *        cell fields (U, F, R, TMP, ALPHA, DINV)   (lnz_local, gny, gnx)
 *        SF_BETA_I  (face i between cells i-1, i)   (lnz_local, gny, gnx+1)
 *        SF_BETA_J                                  (lnz_local, gny+1, gnx)
 *        SF_BETA_K                                  (lnz_local+1, gny, gnx)
 *    (lnz_local = lnz * local parts).  Host arrays are never retained.
 *  - Streams: every call enqueues on the level's CUDA stream and returns
 *    without a host synchronisation, EXCEPT sf_level_download, sf_norm,
 *    sf_solve and sf_sync, which synchronise that stream.  Host buffers
 *    passed to sf_level_upload must stay valid until the next synchronising
 *    call (pinned memory makes the copy asynchronous).
 *  - Errors: argument/shape errors are returned synchronously
 *    (SF_ERR_INVALID / SF_ERR_SHAPE).  Asynchronous CUDA/NCCL faults surface
 *    at the next synchronising call as SF_ERR_CUDA / SF_ERR_NCCL.  There is no
 *    CPU fallback: without an sm_100 device every constructor fails with
 *    SF_ERR_CUDA.
 *  - Ghost state: interiors are the contract.  Ghost zones hold valid
 *    boundary values only after sf_apply_bc; the stencil kernels fold the
 *    Dirichlet condition (ghost = -inside) into their arithmetic and refresh
 *    slab halos themselves.
 *  - Thread safety: one level / mg object must not be used concurrently from
 *    two host threads.
 */
#ifndef SF_H_
#define SF_H_

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SF_OK = 0,
    SF_ERR_INVALID = 1,        /* bad argument (NULL handle, bad field id, ...) */
    SF_ERR_SHAPE = 2,          /* dims not even/compatible, gnz % nparts != 0 */
    SF_ERR_OOM = 3,            /* device allocation failed / buffer too small */
    SF_ERR_CUDA = 4,           /* CUDA runtime error, or no sm_100 device */
    SF_ERR_NCCL = 5,           /* NCCL error (or libnccl.so.2 not loadable) */
    SF_ERR_NOT_CONVERGED = 6,  /* sf_solve hit max_cycles */
    SF_ERR_NUMERIC = 7         /* NaN/Inf residual */
} sf_status;

/* Fields stored per level (A1 of DESIGN.md). */
enum sf_field {
    SF_U = 0,      /* solution (finest) / correction e (coarse levels)        */
    SF_F = 1,      /* right-hand side (finest) / restricted residual (coarse) */
    SF_R = 2,      /* residual scratch                                          */
    SF_TMP = 3,    /* scratch; ping-pong target of the colour-fused smoother   */
    SF_ALPHA = 4,  /* alpha(c), cell-centred                                    */
    SF_BETA_I = 5, /* beta on x-faces                                           */
    SF_BETA_J = 6, /* beta on y-faces                                           */
    SF_BETA_K = 7, /* beta on z-faces                                           */
    SF_DINV = 8,   /* lambda = 1/diag(A) (A4)                                   */
    SF_NFIELDS = 9
};

enum sf_restrict_kind { SF_RESTRICT_CELL = 0, SF_RESTRICT_FACE_I = 1,
                        SF_RESTRICT_FACE_J = 2, SF_RESTRICT_FACE_K = 3 };
enum sf_interp_kind { SF_INTERP_P0 = 0 /* piecewise constant */,
                      SF_INTERP_PL = 1 /* trilinear on cell centres */ };
enum sf_norm_kind { SF_NORM_MAX = 0, SF_NORM_L2 = 1 };
enum sf_smoother_kind { SF_SMOOTH_AUTO = 0,     /* fused when the shape allows */
                        SF_SMOOTH_COLOUR = 1,   /* one kernel per colour sweep  */
                        SF_SMOOTH_FUSED = 2,    /* colour-fused RB pair         */
                        SF_SMOOTH_CHEBY = 3,    /* NEXT-3 Chebyshev (mg option) */
                        SF_SMOOTH_FUSED2 = 4 }; /* NEXT-1 two RB pairs per pass  */

typedef struct sf_comm sf_comm;
typedef struct sf_level sf_level;
typedef struct sf_mg sf_mg;

typedef struct {
    int pre_pairs;          /* RB pairs before coarse correction (HPGMG: 2) */
    int post_pairs;         /* RB pairs after (2) */
    int vcycle_interp;      /* SF_INTERP_P0 (reading R-7) */
    int fcycle_interp;      /* SF_INTERP_PL (reading R-7) */
    int agglom_min_planes;  /* agglomerate a level whose slabs would hold fewer planes */
    int max_cycles;         /* sf_solve cap (50) */
    int use_graph;          /* capture V-cycles as CUDA graphs (1) */
    int smoother;           /* enum sf_smoother_kind */
    double rtol;            /* ||f-Au||inf/||f||inf target (1e-10, reading R-9) */
    int cheby_degree;       /* SF_SMOOTH_CHEBY: steps per pair count (2: pre=post=2 -> 4 steps) */
} sf_mg_opts;

/* Default options (pre=post=2, P0/PL, agglomerate below 16 planes, 50 cycles,
 * graphs on, AUTO smoother, rtol 1e-10). */
void sf_mg_opts_default(sf_mg_opts* o);

const char* sf_last_error(void);
/* Library build/version string; never fails. */
const char* sf_version(void);

/* -------------------------------------------------------------- comm
 * Slab decomposition across parts.
 * sf_comm_create_local: nparts slabs held by this process on the current
 *   device; halos move with cudaMemcpyAsync (single-GPU test fixture and
 *   the nranks==1 case).  nparts >= 1.
 * sf_get_unique_id: rank 0 creates an NCCL id (128 bytes, caller buffer);
 *   the caller broadcasts it (e.g. torch.distributed) to every rank.
 * sf_comm_create_nccl: one part per rank; rank in [0,nranks); the current
 *   device must be this rank's GPU.  NCCL is loaded at run time
 *   (libnccl.so.2, the one torch already loaded if any).
 */
sf_status sf_comm_create_local(sf_comm** out, int nparts);
sf_status sf_get_unique_id(unsigned char id[128]);
sf_status sf_comm_create_nccl(sf_comm** out, const unsigned char id[128], int nranks, int rank);
/* Test transport: one part per PROCESS with all
 * processes on the same GPU (NCCL refuses two ranks per device), halos and
 * agglomeration by copies from peer buffers opened through CUDA IPC, host
 * synchronisation and scalar reductions through the caller's all-gather
 * callback (e.g. torch.distributed/gloo).  allgather(send, n, recv, user)
 * must gather n bytes from every rank into recv (rank order) and return 0.
 * Levels created with such a comm (and their agglomerated coarse levels) are
 * collective; CUDA graphs are not used with it. */
typedef int (*sf_host_allgather_fn)(const void* send, size_t nbytes, void* recv, void* user);
sf_status sf_comm_create_hostipc(sf_comm** out, int nranks, int rank, sf_host_allgather_fn allgather,
                                 void* user);
/* Device-initiated transport: one part per process
 * (one GPU each, or several processes sharing a GPU in tests); every level's
 * buffer is opened by every peer through CUDA IPC (peer access over NVLink
 * when the processes own different GPUs) and halos, agglomeration and scalar
 * all-reduces are kernels that read the peers' memory directly and
 * synchronise through flags in device memory (no NCCL, no host round trip;
 * CUDA-graph capturable).  The host all-gather is used only at level
 * creation to exchange the IPC handles; same contract as hostipc.  Every wait
 * on a peer's flag is bounded (environment SF_P2P_TIMEOUT_S, default 60 s, on
 * the GPU's global timer): a dead or hung peer makes the waiting kernel trap,
 * and the next synchronising call returns SF_ERR_CUDA naming the flag, peer
 * slot and op ("p2p peer wait timed out") instead of blocking forever; the
 * CUDA context is unusable afterwards (the process should exit).  With the
 * NCCL transport, synchronising calls poll ncclCommGetAsyncError and abort the
 * communicator on an asynchronous error or after SF_NCCL_TIMEOUT_S (default
 * 600 s), returning SF_ERR_NCCL. */
sf_status sf_comm_create_p2p(sf_comm** out, int nranks, int rank, sf_host_allgather_fn allgather,
                             void* user);
sf_status sf_comm_destroy(sf_comm* comm);
/* Transport self-test (collective): with the NCCL transport, runs once on a few
 * device doubles every collective the slab path uses -- ncclAllReduce (max,
 * sum), ncclBroadcast, ncclAllGather and, for nranks > 1, grouped ring
 * ncclSend/ncclRecv -- on `stream` (cudaStream_t), checks the values on the
 * host and returns SF_ERR_NCCL on any failure or wrong value.  Other transports
 * have nothing to check without a level: SF_OK.  Synchronises. */
sf_status sf_comm_check(const sf_comm* comm, void* stream);
/* number of parts in the job, parts local to this process, first local part */
sf_status sf_comm_info(const sf_comm* comm, int* nparts, int* nlocal, int* first);

/* -------------------------------------------------------------- level (A1)
 * sf_level_bytes_needed: device bytes for a level's fields (all local parts).
 * sf_level_create: dims must be >= 2 and gnz % nparts == 0 (SF_ERR_SHAPE);
 *   comm NULL == one local part.  stream: a cudaStream_t (NULL = legacy
 *   default).  dev_buf: NULL -> the library allocates (and frees on destroy);
 *   else a caller-owned device buffer of >= buf_bytes (e.g. a torch tensor),
 *   256-byte aligned, kept alive by the caller until sf_level_destroy.
 *   Fields are zero-initialised.  The level borrows comm (keep it alive).
 */
sf_status sf_level_bytes_needed(int gnx, int gny, int gnz, const sf_comm* comm, size_t* bytes);
sf_status sf_level_create(sf_level** out, int gnx, int gny, int gnz, double h,
                          const sf_comm* comm, void* stream, void* dev_buf, size_t buf_bytes);
sf_status sf_level_destroy(sf_level* level);
sf_status sf_level_upload(sf_level* level, int field, const double* host);
sf_status sf_level_download(sf_level* level, int field, double* host);   /* syncs */
/* Set every element of `field` (interior, ghosts and halo planes of every
 * local part) to 0 on the device, enqueued on the level's stream -- e.g. the
 * zero initial guess u = 0 of a V-cycle solve.
 * SF_ERR_INVALID for a bad field id. */
sf_status sf_level_zero(sf_level* level, int field);
/* Borrowed device pointer of (local part `part`, field) and its strides in
 * doubles: element (i,j,k) of the part is dev[k*strides[2] + j*strides[1] + i]
 * for -2 <= i,j,k (ghost/padding).  Valid until the next
 * sf_smooth_gsrb on that level (the fused smoother may swap U and TMP). */
sf_status sf_level_field_ptr(sf_level* level, int part, int field, double** dev, long strides[3]);
/* Fill ALPHA, BETA_* (and, if want_rhs, F with the manufactured right-hand
 * side; U zeroed) with the HPGMG-shaped problem of DESIGN.md "Input recipe",
 * on the device.  problem 0 = constant-coefficient (alpha=beta=1), 1 = HPGMG
 * variable-coefficient (tanh beta). */
sf_status sf_init_problem(sf_level* level, int problem, double a, double b, int want_rhs);
/* A4: Dinv = 1/diag(A) with the Dirichlet fold (R-4);
 * also refreshes coefficient halo planes between parts. */
sf_status sf_rebuild_operator(sf_level* level, double a, double b);

/* -------------------------------------------------------------- operators
 * All take field ids of one level.  a, b are the Helmholtz scalars of
 *   A x = a*alpha*x - b*div(beta grad x)
 */
/* A2: ghost fill, ghost = (-1)^m * mirror (R-5) */
sf_status sf_apply_bc(sf_level* level, int field);
/* A3: out = A x (out != x) */
sf_status sf_apply_op(sf_level* level, int out, int x, double a, double b);
/* A5: rb_pairs x (BC, red, BC, black) in place on field x with rhs field rhs
 * and the level's DINV.  Red = (i+j+k) even in
 * global 0-based cell indices (R-2).  x must be SF_U or SF_TMP when the fused
 * smoother is used: it writes each pair into the other of U / TMP and swaps the
 * two ids, so with x = SF_TMP and kind SF_SMOOTH_FUSED the buffer U named before
 * the call is overwritten.  SF_SMOOTH_AUTO takes the fused kernel only for
 * x = SF_U (TMP is then the clobbered scratch), otherwise the colour sweeps.
 * SF_SMOOTH_FUSED2 (NEXT-1): every two pairs
 * run as ONE pass of a temporally blocked kernel (4 sweeps per HBM pass, the
 * result bit-identical to two fused pairs), an odd last pair as one fused
 * pair; same field rules as FUSED, single-part levels with nx % 32 == 0 and
 * ny % 8 == 0 (SF_ERR_SHAPE otherwise).
 * kind: enum sf_smoother_kind. */
sf_status sf_smooth_gsrb(sf_level* level, int x, int rhs, double a, double b, int rb_pairs, int kind);
/* A6: res = rhs - A x */
sf_status sf_residual(sf_level* level, int res, int x, int rhs, double a, double b);
/* A5 + A6 + A7, the tail of V(l)'s pre-smoothing: one RB
 * pair on fine.x (exactly sf_smooth_gsrb with rb_pairs = 1), then
 * coarse.c_field = R_cell(rhs - A x) of the smoothed x.  On single-part fine and
 * coarse levels with x = SF_U, nx % 32 == 0, ny % 8 == 0, even nz and at least
 * SF_RRF_CELLS fine cells (default 2^21; SF_RRF=0 disables), the pair forms the
 * restricted residual itself in delta form (gsrb_rr.cu, DESIGN.md section 6:
 * a red cell's residual after the pair is b h^-2 sum_f beta_f delta of its
 * black neighbours; equal to rhs - A x up to rounding, reading R-19) and a
 * small fix-up pass writes coarse.c_field (the U/TMP ids are swapped as by the
 * fused smoother); the fine level keeps partial arrays for that coarse shape,
 * allocated (zeroed) on first use (sf_mg_create allocates its levels'; a call
 * inside a graph capture without them takes the composite path).  Otherwise the
 * pair, then one residual + restriction pass (even nx: the residual is never
 * stored; odd nx: residual into SF_R, then the restriction).
 * x must differ from rhs, SF_R and SF_DINV.  coarse dims must be fine dims / 2
 * (SF_ERR_SHAPE); c_field must not be SF_DINV.  Enqueued on the fine level's
 * stream; the coarse level must be idle on its own stream. */
sf_status sf_smooth_residual_restrict(sf_level* fine, int x, int rhs, double a, double b,
                                      sf_level* coarse, int c_field);
/* A8 + A5, the head of V(l)'s post-smoothing:
 * fine.x += P0(coarse.c_field) (piecewise-constant interpolation, prescale 1),
 * then one RB pair on fine.x with rhs -- exactly sf_interpolate(P0, 1.0)
 * followed by sf_smooth_gsrb(rb_pairs = 1).  With x = SF_U, rhs != SF_TMP and a
 * level the colour-fused smoother supports, the correction is applied inside
 * the fused pair's single HBM pass (TMP is clobbered and the U/TMP ids are
 * swapped, as by the fused smoother); otherwise P0 then the smoother.  coarse
 * dims must be fine dims / 2 (SF_ERR_SHAPE).  Enqueued on the fine level's
 * stream; the coarse level must be idle on its own stream. */
sf_status sf_interpolate_smooth(sf_level* fine, int x, int rhs, double a, double b,
                                sf_level* coarse, int c_field);
/* A7: coarse.c_field = R(fine.f_field); coarse dims must be fine dims / 2
 * (PAPER.md:293-297, 466-468).  kind: enum sf_restrict_kind. */
sf_status sf_restrict(sf_level* coarse, int c_field, sf_level* fine, int f_field, int kind);
/* A8: fine.f_field = prescale*fine.f_field + P(coarse.c_field)
 * (PAPER.md:293-297, 597).  kind: enum sf_interp_kind.  PL refreshes the
 * coarse field's ghosts (A2) first. */
sf_status sf_interpolate(sf_level* fine, int f_field, double prescale,
                         sf_level* coarse, int c_field, int kind);
/* NEXT-2, the other two operators of the paper's Fig 7:
 * sf_apply_laplacian: out = L x, the canonical constant-coefficient 7-point
 *   Laplacian h^-2 * sum_n (x(c) - x(n)) with the Dirichlet fold (A3 with a = 0,
 *   b = 1, beta = 1, but no coefficient array is read).  out != x.
 * sf_jacobi: out = x + omega * D^-1 (f - L x), D = diag(L) with the fold
 *   (reading R-11: omega = 2/3 in the paper).  Out of place: out != x, f.
 * Both need an even gnx (SF_ERR_SHAPE otherwise). */
sf_status sf_apply_laplacian(sf_level* level, int out, int x);
sf_status sf_jacobi(sf_level* level, int out, int x, int f, double omega);
/* NEXT-3, the Chebyshev smoother the paper names as an in-place technique
 * (formula = reading R-16, Saad Alg. 12.1 with the Jacobi
 * preconditioner D = diag(A)):
 * sf_smooth_chebyshev: `degree` steps damping the eigenvalues of D^-1 A in
 *   [lo, hi] (0 < lo < hi), in place on x; uses TMP and R as scratch (x, rhs
 *   must be other fields).  Field ids of TMP/R may be permuted afterwards.
 * sf_lambda_max: power iteration estimate of lambda_max(D^-1 A): `iters` (>= 2)
 *   steps v <- D^-1 A v / ||.||_2 from the current v, or from the start vector
 *   v = 1 + ((7i + 13j + 29k) mod 17)/17 if start != 0; uses R; syncs. */
sf_status sf_smooth_chebyshev(sf_level* level, int x, int rhs, double a, double b, int degree,
                              double lo, double hi);
sf_status sf_lambda_max(sf_level* level, int v, double a, double b, int iters, int start,
                        double* out);
/* A10: norm of the interior over all parts/ranks; syncs. */
sf_status sf_norm(sf_level* level, int field, int kind, double* out);
sf_status sf_sync(sf_level* level);
/* Live duration of the colour-fused RB-pair kernel (A5) on this level, for the
 * roofline measured inside a timed region: op 1 resets and arms an in-kernel
 * timer (per launch: first CTA start to last CTA end on the global timer,
 * booked by the last CTA), op 0 disarms it and returns the mean ms per RB pair
 * and the number of pairs since arming (a pair split into interior and
 * boundary launches around a halo exchange counts once, with both durations).  Both ops synchronise the level's stream;
 * the timer works inside captured graphs (it lives in the level's scratch). */
sf_status sf_level_pair_timing(sf_level* level, int op, double* mean_ms, long long* count);
/* Per-variant split of the last sf_level_pair_timing(op 0) read-out: mean ms and
 * pairs of the plain [0], input-residual check-fused RESID [1], output-residual
 * BRES [2] and P0-fused INTERP [3] (incl. INTERP + BRES) launches.  Host only. */
sf_status sf_level_pair_timing_variants(const sf_level* level, double mean_ms[4], long long counts[4]);
/* Same read-out for the V-cycle's fused pair + residual + restriction launches
 * (the last pre-smoothing pair with the delta-form restricted residual,
 * gsrb_rr.cu) on this level, which the pair mean above excludes.  Host only. */
sf_status sf_level_pair_timing_rrf(const sf_level* level, double* mean_ms, long long* count);

/* -------------------------------------------------------------- multigrid (A9)
 * sf_mg_create: builds the hierarchy below `finest` (which must hold ALPHA and
 *   BETA_*): coarse coefficients by A7 (cell/face), h_c = 2h, Dinv by A4 on
 *   every level, down to min dim 2 (exact bottom solve, R-8).  Levels whose
 *   slabs would hold fewer than opts->agglom_min_planes planes are
 *   agglomerated (replicated on every part/rank).  opts NULL = defaults.
 *   From the first single-part power-of-two level of <= 32^3 cells down, a
 *   V-cycle runs as ONE thread-block-cluster launch (up to 16 CTAs, operands
 *   in registers / shared memory; coarse.cu); same arithmetic as the per-phase
 *   kernels up to rounding (the sweeps in the fused pairs' lambda form).  The
 *   environment variable SF_COARSE_KERNEL=0, read at sf_mg_create, keeps the
 *   per-phase launches.
 * sf_vcycle: one V-cycle on level l (U_l corrected for rhs F_l), enqueued.
 * sf_fcycle: one F-cycle from scratch for rhs F_0 into U_0, enqueued.
 * sf_solve: optional F-cycle, then V-cycles until ||F-AU||inf/||F||inf <
 *   rtol; fills *cycles and hist[0..*cycles-1] (may be NULL; caller array of
 *   max_cycles+1 doubles); max_cycles < 1 is SF_ERR_INVALID; rtol <= 0 takes
 *   opts->rtol; syncs.  F = 0 gives U = 0 and *cycles = 0; a NaN/Inf
 *   in F returns SF_ERR_NUMERIC with *cycles = 0.  With use_graph and the
 *   colour-fused smoother (max_cycles <= 256, no NCCL transport) the whole
 *   solve is ONE CUDA graph launch whose WHILE node is driven by the
 *   termination test evaluated on the device, and the call synchronises once;
 *   otherwise the host tests after every cycle.  Both give the same iterate,
 *   cycle count and history bits.  On SF_ERR_NOT_CONVERGED U holds the iterate
 *   after exactly max_cycles cycles.
 */
sf_status sf_mg_create(sf_mg** out, sf_level* finest, double a, double b, const sf_mg_opts* opts);
/* Host-only (no device needed): the hierarchy sf_mg_create builds for a
 * gnx x gny x gnz level split into nparts z-slabs -- coarsen while every dim is
 * even and the min dim > 2; a level stays decomposed while its slabs keep >=
 * agglom_min_planes planes (and it is not the bottom), else it and all coarser
 * levels are replicated (agglomerated).  Fills up to max_levels entries of
 * dims[3*l .. 3*l+2] and distributed[l]; *nlevels = levels.  SF_ERR_SHAPE if the
 * bottom would exceed 64 cells or slabs cannot be halved. */
sf_status sf_mg_plan(int gnx, int gny, int gnz, int nparts, int agglom_min_planes, int max_levels,
                     int* nlevels, int* dims, int* distributed);
sf_status sf_mg_num_levels(const sf_mg* mg, int* n);
sf_status sf_mg_level(sf_mg* mg, int l, sf_level** out);
sf_status sf_vcycle(sf_mg* mg, int l);
sf_status sf_fcycle(sf_mg* mg);
sf_status sf_solve(sf_mg* mg, int fcycle, double rtol, int max_cycles, int* cycles, double* hist);
sf_status sf_mg_destroy(sf_mg* mg);
/* Pipelined multi-RHS solve (the serving path): for k = 0..n-1 solve
 * A u_k = f_k exactly as sf_solve does (F-cycle first when fcycle, else from
 * u = 0), reading f_k from host_f[k] and writing u_k to host_u[k] (packed
 * interior host layout of the finest level's local parts, as
 * sf_level_upload/download; pinned memory makes the copies asynchronous).
 * The host->device copy of f_{k+1} and the device->host copy of u_{k-1} run
 * on their own streams while solve k runs, through two packed device staging
 * buffers (2 x one field, allocated on the first call and kept by the
 * hierarchy until sf_mg_destroy).  cycles[k] (may be NULL)
 * receives each solve's cycle count.  Synchronises; returns the first failing
 * solve's status (later right-hand sides are not solved).  Leaves F = f_{last}
 * and U = u_{last} on the level. */
sf_status sf_solve_stream(sf_mg* mg, int fcycle, double rtol, int max_cycles, int n,
                          const double* const* host_f, double* const* host_u, int* cycles);
/* Phase times of the last sf_solve_stream call (CUDA events on the three
 * streams): stats[0] mean H2D copy of one f, [1] mean solve incl. (un)packing,
 * [2] mean D2H copy of one u (ms), [3] host wall ms per right-hand side. */
sf_status sf_solve_stream_stats(const sf_mg* mg, double stats[4]);

/* -------------------------------------------------------------- measurement
 * Number of kernels libsf launched since the counter was last reset (host-side
 * count of launches it issued; a replayed CUDA graph counts its nodes). */
sf_status sf_launch_count(long long* count, int reset);
/* Per-launch device time of the most recent sf_smooth_gsrb kernels is not
 * tracked here; bench.py times sf_smooth_gsrb with CUDA events. */

/* ------------------------------------------- generic stencils (NEXT-4)
 * The paper's language core (Table I, Fig 4): a Stencil
 * associates an expression over meshes (Components = weight arrays applied to
 * a mesh; weights may themselves be mesh expressions -- variable coefficients),
 * an output mesh (possibly one of the inputs: in place) and a domain that is a
 * union of strided RectDomains whose negative bounds are relative to the grid
 * size; a StencilGroup runs stencils consecutively.  Compiling a group renders
 * ONE CUDA kernel for it and compiles it at run time for sm_100a (NVRTC), the
 * B200 counterpart of the paper's JIT micro-compilers.
 *
 * Coordinates (reading R-17): ghost-inclusive, one ghost layer as in Fig 4 --
 * interior cell i of axis d has coordinate i+1, so interior = [1, n_d] and the
 * Dirichlet ghost layer is 0 and n_d+1.  Rect bounds b < 0 mean N_d + b with
 * N_d = n_d + 2 (so hi = -1 is the exclusive end n_d+1); lo inclusive, hi
 * exclusive, stride >= 1; stride 0 makes the axis the single coordinate lo
 * (Fig 4 l.17's boundary domain).  A READ node reads mesh `mesh` of the output level
 * (src 0) or of the source level (src 1) at, per axis,
 *     q = floor((mul*p + pre) / div) + off            (p = output point)
 * -- plain offsets have mul = div = 1, pre = 0; restriction reads a fine level
 * at 2p + o (mul 2), P0 interpolation a coarse level at floor((p+1)/2) (div 2,
 * pre 1).  Reads may reach the storage ghost zone (2 layers on every axis).
 *
 * Semantics: every point of a stencil's domain is computed from the values
 * before the stencil (points of one stencil are independent); stencils of a
 * group apply in order.  sf_stencil_apply verifies this with the paper's
 * Diophantine analysis (exact per-axis lattice intersection
 * by the extended Euclidean algorithm): an in-place stencil whose reads of its
 * output mesh hit points it writes, other than each point's own, is rejected
 * (SF_ERR_INVALID); consecutive independent stencils (no RAW/WAR/WAW overlap)
 * share one launch, a dependence starts a new launch (the paper's greedy
 * barrier placement). */
typedef struct sf_stencil sf_stencil;
enum sf_sx_op {
    SF_SX_CONST = 0, /* value                                   */
    SF_SX_READ = 1,  /* mesh[src](affine(p))                     */
    SF_SX_ADD = 2,   /* node a + node b                          */
    SF_SX_SUB = 3,   /* node a - node b                          */
    SF_SX_MUL = 4,   /* node a * node b                          */
    SF_SX_DIV = 5,   /* node a / node b                          */
    SF_SX_NEG = 6    /* -node a                                  */
};
typedef struct {
    int op;          /* sf_sx_op                                              */
    int a, b;        /* operand node indices (must be < this node's index)     */
    int mesh, src;   /* READ: sf_field, 0 = output level, 1 = source level     */
    int off[3], mul[3], div[3], pre[3];   /* READ: affine map per axis (x,y,z) */
    double value;    /* CONST                                                 */
} sf_sx_node;
typedef struct {
    int lo[3], hi[3], stride[3];   /* x, y, z; see coordinates above          */
} sf_rect;
typedef struct {
    int n_nodes;
    const sf_sx_node* nodes;       /* expression DAG in topological order      */
    int root;                      /* node whose value is stored               */
    int out_mesh;                  /* sf_field written on the output level     */
    int n_rects;                   /* DomainUnion: 1..SF_STENCIL_MAX_RECTS      */
    const sf_rect* rects;
} sf_stencil_desc;
#define SF_STENCIL_MAX_RECTS 64
/* Validate and render the group (host only; no GPU needed).  The descriptions
 * are copied.  SF_ERR_INVALID on malformed input. */
sf_status sf_stencil_compile(sf_stencil** out, const sf_stencil_desc* stencils, int n_stencils);
/* The rendered CUDA source (NUL-terminated; *len = its length without NUL;
 * copies min(cap-1, len) bytes when buf != NULL). */
sf_status sf_stencil_source(const sf_stencil* s, char* buf, size_t cap, size_t* len);
/* Run the group on `level` (output level, src 0) reading `src` (src 1; NULL =
 * `level`).  JIT-compiles on first use (NVRTC, sm_100a; SF_ERR_CUDA if NVRTC or
 * the device is unavailable).  Multi-part levels: same-level reads only, z
 * halos of read meshes exchanged before each launch (depth <= 2); cross-level
 * groups need single-part levels.  Enqueued on level's stream.  Errors:
 * SF_ERR_SHAPE when a domain point or read falls outside the storage,
 * SF_ERR_INVALID for a racy in-place stencil. */
sf_status sf_stencil_apply(sf_stencil* s, sf_level* level, sf_level* src);
/* Host-only dependence analysis of the group on a gnx x gny x gnz grid
 * (src_is_output: source-level reads hit the output level): *phases = the
 * launches apply would use; SF_ERR_INVALID for a racy in-place stencil. */
sf_status sf_stencil_plan(const sf_stencil* s, int gnx, int gny, int gnz, int src_is_output,
                          int* phases);
/* Number of launches (dependence phases) the last apply used. */
sf_status sf_stencil_phases(const sf_stencil* s, int* phases);
sf_status sf_stencil_destroy(sf_stencil* s);

#ifdef __cplusplus
}
#endif
#endif /* SF_H_ */
