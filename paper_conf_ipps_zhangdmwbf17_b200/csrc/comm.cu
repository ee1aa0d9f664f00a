// Slab decomposition plumbing: z-halo exchange between
// neighbouring parts, coarse-level agglomeration and scalar all-reduce.
//
// Parts local to this process exchange with cudaMemcpyAsync (the loopback
// fixture that lets one GPU run the decomposed code path); parts on other
// ranks exchange with NCCL point-to-point over NVLink.  NCCL is resolved at
// run time from libnccl.so.2 (torch's copy when torch is loaded), so libsf
// has no link-time NCCL dependency and the CPU-only build box can build it.
#include <dlfcn.h>
#include <nccl.h>

#include <cuda.h>

#include <chrono>
#include <mutex>
#include <thread>

#include <algorithm>
#include <cmath>

#include <cstdlib>
#include <cstring>

#include "sf_internal.h"

namespace {

struct NcclApi {
    void* h = nullptr;
    decltype(&ncclGetUniqueId) getUniqueId;
    decltype(&ncclCommInitRank) commInitRank;
    decltype(&ncclCommDestroy) commDestroy;
    decltype(&ncclSend) send;
    decltype(&ncclRecv) recv;
    decltype(&ncclGroupStart) groupStart;
    decltype(&ncclGroupEnd) groupEnd;
    decltype(&ncclAllReduce) allReduce;
    decltype(&ncclAllGather) allGather;
    decltype(&ncclBroadcast) broadcast;
    decltype(&ncclGetErrorString) errStr;
    decltype(&ncclCommGetAsyncError) asyncErr;
    decltype(&ncclCommAbort) abort;
};

NcclApi g_nccl;
std::mutex g_nccl_mu;

sf_status nccl_load() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.h) return SF_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return sf_fail(SF_ERR_NCCL, "cannot load libnccl.so.2: %s", dlerror());
#define SYM(field, name)                                                             \
    g_nccl.field = (decltype(g_nccl.field))dlsym(h, name);                           \
    if (!g_nccl.field) return sf_fail(SF_ERR_NCCL, "libnccl.so.2 lacks %s", name);
    SYM(getUniqueId, "ncclGetUniqueId");
    SYM(commInitRank, "ncclCommInitRank");
    SYM(commDestroy, "ncclCommDestroy");
    SYM(send, "ncclSend");
    SYM(recv, "ncclRecv");
    SYM(groupStart, "ncclGroupStart");
    SYM(groupEnd, "ncclGroupEnd");
    SYM(allReduce, "ncclAllReduce");
    SYM(allGather, "ncclAllGather");
    SYM(broadcast, "ncclBroadcast");
    SYM(errStr, "ncclGetErrorString");
    SYM(asyncErr, "ncclCommGetAsyncError");
    SYM(abort, "ncclCommAbort");
#undef SYM
    g_nccl.h = h;
    return SF_OK;
}

#define SF_NCCL(call)                                                                    \
    do {                                                                                 \
        ncclResult_t r_ = (call);                                                        \
        if (r_ != ncclSuccess)                                                           \
            return sf_fail(SF_ERR_NCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call,       \
                           g_nccl.errStr ? g_nccl.errStr(r_) : "?");                     \
    } while (0)

}  // namespace

extern "C" sf_status sf_comm_create_local(sf_comm** out, int nparts) {
    if (!out || nparts < 1) return sf_fail(SF_ERR_INVALID, "bad arguments");
    sf_comm* c = new sf_comm();
    c->kind = 0;
    c->nparts = nparts; c->nlocal = nparts; c->first = 0;
    c->rank = 0; c->nranks = 1;
    c->nccl = nullptr;
    *out = c;
    return SF_OK;
}

extern "C" sf_status sf_get_unique_id(unsigned char id[128]) {
    if (!id) return sf_fail(SF_ERR_INVALID, "id is NULL");
    SF_TRY(nccl_load());
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId u;
    SF_NCCL(g_nccl.getUniqueId(&u));
    memcpy(id, &u, 128);
    return SF_OK;
}

extern "C" sf_status sf_comm_create_nccl(sf_comm** out, const unsigned char id[128], int nranks,
                                         int rank) {
    if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks)
        return sf_fail(SF_ERR_INVALID, "bad arguments");
    SF_TRY(nccl_load());
    ncclUniqueId u;
    memcpy(&u, id, 128);
    ncclComm_t comm;
    SF_NCCL(g_nccl.commInitRank(&comm, nranks, u, rank));
    sf_comm* c = new sf_comm();
    c->kind = 1;
    c->nparts = nranks; c->nlocal = 1; c->first = rank;
    c->rank = rank; c->nranks = nranks;
    c->nccl = comm;
    *out = c;
    return SF_OK;
}

static void ensure_err_word();

static sf_status create_ipc_comm(sf_comm** out, int nranks, int rank, sf_host_allgather_fn fn,
                                 void* user, int kind) {
    if (!out || !fn || nranks < 1 || rank < 0 || rank >= nranks)
        return sf_fail(SF_ERR_INVALID, "bad arguments");
    if (kind == 3 && nranks > SF_P2P_MAX_RANKS)
        return sf_fail(SF_ERR_INVALID, "p2p comm supports <= %d ranks", SF_P2P_MAX_RANKS);
    sf_comm* c = new sf_comm();
    c->kind = kind;
    c->nparts = nranks; c->nlocal = 1; c->first = rank;
    c->rank = rank; c->nranks = nranks;
    c->nccl = nullptr;
    c->hostfn = fn;
    c->hostuser = user;
    // the p2p timeout's mapped host word is allocated here, never inside a
    // stream capture (a pinned allocation there would abort the capture)
    if (kind == 3) ensure_err_word();
    *out = c;
    return SF_OK;
}

extern "C" sf_status sf_comm_create_hostipc(sf_comm** out, int nranks, int rank,
                                            sf_host_allgather_fn fn, void* user) {
    return create_ipc_comm(out, nranks, rank, fn, user, 2);
}

extern "C" sf_status sf_comm_create_p2p(sf_comm** out, int nranks, int rank, sf_host_allgather_fn fn,
                                        void* user) {
    return create_ipc_comm(out, nranks, rank, fn, user, 3);
}

namespace {
sf_status host_allgather(const sf_comm* c, const void* send, size_t n, void* recv) {
    if (c->hostfn(send, n, recv, c->hostuser) != 0)
        return sf_fail(SF_ERR_NCCL, "host all-gather callback failed");
    return SF_OK;
}
sf_status host_barrier(const sf_comm* c) {
    char b = 0;
    std::vector<char> r(c->nranks);
    return host_allgather(c, &b, 1, r.data());
}
double* peer_field(const sf_level* L, int rank, const double* mine) {
    return (double*)(L->peer[rank] + ((const char*)mine - (const char*)L->buf));
}
}  // namespace

// ------------------------------------------------------------ kind 3: P2P
// Device-initiated exchanges over peer memory.  Every exchange is one op of a
// per-level sequence that all ranks run in the same order (SPMD); op s:
//   1. "ready = s" (release, system scope): my data for op s is final (all
//      earlier kernels of the stream are done);
//   2. wait until every peer involved shows ready >= s (acquire), read its
//      data straight from its memory (NVLink loads), write mine;
//   3. "consumed = s", then wait until those peers show consumed >= s: nobody
//      overwrites data a peer is still reading, and a peer can be at most one
//      op ahead.
// The sequence number lives in device memory (read at kernel start, advanced
// by the last CTA), so the kernels replay correctly from CUDA graphs.
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long p2p_clock() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

struct P2PPeers {
    const unsigned long long* sync[SF_P2P_MAX_RANKS];   // peers' sync blocks (nullptr: not involved)
    unsigned long long* err;        // mapped host word written before a timed-out wait traps
    unsigned long long timeout_ns;  // bound of every wait on a peer's flag
};

// Wait until *p >= v.  A peer that never gets there (dead, hung, or not
// running the same op sequence) must not wedge this GPU forever: after
// timeout_ns on the global timer the waiting thread records (what, peer, op)
// in mapped host memory and traps, which fails the stream with a CUDA error
// that sf_stream_sync reports as SF_ERR_CUDA with that description.
__device__ __forceinline__ void wait_ge(const unsigned long long* p, unsigned long long v,
                                        const P2PPeers& pe, int peer, int what) {
    if (ld_acquire_sys(p) >= v) return;
    const unsigned long long t0 = p2p_clock();
    unsigned ns = 32;
    while (ld_acquire_sys(p) < v) {
        __nanosleep(ns);
        if (ns < 1024) ns *= 2;
        if (p2p_clock() - t0 > pe.timeout_ns) {
            if (pe.err) {
                *(volatile unsigned long long*)pe.err =
                    (1ull << 63) | ((unsigned long long)what << 56) |
                    ((unsigned long long)(peer & 0xffff) << 40) | (v & 0xffffffffffull);
                __threadfence_system();
            }
            __trap();
        }
    }
}

// op start: every CTA learns s; CTA 0 publishes ready; thread 0 of each CTA
// waits for the peers' ready
__device__ __forceinline__ unsigned long long p2p_begin(unsigned long long* my, const P2PPeers& pe,
                                                        int npeers) {
    __shared__ unsigned long long s_seq;
    if (threadIdx.x == 0) {
        const unsigned long long s = *(volatile unsigned long long*)&my[2] + 1;
        if (blockIdx.x == 0) st_release_sys(&my[0], s);
        for (int q = 0; q < npeers; q++)
            if (pe.sync[q]) wait_ge(&pe.sync[q][0], s, pe, q, 1);
        s_seq = s;
    }
    __syncthreads();
    return s_seq;
}

// op end: the last CTA publishes consumed, waits for the peers', advances s
__device__ __forceinline__ void p2p_end(unsigned long long* my, const P2PPeers& pe, int npeers,
                                        unsigned long long s) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned prev = atomicAdd((unsigned*)&my[3], 1u);
        if (prev == gridDim.x - 1) {
            __threadfence();
            my[3] = 0;
            st_release_sys(&my[1], s);
            for (int q = 0; q < npeers; q++)
                if (pe.sync[q]) wait_ge(&pe.sync[q][1], s, pe, q, 2);
            *(volatile unsigned long long*)&my[2] = s;
        }
    }
}

// halo: my ghosts <- the neighbours' boundary planes (peers 0 = lower, 1 = upper)
__global__ void __launch_bounds__(256) p2p_halo_kernel(double* x, const double* lo_x, const double* hi_x,
                                                       unsigned long long* my, P2PPeers pe, long lo_dst,
                                                       long hi_src, long hi_dst, long lo_src, long cnt) { pdl_wait();
    const unsigned long long s = p2p_begin(my, pe, 2);
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride) {
        if (lo_x) x[lo_dst + i] = lo_x[hi_src + i];
        if (hi_x) x[hi_dst + i] = hi_x[lo_src + i];
    }
    p2p_end(my, pe, 2, s);
}

struct P2PPtrs {
    const double* p[SF_P2P_MAX_RANKS];
};

// all-reduce of one scalar: my slot <- v; every rank reduces all ranks' slots
// in rank order (the same result on every rank)
__global__ void p2p_allreduce_kernel(double* v, unsigned long long* my, P2PPeers pe, P2PPtrs slot,
                                     int nranks, int op) { pdl_wait();
    // my slot is rewritten only after every peer consumed the previous op
    if (threadIdx.x == 0) *(double*)(my + 8) = *v;
    const unsigned long long s = p2p_begin(my, pe, nranks);
    if (threadIdx.x == 0) {
        double r = 0.0;
        for (int q = 0; q < nranks; q++) {
            const double y = *(const volatile double*)slot.p[q];
            if (q == 0) r = y;
            else if (op == 0) r = (y > r || y != y) ? y : r;
            else r = r + y;
        }
        *v = r;
    }
    p2p_end(my, pe, nranks, s);
}

// agglomeration: copy every other rank's planes of a replicated level
__global__ void __launch_bounds__(256) p2p_gather_kernel(double* base, P2PPtrs peer_base,
                                                         unsigned long long* my, P2PPeers pe, int nranks,
                                                         int rank, long cnt, double* top,
                                                         const double* peer_top, long topcnt) { pdl_wait();
    const unsigned long long s = p2p_begin(my, pe, nranks);
    const long stride = (long)gridDim.x * blockDim.x;
    for (int q = 0; q < nranks; q++) {
        if (q == rank) continue;
        const double* src = peer_base.p[q] + q * cnt;
        double* dst = base + q * cnt;
        for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride) dst[i] = src[i];
    }
    if (peer_top)
        for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < topcnt; i += stride) top[i] = peer_top[i];
    p2p_end(my, pe, nranks, s);
}

static sf_status sync_failure(cudaError_t e, const char* what);

// process-wide mapped host word for the p2p timeout diagnosis (see wait_ge)
static unsigned long long* g_err_host = nullptr;
static unsigned long long* g_err_dev = nullptr;
static std::mutex g_err_mu;

static void ensure_err_word() {
    std::lock_guard<std::mutex> lk(g_err_mu);
    if (g_err_host) return;
    void* h = nullptr;
    void* d = nullptr;
    if (cudaHostAlloc(&h, 64, cudaHostAllocMapped) == cudaSuccess &&
        cudaHostGetDevicePointer(&d, h, 0) == cudaSuccess) {
        memset(h, 0, 64);
        g_err_host = (unsigned long long*)h;
        g_err_dev = (unsigned long long*)d;
    } else {
        cudaGetLastError();
    }
}

static P2PPeers peers_init() {
    P2PPeers pe = {};
    ensure_err_word();
    pe.err = g_err_dev;
    static const double secs = getenv("SF_P2P_TIMEOUT_S") ? atof(getenv("SF_P2P_TIMEOUT_S")) : 60.0;
    pe.timeout_ns = (unsigned long long)(std::max(secs, 1e-3) * 1e9);
    return pe;
}

// Status of a CUDA call that returned e; a timed-out peer wait is named (the
// trap it caused is a sticky error, so whichever call sees it first reports it).
sf_status sf_cuda_failure(cudaError_t e, const char* what) { return sync_failure(e, what); }

static sf_status sync_failure(cudaError_t e, const char* what) {
    const unsigned long long w = g_err_host ? *(volatile unsigned long long*)g_err_host : 0ull;
    if (w >> 63)
        return sf_fail(SF_ERR_CUDA,
                       "%s: p2p peer wait timed out (%s flag of peer slot %d, op %llu; the peer "
                       "rank is dead, hung or off the op sequence): %s",
                       what, ((w >> 56) & 0x7f) == 1 ? "ready" : "consumed", (int)((w >> 40) & 0xffff),
                       w & 0xffffffffffull, cudaGetErrorString(e));
    return sf_fail(SF_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

// Host synchronisation of a level's stream.  With the NCCL transport the wait
// polls ncclCommGetAsyncError (a peer's failure aborts the communicator instead
// of blocking forever; SF_NCCL_TIMEOUT_S bounds the wait, default 600 s).
sf_status sf_stream_sync(sf_level* L) {
    const sf_comm* c = L->comm ? L->comm : L->rep_comm;
    if (c && c->kind == 1 && c->nccl && g_nccl.asyncErr) {
        static const double secs =
            getenv("SF_NCCL_TIMEOUT_S") ? atof(getenv("SF_NCCL_TIMEOUT_S")) : 600.0;
        const auto t0 = std::chrono::steady_clock::now();
        for (;;) {
            cudaError_t e = cudaStreamQuery(L->stream);
            if (e == cudaSuccess) return SF_OK;
            if (e != cudaErrorNotReady) return sync_failure(e, "stream");
            ncclResult_t ar = ncclSuccess;
            if (g_nccl.asyncErr((ncclComm_t)c->nccl, &ar) != ncclSuccess ||
                (ar != ncclSuccess && ar != ncclInProgress)) {
                g_nccl.abort((ncclComm_t)c->nccl);
                const_cast<sf_comm*>(c)->nccl = nullptr;
                return sf_fail(SF_ERR_NCCL, "NCCL asynchronous error: %s",
                               g_nccl.errStr ? g_nccl.errStr(ar) : "?");
            }
            if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > secs) {
                g_nccl.abort((ncclComm_t)c->nccl);
                const_cast<sf_comm*>(c)->nccl = nullptr;
                return sf_fail(SF_ERR_NCCL, "NCCL wait exceeded %.0f s (SF_NCCL_TIMEOUT_S); "
                               "communicator aborted", secs);
            }
            // spin for the first millisecond (a solve cycle's sync), then back off
            if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > 1e-3)
                std::this_thread::sleep_for(std::chrono::microseconds(50));
        }
    }
    cudaError_t e = cudaStreamSynchronize(L->stream);
    if (e != cudaSuccess) return sync_failure(e, "stream");
    return SF_OK;
}

static unsigned long long* peer_sync(const sf_level* L, int r) {
    return (unsigned long long*)(L->peer[r] + ((const char*)L->dsync - (const char*)L->buf));
}

sf_status sf_ipc_register(sf_level* L, const sf_comm* c) {
    if (!c || (c->kind != 2 && c->kind != 3)) return SF_OK;
    if (c->kind == 3) {   // fresh sync block (the buffer may be recycled memory)
        SF_CUDA(cudaMemsetAsync(L->dsync, 0, SF_SCRATCH_BYTES - 256, L->stream));
    }
    SF_CUDA(cudaStreamSynchronize(L->stream));
    // base of the allocation holding the level buffer (a torch block may sit inside one)
    static decltype(&cuMemGetAddressRange) range = nullptr;
    if (!range) {
        cudaDriverEntryPointQueryResult q;
        void* fn = nullptr;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) !=
                cudaSuccess || !fn)
            return sf_fail(SF_ERR_CUDA, "cuMemGetAddressRange unavailable");
        range = (decltype(range))fn;
    }
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)L->buf) != CUDA_SUCCESS)
        return sf_fail(SF_ERR_CUDA, "cuMemGetAddressRange failed");
    struct Rec {
        cudaIpcMemHandle_t h;
        unsigned long long off;
        int ok;
    } mine, all[64];
    if (c->nranks > 64) return sf_fail(SF_ERR_INVALID, "hostipc supports <= 64 ranks");
    // every rank reaches both all-gathers whatever fails locally, and all of
    // them return the same error: a rank that cannot export or open a peer
    // buffer must not leave the others waiting (callers fall back collectively)
    memset(&mine, 0, sizeof(mine));
    cudaError_t e = cudaIpcGetMemHandle(&mine.h, (void*)base);
    mine.ok = e == cudaSuccess;
    mine.off = (unsigned long long)((char*)L->buf - (char*)base);
    cudaGetLastError();
    SF_TRY(host_allgather(c, &mine, sizeof(Rec), all));
    int ok = 1;
    for (int r = 0; r < c->nranks; r++) ok &= all[r].ok;
    if (const char* t = getenv("SF_TEST_IPC_FAIL_RANK"))   // tests: one rank cannot open
        if (atoi(t) == c->rank) ok = 0;
    L->peer.assign(c->nranks, nullptr);
    for (int r = 0; r < c->nranks && ok; r++) {
        if (r == c->rank) continue;
        void* p = nullptr;
        e = cudaIpcOpenMemHandle(&p, all[r].h, cudaIpcMemLazyEnablePeerAccess);   // NVLink P2P
        if (e != cudaSuccess) {
            cudaGetLastError();
            ok = 0;
            break;
        }
        L->ipc_opened.push_back(p);
        L->peer[r] = (char*)p + all[r].off;
    }
    int oks[64];
    SF_TRY(host_allgather(c, &ok, sizeof(int), oks));   // doubles as the barrier
    for (int r = 0; r < c->nranks; r++)
        if (!oks[r]) {
            sf_ipc_close(L);
            return sf_fail(SF_ERR_CUDA, "CUDA IPC: rank %d could not export or open a peer level buffer (%s)",
                           r, cudaGetErrorString(e));
        }
    return SF_OK;
}

void sf_ipc_close(sf_level* L) {
    for (void* p : L->ipc_opened) cudaIpcCloseMemHandle(p);
    L->ipc_opened.clear();
    L->peer.clear();
}

extern "C" sf_status sf_comm_destroy(sf_comm* c) {
    if (!c) return SF_OK;
    if (c->kind == 1 && c->nccl) g_nccl.commDestroy((ncclComm_t)c->nccl);
    delete c;
    return SF_OK;
}

// Transport self-test: every NCCL collective the slab path uses, once, on a
// few device doubles, results checked on the host.
extern "C" sf_status sf_comm_check(const sf_comm* c, void* stream) {
    if (!c) return sf_fail(SF_ERR_INVALID, "NULL comm");
    if (c->kind != 1) return SF_OK;
    if (!c->nccl) return sf_fail(SF_ERR_NCCL, "communicator was aborted");
    cudaStream_t s = (cudaStream_t)stream;
    ncclComm_t nc = (ncclComm_t)c->nccl;
    const int n = c->nranks, r = c->rank;
    const int G = 4;   // all-gather doubles per rank
    std::vector<double> h(8 + (size_t)G * n + 4, 0.0);
    h[0] = r;          // all-reduce max
    h[1] = r + 1;      // all-reduce sum
    h[2] = (r == n - 1) ? 1000.0 + r : -1.0;   // broadcast from the last rank
    h[3] = 100.0 + r;  // ring send
    for (int i = 0; i < G; i++) h[8 + (size_t)G * r + i] = 10.0 * r + i;
    double* d = nullptr;
    SF_CUDA(cudaMalloc(&d, h.size() * sizeof(double)));
    sf_status st = SF_OK;
    auto nccl = [&](ncclResult_t e, const char* what) {
        if (e != ncclSuccess && st == SF_OK)
            st = sf_fail(SF_ERR_NCCL, "%s: %s", what, g_nccl.errStr ? g_nccl.errStr(e) : "?");
    };
    if (cudaMemcpyAsync(d, h.data(), h.size() * sizeof(double), cudaMemcpyHostToDevice, s) != cudaSuccess)
        st = sf_fail(SF_ERR_CUDA, "upload");
    if (st == SF_OK) nccl(g_nccl.allReduce(d, d, 1, ncclDouble, ncclMax, nc, s), "ncclAllReduce(max)");
    if (st == SF_OK) nccl(g_nccl.allReduce(d + 1, d + 1, 1, ncclDouble, ncclSum, nc, s), "ncclAllReduce(sum)");
    if (st == SF_OK) nccl(g_nccl.broadcast(d + 2, d + 2, 1, ncclDouble, n - 1, nc, s), "ncclBroadcast");
    if (st == SF_OK)
        nccl(g_nccl.allGather(d + 8 + (size_t)G * r, d + 8, G, ncclDouble, nc, s), "ncclAllGather");
    if (st == SF_OK && n > 1) {   // ring point-to-point, as the halo exchange groups it
        nccl(g_nccl.groupStart(), "ncclGroupStart");
        if (st == SF_OK) nccl(g_nccl.send(d + 3, 1, ncclDouble, (r + 1) % n, nc, s), "ncclSend");
        if (st == SF_OK) nccl(g_nccl.recv(d + 4, 1, ncclDouble, (r + n - 1) % n, nc, s), "ncclRecv");
        nccl(g_nccl.groupEnd(), "ncclGroupEnd");
    }
    if (st == SF_OK &&
        cudaMemcpyAsync(h.data(), d, h.size() * sizeof(double), cudaMemcpyDeviceToHost, s) != cudaSuccess)
        st = sf_fail(SF_ERR_CUDA, "download");
    if (st == SF_OK) {
        sf_level tmp;   // a level shell carrying the stream and the comm for the polled wait
        tmp.comm = c;
        tmp.rep_comm = nullptr;
        tmp.stream = s;
        st = sf_stream_sync(&tmp);
    }
    cudaFree(d);
    if (st != SF_OK) return st;
    bool ok = h[0] == n - 1 && h[1] == 0.5 * n * (n + 1) && h[2] == 1000.0 + (n - 1);
    for (int q = 0; q < n; q++)
        for (int i = 0; i < G; i++) ok = ok && h[8 + (size_t)G * q + i] == 10.0 * q + i;
    if (n > 1) ok = ok && h[4] == 100.0 + (r + n - 1) % n;
    if (!ok) return sf_fail(SF_ERR_NCCL, "NCCL self-test returned wrong values");
    return SF_OK;
}

extern "C" sf_status sf_comm_info(const sf_comm* c, int* nparts, int* nlocal, int* first) {
    if (!c) return sf_fail(SF_ERR_INVALID, "NULL comm");
    if (nparts) *nparts = c->nparts;
    if (nlocal) *nlocal = c->nlocal;
    if (first) *first = c->first;
    return SF_OK;
}

sf_status sf_halo(sf_level* L, int field, int depth) { return sf_halo_on(L, field, depth, L->stream); }

sf_status sf_halo_on(sf_level* L, int field, int depth, cudaStream_t stream) {
    if (L->nparts <= 1 || !L->comm) return SF_OK;
    // beside a running sweep (stream != the level's) the device-initiated copy
    // keeps to a few CTAs: the sweep leaves only a couple of SMs free
    const int max_ctas = stream == L->stream ? 148 : 16;
    if (depth > SF_GZ || depth > L->lnz) return sf_fail(SF_ERR_SHAPE, "halo depth %d too deep", depth);
    size_t cnt = (size_t)depth * L->ks;
    const long lo_src = (long)SF_GZ * L->ks;                  // planes [0, d)
    const long hi_src = (long)(L->lnz - depth + SF_GZ) * L->ks;  // planes [lnz-d, lnz)
    const long lo_dst = (long)(SF_GZ - depth) * L->ks;        // ghosts [-d, 0)
    const long hi_dst = (long)(L->lnz + SF_GZ) * L->ks;       // ghosts [lnz, lnz+d)
    if (L->comm->kind == 0) {
        for (int q = 0; q + 1 < L->nlocal; q++) {
            double* lo = L->parts[q].f[field];
            double* hi = L->parts[q + 1].f[field];
            SF_CUDA(cudaMemcpyAsync(hi + lo_dst, lo + hi_src, cnt * sizeof(double),
                                    cudaMemcpyDeviceToDevice, stream));
            SF_CUDA(cudaMemcpyAsync(lo + hi_dst, hi + lo_src, cnt * sizeof(double),
                                    cudaMemcpyDeviceToDevice, stream));
        }
        return SF_OK;
    }
    if (L->comm->kind == 3) {  // device-initiated: neighbours' planes over peer memory
        const sf_comm* c = L->comm;
        const int r = c->rank, n = c->nranks;
        double* x = L->parts[0].f[field];
        P2PPeers pe = peers_init();
        const double* lo_x = nullptr;
        const double* hi_x = nullptr;
        if (r > 0) { pe.sync[0] = peer_sync(L, r - 1); lo_x = peer_field(L, r - 1, x); }
        if (r < n - 1) { pe.sync[1] = peer_sync(L, r + 1); hi_x = peer_field(L, r + 1, x); }
        const int grid = (int)std::min<long>(max_ctas, ((long)cnt + 255) / 256);
        sf_launch(p2p_halo_kernel, grid, 256, 0, stream, x, lo_x, hi_x, L->dsync, pe, lo_dst, hi_src, hi_dst,
                                                     lo_src, (long)cnt);
        SF_LAUNCHED();
        return sf_check_launch("p2p_halo");
    }
    if (L->comm->kind == 2) {  // pull the neighbours' boundary planes through IPC
        const sf_comm* c = L->comm;
        int r = c->rank, n = c->nranks;
        double* x = L->parts[0].f[field];
        SF_CUDA(cudaStreamSynchronize(L->stream));
        SF_TRY(host_barrier(c));
        if (r > 0)
            SF_CUDA(cudaMemcpyAsync(x + lo_dst, peer_field(L, r - 1, x) + hi_src, cnt * sizeof(double),
                                    cudaMemcpyDeviceToDevice, L->stream));
        if (r < n - 1)
            SF_CUDA(cudaMemcpyAsync(x + hi_dst, peer_field(L, r + 1, x) + lo_src, cnt * sizeof(double),
                                    cudaMemcpyDeviceToDevice, L->stream));
        SF_CUDA(cudaStreamSynchronize(L->stream));
        return host_barrier(c);
    }
    ncclComm_t comm = (ncclComm_t)L->comm->nccl;
    int r = L->comm->rank, n = L->comm->nranks;
    double* x = L->parts[0].f[field];
    SF_NCCL(g_nccl.groupStart());
    if (r > 0) {
        SF_NCCL(g_nccl.send(x + lo_src, cnt, ncclDouble, r - 1, comm, stream));
        SF_NCCL(g_nccl.recv(x + lo_dst, cnt, ncclDouble, r - 1, comm, stream));
    }
    if (r < n - 1) {
        SF_NCCL(g_nccl.send(x + hi_src, cnt, ncclDouble, r + 1, comm, stream));
        SF_NCCL(g_nccl.recv(x + hi_dst, cnt, ncclDouble, r + 1, comm, stream));
    }
    SF_NCCL(g_nccl.groupEnd());
    return SF_OK;
}

sf_status sf_agglomerate(sf_level* C, int field, int parts, int lnz_per_part) {
    // Loopback: every fine part is local and already wrote its planes.
    const sf_comm* cm = C->rep_comm;
    if (!cm || cm->kind == 0) return SF_OK;
    if (cm->nranks != parts) return sf_fail(SF_ERR_SHAPE, "agglomeration across %d parts", parts);
    if (cm->kind == 3) {  // device-initiated gather over peer memory
        double* base = C->parts[0].f[field] + (long)SF_GZ * C->ks;
        const long cnt = (long)lnz_per_part * C->ks;
        P2PPeers pe = peers_init();
        P2PPtrs pb = {};
        for (int q = 0; q < parts; q++)
            if (q != cm->rank) {
                pe.sync[q] = peer_sync(C, q);
                pb.p[q] = peer_field(C, q, base);
            }
        double* top = base + (size_t)C->gnz * C->ks;
        const double* ptop = (field == SF_BETA_K && cm->rank != parts - 1) ? peer_field(C, parts - 1, top)
                                                                           : nullptr;
        const int grid = (int)std::min<long>(148, (cnt + 255) / 256);
        sf_launch(p2p_gather_kernel, grid, 256, 0, C->stream, base, pb, C->dsync, pe, parts, cm->rank, cnt, top,
                                                       ptop, C->ks);
        SF_LAUNCHED();
        return sf_check_launch("p2p_gather");
    }
    if (cm->kind == 2) {  // every rank copies the other ranks' planes from their buffers
        double* base = C->parts[0].f[field] + (long)SF_GZ * C->ks;
        size_t cnt = (size_t)lnz_per_part * C->ks;
        SF_CUDA(cudaStreamSynchronize(C->stream));
        SF_TRY(host_barrier(cm));
        for (int q = 0; q < parts; q++) {
            if (q == cm->rank) continue;
            SF_CUDA(cudaMemcpyAsync(base + q * cnt, peer_field(C, q, base) + q * cnt,
                                    cnt * sizeof(double), cudaMemcpyDeviceToDevice, C->stream));
        }
        if (field == SF_BETA_K && cm->rank != parts - 1) {
            double* top = base + (size_t)C->gnz * C->ks;
            SF_CUDA(cudaMemcpyAsync(top, peer_field(C, parts - 1, top), C->ks * sizeof(double),
                                    cudaMemcpyDeviceToDevice, C->stream));
        }
        SF_CUDA(cudaStreamSynchronize(C->stream));
        return host_barrier(cm);
    }
    ncclComm_t comm = (ncclComm_t)cm->nccl;
    double* base = C->parts[0].f[field] + (long)SF_GZ * C->ks;
    size_t cnt = (size_t)lnz_per_part * C->ks;
    SF_NCCL(g_nccl.allGather(base + cm->rank * cnt, base, cnt, ncclDouble, comm, C->stream));
    if (field == SF_BETA_K) {  // the top boundary face belongs to the last part only
        double* top = base + (size_t)C->gnz * C->ks;
        SF_NCCL(g_nccl.broadcast(top, top, C->ks, ncclDouble, parts - 1, comm, C->stream));
    }
    return SF_OK;
}

sf_status sf_allreduce_scalar(sf_level* L, const sf_comm* cm, double* dev, int op) {
    if (!cm || cm->kind == 0 || cm->nranks == 1) return SF_OK;
    cudaStream_t s = L->stream;
    if (cm->kind == 3) {
        P2PPeers pe = peers_init();
        P2PPtrs sl = {};
        for (int q = 0; q < cm->nranks; q++) {
            if (q != cm->rank) pe.sync[q] = peer_sync(L, q);
            sl.p[q] = (const double*)((q == cm->rank ? L->dsync : peer_sync(L, q)) + 8);
        }
        sf_launch(p2p_allreduce_kernel, 1, 32, 0, s, dev, L->dsync, pe, sl, cm->nranks, op);
        SF_LAUNCHED();
        return sf_check_launch("p2p_allreduce");
    }
    if (cm->kind == 2) {
        double v;
        SF_CUDA(cudaMemcpyAsync(&v, dev, sizeof(double), cudaMemcpyDeviceToHost, s));
        SF_CUDA(cudaStreamSynchronize(s));
        std::vector<double> all(cm->nranks);
        SF_TRY(host_allgather(cm, &v, sizeof(double), all.data()));
        double r = all[0];
        for (int q = 1; q < cm->nranks; q++)
            r = op == 0 ? ((all[q] > r || all[q] != all[q]) ? all[q] : r) : r + all[q];
        SF_CUDA(cudaMemcpyAsync(dev, &r, sizeof(double), cudaMemcpyHostToDevice, s));
        SF_CUDA(cudaStreamSynchronize(s));
        return SF_OK;
    }
    SF_NCCL(g_nccl.allReduce(dev, dev, 1, ncclDouble, op == 0 ? ncclMax : ncclSum,
                             (ncclComm_t)cm->nccl, s));
    return SF_OK;
}

// Depth-2 x halo + fused RB pair with the exchange hidden under the interior
// (SURVEY 8e performance variant).  On a multi-part level the halo runs on a
// side stream (fork/join by events, so CUDA graphs capture it) while the
// interior z-chunks [1, nch-1) are smoothed -- they read no ghost plane -- and
// the boundary chunks 0 and nch-1 run after the join.  Same arithmetic per
// cell as one launch over all chunks (bit-identical).  SF_HALO_OVERLAP=0 turns
// it off (exchange, then one launch).
sf_status k_gsrb_pair_halo(sf_level* L, int xin, int xout, int rhs, double a, double b, double* rmax,
                           sf_level* C, int cf, int rmode) {
    const char* ev = getenv("SF_HALO_OVERLAP");
    const int ov = ev ? atoi(ev) : -1;   // 1 always split, 0 never, -1 (default) by cost
    bool split = ov != 0 && L->nparts > 1 && L->comm && L->comm->kind != 2 && L->lnz >= 24;
    if (split && ov < 0) {
        // Overlap pays when the exchange it hides costs more than the boundary
        // launch it adds: that launch walks 2 * tiles two-plane items (5 z steps
        // each) over the resident CTAs, ~G * 512 cells * 56 B per step at
        // ~5.5 TB/s; the exchange moves 2 neighbours x 2 planes, ~10 us of flag
        // synchronisation plus the bytes at ~600 GB/s over NVLink (a copy
        // engine on one device: ~3 us + 2.5 TB/s).  With NVLink both grow with
        // the plane area at similar rates (bench's 512^2..1024^2 slabs: no split),
        // the fixed synchronisation cost makes small planes split.
        const double plane = (double)L->nx * L->ny;
        const bool local = L->comm->kind == 0;
        const double t_halo = (local ? 3e-6 : 10e-6) + 4.0 * plane * 8.0 / (local ? 2.5e12 : 6e11);
        const double tiles = plane / 512.0, G = 148.0;
        const double t_step = G * 512.0 * 56.0 / 5.5e12;
        const double t_split = std::ceil(2.0 * tiles / G) * 5.0 * t_step;
        split = t_halo > t_split;
    }
    if (!split) {
        SF_TRY(sf_halo(L, xin, 2));
        return k_gsrb_pair_fused(L, xin, xout, rhs, a, b, rmax, C, cf, 0, 0, rmode);
    }
    if (!L->side) {
        SF_CUDA(cudaStreamCreateWithFlags(&L->side, cudaStreamNonBlocking));
        SF_CUDA(cudaEventCreateWithFlags(&L->ev_fork, cudaEventDisableTiming));
        SF_CUDA(cudaEventCreateWithFlags(&L->ev_join, cudaEventDisableTiming));
    }
    SF_CUDA(cudaEventRecord(L->ev_fork, L->stream));
    SF_CUDA(cudaStreamWaitEvent(L->side, L->ev_fork, 0));
    SF_TRY(sf_halo_on(L, xin, 2, L->side));
    SF_CUDA(cudaEventRecord(L->ev_join, L->side));
    // copy-engine transfers (kind 0) need no SM; kernels / NCCL get two
    const int reserve = L->comm->kind == 0 ? 0 : 2;
    SF_TRY(k_gsrb_pair_fused(L, xin, xout, rhs, a, b, rmax, C, cf, 1, reserve, rmode));
    SF_CUDA(cudaStreamWaitEvent(L->stream, L->ev_join, 0));
    return k_gsrb_pair_fused(L, xin, xout, rhs, a, b, rmax, C, cf, 2, 0, rmode);
}
