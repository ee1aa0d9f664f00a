// Generic strided-domain stencils: the paper's language core
// (Table I, Fig 4) with a run-time CUDA micro-compiler for
// sm_100a, the B200 counterpart of Snowflake's JIT backends.
//
//   sf_stencil_compile   validate the expression DAGs + domain unions of a
//                        StencilGroup and render ONE CUDA kernel for it
//                        (a switch over the group's stencils; each thread owns
//                        one domain point of one RectDomain);
//   sf_stencil_apply     resolve the size-relative domains on the level, run
//                        the paper's Diophantine dependence analysis
//                         -- exact lattice intersection of
//                        strided rects by the extended Euclidean algorithm --
//                        to reject racy in-place stencils and to pack
//                        consecutive independent stencils into one launch
//                        (greedy barrier placement), compile
//                        with NVRTC on first use, and launch per phase.
//
// The generated kernel evaluates the DAG in its stored order with IEEE
// operations (NVRTC --fmad=false, IEEE division): the result is the oracle's
// (oracle/stencil.py) bit for bit.  HBM-bound like every stencil here; the
// hand-written kernels remain the hot path, this is the general engine.
#include <cuda.h>
#include <dlfcn.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <sstream>

#include "sf_internal.h"

namespace {

// ------------------------------------------------------------------ NVRTC
struct Nvrtc {
    bool tried = false, ok = false;
    int (*create)(void**, const char*, const char*, int, const char* const*, const char* const*);
    int (*compile)(void*, int, const char* const*);
    int (*log_size)(void*, size_t*);
    int (*log)(void*, char*);
    int (*cubin_size)(void*, size_t*);
    int (*cubin)(void*, char*);
    int (*destroy)(void**);
};
Nvrtc g_rtc;
std::mutex g_rtc_mu;

sf_status load_nvrtc() {
    std::lock_guard<std::mutex> lk(g_rtc_mu);
    if (g_rtc.tried) return g_rtc.ok ? SF_OK : sf_fail(SF_ERR_CUDA, "libnvrtc.so.12 not found");
    g_rtc.tried = true;
    const char* names[] = {"libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so"};
    void* h = nullptr;
    for (const char* n : names)
        if ((h = dlopen(n, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) return sf_fail(SF_ERR_CUDA, "libnvrtc.so.12 not found");
#define SF_RTC_SYM(field, name)                                                \
    *(void**)&g_rtc.field = dlsym(h, name);                                   \
    if (!g_rtc.field) return sf_fail(SF_ERR_CUDA, "NVRTC symbol %s missing", name);
    SF_RTC_SYM(create, "nvrtcCreateProgram");
    SF_RTC_SYM(compile, "nvrtcCompileProgram");
    SF_RTC_SYM(log_size, "nvrtcGetProgramLogSize");
    SF_RTC_SYM(log, "nvrtcGetProgramLog");
    SF_RTC_SYM(cubin_size, "nvrtcGetCUBINSize");
    SF_RTC_SYM(cubin, "nvrtcGetCUBIN");
    SF_RTC_SYM(destroy, "nvrtcDestroyProgram");
#undef SF_RTC_SYM
    g_rtc.ok = true;
    return SF_OK;
}

// driver entry points (the runtime's primary context is current)
struct Drv {
    bool ok = false;
    CUresult (*load)(CUmodule*, const void*);
    CUresult (*get)(CUfunction*, CUmodule, const char*);
    CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                       unsigned, CUstream, void**, void**);
    CUresult (*unload)(CUmodule);
    CUresult (*occ)(int*, CUfunction, int, size_t);
};
Drv g_drv;

sf_status load_driver() {
    if (g_drv.ok) return SF_OK;
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
#define SF_DRV_SYM(field, name)                                                          \
    if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) \
        return sf_fail(SF_ERR_CUDA, "driver entry point %s unavailable", name);          \
    *(void**)&g_drv.field = fn;
    SF_DRV_SYM(load, "cuModuleLoadData");
    SF_DRV_SYM(get, "cuModuleGetFunction");
    SF_DRV_SYM(launch, "cuLaunchKernel");
    SF_DRV_SYM(unload, "cuModuleUnload");
    SF_DRV_SYM(occ, "cuOccupancyMaxActiveBlocksPerMultiprocessor");
#undef SF_DRV_SYM
    g_drv.ok = true;
    return SF_OK;
}

// ------------------------------------------------------------------ IR
struct Rect {
    int lo[3], hi[3], st[3];
};
struct St {
    std::vector<sf_sx_node> nodes;
    int root, out;
    std::vector<Rect> rects;
};

// a resolved (size-bound) rect: lattice lo + st*i, i in [0, cnt)
struct RR {
    long lo[3], st[3], cnt[3];
    bool empty() const { return cnt[0] <= 0 || cnt[1] <= 0 || cnt[2] <= 0; }
    long last(int d) const { return lo[d] + st[d] * (cnt[d] - 1); }
};

bool is_identity(const sf_sx_node& n) {
    for (int d = 0; d < 3; d++)
        if (n.mul[d] != 1 || n.div[d] != 1 || n.pre[d] != 0) return false;
    return true;
}

long fdiv(long a, long b) {   // floor division, b > 0
    long q = a / b;
    return (q * b > a) ? q - 1 : q;
}
long amap(const sf_sx_node& n, int d, long p) {
    return fdiv((long)n.mul[d] * p + n.pre[d], n.div[d]) + n.off[d];
}

// ------------------------------------------------------------------ analysis
long egcd(long a, long b, long& x, long& y) {
    if (b == 0) { x = 1; y = 0; return a; }
    long x1, y1;
    long g = egcd(b, a % b, x1, y1);
    x = y1;
    y = x1 - (a / b) * y1;
    return g;
}

// do the lattices {a0 + sa i | 0 <= i < ca} and {b0 + sb j | 0 <= j < cb} meet?
// (the affine Diophantine equation sa i - sb j = b0 - a0, solved by the
// extended Euclidean algorithm, then intersected with the bounds)
bool axis_meet(long a0, long sa, long ca, long b0, long sb, long cb) {
    if (ca <= 0 || cb <= 0) return false;
    const long lo = std::max(a0, b0);
    const long hi = std::min(a0 + sa * (ca - 1), b0 + sb * (cb - 1));
    if (lo > hi) return false;
    long u, v;
    const long g = egcd(sa, sb, u, v);   // sa u + sb v = g
    const long diff = b0 - a0;
    if (diff % g != 0) return false;
    const long L = sa / g * sb;
    // x0 = a0 + sa * u * diff/g  solves both congruences; reduce mod L
    long t = (u % (sb / g)) * ((diff / g) % (sb / g)) % (sb / g);
    long x0 = a0 + sa * t;
    x0 = lo + (((x0 - lo) % L) + L) % L;   // smallest solution >= lo
    return x0 <= hi;
}

bool rect_meet(const RR& A, const RR& B) {
    for (int d = 0; d < 3; d++)
        if (!axis_meet(A.lo[d], A.st[d], A.cnt[d], B.lo[d], B.st[d], B.cnt[d])) return false;
    return true;
}

// the set a READ touches over a rect: exact lattice for identity maps, else a
// dense bounding box (conservative)
RR read_image(const sf_sx_node& n, const RR& r) {
    RR o;
    for (int d = 0; d < 3; d++) {
        if (is_identity(n)) {
            o.lo[d] = r.lo[d] + n.off[d];
            o.st[d] = r.st[d];
            o.cnt[d] = r.cnt[d];
        } else {
            const long a = amap(n, d, r.lo[d]), b = amap(n, d, r.last(d));
            o.lo[d] = a;
            o.st[d] = 1;
            o.cnt[d] = r.cnt[d] > 0 ? b - a + 1 : 0;
        }
    }
    return o;
}

// reads of mesh m on the output level by stencil s (src 0, or src 1 when same)
template <class F>
void for_level_reads(const St& s, bool same, F&& f) {
    for (const sf_sx_node& n : s.nodes)
        if (n.op == SF_SX_READ && (n.src == 0 || same)) f(n);
}

RR resolve(const Rect& r, const int n[3], long zlo, long zhi) {
    RR o;
    for (int d = 0; d < 3; d++) {
        const long N = n[d] + 2;
        long lo = r.lo[d] < 0 ? N + r.lo[d] : r.lo[d];
        long hi = r.hi[d] < 0 ? N + r.hi[d] : r.hi[d];
        long st = r.st[d];
        if (st == 0) {   // degenerate axis: the single coordinate lo
            hi = lo + 1;
            st = 1;
        }
        if (d == 2) {   // clip to the part's owned planes
            if (zlo > lo) lo = lo + (zlo - lo + st - 1) / st * st;
            hi = std::min(hi, zhi);
        }
        o.lo[d] = lo;
        o.st[d] = st;
        o.cnt[d] = hi > lo ? (hi - lo + st - 1) / st : 0;
    }
    return o;
}

// is stencil s racy in place (reads of its output mesh at points it writes,
// other than each point's own)?
bool racy(const St& s, const std::vector<RR>& D, bool same) {
    bool bad = false;
    for_level_reads(s, same, [&](const sf_sx_node& n) {
        if (bad || n.mesh != s.out) return;
        const bool self = is_identity(n) && !n.off[0] && !n.off[1] && !n.off[2];
        for (size_t a = 0; a < D.size() && !bad; a++)
            for (size_t b = 0; b < D.size() && !bad; b++) {
                if (self && a == b) continue;   // a point reading itself
                if (rect_meet(read_image(n, D[a]), D[b])) bad = true;
            }
    });
    return bad;
}

// does stencil t depend on stencil s (RAW, WAR or WAW on the output level)?
bool depends(const St& s, const std::vector<RR>& Ds, const St& t, const std::vector<RR>& Dt,
             bool same) {
    auto reads_hit = [&](const St& r, const std::vector<RR>& Dr, int mesh,
                         const std::vector<RR>& Dw) {
        bool hit = false;
        for_level_reads(r, same, [&](const sf_sx_node& n) {
            if (hit || n.mesh != mesh) return;
            for (const RR& a : Dr)
                for (const RR& b : Dw)
                    if (!hit && rect_meet(read_image(n, a), b)) hit = true;
        });
        return hit;
    };
    if (reads_hit(t, Dt, s.out, Ds)) return true;   // RAW
    if (reads_hit(s, Ds, t.out, Dt)) return true;   // WAR
    if (s.out == t.out)                              // WAW
        for (const RR& a : Ds)
            for (const RR& b : Dt)
                if (rect_meet(a, b)) return true;
    return false;
}

// ------------------------------------------------------------------ codegen
const char* kPrelude = R"(// rendered by libsf sf_stencil_compile (NEXT-4 generic stencil engine)
#define SF_MAXR 64
struct SfRect { int lo[3]; int st[3]; int cnt[3]; int ax[3]; int sid; long long start; };
struct SfArgs {
    double* f[2][9];
    long long js[2], ks[2];
    int xb, yb, zb[2];
    int nrect;
    int ilv;            // > 0: the rects share one line lattice; line t -> rect t % ilv
    long long total;
    SfRect r[SF_MAXR];
};
__device__ __forceinline__ int sf_fdiv(int a, int b) { int q = a / b; return (q * b > a) ? q - 1 : q; }
)";

std::string axis_expr(const sf_sx_node& n, int d) {
    static const char* P[3] = {"X", "Y", "Z"};
    std::ostringstream o;
    if (n.mul[d] == 1 && n.div[d] == 1 && n.pre[d] == 0) {
        o << "(" << P[d] << " + (" << n.off[d] << "))";
    } else if (n.div[d] == 1) {
        o << "(" << n.mul[d] << " * " << P[d] << " + (" << (n.pre[d] + n.off[d]) << "))";
    } else {
        o << "(sf_fdiv(" << n.mul[d] << " * " << P[d] << " + (" << n.pre[d] << "), " << n.div[d]
          << ") + (" << n.off[d] << "))";
    }
    return o.str();
}

std::string index_expr(int src, const std::string& x, const std::string& y, const std::string& z) {
    std::ostringstream o;
    o << "((long long)(" << z << " + a.zb[" << src << "]) * a.ks[" << src << "] + (long long)(" << y
      << " + a.yb) * a.js[" << src << "] + (" << x << " + a.xb))";
    return o.str();
}

std::string render(const std::vector<St>& group) {
    std::ostringstream o;
    o << kPrelude;
    // one evaluation function per stencil: the DAG in stored order
    for (size_t s = 0; s < group.size(); s++) {
        const St& st = group[s];
        o << "__device__ __forceinline__ double sf_ev" << s
          << "(const SfArgs& a, const int X, const int Y, const int Z) {\n";
        for (size_t i = 0; i < st.nodes.size(); i++) {
            const sf_sx_node& n = st.nodes[i];
            o << "    const double v" << i << " = ";
            switch (n.op) {
                case SF_SX_CONST: {
                    char buf[64];
                    snprintf(buf, sizeof buf, "%a", n.value);
                    o << buf;
                    break;
                }
                case SF_SX_READ:
                    // read-only path: the phase analysis guarantees no point read
                    // in a launch is written by another point of it
                    o << "__ldg(&a.f[" << n.src << "][" << n.mesh << "]["
                      << index_expr(n.src, axis_expr(n, 0), axis_expr(n, 1), axis_expr(n, 2)) << "])";
                    break;
                case SF_SX_ADD: o << "v" << n.a << " + v" << n.b; break;
                case SF_SX_SUB: o << "v" << n.a << " - v" << n.b; break;
                case SF_SX_MUL: o << "v" << n.a << " * v" << n.b; break;
                case SF_SX_DIV: o << "v" << n.a << " / v" << n.b; break;
                case SF_SX_NEG: o << "-v" << n.a; break;
            }
            o << ";\n";
        }
        o << "    return v" << st.root << ";\n}\n";
    }
    // one block row per (rect, j, k) line of the domain: blockIdx.y walks the
    // lines of all rects of the launch (start = first line of a rect), the x
    // threads the points of the line -- one division per line, coalesced x;
    // each thread evaluates two points before storing either (their loads overlap)
    o << "extern \"C\" __global__ void __launch_bounds__(256) sf_stencil_group(const __grid_constant__ SfArgs a) {\n"
         "    const int step = gridDim.x * blockDim.x;\n"
         "    for (long long row = blockIdx.y; row < a.total; row += gridDim.y) {\n"
         "        int lo, l;\n"
         "        if (a.ilv) {   // interleaved: consecutive lines of all rects plane by plane\n"
         "            lo = (int)(row % a.ilv);\n"
         "            l = (int)(row / a.ilv);\n"
         "        } else {       // rect by rect: last start <= row\n"
         "            lo = 0;\n"
         "            int hi = a.nrect - 1;\n"
         "            while (lo < hi) { int m = (lo + hi + 1) >> 1; if (a.r[m].start <= row) lo = m; else hi = m - 1; }\n"
         "            l = (int)(row - a.r[lo].start);\n"
         "        }\n"
         "        const SfRect& R = a.r[lo];\n"
         "        const int n0 = R.cnt[R.ax[0]], n1 = R.cnt[R.ax[1]];\n"
         "        const int j = l % n1, k = l / n1;\n"
         "        for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n0; i += 2 * step) {\n"
         "        const int i2 = i + step < n0 ? i + step : i;\n"
         "        const int X = R.lo[0] + R.st[0] * (R.ax[0] == 0 ? i : R.ax[1] == 0 ? j : k);\n"
         "        const int Y = R.lo[1] + R.st[1] * (R.ax[0] == 1 ? i : R.ax[1] == 1 ? j : k);\n"
         "        const int Z = R.lo[2] + R.st[2] * (R.ax[0] == 2 ? i : R.ax[1] == 2 ? j : k);\n"
         "        const int X2 = R.lo[0] + R.st[0] * (R.ax[0] == 0 ? i2 : R.ax[1] == 0 ? j : k);\n"
         "        const int Y2 = R.lo[1] + R.st[1] * (R.ax[0] == 1 ? i2 : R.ax[1] == 1 ? j : k);\n"
         "        const int Z2 = R.lo[2] + R.st[2] * (R.ax[0] == 2 ? i2 : R.ax[1] == 2 ? j : k);\n"
         "        switch (R.sid) {\n";
    for (size_t s = 0; s < group.size(); s++) {
        const St& st = group[s];
        o << "        case " << s << ": {\n"
          << "            const double r1 = sf_ev" << s << "(a, X, Y, Z);\n"
          << "            const double r2 = sf_ev" << s << "(a, X2, Y2, Z2);\n"
          << "            a.f[0][" << st.out << "][" << index_expr(0, "X", "Y", "Z") << "] = r1;\n"
          << "            if (i2 != i) a.f[0][" << st.out << "][" << index_expr(0, "X2", "Y2", "Z2")
          << "] = r2;\n"
          << "        } break;\n";
    }
    o << "        }\n        }\n    }\n}\n";
    return o.str();
}

// host mirror of the generated argument block
struct SfRectH {
    int lo[3], st[3], cnt[3], ax[3], sid;
    long long start;
};
struct SfArgsH {
    double* f[2][9];
    long long js[2], ks[2];
    int xb, yb, zb[2];
    int nrect;
    int ilv;
    long long total;
    SfRectH r[SF_STENCIL_MAX_RECTS];
};
static_assert(SF_NFIELDS == 9, "generated SfArgs assumes 9 fields");

}  // namespace

struct sf_stencil {
    std::vector<St> st;
    std::string src;
    CUmodule mod = nullptr;
    CUfunction fn = nullptr;
    int sms = 0;
    int occ[9] = {0};   // resident blocks per SM for 32 << b threads
    int phases = 0;
};

extern "C" sf_status sf_stencil_compile(sf_stencil** out, const sf_stencil_desc* d, int n) {
    if (!out || !d || n < 1) return sf_fail(SF_ERR_INVALID, "NULL argument or empty group");
    *out = nullptr;
    std::vector<St> group;
    for (int s = 0; s < n; s++) {
        const sf_stencil_desc& D = d[s];
        if (D.n_nodes < 1 || !D.nodes || D.root < 0 || D.root >= D.n_nodes)
            return sf_fail(SF_ERR_INVALID, "stencil %d: bad node list / root", s);
        if (D.out_mesh < 0 || D.out_mesh >= SF_NFIELDS)
            return sf_fail(SF_ERR_INVALID, "stencil %d: bad output mesh %d", s, D.out_mesh);
        if (D.n_rects < 1 || D.n_rects > SF_STENCIL_MAX_RECTS || !D.rects)
            return sf_fail(SF_ERR_INVALID, "stencil %d: 1..%d rects", s, SF_STENCIL_MAX_RECTS);
        St st;
        st.root = D.root;
        st.out = D.out_mesh;
        for (int i = 0; i < D.n_nodes; i++) {
            const sf_sx_node& x = D.nodes[i];
            const bool bin = x.op == SF_SX_ADD || x.op == SF_SX_SUB || x.op == SF_SX_MUL ||
                             x.op == SF_SX_DIV;
            if (x.op < SF_SX_CONST || x.op > SF_SX_NEG)
                return sf_fail(SF_ERR_INVALID, "stencil %d node %d: bad op %d", s, i, x.op);
            if ((bin || x.op == SF_SX_NEG) && (x.a < 0 || x.a >= i))
                return sf_fail(SF_ERR_INVALID, "stencil %d node %d: operand a", s, i);
            if (bin && (x.b < 0 || x.b >= i))
                return sf_fail(SF_ERR_INVALID, "stencil %d node %d: operand b", s, i);
            if (x.op == SF_SX_CONST && !std::isfinite(x.value))
                return sf_fail(SF_ERR_INVALID, "stencil %d node %d: non-finite constant", s, i);
            if (x.op == SF_SX_READ) {
                if (x.mesh < 0 || x.mesh >= SF_NFIELDS || (x.src != 0 && x.src != 1))
                    return sf_fail(SF_ERR_INVALID, "stencil %d node %d: bad mesh/src", s, i);
                for (int k = 0; k < 3; k++)
                    if (x.mul[k] < 1 || x.div[k] < 1 || x.mul[k] > 64 || x.div[k] > 64 ||
                        std::abs(x.off[k]) > 64 || std::abs(x.pre[k]) > 64)
                        return sf_fail(SF_ERR_INVALID, "stencil %d node %d: bad affine map", s, i);
            }
            st.nodes.push_back(x);
        }
        for (int r = 0; r < D.n_rects; r++) {
            Rect R;
            for (int k = 0; k < 3; k++) {
                R.lo[k] = D.rects[r].lo[k];
                R.hi[k] = D.rects[r].hi[k];
                R.st[k] = D.rects[r].stride[k];
                if (R.st[k] < 0) return sf_fail(SF_ERR_INVALID, "stencil %d rect %d: stride < 0", s, r);
            }
            st.rects.push_back(R);
        }
        group.push_back(std::move(st));
    }
    sf_stencil* S = new sf_stencil();
    S->st = std::move(group);
    S->src = render(S->st);
    *out = S;
    return SF_OK;
}

extern "C" sf_status sf_stencil_source(const sf_stencil* s, char* buf, size_t cap, size_t* len) {
    if (!s) return sf_fail(SF_ERR_INVALID, "NULL stencil");
    if (len) *len = s->src.size();
    if (buf && cap) {
        size_t m = std::min(cap - 1, s->src.size());
        memcpy(buf, s->src.data(), m);
        buf[m] = 0;
    }
    return SF_OK;
}

extern "C" sf_status sf_stencil_phases(const sf_stencil* s, int* phases) {
    if (!s || !phases) return sf_fail(SF_ERR_INVALID, "NULL argument");
    *phases = s->phases;
    return SF_OK;
}

extern "C" sf_status sf_stencil_destroy(sf_stencil* s) {
    if (!s) return SF_OK;
    if (s->mod && g_drv.ok) g_drv.unload(s->mod);
    delete s;
    return SF_OK;
}

static sf_status jit(sf_stencil* s) {
    if (s->fn) return SF_OK;
    SF_TRY(load_nvrtc());
    SF_TRY(load_driver());
    int dev;
    SF_CUDA(cudaGetDevice(&dev));
    cudaDeviceProp p;
    SF_CUDA(cudaGetDeviceProperties(&p, dev));
    if (p.major != 10 || p.minor != 0)
        return sf_fail(SF_ERR_CUDA, "stencil JIT targets sm_100a; device is sm_%d%d", p.major, p.minor);
    void* prog = nullptr;
    if (g_rtc.create(&prog, s->src.c_str(), "sf_stencil.cu", 0, nullptr, nullptr) != 0)
        return sf_fail(SF_ERR_CUDA, "nvrtcCreateProgram failed");
    const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "--fmad=false",
                          "--prec-div=true", "--prec-sqrt=true", "-lineinfo"};
    int rc = g_rtc.compile(prog, 6, opts);
    if (rc != 0) {
        size_t n = 0;
        g_rtc.log_size(prog, &n);
        std::string log(n, '\0');
        if (n) g_rtc.log(prog, &log[0]);
        g_rtc.destroy(&prog);
        return sf_fail(SF_ERR_CUDA, "NVRTC compile failed: %.400s", log.c_str());
    }
    size_t n = 0;
    g_rtc.cubin_size(prog, &n);
    std::vector<char> cubin(n);
    g_rtc.cubin(prog, cubin.data());
    g_rtc.destroy(&prog);
    SF_CUDA(cudaFree(nullptr));   // make the primary context current
    if (g_drv.load(&s->mod, cubin.data()) != CUDA_SUCCESS)
        return sf_fail(SF_ERR_CUDA, "cuModuleLoadData failed");
    if (g_drv.get(&s->fn, s->mod, "sf_stencil_group") != CUDA_SUCCESS)
        return sf_fail(SF_ERR_CUDA, "cuModuleGetFunction failed");
    s->sms = p.multiProcessorCount;
    for (int b = 0; b < 4; b++)   // 32, 64, 128, 256 threads
        if (g_drv.occ(&s->occ[b], s->fn, 32 << b, 0) != CUDA_SUCCESS || s->occ[b] < 1) s->occ[b] = 1;
    return SF_OK;
}

// the race / dependence structure of the group on a grid of gdim cells (the
// same on every z-slab part): reject racy stencils, pack phases greedily
static sf_status analyse(const sf_stencil* s, const int gdim[3], bool same,
                         std::vector<std::vector<int>>& phases) {
    const int ng = (int)s->st.size();
    std::vector<std::vector<RR>> G(ng);
    for (int i = 0; i < ng; i++)
        for (const Rect& r : s->st[i].rects) G[i].push_back(resolve(r, gdim, LONG_MIN / 4, LONG_MAX / 4));
    for (int i = 0; i < ng; i++)
        if (racy(s->st[i], G[i], same))
            return sf_fail(SF_ERR_INVALID,
                           "stencil %d of the group reads points of its output mesh that it writes "
                           "(loop-carried dependence, Diophantine test): write out of place", i);
    phases.clear();
    for (int i = 0; i < ng; i++) {
        bool dep = phases.empty();
        if (!dep)
            for (int j : phases.back())
                if (depends(s->st[j], G[j], s->st[i], G[i], same)) { dep = true; break; }
        if (dep) phases.emplace_back();
        phases.back().push_back(i);
    }
    return SF_OK;
}

extern "C" sf_status sf_stencil_plan(const sf_stencil* s, int gnx, int gny, int gnz, int src_is_output,
                                     int* nphases) {
    if (!s || !nphases || gnx < 1 || gny < 1 || gnz < 1) return sf_fail(SF_ERR_INVALID, "bad arguments");
    const int gdim[3] = {gnx, gny, gnz};
    std::vector<std::vector<int>> ph;
    SF_TRY(analyse(s, gdim, src_is_output != 0, ph));
    *nphases = (int)ph.size();
    return SF_OK;
}

// storage window of a level part in stencil coordinates, per axis [lo, hi)
static void window(const sf_level* L, int z0, long lo[3], long hi[3]) {
    lo[0] = 1 - SF_OX;            hi[0] = L->js - SF_OX + 1;
    lo[1] = 1 - SF_GY;            hi[1] = L->ny + SF_GY + 1;
    lo[2] = 1 + z0 - SF_GZ;       hi[2] = z0 + L->lnz + SF_GZ + 1;
}

extern "C" sf_status sf_stencil_apply(sf_stencil* s, sf_level* L, sf_level* Src) {
    if (!s || !L) return sf_fail(SF_ERR_INVALID, "NULL argument");
    const bool same = (Src == nullptr || Src == L);
    sf_level* S = same ? L : Src;
    const bool uses_src = [&] {
        for (const St& t : s->st)
            for (const sf_sx_node& n : t.nodes)
                if (n.op == SF_SX_READ && n.src == 1) return true;
        return false;
    }();
    const bool multi = L->nparts > 1;
    if (!same && uses_src && (multi || S->nparts > 1 || L->nlocal != 1 || S->nlocal != 1))
        return sf_fail(SF_ERR_INVALID, "cross-level stencils need single-part levels");
    const int gdim[3] = {L->gnx, L->gny, L->gnz};
    const int ng = (int)s->st.size();
    std::vector<std::vector<int>> phases;
    SF_TRY(analyse(s, gdim, same, phases));
    // multi-part: same-level reads only with plain offsets; z halo depth per mesh
    if (multi) {
        for (const St& t : s->st)
            for (const sf_sx_node& n : t.nodes)
                if (n.op == SF_SX_READ && !is_identity(n))
                    return sf_fail(SF_ERR_INVALID, "affine reads need a single-part level");
    }
    // ---- bounds: every write and read inside the storage windows
    for (int p = 0; p < L->nlocal; p++) {
        const int z0 = L->parts[p].z0;
        const int gi = L->parts[p].index;
        const long zlo = gi == 0 ? LONG_MIN / 4 : z0 + 1;
        const long zhi = gi == L->nparts - 1 ? LONG_MAX / 4 : z0 + L->lnz + 1;
        long wl[3], wh[3], sl[3], sh[3];
        window(L, z0, wl, wh);
        window(S, same ? z0 : 0, sl, sh);
        for (int i = 0; i < ng; i++)
            for (const Rect& r : s->st[i].rects) {
                RR R = resolve(r, gdim, zlo, zhi);
                if (R.empty()) continue;
                for (int d = 0; d < 3; d++)
                    if (R.lo[d] < wl[d] || R.last(d) >= wh[d])
                        return sf_fail(SF_ERR_SHAPE, "stencil %d writes outside the level storage (axis %d)", i, d);
                for (const sf_sx_node& n : s->st[i].nodes) {
                    if (n.op != SF_SX_READ) continue;
                    const bool onL = n.src == 0 || same;
                    const long* lo = onL ? wl : sl;
                    const long* hi = onL ? wh : sh;
                    for (int d = 0; d < 3; d++) {
                        const long a = amap(n, d, R.lo[d]), b = amap(n, d, R.last(d));
                        if (a < lo[d] || b >= hi[d])
                            return sf_fail(SF_ERR_SHAPE, "stencil %d reads outside the %s level storage (axis %d)",
                                           i, onL ? "output" : "source", d);
                    }
                }
            }
    }
    SF_TRY(jit(s));
    s->phases = (int)phases.size();

    SfArgsH A;
    for (const std::vector<int>& ph : phases) {
        if (multi) {   // z halos of the meshes this phase reads across planes
            int depth[SF_NFIELDS] = {0};
            for (int i : ph)
                for (const sf_sx_node& n : s->st[i].nodes)
                    if (n.op == SF_SX_READ)
                        depth[n.mesh] = std::max(depth[n.mesh], std::abs(n.off[2]));
            for (int m = 0; m < SF_NFIELDS; m++)
                if (depth[m]) SF_TRY(sf_halo(L, m, depth[m]));
        }
        for (int p = 0; p < L->nlocal; p++) {
            const int z0 = L->parts[p].z0;
            const int gi = L->parts[p].index;
            const long zlo = gi == 0 ? LONG_MIN / 4 : z0 + 1;
            const long zhi = gi == L->nparts - 1 ? LONG_MAX / 4 : z0 + L->lnz + 1;
            memset(&A, 0, sizeof A);
            PV v = sf_view(L, p);
            PV w = sf_view(S, same ? p : 0);
            for (int m = 0; m < SF_NFIELDS; m++) {
                A.f[0][m] = v.f[m];
                A.f[1][m] = w.f[m];
            }
            A.js[0] = L->js; A.ks[0] = L->ks;
            A.js[1] = S->js; A.ks[1] = S->ks;
            A.xb = SF_OX - 1;
            A.yb = SF_GY - 1;
            A.zb[0] = SF_GZ - 1 - z0;
            A.zb[1] = same ? A.zb[0] : SF_GZ - 1;
            long long total = 0;   // lines (j, k) of all rects of the phase
            int nr = 0, maxc0 = 0;
            for (int i : ph)
                for (const Rect& r : s->st[i].rects) {
                    RR R = resolve(r, gdim, zlo, zhi);
                    if (R.empty()) continue;
                    if (nr == SF_STENCIL_MAX_RECTS)
                        return sf_fail(SF_ERR_INVALID, "more than %d rects in one phase", SF_STENCIL_MAX_RECTS);
                    // line axis: x unless the rect is one point wide in x (e.g.
                    // an x-face ghost layer), then the longer of y / z
                    int a0 = 0;
                    if (R.cnt[0] == 1) a0 = R.cnt[1] >= R.cnt[2] ? 1 : 2;
                    const int a1 = a0 == 0 ? 1 : 0, a2 = 3 - a0 - a1;
                    const long long lines = (long long)R.cnt[a1] * R.cnt[a2];
                    if (lines > INT_MAX) return sf_fail(SF_ERR_SHAPE, "rect of more than 2^31 lines");
                    SfRectH& h = A.r[nr++];
                    for (int d = 0; d < 3; d++) {
                        h.lo[d] = (int)R.lo[d];
                        h.st[d] = (int)R.st[d];
                        h.cnt[d] = (int)R.cnt[d];
                    }
                    h.ax[0] = a0; h.ax[1] = a1; h.ax[2] = a2;
                    h.sid = i;
                    h.start = total;
                    total += lines;
                    maxc0 = std::max(maxc0, (int)R.cnt[a0]);
                }
            if (total == 0) continue;
            A.nrect = nr;
            A.total = total;
            // rects sharing one line lattice (e.g. the 4 rects of a colour) are
            // walked interleaved, ordered by (outer, middle) start, so the
            // lines in flight sit in a few neighbouring planes (L2 reuse of
            // the neighbour planes / rows instead of 4 sweeps of the volume)
            A.ilv = 0;
            if (nr > 1) {
                bool same = true;
                for (int q = 1; q < nr && same; q++)
                    for (int d = 0; d < 3; d++)
                        if (A.r[q].st[d] != A.r[0].st[d] || A.r[q].cnt[d] != A.r[0].cnt[d] ||
                            A.r[q].ax[d] != A.r[0].ax[d])
                            same = false;
                if (same) {
                    const int a1 = A.r[0].ax[1], a2 = A.r[0].ax[2];
                    std::sort(A.r, A.r + nr, [&](const SfRectH& x, const SfRectH& y) {
                        if (x.lo[a2] != y.lo[a2]) return x.lo[a2] < y.lo[a2];
                        return x.lo[a1] < y.lo[a1];
                    });
                    A.ilv = nr;
                }
            }
            const int half = (maxc0 + 1) / 2;   // two points per thread
            const int bx = half >= 256 ? 256 : half > 64 ? 128 : half > 32 ? 64 : 32;
            const unsigned gx = (unsigned)std::min(4, (half + bx - 1) / bx);
            // persistent: exactly the resident blocks (one wave) walk the lines
            const int bi = bx == 32 ? 0 : bx == 64 ? 1 : bx <= 128 ? 2 : 3;
            const int bxr = 32 << bi;
            const unsigned gy = (unsigned)std::min<long long>(
                total, std::max(1, s->sms * s->occ[bi] / (int)gx));
            void* params[] = {&A};
            if (g_drv.launch(s->fn, gx, gy, 1, bxr, 1, 1, 0, L->stream, params, nullptr) != CUDA_SUCCESS)
                return sf_fail(SF_ERR_CUDA, "cuLaunchKernel failed");
            SF_LAUNCHED();
        }
    }
    return sf_check_launch("sf_stencil_group");
}
