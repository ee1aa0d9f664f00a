// Device helpers shared by the TMA-fed smoothers (gsrb_fused.cu, gsrb_twopair.cu,
// gsrb_rr.cu) and the coarse V-cycle (coarse.cu): mbarrier /
// cp.async.bulk.tensor wrappers and the lambda-form stencil sum.  Included
// inside each translation unit's anonymous namespace.
#pragma once

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
__device__ __forceinline__ void mbar_expect_u(unsigned b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void tma3u(unsigned dst, const CUtensorMap* m, int c0, int c1, int c2,
                                      unsigned bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(dst),
        "l"((unsigned long long)m), "r"(c0), "r"(c1), "r"(c2), "r"(bar)
        : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ int md(int k, int m) { return ((k % m) + m) % m; }

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Gauss-Seidel update in lambda-form.  With lambda = Dinv the EXACT inverse
// diagonal of A including the Dirichlet fold (reading R-4),
//     x + lambda (rhs - A x)  ==  lambda (rhs + b h^-2 S),
//     S = sum over the cell's interior faces of beta_f * x(nbr_f),
// because A x = D x(c) - b h^-2 S (a boundary face's ghost term -2 beta x(c)
// is part of D).  The smoother therefore never reads alpha: 56 instead of the
// 64 compulsory bytes of PAPER.md:669-672.  Boundary neighbours enter S as 0.
// S is summed as a tree (depth 3): the per-plane step is latency-bound.
// 1/d for the check-fused residual: hardware reciprocal estimate + two Newton
// steps (relative error ~1e-16, far below what the 1e-10 convergence test needs;
// avoids the long IEEE division sequence in the hot loop)
__device__ __forceinline__ double inv_fast(double d) {
    double y;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(d));
    y = y * (2.0 - d * y);
    y = y * (2.0 - d * y);
    return y;
}

__device__ __forceinline__ double sum6(double xw, double xe, double xs, double xn, double xb,
                                      double xt, double bw, double be, double bs, double bn,
                                      double bb, double bt) {
    // explicit contraction: every kernel that includes this header forms S
    // with the same roundings (the fused pair variants are bit-identical)
    const double sx = __fma_rn(be, xe, __dmul_rn(bw, xw));
    const double sy = __fma_rn(bn, xn, __dmul_rn(bs, xs));
    const double sz = __fma_rn(bt, xt, __dmul_rn(bb, xb));
    return __dadd_rn(__dadd_rn(sx, sy), sz);
}

// q = rhs + b h^-2 S (one rounding) and the update lambda * q
__device__ __forceinline__ double gs_q(double rhs, double bh2, double S) {
    return __fma_rn(bh2, S, rhs);
}
__device__ __forceinline__ double gs_upd(double dinv, double rhs, double bh2, double S) {
    return __dmul_rn(dinv, gs_q(rhs, bh2, S));
}

__device__ __forceinline__ unsigned long long abits(double v) {
    return (unsigned long long)__double_as_longlong(fabs(v));
}
