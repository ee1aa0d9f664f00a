// Per-cell A3 operator of the one-thread-per-cell kernels (kernels.cu): one
// definition, so every one of them evaluates the operator with the same terms,
// order and roundings.
#pragma once

// x loads: plain (L1-cached) or .cg (L2 only: the cluster kernel reads values
// other SMs wrote in an earlier phase of the same launch)
template <bool CG>
__device__ __forceinline__ double ldx(const double* p) {
    if (CG) return __ldcg(p);
    return *p;
}

// A3 at cell (i,j,k) with the Dirichlet fold.  Summation order matches the
// operator definition term by term (A3).
template <bool CG = false>
__device__ __forceinline__ double op_at(const PV& v, const double* __restrict__ x, int i, int j,
                                        int k, double a, double bh2) {
    const double* al = v.f[SF_ALPHA];
    const double* bi = v.f[SF_BETA_I];
    const double* bj = v.f[SF_BETA_J];
    const double* bk = v.f[SF_BETA_K];
    long c = sf_ix(v, i, j, k);
    double xc = ldx<CG>(x + c);
    int gk = v.z0 + k;
    double xw = (i == 0) ? -xc : ldx<CG>(x + c - 1);
    double xe = (i == v.nx - 1) ? -xc : ldx<CG>(x + c + 1);
    double xs = (j == 0) ? -xc : ldx<CG>(x + c - v.js);
    double xn = (j == v.ny - 1) ? -xc : ldx<CG>(x + c + v.js);
    double xb = (gk == 0) ? -xc : ldx<CG>(x + c - v.ks);
    double xt = (gk == v.gnz - 1) ? -xc : ldx<CG>(x + c + v.ks);
    double flux = bi[c + 1] * (xe - xc);
    flux += bi[c] * (xw - xc);
    flux += bj[c + v.js] * (xn - xc);
    flux += bj[c] * (xs - xc);
    flux += bk[c + v.ks] * (xt - xc);
    flux += bk[c] * (xb - xc);
    return a * al[c] * xc - bh2 * flux;
}
