// The V-cycle's last pre-smoothing RB pair fused with its residual and the
// residual's 2:1 cell restriction (A5 + A6 + A7).
//
// Done separately, the residual pass re-reads x, rhs, alpha and the three face
// coefficients right after the smoother streamed them (48 B per fine cell,
// residual_restrict_zs_kernel).  Here the colour-fused pair itself (its RRF
// variant, gsrb_fused.cu) forms the restricted residual of its OUTPUT from
// values it already holds, in delta form:
//
//   * a red cell c had zero residual right after its own update (the update
//     uses lambda = 1/diag(A) exactly), and the black sweep
//     then changed only its six black neighbours n_f, so
//         r(c) = rhs - A x_out at c = b h^-2 sum_f beta_f delta(n_f),
//     delta = x_out - x_in of a black cell;
//   * a black cell's residual after its update vanishes the same way (its
//     neighbours are red and final);
//
// both up to rounding, the same order as the rounding of rhs - A x itself.  The
// restriction R(C) = 1/8 sum_{c in block C} r(c) then becomes
// a scatter of every black cell's b h^-2 beta_f delta over its six faces: three
// land in its own 2x2x2 block, one per axis in the neighbouring block.  Each
// thread of the pair accumulates its pair column's two planes of a block in
// registers; x shares move to the next pair column by a lane shuffle and z
// shares stay in the thread (carried to the next / previous coarse plane), so a
// thread writes two partials per coarse cell (its block's and the y share for
// the neighbouring block row), plus the shares that cross a tile or z-chunk
// edge into edge arrays (SfRRF, sf_internal.h).  Each entry has at most one
// writer, so the result does not depend on scheduling; the fix-up kernel below
// sums them in a fixed order into the coarse rhs.  Extra work in the pair: one
// shared-memory load (the black cell's old value), ~10 FP64 operations, a
// shuffle and ~4 B of stores per fine cell -- instead of a 48 B/cell pass.
//
// Scope: single-part fine and coarse levels (the headline's 512^3 hierarchy;
// slab-decomposed levels keep pair + residual_restrict), the 32x8 fused-pair
// build, even nz, levels of at least SF_RRF_CELLS cells (default 2^21; tests set
// 0).  SF_RRF=0 disables it.  The partial arrays belong to the fine level and are
// allocated (zeroed) by sf_mg_create / the first eager call, never inside a
// graph capture.
#include <cstdlib>

#include "sf_internal.h"

namespace {

constexpr int NPART = 12;

// coarse rhs = 1/8 of the partials, summed in array order; the edge arrays are
// read only where the current launch wrote them (tile-edge columns: the 32x8
// build's coarse tiles are 16 wide; z-chunk edge planes: zdepth / 2 per chunk)
__global__ void rrf_fixup_kernel(double* __restrict__ out, SfRRF rv, int trig) {
    pdl_wait();
    // trig: the next launch (the coarse cluster V-cycle) may start now -- it
    // stages its constant operands and waits for this output in griddepcontrol.wait
    if (trig) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int i = blockIdx.x * blockDim.x + threadIdx.x, j = blockIdx.y, k = blockIdx.z;
    if (i >= rv.ncx) return;
    const long q = (long)(k + SF_GZ) * rv.cks + (long)(j + SF_GY) * rv.cjs + SF_OX + i;
    const int cd = rv.zdepth / 2;
    // last coarse plane of a z-chunk (the last chunk may be shorter): every y share
    const bool klast = k % cd == cd - 1 || k == rv.ncz - 1;
    double s = rv.a[0][q] + rv.a[1][q];
    if ((i & 15) == 15 && i + 1 < rv.ncx) s = s + rv.a[2][q] + rv.a[3][q];
    if ((i & 15) == 0 && i > 0) s = s + rv.a[4][q] + rv.a[5][q];
    // y shares through memory: the tile-edge block rows (coarse tiles are 4 rows
    // high), and every row on a chunk's last coarse plane
    if ((klast || (j & 3) == 3) && j + 1 < rv.ncy) s = s + rv.a[6][q];
    if ((klast || (j & 3) == 0) && j > 0) s = s + rv.a[7][q];
    if (k % cd == cd - 1 && k + 1 < rv.ncz) s = s + rv.a[8][q] + rv.a[9][q];
    if (k % cd == 0 && k > 0) s = s + rv.a[10][q] + rv.a[11][q];
    out[q] = 0.125 * s;
}

long rrf_min_cells() {   // read per call: tests switch it
    const char* e = getenv("SF_RRF_CELLS");
    return e ? atol(e) : (1L << 21);
}

}  // namespace

bool gsrb_rr_supported(const sf_level* F, const sf_level* C) {
    const bool on = !(getenv("SF_RRF") && atoi(getenv("SF_RRF")) == 0);
    return on && F->nparts == 1 && F->nlocal == 1 && C->nparts == 1 && C->nlocal == 1 &&
           gsrb_fused_supported_t32w4(F) && F->lnz % 2 == 0 && C->nx * 2 == F->nx &&
           C->ny * 2 == F->ny && C->lnz * 2 == F->lnz &&
           (long)F->nx * F->ny * F->lnz >= rrf_min_cells();
}

// the partial arrays exist, or can be allocated now (the stream is not capturing)
bool sf_rrf_usable(const sf_level* F, const sf_level* C) {
    if (F->rrf_buf && F->rrf_felems == C->felems) return true;
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    return cudaStreamIsCapturing(F->stream, &cs) == cudaSuccess && cs == cudaStreamCaptureStatusNone;
}

// allocate (once, zeroed) the partial arrays of F for coarse level C
sf_status sf_rrf_prepare(sf_level* F, const sf_level* C) {
    if (F->rrf_buf && F->rrf_felems == C->felems) return SF_OK;
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    SF_CUDA(cudaStreamIsCapturing(F->stream, &cs));
    if (cs != cudaStreamCaptureStatusNone)
        return sf_fail(SF_ERR_INVALID, "RRF partial arrays must be allocated before graph capture");
    if (F->rrf_buf) cudaFree(F->rrf_buf);
    F->rrf_buf = nullptr;
    const size_t bytes = (size_t)NPART * C->felems * sizeof(double);
    cudaError_t e = cudaMalloc(&F->rrf_buf, bytes);
    if (e != cudaSuccess) {
        F->rrf_buf = nullptr;
        cudaGetLastError();
        return sf_fail(SF_ERR_OOM, "cudaMalloc(%zu) for RRF partials: %s", bytes, cudaGetErrorString(e));
    }
    // never-written entries (neighbour blocks outside the domain) stay 0
    SF_CUDA(cudaMemsetAsync(F->rrf_buf, 0, bytes, F->stream));
    SF_CUDA(cudaStreamSynchronize(F->stream));
    F->rrf_felems = C->felems;
    return SF_OK;
}

sf_status k_gsrb_pair_rr(sf_level* L, int xin, int xout, int rhs, double a, double b, sf_level* C,
                         int cf, bool trigger_next) {
    if (!gsrb_rr_supported(L, C)) return sf_fail(SF_ERR_SHAPE, "fused pair+residual+restriction unsupported");
    SF_TRY(sf_rrf_prepare(L, C));
    SfRRF rv;
    for (int m = 0; m < NPART; m++) rv.a[m] = L->rrf_buf + (size_t)m * C->felems;
    rv.cjs = (int)C->js;
    rv.cks = (int)C->ks;
    rv.ncx = C->nx;
    rv.ncy = C->ny;
    rv.ncz = C->lnz;
    rv.zdepth = 2;
    SF_TRY(k_gsrb_pair_fused_t32w4(L, xin, xout, rhs, a, b, nullptr, nullptr, 0, 0, 0, SF_RM_NONE, &rv));
    PV c = sf_view(C, 0);
    sf_launch(rrf_fixup_kernel, dim3((C->nx + 127) / 128, C->ny, C->lnz), 128, 0, L->stream, c.f[cf], rv,
              trigger_next ? 1 : 0);
    SF_LAUNCHED();
    return sf_check_launch("rrf_fixup");
}
