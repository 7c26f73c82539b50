// spmv_dia.cu — MPK SpMV step (Fig. 4; Newton shift fused) specialised for the
// dominant DIA slice width of the matrix (CAGMRES_OPT_SPMV 16, 17; the default on DIA matrices).
//
// The persistent kernel of kernels.cu (variant 5) is latency-bound (ncu: issue active 56 %,
// long-scoreboard the top stall, ~255 instructions per 32-row slice): its generic batched loop
// pays predicates, selects and 64-bit index arithmetic per entry and issues the shift operand
// loads only after the dot product.  Here a slice whose width equals the matrix's most common
// DIA width WT (7 for the 7-point stencil, 5 / 27 for the 5- and 27-point ones; A.dia_w) and
// needs no clamping runs a fully unrolled body: WT value loads, WT x gathers and the u / w
// loads are all in flight together (one dependent latency per slice), no predicates.  Other
// slices take the generic sell_slice_dot path.  The slice descriptors are software-pipelined
// one / two grid strides ahead exactly as in k_spmv_sell32_persist.
// Per row the FMAs run t = 0..W-1 from 0.0 and the epilogue is out = fma(bu, u, acc), then
// fma(bw, w, .): the same operations in the same order as every other variant (bitwise
// identical results; tests/test_gpu_parity.py::test_spmv_variants_bitwise).
// (A cp.async shared-memory ring version of this step — every value, x gather and shift
// operand staged per slice — was measured 2x slower: 8 warps/SM, issue-latency bound.)
#include <cstdint>

#include "kernels.h"

namespace kern {

namespace {
constexpr int DT_NT = 256;

struct DiaArgs {
    int64_t nrows;
    const int64_t* sptr; const int64_t* sinfo; const int32_t* dcol; int64_t ncols;
    const double* val;
    const double* x;
    const double* u; double bu;
    const double* w; double bw;
    double* y;
    const double* xnrm;     // SX: x is an unnormalised w, the operand is w * (1 / *xnrm)
    double* xs;             // SX: the normalised operand's rows [0, nrows) are stored here
    int rev;                // 1: slices visited in descending order (serpentine order, Dev::rev)
};
}  // namespace

// value stream: read once, keep it out of L1 so L1 holds the x lines neighbouring warps reuse
__device__ __forceinline__ double ldg_stream(const double* p) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

// While slice i is computed, the value lines of slice i + stride (descriptor already in
// registers) are prefetched into L2, so next iteration's value loads are L2 hits: one more
// slice of HBM requests in flight per warp without holding registers.  Slices are grid-strided
// over all warps of the persistent grid.
// SX (fused normalisation, MODE 0 / 1 only): the input vector is w with ||w|| = *xnrm on the
// device (the Arnoldi / residual norm just computed); every x operand is w[c] * (1 / ||w||) —
// exactly the product the separate scaling kernel k_scale1 forms — and each thread also stores
// its row of the normalised vector to xs.  So the q = w / ||w|| pass (a read and a write of the
// vector, one launch) disappears and the results are bitwise those of scale-then-SpMV.
template <int MODE, int WT, int MINB, bool SX = false>   // MODE 0: Ax  1: + bu u  2: + bw w  3: u - Ax
__global__ void __launch_bounds__(DT_NT, MINB) k_spmv_dia(DiaArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t nsl = (a.nrows + 31) >> 5;
    const int64_t stride = int64_t(gridDim.x) * (DT_NT / 32);
    int64_t sl = (int64_t(blockIdx.x) * DT_NT + threadIdx.x) >> 5;
    if (sl >= nsl) { pdl_wait(); pdl_trigger(); return; }
    // serpentine order (rev): the grid walks the slices from the end, so the first slices read
    // are the ones the previous MPK step read last — their A values and x lines are L2 hits
    const int64_t rx = a.rev ? nsl - 1 : 0, rs = a.rev ? -1 : 1;     // slice = rx + rs * sl
    int64_t b0, i0, b1 = 0, i1 = 1, b2 = 0, i2 = 1;
    int W0, W1 = 0, W2 = 0, o0, o1;
    // slice descriptors (static during a solve) are loaded before the PDL wait
    sell_slice_meta(rx + rs * sl, a.sptr, a.sinfo, b0, W0, i0);
    if (sl + stride < nsl) sell_slice_meta(rx + rs * (sl + stride), a.sptr, a.sinfo, b1, W1, i1);
    o0 = sell_slice_off(lane, W0, i0, a.dcol);
    pdl_wait();
    pdl_trigger();
    const double inv = SX ? 1.0 / __ldg(a.xnrm) : 1.0;
#pragma unroll 1
    for (; sl < nsl; sl += stride) {
        b2 = 0; W2 = 0; i2 = 1;
        if (sl + 2 * stride < nsl) sell_slice_meta(rx + rs * (sl + 2 * stride), a.sptr, a.sinfo, b2, W2, i2);
        o1 = sell_slice_off(lane, W1, i1, a.dcol);
        if (lane < 2 * W1) prefetch_l2(a.val + b1 + 16 * lane);        // 128-B lines of slice +1
        const int64_t r = (rx + rs * sl) * 32 + lane;
        const bool live = r < a.nrows;
        double uu = 0.0, ww = 0.0, acc = 0.0;
        if (SX && live) {                                               // own row of q = w / ||w||
            uu = __ldg(a.x + r) * inv;
            a.xs[r] = uu;
        }
        if (W0 == WT && (i0 & 3) == 1) {
            const double* vp = a.val + b0 + lane;
            const double* xr = a.x + r;
            if (!SX && MODE >= 1 && live) uu = __ldg(a.u + r);
            if (MODE == 2 && live) ww = __ldg(a.w + r);
            // 27-point rows: three groups of 9 value / x pairs in flight (all 27 at once spilled
            // 480 B of stack at the 64-register cap); the FMA order t = 0..WT-1 is unchanged
            constexpr int GT = WT > 9 ? 9 : WT;
            static_assert(WT % GT == 0, "DIA width must split into equal groups");
#pragma unroll
            for (int g0 = 0; g0 < WT; g0 += GT) {
                double v[GT], xv[GT];
#pragma unroll
                for (int t = 0; t < GT; ++t) {
                    const int o = __shfl_sync(0xffffffffu, o0, g0 + t);
                    v[t] = ldg_stream(vp + 32 * (g0 + t));
                    xv[t] = __ldg(xr + o);
                }
                if (SX) {
#pragma unroll
                    for (int t = 0; t < GT; ++t) xv[t] *= inv;
                }
#pragma unroll
                for (int t = 0; t < GT; ++t) acc = fma(v[t], xv[t], acc);
            }
        } else {
            acc = sell_slice_dot<4, true, SX>(r, b0, W0, i0, o0, a.dcol, a.ncols, a.val, a.x, false, inv);
            if (!SX && MODE >= 1 && live) uu = __ldg(a.u + r);
            if (MODE == 2 && live) ww = __ldg(a.w + r);
        }
        if (live) {
            double out;
            if constexpr (MODE == 3) {
                out = uu - acc;
            } else {
                out = acc;
                if constexpr (MODE >= 1) out = fma(a.bu, uu, out);
                if constexpr (MODE >= 2) out = fma(a.bw, ww, out);
            }
            a.y[r] = out;
        }
        b0 = b1; W0 = W1; i0 = i1; o0 = o1;
        b1 = b2; W1 = W2; i1 = i2;
    }
}

namespace {
template <int MODE, int WT, int MINB, bool SX = false>
void go_dia(const Dev& d, const DiaArgs& a, cudaStream_t st) {
    static int occ = 0;
    if (occ == 0) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_spmv_dia<MODE, WT, MINB, SX>, DT_NT, 0);
        if (occ < 1) occ = 1;
    }
    const int64_t nsl = (a.nrows + 31) >> 5;
    int64_t g = int64_t(d.sms) * occ;
    const int64_t need = (nsl + DT_NT / 32 - 1) / (DT_NT / 32);
    if (g > need) g = need;
    launch_pdl(k_spmv_dia<MODE, WT, MINB, SX>, dim3(unsigned(g)), dim3(DT_NT), 0, st, a);
}

template <int WT, int MINB>
void go_modes(const Dev& d, const DiaArgs& a, cudaStream_t st, int mode) {
    switch (mode) {
        case 0: go_dia<0, WT, MINB>(d, a, st); break;
        case 1: go_dia<1, WT, MINB>(d, a, st); break;
        case 2: go_dia<2, WT, MINB>(d, a, st); break;
        case 4: go_dia<0, WT, MINB, true>(d, a, st); break;      // 4 / 5: modes 0 / 1 with SX
        case 5: go_dia<1, WT, MINB, true>(d, a, st); break;
        default: go_dia<3, WT, MINB>(d, a, st); break;
    }
}

template <int MINB>
void go_width(const Dev& d, const DiaArgs& a, int wt, cudaStream_t st, int mode) {
    switch (wt) {
        case 5: go_modes<5, MINB>(d, a, st, mode); break;
        case 27: go_modes<27, MINB>(d, a, st, mode); break;
        default: go_modes<7, MINB>(d, a, st, mode); break;     // other widths: generic path
    }
}
}  // namespace

// variants 16 / 17: at least 4 / 5 CTAs per SM, grid-strided slices, L2 prefetch of the next
// slice's values (L1::no_allocate value loads).  (Round 1's other settings — 3 / 6 CTAs per SM,
// CTA-contiguous slice ranges, a two-slice-deep prefetch — and round 2's L2 evict-first hints
// and TMA-streamed value rings measured slower: DESIGN.md §6.)
void spmv_dia(const Dev& d, const Sell& A, int variant, int64_t nrows, const double* x, double* y,
              const double* u, double bu, const double* w, double bw, int mode, cudaStream_t st,
              const double* xnrm, double* xs) {
    DiaArgs a{nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, u, bu, w, bw, y, xnrm, xs, d.rev};
    if (variant == 17) go_width<5>(d, a, A.dia_w, st, mode);
    else go_width<4>(d, a, A.dia_w, st, mode);
}

}  // namespace kern
