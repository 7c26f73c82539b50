// spmv_dia.cu — MPK SpMV step (Fig. 4; Newton shift fused) specialised for the
// dominant DIA slice width of the matrix (CAGMRES_OPT_SPMV 10..13).
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

// L2 eviction-priority hints (PF = 3): the value stream is read exactly once per step, so it is
// loaded / prefetched as evict_first and does not push the basis columns out of the 126 MB L2:
// the x operand (the column the previous step just wrote) and the y column this step writes
// (next step's x) stay L2-resident instead of making a DRAM round trip per step.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ double ldg_stream_hint(const double* p, uint64_t pol) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    return v;
}
// one TMA-engine instruction prefetches a whole slice's values (16-B aligned, multiple of 16 B)
__device__ __forceinline__ void bulk_prefetch_l2(const void* p, uint32_t bytes, uint64_t pol) {
    asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(p), "r"(bytes), "l"(pol)
                 : "memory");
}

// PF = 1: while slice i is computed, the value lines of slice i + stride (descriptor already in
// registers) are prefetched into L2, so next iteration's value loads are L2 hits: one more
// slice of HBM requests in flight per warp without holding registers.
// CONTIG = 0: slices grid-strided over all warps.  CONTIG = 1: each CTA owns a contiguous
// range of slices and its 8 warps walk it side by side, so the x lines of the +-1 and +-nx
// offsets (and, for thin 3-D grids, +-nx*ny) are L1 hits from the CTA's own recent loads.
template <int MODE, int WT, int MINB, int CONTIG = 0, int PF = 0>   // MODE 0: Ax  1: + bu u  2: + bw w  3: u - Ax
__global__ void __launch_bounds__(DT_NT, MINB) k_spmv_dia(DiaArgs a) {
    const int lane = threadIdx.x & 31;
    const uint64_t pol = PF == 3 ? policy_evict_first() : 0;
    const int64_t nsl_all = (a.nrows + 31) >> 5;
    int64_t stride, sl, nsl;
    if (CONTIG) {
        stride = DT_NT / 32;
        const int64_t c0 = int64_t(blockIdx.x) * nsl_all / gridDim.x;
        nsl = int64_t(blockIdx.x + 1) * nsl_all / gridDim.x;
        sl = c0 + (threadIdx.x >> 5);
    } else {
        stride = int64_t(gridDim.x) * (DT_NT / 32);
        nsl = nsl_all;
        sl = (int64_t(blockIdx.x) * DT_NT + threadIdx.x) >> 5;
    }
    if (sl >= nsl) { pdl_wait(); pdl_trigger(); return; }
    int64_t b0, i0, b1 = 0, i1 = 1, b2 = 0, i2 = 1, b3, i3;
    int W0, W1 = 0, W2 = 0, W3, o0, o1;
    // slice descriptors (static during a solve) are loaded before the PDL wait
    sell_slice_meta(sl, a.sptr, a.sinfo, b0, W0, i0);
    if (sl + stride < nsl) sell_slice_meta(sl + stride, a.sptr, a.sinfo, b1, W1, i1);
    if (PF == 2 && sl + 2 * stride < nsl) sell_slice_meta(sl + 2 * stride, a.sptr, a.sinfo, b2, W2, i2);
    o0 = sell_slice_off(lane, W0, i0, a.dcol);
    pdl_wait();
    pdl_trigger();
#pragma unroll 1
    for (; sl < nsl; sl += stride) {
        if (PF == 2) {                                                   // 3-deep descriptor pipeline
            b3 = 0; W3 = 0; i3 = 1;
            if (sl + 3 * stride < nsl) sell_slice_meta(sl + 3 * stride, a.sptr, a.sinfo, b3, W3, i3);
            if (lane < 2 * W2) prefetch_l2(a.val + b2 + 16 * lane);      // 128-B lines of slice +2
        } else {
            b2 = 0; W2 = 0; i2 = 1;
            if (sl + 2 * stride < nsl) sell_slice_meta(sl + 2 * stride, a.sptr, a.sinfo, b2, W2, i2);
        }
        o1 = sell_slice_off(lane, W1, i1, a.dcol);
        if (PF == 1 && lane < 2 * W1) prefetch_l2(a.val + b1 + 16 * lane);     // 128-B lines of slice +1
        if (PF == 3 && lane == 0 && W1 > 0) bulk_prefetch_l2(a.val + b1, uint32_t(W1) * 256u, pol);
        const int64_t r = sl * 32 + lane;
        const bool live = r < a.nrows;
        double uu = 0.0, ww = 0.0, acc = 0.0;
        if (W0 == WT && (i0 & 3) == 1) {
            const double* vp = a.val + b0 + lane;
            const double* xr = a.x + r;
            if (MODE >= 1 && live) uu = __ldg(a.u + r);
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
                    if constexpr (PF == 3) v[t] = ldg_stream_hint(vp + 32 * (g0 + t), pol);
                    else v[t] = (CONTIG || PF) ? ldg_stream(vp + 32 * (g0 + t)) : __ldg(vp + 32 * (g0 + t));
                    xv[t] = __ldg(xr + o);
                }
#pragma unroll
                for (int t = 0; t < GT; ++t) acc = fma(v[t], xv[t], acc);
            }
        } else {
            acc = sell_slice_dot<4, true>(r, b0, W0, i0, o0, a.dcol, a.ncols, a.val, a.x, false);
            if (MODE >= 1 && live) uu = __ldg(a.u + r);
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
        if (PF == 2) { b2 = b3; W2 = W3; i2 = i3; }
    }
}

namespace {
template <int MODE, int WT, int MINB, int CONTIG, int PF>
void go_dia(const Dev& d, const DiaArgs& a, cudaStream_t st) {
    static int occ = 0;
    if (occ == 0) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_spmv_dia<MODE, WT, MINB, CONTIG, PF>, DT_NT, 0);
        if (occ < 1) occ = 1;
    }
    const int64_t nsl = (a.nrows + 31) >> 5;
    int64_t g = int64_t(d.sms) * occ;
    const int64_t need = (nsl + DT_NT / 32 - 1) / (DT_NT / 32);
    if (g > need) g = need;
    launch_pdl(k_spmv_dia<MODE, WT, MINB, CONTIG, PF>, dim3(unsigned(g)), dim3(DT_NT), 0, st, a);
}

template <int WT, int MINB, int CONTIG, int PF>
void go_modes(const Dev& d, const DiaArgs& a, cudaStream_t st, int mode) {
    switch (mode) {
        case 0: go_dia<0, WT, MINB, CONTIG, PF>(d, a, st); break;
        case 1: go_dia<1, WT, MINB, CONTIG, PF>(d, a, st); break;
        case 2: go_dia<2, WT, MINB, CONTIG, PF>(d, a, st); break;
        default: go_dia<3, WT, MINB, CONTIG, PF>(d, a, st); break;
    }
}

template <int MINB, int CONTIG, int PF = 0>
void go_width(const Dev& d, const DiaArgs& a, int wt, cudaStream_t st, int mode) {
    switch (wt) {
        case 5: go_modes<5, MINB, CONTIG, PF>(d, a, st, mode); break;
        case 27: go_modes<27, MINB, CONTIG, PF>(d, a, st, mode); break;
        default: go_modes<7, MINB, CONTIG, PF>(d, a, st, mode); break;     // other widths: generic path
    }
}
}  // namespace

// variants 10 / 11 / 12 / 13: at least 3 / 4 / 5 / 6 CTAs per SM (register cap), grid-strided
// slices; 14 / 15: 4 / 5 CTAs per SM, CTA-contiguous slice ranges (L1 reuse of x); 16 / 17:
// 4 / 5 CTAs per SM, grid-strided, L2 prefetch of the next slice's values (L1::no_allocate value
// loads); 18: 4 CTAs per SM, prefetch two slices ahead (3-deep descriptor pipeline)
void spmv_dia(const Dev& d, const Sell& A, int variant, int64_t nrows, const double* x, double* y,
              const double* u, double bu, const double* w, double bw, int mode, cudaStream_t st) {
    DiaArgs a{nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, u, bu, w, bw, y};
    switch (variant) {
        case 10: go_width<3, 0>(d, a, A.dia_w, st, mode); break;
        case 11: go_width<4, 0>(d, a, A.dia_w, st, mode); break;
        case 12: go_width<5, 0>(d, a, A.dia_w, st, mode); break;
        case 14: go_width<4, 1>(d, a, A.dia_w, st, mode); break;
        case 15: go_width<5, 1>(d, a, A.dia_w, st, mode); break;
        case 16: go_width<4, 0, 1>(d, a, A.dia_w, st, mode); break;
        case 17: go_width<5, 0, 1>(d, a, A.dia_w, st, mode); break;
        case 18: go_width<4, 0, 2>(d, a, A.dia_w, st, mode); break;
        case 19: go_width<4, 0, 3>(d, a, A.dia_w, st, mode); break;
        case 20: go_width<5, 0, 3>(d, a, A.dia_w, st, mode); break;
        default: go_width<6, 0>(d, a, A.dia_w, st, mode); break;
    }
}

}  // namespace kern
