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
    int64_t b0, i0, b1 = 0, i1 = 1, b2 = 0, i2 = 1;
    int W0, W1 = 0, W2 = 0, o0, o1;
    // slice descriptors (static during a solve) are loaded before the PDL wait
    sell_slice_meta(sl, a.sptr, a.sinfo, b0, W0, i0);
    if (sl + stride < nsl) sell_slice_meta(sl + stride, a.sptr, a.sinfo, b1, W1, i1);
    o0 = sell_slice_off(lane, W0, i0, a.dcol);
    pdl_wait();
    pdl_trigger();
    const double inv = SX ? 1.0 / __ldg(a.xnrm) : 1.0;
#pragma unroll 1
    for (; sl < nsl; sl += stride) {
        b2 = 0; W2 = 0; i2 = 1;
        if (sl + 2 * stride < nsl) sell_slice_meta(sl + 2 * stride, a.sptr, a.sinfo, b2, W2, i2);
        o1 = sell_slice_off(lane, W1, i1, a.dcol);
        if (lane < 2 * W1) prefetch_l2(a.val + b1 + 16 * lane);        // 128-B lines of slice +1
        const int64_t r = sl * 32 + lane;
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
// Two rows per lane (variant 18; DIA widths <= 16).  A warp takes a PAIR of consecutive SELL-32
// slices; lane l handles rows 2 (l & 15), 2 (l & 15) + 1 of slice 2p + (l >> 4), so every value
// load is a 16-B double2 (the two rows are adjacent in the slice's column-major layout) and so is
// every x gather whose offset is even (the row pair starts at an even row); odd offsets take two
// 8-B loads.  Half the load instructions per row and twice the bytes in flight per warp for the
// same register budget as two independent slices.  Per row the FMA order (t = 0..W-1) and the
// epilogue are those of k_spmv_dia: bitwise identical.  A pair that is not uniformly "width WT,
// no clamping" is done slice by slice with the generic body.
template <int MODE, int WT, int MINB, bool SX = false>
__global__ void __launch_bounds__(DT_NT, MINB) k_spmv_dia64(DiaArgs a) {
    static_assert(WT <= 16, "two rows per lane: <= 16 diagonals per half warp");
    const int lane = threadIdx.x & 31, hl = lane >> 4, li = lane & 15;
    const int64_t nsl = (a.nrows + 31) >> 5;
    const int64_t npr = (nsl + 1) >> 1;
    const int64_t stride = int64_t(gridDim.x) * (DT_NT / 32);
    int64_t pr = (int64_t(blockIdx.x) * DT_NT + threadIdx.x) >> 5;
    if (pr >= npr) { pdl_wait(); pdl_trigger(); return; }
    // this lane's slice descriptor (its half's slice) for the current and the next pair
    auto meta = [&](int64_t p, int64_t& b, int& W, int64_t& in, int& off) {
        const int64_t sl = 2 * p + hl;
        if (p < npr && sl < nsl) {
            sell_slice_meta(sl, a.sptr, a.sinfo, b, W, in);
            off = ((in & 1) && li < W) ? __ldg(a.dcol + (in >> 2) + li) : 0;
        } else {
            b = 0; W = 0; in = 1; off = 0;
        }
    };
    int64_t b0, i0, b1, i1;
    int W0, W1, o0, o1;
    meta(pr, b0, W0, i0, o0);
    meta(pr + stride, b1, W1, i1, o1);
    pdl_wait();
    pdl_trigger();
    const double inv = SX ? 1.0 / __ldg(a.xnrm) : 1.0;
#pragma unroll 1
    for (; pr < npr; pr += stride) {
        if (li < W1) prefetch_l2(a.val + b1 + 16 * li);          // next pair: 2 x 128-B lines / diag
        const int64_t sl = 2 * pr + hl;
        const bool have = sl < nsl;
        const int64_t r = sl * 32 + 2 * li;                       // even: rows r, r + 1
        const bool live0 = have && r < a.nrows, live1 = have && r + 1 < a.nrows;
        const bool fast = __all_sync(0xffffffffu, !have || (W0 == WT && (i0 & 3) == 1));
        double acc0 = 0.0, acc1 = 0.0, u0 = 0.0, u1 = 0.0, w0 = 0.0, w1 = 0.0;
        if (fast) {
            if (have) {
                const double* vp = a.val + b0 + 2 * li;
                double2 v[WT];
                double x0[WT], x1[WT];
#pragma unroll
                for (int t = 0; t < WT; ++t) {
                    const int o = __shfl_sync(0xffffffffu, o0, (lane & 16) + t);
                    v[t] = __ldg(reinterpret_cast<const double2*>(vp + 32 * t));
                    const int64_t c = r + o;
                    if ((o & 1) == 0) {
                        const double2 xx = __ldg(reinterpret_cast<const double2*>(a.x + c));
                        x0[t] = xx.x; x1[t] = xx.y;
                    } else {
                        x0[t] = __ldg(a.x + c);
                        x1[t] = __ldg(a.x + c + 1);
                    }
                }
                if (SX) {
                    const double2 xx = __ldg(reinterpret_cast<const double2*>(a.x + r));
                    u0 = xx.x * inv; u1 = xx.y * inv;
                    if (live0) a.xs[r] = u0;
                    if (live1) a.xs[r + 1] = u1;
                } else if (MODE >= 1) {
                    if (live0) u0 = __ldg(a.u + r);
                    if (live1) u1 = __ldg(a.u + r + 1);
                }
                if (MODE == 2) {
                    if (live0) w0 = __ldg(a.w + r);
                    if (live1) w1 = __ldg(a.w + r + 1);
                }
#pragma unroll
                for (int t = 0; t < WT; ++t) {
                    acc0 = fma(v[t].x, SX ? x0[t] * inv : x0[t], acc0);
                    acc1 = fma(v[t].y, SX ? x1[t] * inv : x1[t], acc1);
                }
            }
        } else {
            // slice by slice, one row per lane, with the generic body
#pragma unroll 1
            for (int hh = 0; hh < 2; ++hh) {
                const int64_t s2 = 2 * pr + hh;
                if (s2 >= nsl) break;
                int64_t bb, ii;
                int WW;
                sell_slice_meta(s2, a.sptr, a.sinfo, bb, WW, ii);
                const int oo = sell_slice_off(lane, WW, ii, a.dcol);
                const int64_t rr = s2 * 32 + lane;
                const double acc = sell_slice_dot<4, true, SX>(rr, bb, WW, ii, oo, a.dcol, a.ncols, a.val, a.x, false, inv);
                if (rr < a.nrows) {
                    double uu = 0.0, ww = 0.0;
                    if (SX) { uu = __ldg(a.x + rr) * inv; a.xs[rr] = uu; }
                    else if (MODE >= 1) uu = __ldg(a.u + rr);
                    if (MODE == 2) ww = __ldg(a.w + rr);
                    double out;
                    if constexpr (MODE == 3) {
                        out = uu - acc;
                    } else {
                        out = acc;
                        if constexpr (MODE >= 1) out = fma(a.bu, uu, out);
                        if constexpr (MODE >= 2) out = fma(a.bw, ww, out);
                    }
                    a.y[rr] = out;
                }
            }
        }
        if (fast && have) {
            double out0, out1;
            if constexpr (MODE == 3) {
                out0 = u0 - acc0; out1 = u1 - acc1;
            } else {
                out0 = acc0; out1 = acc1;
                if constexpr (MODE >= 1) { out0 = fma(a.bu, u0, out0); out1 = fma(a.bu, u1, out1); }
                if constexpr (MODE >= 2) { out0 = fma(a.bw, w0, out0); out1 = fma(a.bw, w1, out1); }
            }
            if (live1) *reinterpret_cast<double2*>(a.y + r) = make_double2(out0, out1);
            else if (live0) a.y[r] = out0;
        }
        b0 = b1; W0 = W1; i0 = i1; o0 = o1;
        meta(pr + 2 * stride, b1, W1, i1, o1);
    }
}

template <int MODE, int WT, int MINB, bool SX = false>
void go_dia64(const Dev& d, const DiaArgs& a, cudaStream_t st) {
    static int occ = 0;
    if (occ == 0) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_spmv_dia64<MODE, WT, MINB, SX>, DT_NT, 0);
        if (occ < 1) occ = 1;
    }
    const int64_t npr = (((a.nrows + 31) >> 5) + 1) >> 1;
    int64_t g = int64_t(d.sms) * occ;
    const int64_t need = (npr + DT_NT / 32 - 1) / (DT_NT / 32);
    if (g > need) g = need;
    if (g < 1) g = 1;
    launch_pdl(k_spmv_dia64<MODE, WT, MINB, SX>, dim3(unsigned(g)), dim3(DT_NT), 0, st, a);
}

template <int WT, int MINB>
void go_modes64(const Dev& d, const DiaArgs& a, cudaStream_t st, int mode) {
    switch (mode) {
        case 0: go_dia64<0, WT, MINB>(d, a, st); break;
        case 1: go_dia64<1, WT, MINB>(d, a, st); break;
        case 2: go_dia64<2, WT, MINB>(d, a, st); break;
        case 4: go_dia64<0, WT, MINB, true>(d, a, st); break;
        case 5: go_dia64<1, WT, MINB, true>(d, a, st); break;
        default: go_dia64<3, WT, MINB>(d, a, st); break;
    }
}

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
    DiaArgs a{nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, u, bu, w, bw, y, xnrm, xs};
    if ((variant == 18 || variant == 19) && A.dia_w != 27) { // two rows per lane (widths <= 16)
        if (A.dia_w == 5) { if (variant == 18) go_modes64<5, 3>(d, a, st, mode); else go_modes64<5, 2>(d, a, st, mode); }
        else { if (variant == 18) go_modes64<7, 3>(d, a, st, mode); else go_modes64<7, 2>(d, a, st, mode); }
        return;
    }
    if (variant == 17) go_width<5>(d, a, A.dia_w, st, mode);
    else go_width<4>(d, a, A.dia_w, st, mode);
}

}  // namespace kern
