// mpk_sweep.cu — one MPK block (s_b SpMV steps, Fig. 4; Newton shifts fused) in ONE
// persistent launch on a single GPU (CAGMRES_OPT_MPK_WAVE = 3).
//
// The stepwise MPK launches one DIA SpMV per step; every launch pays its ramp (first loads'
// latency, CTA rasterisation, slice-descriptor prologue) and its drain (the slowest warp), a
// fixed ~5-7 µs per launch against ~20-25 µs of streaming (tools/stream_probe.cu).  Here the
// grid (all CTAs resident: #SMs x occupancy) runs the steps back to back with a grid barrier
// between them: after step k every CTA arrives on a monotonically increasing counter and
// spins (acquire loads) until all have; the next step's first slice descriptors are loaded
// before the barrier (A is static).  Each step is the stepwise kernel's row body — the same
// loads and the same FMA order — so the basis is bitwise the stepwise MPK's; the sweep
// direction alternates per step (serpentine order).
// x is read with L1-cached coherent loads: L1 is invalidated at launch and a column is only
// read after the barrier that follows the step writing it, so no stale line can be hit.
// Dependents are triggered only after the last barrier: until then no later kernel can take
// an SM that a not-yet-resident CTA of this grid is waiting for.
#include <cstdint>

#include "kernels.h"

namespace kern {

namespace {
constexpr int SW_NT = 256;
constexpr int SW_NW = SW_NT / 32;

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double ld_stream_sw(const double* p) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void prefetch_l2_sw(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }
}  // namespace

template <int WT, int MINB>
__global__ void __launch_bounds__(SW_NT, MINB) k_mpk_sweep(SweepArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t nsl = (a.n + 31) >> 5;
    const int64_t stride = int64_t(gridDim.x) * SW_NW;
    const int64_t g = (int64_t(blockIdx.x) * SW_NT + threadIdx.x) >> 5;
    pdl_wait();
    for (int k = 1; k <= a.sb; ++k) {
        const int rev = a.rev0 ^ ((k - 1) & 1);
        const int64_t rx = rev ? nsl - 1 : 0, rs = rev ? -1 : 1;        // slice = rx + rs * sl
        const double* x = a.V + a.ldv * (a.j + k - 1);
        double* y = a.V + a.ldv * (a.j + k);
        const int kind = a.kind[k - 1];
        const double bu = -a.theta[k - 1], bw = a.b2[k - 1];
        const bool use_u = bu != 0.0 || kind == 2;                       // the stepwise MODE >= 1
        const double* wv = kind == 2 ? a.V + a.ldv * (a.j + k - 2) : nullptr;
        int64_t sl = g;
        int64_t b0 = 0, i0 = 1, b1 = 0, i1 = 1, b2 = 0, i2 = 1;
        int W0 = 0, W1 = 0, W2 = 0, o0 = 0, o1;
        if (sl < nsl) {
            sell_slice_meta(rx + rs * sl, a.sptr, a.sinfo, b0, W0, i0);
            o0 = sell_slice_off(lane, W0, i0, a.dcol);
        }
        if (sl + stride < nsl) sell_slice_meta(rx + rs * (sl + stride), a.sptr, a.sinfo, b1, W1, i1);
        if (k > 1) {                                                     // grid barrier: step k-1 done
            __syncthreads();
            if (threadIdx.x == 0) {
                const unsigned target = a.bar_base + unsigned(k - 1) * gridDim.x;
                while (int(ld_acquire_u32(a.bar) - target) < 0) __nanosleep(40);
            }
            __syncthreads();
        }
#pragma unroll 1
        for (; sl < nsl; sl += stride) {
            b2 = 0; W2 = 0; i2 = 1;
            if (sl + 2 * stride < nsl) sell_slice_meta(rx + rs * (sl + 2 * stride), a.sptr, a.sinfo, b2, W2, i2);
            o1 = sell_slice_off(lane, W1, i1, a.dcol);
            if (lane < 2 * W1) prefetch_l2_sw(a.val + b1 + 16 * lane);
            const int64_t r = (rx + rs * sl) * 32 + lane;
            const bool live = r < a.n;
            double uu = 0.0, ww = 0.0, acc = 0.0;
            if (WT > 0 && W0 == WT && (i0 & 3) == 1) {
                const double* vp = a.val + b0 + lane;
                const double* xr = x + r;
                if (use_u && live) uu = __ldca(x + r);
                if (wv && live) ww = __ldca(wv + r);
                constexpr int GT = WT > 9 ? 9 : (WT > 0 ? WT : 1);
#pragma unroll
                for (int g0 = 0; g0 < WT; g0 += GT) {
                    double v[GT], xv[GT];
#pragma unroll
                    for (int t = 0; t < GT; ++t) {
                        const int o = __shfl_sync(0xffffffffu, o0, g0 + t);
                        v[t] = ld_stream_sw(vp + 32 * (g0 + t));
                        xv[t] = __ldca(xr + o);
                    }
#pragma unroll
                    for (int t = 0; t < GT; ++t) acc = fma(v[t], xv[t], acc);
                }
            } else {
                acc = sell_slice_dot<4, true>(r, b0, W0, i0, o0, a.dcol, a.ncols, a.val, x, true);
                if (use_u && live) uu = __ldca(x + r);
                if (wv && live) ww = __ldca(wv + r);
            }
            if (live) {
                double out = acc;                       // the stepwise epilogue, same order
                if (use_u) out = fma(bu, uu, out);
                if (wv) out = fma(bw, ww, out);
                __stcg(y + r, out);
            }
            b0 = b1; W0 = W1; i0 = i1; o0 = o1;
            b1 = b2; W1 = W2; i1 = i2;
        }
        if (k < a.sb) {                                 // arrive (release: y visible to all CTAs)
            __syncthreads();
            if (threadIdx.x == 0) {
                __threadfence();
                atomicAdd(a.bar, 1u);
            }
        }
    }
    pdl_trigger();
}

namespace {
template <int WT, int MINB>
int go_sweep(const Dev& d, SweepArgs a, cudaStream_t st, unsigned* next_base) {
    static int occ = 0;
    if (occ == 0) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mpk_sweep<WT, MINB>, SW_NT, 0);
        if (occ < 1) occ = 1;
    }
    const int64_t nsl = (a.n + 31) >> 5;
    int64_t g = int64_t(d.sms) * occ;                   // all CTAs co-resident (grid barrier)
    const int64_t need = (nsl + SW_NW - 1) / SW_NW;
    if (g > need) g = need;
    if (g < 1) g = 1;
    *next_base = a.bar_base + unsigned(a.sb - 1) * unsigned(g);
    ++g_launches;
    launch_pdl(k_mpk_sweep<WT, MINB>, dim3(unsigned(g)), dim3(SW_NT), 0, st, a);
    return 0;
}
}  // namespace

int mpk_sweep(const Dev& d, const SweepArgs& a, cudaStream_t st, unsigned* next_base) {
    if (a.sb < 1 || a.sb > 32) return -1;
    switch (a.dia_w) {
        case 5: return go_sweep<5, 4>(d, a, st, next_base);
        case 7: return go_sweep<7, 4>(d, a, st, next_base);
        case 27: return go_sweep<27, 4>(d, a, st, next_base);
        default: return go_sweep<0, 4>(d, a, st, next_base);
    }
}

}  // namespace kern
