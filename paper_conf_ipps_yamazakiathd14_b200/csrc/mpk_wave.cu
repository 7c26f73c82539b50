// mpk_wave.cu — single-GPU matrix powers kernel with temporal blocking ("reducing
// communication of MPK on a single GPU").
//
// Plain MPK reads A from HBM once per SpMV step (s times per block).  For a naturally
// ordered matrix with half-bandwidth b (|col - row| <= b: stencils, banded operators), the
// rows of step k in a chunk [r0, r1) depend only on step k-1 rows [r0 - b, r1 + b).  One
// persistent kernel executes all (chunk, step) items of a block as a dataflow wavefront:
//   * items are ordered by tau = c + L*k.  With L > ceil((b + 16) / CH) every dependency has
//     a smaller tau; CTAs take items from a global ticket counter in that order, so an item
//     only ever waits for items already held by running (resident) CTAs: no deadlock;
//   * L - b/CH chunks of slack per step leave ~G/s runnable items per step for the G resident
//     CTAs, while the reuse distance of a chunk of A (s*L chunks) stays within L2, so A is
//     read from HBM about once per block and re-read from L2 for the other s-1 steps;
//   * warp 0 of a CTA waits (acquire loads) on the epoch-stamped completion flags of the
//     step-(k-1) chunks the item reads — no grid barrier, no memset of the flags.
// Inside an item every warp runs the DIA-specialised row body of spmv_dia.cu over its slices
// (WT value loads + WT x gathers in flight, slice descriptors pipelined one slice ahead), so
// each row is computed with exactly the operations of the stepwise SpMV: the basis is bitwise
// identical (tests/test_gpu_parity.py).  x gathers use L1-cached loads: L1 is invalidated at
// every launch, nothing is read before the chunk that wrote it is complete, and the waited
// range is widened by one L1 line (16 rows), so no stale line can be hit.
#include <cstdint>

#include "kernels.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NW = NT / 32;

__device__ __forceinline__ int ld_acquire(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ double ld_stream(const double* p) {
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}
}  // namespace

template <int WT>
__global__ void __launch_bounds__(NT, 4) k_mpk_wave(WaveArgs a) {
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    __shared__ int s_item;
    for (;;) {
        if (threadIdx.x == 0) s_item = atomicAdd(a.queue, 1);
        __syncthreads();
        const int idx = s_item;
        if (idx >= a.npairs) break;
        const int2 ck = __ldg(a.pairs + idx);
        const int c = ck.x, k = ck.y;
        const int64_t r0 = int64_t(c) * a.CH;
        const int64_t r1 = min(a.n, r0 + a.CH);
        // slices of this item and this warp's first two descriptors (static: before the wait)
        const int64_t sl_end = (r1 + 31) >> 5;
        int64_t sl = (r0 >> 5) + wp;
        int64_t b0 = 0, i0 = 1, b1 = 0, i1 = 1;
        int W0 = 0, W1 = 0, o0 = 0;
        if (sl < sl_end) {
            sell_slice_meta(sl, a.sptr, a.sinfo, b0, W0, i0);
            o0 = sell_slice_off(lane, W0, i0, a.dcol);
        }
        if (sl + NW < sl_end) sell_slice_meta(sl + NW, a.sptr, a.sinfo, b1, W1, i1);
        if (k > 1 && wp == 0) {
            // rows read: [r0 - bw, r1 - 1 + bw], widened by one 128-B line (16 rows)
            const int64_t lo_r = r0 - a.bw - 16 < 0 ? 0 : r0 - a.bw - 16;
            const int64_t hi_r = min(a.n - 1, r1 - 1 + a.bw + 16);
            const int clo = int(lo_r / a.CH), chi = int(hi_r / a.CH);
            const int* f = a.done + int64_t(k - 1) * a.nC;
            for (int base = clo; base <= chi; base += 32) {
                const int cc = base + lane;
                bool ok = cc > chi;
                while (true) {
                    if (!ok) ok = ld_acquire(f + cc) == a.epoch;
                    if (__all_sync(0xffffffffu, ok)) break;
                    __nanosleep(32);
                }
            }
        }
        __syncthreads();
        const double* x = a.V + a.ldv * (a.j + k - 1);
        double* y = a.V + a.ldv * (a.j + k);
        const double th = a.theta[k - 1], b2 = a.b2[k - 1];
        const double* xp = a.kind[k - 1] == 2 ? a.V + a.ldv * (a.j + k - 2) : nullptr;
#pragma unroll 1
        for (; sl < sl_end; sl += NW) {
            int64_t b2d = 0, i2 = 1;
            int W2 = 0;
            if (sl + 2 * NW < sl_end) sell_slice_meta(sl + 2 * NW, a.sptr, a.sinfo, b2d, W2, i2);
            const int o1 = sell_slice_off(lane, W1, i1, a.dcol);
            const int64_t r = sl * 32 + lane;
            const bool live = r < r1;
            double acc = 0.0, uu = 0.0, ww = 0.0;
            if (WT > 0 && W0 == WT && (i0 & 3) == 1) {
                const double* vp = a.val + b0 + lane;
                const double* xr = x + r;
                if (live) uu = __ldca(x + r);
                if (xp && live) ww = __ldca(xp + r);
                constexpr int GT = WT > 9 ? 9 : (WT > 0 ? WT : 1);
#pragma unroll
                for (int g0 = 0; g0 < WT; g0 += GT) {
                    double v[GT], xv[GT];
#pragma unroll
                    for (int t = 0; t < GT; ++t) {
                        const int o = __shfl_sync(0xffffffffu, o0, g0 + t);
                        v[t] = ld_stream(vp + 32 * (g0 + t));
                        xv[t] = __ldca(xr + o);
                    }
#pragma unroll
                    for (int t = 0; t < GT; ++t) acc = fma(v[t], xv[t], acc);
                }
            } else {
                acc = sell_slice_dot<4, true>(r, b0, W0, i0, o0, a.dcol, a.ncols, a.val, x, true);
                if (live) uu = __ldca(x + r);
                if (xp && live) ww = __ldca(xp + r);
            }
            if (live) {
                // the stepwise SpMV's epilogue: out = fma(bu, u, acc) [, fma(bw, w, .)]
                double out = acc;
                if (th != 0.0 || xp) out = fma(-th, uu, out);
                if (xp) out = fma(b2, ww, out);
                __stcg(y + r, out);
            }
            b0 = b1; W0 = W1; i0 = i1; o0 = o1;
            b1 = b2d; W1 = W2; i1 = i2;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            st_release(a.done + int64_t(k) * a.nC + c, a.epoch);
        }
    }
}

void mpk_wave(const Dev& d, const WaveArgs& a, int ctas_per_sm, cudaStream_t st) {
    auto go = [&](auto kfn) {
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kfn, NT, 0);
        if (occ < 1) occ = 1;
        if (ctas_per_sm > 0 && ctas_per_sm < occ) occ = ctas_per_sm;
        int64_t g = int64_t(d.sms) * occ;                 // all CTAs resident (no deadlock)
        if (g > a.npairs) g = a.npairs;
        if (g < 1) g = 1;
        ++g_launches;
        kfn<<<unsigned(g), NT, 0, st>>>(a);
    };
    switch (a.dia_w) {
        case 5: go(k_mpk_wave<5>); break;
        case 7: go(k_mpk_wave<7>); break;
        case 27: go(k_mpk_wave<27>); break;
        default: go(k_mpk_wave<0>); break;
    }
}

}  // namespace kern
