// mpk_wave.cu — single-GPU matrix powers kernel with temporal blocking ("reducing
// communication of MPK on a single GPU").
//
// Plain MPK reads A from HBM once per SpMV step (s times per block).  For a naturally
// ordered matrix with half-bandwidth b (|col - row| <= b: stencils, banded operators), the
// rows of step k in a chunk [r0, r1) depend only on step k-1 rows [r0 - b, r1 + b).  One
// persistent kernel executes all (chunk, step) items of a block as a dataflow wavefront:
//   * items are ordered by tau = c + L*k.  With L > ceil(b/CH) every dependency has a
//     smaller tau, so round-robin assignment to resident CTAs cannot deadlock;
//   * L - b/CH chunks of slack per step give ~G/s runnable chunks per step (G resident
//     CTAs), while the reuse distance of a chunk of A (s*L chunks) stays within L2, so A is
//     read from HBM about once per block and re-read from L2 for the other s-1 steps;
//   * a chunk waits (one warp, acquire loads) on the epoch-stamped completion flags of the
//     <= 2*ceil(b/CH)+1 step-(k-1) chunks it reads — no grid barrier, no memset.
// Each row is computed with exactly the operations of k_spmv_sell32, so the basis is bitwise
// identical to the step-by-step MPK (tests/test_gpu_parity.py).  x gathers use L1-cached
// loads: L1 is invalidated at every launch, nothing is read before the chunk that wrote it is
// complete, and the waited range is widened by one L1 line, so no stale line can be hit.
#include <cstdint>

#include "kernels.h"

namespace kern {

namespace {
constexpr int NT = 256;

__device__ __forceinline__ int ld_acquire(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
}  // namespace

__global__ void __launch_bounds__(NT) k_mpk_wave(WaveArgs a) {
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    for (int64_t idx = blockIdx.x; idx < a.npairs; idx += gridDim.x) {
        const int2 ck = a.pairs[idx];
        const int c = ck.x, k = ck.y;
        const int64_t r0 = int64_t(c) * a.CH;
        const int64_t r1 = min(a.n, r0 + a.CH);
        if (k > 1 && wp == 0) {
            // rows read: [r0 - bw, r1 - 1 + bw], widened by one 128-B line (16 rows) so no L1
            // line this chunk caches can hold rows of a not-yet-complete chunk
            const int64_t lo_r = r0 - a.bw - 16 < 0 ? 0 : r0 - a.bw - 16;
            const int64_t hi_r = min(a.n - 1, r1 - 1 + a.bw + 16);
            const int clo = int(lo_r / a.CH), chi = int(hi_r / a.CH);
            const int* f = a.done + int64_t(k - 1) * a.nC;
            for (int base = clo; base <= chi; base += 32) {
                const int cc = base + lane;
                bool ok = cc > chi;
                int ns = 32;
                while (true) {
                    if (!ok) ok = ld_acquire(f + cc) == a.epoch;
                    if (__all_sync(0xffffffffu, ok)) break;
                    __nanosleep(ns);
                    ns = ns < 512 ? ns * 2 : 512;
                }
            }
        }
        __syncthreads();
        const double* x = a.V + a.ldv * (a.j + k - 1);
        double* y = a.V + a.ldv * (a.j + k);
        const double th = a.theta[k - 1], b2 = a.b2[k - 1];
        const double* xp = a.kind[k - 1] == 2 ? a.V + a.ldv * (a.j + k - 2) : nullptr;
        // same row computation as k_spmv_sell32 (sell_row_dot), x through L1 (see header)
        for (int64_t r = r0 + threadIdx.x; (r & ~int64_t(31)) < r1; r += NT) {
            const double acc = sell_row_dot<4>(r, a.sptr, a.sinfo, a.dcol, a.ncols, a.val, x, true);
            if (r < r1) {
                double out = acc;
                if (th != 0.0) out = fma(-th, __ldca(x + r), out);
                if (xp) out = fma(b2, __ldca(xp + r), out);
                __stcg(y + r, out);
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            st_release(a.done + int64_t(k) * a.nC + c, a.epoch);
        }
    }
}

void mpk_wave(const Dev& d, const WaveArgs& a, int ctas_per_sm, cudaStream_t st) {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mpk_wave, NT, 0);
    if (occ < 1) occ = 1;
    if (ctas_per_sm > 0 && ctas_per_sm < occ) occ = ctas_per_sm;
    int64_t g = int64_t(d.sms) * occ;                     // all CTAs resident (no deadlock)
    if (g > a.npairs) g = a.npairs;
    if (g < 1) g = 1;
    ++g_launches;
    k_mpk_wave<<<unsigned(g), NT, 0, st>>>(a);
}

}  // namespace kern
