// mpk_wave.cu — single-GPU matrix powers kernel with temporal blocking ("reducing
// communication of MPK on a single GPU").
//
// Plain MPK reads A from HBM once per SpMV step (s times per block).  For a naturally
// ordered matrix with half-bandwidth b (|col - row| <= b: stencils, banded operators), rows
// are cut into tiles of R >= b rows, so step k on tile t depends only on step k-1 on tiles
// t-1, t, t+1.  One persistent kernel executes all (tile, step) items of a block as a
// dataflow wavefront: items are ordered by tau = t + 2k (a topological order, since every
// dependency has a smaller tau), split into chunks of CH rows handed round-robin to the
// resident CTAs, and a chunk waits on per-(step, tile) completion counters instead of a
// grid barrier.  The live window is ~2*s tiles, so a tile of A stays in L2 across its s
// steps: A is read from HBM about once per block instead of s times, vectors are written
// once and re-read from L2.  Each row is computed exactly as in k_spmv_sell32 (same order of
// the same operations), so the result is bitwise identical to the step-by-step MPK.
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
}  // namespace

__global__ void __launch_bounds__(NT) k_mpk_wave(WaveArgs a) {
    const int64_t nchunks = int64_t(a.npairs) * a.C;
    __shared__ int s_ok;
    for (int64_t idx = blockIdx.x; idx < nchunks; idx += gridDim.x) {
        const int pi = int(idx / a.C), c = int(idx - int64_t(pi) * a.C);
        const int2 tk = a.pairs[pi];
        const int t = tk.x, k = tk.y;
        const int64_t r0 = int64_t(t) * a.R + int64_t(c) * a.CH;
        if (r0 < a.n && k > 1) {
            if (threadIdx.x == 0) {
                for (int d = -1; d <= 1; ++d) {
                    const int tt = t + d;
                    if (tt < 0 || tt >= a.nT) continue;
                    const int* f = a.done + (k - 1) * a.nT + tt;
                    const int want = a.cnt[tt];
                    int ns = 32;
                    while (ld_acquire(f) < want) {
                        __nanosleep(ns);
                        ns = ns < 1024 ? ns * 2 : 1024;
                    }
                }
                s_ok = 1;
            }
            __syncthreads();
        }
        if (r0 < a.n) {
            const int64_t r1 = min(a.n, r0 + a.CH);
            const double* x = a.V + a.ldv * (a.j + k - 1);
            double* y = a.V + a.ldv * (a.j + k);
            const double th = a.theta[k - 1], b2 = a.b2[k - 1];
            const double* xp = a.kind[k - 1] == 2 ? a.V + a.ldv * (a.j + k - 2) : nullptr;
            for (int64_t r = r0 + threadIdx.x; r < r1; r += NT) {
                const int64_t sl = r >> 5;
                const int lane = int(r & 31);
                int64_t o = __ldg(a.sptr + sl) + lane;
                const int64_t e = __ldg(a.sptr + sl + 1);
                double acc = 0.0;
#pragma unroll 4
                for (; o < e; o += 32) acc = fma(__ldg(a.val + o), __ldcg(x + __ldg(a.col + o)), acc);
                double out = acc;
                if (th != 0.0) out = fma(-th, __ldcg(x + r), out);
                if (xp) out = fma(b2, __ldcg(xp + r), out);
                y[r] = out;
            }
        }
        __syncthreads();
        if (threadIdx.x == 0 && r0 < a.n) {
            __threadfence();
            atomicAdd(a.done + k * a.nT + t, 1);
        }
    }
    (void)s_ok;
}

void mpk_wave(const Dev& d, const WaveArgs& a, cudaStream_t st) {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mpk_wave, NT, 0);
    if (occ < 1) occ = 1;
    const int64_t nchunks = int64_t(a.npairs) * a.C;
    int64_t g = int64_t(d.sms) * occ;                     // all CTAs resident (no deadlock)
    if (g > nchunks) g = nchunks;
    if (g < 1) g = 1;
    ++g_launches;
    k_mpk_wave<<<unsigned(g), NT, 0, st>>>(a);
}

}  // namespace kern
