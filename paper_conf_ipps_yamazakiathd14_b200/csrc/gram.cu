// gram.cu — CholQR Gram G = P^T P (P: n x W, W <= 12) on the FP64 CUDA cores.
//
// Why not the tensor core here: one DMMA (m8n8k4) yields an 8x8 block for 4 rows, so the
// symmetric W = 11 Gram takes 3 DMMAs per 4 rows for 66 useful products out of 192 — at
// HBM speed (6.4 TB/s / 88 B per row = 73 G rows/s) that is 55 G DMMA/s, more than the FP64
// tensor pipe sustains (tools/fp64_probe.cu).  The scalar form needs W(W+1)/2 = 66 DFMAs
// per row, a fraction of the DFMA pipe.
//
// Data movement: the warps of a CTA work in pairs; each pair streams its band-order share
// (kern::band_tile: tiles g, g + 8 x 148, ...; descending in serpentine order) of the 64-row tiles of the W columns through an S-stage shared-memory ring with 16-B
// cp.async copies (both warps issue half of every tile's copies), so the bytes in flight
// (~150 KB per SM) live in shared memory, not in registers.  Lane l of both warps owns rows
// 2l, 2l+1 of a tile (one 16-B shared load per column; 32-row tiles with one row per lane
// measured 49 us for W = 11 at n = 2.1M: barrier / MIO-throttle bound); the W(W+1)/2 upper-triangle
// products are split between the two warps (33 + 33 sums at W = 11), which halves the
// registers per thread and so doubles the warps per SM that hide the latencies.  One named
// barrier per tile and pair publishes the tile and frees the slot read in the previous step.
// Reduction: a fixed xor-shuffle tree in the warp, a fixed-order sum over the CTA's pairs,
// and the last CTA (atomic ticket) sums the per-CTA partials in a fixed order (reduce.cuh)
// and, for CholQR on one GPU, runs the Cholesky in the same launch — deterministic for a
// given grid.
#include <algorithm>
#include <cstdint>

#include "dense_dev.cuh"
#include "kernels.h"
#include "ptx.h"
#include "reduce.cuh"

namespace kern {

namespace {
constexpr int GR_NT = 512;               // 16 warps = 8 pairs, one CTA per SM
constexpr int GR_TW = 64;                // rows per tile (2 per lane: one LDS.128 per column)
constexpr int GR_NP = GR_NT / 64;        // warp pairs

template <int W>
__host__ __device__ constexpr int gram_stages() { return W <= 6 ? 6 : (W <= 8 ? 5 : 4); }

__device__ __forceinline__ void pair_sync(int pair) {
    asm volatile("bar.sync %0, 64;" ::"r"(pair + 1) : "memory");
}

// acc[e - lo] += v_i v_k for the upper-triangle entries e in [lo, hi) (row-major order), for
// the two rows 2 lane, 2 lane + 1 of the tile (in that order)
template <int W, int LO, int HI>
__device__ __forceinline__ void rank1_part(const double* __restrict__ sl, int lane, double (&acc)[HI - LO]) {
    double2 v[W];
#pragma unroll
    for (int c = 0; c < W; ++c)                                    // unused columns: dead code
        v[c] = *reinterpret_cast<const double2*>(sl + c * GR_TW + 2 * lane);
    int e = 0;
#pragma unroll
    for (int i = 0; i < W; ++i)
#pragma unroll
        for (int k = i; k < W; ++k, ++e)
            if (e >= LO && e < HI) {
                acc[e - LO] = fma(v[i].x, v[k].x, acc[e - LO]);
                acc[e - LO] = fma(v[i].y, v[k].y, acc[e - LO]);
            }
}
}  // namespace

template <int W, int H>
__device__ __forceinline__ void gram_pair_body(const GramArgs& a, double* smg, double* red, int pair, int h) {
    constexpr int S = gram_stages<W>();
    constexpr int NE = W * (W + 1) / 2;
    constexpr int HALF = (NE + 1) / 2;
    constexpr int LO = H ? HALF : 0, HI = H ? NE : HALF;
    constexpr int NA = HI - LO > 0 ? HI - LO : 1;
    const int lane = threadIdx.x & 31;
    constexpr int stage_d = W * GR_TW;
    double* ring = smg + int64_t(pair) * S * stage_d;
    const int64_t T = a.n / GR_TW;                                 // full tiles
    const int64_t NPg = int64_t(gridDim.x) * GR_NP;
    const int64_t g = int64_t(blockIdx.x) * GR_NP + pair;
    const int64_t cnt = band_count(T, NPg, g);                    // tiles of this pair (band order)
    // this thread's 16-B chunks of a tile (pair-thread q = 64 k + pt): fixed offsets
    constexpr int CPC = GR_TW * 8 / 16;                            // 16-B chunks per column tile
    constexpr int NCH = W * CPC;
    constexpr int KC = (NCH + 63) / 64;
    const int pt = h * 32 + lane;
    int64_t gof[KC];
    int sof[KC];
#pragma unroll
    for (int k = 0; k < KC; ++k) {
        const int q = pt + 64 * k;
        const int c = q / CPC, part = q - c * CPC;
        gof[k] = q < NCH ? a.ldp * c + part * 2 : -1;
        sof[k] = c * GR_TW + part * 2;
    }
    auto issue = [&](int64_t i, double* slot) {
        if (i < cnt) {
            const double* src = a.P + band_tile(T, NPg, g, i, a.rev) * GR_TW;
#pragma unroll
            for (int k = 0; k < KC; ++k)
                if (k * 64 + 63 < NCH || gof[k] >= 0) ptx::cp_async16(slot + sof[k], src + gof[k]);
        }
        ptx::cp_async_commit();
    };
    double acc[NA];
#pragma unroll
    for (int e = 0; e < NA; ++e) acc[e] = 0.0;
#pragma unroll
    for (int s = 0; s < S - 1; ++s) issue(s, ring + s * stage_d);
    double* cur = ring;                                            // slot of tile t
    double* nxt = ring + (S - 1) * stage_d;                        // slot refilled at step t
    double* const rend = ring + S * stage_d;
    for (int64_t i = 0; i < cnt; ++i) {
        ptx::cp_async_wait<S - 2>();                               // my copies of tile i landed
        pair_sync(pair);                                           // ... and my partner's; slot
        issue(i + S - 1, nxt);                                     //  of step i-1 is free
        if (HI > LO) rank1_part<W, LO, (HI > LO ? HI : LO + 1)>(cur, lane, acc);
        cur += stage_d; if (cur == rend) cur = ring;
        nxt += stage_d; if (nxt == rend) nxt = ring;
    }
    ptx::cp_async_wait<0>();
    if (blockIdx.x == 0 && pair == 0 && T * GR_TW < a.n) {         // ragged tail rows [T*64, n)
        pair_sync(pair);
        double* sl = ring;                                         // ring idle: stage the tail
        const int64_t r0 = T * GR_TW;
        for (int q = pt; q < W * GR_TW; q += 64) {
            const int c = q / GR_TW, r = q - c * GR_TW;
            sl[q] = r0 + r < a.n ? a.P[a.ldp * c + r0 + r] : 0.0;
        }
        pair_sync(pair);
        if (HI > LO) rank1_part<W, LO, (HI > LO ? HI : LO + 1)>(sl, lane, acc);
    }
#pragma unroll
    for (int e = 0; e < NA; ++e) {
        double sum = acc[e];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
        if (lane == 0 && LO + e < HI) red[pair * NE + LO + e] = sum;
    }
}

template <int W>
__global__ void __launch_bounds__(GR_NT, 1) k_gram_ring(GramArgs a) {
    extern __shared__ __align__(16) double smg[];
    constexpr int NE = W * (W + 1) / 2;
    __shared__ double red[GR_NP * NE];                             // per-pair sums (not aliased)
    const int wp = threadIdx.x >> 5, pair = wp >> 1, h = wp & 1;
    pdl_wait();
    pdl_trigger();
    if (h == 0) gram_pair_body<W, 0>(a, smg, red, pair, 0);
    else gram_pair_body<W, 1>(a, smg, red, pair, 1);
    __syncthreads();
    constexpr int nent = W * W;
    double* part = a.part + int64_t(blockIdx.x) * nent;
    for (int q = threadIdx.x; q < nent; q += GR_NT) {
        int i = q % W, k = q / W;
        if (i > k) { const int tt = i; i = k; k = tt; }
        const int e = i * W - i * (i - 1) / 2 + (k - i);           // upper-triangle index
        double s = 0.0;
#pragma unroll
        for (int u = 0; u < GR_NP; ++u) s += red[u * NE + e];
        part[q] = s;
    }
    const bool fin = tree_reduce(a.part, a.part + int64_t(gridDim.x) * nent, int(gridDim.x), int(blockIdx.x),
                                 nent, nent, a.counter, [&](int q, double tot) { a.out[q] = tot; });
    if (fin && a.fin_chol && threadIdx.x < 32) {
        __threadfence_block();
        chol_upper_warp(a.out, W, W, a.R, a.status, smg);       // rings idle
    }
}

// Per-warp variant (CAGMRES_OPT_GRAM = 2): every warp streams its own 32-row tiles through a
// private cp.async ring (no pair barrier) and accumulates all W(W+1)/2 sums for its lane's row
// (up to 78 accumulators: 8 warps per SM at <= 255 registers).
constexpr int GW_NW = 8, GW_S = 4;
template <int W>
__global__ void __launch_bounds__(GW_NW * 32, 1) k_gram_warp(GramArgs a) {
    extern __shared__ __align__(16) double smg[];
    constexpr int NE = W * (W + 1) / 2;
    __shared__ double red[GW_NW * NE];
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    pdl_wait();
    pdl_trigger();
    constexpr int SD = W * 32;
    double* ring = smg + int64_t(wp) * GW_S * SD;
    const int64_t T = a.n / 32;
    const int64_t Wn = int64_t(gridDim.x) * GW_NW;
    const int64_t g = int64_t(blockIdx.x) * GW_NW + wp;
    const int64_t cnt = band_count(T, Wn, g);
    const int part2 = 2 * (lane & 15), cfirst = lane >> 4;
    const double* srcl = a.P + a.ldp * cfirst + part2;
    const int64_t cstride = 2 * a.ldp;
    auto issue = [&](int64_t i, int stage) {
        if (i < cnt) {
            double* dst = ring + stage * SD + cfirst * 32 + part2;
            const double* src = srcl + band_tile(T, Wn, g, i, a.rev) * 32;
#pragma unroll
            for (int c = cfirst; c < W; c += 2, dst += 64, src += cstride) ptx::cp_async16(dst, src);
        }
        ptx::cp_async_commit();
    };
    double acc[NE];
#pragma unroll
    for (int e = 0; e < NE; ++e) acc[e] = 0.0;
    auto rank1 = [&](const double* sl) {
        double v[W];
#pragma unroll
        for (int c = 0; c < W; ++c) v[c] = sl[c * 32];
        int e = 0;
#pragma unroll
        for (int i = 0; i < W; ++i)
#pragma unroll
            for (int k = i; k < W; ++k, ++e) acc[e] = fma(v[i], v[k], acc[e]);
    };
#pragma unroll
    for (int s = 0; s < GW_S - 1; ++s) issue(s, s);
    int stage = 0;
    for (int64_t i = 0; i < cnt; ++i) {
        issue(i + GW_S - 1, stage == 0 ? GW_S - 1 : stage - 1);
        ptx::cp_async_wait<GW_S - 1>();
        __syncwarp();
        rank1(ring + stage * SD + lane);
        __syncwarp();
        stage = stage == GW_S - 1 ? 0 : stage + 1;
    }
    ptx::cp_async_wait<0>();
    if (blockIdx.x == 0 && wp == 0 && T * 32 + lane < a.n) {      // ragged tail rows [32 T, n)
        double* sl = ring + lane;
        const int64_t r = T * 32 + lane;
        for (int c = 0; c < W; ++c) sl[c * 32] = a.P[a.ldp * c + r];
        rank1(sl);
    }
#pragma unroll
    for (int e = 0; e < NE; ++e) {
        double sum = acc[e];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
        if (lane == 0) red[wp * NE + e] = sum;
    }
    __syncthreads();
    constexpr int nent = W * W;
    double* part = a.part + int64_t(blockIdx.x) * nent;
    for (int q = threadIdx.x; q < nent; q += blockDim.x) {
        int i = q % W, k = q / W;
        if (i > k) { const int tt = i; i = k; k = tt; }
        const int e = i * W - i * (i - 1) / 2 + (k - i);
        double s = 0.0;
#pragma unroll
        for (int u = 0; u < GW_NW; ++u) s += red[u * NE + e];
        part[q] = s;
    }
    const bool fin = tree_reduce(a.part, a.part + int64_t(gridDim.x) * nent, int(gridDim.x), int(blockIdx.x),
                                 nent, nent, a.counter, [&](int q, double tot) { a.out[q] = tot; });
    if (fin && a.fin_chol && threadIdx.x < 32) {
        __threadfence_block();
        chol_upper_warp(a.out, W, W, a.R, a.status, smg);
    }
}

int gram_warp(const Dev& d, const GramArgs& a0, cudaStream_t st) {
    GramArgs a = a0;
    a.rev = d.rev;
    auto go = [&](auto kfn) {
        size_t smem = size_t(GW_NW) * GW_S * a.w * 32 * sizeof(double);
        const size_t need = size_t(32 * 32) * sizeof(double);
        smem = smem < need ? need : smem;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        launch_pdl(kfn, dim3(unsigned(d.sms)), dim3(GW_NW * 32), smem, st, a);
    };
    switch (a.w) {
        case 6: go(k_gram_warp<6>); break;
        case 7: go(k_gram_warp<7>); break;
        case 8: go(k_gram_warp<8>); break;
        case 9: go(k_gram_warp<9>); break;
        case 10: go(k_gram_warp<10>); break;
        case 11: go(k_gram_warp<11>); break;
        case 12: go(k_gram_warp<12>); break;
        default: return -1;
    }
    return 0;
}

int gram_dfma(const Dev& d, const GramArgs& a0, cudaStream_t st) {
    GramArgs a = a0;
    a.rev = d.rev;
    const bool aligned = (reinterpret_cast<uintptr_t>(a.P) % 16 == 0) && a.ldp % 2 == 0;
    if (!aligned || a.w < 1 || a.w > 12 || a.n < 64 * GR_TW) return -1;
    if (d.gram == 2 && gram_warp(d, a, st) == 0) return 0;
    auto go = [&](auto kfn, int S) {
        size_t smem = size_t(GR_NP) * S * a.w * GR_TW * sizeof(double);
        const size_t need = size_t(32 * 32) * sizeof(double);     // Cholesky scratch
        smem = smem < need ? need : smem;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        launch_pdl(kfn, dim3(unsigned(d.sms)), dim3(GR_NT), smem, st, a);
    };
    switch (a.w) {
        case 1: go(k_gram_ring<1>, gram_stages<1>()); break;
        case 2: go(k_gram_ring<2>, gram_stages<2>()); break;
        case 3: go(k_gram_ring<3>, gram_stages<3>()); break;
        case 4: go(k_gram_ring<4>, gram_stages<4>()); break;
        case 5: go(k_gram_ring<5>, gram_stages<5>()); break;
        case 6: go(k_gram_ring<6>, gram_stages<6>()); break;
        case 7: go(k_gram_ring<7>, gram_stages<7>()); break;
        case 8: go(k_gram_ring<8>, gram_stages<8>()); break;
        case 9: go(k_gram_ring<9>, gram_stages<9>()); break;
        case 10: go(k_gram_ring<10>, gram_stages<10>()); break;
        case 11: go(k_gram_ring<11>, gram_stages<11>()); break;
        case 12: go(k_gram_ring<12>, gram_stages<12>()); break;
        default: return -1;
    }
    return 0;
}

}  // namespace kern
