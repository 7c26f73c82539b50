// fused.cu — BOrth pass 2 fused with the CholQR Gram of the updated panel.
//   P' = P - X C            (BOrth)
//   B  = [q_j P']^T [q_j P'] (CholQR Gram) and, on one GPU, R = chol(B)
// in one pass: the per-warp cp.async ring holds X, P and q_j tiles; each 8-row group's P'
// (tensor-core DMMA against the register-resident C) is stored to global memory AND written
// back into the warp's ring slot, from which the Gram fragments of the 32-row tile are read
// for the symmetric DMMA accumulation.  Saves the Gram kernel's separate read of the panel.
// Column stride TW+8 (== 8 mod 16) keeps the update's 8-row x 4-column fragment reads
// conflict-free; the Gram reads (4 rows x 8 columns) take a 2-way conflict there.
#include <algorithm>
#include <cstdint>

#include "dense_dev.cuh"
#include "kernels.h"
#include "ptx.h"
#include "reduce.cuh"

namespace kern {

namespace {
constexpr int UG_S = 3;
constexpr int UG_TW = 32;
}

template <int KTM, int NTN, int NTG>
__global__ void __launch_bounds__(512, 1) k_update_gram(UpdGramArgs a) {
    extern __shared__ __align__(16) double smp[];
    constexpr int TW = UG_TW, SP = TW + 8;
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w, jx = a.jx, wg = w + 1;
    // B fragments of C: b[kt][nt] = C[4kt + tig][8nt + gid]
    double b[KTM][NTN];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            const int k = 4 * kt + tig, c = 8 * nt + gid;
            b[kt][nt] = (k < jx && c < w) ? a.C[k + int64_t(jx) * c] : 0.0;
        }
    const int ncol = jx + w + 1;                                    // X | P | q_j
    const int64_t stage_d = int64_t(ncol) * SP;
    double* ring = smp + int64_t(wp) * UG_S * stage_d;
    const int64_t T = a.n / TW;
    const int64_t W = int64_t(gridDim.x) * nw;
    const int64_t g = int64_t(blockIdx.x) * nw + wp;
    const int64_t t0 = g * T / W, t1 = (g + 1) * T / W;
    auto colptr = [&](int c) -> const double* {
        return c < jx ? a.X + a.ldx * c : (c < jx + w ? a.P + a.ldp * (c - jx) : a.q0);
    };
    constexpr int CPC = TW * 8 / 16;
    auto issue = [&](int64_t t, int stage) {
        if (t < t1) {
            double* dst = ring + stage * stage_d;
            const int64_t r0 = t * TW;
            for (int q = lane; q < ncol * CPC; q += 32) {
                const int c = q / CPC, part = q - c * CPC;
                ptx::cp_async16(dst + c * SP + part * 2, colptr(c) + r0 + part * 2);
            }
        }
        ptx::cp_async_commit();
    };
    const int KT = (jx + 3) / 4;
    int acol[KTM];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt) acol[kt] = min(4 * kt + tig, jx - 1);
    int pcol[NTN][2];
    bool wcol[NTN][2];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = 8 * nt + 2 * tig + h;
            pcol[nt][h] = min(c, w - 1);
            wcol[nt][h] = c < w;
        }
    // Gram panel column p (0 = q_j, p >= 1: P' column p-1) -> slot column
    int gcol[NTG];
#pragma unroll
    for (int nt = 0; nt < NTG; ++nt) {
        const int p = min(8 * nt + gid, wg - 1);
        gcol[nt] = p == 0 ? jx + w : jx + p - 1;
    }
    double acc[NTG][NTG][2];
#pragma unroll
    for (int i = 0; i < NTG; ++i)
#pragma unroll
        for (int k = 0; k < NTG; ++k) acc[i][k][0] = acc[i][k][1] = 0.0;

    auto process = [&](double* sl, int64_t rbase, int rows_valid) {
        // (1) update: P' rows of 4 groups of 8, stored to global and back into the slot
#pragma unroll 1
        for (int g8 = 0; g8 < TW / 8; ++g8) {
            const int row = 8 * g8 + gid;
            double d[NTN][2];
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h) d[nt][h] = sl[(jx + pcol[nt][h]) * SP + row];
#pragma unroll
            for (int kt = 0; kt < KTM; ++kt)
                if (kt < KT) {
                    const double am = -sl[acol[kt] * SP + row];
#pragma unroll
                    for (int nt = 0; nt < NTN; ++nt) ptx::dmma(d[nt][0], d[nt][1], am, b[kt][nt]);
                }
            __syncwarp();
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h)
                    if (wcol[nt][h]) {
                        const int c = 8 * nt + 2 * tig + h;
                        sl[(jx + c) * SP + row] = d[nt][h];
                        if (row < rows_valid) __stcs(a.P + a.ldp * c + rbase + row, d[nt][h]);
                    }
        }
        __syncwarp();
        // (2) Gram of [q_j P'] over the tile's rows
#pragma unroll
        for (int u = 0; u < TW / 4; ++u) {
            const int row = 4 * u + tig;
            double bn[NTG];
#pragma unroll
            for (int nt = 0; nt < NTG; ++nt) bn[nt] = row < rows_valid ? sl[gcol[nt] * SP + row] : 0.0;
#pragma unroll
            for (int i = 0; i < NTG; ++i)
#pragma unroll
                for (int k = i; k < NTG; ++k) ptx::dmma(acc[i][k][0], acc[i][k][1], bn[i], bn[k]);
        }
        __syncwarp();
    };
#pragma unroll
    for (int s = 0; s < UG_S - 1; ++s) issue(t0 + s, s);
    int stage = 0;
    for (int64_t t = t0; t < t1; ++t) {
        issue(t + UG_S - 1, (stage + UG_S - 1) % UG_S);
        ptx::cp_async_wait<UG_S - 1>();
        __syncwarp();
        process(ring + stage * stage_d, t * TW, TW);
        stage = (stage + 1) % UG_S;
    }
    ptx::cp_async_wait<0>();
    if (blockIdx.x == 0 && wp == 0 && T * TW < a.n) {            // ragged tail through the slot
        double* sl = ring;                                        // ring idle now
        const int64_t r0 = T * TW;
        const int rows = int(a.n - r0);
        for (int q = lane; q < ncol * TW; q += 32) {
            const int c = q / TW, r = q - c * TW;
            sl[c * SP + r] = r < rows ? colptr(c)[r0 + r] : 0.0;
        }
        __syncwarp();
        process(sl, r0, rows);
    }
    // ---- CTA reduction of the Gram accumulators (fixed order) + last-CTA total ----
    __syncthreads();
    double* red = smp;
    constexpr int FR = NTG * NTG * 64;
#pragma unroll
    for (int i = 0; i < NTG; ++i)
#pragma unroll
        for (int k = 0; k < NTG; ++k) {
            red[wp * FR + (i * NTG + k) * 64 + lane * 2 + 0] = acc[i][k][0];
            red[wp * FR + (i * NTG + k) * 64 + lane * 2 + 1] = acc[i][k][1];
        }
    __syncthreads();
    const int nent = wg * wg;
    double* part = a.part + int64_t(blockIdx.x) * nent;
    for (int e = threadIdx.x; e < nent; e += blockDim.x) {
        const int i0 = e % wg, c0 = e / wg;
        int mt = i0 >> 3, nt = c0 >> 3, ml = i0 & 7, nl = c0 & 7;
        if (mt > nt) { const int tt = mt; mt = nt; nt = tt; const int q = ml; ml = nl; nl = q; }
        const int ln = ml * 4 + (nl >> 1), h = nl & 1;
        double sum = 0.0;
        for (int q = 0; q < nw; ++q) sum += red[q * FR + (mt * NTG + nt) * 64 + ln * 2 + h];
        part[e] = sum;
    }
    const bool fin = tree_reduce(a.part, a.part + int64_t(gridDim.x) * nent, int(gridDim.x), int(blockIdx.x),
                                 nent, nent, a.counter, [&](int e, double tot) { a.out[e] = tot; });
    if (fin && a.fin_chol && threadIdx.x < 32) {
        __threadfence_block();
        chol_upper_warp(a.out, wg, wg, a.R, a.status, smp);
    }
}

int update_gram(const Dev& d, const UpdGramArgs& a, cudaStream_t st) {
    const int w = a.w, jx = a.jx, wg = w + 1;
    const bool aligned = ((reinterpret_cast<uintptr_t>(a.X) | reinterpret_cast<uintptr_t>(a.P) |
                           reinterpret_cast<uintptr_t>(a.q0)) % 16 == 0) && a.ldx % 2 == 0 && a.ldp % 2 == 0;
    if (!aligned || jx < 1 || jx > 64 || wg > 16 || a.n < 64 * UG_TW) return -1;
    const int ncol = jx + w + 1;
    const size_t ring_w = size_t(UG_S) * ncol * (UG_TW + 8) * sizeof(double);
    int nw = int((200 * 1024) / ring_w);
    nw = nw < 2 ? 2 : (nw > 16 ? 16 : nw);
    const int ntg = wg <= 8 ? 1 : 2;
    size_t smem = std::max(size_t(nw) * ring_w, size_t(nw) * ntg * ntg * 64 * sizeof(double));
    smem = std::max(smem, size_t(32 * nw) * sizeof(double));
    const int ntn = w <= 8 ? 1 : 2;
    const int ktm = jx <= 4 ? 1 : (jx <= 8 ? 2 : (jx <= 16 ? 4 : (jx <= 32 ? 8 : 16)));
    auto go = [&](auto kfn) {
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        kfn<<<unsigned(d.sms), 32 * nw, smem, st>>>(a);
    };
    switch (ktm * 100 + ntn * 10 + ntg) {
        case 111: go(k_update_gram<1, 1, 1>); break;
        case 211: go(k_update_gram<2, 1, 1>); break;
        case 411: go(k_update_gram<4, 1, 1>); break;
        case 811: go(k_update_gram<8, 1, 1>); break;
        case 1611: go(k_update_gram<16, 1, 1>); break;
        case 112: go(k_update_gram<1, 1, 2>); break;
        case 212: go(k_update_gram<2, 1, 2>); break;
        case 412: go(k_update_gram<4, 1, 2>); break;
        case 812: go(k_update_gram<8, 1, 2>); break;
        case 1612: go(k_update_gram<16, 1, 2>); break;
        case 122: go(k_update_gram<1, 2, 2>); break;
        case 222: go(k_update_gram<2, 2, 2>); break;
        case 422: go(k_update_gram<4, 2, 2>); break;
        case 822: go(k_update_gram<8, 2, 2>); break;
        case 1622: go(k_update_gram<16, 2, 2>); break;
        default: return -1;
    }
    return 0;
}

size_t update_gram_ws_doubles(const Dev& d) { return 2 * size_t(d.sms) * 16 * 16; }

}  // namespace kern
