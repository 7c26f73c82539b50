// stream.cu — row-streaming panel kernels on the FP64 tensor core (sm_100a DMMA).
//   K9  update : P[:, 0:w] -= X C                 (BOrth pass 2; x += V y)
//   K8  trsm   : P[:, c0:w] = (P R^{-1})[:, c0:w] (CholQR/SVQR update)
//       gemm   : P[:, c0:w] = (X M)[:, c0:w], X = [Q | P] contiguous (one-pass BOrth+CholQR
//                update (P - Q C) R^{-1} = [Q P] [-C R^{-1}; R^{-1}])
// Each warp forms 8-row x w output tiles with mma.sync.m8n8k4.f64 against the small
// right-hand matrix (C, or R^{-1}), whose B-fragments live in registers for the whole
// kernel.  A fragments (8 rows x 4 columns) and the P tile are loaded straight from global
// memory — each warp keeps U 8-row groups of loads in flight before its DMMAs — and results
// are stored straight back (one pass: read X and P once, write P once).
// TRSM uses the explicit inverse of the w x w triangular factor, formed once per CTA in
// shared memory by column back-substitution (what blocked GPU TRSMs do for their diagonal
// blocks); the product with P then runs on the tensor core like the update.
#include <cstdint>

#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NWARP = NT / 32;

struct StreamArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;     // update: X (n x jx); trsm: unused (A = P)
    double* P; int64_t ldp; int w;
    const double* M; int64_t ldm;             // C (jx x w) or R (w x w), leading dim ldm
    int c0;                                   // trsm: first column written
    int pf = 0;                               // L2 prefetch ahead of the ring (Dev::panel_pf)
    // 1: the kernel immediately before this one in the stream does not write X or P (it only
    // produced C / R), so the ring kernels issue their first tile copies BEFORE
    // griddepcontrol.wait and fill their pipelines while that kernel drains (PDL)
    int early = 0;
    int rev = 0;                              // tile order (band_tile), from Dev::rev
};

// R^{-1} (upper, w x w) into sRi[k*32 + c]; one thread per column (back substitution)
__device__ __forceinline__ void upper_inverse(const double* R, int w, double* sRi, double* sInv) {
    for (int k = threadIdx.x; k < 32; k += NT) sInv[k] = k < w ? 1.0 / R[k + int64_t(w) * k] : 0.0;
    __syncthreads();
    for (int c = threadIdx.x; c < 32; c += NT) {
        for (int k = 0; k < 32; ++k) sRi[k * 32 + c] = 0.0;
        if (c >= w) continue;
        sRi[c * 32 + c] = sInv[c];
        for (int k = c - 1; k >= 0; --k) {
            double s = 0.0;
            for (int l = k + 1; l <= c; ++l) s = fma(R[k + int64_t(w) * l], sRi[l * 32 + c], s);
            sRi[k * 32 + c] = -s * sInv[k];
        }
    }
    __syncthreads();
}

// MODE 0: update (A = X, B = C, D = P - A B); MODE 1: trsm (A = P, B = R^{-1}, D = A B);
// MODE 2: gemm (A = X with jx = K columns that include P, B = M, D = A B).
template <int MODE, int KTM, int NTN, int U>
__global__ void __launch_bounds__(NT) k_rows_mma(StreamArgs a) {
    __shared__ double sB[32 * 32 + 32];
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w;
    const int K = MODE == 1 ? w : a.jx;
    if (MODE == 1) upper_inverse(a.M, w, sB, sB + 32 * 32);   // (ldm == w for R)
    // B fragments: b[kt][nt] = B[4kt + tig][8nt + gid]
    double b[KTM][NTN];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            const int k = 4 * kt + tig, c = 8 * nt + gid;
            double v = 0.0;
            if (k < K && c < w) v = MODE != 1 ? a.M[k + a.ldm * c] : sB[k * 32 + c];
            b[kt][nt] = v;
        }
    // per-lane column pointers (clamped: the matching B rows / stored columns are masked)
    const double* acol[KTM];
    const double* Abase = MODE != 1 ? a.X : a.P;
    const int64_t ldA = MODE != 1 ? a.ldx : a.ldp;
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt) acol[kt] = Abase + ldA * min(4 * kt + tig, K - 1);
    double* pcol[NTN][2];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) pcol[nt][h] = a.P + a.ldp * min(8 * nt + 2 * tig + h, w - 1);
    bool wcol[NTN][2];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = 8 * nt + 2 * tig + h;
            wcol[nt][h] = c < w && (MODE == 0 || c >= a.c0);
        }
    const int KT = (K + 3) / 4;
    // MODE 2 writes P in place: every output row depends only on the same row of X (which
    // holds P), loaded by the same warp before it stores — rows are private to a warp.

    const int64_t ngroups = (a.n + 7) / 8;
    const int64_t nsg = (ngroups + U - 1) / U;
    const int64_t wstride = int64_t(gridDim.x) * NWARP;
    for (int64_t sg = int64_t(blockIdx.x) * NWARP + wp; sg < nsg; sg += wstride) {
        double av[U][KTM];
        double d[U][NTN][2];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t row = (sg * U + u) * 8 + gid;
            const bool ok = row < a.n;
#pragma unroll
            for (int kt = 0; kt < KTM; ++kt) av[u][kt] = (ok && kt < KT) ? __ldcs(acol[kt] + row) : 0.0;
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h) d[u][nt][h] = (MODE == 0 && ok) ? __ldcs(pcol[nt][h] + row) : 0.0;
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int kt = 0; kt < KTM; ++kt) {
                const double am = MODE == 0 ? -av[u][kt] : av[u][kt];
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt) ptx::dmma(d[u][nt][0], d[u][nt][1], am, b[kt][nt]);
            }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t row = (sg * U + u) * 8 + gid;
            if (row < a.n) {
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (wcol[nt][h]) __stcs(pcol[nt][h] + row, d[u][nt][h]);
            }
        }
    }
}

// Per-warp cp.async pipeline (aligned panels): each warp streams its band-order share (kern::band_tile) of the TW-row tiles of
// the input columns (X then P for the update, P for TRSM) through its own S-stage shared
// ring; 8-row groups read A fragments (8 rows x 4 cols) from the ring with a column stride
// of TW+8 doubles (== 8 mod 16: conflict free for that pattern) and store results directly.
constexpr int RP_S = 3;

template <int MODE, int KTM, int NTN, int TW, int MAXT = 512>   // MAXT 256: up to 255 registers
__global__ void __launch_bounds__(MAXT, 1) k_rows_pipe(StreamArgs a) {
    extern __shared__ __align__(16) double smp[];
    constexpr int SP = TW + 4;     // == 4 mod 16 doubles: A (8 rows x 4 cols) and P (8 rows x cols
                                   // 2 tig + h) fragment reads both take the 2 ideal wavefronts
                                   // (TW + 8 put the 4 P columns of a lane quad on the same banks)
    __shared__ double sB[32 * 32 + 32];
    __shared__ const double* sCol[96];                         // column base pointers (ncol <= 96)
    if (!a.early) {
        pdl_wait();
        pdl_trigger();
    }
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w;
    const int K = MODE == 1 ? w : a.jx;
    const int jxl = MODE != 1 ? a.jx : 0;
    const int ncol = MODE == 2 ? a.jx : jxl + w;               // gemm: P is inside X
    for (int c = threadIdx.x; c < ncol; c += blockDim.x)
        sCol[c] = c < jxl ? a.X + a.ldx * c : a.P + a.ldp * (c - jxl);
    __syncthreads();
    // measured (profiles/r1_launches_C2_pf.txt): prefetch helps narrow panels, hurts wide ones
    const bool d_pf = a.pf != 0 && TW == 32 && ncol <= 24;
    const int64_t stage_d = int64_t(ncol) * SP;
    double* ring = smp + int64_t(wp) * RP_S * stage_d;
    const int64_t T = a.n / TW;
    const int64_t W = int64_t(gridDim.x) * nw;
    const int64_t g = int64_t(blockIdx.x) * nw + wp;
    const int64_t cnt = band_count(T, W, g);                  // tiles of this warp (band order)
    auto colptr = [&](int c) -> const double* { return sCol[c]; };
    // copy slots: lane covers 16-B part (lane % CPC) of columns lane / CPC, + 32 / CPC, ...
    constexpr int CPC = TW * 8 / 16;
    constexpr int CSTEP = 32 / CPC;
    const int part2 = 2 * (lane % CPC), cfirst = lane / CPC;
    auto issue = [&](int64_t i, int stage) {
        if (i < cnt) {
            double* dst = ring + stage * stage_d + part2;
            const int64_t r0 = band_tile(T, W, g, i, a.rev) * TW + part2;
#pragma unroll 4
            for (int c = cfirst; c < ncol; c += CSTEP) ptx::cp_async16(dst + c * SP, sCol[c] + r0);
        }
        ptx::cp_async_commit();
    };
    const int KT = (K + 3) / 4;
    int acol[KTM];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt) acol[kt] = ((MODE == 1 ? jxl : 0) + min(4 * kt + tig, K - 1)) * SP;
    int pcol[NTN][2];
    bool wcol[NTN][2];
    double* pst[NTN][2];                                       // per-lane output column pointers
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = 8 * nt + 2 * tig + h;
            pcol[nt][h] = (jxl + min(c, w - 1)) * SP;
            wcol[nt][h] = c < w && (MODE == 0 || c >= a.c0);
            pst[nt][h] = a.P + a.ldp * min(c, w - 1) + gid;
        }
#pragma unroll
    for (int s = 0; s < RP_S - 1; ++s) issue(s, s);
    if (a.early) {                                             // X, P final before the predecessor
        pdl_wait();
        pdl_trigger();
    }
    if (MODE == 1) upper_inverse(a.M, w, sB, sB + 32 * 32);  // (has __syncthreads)
    // B fragments (update: -C, so d = P + A (-C) needs no per-element negation)
    double b[KTM][NTN];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            const int k = 4 * kt + tig, c = 8 * nt + gid;
            double v = 0.0;
            if (k < K && c < w) v = MODE != 1 ? a.M[k + a.ldm * c] : sB[k * 32 + c];
            b[kt][nt] = MODE == 0 ? -v : v;
        }
    int stage = 0, stage_in = RP_S - 1;
    for (int64_t i = 0; i < cnt; ++i) {
        issue(i + RP_S - 1, stage_in);
        if (d_pf && i + RP_S - 1 + ptx::PF_DIST < cnt) {
            const int64_t rp = band_tile(T, W, g, i + RP_S - 1 + ptx::PF_DIST, a.rev) * TW;
            constexpr int LPC = TW / 16;                        // 128-B lines per column tile
            for (int q = lane; q < ncol * LPC; q += 32) ptx::prefetch_l2(colptr(q / LPC) + rp + 16 * (q % LPC));
        }
        ptx::cp_async_wait<RP_S - 1>();
        __syncwarp();
        const double* sl = ring + stage * stage_d + gid;
        const int64_t toff = band_tile(T, W, g, i, a.rev) * TW;
        // per-tile operand pointers; the 8-row groups below are unrolled, so every shared load
        // and global store is [register + immediate]
        const double* sa[KTM];
#pragma unroll
        for (int kt = 0; kt < KTM; ++kt) sa[kt] = sl + acol[kt];
        const double* sd[NTN][2];
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) sd[nt][h] = sl + pcol[nt][h];
#pragma unroll
        for (int g8 = 0; g8 < TW / 8; ++g8) {
            double d[NTN][2];
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h) d[nt][h] = MODE == 0 ? sd[nt][h][8 * g8] : 0.0;
#pragma unroll
            for (int kt = 0; kt < KTM; ++kt) {
                if (kt >= KT) break;                            // uniform: skip padded k-steps
                const double av = sa[kt][8 * g8];
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt) ptx::dmma(d[nt][0], d[nt][1], av, b[kt][nt]);
            }
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h)
                    if (wcol[nt][h]) pst[nt][h][toff + 8 * g8] = d[nt][h];   // (L2-normal: the next
        }                                                             //  kernel reads it, serpentine)
        __syncwarp();
        stage = stage == RP_S - 1 ? 0 : stage + 1;
        stage_in = stage_in == RP_S - 1 ? 0 : stage_in + 1;
    }
    ptx::cp_async_wait<0>();
    // ragged tail rows [T*TW, n): warp 0 of CTA 0, direct zero-padded loads
    if (blockIdx.x == 0 && wp == 0) {
        for (int64_t r0 = T * TW; r0 < a.n; r0 += 8) {
            const int64_t row = r0 + gid;
            const bool ok = row < a.n;
            double d[NTN][2];
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                for (int h = 0; h < 2; ++h) d[nt][h] = (MODE == 0 && ok) ? sCol[pcol[nt][h] / SP][row] : 0.0;
#pragma unroll
            for (int kt = 0; kt < KTM; ++kt) {
                if (kt < KT) {
                    const double av = ok ? sCol[acol[kt] / SP][row] : 0.0;
#pragma unroll
                    for (int nt = 0; nt < NTN; ++nt) ptx::dmma(d[nt][0], d[nt][1], av, b[kt][nt]);
                }
            }
            if (ok) {
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (wcol[nt][h]) a.P[a.ldp * (8 * nt + 2 * tig + h) + row] = d[nt][h];
            }
        }
    }
}

template <int MODE, int KTM, int NTN, int TW>
bool run_pipe_tw(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    const bool aligned = ((reinterpret_cast<uintptr_t>(a.P) | reinterpret_cast<uintptr_t>(MODE != 1 ? a.X : a.P)) % 16 == 0) &&
                         (a.ldp % 2 == 0) && (MODE == 1 || a.ldx % 2 == 0);
    if (!aligned || a.n < 64 * TW) return false;
    const int ncol = MODE == 2 ? a.jx : (MODE == 0 ? a.jx : 0) + a.w;
    const size_t ring_w = size_t(RP_S) * ncol * (TW + 4) * sizeof(double);
    int nw = int((200 * 1024) / ring_w);
    nw = nw < 2 ? 2 : (nw > 16 ? 16 : nw);
    const size_t smem = size_t(nw) * ring_w;
    ++g_launches;
    if (nw <= 8) {      // wide panels: few warps fit anyway -> let them keep every pointer in registers
        cudaFuncSetAttribute(k_rows_pipe<MODE, KTM, NTN, TW, 256>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        launch_pdl(k_rows_pipe<MODE, KTM, NTN, TW, 256>, dim3(unsigned(d.sms)), dim3(32 * nw), smem, st, a);
    } else {
        cudaFuncSetAttribute(k_rows_pipe<MODE, KTM, NTN, TW, 512>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        launch_pdl(k_rows_pipe<MODE, KTM, NTN, TW, 512>, dim3(unsigned(d.sms)), dim3(32 * nw), smem, st, a);
    }
    return true;
}

// wide panels: 16-row tiles, about twice the warps per SM
template <int MODE, int KTM, int NTN>
bool run_pipe(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    // measured (profiles/r1_launches_C2_tw*.txt): 16-row tiles win for wide light-compute
    // panels (x += V y, w = 1) and the one-pass gemm, lose for the BOrth update (w = 10)
    const int ncol = MODE == 2 ? a.jx : (MODE == 0 ? a.jx : 0) + a.w;
    if (d.panel_tw16 && ncol >= 24 && (MODE == 2 || a.w <= 8)) return run_pipe_tw<MODE, KTM, NTN, 16>(d, a, st);
    return run_pipe_tw<MODE, KTM, NTN, 32>(d, a, st);
}

template <int MODE, int KTM, int NTN, int U>
void run(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    if (run_pipe<MODE, KTM, NTN>(d, a, st)) return;
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_rows_mma<MODE, KTM, NTN, U>, NT, 0);
    if (occ < 1) occ = 1;
    const int64_t nsg = ((a.n + 7) / 8 + U - 1) / U;
    int64_t g = int64_t(d.sms) * occ;
    const int64_t cap = (nsg + NWARP - 1) / NWARP;
    if (g > cap) g = cap;
    if (g < 1) g = 1;
    ++g_launches;
    k_rows_mma<MODE, KTM, NTN, U><<<unsigned(g), NT, 0, st>>>(a);
}

template <int MODE>
int dispatch(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    const int w = a.w, K = MODE == 1 ? w : a.jx;
    const int ntn = w <= 8 ? 1 : (w <= 16 ? 2 : 4);
    const int ktm = K <= 4 ? 1 : (K <= 8 ? 2 : (K <= 16 ? 4 : (K <= 32 ? 8 : (K <= 64 ? 16 : 0))));
    switch (ktm * 10 + ntn) {
        case 11: run<MODE, 1, 1, 4>(d, a, st); return 0;
        case 21: run<MODE, 2, 1, 4>(d, a, st); return 0;
        case 41: run<MODE, 4, 1, 2>(d, a, st); return 0;
        case 81: run<MODE, 8, 1, 2>(d, a, st); return 0;
        case 161: run<MODE, 16, 1, 1>(d, a, st); return 0;
        case 12: run<MODE, 1, 2, 4>(d, a, st); return 0;
        case 22: run<MODE, 2, 2, 2>(d, a, st); return 0;
        case 42: run<MODE, 4, 2, 2>(d, a, st); return 0;
        case 82: run<MODE, 8, 2, 2>(d, a, st); return 0;
        case 162: run<MODE, 16, 2, 1>(d, a, st); return 0;
        case 14: run<MODE, 1, 4, 2>(d, a, st); return 0;
        case 24: run<MODE, 2, 4, 2>(d, a, st); return 0;
        case 44: run<MODE, 4, 4, 1>(d, a, st); return 0;
        case 84: run<MODE, 8, 4, 1>(d, a, st); return 0;
        case 164: run<MODE, 16, 4, 1>(d, a, st); return 0;
        default: return -1;
    }
}
// w = 1 TRSM (Arnoldi normalisation v /= h, q_0 = r / beta): P[:,0] *= 1 / R[0].  A DMMA
// tile would waste 7/8 of its work and 12 M instructions on 2 M rows; this is a plain
// vectorised stream (16-B loads/stores, grid = SMs x 4).  The product p * (1/r) is rounded once,
// exactly like the DMMA path (fma(p, 1/r, 0)), so results are bitwise identical.
__global__ void __launch_bounds__(256) k_scale1(int64_t n, double* __restrict__ p, const double* __restrict__ r) {
    pdl_wait();
    pdl_trigger();
    const double inv = 1.0 / __ldg(r);
    const int64_t i0 = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const int64_t stride = int64_t(gridDim.x) * blockDim.x;
    const bool al = (reinterpret_cast<uintptr_t>(p) & 15) == 0;
    if (al) {
        double2* p2 = reinterpret_cast<double2*>(p);
        const int64_t n2 = n >> 1;
        int64_t i = i0;
        for (; i + 3 * stride < n2; i += 4 * stride) {       // 4 x 16 B in flight per thread
            double2 v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = __ldcs(p2 + i + u * stride);
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                v[u].x *= inv; v[u].y *= inv;
                p2[i + u * stride] = v[u];
            }
        }
        for (; i < n2; i += stride) {
            double2 v = __ldcs(p2 + i);
            v.x *= inv; v.y *= inv;
            p2[i] = v;
        }
        if (i0 == 0 && (n & 1)) p[n - 1] *= inv;
    } else {
        for (int64_t i = i0; i < n; i += stride) p[i] *= inv;
    }
}
// Scalar-FP64 TRSM on a per-warp cp.async ring (CAGMRES_OPT_TRSM = 1, default for w <= 16).
// The DMMA form pads the w x w triangular R^{-1} to 16 x 16 tiles (34 % useful MACs at w = 11)
// and was tensor-pipe co-limited (ncu: 67 us, 4.4 TB/s at n = 2.1M, w = 11); here lane l owns
// row l of a 32-row tile, reads its W panel values from the ring once and forms
// out[c] = sum_{k <= c} p[k] Ri[k][c] for c >= c0 with R^{-1} broadcast from shared memory:
// w(w+1)/2 DFMAs per row, no padding.
template <int W, int RS>
__global__ void __launch_bounds__(256, 1) k_trsm_ring(StreamArgs a) {
    extern __shared__ __align__(16) double smt[];
    __shared__ double sB[32 * 32 + 32];
    constexpr int WP = W + (W & 1);                             // even row stride: 16-B pairs
    __shared__ __align__(16) double sRi[W * WP];
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (!a.early) {
        pdl_wait();
        pdl_trigger();
    }
    // 64-row tiles, two rows per lane (rows 2 lane, 2 lane + 1: one 16-B shared load per column):
    // every broadcast load of two R^{-1} entries feeds four FMAs (ncu, 32-row tiles with one row
    // per lane: MIO-throttle / short-scoreboard bound on the R^{-1} loads)
    constexpr int TR = 64;
    constexpr int SD = W * TR;
    double* ring = smt + int64_t(wp) * RS * SD;
    const int64_t T = a.n / TR;
    const int64_t Wn = int64_t(gridDim.x) * nw;
    const int64_t g = int64_t(blockIdx.x) * nw + wp;
    const int64_t cnt = band_count(T, Wn, g);
    const int c0 = a.c0;
    auto issue = [&](int64_t i, int stage) {
        if (i < cnt) {
            double* dst = ring + stage * SD + 2 * lane;
            const double* src = a.P + band_tile(T, Wn, g, i, a.rev) * TR + 2 * lane;
#pragma unroll
            for (int c = 0; c < W; ++c) ptx::cp_async16(dst + c * TR, src + a.ldp * c);
        }
        ptx::cp_async_commit();
    };
    // two output columns per 16-B broadcast load of R^{-1}: out[c], out[c+1] = sum_k p[k] Ri[k][.]
    // (Ri[c+1][c] = 0: the extra term adds an exact zero); per output the FMAs run k = 0..c+1
    auto rowout2 = [&](const double (&v0)[W], const double (&v1)[W], double* out) {
#pragma unroll
        for (int c = 0; c < W; c += 2) {
            if (c + 1 < c0) continue;
            double a00 = 0.0, a01 = 0.0, a10 = 0.0, a11 = 0.0;
#pragma unroll
            for (int k = 0; k <= c + 1 && k < W; ++k) {
                const double2 r2 = *reinterpret_cast<const double2*>(&sRi[k * WP + c]);
                a00 = fma(v0[k], r2.x, a00);
                a01 = fma(v0[k], r2.y, a01);
                a10 = fma(v1[k], r2.x, a10);
                a11 = fma(v1[k], r2.y, a11);
            }
            if (c >= c0) *reinterpret_cast<double2*>(out + a.ldp * c) = make_double2(a00, a10);
            if (c + 1 < W) *reinterpret_cast<double2*>(out + a.ldp * (c + 1)) = make_double2(a01, a11);
        }
    };
    auto rowout = [&](const double (&v)[W], double* out) {           // one row (ragged tail)
#pragma unroll
        for (int c = 0; c < W; c += 2) {
            if (c + 1 < c0) continue;
            double acc0 = 0.0, acc1 = 0.0;
#pragma unroll
            for (int k = 0; k <= c + 1 && k < W; ++k) {
                const double2 r2 = *reinterpret_cast<const double2*>(&sRi[k * WP + c]);
                acc0 = fma(v[k], r2.x, acc0);
                acc1 = fma(v[k], r2.y, acc1);
            }
            if (c >= c0) out[a.ldp * c] = acc0;
            if (c + 1 < W) out[a.ldp * (c + 1)] = acc1;
        }
    };
#pragma unroll
    for (int s = 0; s < RS - 1; ++s) issue(s, s);
    if (a.early) {                                             // P final before the Gram / Cholesky
        pdl_wait();
        pdl_trigger();
    }
    upper_inverse(a.M, W, sB, sB + 32 * 32);
    for (int q = threadIdx.x; q < W * WP; q += blockDim.x) {
        const int k = q / WP, c = q - k * WP;
        sRi[q] = c < W ? sB[k * 32 + c] : 0.0;                 // [k * WP + c] = R^{-1}[k][c]
    }
    __syncthreads();
    int stage = 0;
    for (int64_t i = 0; i < cnt; ++i) {
        issue(i + RS - 1, stage == 0 ? RS - 1 : stage - 1);
        ptx::cp_async_wait<RS - 1>();
        __syncwarp();
        const double* sl = ring + stage * SD + 2 * lane;
        double v0[W], v1[W];
#pragma unroll
        for (int k = 0; k < W; ++k) {
            const double2 p2 = *reinterpret_cast<const double2*>(sl + k * TR);
            v0[k] = p2.x;
            v1[k] = p2.y;
        }
        rowout2(v0, v1, a.P + band_tile(T, Wn, g, i, a.rev) * TR + 2 * lane);
        __syncwarp();
        stage = stage == RS - 1 ? 0 : stage + 1;
    }
    ptx::cp_async_wait<0>();
    if (blockIdx.x == 0 && wp == 0) {                          // ragged tail rows [64 T, n)
        for (int64_t r = T * TR + lane; r < a.n; r += 32) {
            double v[W];
#pragma unroll
            for (int k = 0; k < W; ++k) v[k] = a.P[a.ldp * k + r];
            rowout(v, a.P + r);
        }
    }
}

template <int W, int RS>
bool go_trsm_rs(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    const size_t ring_w = size_t(RS) * W * 64 * sizeof(double);
    int nw = int((200 * 1024) / ring_w);
    nw = nw < 2 ? 2 : (nw > 8 ? 8 : nw);              // <= 256 threads: R^{-1} stays in registers
    const size_t smem = size_t(nw) * ring_w;
    cudaFuncSetAttribute(k_trsm_ring<W, RS>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    launch_pdl(k_trsm_ring<W, RS>, dim3(unsigned(d.sms)), dim3(32 * nw), smem, st, a);
    return true;
}

template <int W>
bool go_trsm_ring(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    const bool aligned = (reinterpret_cast<uintptr_t>(a.P) % 16 == 0) && (a.ldp % 2 == 0);
    if (!aligned || a.n < 64 * 32) return false;
    switch (d.trsm_scalar) {             // ring stages (CAGMRES_OPT_TRSM 1..4 -> 3, 4, 6, 8)
        case 2: return go_trsm_rs<W, 4>(d, a, st);
        case 3: return go_trsm_rs<W, 6>(d, a, st);
        case 4: return go_trsm_rs<W, 8>(d, a, st);
        default: return go_trsm_rs<W, 3>(d, a, st);
    }
}

bool trsm_ring(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    switch (a.w) {
        case 2: return go_trsm_ring<2>(d, a, st);
        case 3: return go_trsm_ring<3>(d, a, st);
        case 4: return go_trsm_ring<4>(d, a, st);
        case 5: return go_trsm_ring<5>(d, a, st);
        case 6: return go_trsm_ring<6>(d, a, st);
        case 7: return go_trsm_ring<7>(d, a, st);
        case 8: return go_trsm_ring<8>(d, a, st);
        case 9: return go_trsm_ring<9>(d, a, st);
        case 10: return go_trsm_ring<10>(d, a, st);
        case 11: return go_trsm_ring<11>(d, a, st);
        case 12: return go_trsm_ring<12>(d, a, st);
        case 13: return go_trsm_ring<13>(d, a, st);
        case 14: return go_trsm_ring<14>(d, a, st);
        case 15: return go_trsm_ring<15>(d, a, st);
        case 16: return go_trsm_ring<16>(d, a, st);
        default: return false;
    }
}
}  // namespace

void update(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* P,
            int64_t ldp, int w, const double* C, cudaStream_t st, bool early) {
    if (n <= 0 || w <= 0) return;
    if (w == 1 && jx <= 32 && update_w1(d, n, X, ldx, jx, P, C, st) == 0) return;
    // wide X (> 64 columns): P -= X[:, s] C[s, :] in 64-column slabs (C viewed with ld jx);
    // a later slab follows a launch that wrote P: no early start for it
    for (int s0 = 0; s0 < jx; s0 += 64) {
        const int js = jx - s0 < 64 ? jx - s0 : 64;
        StreamArgs a{n, X + ldx * s0, ldx, js, P, ldp, w, C + s0, jx, 0, d.panel_pf, early && s0 == 0 ? 1 : 0, d.rev};
        dispatch<0>(d, a, st);
    }
}

int gemm_rows(const Dev& d, int64_t n, const double* X, int64_t ldx, int K, double* P, int64_t ldp, int w,
              const double* M, int64_t ldm, int c0, cudaStream_t st, bool early) {
    if (n <= 0 || w <= 0) return 0;
    if (K > 64 || w > 32) return -1;
    StreamArgs a{n, X, ldx, K, P, ldp, w, M, ldm, c0, d.panel_pf, early ? 1 : 0, d.rev};
    return dispatch<2>(d, a, st);
}

void trsm(const Dev& d, int64_t n, double* P, int64_t ldp, int w, const double* R, int c0,
          cudaStream_t st, bool early) {
    if (n <= 0 || w <= 0) return;
    if (w == 1 && c0 == 0) {
        int64_t g = int64_t(d.sms) * 4;
        const int64_t need = ((n >> 1) + 255) / 256;
        if (g > need) g = need < 1 ? 1 : need;
        ++g_launches;
        launch_pdl(k_scale1, dim3(unsigned(g)), dim3(256), 0, st, n, P, R);
        return;
    }
    StreamArgs a{n, nullptr, 0, 0, P, ldp, w, R, w, c0, d.panel_pf, early ? 1 : 0, d.rev};
    if (d.trsm_scalar && trsm_ring(d, a, st)) return;
    dispatch<1>(d, a, st);
}

}  // namespace kern
