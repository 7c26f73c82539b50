// xty.cu — K4/K5: C = X^T Y for tall-skinny X (n x jx) and Y (n x w <= 32), FP64.
//   * BOrth pass 1: C = Q[:,0:j]^T P            ("MAGMA tall-skinny DGEMV")
//   * CholQR Gram:  B = V^T V, then R = chol(B)  ("batched DGEMM")
//
// The contraction over rows runs on the FP64 tensor core (mma.sync.m8n8k4.f64, 256 FMAs
// per warp instruction): with scalar DFMA the kernel was issue-bound at the occupancy its
// accumulators allow (ncu: 107 M instructions, 0.73 IPC).  Fragments are loaded straight
// from global memory: an A/B fragment is 8 columns x 4 consecutive rows, i.e. eight fully
// used 32-B sectors per warp load, and each warp keeps U k-steps (4U rows) of fragments in
// flight before issuing its DMMAs, so bytes in flight scale with the resident warps.  (A
// TMA bulk-copy ring was measured slower on this shape: tools/tma_probe.cu.)
// Gram (X == Y): the A fragment is reused as B and only the upper block triangle is formed.
// Each CTA reduces its warps' 8x8 accumulators in a fixed order; the LAST CTA (atomic
// ticket) sums all CTA partials in a fixed order (run-to-run bitwise reproducible) and, for
// CholQR on one GPU, factors the Gram in the same launch.
#include <algorithm>
#include <cstdint>

#include "dense_dev.cuh"
#include "reduce.cuh"
#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 512;                 // one CTA per SM: few partials for the final reduction
constexpr int NWARP = NT / 32;
}

struct XtyArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;
    const double* Y; int64_t ldy; int w;
    int chunk;                  // X columns per blockIdx.y chunk (= 8*MT)
    double* part;               // per-CTA partials (chunk x w each)
    double* out;                // jx x w, ld jx
    unsigned int* counter;
    int fin_chol;
    double* R;
    int* status;
    int pf = 0;                 // L2 prefetch ahead of the ring (Dev::panel_pf)
    int rev = 0;                // tile order (band_tile), from Dev::rev
};

// ---- CTA partial -> two-level fixed-order total (+ Cholesky) ---------------------------
// Partials of y-chunk `by` live at part[(by * gx + bx) * nent]; its group partials after all
// CTA partials; its counters at counter[by * TR_CNT].
__device__ __forceinline__ void xty_finish(const XtyArgs& a, int nent_cta) {
    const int gx = int(gridDim.x), by = int(blockIdx.y);
    const int ng = (gx + TR_GS - 1) / TR_GS;
    const double* pb = a.part + int64_t(by) * gx * nent_cta;
    double* gp = a.part + int64_t(gridDim.y) * gx * nent_cta + int64_t(by) * ng * nent_cta;
    const int jx = a.jx, w = a.w;
    const bool fin = tree_reduce(pb, gp, gx, int(blockIdx.x), nent_cta, a.chunk * w, a.counter + by * TR_CNT,
                                 [&](int e, double tot) {
                                     const int il = e % a.chunk, c = e / a.chunk, i = by * a.chunk + il;
                                     if (i < jx) a.out[i + int64_t(jx) * c] = tot;
                                 });
    if (fin && a.fin_chol && threadIdx.x < 32) {                 // gy == 1 for the Gram
        extern __shared__ double red[];
        __threadfence_block();
        chol_upper_warp(a.out, jx, w, a.R, a.status, red);
    }
}

// MT = 8-column tiles of X per chunk, NTN = 8-column tiles of Y, U = k-steps in flight.
template <int MT, int NTN, int U, bool SYM>
__global__ void __launch_bounds__(NT, 1) k_xty_mma(XtyArgs a) {
    extern __shared__ double red[];                              // NWARP x MT x NTN x 64 (>= NT)
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w;
    const int colbase = SYM ? 0 : blockIdx.y * a.chunk;
    const int nxc = SYM ? w : min(a.chunk, a.jx - colbase);
    // per-lane column pointers (clamped columns feed only discarded accumulator entries)
    const double* ycol[NTN];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt) ycol[nt] = a.Y + a.ldy * min(8 * nt + gid, w - 1);
    const double* xcol[SYM ? 1 : MT];
    if constexpr (!SYM) {
#pragma unroll
        for (int mt = 0; mt < MT; ++mt) xcol[mt] = a.X + a.ldx * (colbase + min(8 * mt + gid, nxc - 1));
    }
    double acc[MT][NTN][2];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) acc[mt][nt][0] = acc[mt][nt][1] = 0.0;

    const int64_t rows_per_ss = 4 * U;
    const int64_t nss = (a.n + rows_per_ss - 1) / rows_per_ss;
    const int64_t wstride = int64_t(gridDim.x) * NWARP;
    for (int64_t ss = int64_t(blockIdx.x) * NWARP + wp; ss < nss; ss += wstride) {
        const int64_t r0 = ss * rows_per_ss + tig;
        double bv[U][NTN];
        double av[SYM ? 1 : U][SYM ? 1 : MT];
        if (r0 + 4 * (U - 1) < a.n) {                              // full super-step
#pragma unroll
            for (int u = 0; u < U; ++u) {
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt) bv[u][nt] = __ldcs(ycol[nt] + r0 + 4 * u);
                if constexpr (!SYM) {
#pragma unroll
                    for (int mt = 0; mt < MT; ++mt) av[u][mt] = __ldcs(xcol[mt] + r0 + 4 * u);
                }
            }
        } else {                                                    // ragged tail: zero padded
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const bool ok = r0 + 4 * u < a.n;
#pragma unroll
                for (int nt = 0; nt < NTN; ++nt) bv[u][nt] = ok ? ycol[nt][r0 + 4 * u] : 0.0;
                if constexpr (!SYM) {
#pragma unroll
                    for (int mt = 0; mt < MT; ++mt) av[u][mt] = ok ? xcol[mt][r0 + 4 * u] : 0.0;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if constexpr (SYM) {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                    for (int nt = mt; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], bv[u][mt], bv[u][nt]);
            } else {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                    for (int nt = 0; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], av[u][mt], bv[u][nt]);
            }
        }
    }
    // ---- CTA reduction over warps (fixed order) ----
    constexpr int FR = MT * NTN * 64;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 0] = acc[mt][nt][0];
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 1] = acc[mt][nt][1];
        }
    __syncthreads();
    const int nent = a.chunk * w;
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * nent;
    for (int e = threadIdx.x; e < nent; e += NT) {
        const int il = e % a.chunk, c = e / a.chunk;
        int mt = il >> 3, nt = c >> 3, ml = il & 7, nl = c & 7;
        if (SYM && mt > nt) { const int t = mt; mt = nt; nt = t; const int q = ml; ml = nl; nl = q; }
        const int ln = ml * 4 + (nl >> 1), h = nl & 1;
        double sum = 0.0;
        if (mt < MT && nt < NTN)
            for (int q = 0; q < NWARP; ++q) sum += red[q * FR + (mt * NTN + nt) * 64 + ln * 2 + h];
        part[il + int64_t(a.chunk) * c] = sum;
    }
    xty_finish(a, nent);
}

// ======================================================================================
// Per-warp cp.async pipeline (aligned panels).  Each warp streams its band-order share
// (kern::band_tile) of the TW-row tiles of all ncol needed columns through its own S-stage shared-memory ring
// (LDGSTS 16-B copies, commit/wait groups, __syncwarp only — no CTA barrier), so the bytes
// in flight (~(S-1) stages per warp) live in shared memory instead of registers; the
// register-load kernel above was latency-bound (ncu: long_scoreboard, 16 warps/SM).
// Fragment reads use a column stride of TW+4 doubles (== 4 mod 16): conflict free.
// ======================================================================================
constexpr int PIPE_S = 3;

template <int MT, int NTN, bool SYM, int TW>
__global__ void __launch_bounds__(NT, 1) k_xty_pipe(XtyArgs a) {
    extern __shared__ __align__(16) double smp[];
    pdl_wait();
    pdl_trigger();
    constexpr int SP = TW + 4;
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w;
    const int colbase = SYM ? 0 : blockIdx.y * a.chunk;
    const int nxc = SYM ? w : min(a.chunk, a.jx - colbase);
    const int nx = (SYM || a.X == a.Y) ? 0 : nxc;                 // X columns streamed
    const int ncol = w + nx;
    const int64_t stage_d = int64_t(ncol) * SP;
    double* ring = smp + int64_t(wp) * PIPE_S * stage_d;
    const int64_t T = a.n / TW;                                    // full tiles
    const int64_t W = int64_t(gridDim.x) * nw;
    const int64_t g = int64_t(blockIdx.x) * nw + wp;
    const int64_t cnt = band_count(T, W, g);                      // tiles of this warp (band order)
    // columns: Y cols 0..w-1 at slot cols 0..w-1; X cols (if streamed) at w..w+nx-1
    const double* xbase = a.X == a.Y && !SYM ? a.Y + a.ldy * colbase : a.X + a.ldx * colbase;
    __shared__ const double* sCol[96];                             // column base pointers
    for (int c = threadIdx.x; c < ncol; c += blockDim.x) sCol[c] = c < w ? a.Y + a.ldy * c : xbase + a.ldx * (c - w);
    __syncthreads();
    auto colptr = [&](int c) -> const double* { return sCol[c]; };
    constexpr int CPC = TW * 8 / 16;                               // 16-B chunks per column
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
    // two accumulator sets, even / odd 4-row k-steps: twice the independent DMMA chains per warp
    // (ncu: the single set stalled on the DMMA dependency, "wait"); summed in a fixed order at the end
    double acc[MT][NTN][2], acc2[MT][NTN][2];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) acc[mt][nt][0] = acc[mt][nt][1] = acc2[mt][nt][0] = acc2[mt][nt][1] = 0.0;
    // slot column of each fragment lane (clamped: padded lanes feed discarded entries)
    int ycol[NTN], xcol[SYM ? 1 : MT];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt) ycol[nt] = min(8 * nt + gid, w - 1);
    if constexpr (!SYM) {
#pragma unroll
        for (int mt = 0; mt < MT; ++mt) xcol[mt] = (nx ? w : 0) + min(8 * mt + gid, nxc - 1);
    }
#pragma unroll
    for (int s = 0; s < PIPE_S - 1; ++s) issue(s, s);
    int stage = 0;
    for (int64_t i = 0; i < cnt; ++i) {
        issue(i + PIPE_S - 1, (stage + PIPE_S - 1) % PIPE_S);
        if (a.pf && TW == 32 && ncol <= 24 && i + PIPE_S - 1 + ptx::PF_DIST < cnt) {   // narrow panels only
            const int64_t rp = band_tile(T, W, g, i + PIPE_S - 1 + ptx::PF_DIST, a.rev) * TW;
            constexpr int LPC = TW / 16;
            for (int q = lane; q < ncol * LPC; q += 32) ptx::prefetch_l2(colptr(q / LPC) + rp + 16 * (q % LPC));
        }
        ptx::cp_async_wait<PIPE_S - 1>();
        __syncwarp();
        const double* sl = ring + stage * stage_d + tig;
        // per-tile fragment pointers: the unrolled k-steps below load [register + immediate]
        const double* sy[NTN];
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) sy[nt] = sl + ycol[nt] * SP;
        const double* sx[SYM ? 1 : MT];
        if constexpr (!SYM) {
#pragma unroll
            for (int mt = 0; mt < MT; ++mt) sx[mt] = sl + xcol[mt] * SP;
        }
#pragma unroll
        for (int u = 0; u < TW / 4; ++u) {
            double bn[NTN];
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt) bn[nt] = sy[nt][4 * u];
            constexpr bool SPLIT = MT * NTN <= 8;                    // (wider tiles: registers)
            auto& A = (SPLIT && (u & 1)) ? acc2 : acc;
            if constexpr (SYM) {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                    for (int nt = mt; nt < NTN; ++nt) ptx::dmma(A[mt][nt][0], A[mt][nt][1], bn[mt], bn[nt]);
            } else {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt) {
                    const double am = sx[mt][4 * u];
#pragma unroll
                    for (int nt = 0; nt < NTN; ++nt) ptx::dmma(A[mt][nt][0], A[mt][nt][1], am, bn[nt]);
                }
            }
        }
        __syncwarp();
        stage = (stage + 1) % PIPE_S;
    }
    ptx::cp_async_wait<0>();
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            acc[mt][nt][0] += acc2[mt][nt][0];
            acc[mt][nt][1] += acc2[mt][nt][1];
        }
    // ragged tail rows [T*TW, n): warp 0 of CTA 0, direct zero-padded loads
    if (blockIdx.x == 0 && wp == 0) {
        for (int64_t kr = T * TW; kr < a.n; kr += 4) {
            const int64_t row = kr + tig;
            const bool ok = row < a.n;
            double bn[NTN];
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt) bn[nt] = ok ? colptr(ycol[nt])[row] : 0.0;
            if constexpr (SYM) {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                    for (int nt = mt; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], bn[mt], bn[nt]);
            } else {
#pragma unroll
                for (int mt = 0; mt < MT; ++mt) {
                    const double am = ok ? (xbase + a.ldx * min(8 * mt + gid, nxc - 1))[row] : 0.0;
#pragma unroll
                    for (int nt = 0; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], am, bn[nt]);
                }
            }
        }
    }
    // ---- CTA reduction over warps (fixed order), reusing the ring ----
    __syncthreads();
    double* red = smp;
    constexpr int FR = MT * NTN * 64;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 0] = acc[mt][nt][0];
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 1] = acc[mt][nt][1];
        }
    __syncthreads();
    const int nent = a.chunk * w;
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * nent;
    for (int e = threadIdx.x; e < nent; e += blockDim.x) {
        const int il = e % a.chunk, c = e / a.chunk;
        int mt = il >> 3, nt = c >> 3, ml = il & 7, nl = c & 7;
        if (SYM && mt > nt) { const int tt = mt; mt = nt; nt = tt; const int q = ml; ml = nl; nl = q; }
        const int ln = ml * 4 + (nl >> 1), h = nl & 1;
        double sum = 0.0;
        if (mt < MT && nt < NTN)
            for (int q = 0; q < nw; ++q) sum += red[q * FR + (mt * NTN + nt) * 64 + ln * 2 + h];
        part[il + int64_t(a.chunk) * c] = sum;
    }
    __syncthreads();
    xty_finish(a, nent);
}

// ======================================================================================
// host side
// ======================================================================================
namespace {
struct Geo { int MT, NTN, U, chunk, gx, gy; bool sym; };

Geo geometry(const Dev& d, int64_t n, int jx, int w, bool same) {
    Geo o{};
    o.NTN = w <= 8 ? 1 : (w <= 16 ? 2 : 4);
    o.sym = same;
    if (same) {
        o.MT = o.NTN; o.chunk = 8 * o.MT; o.gy = 1;
    } else {
        const int mt = (jx + 7) / 8;
        o.MT = mt <= 1 ? 1 : (mt <= 2 ? 2 : (mt <= 4 ? 4 : 8));
        if (o.NTN == 4 && o.MT > 4) o.MT = 4;                       // register budget
        o.chunk = 8 * o.MT;
        o.gy = (jx + o.chunk - 1) / o.chunk;
    }
    const int per_ks = o.sym ? o.NTN : o.MT + o.NTN;               // loads per k-step per lane
    o.U = per_ks <= 1 ? 16 : (per_ks <= 2 ? 8 : (per_ks <= 6 ? 4 : (per_ks <= 9 ? 2 : 1)));
    const int64_t nss = (n + 4 * o.U - 1) / (4 * o.U);
    int64_t want = int64_t(d.sms) / o.gy;
    if (want < 1) want = 1;
    const int64_t cap = (nss + NWARP - 1) / NWARP;
    if (want > cap) want = cap;
    if (want < 1) want = 1;
    o.gx = int(want);
    return o;
}

template <typename K>
void launch(K kfn, const Geo& o, const XtyArgs& a, cudaStream_t st) {
    size_t smem = size_t(NWARP) * o.MT * o.NTN * 64 * sizeof(double);
    if (smem < NT * sizeof(double)) smem = NT * sizeof(double);
    if (smem > 48 * 1024) cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    kfn<<<dim3(o.gx, o.gy), NT, smem, st>>>(a);
}
}  // namespace

size_t xty_ws_doubles(const Dev& d, int jx, int w) {
    size_t m = 0;
    for (int same = 0; same < 2; ++same) {
        const Geo o = geometry(d, int64_t(1) << 40, same ? w : jx, w, same != 0);
        const size_t v = 2 * size_t(std::max(o.gx, d.sms / o.gy)) * o.gy * o.chunk * w;   // + group partials
        m = v > m ? v : m;
    }
    return m;
}

template <typename K>
void launch_pipe(K kfn, const Geo& o, int nw, size_t smem, const XtyArgs& a, cudaStream_t st) {
    cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    launch_pdl(kfn, dim3(o.gx, o.gy), dim3(32 * nw), smem, st, a);
}

template <int TW>
int xty_pipe_launch(const Dev& d, Geo o, const XtyArgs& a, int ncol, const XtyWs& ws, cudaStream_t st) {
    const size_t ring_w = size_t(PIPE_S) * ncol * (TW + 4) * sizeof(double);
    int nw = int((200 * 1024) / ring_w);
    nw = nw < 2 ? 2 : (nw > 16 ? 16 : nw);
    size_t smem = size_t(nw) * ring_w;
    const size_t red = size_t(nw) * o.MT * o.NTN * 64 * sizeof(double);
    if (smem < red) smem = red;
    if (smem < size_t(32 * nw) * sizeof(double)) smem = size_t(32 * nw) * sizeof(double);
    o.gx = std::max(1, d.sms / o.gy);
    if (size_t(o.gx) * o.gy * o.chunk * a.w * 2 > ws.cap) return -1;
    if (o.sym) {
        if (o.NTN == 1) launch_pipe(k_xty_pipe<1, 1, true, TW>, o, nw, smem, a, st);
        else if (o.NTN == 2) launch_pipe(k_xty_pipe<2, 2, true, TW>, o, nw, smem, a, st);
        else launch_pipe(k_xty_pipe<4, 4, true, TW>, o, nw, smem, a, st);
        return 0;
    }
    switch (o.MT * 10 + o.NTN) {
        case 11: launch_pipe(k_xty_pipe<1, 1, false, TW>, o, nw, smem, a, st); break;
        case 21: launch_pipe(k_xty_pipe<2, 1, false, TW>, o, nw, smem, a, st); break;
        case 41: launch_pipe(k_xty_pipe<4, 1, false, TW>, o, nw, smem, a, st); break;
        case 81: launch_pipe(k_xty_pipe<8, 1, false, TW>, o, nw, smem, a, st); break;
        case 12: launch_pipe(k_xty_pipe<1, 2, false, TW>, o, nw, smem, a, st); break;
        case 22: launch_pipe(k_xty_pipe<2, 2, false, TW>, o, nw, smem, a, st); break;
        case 42: launch_pipe(k_xty_pipe<4, 2, false, TW>, o, nw, smem, a, st); break;
        case 82: launch_pipe(k_xty_pipe<8, 2, false, TW>, o, nw, smem, a, st); break;
        case 14: launch_pipe(k_xty_pipe<1, 4, false, TW>, o, nw, smem, a, st); break;
        case 24: launch_pipe(k_xty_pipe<2, 4, false, TW>, o, nw, smem, a, st); break;
        default: launch_pipe(k_xty_pipe<4, 4, false, TW>, o, nw, smem, a, st); break;
    }
    return 0;
}

int xty(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, const double* Y,
        int64_t ldy, int w, double* out, bool fin_chol, double* R, int* status,
        const XtyWs& ws, cudaStream_t st) {
    if (jx <= 0 || w <= 0 || w > 32 || n < 0) return -1;
    const bool same = (X == Y) && (ldx == ldy) && (jx == w);
    if (same && d.gram >= 1 && size_t(d.sms) * w * w * 2 <= ws.cap) {
        GramArgs g{n, X, ldx, w, d.panel_pf, ws.part, out, ws.counter, fin_chol ? 1 : 0, R, status};
        if (gram_dfma(d, g, st) == 0) return 0;
    }
    Geo o = geometry(d, n, jx, w, same);
    if (size_t(o.gx) * o.gy * o.chunk * w * 2 > ws.cap || o.gy * TR_CNT > XTY_COUNTERS) return -1;
    XtyArgs a{n, X, ldx, jx, Y, ldy, w, o.chunk, ws.part, out, ws.counter, fin_chol ? 1 : 0, R, status, d.panel_pf, d.rev};
    const bool aligned = ((reinterpret_cast<uintptr_t>(X) | reinterpret_cast<uintptr_t>(Y)) % 16 == 0) &&
                         (ldx % 2 == 0) && (ldy % 2 == 0);
    if (aligned && n >= 32 * 64) {
        // per-warp cp.async pipeline: size the warps so the rings use ~200 KB of smem; very
        // wide panels (>= 36 streamed columns, < 6 warps at 32 rows) use 16-row tiles
        const int ncol = w + ((o.sym || X == Y) ? 0 : std::min(o.chunk, jx));
        if (d.panel_tw16 && ncol >= 36) return xty_pipe_launch<16>(d, o, a, ncol, ws, st);
        return xty_pipe_launch<32>(d, o, a, ncol, ws, st);
    }
    if (o.sym) {
        if (o.NTN == 1) launch(k_xty_mma<1, 1, 16, true>, o, a, st);
        else if (o.NTN == 2) launch(k_xty_mma<2, 2, 8, true>, o, a, st);
        else launch(k_xty_mma<4, 4, 4, true>, o, a, st);
        return 0;
    }
    switch (o.MT * 10 + o.NTN) {
        case 11: launch(k_xty_mma<1, 1, 8, false>, o, a, st); break;
        case 21: launch(k_xty_mma<2, 1, 4, false>, o, a, st); break;
        case 41: launch(k_xty_mma<4, 1, 4, false>, o, a, st); break;
        case 81: launch(k_xty_mma<8, 1, 2, false>, o, a, st); break;
        case 12: launch(k_xty_mma<1, 2, 4, false>, o, a, st); break;
        case 22: launch(k_xty_mma<2, 2, 4, false>, o, a, st); break;
        case 42: launch(k_xty_mma<4, 2, 4, false>, o, a, st); break;
        case 82: launch(k_xty_mma<8, 2, 1, false>, o, a, st); break;
        case 14: launch(k_xty_mma<1, 4, 4, false>, o, a, st); break;
        case 24: launch(k_xty_mma<2, 4, 4, false>, o, a, st); break;
        default: launch(k_xty_mma<4, 4, 2, false>, o, a, st); break;
    }
    return 0;
}

}  // namespace kern
