// arnoldi.cu — fused passes of the first (shift-finding) cycle, GMRES(m) with CGS2
// Arnoldi ("we use the standard GMRES iterations"; reading G12).
// One Arnoldi step on Q = V[:, 0:jx] and the new vector v = A q_k is
//     c1 = Q^T v ; v -= Q c1 ; c2 = Q^T v ; v -= Q c2 ; h = ||v|| ; v /= h.
// Unfused that is four passes over Q.  Here the middle two pairs are fused:
//     MODE 1:  v -= Q c_in, and in the same pass  c_out = Q^T v   (new v)
//     MODE 2:  v -= Q c_in, and in the same pass  nrm   = v^T v   (new v; jx = 0: plain norm)
//     MODE 0:  c_out = Q^T v (the first CGS pass; no update)
// so Q is read three times per step (k_xty_mma for c1, then these two).  One thread per
// row: the Q row (jx <= 32 values) is held in registers between the update and the
// reduction; c_in is a warp-broadcast from shared memory.  Partials are reduced in a fixed
// order (warp butterfly -> smem -> last CTA), so results are run-to-run reproducible.
#include <cstdint>

#include "kernels.h"
#include "ptx.h"
#include "reduce.cuh"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NWARP = NT / 32;
}

template <int JX, int MODE>
__global__ void __launch_bounds__(NT) k_arnoldi_fused(ArnoldiArgs a) {
    __shared__ double sc[JX];
    __shared__ double sred[NWARP][JX];
    const int jx = a.jx;
    for (int i = threadIdx.x; i < JX; i += NT) sc[i] = (MODE != 0 && i < jx) ? a.c_in[i] : 0.0;
    __syncthreads();
    constexpr int NA = MODE == 2 ? 1 : JX;
    double acc[NA];
#pragma unroll
    for (int i = 0; i < NA; ++i) acc[i] = 0.0;
    for (int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x; r < a.n; r += int64_t(gridDim.x) * NT) {
        double q[JX];
#pragma unroll
        for (int i = 0; i < JX; ++i) q[i] = i < jx ? __ldg(a.Q + r + a.ldq * i) : 0.0;
        double v = a.v[r];
        if constexpr (MODE != 0) {
#pragma unroll
            for (int i = 0; i < JX; ++i) v = fma(-q[i], sc[i], v);
            if (jx > 0) (a.vout ? a.vout : a.v)[r] = v;
        }
        if constexpr (MODE != 2) {
#pragma unroll
            for (int i = 0; i < JX; ++i) acc[i] = fma(q[i], v, acc[i]);
        } else {
            acc[0] = fma(v, v, acc[0]);
        }
    }
    // fixed-order CTA reduction
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
#pragma unroll
    for (int i = 0; i < NA; ++i) {
        double x = acc[i];
        for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(0xffffffffu, x, off);
        if (lane == 0) sred[wp][i] = x;
    }
    __syncthreads();
    double* part = a.part + int64_t(blockIdx.x) * NA;
    for (int i = threadIdx.x; i < NA; i += NT) {
        double s = 0.0;
        for (int q = 0; q < NWARP; ++q) s += sred[q][i];
        part[i] = s;
    }
    const int nout = MODE == 2 ? 1 : jx;
    tree_reduce(a.part, a.part + int64_t(gridDim.x) * NA, int(gridDim.x), int(blockIdx.x), NA, nout, a.counter,
                [&](int i, double s) {
                    if (MODE == 2 && a.sqrt_out) {
                        if (!(s > 0.0)) atomicOr(a.status, ST_NORM);
                        s = sqrt(s);
                    }
                    a.c_out[i] = s;
                });
}

// Ring version (aligned columns, n >= 64 tiles): the register-load kernel above keeps one row's
// jx loads in flight per thread with <= 16 warps per SM and no prefetch across rows (ncu:
// 2.2-3.6 TB/s at jx ~ 24).  Here each warp streams its band-order share (kern::band_tile) of the 32-row tiles
// of [Q | v] through an AR_S-stage shared-memory ring with 16-B cp.async (no registers held),
// lane l owns row l of a tile and reads its Q row from the ring (column c at c*32 + l:
// conflict-free).  Same per-row operations as k_arnoldi_fused; partials reduced in a fixed order.
constexpr int AR_S = 3;
template <int JX, int MODE>
__global__ void __launch_bounds__(512, 1) k_arnoldi_ring(ArnoldiArgs a) {
    extern __shared__ __align__(16) double sma[];
    __shared__ double sc[JX > 0 ? JX : 1];
    __shared__ double sred[16][JX > 0 ? JX : 1];
    pdl_wait();
    pdl_trigger();
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int jx = a.jx;
    for (int i = threadIdx.x; i < JX; i += blockDim.x) sc[i] = (MODE != 0 && i < jx) ? a.c_in[i] : 0.0;
    __syncthreads();
    constexpr int NA = (MODE == 2 || MODE == 3) ? 1 : JX;      // MODE 3: update only (x += V y)
    double acc[NA];
#pragma unroll
    for (int i = 0; i < NA; ++i) acc[i] = 0.0;
    const int ncol = jx + 1;                                   // Q columns, then v
    const int64_t stage_d = int64_t(ncol) * 32;
    double* ring = sma + int64_t(wp) * AR_S * stage_d;
    const int64_t T = a.n / 32;
    const int64_t Wn = int64_t(gridDim.x) * nw;
    const int64_t g = int64_t(blockIdx.x) * nw + wp;
    const int64_t cnt = band_count(T, Wn, g);                     // tiles of this warp (band order)
    const int part2 = 2 * (lane & 15), cfirst = lane >> 4;
    const int64_t cstride = 2 * a.ldq;
    auto issue = [&](int64_t i, int stage) {
        if (i < cnt) {
            double* dst = ring + stage * stage_d + cfirst * 32 + part2;
            const int64_t r0 = band_tile(T, Wn, g, i, a.rev) * 32 + part2;
            const double* src = a.Q + a.ldq * cfirst + r0;
            int c = cfirst;
#pragma unroll 4
            for (; c < jx; c += 2, dst += 64, src += cstride) ptx::cp_async16(dst, src);
            if (c == jx) ptx::cp_async16(dst, a.v + r0);             // v is slot column jx
        }
        ptx::cp_async_commit();
    };
    auto row = [&](const double* sq, double vv, int64_t r) {
        if constexpr (MODE != 0) {
#pragma unroll
            for (int i = 0; i < JX; ++i)
                if (i < jx) vv = fma(-sq[i * 32], sc[i], vv);
            if (jx > 0) (a.vout ? a.vout : a.v)[r] = vv;
        }
        if constexpr (MODE == 0 || MODE == 1) {
#pragma unroll
            for (int i = 0; i < JX; ++i)
                if (i < jx) acc[i] = fma(sq[i * 32], vv, acc[i]);
        } else if constexpr (MODE == 2) {
            acc[0] = fma(vv, vv, acc[0]);
        }
    };
#pragma unroll
    for (int s = 0; s < AR_S - 1; ++s) issue(s, s);
    int stage = 0;
    for (int64_t i = 0; i < cnt; ++i) {
        issue(i + AR_S - 1, (stage + AR_S - 1) % AR_S);
        if (a.pf && i + AR_S - 1 + ptx::PF_DIST < cnt) {
            const int64_t rp = band_tile(T, Wn, g, i + AR_S - 1 + ptx::PF_DIST, a.rev) * 32;
            for (int q = lane; q < ncol * 2; q += 32)
                ptx::prefetch_l2((q >> 1 < jx ? a.Q + a.ldq * (q >> 1) : a.v) + rp + 16 * (q & 1));
        }
        ptx::cp_async_wait<AR_S - 1>();
        __syncwarp();
        const double* sl = ring + stage * stage_d + lane;
        row(sl, sl[jx * 32], band_tile(T, Wn, g, i, a.rev) * 32 + lane);
        __syncwarp();
        stage = (stage + 1) % AR_S;
    }
    ptx::cp_async_wait<0>();
    if (blockIdx.x == 0 && wp == 0) {                          // ragged tail rows [32 T, n)
        const int64_t r = T * 32 + lane;
        if (r < a.n) {
            double* sl = ring + lane;                          // ring idle: stage this lane's row
            for (int c = 0; c < jx; ++c) sl[c * 32] = a.Q[a.ldq * c + r];
            row(sl, a.v[r], r);
        }
    }
    if constexpr (MODE == 3) return;                           // no reduction
#pragma unroll
    for (int i = 0; i < NA; ++i) {
        double x = acc[i];
        for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(0xffffffffu, x, off);
        if (lane == 0) sred[wp][i] = x;
    }
    __syncthreads();
    double* part = a.part + int64_t(blockIdx.x) * NA;
    for (int i = threadIdx.x; i < NA; i += blockDim.x) {
        double s = 0.0;
        for (int q = 0; q < nw; ++q) s += sred[q][i];
        part[i] = s;
    }
    const int nout = MODE == 2 ? 1 : jx;
    tree_reduce(a.part, a.part + int64_t(gridDim.x) * NA, int(gridDim.x), int(blockIdx.x), NA, nout, a.counter,
                [&](int i, double s) {
                    if (MODE == 2 && a.sqrt_out) {
                        if (!(s > 0.0)) atomicOr(a.status, ST_NORM);
                        s = sqrt(s);
                    }
                    a.c_out[i] = s;
                });
}

namespace {
template <int JX, int MODE>
bool go_ring(const Dev& d, const ArnoldiArgs& a0, cudaStream_t st) {
    ArnoldiArgs a = a0;
    a.rev = d.rev;
    const bool aligned = ((reinterpret_cast<uintptr_t>(a.v) | reinterpret_cast<uintptr_t>(a.Q)) % 16 == 0) &&
                         (a.ldq % 2 == 0 || a.jx == 0);
    if (!aligned || a.n < 64 * 32) return false;
    const size_t ring_w = size_t(AR_S) * size_t(a.jx + 1) * 32 * sizeof(double);
    int nw = int((200 * 1024) / ring_w);
    nw = nw < 2 ? 2 : (nw > 16 ? 16 : nw);
    const size_t smem = size_t(nw) * ring_w;
    cudaFuncSetAttribute(k_arnoldi_ring<JX, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    launch_pdl(k_arnoldi_ring<JX, MODE>, dim3(unsigned(d.sms)), dim3(32 * nw), smem, st, a);
    return true;
}
}  // namespace

// JX buckets of 8: the per-row loops are unrolled to JX with predicates i < jx
template <int MODE>
bool ring_dispatch(const Dev& d, const ArnoldiArgs& a, cudaStream_t st) {
    if (a.jx <= 8) return go_ring<8, MODE>(d, a, st);
    if (a.jx <= 16) return go_ring<16, MODE>(d, a, st);
    if (a.jx <= 24) return go_ring<24, MODE>(d, a, st);
    return go_ring<32, MODE>(d, a, st);
}

// p -= X c for a single column p (x += V y at the end of a cycle): the ring kernel's
// update-only mode, one lane per row (a DMMA tile would waste 7/8 of its columns).
int update_w1(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* p, const double* c,
              cudaStream_t st) {
    if (!d.arnoldi_ring || jx < 1 || jx > 32) return -1;
    ArnoldiArgs a{d.panel_pf, n, X, ldx, jx, p, c, nullptr, nullptr, nullptr, nullptr, 0, nullptr};
    const bool ok = ring_dispatch<3>(d, a, st);
    return ok ? 0 : -1;
}

int arnoldi_fused(const Dev& d, const ArnoldiArgs& a, int mode, cudaStream_t st) {
    if (a.jx < (mode == 2 ? 0 : 1) || a.jx > 32) return -1;   // wider: caller uses unfused passes
    if (d.arnoldi_ring) {
        bool ok;
        if (mode == 0) ok = ring_dispatch<0>(d, a, st);
        else if (mode == 1) ok = ring_dispatch<1>(d, a, st);
        else ok = ring_dispatch<2>(d, a, st);
        if (ok) return 0;
    }
    const int64_t blocks = (a.n + NT - 1) / NT;
    auto go = [&](auto kfn) {
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kfn, NT, 0);
        int64_t g = int64_t(d.sms) * (occ < 1 ? 1 : (occ > 2 ? 2 : occ));   // <= 2 CTAs/SM: few partials
        if (g > blocks) g = blocks;
        if (g < 1) g = 1;
        ++g_launches;
        kfn<<<unsigned(g), NT, 0, st>>>(a);
    };
    if (mode == 0) {
        if (a.jx <= 8) go(k_arnoldi_fused<8, 0>);
        else if (a.jx <= 16) go(k_arnoldi_fused<16, 0>);
        else go(k_arnoldi_fused<32, 0>);
    } else if (mode == 1) {
        if (a.jx <= 8) go(k_arnoldi_fused<8, 1>);
        else if (a.jx <= 16) go(k_arnoldi_fused<16, 1>);
        else go(k_arnoldi_fused<32, 1>);
    } else {
        if (a.jx <= 8) go(k_arnoldi_fused<8, 2>);
        else if (a.jx <= 16) go(k_arnoldi_fused<16, 2>);
        else go(k_arnoldi_fused<32, 2>);
    }
    return 0;
}

size_t arnoldi_ws_doubles(const Dev& d) { return 2 * size_t(d.sms) * 8 * 32; }   // >= 2 * sms * 32 (ring)

}  // namespace kern
