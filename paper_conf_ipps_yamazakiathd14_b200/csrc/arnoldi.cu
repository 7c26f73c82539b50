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
            if (jx > 0) a.v[r] = v;
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

int arnoldi_fused(const Dev& d, const ArnoldiArgs& a, int mode, cudaStream_t st) {
    if (a.jx < (mode == 2 ? 0 : 1) || a.jx > 32) return -1;   // wider: caller uses unfused passes
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

size_t arnoldi_ws_doubles(const Dev& d) { return 2 * size_t(d.sms) * 8 * 32; }

}  // namespace kern
