// xty.cu — K4/K5: C = X^T Y for tall-skinny X (n x jx) and Y (n x w <= 32), FP64.
//   * BOrth pass 1: C = Q[:,0:j]^T P            ("MAGMA tall-skinny DGEMV")
//   * CholQR Gram:  B = V^T V, then R = chol(B)  ("batched DGEMM")
//
// Main path (k_xty_tma): a persistent CTA per SM streams full row tiles of every needed
// column into a 4-stage shared-memory ring with 1-D bulk async copies (the TMA engine,
// cp.async.bulk + mbarrier complete_tx), so ~100 KB per SM is in flight without holding
// registers — the tall-skinny panel is read from HBM exactly once.  Threads then compute
// from shared memory with per-thread register accumulators that persist over all tiles:
//   SYM  (Gram, w <= 12): every thread owns whole rows and accumulates the full upper
//        triangle w(w+1)/2 in registers (one smem load per operand, ~w/2 FMAs per load);
//   general: G groups x TR row-lanes; group g owns X columns g, g+G, .. (JB of them),
//        loads its rows' w Y-values once and feeds JB*w FMAs.
// At the end a fixed-order warp-butterfly + smem reduction produces the CTA partial, and
// the LAST CTA (atomic ticket) sums all partials in a fixed order (run-to-run bitwise
// reproducible) and, for CholQR on one GPU, factors the Gram in the same launch.
// Fallback (k_xty_ldg): register loads, used only when a user panel is not 16-B aligned.
#include <cstdint>

#include "dense_dev.cuh"
#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int XTY_STAGES = 4;
constexpr int XTY_STAGE_BYTES = 32 * 1024;
}

struct XtyArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;
    const double* Y; int64_t ldy; int w;
    int same;                   // X == Y (and jx == w): X columns come from the Y tile
    int G, chunk;               // groups per CTA, X columns per blockIdx.y chunk (= G*JB)
    int TS;                     // rows per tile (TMA path)
    double* part;               // per-CTA partials
    double* out;                // jx x w, ld jx
    unsigned int* counter;
    int fin_chol;
    double* R;
    int* status;
};

// ---- shared epilogue: CTA partial -> last-CTA fixed-order total (+ Cholesky) ---------
__device__ __forceinline__ void xty_finish(const XtyArgs& a, int nent_cta) {
    __shared__ bool s_last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned total = gridDim.x * gridDim.y;
        s_last = (atomicAdd(a.counter, 1u) == total - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    const int jx = a.jx, w = a.w;
    for (int e = threadIdx.x; e < jx * w; e += NT) {
        const int i = e % jx, c = e / jx;
        const int by = i / a.chunk, il = i - by * a.chunk;
        const double* src = a.part + int64_t(by) * gridDim.x * int64_t(nent_cta) + il + int64_t(a.chunk) * c;
        double s = 0.0;
        for (unsigned bx = 0; bx < gridDim.x; ++bx) s += __ldcg(src + int64_t(bx) * nent_cta);
        a.out[i + int64_t(jx) * c] = s;
    }
    if (threadIdx.x == 0) *a.counter = 0u;         // ready for the next launch (stream order)
    if (a.fin_chol) {
        __syncthreads();
        if (threadIdx.x == 0) chol_upper_serial(a.out, jx, w, a.R, a.status);
    }
}

// ======================================================================================
// TMA-pipelined kernel
// ======================================================================================
template <int JB, int WM, bool SYM>
__device__ __forceinline__ void xty_rows(const XtyArgs& a, double (&acc)[SYM ? WM * (WM + 1) / 2 : JB * WM],
                                         const double* Yb, int64_t ldY, const double* Xb, int64_t ldX,
                                         int rows, int g, int rl, int TR, const bool (&xok)[JB],
                                         const int (&xoff)[JB]) {
    const int w = a.w;
    if constexpr (SYM) {
        for (int r = threadIdx.x; r < rows; r += NT) {
            double p[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) p[c] = (c < w) ? Yb[r + ldY * c] : 0.0;
            int idx = 0;
#pragma unroll
            for (int i = 0; i < WM; ++i)
#pragma unroll
                for (int c = i; c < WM; ++c) { acc[idx] = fma(p[i], p[c], acc[idx]); ++idx; }
        }
    } else {
        for (int r = rl; r < rows; r += TR) {
            double p[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) p[c] = (c < w) ? Yb[r + ldY * c] : 0.0;
            double xv[JB];
#pragma unroll
            for (int jb = 0; jb < JB; ++jb) xv[jb] = xok[jb] ? Xb[r + ldX * xoff[jb]] : 0.0;
#pragma unroll
            for (int jb = 0; jb < JB; ++jb)
#pragma unroll
                for (int c = 0; c < WM; ++c) acc[jb * WM + c] = fma(xv[jb], p[c], acc[jb * WM + c]);
        }
    }
    (void)g;
}

template <int JB, int WM, bool SYM>
__global__ void __launch_bounds__(NT, 1) k_xty_tma(XtyArgs a) {
    constexpr int NACC = SYM ? WM * (WM + 1) / 2 : JB * WM;
    extern __shared__ __align__(128) unsigned char smraw[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smraw);
    double* slots = reinterpret_cast<double*>(smraw + 128);
    const int tid = threadIdx.x;
    const int TS = a.TS, w = a.w;
    const int G = SYM ? 1 : a.G, TR = NT / G;
    const int g = tid / TR, rl = tid - g * TR;
    const int colbase = blockIdx.y * a.chunk;
    const int nx = (SYM || a.same) ? 0 : min(a.chunk, a.jx - colbase);   // X columns loaded
    const int ncol = w + nx;
    const int64_t slot_d = int64_t(ncol) * TS;
    const int64_t ntiles = a.n / TS;
    const int64_t my_tiles = ntiles > int64_t(blockIdx.x) ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;

    bool xok[JB];
    int xoff[JB];
#pragma unroll
    for (int jb = 0; jb < JB; ++jb) {
        const int il = g + G * jb;
        xok[jb] = !SYM && (il < a.chunk) && (colbase + il < a.jx);
        xoff[jb] = a.same ? (colbase + il) : il;      // column inside the X source
    }
    double acc[NACC];
#pragma unroll
    for (int e = 0; e < NACC; ++e) acc[e] = 0.0;

    if (tid == 0) {
        for (int s = 0; s < XTY_STAGES; ++s) ptx::mbar_init(&bars[s], 1);
        ptx::fence_mbar_init();
    }
    __syncthreads();
    const uint32_t colbytes = uint32_t(TS) * 8u;
    auto issue = [&](int64_t k) {
        const int s = int(k % XTY_STAGES);
        const int64_t r0 = (int64_t(blockIdx.x) + k * gridDim.x) * TS;
        double* dst = slots + s * slot_d;
        ptx::fence_proxy_async();                      // generic reads of the slot precede the async writes
        ptx::mbar_arrive_expect_tx(&bars[s], colbytes * uint32_t(ncol));
        for (int c = 0; c < w; ++c) ptx::bulk_g2s(dst + int64_t(c) * TS, a.Y + a.ldy * c + r0, colbytes, &bars[s]);
        for (int c = 0; c < nx; ++c)
            ptx::bulk_g2s(dst + int64_t(w + c) * TS, a.X + a.ldx * (colbase + c) + r0, colbytes, &bars[s]);
    };
    if (tid == 0)
        for (int64_t k = 0; k < my_tiles && k < XTY_STAGES; ++k) issue(k);
    for (int64_t k = 0; k < my_tiles; ++k) {
        const int s = int(k % XTY_STAGES);
        ptx::mbar_wait(&bars[s], uint32_t((k / XTY_STAGES) & 1));
        const double* Ys = slots + s * slot_d;
        const double* Xs = a.same ? Ys : Ys + int64_t(w) * TS;
        xty_rows<JB, WM, SYM>(a, acc, Ys, TS, Xs, TS, TS, g, rl, TR, xok, xoff);
        __syncthreads();                               // every thread is done with slot s
        if (tid == 0 && k + XTY_STAGES < my_tiles) issue(k + XTY_STAGES);
    }
    // ragged tail [ntiles*TS, n): CTA x = 0 reads it straight from global memory
    if (blockIdx.x == 0 && ntiles * TS < a.n) {
        const int64_t r0 = ntiles * TS;
        const int rows = int(a.n - r0);
        const double* Xb = a.same ? a.Y + r0 : a.X + a.ldx * colbase + r0;
        xty_rows<JB, WM, SYM>(a, acc, a.Y + r0, a.ldy, Xb, a.same ? a.ldy : a.ldx, rows, g, rl, TR, xok, xoff);
    }
    // ---- CTA reduction (fixed order): butterfly over row-lanes, then smem over warps ----
    __syncthreads();
    double* red = slots;                                    // reuse the ring
    const int lanes = SYM ? 32 : min(TR, 32);               // lanes of one group in a warp
    const int warp = tid >> 5, lane = tid & 31;
#pragma unroll
    for (int e = 0; e < NACC; ++e) {
        double v = acc[e];
        for (int off = lanes >> 1; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
        acc[e] = v;
    }
    const int npg = SYM ? NT / 32 : max(1, TR / 32);        // partials per group
    if ((lane % lanes) == 0) {
        const int k = SYM ? warp : (rl / 32);
#pragma unroll
        for (int e = 0; e < NACC; ++e) red[(int64_t(g) * npg + k) * NACC + e] = acc[e];
    }
    __syncthreads();
    const int nent = a.chunk * w;                           // entries of this CTA's partial
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * nent;
    if constexpr (SYM) {
        for (int e = tid; e < w * w; e += NT) {
            const int i = e % w, c = e / w;
            const int lo = min(i, c), hi = max(i, c);
            const int idx = lo * WM - lo * (lo - 1) / 2 + (hi - lo);
            double s = 0.0;
            for (int k = 0; k < npg; ++k) s += red[int64_t(k) * NACC + idx];
            part[i + int64_t(a.chunk) * c] = s;
        }
    } else {
        for (int e = tid; e < a.chunk * w; e += NT) {
            const int il = e % a.chunk, c = e / a.chunk;
            const int g2 = il % G, jb = il / G;
            double s = 0.0;
            for (int k = 0; k < npg; ++k) s += red[(int64_t(g2) * npg + k) * NACC + jb * WM + c];
            part[il + int64_t(a.chunk) * c] = s;
        }
    }
    xty_finish(a, nent);
}

// ======================================================================================
// Fallback: register loads (unaligned panels)
// ======================================================================================
template <int JB, int WM>
__global__ void __launch_bounds__(NT, 1) k_xty_ldg(XtyArgs a) {
    constexpr int TSZ = 256;
    extern __shared__ double sm[];                  // WM x TSZ
    const int G = a.G, TR = NT / G;
    const int tid = threadIdx.x, g = tid / TR, rl = tid - g * TR;
    const int w = a.w;
    const int colbase = blockIdx.y * a.chunk;
    bool xok[JB];
    const double* xcol[JB];
#pragma unroll
    for (int jb = 0; jb < JB; ++jb) {
        const int il = g + G * jb, i = colbase + il;
        xok[jb] = (il < a.chunk) && (i < a.jx);
        xcol[jb] = a.X + (xok[jb] ? int64_t(i) * a.ldx : 0);
    }
    double acc[JB][WM];
#pragma unroll
    for (int jb = 0; jb < JB; ++jb)
#pragma unroll
        for (int c = 0; c < WM; ++c) acc[jb][c] = 0.0;
    const int64_t ntiles = (a.n + TSZ - 1) / TSZ;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int64_t r0 = t * TSZ;
        const int rows = int(min(int64_t(TSZ), a.n - r0));
        __syncthreads();
        for (int idx = tid; idx < w * TSZ; idx += NT) {
            const int c = idx / TSZ, r = idx - c * TSZ;
            sm[idx] = (r < rows) ? __ldg(a.Y + r0 + r + a.ldy * c) : 0.0;
        }
        __syncthreads();
        for (int r = rl; r < rows; r += TR) {
            double xv[JB];
#pragma unroll
            for (int jb = 0; jb < JB; ++jb) xv[jb] = xok[jb] ? __ldg(xcol[jb] + r0 + r) : 0.0;
            double p[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) p[c] = (c < w) ? sm[c * TSZ + r] : 0.0;
#pragma unroll
            for (int jb = 0; jb < JB; ++jb)
#pragma unroll
                for (int c = 0; c < WM; ++c) acc[jb][c] = fma(xv[jb], p[c], acc[jb][c]);
        }
    }
    const int nent = a.chunk * w;
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * nent;
#pragma unroll
    for (int jb = 0; jb < JB; ++jb) {
        __syncthreads();
#pragma unroll
        for (int c = 0; c < WM; ++c)
            if (c < w) sm[c * NT + tid] = acc[jb][c];
        __syncthreads();
        for (int e = tid; e < G * w; e += NT) {
            const int g2 = e % G, c = e / G;
            const int il = g2 + G * jb;
            if (il >= a.chunk) continue;
            double s = 0.0;
            const double* src = sm + c * NT + g2 * TR;
            for (int q = 0; q < TR; ++q) s += src[q];
            part[il + int64_t(a.chunk) * c] = s;
        }
    }
    xty_finish(a, nent);
}

// ======================================================================================
// host side
// ======================================================================================
namespace {
struct Cfg { int JB, WM; bool sym; };

Cfg cfg_for(int jx, int w, bool same) {
    if (same && w <= 12) {
        if (w <= 1) return {1, 1, true};
        if (w <= 2) return {1, 2, true};
        if (w <= 4) return {1, 4, true};
        if (w <= 8) return {1, 8, true};
        return {1, 12, true};
    }
    (void)jx;
    if (w <= 1) return {8, 1, false};
    if (w <= 2) return {8, 2, false};
    if (w <= 4) return {4, 4, false};
    if (w <= 8) return {4, 8, false};
    if (w <= 12) return {4, 12, false};
    if (w <= 16) return {4, 16, false};
    return {2, 32, false};
}

struct Geo { int G, chunk, gx, gy, TS; bool tma; Cfg cf; };

Geo geometry(const Dev& d, int64_t n, int jx, int w, bool same, bool aligned) {
    Geo o;
    o.cf = cfg_for(jx, w, same);
    if (o.cf.sym) {
        o.G = 1; o.chunk = w; o.gy = 1;
    } else {
        const int need = (jx + o.cf.JB - 1) / o.cf.JB;
        int g = 1;
        while (g < need && g < 16) g *= 2;
        o.G = g; o.chunk = g * o.cf.JB;
        if (same) o.chunk = o.chunk < w ? w : o.chunk;
        o.gy = same ? 1 : (jx + o.chunk - 1) / o.chunk;
    }
    o.tma = aligned;
    const int ncol = w + ((o.cf.sym || same) ? 0 : o.chunk);
    int TS = 4096;
    while (TS > 32 && TS * ncol * 8 > XTY_STAGE_BYTES) TS /= 2;
    o.TS = TS;
    const int64_t tiles = o.tma ? (n / TS) : (n + 255) / 256;
    int64_t want = o.tma ? int64_t(d.sms) / o.gy : int64_t(d.sms) * 2 / o.gy;
    if (want > tiles) want = tiles;
    if (want < 1) want = 1;
    o.gx = int(want);
    return o;
}

size_t smem_bytes(const Geo& o, int w) {
    if (!o.tma) return size_t(o.cf.WM) * 256 * sizeof(double);
    const int ncol = w + (o.cf.sym ? 0 : o.chunk);
    size_t ring = size_t(XTY_STAGES) * size_t(ncol) * size_t(o.TS) * sizeof(double);
    const int nacc = o.cf.sym ? o.cf.WM * (o.cf.WM + 1) / 2 : o.cf.JB * o.cf.WM;
    const size_t red = size_t(16) * size_t(nacc) * sizeof(double);   // G*npg <= 16 partial rows
    return 128 + (ring > red ? ring : red);
}

template <typename K>
void launch(K kfn, const Geo& o, size_t smem, const XtyArgs& a, cudaStream_t st) {
    cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    kfn<<<dim3(o.gx, o.gy), NT, smem, st>>>(a);
}
}  // namespace

size_t xty_ws_doubles(const Dev& d, int jx, int w) {
    size_t m = 0;
    for (int same = 0; same < 2; ++same)
        for (int al = 0; al < 2; ++al) {
            const Geo o = geometry(d, int64_t(1) << 40, same ? w : jx, w, same != 0, al != 0);
            const size_t v = size_t(o.gx) * o.gy * o.chunk * w;
            m = v > m ? v : m;
        }
    return m;
}

int xty(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, const double* Y,
        int64_t ldy, int w, double* out, bool fin_chol, double* R, int* status,
        const XtyWs& ws, cudaStream_t st) {
    if (jx <= 0 || w <= 0 || w > 32 || n < 0) return -1;
    const bool same = (X == Y) && (ldx == ldy) && (jx == w);
    const bool aligned = ((reinterpret_cast<uintptr_t>(X) | reinterpret_cast<uintptr_t>(Y)) % 16 == 0) &&
                         (ldx % 2 == 0) && (ldy % 2 == 0);
    const Geo o = geometry(d, n, jx, w, same, aligned);
    if (size_t(o.gx) * o.gy * o.chunk * w > ws.cap) return -1;
    XtyArgs a{n, X, ldx, jx, Y, ldy, w, same ? 1 : 0, o.G, o.chunk, o.TS, ws.part, out, ws.counter,
              fin_chol ? 1 : 0, R, status};
    const size_t smem = smem_bytes(o, w);
    const Cfg c = o.cf;
    if (o.tma) {
        if (c.sym) {
            switch (c.WM) {
                case 1: launch(k_xty_tma<1, 1, true>, o, smem, a, st); break;
                case 2: launch(k_xty_tma<1, 2, true>, o, smem, a, st); break;
                case 4: launch(k_xty_tma<1, 4, true>, o, smem, a, st); break;
                case 8: launch(k_xty_tma<1, 8, true>, o, smem, a, st); break;
                default: launch(k_xty_tma<1, 12, true>, o, smem, a, st); break;
            }
        } else {
            switch (c.WM) {
                case 1: launch(k_xty_tma<8, 1, false>, o, smem, a, st); break;
                case 2: launch(k_xty_tma<8, 2, false>, o, smem, a, st); break;
                case 4: launch(k_xty_tma<4, 4, false>, o, smem, a, st); break;
                case 8: launch(k_xty_tma<4, 8, false>, o, smem, a, st); break;
                case 12: launch(k_xty_tma<4, 12, false>, o, smem, a, st); break;
                case 16: launch(k_xty_tma<4, 16, false>, o, smem, a, st); break;
                default: launch(k_xty_tma<2, 32, false>, o, smem, a, st); break;
            }
        }
    } else {
        // fallback never uses the symmetric layout
        Geo g2 = o;
        if (c.sym) {
            g2 = geometry(d, n, jx, w, false, false);
            a.G = g2.G; a.chunk = g2.chunk;
            if (size_t(g2.gx) * g2.gy * g2.chunk * w > ws.cap) return -1;
        }
        const Cfg c2 = g2.cf;
        const size_t sm2 = smem_bytes(g2, w);
        switch (c2.WM) {
            case 1: launch(k_xty_ldg<8, 1>, g2, sm2, a, st); break;
            case 2: launch(k_xty_ldg<8, 2>, g2, sm2, a, st); break;
            case 4: launch(k_xty_ldg<4, 4>, g2, sm2, a, st); break;
            case 8: launch(k_xty_ldg<4, 8>, g2, sm2, a, st); break;
            case 12: launch(k_xty_ldg<4, 12>, g2, sm2, a, st); break;
            case 16: launch(k_xty_ldg<4, 16>, g2, sm2, a, st); break;
            default: launch(k_xty_ldg<2, 32>, g2, sm2, a, st); break;
        }
    }
    return 0;
}

}  // namespace kern
