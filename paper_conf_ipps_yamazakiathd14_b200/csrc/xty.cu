// xty.cu — K4/K5: C = X^T Y for tall-skinny X (n x jx) and Y (n x w <= 32), FP64.
//   * BOrth pass 1: C = Q[:,0:j]^T P            ("MAGMA tall-skinny DGEMV")
//   * CholQR Gram:  B = V^T V, then R = chol(B)  ("batched DGEMM")
//
// Main path (k_xty_mma): a persistent CTA per SM streams full row tiles of every needed
// column into a 4-stage shared-memory ring with 1-D bulk async copies (TMA engine,
// cp.async.bulk + mbarrier complete_tx): ~100 KB per SM in flight without holding
// registers, so the panel is read from HBM exactly once at full rate.  The contraction over
// rows runs on the FP64 tensor core: each warp owns a slice of the tile's rows and issues
// mma.sync.m8n8k4.f64 (256 FMAs per warp instruction) for all 8x8 output tiles of its CTA's
// column chunk — with scalar DFMA the kernel was issue-bound at 8 warps/SM (ncu: 107 M
// instructions, 0.7 IPC); DMMA cuts the instruction count ~15x at the same FLOP rate.
// Column stride in shared memory is TS+4 doubles (== 4 mod 16) so the 8-column x 4-row
// fragment loads are bank-conflict free.  Gram (X == Y): A and B fragments coincide and
// only the upper block triangle is multiplied.
// At the end a fixed-order smem reduction over warps produces the CTA partial, and the LAST
// CTA (atomic ticket) sums all partials in a fixed order (run-to-run bitwise reproducible)
// and, for CholQR on one GPU, factors the Gram in the same launch.
// Fallback (k_xty_ldg): register loads, used when a user panel is not 16-B aligned.
#include <cstdint>

#include "dense_dev.cuh"
#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NWARP = NT / 32;
constexpr int XTY_STAGES = 4;
constexpr int XTY_STAGE_BYTES = 32 * 1024;
}

struct XtyArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;
    const double* Y; int64_t ldy; int w;
    int same;                   // X == Y (and jx == w): X columns come from the Y tile
    int G, chunk;               // fallback: groups per CTA; X columns per blockIdx.y chunk
    int TS;                     // rows per tile (TMA path)
    double* part;               // per-CTA partials (chunk x w each)
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
// TMA ring + DMMA kernel.  MT = 8-column tiles of X per chunk (chunk = 8*MT), NTN = 8-col
// tiles of Y.  SYM: X == Y, MT == NTN, upper block triangle only.
// ======================================================================================
template <int MT, int NTN, bool SYM>
__device__ __forceinline__ void xty_kstep(double (&acc)[MT][NTN][2], const double* Ys, int64_t ldY,
                                          const double* Xs, int64_t ldX, int64_t row, int lane, int w,
                                          int nxc, bool valid) {
    const int gid = lane >> 2;
    double bn[NTN];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt) {
        const int c = min(8 * nt + gid, w - 1);
        bn[nt] = valid ? Ys[row + ldY * c] : 0.0;
    }
    if constexpr (SYM) {
#pragma unroll
        for (int mt = 0; mt < MT; ++mt)
#pragma unroll
            for (int nt = mt; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], bn[mt], bn[nt]);
    } else {
#pragma unroll
        for (int mt = 0; mt < MT; ++mt) {
            const int c = min(8 * mt + gid, nxc - 1);
            const double am = valid ? Xs[row + ldX * c] : 0.0;
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt) ptx::dmma(acc[mt][nt][0], acc[mt][nt][1], am, bn[nt]);
        }
    }
}

template <int MT, int NTN, bool SYM>
__global__ void __launch_bounds__(NT, 1) k_xty_mma(XtyArgs a) {
    extern __shared__ __align__(128) unsigned char smraw[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smraw);
    double* slots = reinterpret_cast<double*>(smraw + 128);
    const int tid = threadIdx.x, lane = tid & 31, wp = tid >> 5;
    const int TS = a.TS, SP = TS + 4, w = a.w;
    const int colbase = blockIdx.y * a.chunk;
    const int nxc = SYM ? w : min(a.chunk, a.jx - colbase);          // X columns of this chunk
    const int nx = (SYM || a.same) ? 0 : nxc;                         // X columns loaded
    const int ncol = w + nx;
    const int64_t slot_d = int64_t(ncol) * SP;
    const int64_t ntiles = a.n / TS;
    const int64_t my_tiles = ntiles > int64_t(blockIdx.x) ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;

    double acc[MT][NTN][2];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) acc[mt][nt][0] = acc[mt][nt][1] = 0.0;

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
        for (int c = 0; c < w; ++c) ptx::bulk_g2s(dst + int64_t(c) * SP, a.Y + a.ldy * c + r0, colbytes, &bars[s]);
        for (int c = 0; c < nx; ++c)
            ptx::bulk_g2s(dst + int64_t(w + c) * SP, a.X + a.ldx * (colbase + c) + r0, colbytes, &bars[s]);
    };
    if (tid == 0)
        for (int64_t k = 0; k < my_tiles && k < XTY_STAGES; ++k) issue(k);
    const int rw = TS / NWARP;                                        // rows per warp per tile (mult. of 4)
    for (int64_t k = 0; k < my_tiles; ++k) {
        const int s = int(k % XTY_STAGES);
        ptx::mbar_wait(&bars[s], uint32_t((k / XTY_STAGES) & 1));
        const double* Ys = slots + s * slot_d;
        const double* Xs = a.same ? Ys + int64_t(SP) * colbase : Ys + int64_t(SP) * w;
#pragma unroll 2
        for (int kr = wp * rw; kr < (wp + 1) * rw; kr += 4)
            xty_kstep<MT, NTN, SYM>(acc, Ys, SP, Xs, SP, kr + (lane & 3), lane, w, nxc, true);
        __syncthreads();                               // every warp is done with slot s
        if (tid == 0 && k + XTY_STAGES < my_tiles) issue(k + XTY_STAGES);
    }
    // ragged tail [ntiles*TS, n): CTA x = 0, k-steps of 4 rows from global, zero padded
    if (blockIdx.x == 0 && ntiles * TS < a.n) {
        const int64_t r0 = ntiles * TS;
        const double* Xb = a.same ? a.Y + a.ldy * colbase : a.X + a.ldx * colbase;
        const int64_t ldX = a.same ? a.ldy : a.ldx;
        for (int64_t kr = r0 + 4 * wp; kr < a.n; kr += 4 * NWARP) {
            const int64_t row = kr + (lane & 3);
            xty_kstep<MT, NTN, SYM>(acc, a.Y, a.ldy, Xb, ldX, row, lane, w, nxc, row < a.n);
        }
    }
    // ---- CTA reduction over warps (fixed order) ----
    __syncthreads();
    double* red = slots;                                    // reuse the ring: NWARP x MT x NTN x 64
    constexpr int FR = MT * NTN * 64;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 0] = acc[mt][nt][0];
            red[wp * FR + (mt * NTN + nt) * 64 + lane * 2 + 1] = acc[mt][nt][1];
        }
    __syncthreads();
    const int nent = a.chunk * w;                           // entries of this CTA's partial
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * nent;
    for (int e = tid; e < a.chunk * w; e += NT) {
        const int il = e % a.chunk, c = e / a.chunk;
        int mt = il >> 3, nt = c >> 3, ml = il & 7, nl = c & 7;
        if (SYM && mt > nt) { const int t = mt; mt = nt; nt = t; const int u = ml; ml = nl; nl = u; }
        const int ln = ml * 4 + (nl >> 1), h = nl & 1;
        double sum = 0.0;
        if (mt < MT && nt < NTN)
            for (int q = 0; q < NWARP; ++q) sum += red[q * FR + (mt * NTN + nt) * 64 + ln * 2 + h];
        part[il + int64_t(a.chunk) * c] = sum;
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
struct Geo { int G, chunk, gx, gy, TS, MT, NTN; bool tma, sym; size_t smem; int JB, WM; };

int ceil8(int x) { return (x + 7) / 8; }

Geo geometry(const Dev& d, int64_t n, int jx, int w, bool same, bool aligned) {
    Geo o{};
    o.tma = aligned;
    if (o.tma) {
        o.NTN = w <= 8 ? 1 : (w <= 16 ? 2 : 4);
        o.sym = same;
        if (same) {
            o.MT = o.NTN; o.chunk = 8 * o.MT; o.gy = 1;
        } else {
            const int mt = ceil8(jx);
            o.MT = mt <= 1 ? 1 : (mt <= 2 ? 2 : (mt <= 4 ? 4 : 8));
            if (o.NTN == 4 && o.MT > 4) o.MT = 4;                    // register budget
            o.chunk = 8 * o.MT;
            o.gy = (jx + o.chunk - 1) / o.chunk;
        }
        const int ncol = w + ((same) ? 0 : std::min(o.chunk, jx));
        int TS = 4096;
        while (TS > 64 && int64_t(TS + 4) * ncol * 8 > XTY_STAGE_BYTES) TS /= 2;
        o.TS = TS;
        const size_t ring = size_t(XTY_STAGES) * size_t(ncol) * size_t(TS + 4) * sizeof(double);
        const size_t red = size_t(NWARP) * o.MT * o.NTN * 64 * sizeof(double);
        o.smem = 128 + (ring > red ? ring : red);
        const int64_t tiles = n / TS;
        int64_t want = int64_t(d.sms) / o.gy;
        if (want > tiles) want = tiles;
        if (want < 1) want = 1;
        o.gx = int(want);
    } else {
        if (w <= 1) { o.JB = 8; o.WM = 1; } else if (w <= 2) { o.JB = 8; o.WM = 2; }
        else if (w <= 4) { o.JB = 4; o.WM = 4; } else if (w <= 8) { o.JB = 4; o.WM = 8; }
        else if (w <= 12) { o.JB = 4; o.WM = 12; } else if (w <= 16) { o.JB = 4; o.WM = 16; }
        else { o.JB = 2; o.WM = 32; }
        const int need = (jx + o.JB - 1) / o.JB;
        int g = 1;
        while (g < need && g < 16) g *= 2;
        o.G = g; o.chunk = g * o.JB;
        o.gy = (jx + o.chunk - 1) / o.chunk;
        o.smem = size_t(o.WM) * 256 * sizeof(double);
        const int64_t tiles = (n + 255) / 256;
        int64_t want = int64_t(d.sms) * 2 / o.gy;
        if (want > tiles) want = tiles;
        if (want < 1) want = 1;
        o.gx = int(want);
    }
    return o;
}

template <typename K>
void launch(K kfn, const Geo& o, const XtyArgs& a, cudaStream_t st) {
    cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(o.smem));
    ++g_launches;
    kfn<<<dim3(o.gx, o.gy), NT, o.smem, st>>>(a);
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
    if (o.tma) {
        if (o.sym) {
            if (o.NTN == 1) launch(k_xty_mma<1, 1, true>, o, a, st);
            else if (o.NTN == 2) launch(k_xty_mma<2, 2, true>, o, a, st);
            else launch(k_xty_mma<4, 4, true>, o, a, st);
        } else {
            const int key = o.MT * 10 + o.NTN;
            switch (key) {
                case 11: launch(k_xty_mma<1, 1, false>, o, a, st); break;
                case 21: launch(k_xty_mma<2, 1, false>, o, a, st); break;
                case 41: launch(k_xty_mma<4, 1, false>, o, a, st); break;
                case 81: launch(k_xty_mma<8, 1, false>, o, a, st); break;
                case 12: launch(k_xty_mma<1, 2, false>, o, a, st); break;
                case 22: launch(k_xty_mma<2, 2, false>, o, a, st); break;
                case 42: launch(k_xty_mma<4, 2, false>, o, a, st); break;
                case 82: launch(k_xty_mma<8, 2, false>, o, a, st); break;
                case 14: launch(k_xty_mma<1, 4, false>, o, a, st); break;
                case 24: launch(k_xty_mma<2, 4, false>, o, a, st); break;
                default: launch(k_xty_mma<4, 4, false>, o, a, st); break;
            }
        }
    } else {
        switch (o.WM) {
            case 1: launch(k_xty_ldg<8, 1>, o, a, st); break;
            case 2: launch(k_xty_ldg<8, 2>, o, a, st); break;
            case 4: launch(k_xty_ldg<4, 4>, o, a, st); break;
            case 8: launch(k_xty_ldg<4, 8>, o, a, st); break;
            case 12: launch(k_xty_ldg<4, 12>, o, a, st); break;
            case 16: launch(k_xty_ldg<4, 16>, o, a, st); break;
            default: launch(k_xty_ldg<2, 32>, o, a, st); break;
        }
    }
    return 0;
}

}  // namespace kern
