// kernels.cu — hand-written FP64 kernels for sm_100a (B200) of one CA-GMRES restart cycle.
//
//   spmv_sell32   MPK SpMV step with the Newton shift fused (Fig. 4)      [K1]
//   xty           tall-skinny X^T Y with a deterministic in-kernel final reduction:
//                 BOrth pass 1 C = Q^T P and the CholQR Gram B = V^T V,
//                 optionally followed by R = chol(B) in the same launch       [K4/K5]
//   update        P -= Q C (BOrth pass 2)                                      [K9]
//   trsm          V := V R^{-1}, row-wise triangular solve (P:166, P:275 fn 7)         [K8]
//   svqr_factor   SVQR small factor                                    [K15]
//   gather/scatter halo pack/unpack (Fig. 4 "compress"/"expand")                 [K2]
//
// Everything here is HBM-bandwidth bound in FP64, so the design
// rules are coalescing, enough bytes in flight per SM, one pass over each operand and grids
// sized from the SM count — not tensor cores.
#include <cfloat>
#include <cstdio>

#include "kernels.h"

namespace kern {

constexpr int NT = 256;
long long g_launches = 0;

// ------------------------------------------------------------------------------------
// K1: y = A x + bu*u + bw*w on the first nrows rows of a SELL-32 matrix.
// One thread per row; a warp covers one 32-row slice whose entries are stored column-major
// (entry t of row lane at sptr[slice] + 32 t + lane) so val/col loads are fully coalesced.
// Padding entries have val = 0 and col = the row itself (always a valid, in-range x).
// Per-row summation runs over the stored (= global column) order, so a row's result does
// not depend on the partition.
// ------------------------------------------------------------------------------------
template <int MODE>   // 0: Ax   1: Ax + bu u   2: Ax + bu u + bw w   3: u - Ax
__global__ void __launch_bounds__(NT) k_spmv_sell32(int64_t nrows, const int64_t* __restrict__ sptr,
                                                    const int32_t* __restrict__ col,
                                                    const double* __restrict__ val,
                                                    const double* __restrict__ x,
                                                    const double* __restrict__ u, double bu,
                                                    const double* __restrict__ w, double bw,
                                                    double* __restrict__ y) {
    const int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x;
    if (r >= nrows) return;
    const int64_t sl = r >> 5;
    const int lane = int(r & 31);
    int64_t o = __ldg(sptr + sl) + lane;
    const int64_t e = __ldg(sptr + sl + 1);
    double acc = 0.0;
#pragma unroll 4
    for (; o < e; o += 32) acc = fma(__ldg(val + o), __ldg(x + __ldg(col + o)), acc);
    double out;
    if constexpr (MODE == 3) {
        out = __ldg(u + r) - acc;
    } else {
        out = acc;
        if constexpr (MODE >= 1) out = fma(bu, __ldg(u + r), out);
        if constexpr (MODE >= 2) out = fma(bw, __ldg(w + r), out);
    }
    y[r] = out;
}

void spmv(const Dev& d, const Sell& A, int64_t nrows, const double* x, double* y,
          const double* u, double bu, const double* w, double bw, cudaStream_t st) {
    (void)d;
    if (nrows <= 0) return;
    const unsigned grid = unsigned((nrows + NT - 1) / NT);
    ++g_launches;
    if (w)
        k_spmv_sell32<2><<<grid, NT, 0, st>>>(nrows, A.sptr, A.col, A.val, x, u, bu, w, bw, y);
    else if (u)
        k_spmv_sell32<1><<<grid, NT, 0, st>>>(nrows, A.sptr, A.col, A.val, x, u, bu, nullptr, 0.0, y);
    else
        k_spmv_sell32<0><<<grid, NT, 0, st>>>(nrows, A.sptr, A.col, A.val, x, nullptr, 0.0, nullptr, 0.0, y);
}

void residual(const Dev& d, const Sell& A, int64_t nrows, const double* x, const double* b,
              double* r, cudaStream_t st) {
    (void)d;
    if (nrows <= 0) return;
    const unsigned grid = unsigned((nrows + NT - 1) / NT);
    ++g_launches; k_spmv_sell32<3><<<grid, NT, 0, st>>>(nrows, A.sptr, A.col, A.val, x, b, 1.0, nullptr, 0.0, r);
}

// ------------------------------------------------------------------------------------
// Small dense factorizations on one thread / one CTA (w <= 32).
// ------------------------------------------------------------------------------------
__device__ void chol_upper_serial(const double* G, int ldg, int w, double* R, int* status) {
    // R^T R = G (upper R, positive diagonal), row-oriented: R[k,c] for c >= k.
    bool bad = false;
    for (int k = 0; k < w; ++k) {
        double dkk = G[k + ldg * k];
        for (int i = 0; i < k; ++i) dkk = fma(-R[i + w * k], R[i + w * k], dkk);
        if (!(dkk > 0.0)) { bad = true; dkk = DBL_MIN; }
        const double rkk = sqrt(dkk);
        const double inv = 1.0 / rkk;
        R[k + w * k] = rkk;
        for (int c = k + 1; c < w; ++c) {
            double v = G[k + ldg * c];
            for (int i = 0; i < k; ++i) v = fma(-R[i + w * k], R[i + w * c], v);
            R[k + w * c] = v * inv;
        }
        for (int c = 0; c < k; ++c) R[k + w * c] = 0.0;
    }
    if (bad) atomicOr(status, ST_CHOL);
}

__global__ void k_chol(const double* G, int w, double* R, int* status) {
    if (threadIdx.x == 0) chol_upper_serial(G, w, w, R, status);
}

void chol(const double* G, int w, double* R, int* status, cudaStream_t st) {
    ++g_launches; k_chol<<<1, 32, 0, st>>>(G, w, R, status);
}

// SVQR (reading G14): D = diag(G)^{-1/2}; D G D = U S U^T (cyclic
// Jacobi); s_i <- max(s_i, eps s_max); R_hat = R of qr(S^{1/2} U^T) (Householder, positive
// diagonal); R = R_hat D^{-1}.  One thread, w <= 32 (a comparator-sized cost).
__global__ void k_svqr(const double* G, int w, double* R, int* status) {
    __shared__ double A[32 * 32], V[32 * 32], d[32];
    if (threadIdx.x != 0) return;
    for (int i = 0; i < w; ++i) {
        const double g = G[i + w * i];
        if (!(g > 0.0)) { atomicOr(status, ST_SVQR); d[i] = 1.0; } else d[i] = 1.0 / sqrt(g);
    }
    for (int j = 0; j < w; ++j)
        for (int i = 0; i < w; ++i) {
            const double g = (i <= j) ? G[i + w * j] : G[j + w * i];
            A[i + 32 * j] = d[i] * g * d[j];
            V[i + 32 * j] = (i == j) ? 1.0 : 0.0;
        }
    for (int sweep = 0; sweep < 60; ++sweep) {
        double off = 0.0, dia = 0.0;
        for (int j = 0; j < w; ++j) {
            dia += A[j + 32 * j] * A[j + 32 * j];
            for (int i = 0; i < j; ++i) off += A[i + 32 * j] * A[i + 32 * j];
        }
        if (off <= DBL_EPSILON * DBL_EPSILON * dia * 1e-2) break;
        for (int p = 0; p < w - 1; ++p)
            for (int q = p + 1; q < w; ++q) {
                const double apq = A[p + 32 * q];
                if (apq == 0.0) continue;
                const double tau = (A[q + 32 * q] - A[p + 32 * p]) / (2.0 * apq);
                const double t = (tau >= 0.0 ? 1.0 : -1.0) / (fabs(tau) + sqrt(1.0 + tau * tau));
                const double c = 1.0 / sqrt(1.0 + t * t), s = t * c;
                for (int k = 0; k < w; ++k) {
                    const double akp = A[k + 32 * p], akq = A[k + 32 * q];
                    A[k + 32 * p] = c * akp - s * akq;
                    A[k + 32 * q] = s * akp + c * akq;
                }
                for (int k = 0; k < w; ++k) {
                    const double apk = A[p + 32 * k], aqk = A[q + 32 * k];
                    A[p + 32 * k] = c * apk - s * aqk;
                    A[q + 32 * k] = s * apk + c * aqk;
                }
                for (int k = 0; k < w; ++k) {
                    const double vkp = V[k + 32 * p], vkq = V[k + 32 * q];
                    V[k + 32 * p] = c * vkp - s * vkq;
                    V[k + 32 * q] = s * vkp + c * vkq;
                }
            }
    }
    double smax = 0.0;
    for (int i = 0; i < w; ++i) smax = fmax(smax, A[i + 32 * i]);
    // M = S^{1/2} U^T  (stored in A)
    double sq[32];
    for (int i = 0; i < w; ++i) sq[i] = sqrt(fmax(A[i + 32 * i], DBL_EPSILON * smax));
    for (int i = 0; i < w; ++i)
        for (int k = 0; k < w; ++k) A[i + 32 * k] = sq[i] * V[k + 32 * i];
    // Householder QR of M (w x w), R_hat in the upper triangle of A
    for (int k = 0; k < w; ++k) {
        double nrm = 0.0;
        for (int i = k; i < w; ++i) nrm += A[i + 32 * k] * A[i + 32 * k];
        nrm = sqrt(nrm);
        if (nrm == 0.0) continue;
        const double alpha = -copysign(nrm, A[k + 32 * k]);
        double v[32];
        for (int i = k; i < w; ++i) v[i] = A[i + 32 * k];
        v[k] -= alpha;
        double vv = 0.0;
        for (int i = k; i < w; ++i) vv += v[i] * v[i];
        if (vv == 0.0) continue;
        const double beta = 2.0 / vv;
        for (int c = k; c < w; ++c) {
            double dd = 0.0;
            for (int i = k; i < w; ++i) dd += v[i] * A[i + 32 * c];
            dd *= beta;
            for (int i = k; i < w; ++i) A[i + 32 * c] -= dd * v[i];
        }
    }
    for (int i = 0; i < w; ++i) {
        const double sg = A[i + 32 * i] < 0.0 ? -1.0 : 1.0;
        for (int c = 0; c < w; ++c) R[i + w * c] = (c < i) ? 0.0 : sg * A[i + 32 * c] / d[c];
    }
}

void svqr_factor(const double* G, int w, double* R, int* status, cudaStream_t st) {
    ++g_launches; k_svqr<<<1, 32, 0, st>>>(G, w, R, status);
}

// ------------------------------------------------------------------------------------
// K4/K5: C = X^T Y for tall-skinny X (n x jx) and Y (n x w).
// A CTA walks 256-row tiles (grid-stride).  The Y tile is staged in shared memory (it is
// needed by every column group); X is read straight from global memory into registers,
// each element feeding w FMAs.  Threads form G groups of TR = 256/G row-lanes: group g
// owns X columns g, g+G, ..., (JB of them) of this blockIdx.y chunk, lane rl owns rows
// rl, rl+TR, ... of the tile.  Per-thread accumulators acc[JB][WM] persist over all tiles;
// at the end they are reduced over the TR lanes of each group in a fixed order, the CTA's
// partial is stored, and the LAST CTA to finish (atomic ticket) sums all partials in a
// fixed order (deterministic, run-to-run bitwise reproducible) and optionally factors the
// Gram matrix (fin_chol) — one launch per Gram + Cholesky.
// ------------------------------------------------------------------------------------
struct XtyArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;
    const double* Y; int64_t ldy; int w;
    int G, chunk;               // groups per CTA, X columns per blockIdx.y chunk (= G*JB)
    double* part;
    double* out;                // jx x w, ld jx
    unsigned int* counter;
    int fin_chol;
    double* R;
    int* status;
};

constexpr int XTY_TS = 256;

template <int JB, int WM>
__global__ void __launch_bounds__(NT, 1) k_xty(XtyArgs a) {
    extern __shared__ double sm[];                 // WM x XTY_TS, column-major
    __shared__ bool s_last;
    const int G = a.G, TR = NT / G;
    const int tid = threadIdx.x, g = tid / TR, rl = tid - g * TR;
    const int w = a.w;
    const int colbase = blockIdx.y * a.chunk;
    const double* xcol[JB];
    bool xok[JB];
#pragma unroll
    for (int jb = 0; jb < JB; ++jb) {
        const int il = g + G * jb;
        const int i = colbase + il;
        xok[jb] = (il < a.chunk) && (i < a.jx);
        xcol[jb] = a.X + (xok[jb] ? int64_t(i) * a.ldx : 0);
    }
    double acc[JB][WM];
#pragma unroll
    for (int jb = 0; jb < JB; ++jb)
#pragma unroll
        for (int c = 0; c < WM; ++c) acc[jb][c] = 0.0;

    const int64_t ntiles = (a.n + XTY_TS - 1) / XTY_TS;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int64_t r0 = t * XTY_TS;
        const int rows = int(min(int64_t(XTY_TS), a.n - r0));
        __syncthreads();
        for (int idx = tid; idx < w * XTY_TS; idx += NT) {
            const int c = idx / XTY_TS, r = idx - c * XTY_TS;
            sm[idx] = (r < rows) ? __ldg(a.Y + r0 + r + a.ldy * c) : 0.0;
        }
        __syncthreads();
#pragma unroll 2
        for (int r = rl; r < rows; r += TR) {
            double xv[JB];
#pragma unroll
            for (int jb = 0; jb < JB; ++jb) xv[jb] = xok[jb] ? __ldg(xcol[jb] + r0 + r) : 0.0;
            double p[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) p[c] = (c < w) ? sm[c * XTY_TS + r] : 0.0;
#pragma unroll
            for (int jb = 0; jb < JB; ++jb)
#pragma unroll
                for (int c = 0; c < WM; ++c) acc[jb][c] = fma(xv[jb], p[c], acc[jb][c]);
        }
    }
    // ---- CTA reduction over the TR row-lanes of each group (fixed order) ----
    double* part = a.part + (int64_t(blockIdx.y) * gridDim.x + blockIdx.x) * int64_t(a.chunk) * w;
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
    // ---- last CTA: deterministic sum of all partials (+ optional Cholesky) ----
    __threadfence();
    __syncthreads();
    if (tid == 0) {
        const unsigned total = gridDim.x * gridDim.y;
        s_last = (atomicAdd(a.counter, 1u) == total - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    const int jx = a.jx;
    for (int e = tid; e < jx * w; e += NT) {
        const int i = e % jx, c = e / jx;
        const int by = i / a.chunk, il = i - by * a.chunk;
        const double* src = a.part + int64_t(by) * gridDim.x * int64_t(a.chunk) * w + il + int64_t(a.chunk) * c;
        double s = 0.0;
        for (unsigned bx = 0; bx < gridDim.x; ++bx) s += __ldcg(src + int64_t(bx) * a.chunk * w);
        a.out[i + int64_t(jx) * c] = s;
    }
    if (tid == 0) *a.counter = 0u;                 // ready for the next launch (stream order)
    if (a.fin_chol) {
        __syncthreads();
        if (tid == 0) chol_upper_serial(a.out, jx, w, a.R, a.status);
    }
}

struct XtyCfg { int JB, WM; };

static XtyCfg xty_cfg(int w) {
    if (w <= 1) return {4, 1};
    if (w <= 2) return {4, 2};
    if (w <= 4) return {4, 4};
    if (w <= 8) return {4, 8};
    if (w <= 12) return {4, 12};
    if (w <= 16) return {4, 16};
    return {2, 32};
}

static void xty_geometry(const Dev& d, int64_t n, int jx, int w, int* G, int* chunk, int* gx, int* gy) {
    const XtyCfg cf = xty_cfg(w);
    int need = (jx + cf.JB - 1) / cf.JB;
    int g = 1;
    while (g < need && g < 16) g *= 2;
    *G = g;
    *chunk = g * cf.JB;
    *gy = (jx + *chunk - 1) / *chunk;
    const int64_t ntiles = (n + XTY_TS - 1) / XTY_TS;
    int64_t want = int64_t(d.sms) * 2 / *gy;       // ~2 CTAs per SM in total (1 resident)
    if (want < 1) want = 1;
    if (want > ntiles) want = ntiles;
    if (want < 1) want = 1;
    *gx = int(want);
}

size_t xty_ws_doubles(const Dev& d, int jx, int w) {
    int G, chunk, gx, gy;
    xty_geometry(d, int64_t(1) << 40, jx, w, &G, &chunk, &gx, &gy);
    return size_t(gx) * size_t(gy) * size_t(chunk) * size_t(w);
}

template <int JB, int WM>
static void launch_xty(const XtyArgs& a, int gx, int gy, cudaStream_t st) {
    const size_t smem = size_t(WM) * XTY_TS * sizeof(double);
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_xty<JB, WM>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        attr = true;
    }
    ++g_launches; k_xty<JB, WM><<<dim3(gx, gy), NT, smem, st>>>(a);
}

int xty(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, const double* Y,
        int64_t ldy, int w, double* out, bool fin_chol, double* R, int* status,
        const XtyWs& ws, cudaStream_t st) {
    if (jx <= 0 || w <= 0 || w > 32) return -1;
    int G, chunk, gx, gy;
    xty_geometry(d, n, jx, w, &G, &chunk, &gx, &gy);
    if (size_t(gx) * gy * chunk * w > ws.cap) return -1;
    XtyArgs a{n, X, ldx, jx, Y, ldy, w, G, chunk, ws.part, out, ws.counter, fin_chol ? 1 : 0, R, status};
    const XtyCfg cf = xty_cfg(w);
    switch (cf.WM) {
        case 1: launch_xty<4, 1>(a, gx, gy, st); break;
        case 2: launch_xty<4, 2>(a, gx, gy, st); break;
        case 4: launch_xty<4, 4>(a, gx, gy, st); break;
        case 8: launch_xty<4, 8>(a, gx, gy, st); break;
        case 12: launch_xty<4, 12>(a, gx, gy, st); break;
        case 16: launch_xty<4, 16>(a, gx, gy, st); break;
        default: launch_xty<2, 32>(a, gx, gy, st); break;
    }
    return 0;
}

// ------------------------------------------------------------------------------------
// K9: P[:, 0:w] -= X C   (row-wise; C broadcast from shared memory)
// ------------------------------------------------------------------------------------
template <int WM>
__global__ void __launch_bounds__(NT) k_update(int64_t n, const double* __restrict__ X, int64_t ldx,
                                               int jx, double* __restrict__ P, int64_t ldp, int w,
                                               const double* __restrict__ C) {
    extern __shared__ double sC[];                 // jx x WM (row i contiguous: i*WM + c)
    for (int e = threadIdx.x; e < jx * WM; e += NT) {
        const int i = e / WM, c = e - i * WM;
        sC[e] = (c < w) ? C[i + int64_t(jx) * c] : 0.0;
    }
    __syncthreads();
    for (int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x; r < n; r += int64_t(gridDim.x) * NT) {
        double acc[WM];
#pragma unroll
        for (int c = 0; c < WM; ++c) acc[c] = (c < w) ? P[r + ldp * c] : 0.0;
#pragma unroll 8
        for (int i = 0; i < jx; ++i) {
            const double x = __ldg(X + r + ldx * i);
#pragma unroll
            for (int c = 0; c < WM; ++c) acc[c] = fma(-x, sC[i * WM + c], acc[c]);
        }
#pragma unroll
        for (int c = 0; c < WM; ++c)
            if (c < w) P[r + ldp * c] = acc[c];
    }
}

static int grid_stream(const Dev& d, int64_t n, int per_sm) {
    int64_t g = (n + NT - 1) / NT;
    const int64_t cap = int64_t(d.sms) * per_sm;
    if (g > cap) g = cap;
    return int(g < 1 ? 1 : g);
}

void update(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* P,
            int64_t ldp, int w, const double* C, cudaStream_t st) {
    if (jx <= 0 || n <= 0) return;
    const int grid = grid_stream(d, n, 8);
    auto go = [&](auto kfn, int WM) {
        const size_t smem = size_t(jx) * WM * sizeof(double);
        if (smem > 48 * 1024) cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        kfn<<<grid, NT, smem, st>>>(n, X, ldx, jx, P, ldp, w, C);
    };
    if (w <= 1) go(k_update<1>, 1);
    else if (w <= 2) go(k_update<2>, 2);
    else if (w <= 4) go(k_update<4>, 4);
    else if (w <= 8) go(k_update<8>, 8);
    else if (w <= 12) go(k_update<12>, 12);
    else if (w <= 16) go(k_update<16>, 16);
    else go(k_update<32>, 32);
}

// ------------------------------------------------------------------------------------
// K8: P[:, c0:w] = (P R^{-1})[:, c0:w], forward substitution per row with 1/R_cc.
// ------------------------------------------------------------------------------------
template <int WM>
__global__ void __launch_bounds__(NT) k_trsm(int64_t n, double* __restrict__ P, int64_t ldp, int w,
                                             const double* __restrict__ R, int c0) {
    __shared__ double sR[WM * WM];
    __shared__ double sInv[WM];
    for (int e = threadIdx.x; e < WM * WM; e += NT) {
        const int k = e / WM, c = e - k * WM;     // sR[k*WM + c] = R[k, c]
        sR[e] = (k < w && c < w) ? R[k + int64_t(w) * c] : 0.0;
    }
    for (int c = threadIdx.x; c < WM; c += NT) sInv[c] = (c < w) ? 1.0 / R[c + int64_t(w) * c] : 0.0;
    __syncthreads();
    for (int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x; r < n; r += int64_t(gridDim.x) * NT) {
        double p[WM];
#pragma unroll
        for (int c = 0; c < WM; ++c) p[c] = (c < w) ? P[r + ldp * c] : 0.0;
#pragma unroll
        for (int c = 0; c < WM; ++c) {
            double x = p[c];
#pragma unroll
            for (int k = 0; k < c; ++k) x = fma(-p[k], sR[k * WM + c], x);
            p[c] = x * sInv[c];
        }
#pragma unroll
        for (int c = 0; c < WM; ++c)
            if (c >= c0 && c < w) P[r + ldp * c] = p[c];
    }
}

void trsm(const Dev& d, int64_t n, double* P, int64_t ldp, int w, const double* R, int c0,
          cudaStream_t st) {
    if (n <= 0) return;
    const int grid = grid_stream(d, n, 8);
    if (w <= 1) { ++g_launches; k_trsm<1><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else if (w <= 2) { ++g_launches; k_trsm<2><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else if (w <= 4) { ++g_launches; k_trsm<4><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else if (w <= 8) { ++g_launches; k_trsm<8><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else if (w <= 12) { ++g_launches; k_trsm<12><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else if (w <= 16) { ++g_launches; k_trsm<16><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
    else { ++g_launches; k_trsm<32><<<grid, NT, 0, st>>>(n, P, ldp, w, R, c0); }
}

// ------------------------------------------------------------------------------------
// K2: halo pack / unpack
// ------------------------------------------------------------------------------------
__global__ void k_gather(const double* __restrict__ src, const int64_t* __restrict__ idx, int64_t cnt,
                         double* __restrict__ dst) {
    for (int64_t k = int64_t(blockIdx.x) * NT + threadIdx.x; k < cnt; k += int64_t(gridDim.x) * NT)
        dst[k] = src[idx[k]];
}
__global__ void k_scatter(const double* __restrict__ src, const int64_t* __restrict__ idx, int64_t cnt,
                          double* __restrict__ dst) {
    for (int64_t k = int64_t(blockIdx.x) * NT + threadIdx.x; k < cnt; k += int64_t(gridDim.x) * NT)
        dst[idx[k]] = src[k];
}
void gather(const double* src, const int64_t* idx, int64_t cnt, double* dst, cudaStream_t st) {
    if (cnt <= 0) return;
    const int64_t g = std::min<int64_t>((cnt + NT - 1) / NT, 4096);
    ++g_launches; k_gather<<<unsigned(g), NT, 0, st>>>(src, idx, cnt, dst);
}
void scatter(const double* src, const int64_t* idx, int64_t cnt, double* dst, cudaStream_t st) {
    if (cnt <= 0) return;
    const int64_t g = std::min<int64_t>((cnt + NT - 1) / NT, 4096);
    ++g_launches; k_scatter<<<unsigned(g), NT, 0, st>>>(src, idx, cnt, dst);
}

__global__ void k_add_small(const double* a, const double* b, double* c, int cnt) {
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) c[i] = a[i] + b[i];
}
void add_small(const double* a, const double* b, double* c, int cnt, cudaStream_t st) {
    if (cnt > 0) { ++g_launches; k_add_small<<<1, 256, 0, st>>>(a, b, c, cnt); }
}

}  // namespace kern
