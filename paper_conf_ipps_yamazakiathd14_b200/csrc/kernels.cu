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
#include "dense_dev.cuh"

namespace kern {

constexpr int NT = 256;
constexpr int SPMV_BATCH = 4;           // entries whose loads are issued together
long long g_launches = 0;
int g_pdl = 1;

// ------------------------------------------------------------------------------------
// K1: y = A x + bu*u + bw*w on the first nrows rows of a SELL-32 matrix.
// One thread per row; a warp covers one 32-row slice whose entries are stored column-major
// (entry t of row lane at sptr[slice] + 32 t + lane) so val/col loads are fully coalesced.
// Padding entries have val = 0 and col = the row itself (always a valid, in-range x).
// Per-row summation runs over the stored (= global column) order, so a row's result does
// not depend on the partition.
// ------------------------------------------------------------------------------------
template <int MODE>   // 0: Ax   1: Ax + bu u   2: Ax + bu u + bw w   3: u - Ax
__global__ void __launch_bounds__(NT, 6) k_spmv_sell32(int64_t nrows, const int64_t* __restrict__ sptr,
                                                    const int64_t* __restrict__ sinfo,
                                                    const int32_t* __restrict__ dcol, int64_t ncols,
                                                    const double* __restrict__ val,
                                                    const double* __restrict__ x,
                                                    const double* __restrict__ u, double bu,
                                                    const double* __restrict__ w, double bw,
                                                    double* __restrict__ y) {
    const int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x;
    if ((r & ~int64_t(31)) >= nrows) return;           // whole warp beyond the matrix
    // every lane of the warp takes part (shuffles): lane t must load the slice's offset t.
    // Rows >= nrows of the last slice are padding (val 0, in-range or clamp-flagged columns)
    // or real rows beyond this step's prefix: they compute but do not store.
    const double acc = sell_row_dot<SPMV_BATCH>(r, sptr, sinfo, dcol, ncols, val, x, false);
    if (r >= nrows) return;
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

// Persistent SpMV with a software-pipelined slice descriptor.  In k_spmv_sell32 every warp
// pays a chain of dependent loads before its first x gather (sptr/sinfo -> DIA offsets ->
// x), ~3 L2/HBM latencies for 32 rows of ~7 entries.  Here a grid of (SMs x resident CTAs)
// warps strides over the slices and, while slice i's values and x are in flight, already
// holds slice i+1's (b, W, info) and offsets and loads slice i+2's (b, W, info): one latency
// per slice.  Per row the FMA order is t = 0..W-1 exactly as sell_row_dot: results are
// bitwise identical to k_spmv_sell32.
template <int MODE, int PB, int MINB>
__global__ void __launch_bounds__(NT, MINB) k_spmv_sell32_persist(int64_t nrows, const int64_t* __restrict__ sptr,
                                                             const int64_t* __restrict__ sinfo,
                                                             const int32_t* __restrict__ dcol, int64_t ncols,
                                                             const double* __restrict__ val,
                                                             const double* __restrict__ x,
                                                             const double* __restrict__ u, double bu,
                                                             const double* __restrict__ w, double bw,
                                                             double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int64_t nsl = (nrows + 31) >> 5;
    const int64_t stride = int64_t(gridDim.x) * (NT / 32);
    int64_t sl = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    if (sl >= nsl) { pdl_wait(); pdl_trigger(); return; }
    // descriptors: current slice (b0, W0, i0, o0), next (b1, W1, i1, o1), after next (b2, W2, i2)
    // (the matrix is never written during a solve: loaded before the PDL wait)
    int64_t b0, i0, b1 = 0, i1 = 1, b2, i2;
    int W0, W1 = 0, W2, o0, o1;
    sell_slice_meta(sl, sptr, sinfo, b0, W0, i0);
    if (sl + stride < nsl) sell_slice_meta(sl + stride, sptr, sinfo, b1, W1, i1);
    o0 = sell_slice_off(lane, W0, i0, dcol);
    pdl_wait();
    pdl_trigger();
#pragma unroll 1
    for (; sl < nsl; sl += stride) {
        b2 = 0; W2 = 0; i2 = 1;
        if (sl + 2 * stride < nsl) sell_slice_meta(sl + 2 * stride, sptr, sinfo, b2, W2, i2);
        o1 = sell_slice_off(lane, W1, i1, dcol);
        const int64_t r = sl * 32 + lane;
        const double acc = sell_slice_dot<PB, true>(r, b0, W0, i0, o0, dcol, ncols, val, x, false);
        if (r < nrows) {
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
        b0 = b1; W0 = W1; i0 = i1; o0 = o1;
        b1 = b2; W1 = W2; i1 = i2;
    }
}

template <int MODE, int PB, int MINB>
static void launch_persist(const Dev& d, const Sell& A, int64_t nrows, const double* x, double* y,
                           const double* u, double bu, const double* w, double bw, cudaStream_t st) {
    static int occ = 0;
    if (occ == 0) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_spmv_sell32_persist<MODE, PB, MINB>, NT, 0);
        if (occ < 1) occ = 1;
    }
    const int64_t nsl = (nrows + 31) >> 5;
    int64_t g = int64_t(d.sms) * occ;
    const int64_t need = (nsl + NT / 32 - 1) / (NT / 32);
    if (g > need) g = need;
    launch_pdl(k_spmv_sell32_persist<MODE, PB, MINB>, dim3(unsigned(g)), dim3(NT), 0, st, nrows, A.sptr, A.sinfo,
               A.dcol, A.ncols, A.val, x, u, bu, w, bw, y);
}

// CAGMRES_OPT_SPMV: 0 = one SELL-32 slice per warp (k_spmv_sell32); 5 = persistent grid with
// software-pipelined slice descriptors (k_spmv_sell32_persist); 16, 17 = the DIA-width
// specialised persistent kernel with an L2 prefetch of the next slice (spmv_dia.cu) at >= 4 / 5
// CTAs per SM.  (Round 1 shipped 19 variants; the others were measured slower and removed:
// DESIGN.md §6.)
void spmv(const Dev& d, const Sell& A, int64_t nrows, const double* x, double* y,
          const double* u, double bu, const double* w, double bw, cudaStream_t st) {
    (void)d;
    if (nrows <= 0) return;
    ++g_launches;
    if (w && !u) { u = x; bu = 0.0; }             // pair step with a == 0: keep MODE 2 well formed
    if (A.variant >= 16) {
        spmv_dia(d, A, A.variant, nrows, x, y, u, bu, w, bw, w ? 2 : (u ? 1 : 0), st);
        return;
    }
    if (A.variant == 5) {
        if (w) launch_persist<2, 4, 4>(d, A, nrows, x, y, u, bu, w, bw, st);
        else if (u) launch_persist<1, 4, 4>(d, A, nrows, x, y, u, bu, nullptr, 0.0, st);
        else launch_persist<0, 4, 4>(d, A, nrows, x, y, nullptr, 0.0, nullptr, 0.0, st);
        return;
    }
    const unsigned grid = unsigned((nrows + NT - 1) / NT);
    if (w)
        k_spmv_sell32<2><<<grid, NT, 0, st>>>(nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, u, bu, w, bw, y);
    else if (u)
        k_spmv_sell32<1><<<grid, NT, 0, st>>>(nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, u, bu, nullptr, 0.0, y);
    else
        k_spmv_sell32<0><<<grid, NT, 0, st>>>(nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, nullptr, 0.0, nullptr, 0.0, y);
}

int spmv_scaled(const Dev& d, const Sell& A, int64_t nrows, const double* w, const double* wnrm, double* xs,
                double* y, double bu, bool shift, cudaStream_t st) {
    if (A.variant < 16) return -1;
    if (nrows <= 0) return 0;
    ++g_launches;
    spmv_dia(d, A, A.variant, nrows, w, y, nullptr, bu, nullptr, 0.0, shift ? 5 : 4, st, wnrm, xs);
    return 0;
}

__global__ void __launch_bounds__(256) k_scale_copy(int64_t n, const double* __restrict__ w,
                                                    const double* __restrict__ wnrm, double* __restrict__ xs) {
    pdl_wait();
    pdl_trigger();
    const double inv = 1.0 / __ldg(wnrm);                  // the product k_scale1 forms
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
        xs[i] = __ldg(w + i) * inv;
}

void scale_copy(int64_t n, const double* w, const double* wnrm, double* xs, cudaStream_t st) {
    if (n <= 0) return;
    const int64_t g = std::min<int64_t>((n + 255) / 256, 148 * 8);
    ++g_launches;
    launch_pdl(k_scale_copy, dim3(unsigned(g)), dim3(256), 0, st, n, w, wnrm, xs);
}

void residual(const Dev& d, const Sell& A, int64_t nrows, const double* x, const double* b,
              double* r, cudaStream_t st) {
    (void)d;
    if (nrows <= 0) return;
    ++g_launches;
    if (A.variant >= 16) {
        spmv_dia(d, A, A.variant, nrows, x, r, b, 1.0, nullptr, 0.0, 3, st);
        return;
    }
    if (A.variant == 5) {
        launch_persist<3, 4, 4>(d, A, nrows, x, r, b, 1.0, nullptr, 0.0, st);
        return;
    }
    const unsigned grid = unsigned((nrows + NT - 1) / NT);
    k_spmv_sell32<3><<<grid, NT, 0, st>>>(nrows, A.sptr, A.sinfo, A.dcol, A.ncols, A.val, x, b, 1.0, nullptr, 0.0, r);
}

// ------------------------------------------------------------------------------------
// Small dense factorizations on one thread / one CTA (w <= 32).
// ------------------------------------------------------------------------------------
__global__ void k_chol(const double* G, int w, double* R, int* status) {
    __shared__ double sm[32 * 32];
    pdl_wait();
    pdl_trigger();
    chol_upper_warp(G, w, w, R, status, sm);
}

void chol(const double* G, int w, double* R, int* status, cudaStream_t st) {
    ++g_launches; launch_pdl(k_chol, dim3(1), dim3(32), 0, st, G, w, R, status);
}

// SVQR (reading G14): D = diag(G)^{-1/2}; D G D = U S U^T (cyclic
// Jacobi); s_i <- max(s_i, eps s_max); R_hat = R of qr(S^{1/2} U^T) (Householder, positive
// diagonal); R = R_hat D^{-1}.  One thread, w <= 32 (a comparator-sized cost).
// One warp: lane k owns row/column k of the w x w matrices (w <= 32).  Each Jacobi rotation's
// (c, s) is computed redundantly by every lane from shared memory, then the two columns, the
// two rows and V are updated lane-parallel; sums (off-diagonal norm, Householder norms and dot
// products) are warp shuffle reductions.  (The one-thread version took ~0.5 ms at w = 11.)
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// retry = 1 (G15 opt-in, CAGMRES_SVQR_RETRY): act only if the CholQR of this panel broke down
// (ST_CHOL set by the Gram/Cholesky launch just before), then clear ST_CHOL and count the retry
// in status[1]; R is replaced by the SVQR factor of the same Gram G.
__global__ void k_svqr(const double* G, int w, double* R, int* status, int retry) {
    __shared__ double A[32 * 33], V[32 * 33], d[32];
    constexpr int LD = 33;
    const int k = threadIdx.x;                         // lane
    pdl_wait();
    pdl_trigger();
    if (retry) {
        const int st0 = *(volatile int*)status;
        if (!(st0 & ST_CHOL)) return;
        __syncwarp();
        if (k == 0) {
            atomicAnd(status, ~ST_CHOL);
            atomicAdd(status + 1, 1);
        }
    }
    if (k < w) {
        const double g = G[k + w * k];
        if (!(g > 0.0)) { atomicOr(status, ST_SVQR); d[k] = 1.0; } else d[k] = 1.0 / sqrt(g);
    }
    __syncwarp();
    for (int j = 0; j < w; ++j)
        if (k < w) {
            const double g = (k <= j) ? G[k + w * j] : G[j + w * k];
            A[k + LD * j] = d[k] * g * d[j];
            V[k + LD * j] = (k == j) ? 1.0 : 0.0;
        }
    __syncwarp();
    for (int sweep = 0; sweep < 60; ++sweep) {
        double off = 0.0, dia = 0.0;
        if (k < w) {
            dia = A[k + LD * k] * A[k + LD * k];
            for (int i = 0; i < k; ++i) off += A[i + LD * k] * A[i + LD * k];
        }
        off = warp_sum(off);
        dia = warp_sum(dia);
        if (off <= DBL_EPSILON * DBL_EPSILON * dia * 1e-2) break;
        for (int p = 0; p < w - 1; ++p)
            for (int q = p + 1; q < w; ++q) {
                const double apq = A[p + LD * q];
                if (apq == 0.0) continue;                  // uniform: every lane read the same value
                const double tau = (A[q + LD * q] - A[p + LD * p]) / (2.0 * apq);
                const double t = (tau >= 0.0 ? 1.0 : -1.0) / (fabs(tau) + sqrt(1.0 + tau * tau));
                const double c = 1.0 / sqrt(1.0 + t * t), sn = t * c;
                __syncwarp();
                if (k < w) {                               // columns p, q
                    const double akp = A[k + LD * p], akq = A[k + LD * q];
                    A[k + LD * p] = c * akp - sn * akq;
                    A[k + LD * q] = sn * akp + c * akq;
                    const double vkp = V[k + LD * p], vkq = V[k + LD * q];
                    V[k + LD * p] = c * vkp - sn * vkq;
                    V[k + LD * q] = sn * vkp + c * vkq;
                }
                __syncwarp();
                if (k < w) {                               // rows p, q
                    const double apk = A[p + LD * k], aqk = A[q + LD * k];
                    A[p + LD * k] = c * apk - sn * aqk;
                    A[q + LD * k] = sn * apk + c * aqk;
                }
                __syncwarp();
            }
    }
    double smax = k < w ? A[k + LD * k] : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) smax = fmax(smax, __shfl_xor_sync(0xffffffffu, smax, o));
    // M = S^{1/2} U^T (stored in A): row i = sq[i] * column i of V
    const double sqk = k < w ? sqrt(fmax(A[k + LD * k], DBL_EPSILON * smax)) : 0.0;
    __syncwarp();
    for (int i = 0; i < w; ++i) {
        const double sqi = __shfl_sync(0xffffffffu, sqk, i);
        if (k < w) A[i + LD * k] = sqi * V[k + LD * i];
    }
    __syncwarp();
    // Householder QR of M (w x w); lane = row index
    for (int kk = 0; kk < w; ++kk) {
        const double aik = (k >= kk && k < w) ? A[k + LD * kk] : 0.0;
        const double nrm = sqrt(warp_sum(aik * aik));
        if (nrm == 0.0) continue;
        const double akk = __shfl_sync(0xffffffffu, aik, kk);
        const double alpha = -copysign(nrm, akk);
        const double vi = aik - (k == kk ? alpha : 0.0);
        const double vv = warp_sum(vi * vi);
        if (vv == 0.0) continue;
        const double beta = 2.0 / vv;
        for (int c = kk; c < w; ++c) {
            const double aic = (k >= kk && k < w) ? A[k + LD * c] : 0.0;
            const double dd = warp_sum(vi * aic) * beta;
            __syncwarp();
            if (k >= kk && k < w) A[k + LD * c] = aic - dd * vi;
            __syncwarp();
        }
    }
    if (k < w) {
        const double sg = A[k + LD * k] < 0.0 ? -1.0 : 1.0;
        for (int c = 0; c < w; ++c) R[k + w * c] = (c < k) ? 0.0 : sg * A[k + LD * c] / d[c];
    }
}

void svqr_factor(const double* G, int w, double* R, int* status, cudaStream_t st) {
    ++g_launches; launch_pdl(k_svqr, dim3(1), dim3(32), 0, st, G, w, R, status, 0);
}
void svqr_retry(const double* G, int w, double* R, int* status, cudaStream_t st) {
    ++g_launches; launch_pdl(k_svqr, dim3(1), dim3(32), 0, st, G, w, R, status, 1);
}

// ------------------------------------------------------------------------------------
// K2: halo pack / unpack
// ------------------------------------------------------------------------------------
template <bool SCATTER>
__global__ void k_halo_segs(const double* __restrict__ src, const int64_t* __restrict__ idx, Segs sg,
                            int64_t tot, double* __restrict__ dst) {
    for (int64_t t = int64_t(blockIdx.x) * NT + threadIdx.x; t < tot; t += int64_t(gridDim.x) * NT) {
        int i = 0;
        int64_t k = t;
        while (k >= sg.cnt[i]) { k -= sg.cnt[i]; ++i; }
        k += sg.off[i];
        if (SCATTER) dst[idx[k]] = src[k];
        else dst[k] = src[idx[k]];
    }
}
template <bool SCATTER>
static void halo_segs(const double* src, const int64_t* idx, const Segs& sg, double* dst, cudaStream_t st) {
    int64_t tot = 0;
    for (int i = 0; i < sg.n; ++i) tot += sg.cnt[i];
    if (tot <= 0) return;
    const int64_t g = std::min<int64_t>((tot + NT - 1) / NT, 4096);
    ++g_launches;
    k_halo_segs<SCATTER><<<unsigned(g), NT, 0, st>>>(src, idx, sg, tot, dst);
}
void gather_segs(const double* src, const int64_t* idx, const Segs& sg, double* dst, cudaStream_t st) {
    halo_segs<false>(src, idx, sg, dst, st);
}
void scatter_segs(const double* src, const int64_t* idx, const Segs& sg, double* dst, cudaStream_t st) {
    halo_segs<true>(src, idx, sg, dst, st);
}

__global__ void k_add_small(const double* a, const double* b, double* c, int cnt) {
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) c[i] = a[i] + b[i];
}
void add_small(const double* a, const double* b, double* c, int cnt, cudaStream_t st) {
    if (cnt > 0) { ++g_launches; k_add_small<<<1, 256, 0, st>>>(a, b, c, cnt); }
}

}  // namespace kern
