// onepass.cu — small-matrix step of the one-pass BOrth + CholQR (P:176 fused
// CGS, P:275 fn 7), between the two panel passes:
//   pass 1 (xty.cu)   Mx = [Q P]^T P                           ((j+w) x w, summed over ranks)
//   here  (1 CTA)     C  = Mx[0:j, 1:w]                         (BOrth coefficients, col 0 = 0)
//                     G  = Mx[j:j+w, :] - Cf^T Cf,  Cf = [0 | C] (Pythagoras, Q^T Q = I)
//                     R  = chol(G)                              (upper, positive diagonal)
//                     Mo = [-Cf R^{-1} ; R^{-1}]                ((j+w) x w, ld j+w)
//   pass 2 (stream.cu gemm_rows)  P[:, 1:w] = ([Q P] Mo)[:, 1:w] = ((P - Q Cf) R^{-1})[:, 1:w]
// Same arithmetic as oracle/borth_cholqr_onepass up to summation order.
#include <cfloat>
#include <cstdint>

#include "dense_dev.cuh"
#include "kernels.h"

namespace kern {

__global__ void __launch_bounds__(256) k_onepass_finalize(const double* __restrict__ Mx, int j, int w,
                                                          double* __restrict__ C, double* __restrict__ R,
                                                          double* __restrict__ Mo, int* status) {
    __shared__ double sM[64 * 32], sG[32 * 32], sCh[32 * 32], sRi[32 * 32], sInv[32];
    const int K = j + w;
    pdl_wait();
    pdl_trigger();
    // stage Mx (K x w <= 64 x 32) in shared memory with one coalesced pass (the dot products
    // below would otherwise be chains of dependent L2 loads)
    for (int q = threadIdx.x; q < K * w; q += blockDim.x) sM[q] = Mx[q];
    __syncthreads();
    // G = Mx[j:, :] - Cf^T Cf (upper triangle, ld w); C out (ld j)
    for (int q = threadIdx.x; q < w * w; q += blockDim.x) {
        const int a = q % w, b = q / w;
        double g = 0.0;
        if (a <= b) {
            g = sM[j + a + K * b];
            if (a > 0)
                for (int i = 0; i < j; ++i) g = fma(-sM[i + K * a], sM[i + K * b], g);
        }
        sG[a + w * b] = g;
    }
    for (int q = threadIdx.x; q < j * (w - 1); q += blockDim.x) {
        const int i = q % j, c = q / j;
        C[i + int64_t(j) * c] = sM[i + K * (c + 1)];
    }
    __syncthreads();
    if (threadIdx.x < 32) chol_upper_warp(sG, w, w, R, status, sCh);
    __syncthreads();
    // R^{-1} (upper) by column back substitution, one thread per column; R is in sCh (the
    // warp Cholesky's scratch, ld w, upper part valid)
    for (int k = threadIdx.x; k < w; k += blockDim.x) sInv[k] = 1.0 / sCh[k + w * k];
    __syncthreads();
    for (int c = threadIdx.x; c < w; c += blockDim.x) {
        for (int k = 0; k < w; ++k) sRi[k + 32 * c] = 0.0;
        sRi[c + 32 * c] = sInv[c];
        for (int k = c - 1; k >= 0; --k) {
            double s = 0.0;
            for (int l = k + 1; l <= c; ++l) s = fma(sCh[k + w * l], sRi[l + 32 * c], s);
            sRi[k + 32 * c] = -s * sInv[k];
        }
    }
    __syncthreads();
    // Mo = [-Cf R^{-1}; R^{-1}]
    for (int q = threadIdx.x; q < K * w; q += blockDim.x) {
        const int i = q % K, c = q / K;
        double v;
        if (i >= j) {
            v = sRi[(i - j) + 32 * c];
        } else {
            double s = 0.0;
            for (int a = 1; a <= c; ++a) s = fma(sM[i + K * a], sRi[a + 32 * c], s);
            v = -s;
        }
        Mo[i + int64_t(K) * c] = v;
    }
}

void onepass_finalize(const double* Mx, int j, int w, double* C, double* R, double* Mo, int* status,
                      cudaStream_t st) {
    ++g_launches;
    launch_pdl(k_onepass_finalize, dim3(1), dim3(256), 0, st, Mx, j, w, C, R, Mo, status);
}

}  // namespace kern
