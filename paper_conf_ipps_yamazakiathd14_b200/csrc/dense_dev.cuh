// dense_dev.cuh — tiny dense factorizations run by one device thread (w <= 32).
#pragma once
#include <cfloat>
#include "kernels.h"

namespace kern {

__device__ __forceinline__ void chol_upper_serial(const double* G, int ldg, int w, double* R, int* status) {
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

}  // namespace kern

namespace kern {

// Same factorization by one full warp, register-resident (right-looking; lane c owns column c
// of the upper triangle in registers, w <= WM <= 32).  Step k: the pivot comes from lane k by
// shuffle, inv = rsqrt(pivot) (one MUFU + Newton steps; R[k][k] = pivot * inv), row k is scaled
// by inv, and the trailing update g[i] -= R[k][i] R[k][c] takes R[k][i] from lane i by shuffle
// — no shared-memory round trips or divisions on the serial chain (the shared-memory version
// cost ~3-5 us in the Gram kernel's last CTA).  Writes R (w x w, ld w, zeros below the
// diagonal) to R and to sm.  Must be called by all 32 lanes of a warp.
template <int WM>
__device__ __forceinline__ void chol_upper_regs(const double* G, int ldg, int w, double* R, int* status,
                                                double* sm) {
    const int lane = threadIdx.x & 31;
    double g[WM];
#pragma unroll
    for (int i = 0; i < WM; ++i) g[i] = (i <= lane && lane < w) ? G[i + ldg * lane] : 0.0;
    bool bad = false;
#pragma unroll
    for (int k = 0; k < WM; ++k) {
        if (k >= w) break;
        double dkk = __shfl_sync(0xffffffffu, g[k], k);
        if (!(dkk > 0.0)) { bad = true; dkk = DBL_MIN; }
        const double inv = rsqrt(dkk);
        if (lane == k) g[k] = dkk * inv;
        else if (lane > k) g[k] *= inv;                             // R[k][lane]
#pragma unroll
        for (int i = k + 1; i < WM; ++i) {
            if (i >= w) break;
            const double rki = __shfl_sync(0xffffffffu, g[k], i);  // R[k][i]
            if (lane >= i) g[i] = fma(-rki, g[k], g[i]);
        }
    }
    if (lane < w) {
#pragma unroll
        for (int i = 0; i < WM; ++i)
            if (i < w) {
                const double v = i <= lane ? g[i] : 0.0;
                R[i + w * lane] = v;
                sm[i + w * lane] = v;
            }
    }
    if (bad && lane == 0) atomicOr(status, ST_CHOL);
}

__device__ __forceinline__ void chol_upper_warp(const double* G, int ldg, int w, double* R, int* status,
                                                double* sm) {
    if (w <= 12) chol_upper_regs<12>(G, ldg, w, R, status, sm);
    else chol_upper_regs<32>(G, ldg, w, R, status, sm);
}

}  // namespace kern
