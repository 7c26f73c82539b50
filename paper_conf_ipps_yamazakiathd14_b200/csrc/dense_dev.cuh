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

// Same factorization by one full warp (right-looking; lane c owns column c of the upper
// triangle, w <= 32).  Trailing updates G[i][c] -= R[k][i] R[k][c] are applied for
// k = 0, 1, ... in the order chol_upper_serial's fma chain uses, so R is bitwise identical.
// sm: w*w doubles of shared memory (scratch).  Must be called by all 32 lanes of a warp.
__device__ __forceinline__ void chol_upper_warp(const double* G, int ldg, int w, double* R, int* status,
                                                double* sm) {
    const int lane = threadIdx.x & 31;
    for (int q = lane; q < w * w; q += 32) {
        const int i = q % w, c = q / w;
        sm[q] = i <= c ? G[i + ldg * c] : 0.0;
    }
    __syncwarp();
    bool bad = false;
    for (int k = 0; k < w; ++k) {
        double dkk = sm[k + w * k];
        if (!(dkk > 0.0)) { bad = true; dkk = DBL_MIN; }
        const double rkk = sqrt(dkk);
        const double inv = 1.0 / rkk;
        __syncwarp();
        if (lane == k) sm[k + w * k] = rkk;
        if (lane > k && lane < w) sm[k + w * lane] *= inv;            // R[k][c]
        __syncwarp();
        if (lane > k && lane < w) {
            const double rkc = sm[k + w * lane];
            for (int i = k + 1; i <= lane; ++i) sm[i + w * lane] = fma(-sm[k + w * i], rkc, sm[i + w * lane]);
        }
        __syncwarp();
    }
    for (int q = lane; q < w * w; q += 32) {
        const int i = q % w, c = q / w;
        R[q] = i <= c ? sm[q] : 0.0;
    }
    if (bad && lane == 0) atomicOr(status, ST_CHOL);
}

}  // namespace kern
