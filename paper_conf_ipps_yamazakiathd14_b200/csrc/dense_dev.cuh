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
