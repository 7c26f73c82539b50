// reduce.cuh — fixed-order parallel reduction of per-CTA partials, run by the last CTA of
// a launch (atomic ticket).  out[e] = sum_{b < nblk} part[b * stride + e] for e < nent.
// Every thread sums an (entry, subset) slice with 8 independent loads in flight, and the
// subsets of an entry are combined in a fixed order: the result is deterministic for a
// given launch geometry, and the serial L2-latency chain is ~nblk / (8 S) instead of nblk.
#pragma once
#include <cstdint>

namespace kern {

template <class Store>
__device__ __forceinline__ void final_reduce(const double* part, int nblk, int64_t stride, int nent,
                                             double* red /* blockDim.x doubles of smem */, Store store) {
    const int nth = blockDim.x, t = threadIdx.x;
    int S = nent > 0 ? nth / nent : nth;
    S = S < 1 ? 1 : (S > 32 ? 32 : S);
    const int EB = nth / S;                       // entries per pass
    for (int e0 = 0; e0 < nent; e0 += EB) {
        const int el = t / S, sub = t - el * S, e = e0 + el;
        const bool act = el < EB && e < nent;
        double s = 0.0;
        if (act) {
            int b = sub;
            for (; b + 7 * S < nblk; b += 8 * S) {
                double v[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) v[u] = __ldcg(part + int64_t(b + u * S) * stride + e);
#pragma unroll
                for (int u = 0; u < 8; ++u) s += v[u];
            }
            for (; b < nblk; b += S) s += __ldcg(part + int64_t(b) * stride + e);
        }
        red[t] = s;
        __syncthreads();
        if (act && sub == 0) {
            double tot = 0.0;
            for (int q = 0; q < S; ++q) tot += red[t + q];
            store(e, tot);
        }
        __syncthreads();
    }
}

}  // namespace kern
