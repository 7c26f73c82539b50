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

namespace kern {

// Two-level deterministic reduction of per-CTA partials, replacing "last CTA sums all
// partials" (a ~148 x nent serial read by one SM: 8-20 us, tools/reduce_probe.cu).
// CTA b (of nblk) has written part[b * stride + e], e < nent, and calls this with every
// thread.  CTAs form groups of TR_GS consecutive ids; the last CTA of a group to arrive
// (atomic ticket) sums its group's partials in id order into gpart[g * stride + e]; the last
// group to finish sums the group partials in group order and calls store(e, total).
// Each thread keeps all of its <= TR_GS loads in flight, so each level costs about one L2
// round trip.  Fixed summation order: bitwise reproducible for a given grid.  cnt: >= 65
// zeroed counters (left zeroed on exit).  Returns true only in the CTA that stored.
constexpr int TR_GS = 16;
constexpr int TR_TOP = 64;            // index of the top-level counter (nblk <= 64 * TR_GS)
constexpr int TR_CNT = 72;            // counters per independent reduction

template <class Store>
__device__ __forceinline__ bool tree_reduce(const double* part, double* gpart, int nblk, int b, int64_t stride,
                                            int nent, unsigned int* cnt, Store store) {
    const int ng = (nblk + TR_GS - 1) / TR_GS;
    const int g = b / TR_GS;
    const int gsz = min(TR_GS, nblk - g * TR_GS);
    __shared__ int s_flag;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_flag = atomicAdd(cnt + g, 1u) == unsigned(gsz - 1);
    __syncthreads();
    if (!s_flag) return false;
    __threadfence();
    const double* pg = part + int64_t(g) * TR_GS * stride;
    for (int e = threadIdx.x; e < nent; e += blockDim.x) {
        double v[TR_GS];
#pragma unroll
        for (int u = 0; u < TR_GS; ++u) v[u] = u < gsz ? __ldcg(pg + int64_t(u) * stride + e) : 0.0;
        double s = v[0];
#pragma unroll
        for (int u = 1; u < TR_GS; ++u)
            if (u < gsz) s += v[u];
        if (ng == 1) store(e, s);
        else __stcg(gpart + int64_t(g) * stride + e, s);
    }
    if (threadIdx.x == 0) cnt[g] = 0u;
    if (ng == 1) { __syncthreads(); return true; }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_flag = atomicAdd(cnt + TR_TOP, 1u) == unsigned(ng - 1);
    __syncthreads();
    if (!s_flag) return false;
    __threadfence();
    for (int e = threadIdx.x; e < nent; e += blockDim.x) {
        double s = 0.0;
        for (int g0 = 0; g0 < ng; g0 += TR_GS) {
            double v[TR_GS];
#pragma unroll
            for (int u = 0; u < TR_GS; ++u) v[u] = g0 + u < ng ? __ldcg(gpart + int64_t(g0 + u) * stride + e) : 0.0;
#pragma unroll
            for (int u = 0; u < TR_GS; ++u)
                if (g0 + u < ng) s = (g0 + u == 0) ? v[u] : s + v[u];
        }
        store(e, s);
    }
    if (threadIdx.x == 0) cnt[TR_TOP] = 0u;
    __syncthreads();
    return true;
}

}  // namespace kern
