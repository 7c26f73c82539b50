// reduce_probe.cu — fixed per-launch cost of the panel kernels' epilogue (per-CTA partials +
// __threadfence + atomic ticket + last-CTA fixed-order reduction), isolated from streaming.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -I paper_conf_ipps_yamazakiathd14_b200/csrc \
//        -o /tmp/reduce_probe tools/reduce_probe.cu && /tmp/reduce_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "kernels.h"
#include "reduce.cuh"
#include "dense_dev.cuh"

template <int MODE>   // 0: partials only; 1: + fence/ticket; 2: + last-CTA final_reduce; 3: tree_reduce
__global__ void k_epi(double* part, double* out, unsigned* counter, int nent, int touch_smem) {
    extern __shared__ double sm[];
    if (touch_smem) sm[threadIdx.x] = threadIdx.x;
    for (int e = threadIdx.x; e < nent; e += blockDim.x) part[int64_t(blockIdx.x) * nent + e] = e + blockIdx.x;
    if (MODE == 0) return;
    if (MODE == 3) {
        kern::tree_reduce(part, part + int64_t(gridDim.x) * nent, int(gridDim.x), int(blockIdx.x), nent, nent,
                          counter + 8, [&](int e, double t) { out[e] = t; });
        return;
    }
    __shared__ bool s_last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(counter, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (MODE == 2) {
        __shared__ double red[1024];
        kern::final_reduce(part, int(gridDim.x), nent, nent, red, [&](int e, double t) { out[e] = t; });
    }
    if (threadIdx.x == 0) *counter = 0u;
}

template <typename K>
float timeit(K k, int grid, int nt, size_t smem, double* part, double* out, unsigned* c, int nent, int touch) {
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    for (int i = 0; i < 10; ++i) k<<<grid, nt, smem>>>(part, out, c, nent, touch);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    const int R = 200;
    for (int i = 0; i < R; ++i) k<<<grid, nt, smem>>>(part, out, c, nent, touch);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms * 1000.f / R;
}

__global__ void k_chol_probe(const double* G, int w, double* R, int* st, int warp) {
    __shared__ double sm[32 * 32];
    if (warp) kern::chol_upper_warp(G, w, w, R, st, sm);
    else if (threadIdx.x == 0) kern::chol_upper_serial(G, w, w, R, st);
}

int main() {
    double *part, *out;
    unsigned* c;
    cudaMalloc(&part, sizeof(double) * 2 * 148 * 4096);
    cudaMalloc(&out, sizeof(double) * 4096);
    cudaMalloc(&c, 4 * 256);
    cudaMemset(c, 0, 4 * 256);
    {   // Cholesky of an 11x11 SPD matrix: serial thread vs warp, per launch (incl. launch cost)
        const int w = 11;
        double hG[w * w];
        for (int i = 0; i < w; ++i)
            for (int j = 0; j < w; ++j) hG[i + w * j] = (i == j ? w + 1.0 : 1.0 / (1 + i + j));
        double *G, *R;
        int* st;
        cudaMalloc(&G, sizeof(hG)); cudaMalloc(&R, sizeof(hG)); cudaMalloc(&st, 4);
        cudaMemcpy(G, hG, sizeof(hG), cudaMemcpyHostToDevice);
        for (int warp = 0; warp < 2; ++warp) {
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            k_chol_probe<<<1, 32>>>(G, w, R, st, warp);
            cudaEventRecord(e0);
            for (int i = 0; i < 200; ++i) k_chol_probe<<<1, 32>>>(G, w, R, st, warp);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("{\"chol_w11\": \"%s\", \"us_per_launch\": %.2f}\n", warp ? "warp" : "serial", ms * 5.f);
        }
    }
    for (int nent : {121, 320, 1000}) {
        for (size_t smem : {size_t(0), size_t(180 * 1024)}) {
            for (int nt : {256, 512}) {
                float t0 = timeit(k_epi<0>, 148, nt, smem, part, out, c, nent, smem > 0);
                float t1 = timeit(k_epi<1>, 148, nt, smem, part, out, c, nent, smem > 0);
                float t2 = timeit(k_epi<2>, 148, nt, smem, part, out, c, nent, smem > 0);
                float t3 = timeit(k_epi<3>, 148, nt, smem, part, out, c, nent, smem > 0);
                printf("{\"nent\": %d, \"smem_kb\": %zu, \"threads\": %d, \"us_partials\": %.2f, \"us_ticket\": %.2f, "
                       "\"us_final_reduce\": %.2f, \"us_tree_reduce\": %.2f}\n", nent, smem / 1024, nt, t0, t1, t2, t3);
            }
        }
    }
    return 0;
}
