// fp64_probe.cu — measured FP64 throughput on this GPU: scalar DFMA vs tensor-core DMMA
// (mma.sync.m8n8k4.f64), to decide which pipe the panel contractions (Gram / BOrth) use.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/fp64_probe tools/fp64_probe.cu && /tmp/fp64_probe
#include <cstdio>
#include <cuda_runtime.h>

template <int CH>
__global__ void k_dfma(double* out, int iters, double a, double b) {
    double acc[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) acc[c] = threadIdx.x * 1e-9 + c;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c) acc[c] = fma(acc[c], a, b);
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += acc[c];
    if (s == 12345.678) out[0] = s;
}

template <int CH>
__global__ void k_dmma(double* out, int iters, double a, double b) {
    double d0[CH], d1[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) d0[c] = d1[c] = threadIdx.x * 1e-9 + c;
    double av = a + threadIdx.x * 1e-12, bv = b;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                         : "+d"(d0[c]), "+d"(d1[c])
                         : "d"(av), "d"(bv));
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += d0[c] + d1[c];
    if (s == 12345.678) out[0] = s;
}

template <typename K>
float run(K k, int blocks, int threads, int iters, double* out) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k<<<blocks, threads>>>(out, 10, 1.0000001, 1e-9);
    cudaEventRecord(e0);
    k<<<blocks, threads>>>(out, iters, 1.0000001, 1e-9);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double* out;
    cudaMalloc(&out, 8);
    const int iters = 20000;
    for (int warps : {4, 8, 16, 32}) {
        int thr = 32 * warps;
        float ms = run(k_dfma<8>, sms * 2, thr, iters, out);
        double fl = 2.0 * 8 * iters * double(sms) * 2 * thr;
        printf("{\"probe\": \"dfma\", \"warps_per_cta\": %d, \"ctas\": %d, \"tflops\": %.2f}\n", warps, sms * 2,
               fl / ms / 1e9);
        ms = run(k_dmma<4>, sms * 2, thr, iters, out);
        fl = 512.0 * 4 * iters * double(sms) * 2 * warps;
        printf("{\"probe\": \"dmma_m8n8k4\", \"warps_per_cta\": %d, \"ctas\": %d, \"tflops\": %.2f}\n", warps,
               sms * 2, fl / ms / 1e9);
        ms = run(k_dmma<8>, sms * 2, thr, iters, out);
        fl = 512.0 * 8 * iters * double(sms) * 2 * warps;
        printf("{\"probe\": \"dmma_m8n8k4_ch8\", \"warps_per_cta\": %d, \"ctas\": %d, \"tflops\": %.2f}\n", warps,
               sms * 2, fl / ms / 1e9);
    }
    return 0;
}
