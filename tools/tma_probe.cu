// tma_probe.cu — standalone probe of the streaming pipeline used by xty.cu / stream.cu:
// read an n x w column-major FP64 panel once via (a) the 1-D bulk-copy (TMA) ring with
// various tile sizes / stage counts / CTAs per SM and (b) plain vectorised loads, and report
// GB/s.  Build + run on the GPU box:
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/tma_probe tools/tma_probe.cu && /tmp/tma_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k_ring(const double* __restrict__ P, int64_t ld, int w, int64_t n, int TS, int S, double* out) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* bars = (uint64_t*)sm;
    double* slots = (double*)(sm + 128);
    const int SP = TS + 4;
    const int64_t ntiles = n / TS;
    const int64_t my = ntiles > blockIdx.x ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    auto issue = [&](int64_t k) {
        int s = int(k % S);
        int64_t r0 = (blockIdx.x + k * gridDim.x) * (int64_t)TS;
        double* dst = slots + (int64_t)s * w * SP;
        asm volatile("fence.proxy.async.shared::cta;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bars[s])), "r"(TS * 8 * w));
        for (int c = 0; c < w; ++c)
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(dst + (int64_t)c * SP)),
                         "l"(P + ld * c + r0), "r"(TS * 8), "r"(smem_u32(&bars[s])));
    };
    if (threadIdx.x == 0)
        for (int64_t k = 0; k < my && k < S; ++k) issue(k);
    double acc = 0;
    for (int64_t k = 0; k < my; ++k) {
        int s = int(k % S);
        uint32_t par = (uint32_t)((k / S) & 1);
        asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}" ::"r"(
                         smem_u32(&bars[s])),
                     "r"(par));
        const double* src = slots + (int64_t)s * w * SP;
        for (int e = threadIdx.x; e < TS * w; e += blockDim.x) acc += src[(e / TS) * SP + e % TS];
        __syncthreads();
        if (threadIdx.x == 0 && k + S < my) issue(k + S);
    }
    if (acc == 12345.678) out[0] = acc;
}

__global__ void k_plain(const double* __restrict__ P, int64_t ld, int w, int64_t n, double* out) {
    double acc = 0;
    for (int c = 0; c < w; ++c) {
        const double2* col = (const double2*)(P + ld * c);
        for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n / 2; i += (int64_t)gridDim.x * blockDim.x) {
            double2 v = __ldg(col + i);
            acc += v.x + v.y;
        }
    }
    if (acc == 12345.678) out[0] = acc;
}

int main() {
    const int64_t n = 1 << 21;
    const int wmax = 32;
    const int64_t ld = n;
    double* P;
    double* out;
    cudaMalloc(&P, sizeof(double) * ld * wmax);
    cudaMalloc(&out, 64);
    cudaMemset(P, 0, sizeof(double) * ld * wmax);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaFuncSetAttribute(k_ring, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    int ws[] = {1, 6, 11, 30};
    for (int wi = 0; wi < 4; ++wi) {
        int w = ws[wi];
        double bytes = 8.0 * n * w;
        // plain
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            k_plain<<<sms * 8, 256>>>(P, ld, w, n, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
        }
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("w=%2d plain                         %8.1f GB/s\n", w, bytes / ms / 1e6);
        int TSs[] = {128, 256, 512, 1024, 2048};
        int Ss[] = {2, 4, 6, 8};
        int cps[] = {1, 2, 3};
        for (int ti = 0; ti < 5; ++ti)
            for (int si = 0; si < 4; ++si)
                for (int ci = 0; ci < 3; ++ci) {
                    int TS = TSs[ti], S = Ss[si], cp = cps[ci];
                    size_t smem = 128 + (size_t)S * w * (TS + 4) * 8;
                    if (smem * cp > 227 * 1024) continue;
                    int grid = sms * cp;
                    for (int rep = 0; rep < 2; ++rep) {
                        cudaEventRecord(e0);
                        k_ring<<<grid, 256, smem>>>(P, ld, w, n, TS, S, out);
                        cudaEventRecord(e1);
                        cudaEventSynchronize(e1);
                    }
                    cudaError_t err = cudaGetLastError();
                    cudaEventElapsedTime(&ms, e0, e1);
                    printf("w=%2d ring TS=%4d S=%d cta/sm=%d smem=%6zu  %8.1f GB/s %s\n", w, TS, S, cp, smem,
                           bytes / ms / 1e6, err == cudaSuccess ? "" : cudaGetErrorString(err));
                }
    }
    return 0;
}
