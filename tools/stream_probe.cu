// stream_probe.cu — what one kernel launch can move on this B200, cold L2, as a function of
// size: read-only (sum) and copy (read + write) of a flat buffer with 16-B loads, grid-strided,
// (clean L2: evicted by reading another 512 MB before every timed launch)
// U independent loads in flight per thread.  Calibrates the per-kernel roofline fractions of the
// panel kernels: a 185 MB panel read is not a 2 GB copy.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/sp tools/stream_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int U>
__global__ void __launch_bounds__(256) k_read(const double2* __restrict__ p, long n2, double* sink) {
    double acc = 0.0;
    const long stride = long(gridDim.x) * blockDim.x;
    long i = long(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < n2; i += U * stride) {
        double2 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcg(p + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) acc += v[u].x + v[u].y;
    }
    for (; i < n2; i += stride) acc += p[i].x;
    if (acc == 1.2345) *sink = acc;
}

template <int U>
__global__ void __launch_bounds__(256) k_copy(const double2* __restrict__ p, double2* __restrict__ q, long n2) {
    const long stride = long(gridDim.x) * blockDim.x;
    long i = long(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < n2; i += U * stride) {
        double2 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcg(p + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) q[i + u * stride] = v[u];
    }
    for (; i < n2; i += stride) q[i] = p[i];
}

// Same read with DYNAMIC work distribution: every warp takes 64 KB chunks (16 sub-steps of 8 x
// 16 B per lane) from a global atomic counter, fetching the next chunk index while it reads the
// current one, until the buffer is done — SMs that see more bandwidth do more chunks (static
// shares finish when the slowest SM does).
template <int CH>
__global__ void __launch_bounds__(256) k_read_dyn(const double2* __restrict__ p, long n2, double* sink,
                                                  unsigned long long* ctr) {
    const int lane = threadIdx.x & 31;
    constexpr int SUB = 16;
    const long per = 32L * CH * SUB;
    double acc = 0.0;
    long c = 0;
    if (lane == 0) c = long(atomicAdd(ctr, 1ull));
    c = __shfl_sync(0xffffffffu, c, 0);
    while (c * per < n2) {
        long nx = 0;
        if (lane == 0) nx = long(atomicAdd(ctr, 1ull));                  // next chunk, in flight
        const long c0 = c * per;
        for (int sb = 0; sb < SUB; ++sb) {
            double2 v[CH];
#pragma unroll
            for (int u = 0; u < CH; ++u) {
                const long i = c0 + (long(sb) * CH + u) * 32 + lane;
                v[u] = i < n2 ? __ldcg(p + i) : make_double2(0.0, 0.0);
            }
#pragma unroll
            for (int u = 0; u < CH; ++u) acc += v[u].x + v[u].y;
        }
        c = __shfl_sync(0xffffffffu, nx, 0);
    }
    if (acc == 1.2345) *sink = acc;
}

// Static band + dynamic tail: every warp reads its grid-stride share of the first `split` of the
// buffer (the band order of the panel kernels), then takes 4 KB chunks of the rest from one of 8
// atomic counters (its CTA's counter id = blockIdx % 8, region-interleaved) until all are done —
// so SMs that finish their static share early absorb the stragglers' tail.
__global__ void __launch_bounds__(256) k_read_tail(const double2* __restrict__ p, long n2, double* sink,
                                                   unsigned long long* ctr, double split) {
    const int lane = threadIdx.x & 31;
    const long stride = long(gridDim.x) * blockDim.x;
    const long ns = long(double(n2) * split) / stride * stride;      // statically assigned part
    double acc = 0.0;
    long i = long(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; i + 3 * stride < ns; i += 4 * stride) {
        double2 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) v[u] = __ldcg(p + i + u * stride);
#pragma unroll
        for (int u = 0; u < 4; ++u) acc += v[u].x + v[u].y;
    }
    for (; i < ns; i += stride) acc += p[i].x + p[i].y;
    constexpr int CH = 8;                                           // 8 x 16 B per lane = 4 KB per grab
    const long per = 32L * CH;
    const long rest = n2 - ns;
    const int q = blockIdx.x & 7;                                   // 8 interleaved queues
    const long nchunk = (rest + per - 1) / per;
    for (;;) {
        long c = 0;
        if (lane == 0) c = long(atomicAdd(ctr + q, 1ull)) * 8 + q;
        c = __shfl_sync(0xffffffffu, c, 0);
        if (c >= nchunk) break;
        const long c0 = ns + c * per;
        double2 v[CH];
#pragma unroll
        for (int u = 0; u < CH; ++u) {
            const long k = c0 + u * 32 + lane;
            v[u] = k < n2 ? __ldcg(p + k) : make_double2(0.0, 0.0);
        }
#pragma unroll
        for (int u = 0; u < CH; ++u) acc += v[u].x + v[u].y;
    }
    if (acc == 1.2345) *sink = acc;
}

// L2 eviction by READING another 512 MB: the timed kernel starts with clean lines (a write
// flush would leave ~126 MB of dirty lines whose write-back the timed kernel would pay for)
__global__ void k_flush(const double* f, long m, double* sink) {
    double acc = 0.0;
    for (long i = long(blockIdx.x) * blockDim.x + threadIdx.x; i < m; i += long(gridDim.x) * blockDim.x) acc += f[i];
    if (acc == 1.2345) *sink = acc;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long maxb = 2048L << 20;
    double2 *P, *Q;
    double *F, *sink;
    const long fm = 512L << 17;
    cudaMalloc(&P, maxb);
    cudaMalloc(&Q, maxb);
    cudaMalloc(&F, sizeof(double) * fm);
    cudaMalloc(&sink, 8);
    unsigned long long* ctr;
    cudaMalloc(&ctr, 64);
    cudaMemset(P, 0, maxb);
    cudaMemset(Q, 0, maxb);
    cudaMemset(F, 0, sizeof(double) * fm);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const long sizes_mb[] = {17, 64, 138, 185, 350, 520, 1024, 2048};
    for (long mb : sizes_mb) {
        const long n2 = (mb << 20) / 16;
        for (int kind = 0; kind < 5; ++kind) {
            for (int cpsm : {4, 8}) {
                float best = 1e9f;
                for (int rep = 0; rep < 5; ++rep) {
                    k_flush<<<sms * 4, 512>>>(F, fm, sink);
                    cudaMemsetAsync(ctr, 0, 64);
                    cudaEventRecord(a);
                    if (kind == 0) k_read<8><<<sms * cpsm, 256>>>(P, n2, sink);
                    else if (kind == 1) k_copy<4><<<sms * cpsm, 256>>>(P, Q, n2 / 2);
                    else if (kind == 2) k_read_dyn<8><<<sms * cpsm, 256>>>(P, n2, sink, ctr);
                    else k_read_tail<<<sms * cpsm, 256>>>(P, n2, sink, ctr, kind == 3 ? 0.75 : 0.9);
                    cudaEventRecord(b);
                    cudaEventSynchronize(b);
                    float t = 0.f;
                    cudaEventElapsedTime(&t, a, b);
                    if (t < best) best = t;
                }
                const double bytes = kind == 0 ? double(mb << 20) : double(mb << 20);   // copy: mb/2 read + mb/2 written
                printf("%-8s %5ld MB  ctas/SM %d  %9.1f us  %7.0f GB/s\n", kind == 0 ? "read" : (kind == 1 ? "copy" : (kind == 2 ? "read-dyn" : (kind == 3 ? "tail-25%" : "tail-10%"))), mb, cpsm, best * 1e3,
                       bytes / (best * 1e-3) / 1e9);
            }
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("status: %s\n", cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
