// l2_reuse_probe.cu — does a row-streaming kernel that runs its row ranges in the REVERSE
// temporal order of its predecessor hit the predecessor's lines in the 126 MB L2?
// (serpentine order of consecutive panel kernels.)
// Panel n x W doubles (column-major, the C2 panel: n = 2^21, W = 11 -> 185 MB).
//   K1  read  : every CTA streams its contiguous row range forward, sums all columns
//   K2  rw    : read W columns, write W-1 columns (TRSM-like), forward or reverse
//   K2' read  : read-only again (Gram-like), forward or reverse
// Each measurement: 512 MB flush, K1, then K2 timed with CUDA events.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/l2p tools/l2_reuse_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NT = 256;

template <int W, bool WRITE>
__global__ void __launch_bounds__(NT) k_stream(const double* __restrict__ P, double* __restrict__ Q, long n,
                                               int reverse, double* sink) {
    const long G = gridDim.x;
    const long r0 = (long(blockIdx.x) * (n / 2)) / G * 2, r1 = (long(blockIdx.x + 1) * (n / 2)) / G * 2;
    const long nchunk = (r1 - r0 + 2 * NT - 1) / (2 * NT);
    double acc = 0.0;
    for (long c = 0; c < nchunk; ++c) {
        const long cc = reverse ? nchunk - 1 - c : c;
        const long r = r0 + cc * 2 * NT + 2 * threadIdx.x;
        if (r >= r1) continue;
        double2 v[W];
#pragma unroll
        for (int k = 0; k < W; ++k) v[k] = *reinterpret_cast<const double2*>(P + long(k) * n + r);
        if (WRITE) {
#pragma unroll
            for (int k = 1; k < W; ++k) {
                double2 o;
                o.x = v[k].x * 0.5 + v[k - 1].x;
                o.y = v[k].y * 0.5 + v[k - 1].y;
                *reinterpret_cast<double2*>(Q + long(k) * n + r) = o;
            }
        } else {
#pragma unroll
            for (int k = 0; k < W; ++k) acc += v[k].x * v[k].y;
        }
    }
    if (!WRITE && acc == 12345.678) *sink = acc;
}

__global__ void k_flush(double* f, long m) {
    for (long i = long(blockIdx.x) * blockDim.x + threadIdx.x; i < m; i += long(gridDim.x) * blockDim.x) f[i] += 1.0;
}

int main() {
    constexpr int W = 11;
    const long n = 1L << 21;
    double *P, *F, *sink;
    const long fm = 512L << 17;   // 512 MB of doubles
    cudaMalloc(&P, sizeof(double) * n * W);
    cudaMalloc(&F, sizeof(double) * fm);
    cudaMalloc(&sink, 8);
    cudaMemset(P, 0, sizeof(double) * n * W);
    cudaMemset(F, 0, sizeof(double) * fm);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t a, b, c;
    cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&c);
    const double mb_r = 8.0 * n * W / 1e6, mb_w = 8.0 * n * (W - 1) / 1e6;
    for (int ctas : {4, 8}) {
        const int grid = sms * ctas;
        for (int pred = 0; pred < 3; ++pred) {      // 0: no predecessor (cold), 1: read fwd, 2: rw fwd
            for (int kind = 0; kind < 2; ++kind) {  // K2: 0 read-only, 1 read+write (in place)
                for (int rev = 0; rev < 2; ++rev) {
                    float best = 1e9f, t1 = 0.f;
                    for (int rep = 0; rep < 5; ++rep) {
                        k_flush<<<sms * 4, 512>>>(F, fm);
                        if (pred == 1) k_stream<W, false><<<grid, NT>>>(P, P, n, 0, sink);
                        if (pred == 2) k_stream<W, true><<<grid, NT>>>(P, P, n, 0, sink);
                        cudaEventRecord(a);
                        if (kind == 0) k_stream<W, false><<<grid, NT>>>(P, P, n, rev, sink);
                        else k_stream<W, true><<<grid, NT>>>(P, P, n, rev, sink);
                        cudaEventRecord(b);
                        cudaEventSynchronize(b);
                        float t = 0.f;
                        cudaEventElapsedTime(&t, a, b);
                        if (t < best) best = t;
                        t1 = t;
                    }
                    const double mb = mb_r + (kind ? mb_w : 0.0);
                    printf("ctas/SM %d  pred %-9s  K2 %-10s %-7s  %8.1f us  %7.0f GB/s (algorithmic)\n", ctas,
                           pred == 0 ? "none" : (pred == 1 ? "read-fwd" : "rw-fwd"), kind ? "read+write" : "read",
                           rev ? "reverse" : "forward", best * 1e3, mb / (best * 1e-3) / 1e3);
                    (void)t1;
                }
            }
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("status: %s\n", cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}
