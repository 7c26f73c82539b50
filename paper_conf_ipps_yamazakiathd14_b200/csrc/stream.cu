// stream.cu — row-streaming panel kernels fed by a TMA bulk-copy ring (sm_100a).
//   K9  update : P[:, 0:w] -= X C            (BOrth pass 2; x += V y)
//   K8  trsm   : P[:, c0:w] = (P R^{-1})[:, c0:w]   (CholQR/SVQR update)
// One persistent CTA per SM streams full row tiles of all input columns into a 4-stage
// shared-memory ring (cp.async.bulk + mbarrier), so the loads in flight do not consume
// registers; each thread then finishes its rows from shared memory and writes the result
// straight to global memory (coalesced, one pass).  C / R live in shared memory and are
// read as warp-wide broadcasts.  Ragged tails and unaligned panels use plain loads.
#include <cstdint>

#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int ST = 4;
constexpr int STAGE_BYTES = 32 * 1024;

struct StreamArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;     // update only
    double* P; int64_t ldp; int w;
    const double* M;                          // C (jx x w, ld jx) or R (w x w, ld w)
    int c0;                                   // trsm: first column written
    int TS;
};

template <int WM>
__device__ __forceinline__ void update_row(const StreamArgs& a, const double* Xs, int64_t ldX, const double* Ps,
                                           int64_t ldP, int r, const double* sC, double* out, int64_t ldo) {
    double acc[WM];
#pragma unroll
    for (int c = 0; c < WM; ++c) acc[c] = (c < a.w) ? Ps[r + ldP * c] : 0.0;
#pragma unroll 4
    for (int i = 0; i < a.jx; ++i) {
        const double x = Xs[r + ldX * i];
#pragma unroll
        for (int c = 0; c < WM; ++c) acc[c] = fma(-x, sC[i * WM + c], acc[c]);
    }
#pragma unroll
    for (int c = 0; c < WM; ++c)
        if (c < a.w) out[r + ldo * c] = acc[c];
}

template <int WM>
__device__ __forceinline__ void trsm_row(const StreamArgs& a, const double* Ps, int64_t ldP, int r,
                                         const double* sR, const double* sInv, double* out, int64_t ldo) {
    double p[WM];
#pragma unroll
    for (int c = 0; c < WM; ++c) p[c] = (c < a.w) ? Ps[r + ldP * c] : 0.0;
#pragma unroll
    for (int c = 0; c < WM; ++c) {
        double x = p[c];
#pragma unroll
        for (int k = 0; k < c; ++k) x = fma(-p[k], sR[k * WM + c], x);
        p[c] = x * sInv[c];
    }
#pragma unroll
    for (int c = 0; c < WM; ++c)
        if (c >= a.c0 && c < a.w) out[r + ldo * c] = p[c];
}

// MODE 0: update, MODE 1: trsm
template <int MODE, int WM>
__global__ void __launch_bounds__(NT, 1) k_stream(StreamArgs a) {
    extern __shared__ __align__(128) unsigned char smraw[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smraw);
    const int jxl = MODE == 0 ? a.jx : 0;
    double* sM = reinterpret_cast<double*>(smraw + 128);          // C: jx*WM  |  R: WM*WM + WM
    const int nM = MODE == 0 ? jxl * WM : WM * WM + WM;
    double* slots = sM + ((nM + 15) / 16) * 16;
    const int tid = threadIdx.x, TS = a.TS, w = a.w;
    const int ncol = jxl + w;                                     // X columns then P columns
    const int64_t slot_d = int64_t(ncol) * TS;
    const int64_t ntiles = a.n / TS;
    const int64_t my_tiles = ntiles > int64_t(blockIdx.x) ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    if (MODE == 0) {
        for (int e = tid; e < jxl * WM; e += NT) {
            const int i = e / WM, c = e - i * WM;
            sM[e] = (c < w) ? a.M[i + int64_t(jxl) * c] : 0.0;
        }
    } else {
        for (int e = tid; e < WM * WM; e += NT) {
            const int k = e / WM, c = e - k * WM;
            sM[e] = (k < w && c < w) ? a.M[k + int64_t(w) * c] : 0.0;
        }
        for (int c = tid; c < WM; c += NT) sM[WM * WM + c] = (c < w) ? 1.0 / a.M[c + int64_t(w) * c] : 0.0;
    }
    if (tid == 0) {
        for (int s = 0; s < ST; ++s) ptx::mbar_init(&bars[s], 1);
        ptx::fence_mbar_init();
    }
    __syncthreads();
    const uint32_t colbytes = uint32_t(TS) * 8u;
    auto issue = [&](int64_t k) {
        const int s = int(k % ST);
        const int64_t r0 = (int64_t(blockIdx.x) + k * gridDim.x) * TS;
        double* dst = slots + s * slot_d;
        ptx::fence_proxy_async();
        ptx::mbar_arrive_expect_tx(&bars[s], colbytes * uint32_t(ncol));
        for (int c = 0; c < jxl; ++c) ptx::bulk_g2s(dst + int64_t(c) * TS, a.X + a.ldx * c + r0, colbytes, &bars[s]);
        for (int c = 0; c < w; ++c)
            ptx::bulk_g2s(dst + int64_t(jxl + c) * TS, a.P + a.ldp * c + r0, colbytes, &bars[s]);
    };
    if (tid == 0)
        for (int64_t k = 0; k < my_tiles && k < ST; ++k) issue(k);
    for (int64_t k = 0; k < my_tiles; ++k) {
        const int s = int(k % ST);
        ptx::mbar_wait(&bars[s], uint32_t((k / ST) & 1));
        const double* Xs = slots + s * slot_d;
        const double* Ps = Xs + int64_t(jxl) * TS;
        double* out = a.P + (int64_t(blockIdx.x) + k * gridDim.x) * TS;
#pragma unroll 1
        for (int r = tid; r < TS; r += NT) {
            if (MODE == 0) update_row<WM>(a, Xs, TS, Ps, TS, r, sM, out, a.ldp);
            else trsm_row<WM>(a, Ps, TS, r, sM, sM + WM * WM, out, a.ldp);
        }
        __syncthreads();
        if (tid == 0 && k + ST < my_tiles) issue(k + ST);
    }
    if (blockIdx.x == 0 && ntiles * TS < a.n) {                  // ragged tail, plain loads
        const int64_t r0 = ntiles * TS;
        const int rows = int(a.n - r0);
        double* base = a.P + r0;
        for (int r = tid; r < rows; r += NT) {
            if (MODE == 0) update_row<WM>(a, a.X + r0, a.ldx, base, a.ldp, r, sM, base, a.ldp);
            else trsm_row<WM>(a, base, a.ldp, r, sM, sM + WM * WM, base, a.ldp);
        }
    }
}

// ---- fallback kernels (unaligned user panels): one row per thread, plain loads ----------
template <int MODE, int WM>
__global__ void __launch_bounds__(NT) k_rowwise(StreamArgs a) {
    extern __shared__ double sM[];
    const int w = a.w;
    if (MODE == 0) {
        for (int e = threadIdx.x; e < a.jx * WM; e += NT) {
            const int i = e / WM, c = e - i * WM;
            sM[e] = (c < w) ? a.M[i + int64_t(a.jx) * c] : 0.0;
        }
    } else {
        for (int e = threadIdx.x; e < WM * WM; e += NT) {
            const int k = e / WM, c = e - k * WM;
            sM[e] = (k < w && c < w) ? a.M[k + int64_t(w) * c] : 0.0;
        }
        for (int c = threadIdx.x; c < WM; c += NT) sM[WM * WM + c] = (c < w) ? 1.0 / a.M[c + int64_t(w) * c] : 0.0;
    }
    __syncthreads();
    for (int64_t r0 = int64_t(blockIdx.x) * NT; r0 < a.n; r0 += int64_t(gridDim.x) * NT) {
        const int r = threadIdx.x;
        if (r0 + r >= a.n) break;
        if (MODE == 0) update_row<WM>(a, a.X + r0, a.ldx, a.P + r0, a.ldp, r, sM, a.P + r0, a.ldp);
        else trsm_row<WM>(a, a.P + r0, a.ldp, r, sM, sM + WM * WM, a.P + r0, a.ldp);
    }
}

template <int MODE, int WM>
void run(const Dev& d, StreamArgs a, bool aligned, cudaStream_t st) {
    const int nM = MODE == 0 ? a.jx * WM : WM * WM + WM;
    const int ncol = (MODE == 0 ? a.jx : 0) + a.w;
    if (aligned) {
        int TS = 4096;
        while (TS > 32 && TS * ncol * 8 > STAGE_BYTES) TS /= 2;
        a.TS = TS;
        const int64_t tiles = a.n / TS;
        int64_t g = d.sms;
        if (g > tiles) g = tiles;
        if (g < 1) g = 1;
        const size_t smem = 128 + size_t((nM + 15) / 16) * 16 * 8 + size_t(ST) * ncol * TS * 8;
        cudaFuncSetAttribute(k_stream<MODE, WM>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        k_stream<MODE, WM><<<unsigned(g), NT, smem, st>>>(a);
    } else {
        int64_t g = (a.n + NT - 1) / NT;
        if (g > int64_t(d.sms) * 8) g = int64_t(d.sms) * 8;
        if (g < 1) g = 1;
        const size_t smem = size_t(nM) * 8;
        cudaFuncSetAttribute(k_rowwise<MODE, WM>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        ++g_launches;
        k_rowwise<MODE, WM><<<unsigned(g), NT, smem, st>>>(a);
    }
}

template <int MODE>
void dispatch(const Dev& d, const StreamArgs& a, bool al, cudaStream_t st) {
    const int w = a.w;
    if (w <= 1) run<MODE, 1>(d, a, al, st);
    else if (w <= 2) run<MODE, 2>(d, a, al, st);
    else if (w <= 4) run<MODE, 4>(d, a, al, st);
    else if (w <= 8) run<MODE, 8>(d, a, al, st);
    else if (w <= 12) run<MODE, 12>(d, a, al, st);
    else if (w <= 16) run<MODE, 16>(d, a, al, st);
    else run<MODE, 32>(d, a, al, st);
}

bool al16(const void* p, int64_t ld) { return (reinterpret_cast<uintptr_t>(p) % 16 == 0) && (ld % 2 == 0); }
}  // namespace

void update(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* P,
            int64_t ldp, int w, const double* C, cudaStream_t st) {
    if (jx <= 0 || n <= 0 || w <= 0) return;
    StreamArgs a{n, X, ldx, jx, P, ldp, w, C, 0, 0};
    dispatch<0>(d, a, al16(X, ldx) && al16(P, ldp) && (jx + w) * 32 * 8 <= STAGE_BYTES, st);
}

void trsm(const Dev& d, int64_t n, double* P, int64_t ldp, int w, const double* R, int c0,
          cudaStream_t st) {
    if (n <= 0 || w <= 0) return;
    StreamArgs a{n, nullptr, 0, 0, P, ldp, w, R, c0, 0};
    dispatch<1>(d, a, al16(P, ldp), st);
}

}  // namespace kern
