// stream.cu — row-streaming panel kernels fed by a TMA bulk-copy ring (sm_100a, FP64 DMMA).
//   K9  update : P[:, 0:w] -= X C                 (BOrth pass 2; x += V y)
//   K8  trsm   : P[:, c0:w] = (P R^{-1})[:, c0:w] (CholQR/SVQR update)
// One persistent CTA per SM streams full row tiles of all input columns into a 4-stage
// shared-memory ring (cp.async.bulk + mbarrier), so the loads in flight do not consume
// registers.  Each warp then takes 8-row groups of the tile and forms the 8-row x w output
// with mma.sync.m8n8k4.f64 against the small right-hand matrix (C, or R^{-1}), whose
// B-fragments live in registers for the whole kernel, and writes the rows straight back to
// global memory (one pass: read X and P once, write P once).
// TRSM uses the explicit inverse of the w x w triangular factor, formed once per CTA in
// shared memory by column back-substitution (what blocked GPU TRSMs do for their diagonal
// blocks); the product with P then runs on the tensor core like the update.
// Ragged tails use zero-padded fragment loads; unaligned user panels use k_rowwise.
#include <cstdint>

#include "kernels.h"
#include "ptx.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NWARP = NT / 32;
constexpr int ST = 4;
constexpr int STAGE_BYTES = 32 * 1024;

struct StreamArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;     // update: X (n x jx); trsm: unused (A = P)
    double* P; int64_t ldp; int w;
    const double* M;                          // C (jx x w, ld jx) or R (w x w, ld w)
    int c0;                                   // trsm: first column written
    int TS;
};

// R^{-1} (upper, w x w) into sRi[k*32 + c]; one thread per column (back substitution)
__device__ __forceinline__ void upper_inverse(const double* R, int w, double* sRi, double* sInv) {
    for (int k = threadIdx.x; k < 32; k += NT) sInv[k] = k < w ? 1.0 / R[k + int64_t(w) * k] : 0.0;
    __syncthreads();
    for (int c = threadIdx.x; c < 32; c += NT) {
        for (int k = 0; k < 32; ++k) sRi[k * 32 + c] = 0.0;
        if (c >= w) continue;
        sRi[c * 32 + c] = sInv[c];
        for (int k = c - 1; k >= 0; --k) {
            double s = 0.0;
            for (int l = k + 1; l <= c; ++l) s = fma(R[k + int64_t(w) * l], sRi[l * 32 + c], s);
            sRi[k * 32 + c] = -s * sInv[k];
        }
    }
}

// one 8-row group: D(8 x 8*NTN) = sign * A(8 x K) B(K x 8*NTN) [+ P], then store
template <int MODE, int KTM, int NTN>
__device__ __forceinline__ void group8(const StreamArgs& a, const double* As, int64_t ldA, const double* Ps,
                                       int64_t ldP, int64_t row, bool valid, const double (&b)[KTM][NTN],
                                       int KT, double* outrow_base, int64_t ldo, int lane) {
    const int gid = lane >> 2, tig = lane & 3;
    const int w = a.w;
    double d[NTN][2];
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = min(8 * nt + 2 * tig + h, w - 1);
            d[nt][h] = (MODE == 0 && valid) ? Ps[row + ldP * c] : 0.0;
        }
    }
    const int kmax = MODE == 0 ? a.jx : w;
    (void)gid;
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt) {
        if (kt < KT) {
            const int c = min(4 * kt + tig, kmax - 1);
            // A fragment: A[m = gid][k = tig] = rows of this group, columns 4kt..4kt+3
            const double av = valid ? As[(row - (lane >> 2) + gid) + ldA * c] : 0.0;
            const double am = MODE == 0 ? -av : av;
#pragma unroll
            for (int nt = 0; nt < NTN; ++nt) ptx::dmma(d[nt][0], d[nt][1], am, b[kt][nt]);
        }
    }
#pragma unroll
    for (int nt = 0; nt < NTN; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = 8 * nt + 2 * tig + h;
            if (valid && c < w && (MODE == 0 || c >= a.c0)) outrow_base[row + ldo * c] = d[nt][h];
        }
}

// MODE 0: update (A = X, B = C, D init = P, subtract); MODE 1: trsm (A = P, B = R^{-1}).
template <int MODE, int KTM, int NTN>
__global__ void __launch_bounds__(NT, 1) k_stream_mma(StreamArgs a) {
    extern __shared__ __align__(128) unsigned char smraw[];
    uint64_t* bars = reinterpret_cast<uint64_t*>(smraw);
    double* sB = reinterpret_cast<double*>(smraw + 128);        // 32 x 32 (R^{-1}) or unused
    double* sInv = sB + 32 * 32;                                  // 32 (1 / R_kk)
    double* slots = sInv + 32;
    const int tid = threadIdx.x, lane = tid & 31, wp = tid >> 5;
    const int gid = lane >> 2, tig = lane & 3;
    const int TS = a.TS, SP = TS + 4, w = a.w;
    const int jxl = MODE == 0 ? a.jx : 0;
    const int ncol = jxl + w;                                     // X columns then P columns
    const int64_t slot_d = int64_t(ncol) * SP;
    const int64_t ntiles = a.n / TS;
    const int64_t my_tiles = ntiles > int64_t(blockIdx.x) ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    const int KT = ((MODE == 0 ? a.jx : w) + 3) / 4;

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
        for (int c = 0; c < jxl; ++c) ptx::bulk_g2s(dst + int64_t(c) * SP, a.X + a.ldx * c + r0, colbytes, &bars[s]);
        for (int c = 0; c < w; ++c)
            ptx::bulk_g2s(dst + int64_t(jxl + c) * SP, a.P + a.ldp * c + r0, colbytes, &bars[s]);
    };
    if (tid == 0)
        for (int64_t k = 0; k < my_tiles && k < ST; ++k) issue(k);     // loads overlap the prologue
    // ---- B fragments (registers): b[kt][nt] = B[4kt + tig][8nt + gid] ----
    if (MODE == 1) {
        upper_inverse(a.M, w, sB, sInv);
        __syncthreads();
    }
    double b[KTM][NTN];
#pragma unroll
    for (int kt = 0; kt < KTM; ++kt)
#pragma unroll
        for (int nt = 0; nt < NTN; ++nt) {
            const int k = 4 * kt + tig, c = 8 * nt + gid;
            double v = 0.0;
            if (MODE == 0) {
                if (k < a.jx && c < w) v = a.M[k + int64_t(a.jx) * c];
            } else {
                if (k < w && c < w) v = sB[k * 32 + c];
            }
            b[kt][nt] = v;
        }
    for (int64_t k = 0; k < my_tiles; ++k) {
        const int s = int(k % ST);
        ptx::mbar_wait(&bars[s], uint32_t((k / ST) & 1));
        const double* Xs = slots + s * slot_d;
        const double* Ps = Xs + int64_t(jxl) * SP;
        const double* As = MODE == 0 ? Xs : Ps;
        double* out = a.P + (int64_t(blockIdx.x) + k * gridDim.x) * TS;
#pragma unroll 1
        for (int g8 = wp; g8 < TS / 8; g8 += NWARP)
            group8<MODE, KTM, NTN>(a, As, SP, Ps, SP, 8 * g8 + gid, true, b, KT, out, a.ldp, lane);
        __syncthreads();
        if (tid == 0 && k + ST < my_tiles) issue(k + ST);
    }
    if (blockIdx.x == 0 && ntiles * TS < a.n) {                  // ragged tail, zero padded
        const int64_t r0 = ntiles * TS;
        const int rows = int(a.n - r0);
        double* base = a.P + r0;
        const double* Ab = MODE == 0 ? a.X + r0 : base;
        const int64_t ldA = MODE == 0 ? a.ldx : a.ldp;
        for (int g8 = wp; 8 * g8 < rows; g8 += NWARP) {
            const int64_t row = 8 * g8 + gid;
            group8<MODE, KTM, NTN>(a, Ab, ldA, base, a.ldp, row, row < rows, b, KT, base, a.ldp, lane);
        }
    }
}

// ---- fallback kernels (unaligned user panels / very wide X): one row per thread ---------
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
    for (int64_t r = int64_t(blockIdx.x) * NT + threadIdx.x; r < a.n; r += int64_t(gridDim.x) * NT) {
        if (MODE == 0) {
            double acc[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) acc[c] = (c < w) ? a.P[r + a.ldp * c] : 0.0;
            for (int i = 0; i < a.jx; ++i) {
                const double x = a.X[r + a.ldx * i];
#pragma unroll
                for (int c = 0; c < WM; ++c) acc[c] = fma(-x, sM[i * WM + c], acc[c]);
            }
#pragma unroll
            for (int c = 0; c < WM; ++c)
                if (c < w) a.P[r + a.ldp * c] = acc[c];
        } else {
            double p[WM];
#pragma unroll
            for (int c = 0; c < WM; ++c) p[c] = (c < w) ? a.P[r + a.ldp * c] : 0.0;
#pragma unroll
            for (int c = 0; c < WM; ++c) {
                double x = p[c];
#pragma unroll
                for (int k = 0; k < c; ++k) x = fma(-p[k], sM[k * WM + c], x);
                p[c] = x * sM[WM * WM + c];
            }
#pragma unroll
            for (int c = 0; c < WM; ++c)
                if (c >= a.c0 && c < w) a.P[r + a.ldp * c] = p[c];
        }
    }
}

template <int MODE, int WM>
void run_rowwise(const Dev& d, const StreamArgs& a, cudaStream_t st) {
    const int nM = MODE == 0 ? a.jx * WM : WM * WM + WM;
    int64_t g = (a.n + NT - 1) / NT;
    if (g > int64_t(d.sms) * 8) g = int64_t(d.sms) * 8;
    if (g < 1) g = 1;
    const size_t smem = size_t(nM) * 8;
    cudaFuncSetAttribute(k_rowwise<MODE, WM>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    k_rowwise<MODE, WM><<<unsigned(g), NT, smem, st>>>(a);
}

template <int MODE, int KTM, int NTN>
void run_mma(const Dev& d, StreamArgs a, cudaStream_t st) {
    const int ncol = (MODE == 0 ? a.jx : 0) + a.w;
    int TS = 4096;
    while (TS > 64 && int64_t(TS + 4) * ncol * 8 > STAGE_BYTES) TS /= 2;
    a.TS = TS;
    const int64_t tiles = a.n / TS;
    int64_t g = d.sms;
    if (g > tiles) g = tiles;
    if (g < 1) g = 1;
    const size_t smem = 128 + 33 * 32 * 8 + size_t(ST) * ncol * (TS + 4) * 8;
    cudaFuncSetAttribute(k_stream_mma<MODE, KTM, NTN>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    ++g_launches;
    k_stream_mma<MODE, KTM, NTN><<<unsigned(g), NT, smem, st>>>(a);
}

template <int MODE>
void dispatch(const Dev& d, const StreamArgs& a, bool al, cudaStream_t st) {
    const int w = a.w, K = MODE == 0 ? a.jx : w;
    const int ncol = (MODE == 0 ? a.jx : 0) + w;
    if (al && K <= 64 && w <= 32 && int64_t(68) * ncol * 8 <= STAGE_BYTES) {
        const int ntn = w <= 8 ? 1 : (w <= 16 ? 2 : 4);
        const int ktm = K <= 4 ? 1 : (K <= 8 ? 2 : (K <= 16 ? 4 : (K <= 32 ? 8 : 16)));
        switch (ktm * 10 + ntn) {
            case 11: run_mma<MODE, 1, 1>(d, a, st); return;
            case 21: run_mma<MODE, 2, 1>(d, a, st); return;
            case 41: run_mma<MODE, 4, 1>(d, a, st); return;
            case 81: run_mma<MODE, 8, 1>(d, a, st); return;
            case 161: run_mma<MODE, 16, 1>(d, a, st); return;
            case 12: run_mma<MODE, 1, 2>(d, a, st); return;
            case 22: run_mma<MODE, 2, 2>(d, a, st); return;
            case 42: run_mma<MODE, 4, 2>(d, a, st); return;
            case 82: run_mma<MODE, 8, 2>(d, a, st); return;
            case 162: run_mma<MODE, 16, 2>(d, a, st); return;
            case 14: run_mma<MODE, 1, 4>(d, a, st); return;
            case 24: run_mma<MODE, 2, 4>(d, a, st); return;
            case 44: run_mma<MODE, 4, 4>(d, a, st); return;
            case 84: run_mma<MODE, 8, 4>(d, a, st); return;
            default: break;                                       // K > 32 with w > 16: fallback
        }
    }
    if (w <= 1) run_rowwise<MODE, 1>(d, a, st);
    else if (w <= 2) run_rowwise<MODE, 2>(d, a, st);
    else if (w <= 4) run_rowwise<MODE, 4>(d, a, st);
    else if (w <= 8) run_rowwise<MODE, 8>(d, a, st);
    else if (w <= 12) run_rowwise<MODE, 12>(d, a, st);
    else if (w <= 16) run_rowwise<MODE, 16>(d, a, st);
    else run_rowwise<MODE, 32>(d, a, st);
}

bool al16(const void* p, int64_t ld) { return (reinterpret_cast<uintptr_t>(p) % 16 == 0) && (ld % 2 == 0); }
}  // namespace

void update(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* P,
            int64_t ldp, int w, const double* C, cudaStream_t st) {
    if (jx <= 0 || n <= 0 || w <= 0) return;
    StreamArgs a{n, X, ldx, jx, P, ldp, w, C, 0, 0};
    dispatch<0>(d, a, al16(X, ldx) && al16(P, ldp), st);
}

void trsm(const Dev& d, int64_t n, double* P, int64_t ldp, int w, const double* R, int c0,
          cudaStream_t st) {
    if (n <= 0 || w <= 0) return;
    StreamArgs a{n, nullptr, 0, 0, P, ldp, w, R, c0, 0};
    dispatch<1>(d, a, al16(P, ldp), st);
}

}  // namespace kern
