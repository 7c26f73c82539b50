// caqr.cu — TSQR by CAQR (§V-E; Fig. 9 bottom right; Fig. 10 O(eps)).
//   "each GPU first computes the QR factorization of the local matrix, then the local
//    R-factors are gathered ..., and the final QR factorization is computed ...;
//    V^(d) := V^(d) Q^(d)"  with Q formed explicitly (P:245 fn 6).
// Single-GPU form: a TSQR reduction tree.  Level 0 cuts the n x w panel into blocks of B rows;
// one CTA computes the Householder QR of its block in shared memory and writes R_b (w x w).
// The stacked R's (nb*w x w) are factored by the same kernel, recursively, until one block
// remains (its R is the panel's R, signs normalised to diag(R) > 0, G19).  The explicit Q is
// then formed top-down: a block's Q is (its Householder Q) x (its w x w slice of the parent's
// Q); level 0 recomputes each block's QR from V (deterministic, same result), so the panel is
// read twice and written once, like CholQR, with no Householder vectors stored.
#include <cstdint>
#include <vector>

#include "kernels.h"

namespace kern {

namespace {
constexpr int NT = 256;
constexpr int NWARP = NT / 32;

// Block reduction of up to 32 values per thread -> out[0..cnt) (fixed order).
__device__ void block_sum(const double* vals, int cnt, double* sred /* NWARP*32 */, double* out) {
    const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
    for (int i = 0; i < cnt; ++i) {
        double x = vals[i];
        for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(0xffffffffu, x, off);
        if (lane == 0) sred[wp * 32 + i] = x;
    }
    __syncthreads();
    if (threadIdx.x < cnt) {
        double s = 0.0;
        for (int q = 0; q < NWARP; ++q) s += sred[q * 32 + threadIdx.x];
        out[threadIdx.x] = s;
    }
    __syncthreads();
}

// Householder QR of the rows x w block A (smem, column-major, ld = rows <= NT, one row per
// thread).  On exit A's upper triangle holds R (diag not sign-normalised), the reflectors
// v_k (v_k[k] = 1 implicit) are below the diagonal and tau[k] the scalars.
__device__ void block_householder(double* A, int rows, int w, double* tau, double* sred, double* tmp) {
    const int r = threadIdx.x;
    for (int k = 0; k < w && k < rows; ++k) {
        // norm of A[k:, k]
        double x2[1] = {(r >= k && r < rows) ? A[r + rows * k] * A[r + rows * k] : 0.0};
        block_sum(x2, 1, sred, tmp);
        const double akk = A[k + rows * k];
        const double nrm = sqrt(tmp[0]);
        double beta = 0.0, t = 0.0, scale = 0.0;
        if (nrm > 0.0) {
            beta = akk >= 0.0 ? -nrm : nrm;          // A[k,k] -> beta
            t = (beta - akk) / beta;
            scale = 1.0 / (akk - beta);
        }
        __syncthreads();
        if (r > k && r < rows) A[r + rows * k] *= scale;   // v below the diagonal
        __syncthreads();
        if (r == k) { A[k + rows * k] = nrm > 0.0 ? beta : akk; tau[k] = t; }
        // apply H = I - t v v^T to A[k:, k+1:]: w_c = v^T A[:, c]
        double dots[32];
        const double vk = (r == k) ? 1.0 : ((r > k && r < rows) ? A[r + rows * k] : 0.0);
        int cnt = 0;
        for (int c = k + 1; c < w; ++c) dots[cnt++] = (r >= k && r < rows) ? vk * A[r + rows * c] : 0.0;
        __syncthreads();
        block_sum(dots, cnt, sred, tmp);
        if (r >= k && r < rows)
            for (int c = k + 1; c < w; ++c) A[r + rows * c] -= t * vk * tmp[c - k - 1];
        __syncthreads();
    }
}

// Q (rows x w, explicit, first w columns of H_0 ... H_{w-1}) from the reflectors in A.
__device__ void block_formq(const double* A, int rows, int w, const double* tau, double* Q, double* sred,
                            double* tmp) {
    const int r = threadIdx.x;
    if (r < rows)
        for (int c = 0; c < w; ++c) Q[r + rows * c] = (r == c) ? 1.0 : 0.0;
    __syncthreads();
    for (int k = min(w, rows) - 1; k >= 0; --k) {
        const double vk = (r == k) ? 1.0 : ((r > k && r < rows) ? A[r + rows * k] : 0.0);
        double dots[32];
        for (int c = 0; c < w; ++c) dots[c] = (r >= k && r < rows) ? vk * Q[r + rows * c] : 0.0;
        block_sum(dots, w, sred, tmp);
        if (r >= k && r < rows)
            for (int c = 0; c < w; ++c) Q[r + rows * c] -= tau[k] * vk * tmp[c];
        __syncthreads();
    }
}

struct CaqrArgs {
    int64_t n;                 // rows of this level's input
    const double* in; int64_t ldin;   // input (n x w)
    int w;
    int B;                     // rows per block (multiple of w at levels > 0)
    double* Rout;              // nb*w x w stacked R's (ld nb*w) — level output
    int64_t ldr;
    // pass 2
    const double* Qpar;        // parent explicit Q (nb*w x w), ld ldq
    int64_t ldq;
    double* out; int64_t ldout;// level output Q rows (n x w)
    int c0;                    // first output column written (level 0 in-place: skip q_j)
};

template <int PASS>
__global__ void __launch_bounds__(NT) k_caqr(CaqrArgs a) {
    extern __shared__ double sm[];
    const int w = a.w, B = a.B;
    double* A = sm;                         // B x w
    double* Q = A + B * w;                  // B x w
    double* sred = Q + B * w;               // NWARP x 32
    double* tmp = sred + NWARP * 32;        // 32
    double* tau = tmp + 32;                 // 32
    const int64_t b = blockIdx.x;
    const int64_t r0 = b * B;
    const int rows = int(min(int64_t(B), a.n - r0));
    const int r = threadIdx.x;
    for (int c = 0; c < w; ++c) A[r + B * c] = (r < rows) ? a.in[r0 + r + a.ldin * c] : 0.0;
    __syncthreads();
    block_householder(A, B, w, tau, sred, tmp);   // zero-padded rows keep the block's R exact
    if (PASS == 0) {
        if (r < w)
            for (int c = 0; c < w; ++c)
                a.Rout[b * w + r + a.ldr * c] = (c >= r) ? A[r + B * c] : 0.0;
        return;
    }
    block_formq(A, B, w, tau, Q, sred, tmp);
    // out rows = Q_b (rows x w) * Qpar[b*w : b*w + w, :]
    if (r < rows) {
        double q[32];
        for (int k = 0; k < w; ++k) q[k] = Q[r + B * k];
        for (int c = a.c0; c < w; ++c) {
            double s = 0.0;
            for (int k = 0; k < w; ++k) s = fma(q[k], a.Qpar[b * w + k + a.ldq * c], s);
            a.out[r0 + r + a.ldout * c] = s;
        }
    }
}

// final block: QR of the top (rows <= B) matrix, sign-normalised R and explicit Q
__global__ void __launch_bounds__(NT) k_caqr_top(const double* in, int64_t ld, int rows, int w, double* R,
                                               double* Qout /* rows x w, ld rows */, int B) {
    extern __shared__ double sm[];
    double* A = sm;
    double* Q = A + B * w;
    double* sred = Q + B * w;
    double* tmp = sred + NWARP * 32;
    double* tau = tmp + 32;
    const int r = threadIdx.x;
    for (int c = 0; c < w; ++c) A[r + B * c] = (r < rows) ? in[r + ld * c] : 0.0;
    __syncthreads();
    block_householder(A, B, w, tau, sred, tmp);
    block_formq(A, B, w, tau, Q, sred, tmp);
    // D = sign(diag R): R <- D R, Q <- Q D
    if (r < rows)
        for (int c = 0; c < w; ++c) {
            const double dc = A[c + B * c] < 0.0 ? -1.0 : 1.0;
            Qout[r + int64_t(rows) * c] = Q[r + B * c] * dc;
        }
    if (r < w) {
        const double dr = A[r + B * r] < 0.0 ? -1.0 : 1.0;
        for (int c = 0; c < w; ++c) R[r + int64_t(w) * c] = (c >= r) ? dr * A[r + B * c] : 0.0;
    }
}

size_t smem_for(int B, int w) { return sizeof(double) * (size_t(2) * B * w + NWARP * 32 + 64); }
}  // namespace

// Workspace: caqr_ws_doubles(n, w) doubles.  R: w x w (ld w).  P overwritten by Q (cols >= c0).
size_t caqr_ws_doubles(int64_t n, int w) {
    size_t tot = 0;
    int64_t rows = n;
    const int B = NT;
    while (rows > B) {
        const int64_t nb = (rows + B - 1) / B;
        tot += size_t(nb) * w * w * 2;      // stacked R + its explicit Q
        rows = nb * w;
    }
    return tot + size_t(B) * w + 64;
}

int caqr(const Dev& d, int64_t n, double* P, int64_t ldp, int w, double* R, int c0, double* ws,
         cudaStream_t st) {
    (void)d;
    if (w < 1 || w > 32 || n < w) return -1;
    const int B = NT;
    const size_t smem = smem_for(B, w);
    if (smem > 48 * 1024) {
        cudaFuncSetAttribute(k_caqr<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        cudaFuncSetAttribute(k_caqr<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        cudaFuncSetAttribute(k_caqr_top, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    }
    // ---- up-sweep: levels of stacked R's ----
    struct Lvl { int64_t rows; const double* in; int64_t ldin; double* Rs; int64_t nb; double* Qs; };
    std::vector<Lvl> lv;
    int64_t rows = n;
    const double* in = P;
    int64_t ldin = ldp;
    double* cur = ws;
    while (rows > B) {
        const int64_t nb = (rows + B - 1) / B;
        Lvl L{rows, in, ldin, cur, nb, cur + nb * w * w};
        cur += size_t(nb) * w * w * 2;
        CaqrArgs a{rows, in, ldin, w, B, L.Rs, nb * w, nullptr, 0, nullptr, 0, 0};
        ++g_launches;
        k_caqr<0><<<unsigned(nb), NT, smem, st>>>(a);
        lv.push_back(L);
        in = L.Rs; ldin = nb * w; rows = nb * w;
    }
    // ---- top ----
    double* Qtop = cur;
    ++g_launches;
    k_caqr_top<<<1, NT, smem, st>>>(in, ldin, int(rows), w, R, Qtop, B);
    // ---- down-sweep: explicit Q of each level ----
    const double* Qpar = Qtop;
    int64_t ldq = rows;
    for (int i = int(lv.size()) - 1; i >= 0; --i) {
        const Lvl& L = lv[size_t(i)];
        double* out = i == 0 ? P : lv[size_t(i) - 1].Qs;          // level i-1's R stack -> its Q stack
        const int64_t ldout = i == 0 ? ldp : lv[size_t(i) - 1].nb * w;
        CaqrArgs a{L.rows, L.in, L.ldin, w, B, nullptr, 0, Qpar, ldq, out, ldout, i == 0 ? c0 : 0};
        ++g_launches;
        k_caqr<1><<<unsigned(L.nb), NT, smem, st>>>(a);
        Qpar = out;
        ldq = ldout;
    }
    if (lv.empty()) {                     // n <= B: the top block is the whole panel
        for (int c = c0; c < w; ++c)
            cudaMemcpyAsync(P + ldp * c, Qtop + rows * c, sizeof(double) * size_t(rows), cudaMemcpyDeviceToDevice, st);
    }
    return 0;
}

}  // namespace kern
