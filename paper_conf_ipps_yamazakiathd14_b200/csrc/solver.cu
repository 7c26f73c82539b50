// solver.cu — the CA-GMRES(s, m) handle: setup, MPK / BOrth / TSQR drivers, NCCL halo and
// allreduces, and the restart loop of cagmres_solve (§III-§V).
//
// Data layout in HBM:
//   V   : ldv x (m+1) column-major, ldv = round_up(n_ext, 32).  Rows [0, n_loc) of column k
//         hold the k-th basis vector's owned rows; rows [n_loc, n_ext) are the MPK ghost
//         scratch of that column (P:66 z^(d,k)), so the matrix powers kernel writes its
//         outputs straight into the basis — no expand/copy step (P:66, P:132 fn 4).
//   A   : extended rows in SELL-32 (kern::Sell), columns in extended local ids.
//   tab : per-cycle device table of the BOrth coefficients C and TSQR factors R of every
//         block (and of the reorthogonalisation pass); copied to the host once per cycle
//         for the Hessenberg update and the least-squares solve.
#include <algorithm>
#include <chrono>
#include <climits>
#include <cmath>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include <memory>

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "internal.h"
#include "kernels.h"
#include "transport.h"

#define CU(x)                                                       \
    do {                                                            \
        cudaError_t e_ = (x);                                       \
        if (e_ != cudaSuccess) { return CAGMRES_ECUDA; }            \
    } while (0)
#define TRY(x)                                                      \
    do {                                                            \
        int s_ = (x);                                               \
        if (s_ < 0) return s_;                                      \
    } while (0)

namespace {

enum Phase { PH_MPK = 0, PH_BORTH = 1, PH_TSQR = 2, PH_OTHER = 3, PH_SPMV = 4, PH_N = 5 };

struct Timer {
    bool on = false;
    bool light = false;                    // record only the dominant (MPK) kernel launches
    std::vector<cudaEvent_t> pool;
    size_t used = 0;
    std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> rec;
    cudaEvent_t get() {
        if (used == pool.size()) {
            cudaEvent_t e;
            cudaEventCreate(&e);
            pool.push_back(e);
        }
        return pool[used++];
    }
    void reset() { used = 0; rec.clear(); }
    ~Timer() { for (auto e : pool) cudaEventDestroy(e); }
};

struct Block { int j, sb; size_t c1, r1, c2, r2; };

}  // namespace

struct cagmres {
    int s = 1, m = 1, basis = CAGMRES_NEWTON, orth = CAGMRES_CHOLQR;
    int64_t n = 0, n_loc = 0, n_ext = 0, ldv = 0;
    int rank = 0, nranks = 1;
    std::unique_ptr<Transport> tr;         // NCCL or in-process group (transport.h); null on 1 rank
    kern::Dev dev;
    cudaStream_t stream = nullptr, own_stream = nullptr;
    kern::Sell A;
    double spmv_tuned_us = 0.0;            // setup-time SpMV autotune result (diagnostic)
    std::vector<int64_t> level_len;        // ext rows with distance <= h
    std::vector<int64_t> nnz_prefix;       // nnz of stored rows with distance <= h (h <= s-1)
    double* V = nullptr;
    double* xe = nullptr;                  // ext scratch for the residual (distributed)
    // Fused normalisation (CAGMRES_OPT_FUSE bit 2, default on): the residual r and each Arnoldi
    // vector w are left unnormalised in S (ext length) with their norm on the device; the SpMV
    // that consumes them forms q = w * (1/||w||) on the fly and stores q into V[:, pend_col]
    // (kern::spmv_scaled) — bitwise the separate scaling pass, one launch and one vector pass less.
    double* S = nullptr;
    bool fuse_scale = true;
    bool pend = false;                     // V[:, pend_col] = S / *pend_nrm still to be formed
    const double* pend_nrm = nullptr;
    int pend_col = 0;
    double* tab = nullptr; size_t tab_cap = 0;
    double* gbuf = nullptr;                // Gram / small scratch
    double* ybuf = nullptr;                // LS solution (m)
    double* caqr_ws = nullptr;             // CAQR tree workspace (lazy)
    double* op_M = nullptr;                // one-pass BOrth+CholQR: [-C R^{-1}; R^{-1}] (64 x 32)
    // pinned host mirrors + events of the per-cycle host <-> device exchange
    double* h_tab = nullptr;
    double* h_y = nullptr;
    double* h_beta = nullptr;
    int* h_stat = nullptr;
    cudaEvent_t ev_tab = nullptr, ev_beta = nullptr;
    size_t caqr_cap = 0;
    kern::XtyWs ws;
    double* arn_part = nullptr;            // fused Arnoldi partials
    unsigned int* arn_counter = nullptr;
    bool arnoldi_fuse = true;
    bool fuse_borth_gram = false;          // BOrth pass 2 + CholQR Gram in one pass (fused.cu; slower)
    // CAGMRES_OPT_FOLD (default on): the last block's final panel update (P R^{-1}, or the
    // one-pass [Q P] M) is never formed — the restart only needs x += V y, and
    // Q_new y_new = P (R^{-1} [0; y_new]) — so it is folded into the solution update.
    // fold_kind of the cycle just enqueued: 0 = none, 1 = P R^{-1}, 2 = one-pass; fold_pass = the
    // pass whose R (and C) the host applies.
    bool fold = true;
    int fold_kind = 0, fold_pass = 0;
    // CAGMRES_OPT_SERP (default on): serpentine order — every streaming launch (SpMV, panel ring
    // kernels) sweeps the rows opposite to the previous one (kern::band_tile), so it first reads
    // what its predecessor touched last, still in L2.  Reset at the start of every cycle.
    bool serp = true;
    int* status = nullptr;
    double ms_setup = 0.0;                 // wall time of create
    // CUDA graph of one CA cycle (single rank, untimed solves): captured once per configuration
    // (shifts, options) on a private stream and replayed every cycle
    cudaStream_t cap_stream = nullptr;
    cudaGraphExec_t cyc_exec = nullptr;
    uint64_t cfg_version = 1, cyc_version = 0;
    double cyc_bytes[PH_N] = {0, 0, 0, 0, 0};
    int cyc_spmv = 0;
    long long cyc_launches = 0;
    int cyc_rev_end = 0;
    bool use_graphs = false;               // CAGMRES_OPT_GRAPH (measured neutral on C2: off)
    bool capturing = false;
    int graph_err = 0;                     // cudaError_t of a failed capture (graphs then off)
    // per-panel diagnostics (cagmres_stats.collect_diag): per block [W^T W | Q_p^T Q_p], (s+1)^2 each
    bool diag_on = false;
    double* dg = nullptr;
    double* h_dg = nullptr;
    size_t dg_cap = 0;
    // halo (distributed)
    std::vector<int64_t> send_off, recv_off;
    std::vector<std::vector<int64_t>> send_pre, recv_pre;   // [rank][depth]
    int64_t nsend = 0, nrecv = 0;
    int64_t* d_send_idx = nullptr;
    int64_t* d_recv_ext = nullptr;
    int64_t* d_recv_src = nullptr;         // owner-local row of each requested value (peer pull)
    bool peer_ok = false;                  // transport offers one-sided peer access (in-process group)
    bool peer_pull = true;                 // CAGMRES_OPT_PEER: use it (1, default) or the copies (0)
    double* gsum = nullptr;                // fused cross-rank Gram sum (32 x 32)
    double* d_sendbuf = nullptr;
    double* d_recvbuf = nullptr;
    // shifts
    std::vector<double> sh_re, sh_im;
    bool have_shifts = false;
    Timer timer;
    double bytes[PH_N] = {0, 0, 0, 0, 0};
    int spmv_launches = 0;
    // single-GPU temporally blocked MPK (mpk_wave.cu)
    bool wave_ok = false, wave_on = false;   // off until it beats the stepwise MPK
    bool wave_force = false;               // option value 2: skip the L2-fit heuristic
    bool sweep_on = false;                 // option value 3: one persistent launch per MPK block
    unsigned* sweep_bar = nullptr;         // its grid-barrier counter (only grows)
    unsigned sweep_base = 0;
    int64_t wave_bw = 0;
    int wave_CH = 1024, wave_ctas = 4, wave_lag = 0, wave_nC = 0, wave_epoch = 0;
    int* d_done = nullptr;
    std::vector<int2*> d_pairs;            // indexed by sb (built lazily)
    std::vector<int> npairs;

    ~cagmres() {
        cudaFree(d_done);
        for (int2* p : d_pairs) cudaFree(p);
        cudaFree(A.sptr); cudaFree(A.sinfo); cudaFree(A.dcol); cudaFree(A.val);
        cudaFree(sweep_bar);
        cudaFree(V); cudaFree(xe); cudaFree(S); cudaFree(tab); cudaFree(gbuf); cudaFree(ybuf); cudaFree(caqr_ws); cudaFree(op_M);
        cudaFreeHost(h_tab); cudaFreeHost(h_y); cudaFreeHost(h_beta); cudaFreeHost(h_stat);
        cudaFree(dg); cudaFreeHost(h_dg);
        if (ev_tab) cudaEventDestroy(ev_tab);
        if (ev_beta) cudaEventDestroy(ev_beta);
        cudaFree(ws.part); cudaFree(ws.counter); cudaFree(status);
        cudaFree(arn_part); cudaFree(arn_counter);
        cudaFree(d_send_idx); cudaFree(d_recv_ext); cudaFree(d_recv_src); cudaFree(d_sendbuf); cudaFree(d_recvbuf);
        cudaFree(gsum);
        tr.reset();
        if (own_stream) cudaStreamDestroy(own_stream);
        if (cyc_exec) cudaGraphExecDestroy(cyc_exec);
        if (cap_stream) cudaStreamDestroy(cap_stream);
    }
};

namespace {

// ---- timing helpers --------------------------------------------------------------------
// A phase of the cycle (SURVEY §5 tracing): an NVTX range on the host thread that enqueues it
// (visible to Nsight Systems / any NVTX tool; a no-op without one) and, with collect_timing, a
// pair of CUDA events on the handle's stream.
const char* const kPhaseName[] = {"MPK", "BOrth", "TSQR", "other", "SpMV"};
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};
struct Scope {
    cagmres* h; int ph; cudaEvent_t e0 = nullptr;
    bool act;
    Scope(cagmres* hh, int p) : h(hh), ph(p), act(hh->timer.on && (!hh->timer.light || p == PH_SPMV)) {
        nvtxRangePushA(kPhaseName[p]);
        if (act) { e0 = h->timer.get(); cudaEventRecord(e0, h->stream); }
    }
    ~Scope() {
        nvtxRangePop();
        if (act) {
            cudaEvent_t e1 = h->timer.get();
            cudaEventRecord(e1, h->stream);
            h->timer.rec.push_back({ph, {e0, e1}});
        }
    }
};

int64_t round_up(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

// Device descriptor for the next streaming launch: flips the sweep direction (OPT_SERP).
kern::Dev& sdev(cagmres* h) {
    h->dev.rev = h->serp ? (h->dev.rev ^ 1) : 0;
    return h->dev;
}

// ---- SELL-32 build (host) + upload ------------------------------------------------------
// SELL-32 upload of the host layout built by sell_build (sell.cpp).
int build_sell(cagmres* h, const cagmres_plan& p) {
    SellHost sh;
    try {
        sell_build(p, sh);
    } catch (...) {
        return CAGMRES_ENOMEM;
    }
    const int64_t nr = p.n_mat, ns = sh.nslices, tot = sh.sptr[size_t(ns)], ndcol = int64_t(sh.dcol.size());
    const std::vector<int64_t>& sptr = sh.sptr;
    const std::vector<int64_t>& sinfo = sh.sinfo;
    const std::vector<int32_t>& dcol = sh.dcol;
    const std::vector<double>& val = sh.val;
    const int64_t ndia = sh.ndia;
    h->A.nrows = nr; h->A.nslices = ns; h->A.nstored = tot; h->A.nnz = p.nnz_mat;
    h->A.ncols = p.n_ext; h->A.ndcol = ndcol; h->A.ndia = ndia;
    {   // most common width among unclamped DIA slices (the specialised SpMV's fast path)
        std::vector<int64_t> cnt(33, 0);
        for (int64_t sl = 0; sl < ns; ++sl)
            if ((sinfo[size_t(sl)] & 3) == 1) {
                const int64_t wdt = (sptr[size_t(sl) + 1] - sptr[size_t(sl)]) / 32;
                if (wdt <= 32) ++cnt[size_t(wdt)];
            }
        h->A.dia_w = int(std::max_element(cnt.begin(), cnt.end()) - cnt.begin());
    }
    CU(cudaMalloc(&h->A.sptr, sizeof(int64_t) * size_t(ns + 1)));
    CU(cudaMalloc(&h->A.sinfo, sizeof(int64_t) * size_t(std::max<int64_t>(ns, 1))));
    CU(cudaMalloc(&h->A.dcol, sizeof(int32_t) * size_t(std::max<int64_t>(ndcol, 1))));
    CU(cudaMalloc(&h->A.val, sizeof(double) * size_t(std::max<int64_t>(tot, 1))));
    CU(cudaMemcpy(h->A.sptr, sptr.data(), sizeof(int64_t) * size_t(ns + 1), cudaMemcpyHostToDevice));
    if (ns) CU(cudaMemcpy(h->A.sinfo, sinfo.data(), sizeof(int64_t) * size_t(ns), cudaMemcpyHostToDevice));
    if (ndcol) CU(cudaMemcpy(h->A.dcol, dcol.data(), sizeof(int32_t) * size_t(ndcol), cudaMemcpyHostToDevice));
    if (tot) CU(cudaMemcpy(h->A.val, val.data(), sizeof(double) * size_t(tot), cudaMemcpyHostToDevice));
    // nnz of the first level_len[h] rows (algorithmic byte model of a prefix SpMV)
    h->nnz_prefix.assign(size_t(h->s) + 1, 0);
    for (int hh = 0; hh <= h->s; ++hh) {
        const int64_t rows = std::min(nr, p.level_len[size_t(hh)]);
        h->nnz_prefix[size_t(hh)] = p.rowptr[size_t(rows)];
    }
    return CAGMRES_OK;
}

size_t tab_doubles(int s, int m) {
    const size_t M = size_t(m) + 2, W = size_t(s) + 2;
    return 4 * M * M + 4 * M * W * W + 64;
}

int common_alloc(cagmres* h) {
    h->ldv = round_up(std::max<int64_t>(h->n_ext, 1), 32);
    const size_t vbytes = sizeof(double) * size_t(h->ldv) * size_t(h->m + 1);
    if (cudaMalloc(&h->V, vbytes) != cudaSuccess) return CAGMRES_ENOMEM;
    CU(cudaMemset(h->V, 0, vbytes));
    if (cudaMalloc(&h->S, sizeof(double) * size_t(h->ldv)) != cudaSuccess) return CAGMRES_ENOMEM;
    CU(cudaMemset(h->S, 0, sizeof(double) * size_t(h->ldv)));
    if (h->nranks > 1) {
        if (cudaMalloc(&h->xe, sizeof(double) * size_t(h->ldv)) != cudaSuccess) return CAGMRES_ENOMEM;
        CU(cudaMemset(h->xe, 0, sizeof(double) * size_t(h->ldv)));
    }
    h->tab_cap = tab_doubles(h->s, h->m);
    CU(cudaMalloc(&h->tab, sizeof(double) * h->tab_cap));
    CU(cudaMemset(h->tab, 0, sizeof(double) * h->tab_cap));
    CU(cudaMalloc(&h->gbuf, sizeof(double) * size_t(h->m + 2) * size_t(std::max(h->m, 32) + 2)));
    CU(cudaMalloc(&h->ybuf, sizeof(double) * size_t(h->m + 2)));
    CU(cudaMalloc(&h->op_M, sizeof(double) * 64 * 32));
    CU(cudaMallocHost(&h->h_tab, sizeof(double) * h->tab_cap));
    CU(cudaMallocHost(&h->h_y, sizeof(double) * size_t(h->m + 2)));
    CU(cudaMallocHost(&h->h_beta, sizeof(double) * 2));
    CU(cudaMallocHost(&h->h_stat, sizeof(int) * 2));
    CU(cudaEventCreateWithFlags(&h->ev_tab, cudaEventDisableTiming));
    CU(cudaEventCreateWithFlags(&h->ev_beta, cudaEventDisableTiming));
    size_t cap = 0;
    for (int w = 1; w <= 32; ++w) cap = std::max(cap, kern::xty_ws_doubles(h->dev, h->m + 1, w));
    cap = std::max(cap, kern::update_gram_ws_doubles(h->dev));
    cap = std::max(cap, size_t(2) * size_t(h->dev.sms) * 12 * 12);     // scalar Gram (+ group partials)
    h->ws.cap = cap;
    CU(cudaMalloc(&h->ws.part, sizeof(double) * cap));
    CU(cudaMalloc(&h->ws.counter, sizeof(unsigned int) * kern::XTY_COUNTERS));
    CU(cudaMemset(h->ws.counter, 0, sizeof(unsigned int) * kern::XTY_COUNTERS));
    CU(cudaMalloc(&h->arn_part, sizeof(double) * kern::arnoldi_ws_doubles(h->dev)));
    CU(cudaMalloc(&h->arn_counter, sizeof(unsigned int) * kern::XTY_COUNTERS));
    CU(cudaMemset(h->arn_counter, 0, sizeof(unsigned int) * kern::XTY_COUNTERS));
    CU(cudaMalloc(&h->status, sizeof(int) * 2));            // [0] breakdown flags, [1] SVQR retries
    CU(cudaMemset(h->status, 0, sizeof(int) * 2));
    return CAGMRES_OK;
}

// Temporal blocking is used when the matrix is banded enough that the reuse window of a
// chunk of A (s * L chunks) fits comfortably in the 126 MB L2.
int wave_setup(cagmres* h, const cagmres_plan& p) {
    int64_t bw = 0;
    for (int64_t r = 0; r < p.n_mat; ++r)
        for (int64_t e = p.rowptr[size_t(r)]; e < p.rowptr[size_t(r) + 1]; ++e)
            bw = std::max<int64_t>(bw, std::llabs(int64_t(p.colind[size_t(e)]) - r));
    h->wave_bw = bw;
    h->wave_ok = bw < h->n_loc / 4;                      // otherwise no reuse window exists
    return CAGMRES_OK;
}

int wave_lag(const cagmres* h) {
    // L > ceil(b/CH) keeps the order topological; the extra ~2*G/s chunks of slack give
    // every step enough runnable chunks for the G resident CTAs.
    const int minlag = int((h->wave_bw + h->wave_CH - 1) / h->wave_CH) + 1;   // topological order
    if (h->wave_lag > 0) return std::max(h->wave_lag, minlag);
    const int G = h->dev.sms * std::max(1, h->wave_ctas);
    return minlag + (2 * G + h->s - 1) / h->s;
}

bool wave_fits(const cagmres* h) {
    const double nnz_row = h->n_loc > 0 ? double(h->A.nnz) / double(h->n_loc) : 0.0;
    const double chunk_bytes = double(h->wave_CH) * (12.0 * nnz_row + 16.0);
    if (h->wave_force) return h->wave_ok;
    return h->wave_ok && double(h->s) * wave_lag(h) * chunk_bytes <= 80.0e6 &&
           h->n_loc >= 8 * int64_t(h->wave_CH);
}

// (chunk, step) items of a block of sb steps in wavefront order tau = c + L*k
int wave_pairs(cagmres* h, int sb) {
    const int nC = int((h->n_loc + h->wave_CH - 1) / h->wave_CH);
    if (h->wave_nC != nC || h->d_pairs.size() != size_t(h->s) + 1) {
        for (int2* q : h->d_pairs) cudaFree(q);
        h->d_pairs.assign(size_t(h->s) + 1, nullptr);
        h->npairs.assign(size_t(h->s) + 1, 0);
        cudaFree(h->d_done);
        h->d_done = nullptr;
        CU(cudaMalloc(&h->d_done, sizeof(int) * (size_t(nC) * size_t(h->s + 1) + 1)));
        CU(cudaMemset(h->d_done, 0, sizeof(int) * (size_t(nC) * size_t(h->s + 1) + 1)));
        h->wave_nC = nC;
        h->wave_epoch = 0;
    }
    if (h->d_pairs[size_t(sb)]) return CAGMRES_OK;
    const int64_t L = wave_lag(h);
    std::vector<int2> pr;
    pr.reserve(size_t(nC) * size_t(sb));
    for (int64_t tau = 0; tau <= nC - 1 + L * sb; ++tau)
        for (int k = 1; k <= sb; ++k) {
            const int64_t c = tau - L * k;
            if (c >= 0 && c < nC) pr.push_back(make_int2(int(c), k));
        }
    CU(cudaMalloc(&h->d_pairs[size_t(sb)], sizeof(int2) * pr.size()));
    CU(cudaMemcpy(h->d_pairs[size_t(sb)], pr.data(), sizeof(int2) * pr.size(), cudaMemcpyHostToDevice));
    h->npairs[size_t(sb)] = int(pr.size());
    return CAGMRES_OK;
}

void wave_reset_pairs(cagmres* h) {
    for (int2* q : h->d_pairs) cudaFree(q);
    h->d_pairs.clear();
    h->wave_nC = 0;
}

// SpMV kernel selection (setup, once): every CAGMRES_OPT_SPMV variant computes each row with
// the same operations in the same order (bitwise identical results), so the fastest one on
// this matrix is picked by timing y = A x over all stored rows (x = V[:,0], y = V[:,1]).
int spmv_autotune(cagmres* h) {
    static const int cand[] = {0, 5, 16, 17};
    if (h->m < 1 || h->A.nrows <= 0) return CAGMRES_OK;
    double* x = h->V;
    double* y = h->V + h->ldv;
    cudaEvent_t e0, e1;
    CU(cudaEventCreate(&e0));
    CU(cudaEventCreate(&e1));
    constexpr int NC = int(sizeof(cand) / sizeof(cand[0]));
    constexpr int CHAIN = 8;                 // an MPK-like chain of dependent launches
    float tmin[NC];
    for (int i = 0; i < NC; ++i) {
        tmin[i] = 1e30f;
        h->A.variant = cand[i];
        for (int k = 0; k < 2; ++k)          // warm-up (and the clock ramp) for every candidate
            kern::spmv(h->dev, h->A, h->A.nrows, k ? y : x, k ? x : y, nullptr, 0.0, nullptr, 0.0, h->stream);
    }
    // round-robin over the candidates (5 rounds, best of each): clock ramp or drift does not
    // favour a candidate by its position in the list
    for (int r = 0; r < 5; ++r)
        for (int i = 0; i < NC; ++i) {
            h->A.variant = cand[i];
            CU(cudaEventRecord(e0, h->stream));
            for (int k = 0; k < CHAIN; ++k)
                kern::spmv(h->dev, h->A, h->A.nrows, (k & 1) ? y : x, (k & 1) ? x : y, nullptr, 0.0, nullptr, 0.0,
                           h->stream);
            CU(cudaEventRecord(e1, h->stream));
            CU(cudaEventSynchronize(e1));
            float ms = 0.f;
            CU(cudaEventElapsedTime(&ms, e0, e1));
            tmin[i] = std::min(tmin[i], ms / CHAIN);
        }
    int bi = 0;
    for (int i = 1; i < NC; ++i)
        if (tmin[i] < tmin[bi]) bi = i;
    // the DIA kernels also fuse the q = w / ||w|| normalisations: prefer them within 3 %
    int bd = -1;
    for (int i = 0; i < NC; ++i)
        if (cand[i] >= 16 && (bd < 0 || tmin[i] < tmin[bd])) bd = i;
    if (cand[bi] < 16 && bd >= 0 && tmin[bd] <= 1.03f * tmin[bi]) bi = bd;
    const float best = tmin[bi];
    const int pick = cand[bi];
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    h->A.variant = pick;
    h->spmv_tuned_us = double(best) * 1e3;
    CU(cudaMemsetAsync(h->V, 0, sizeof(double) * size_t(h->ldv) * 2, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    return CAGMRES_OK;
}

int init_common_(cagmres* h, const cagmres_csr* A, const int64_t* row_starts, int s, int m,
                 int basis, int orth);
int init_common(cagmres* h, const cagmres_csr* A, const int64_t* row_starts, int s, int m,
                int basis, int orth) {
    const auto t0 = std::chrono::steady_clock::now();
    const int st = init_common_(h, A, row_starts, s, m, basis, orth);
    h->ms_setup = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return st;
}
int init_common_(cagmres* h, const cagmres_csr* A, const int64_t* row_starts, int s, int m,
                 int basis, int orth) {
    if (s < 1 || m < 1 || s > m || s > 31 || (basis != CAGMRES_MONOMIAL && basis != CAGMRES_NEWTON && basis != CAGMRES_GMRES))
        return CAGMRES_EINVAL;
    const int kind = orth & CAGMRES_TSQR_MASK;
    if (kind > CAGMRES_CAQR) return CAGMRES_EINVAL;
    if ((orth & CAGMRES_ONEPASS) && (kind != CAGMRES_CHOLQR || (orth & CAGMRES_BORTH_MGS))) return CAGMRES_EINVAL;
    if ((orth & CAGMRES_SVQR_RETRY) && kind != CAGMRES_CHOLQR) return CAGMRES_EINVAL;
    h->s = s; h->m = m; h->basis = basis; h->orth = orth;
    int dv = 0;
    CU(cudaGetDevice(&dv));
    h->dev.device = dv;
    CU(cudaDeviceGetAttribute(&h->dev.sms, cudaDevAttrMultiProcessorCount, dv));
    CU(cudaStreamCreateWithFlags(&h->own_stream, cudaStreamNonBlocking));
    h->stream = h->own_stream;
    cagmres_plan plan;
    try {
        TRY(plan_build(&plan, A, row_starts, h->nranks, h->rank, s));
    } catch (...) {
        return CAGMRES_ENOMEM;
    }
    h->n = A->n; h->n_loc = plan.n_loc; h->n_ext = plan.n_ext;
    h->level_len = plan.level_len;
    TRY(build_sell(h, plan));
    TRY(common_alloc(h));
    TRY(spmv_autotune(h));
    if (h->nranks == 1) TRY(wave_setup(h, plan));
    if (h->nranks > 1) {
        // ---- exchange request lists (setup, "compress ... needed by other GPUs") ----
        const int P = h->nranks;
        std::vector<int64_t> myc(plan.req_counts);
        int64_t *d_cnt = nullptr, *d_all = nullptr;
        CU(cudaMalloc(&d_cnt, sizeof(int64_t) * size_t(P)));
        CU(cudaMalloc(&d_all, sizeof(int64_t) * size_t(P) * size_t(P)));
        CU(cudaMemcpy(d_cnt, myc.data(), sizeof(int64_t) * size_t(P), cudaMemcpyHostToDevice));
        TRY(h->tr->allgather(d_cnt, d_all, sizeof(int64_t) * size_t(P), h->stream));
        std::vector<int64_t> all(size_t(P) * size_t(P));
        CU(cudaMemcpyAsync(all.data(), d_all, sizeof(int64_t) * all.size(), cudaMemcpyDeviceToHost, h->stream));
        CU(cudaStreamSynchronize(h->stream));
        cudaFree(d_cnt); cudaFree(d_all);
        std::vector<int64_t> inc(static_cast<size_t>(P));                // what q requests of me
        int64_t tin = 0, tout = int64_t(plan.req_gid.size());
        for (int q = 0; q < P; ++q) { inc[size_t(q)] = all[size_t(q) * P + size_t(h->rank)]; tin += inc[size_t(q)]; }
        int64_t *d_og = nullptr, *d_ig = nullptr;
        int32_t *d_ol = nullptr, *d_il = nullptr;
        CU(cudaMalloc(&d_og, sizeof(int64_t) * size_t(std::max<int64_t>(tout, 1))));
        CU(cudaMalloc(&d_ol, sizeof(int32_t) * size_t(std::max<int64_t>(tout, 1))));
        CU(cudaMalloc(&d_ig, sizeof(int64_t) * size_t(std::max<int64_t>(tin, 1))));
        CU(cudaMalloc(&d_il, sizeof(int32_t) * size_t(std::max<int64_t>(tin, 1))));
        if (tout) {
            CU(cudaMemcpy(d_og, plan.req_gid.data(), sizeof(int64_t) * size_t(tout), cudaMemcpyHostToDevice));
            CU(cudaMemcpy(d_ol, plan.req_level.data(), sizeof(int32_t) * size_t(tout), cudaMemcpyHostToDevice));
        }
        std::vector<Msg> sends, recvs;
        int64_t oo = 0, io = 0;
        for (int q = 0; q < P; ++q) {
            const int64_t so = plan.req_counts[size_t(q)], si = inc[size_t(q)];
            if (so) { sends.push_back({q, d_og + oo, sizeof(int64_t) * size_t(so)});
                      sends.push_back({q, d_ol + oo, sizeof(int32_t) * size_t(so)}); }
            if (si) { recvs.push_back({q, d_ig + io, sizeof(int64_t) * size_t(si)});
                      recvs.push_back({q, d_il + io, sizeof(int32_t) * size_t(si)}); }
            oo += so; io += si;
        }
        TRY(h->tr->exchange(sends, recvs, h->stream));
        std::vector<int64_t> ig(static_cast<size_t>(tin));
        std::vector<int32_t> il(static_cast<size_t>(tin));
        if (tin) {
            CU(cudaMemcpyAsync(ig.data(), d_ig, sizeof(int64_t) * size_t(tin), cudaMemcpyDeviceToHost, h->stream));
            CU(cudaMemcpyAsync(il.data(), d_il, sizeof(int32_t) * size_t(tin), cudaMemcpyDeviceToHost, h->stream));
        }
        CU(cudaStreamSynchronize(h->stream));
        cudaFree(d_og); cudaFree(d_ol); cudaFree(d_ig); cudaFree(d_il);
        TRY(cagmres_plan_set_sends(&plan, inc.data(), ig.data(), il.data()));
        // ---- device halo tables -------------------------------------------------------
        h->nsend = tin; h->nrecv = tout;
        h->send_off.assign(size_t(P) + 1, 0); h->recv_off.assign(size_t(P) + 1, 0);
        h->send_pre.assign(size_t(P), std::vector<int64_t>(size_t(s) + 1, 0));
        h->recv_pre.assign(size_t(P), std::vector<int64_t>(size_t(s) + 1, 0));
        for (int q = 0; q < P; ++q) {
            h->send_off[size_t(q) + 1] = h->send_off[size_t(q)] + inc[size_t(q)];
            h->recv_off[size_t(q) + 1] = h->recv_off[size_t(q)] + plan.req_counts[size_t(q)];
            for (int d = 0; d <= s; ++d) {
                h->send_pre[size_t(q)][size_t(d)] = plan_prefix_count(plan.send_counts, plan.send_level, q, d);
                h->recv_pre[size_t(q)][size_t(d)] = plan_prefix_count(plan.req_counts, plan.req_level, q, d);
            }
        }
        CU(cudaMalloc(&h->d_send_idx, sizeof(int64_t) * size_t(std::max<int64_t>(tin, 1))));
        CU(cudaMalloc(&h->d_recv_ext, sizeof(int64_t) * size_t(std::max<int64_t>(tout, 1))));
        CU(cudaMalloc(&h->d_sendbuf, sizeof(double) * size_t(std::max<int64_t>(tin, 1))));
        CU(cudaMalloc(&h->d_recvbuf, sizeof(double) * size_t(std::max<int64_t>(tout, 1))));
        CU(cudaMemset(h->d_sendbuf, 0, sizeof(double) * size_t(std::max<int64_t>(tin, 1))));
        CU(cudaMemset(h->d_recvbuf, 0, sizeof(double) * size_t(std::max<int64_t>(tout, 1))));
        if (tin) CU(cudaMemcpy(h->d_send_idx, plan.send_idx.data(), sizeof(int64_t) * size_t(tin), cudaMemcpyHostToDevice));
        if (tout) CU(cudaMemcpy(h->d_recv_ext, plan.req_ext.data(), sizeof(int64_t) * size_t(tout), cudaMemcpyHostToDevice));
        {   // owner-local rows of the requested values, for the one-sided halo pull
            std::vector<int64_t> src(static_cast<size_t>(std::max<int64_t>(tout, 1)), 0);
            int64_t k = 0;
            for (int q = 0; q < P; ++q)
                for (int64_t e = 0; e < plan.req_counts[size_t(q)]; ++e, ++k)
                    src[size_t(k)] = plan.req_gid[size_t(k)] - row_starts[q];
            CU(cudaMalloc(&h->d_recv_src, sizeof(int64_t) * src.size()));
            CU(cudaMemcpy(h->d_recv_src, src.data(), sizeof(int64_t) * src.size(), cudaMemcpyHostToDevice));
        }
        CU(cudaMalloc(&h->gsum, sizeof(double) * 32 * 32));
        h->peer_ok = h->tr->peer_capable() && h->peer_pull;
    }
    return CAGMRES_OK;
}

// ---- collectives (transport.h: NCCL, or the in-process group) -------------------------
int allreduce(cagmres* h, double* buf, size_t cnt) {
    if (h->nranks == 1 || cnt == 0) return CAGMRES_OK;
    return h->tr->allreduce_sum(buf, cnt, h->stream);
}

// Halo exchange of the ghost rows (distance <= depth) of an extended vector (Fig. 4 setup,
// P:66): pack the owned values the peers need at this depth, grouped send / recv (NVLink),
// unpack.  Every peer's send / request list is sorted by level, so the depth-limited message
// to or from a peer is a prefix of its segment; only those prefixes are packed and unpacked.
int halo(cagmres* h, double* vec, int depth) {
    if (h->nranks == 1 || depth <= 0) return CAGMRES_OK;
    depth = std::min(depth, h->s);
    if (h->peer_ok && h->nranks <= 16) {
        // one-sided: every rank posts its vector, then ONE kernel pulls the depth-limited
        // prefix of each owner's list straight from the owner's owned rows (peer memory)
        std::vector<const void*> peers;
        TRY(h->tr->peer_acquire(vec, peers, h->stream));
        kern::PullSegs sg{};
        for (int q = 0; q < h->nranks; ++q) {
            const int64_t rc = h->recv_pre[size_t(q)][size_t(depth)];
            if (!rc) continue;
            sg.src[sg.n] = static_cast<const double*>(peers[size_t(q)]);
            sg.off[sg.n] = h->recv_off[size_t(q)];
            sg.cnt[sg.n] = rc;
            ++sg.n;
        }
        kern::halo_pull(sg, h->d_recv_src, h->d_recv_ext, vec, h->stream);
        TRY(h->tr->peer_release(h->stream));
        return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
    }
    std::vector<std::pair<int64_t, int64_t>> ss, rs;          // (offset, count) per peer
    std::vector<Msg> sends, recvs;
    for (int q = 0; q < h->nranks; ++q) {
        const int64_t sc = h->send_pre[size_t(q)][size_t(depth)], rc = h->recv_pre[size_t(q)][size_t(depth)];
        if (sc) {
            ss.push_back({h->send_off[size_t(q)], sc});
            sends.push_back({q, h->d_sendbuf + h->send_off[size_t(q)], sizeof(double) * size_t(sc)});
        }
        if (rc) {
            rs.push_back({h->recv_off[size_t(q)], rc});
            recvs.push_back({q, h->d_recvbuf + h->recv_off[size_t(q)], sizeof(double) * size_t(rc)});
        }
    }
    auto segs = [](const std::vector<std::pair<int64_t, int64_t>>& v, size_t i0) {
        kern::Segs sg{};
        for (size_t i = i0; i < v.size() && i < i0 + 32; ++i) sg.add(v[i].first, v[i].second);
        return sg;
    };
    for (size_t i = 0; i < ss.size(); i += 32) kern::gather_segs(vec, h->d_send_idx, segs(ss, i), h->d_sendbuf, h->stream);
    TRY(h->tr->exchange(sends, recvs, h->stream));
    for (size_t i = 0; i < rs.size(); i += 32) kern::scatter_segs(h->d_recvbuf, h->d_recv_ext, segs(rs, i), vec, h->stream);
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

// ---- building blocks ------------------------------------------------------------------
// C = X^T Y summed over ranks (out ld ldo); optional R = chol(C) (CholQR Gram)
int xty_global(cagmres* h, const double* X, int64_t ldx, int jx, const double* Y, int64_t ldy,
               int w, double* out, bool chol, double* R) {
    if (h->nranks == 1) {
        if (kern::xty(sdev(h), h->n_loc, X, ldx, jx, Y, ldy, w, out, chol, R, h->status, h->ws, h->stream))
            return CAGMRES_EINVAL;
        return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
    }
    if (kern::xty(sdev(h), h->n_loc, X, ldx, jx, Y, ldy, w, out, false, nullptr, h->status, h->ws, h->stream))
        return CAGMRES_EINVAL;
    if (chol && h->peer_ok && w <= 32) {
        // one-sided: the cross-rank sum of the Gram and its Cholesky in one launch reading the
        // peers' partial Grams directly; the sum then replaces this rank's partial
        std::vector<const void*> peers;
        TRY(h->tr->peer_acquire(out, peers, h->stream));
        std::vector<const double*> src(peers.size());
        for (size_t q = 0; q < peers.size(); ++q) src[q] = static_cast<const double*>(peers[q]);
        kern::sum_chol(src.data(), h->nranks, w, h->gsum, R, h->status, h->stream);
        TRY(h->tr->peer_release(h->stream));
        CU(cudaMemcpyAsync(out, h->gsum, sizeof(double) * size_t(w) * size_t(w), cudaMemcpyDeviceToDevice, h->stream));
        return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
    }
    TRY(allreduce(h, out, size_t(jx) * size_t(w)));
    if (chol) kern::chol(out, w, R, h->status, h->stream);
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

double spmv_bytes(cagmres* h, int64_t rows_out, int depth_in, bool pair2) {
    // 12 nnz + 4 (r+1) + 8 r' + 8 r (+ 8 r for the pair's second step)
    const int64_t r = rows_out;
    int hh = 0;
    while (hh < h->s && h->level_len[size_t(hh)] < r) ++hh;
    const double nnz = double(h->nnz_prefix[size_t(std::min(hh, h->s))]);
    const double rin = double(h->level_len[size_t(std::min(depth_in, h->s))]);
    return 12.0 * nnz + 4.0 * double(r + 1) + 8.0 * rin + 8.0 * double(r) + (pair2 ? 8.0 * double(r) : 0.0);
}

// Forms a pending normalised vector V[:, pend_col] = S / ||S|| on its first `rows` extended rows
// for a consumer that cannot fuse it (generic SpMV variants, the temporally blocked MPK).
int materialize(cagmres* h, int64_t rows) {
    if (!h->pend) return CAGMRES_OK;
    kern::scale_copy(rows, h->S, h->pend_nrm, h->V + size_t(h->ldv) * h->pend_col, h->stream);
    h->pend = false;
    h->bytes[PH_OTHER] += 16.0 * double(rows);
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

// Halo of the start vector of an SpMV chain at column col, depth `depth`.  With a pending
// normalisation the UNNORMALISED S is exchanged on every rank (the pending state is the same on
// all ranks; the SpMV variant — fused or not — may differ per rank, so the exchanged
// representation must not depend on it); a rank that cannot fuse then forms V[:, col] = S/||S||
// on its owned AND ghost rows.  Returns true when the caller's first SpMV must fuse (read S).
int start_halo(cagmres* h, int col, int depth, bool& fuse) {
    fuse = false;
    if (!(h->pend && h->pend_col == col)) {
        TRY(materialize(h, h->n_loc));
        return halo(h, h->V + size_t(h->ldv) * col, depth);
    }
    TRY(halo(h, h->S, depth));
    if (h->A.variant >= 16) { fuse = true; return CAGMRES_OK; }
    return materialize(h, h->level_len[size_t(std::min(depth, h->s))]);
}

// MPK of one block (Fig. 4): V[:, j+1 .. j+sb] from V[:, j].  Step k computes the rows at
// distance <= sb-k (a prefix of the extended numbering) from the rows at distance <= sb-k+1.
int mpk_block(cagmres* h, int j, int sb, const std::vector<host::Step>& steps) {
    Scope sc(h, PH_MPK);
    if (h->sweep_on && h->nranks == 1 && sb >= 2 && h->A.variant >= 16 && h->sweep_bar) {
        TRY(materialize(h, h->n_loc));
        kern::SweepArgs a{};
        a.sptr = h->A.sptr; a.sinfo = h->A.sinfo; a.dcol = h->A.dcol; a.val = h->A.val; a.ncols = h->A.ncols;
        a.V = h->V; a.ldv = h->ldv; a.j = j; a.sb = sb; a.n = h->n_loc; a.dia_w = h->A.dia_w;
        a.bar = h->sweep_bar; a.bar_base = h->sweep_base;
        for (int k = 1; k <= sb; ++k) {
            a.theta[k - 1] = steps[size_t(k - 1)].a;
            a.b2[k - 1] = steps[size_t(k - 1)].b2;
            a.kind[k - 1] = steps[size_t(k - 1)].kind;
        }
        kern::Dev& d = sdev(h);
        a.rev0 = d.rev;
        {
            Scope sv(h, PH_SPMV);
            if (kern::mpk_sweep(d, a, h->stream, &h->sweep_base)) return CAGMRES_EINVAL;
        }
        h->dev.rev = a.rev0 ^ ((sb - 1) & 1);            // direction of the block's last step
        double by = 0.0;
        for (int k = 1; k <= sb; ++k) by += spmv_bytes(h, h->n_loc, 1, steps[size_t(k - 1)].kind == 2);
        h->bytes[PH_MPK] += by;
        h->bytes[PH_SPMV] += by;
        h->spmv_launches++;
        return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
    }
    if (h->wave_on && h->nranks == 1 && sb >= 2 && wave_fits(h)) {
        TRY(materialize(h, h->n_loc));
        TRY(wave_pairs(h, sb));
        kern::WaveArgs a{};
        a.sptr = h->A.sptr; a.sinfo = h->A.sinfo; a.dcol = h->A.dcol; a.val = h->A.val; a.ncols = h->A.ncols;
        a.V = h->V; a.ldv = h->ldv; a.j = j;
        a.n = h->n_loc; a.bw = h->wave_bw; a.CH = h->wave_CH; a.nC = h->wave_nC;
        a.pairs = h->d_pairs[size_t(sb)]; a.npairs = h->npairs[size_t(sb)];
        a.done = h->d_done;
        a.queue = h->d_done + size_t(h->wave_nC) * size_t(h->s + 1);
        a.dia_w = h->A.dia_w;
        if (++h->wave_epoch == 0x7fffffff) {                 // epoch wrap: clear the flags
            CU(cudaMemsetAsync(h->d_done, 0, sizeof(int) * size_t(h->wave_nC) * size_t(h->s + 1), h->stream));
            h->wave_epoch = 1;
        }
        CU(cudaMemsetAsync(a.queue, 0, sizeof(int), h->stream));
        a.epoch = h->wave_epoch;
        for (int k = 1; k <= sb; ++k) {
            a.theta[k - 1] = steps[size_t(k - 1)].a;
            a.b2[k - 1] = steps[size_t(k - 1)].b2;
            a.kind[k - 1] = steps[size_t(k - 1)].kind;
        }
        {
            Scope sv(h, PH_SPMV);
            kern::mpk_wave(h->dev, a, h->wave_ctas, h->stream);
        }
        double by = 0.0;
        for (int k = 1; k <= sb; ++k) by += spmv_bytes(h, h->n_loc, 1, steps[size_t(k - 1)].kind == 2);
        h->bytes[PH_MPK] += by;
        h->bytes[PH_SPMV] += by;
        h->spmv_launches++;
        return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
    }
    bool fused_q = false;
    TRY(start_halo(h, j, sb, fused_q));
    for (int k = 1; k <= sb; ++k) {
        const host::Step& stp = steps[size_t(k - 1)];
        const double* x = h->V + size_t(h->ldv) * (j + k - 1);
        double* y = h->V + size_t(h->ldv) * (j + k);
        const int64_t rows = h->level_len[size_t(sb - k)];
        const bool pair2 = stp.kind == 2;
        {
            Scope sv(h, PH_SPMV);
            if (k == 1 && fused_q) {       // q_j = S / ||S|| formed inside the first step (stored to V[:, j])
                if (kern::spmv_scaled(sdev(h), h->A, rows, h->S, h->pend_nrm, h->V + size_t(h->ldv) * j, y, -stp.a,
                                      stp.a != 0.0, h->stream))
                    return CAGMRES_EINVAL;
                h->pend = false;
            } else {
                kern::spmv(sdev(h), h->A, rows, x, y, (stp.a != 0.0 || pair2) ? x : nullptr, -stp.a,
                           pair2 ? h->V + size_t(h->ldv) * (j + k - 2) : nullptr, stp.b2, h->stream);
            }
        }
        const double by = spmv_bytes(h, rows, sb - k + 1, pair2);
        h->bytes[PH_MPK] += by;
        h->bytes[PH_SPMV] += by;
        h->spmv_launches++;
    }
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

// BOrth of the panel columns P (n_loc x w, ld ldp) against Q (n_loc x j): CGS or MGS
// (P:144).  C: device j x w, ld j.
int borth_panel(cagmres* h, const double* Q, int64_t ldq, int j, double* P, int64_t ldp, int w,
                double* C, bool mgs) {
    if (j <= 0) return CAGMRES_OK;
    Scope sc(h, PH_BORTH);
    if (!mgs) {
        TRY(xty_global(h, Q, ldq, j, P, ldp, w, C, false, nullptr));
        // C is jx x w with ld jx = j: xty writes ld jx
        kern::update(sdev(h), h->n_loc, Q, ldq, j, P, ldp, w, C, h->stream, true);   // after xty: early start
        h->bytes[PH_BORTH] += 8.0 * double(h->n_loc) * (2.0 * j + 3.0 * w);
    } else {
        // row l of C (1 x w, ld j) via a scratch row then copied with ld j on the host view:
        for (int l = 0; l < j; ++l) {
            double* row = h->gbuf;
            TRY(xty_global(h, Q + size_t(ldq) * l, ldq, 1, P, ldp, w, row, false, nullptr));
            kern::update(sdev(h), h->n_loc, Q + size_t(ldq) * l, ldq, 1, P, ldp, w, row, h->stream);
            CU(cudaMemcpy2DAsync(C + l, sizeof(double) * size_t(j), row, sizeof(double), sizeof(double),
                                 size_t(w), cudaMemcpyDeviceToDevice, h->stream));
            h->bytes[PH_BORTH] += 8.0 * double(h->n_loc) * (2.0 + 3.0 * w);
        }
    }
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

// TSQR of the panel P (n_loc x w, ld ldp), R (device w x w, ld w).  c0 = 1 leaves column 0
// unwritten (the block's start vector q_j is kept, reading G2).
// skip_update (CholQR / SVQR only): R is formed but P is left as is (OPT_FOLD).
int tsqr_panel(cagmres* h, double* P, int64_t ldp, int w, double* R, int kind, int c0, bool retry = false,
               bool skip_update = false) {
    Scope sc(h, PH_TSQR);
    const double nl = double(h->n_loc);
    if (kind == CAGMRES_CHOLQR || kind == CAGMRES_SVQR) {
        if (kind == CAGMRES_CHOLQR) {
            TRY(xty_global(h, P, ldp, w, P, ldp, w, h->gbuf, true, R));     // B = V^T V ; R = chol(B)
            if (retry) kern::svqr_retry(h->gbuf, w, R, h->status, h->stream);   // G15 opt-in
        } else {
            TRY(xty_global(h, P, ldp, w, P, ldp, w, h->gbuf, false, nullptr));
            kern::svqr_factor(h->gbuf, w, R, h->status, h->stream);
        }
        if (skip_update) {
            h->bytes[PH_TSQR] += 8.0 * nl * w;
        } else {
            kern::trsm(sdev(h), h->n_loc, P, ldp, w, R, c0, h->stream, true);    // V := V R^{-1} (P final: early)
            h->bytes[PH_TSQR] += 8.0 * nl * (2.0 * w + double(w - c0));
        }
    } else if (kind == CAGMRES_CAQR) {                       // Fig. 9 CAQR: TSQR tree
        // Multi-rank: "each GPU first computes the QR factorization of the local
        // matrix, then the local R-factors are gathered ..., and the final QR factorization is
        // computed ...; V^(d) := V^(d) Q^(d)": local tree -> all-gather of the w x w R's ->
        // QR of the stacked R's (redundantly on every rank) -> P := Q_loc Q_s[rank block].
        const int Pn = h->nranks;
        const size_t W2 = size_t(w) * size_t(w);
        const int64_t sr = int64_t(Pn) * w;                      // rows of the stacked R's
        const size_t need_loc = kern::caqr_ws_doubles(h->n_loc, w);
        const size_t need = need_loc + (Pn > 1 ? 3 * size_t(Pn) * W2 + kern::caqr_ws_doubles(sr, w) +
                                                     size_t(h->n_loc) + W2 : 0);
        if (need > h->caqr_cap) {
            cudaFree(h->caqr_ws);
            h->caqr_ws = nullptr;
            CU(cudaMalloc(&h->caqr_ws, sizeof(double) * need));
            h->caqr_cap = need;
        }
        if (Pn == 1) {
            if (kern::caqr(h->dev, h->n_loc, P, ldp, w, R, c0, h->caqr_ws, h->stream)) return CAGMRES_EINVAL;
        } else {
            double* Rloc = h->caqr_ws + need_loc;                // w x w
            double* Rall = Rloc + W2;                            // Pn blocks of w x w
            double* Stk = Rall + size_t(Pn) * W2;                // sr x w, column-major
            double* q0 = Stk + size_t(Pn) * W2;                  // saved column 0 (c0 = 1)
            double* ws2 = q0 + size_t(h->n_loc);
            if (c0 == 1) CU(cudaMemcpyAsync(q0, P, sizeof(double) * size_t(h->n_loc), cudaMemcpyDeviceToDevice, h->stream));
            if (kern::caqr(h->dev, h->n_loc, P, ldp, w, Rloc, 0, h->caqr_ws, h->stream)) return CAGMRES_EINVAL;
            TRY(h->tr->allgather(Rloc, Rall, sizeof(double) * W2, h->stream));
            // stacked column-major: row q*w + i of column c = R_q[i, c]
            for (int q = 0; q < Pn; ++q)
                CU(cudaMemcpy2DAsync(Stk + size_t(q) * w, sizeof(double) * size_t(sr), Rall + size_t(q) * W2,
                                     sizeof(double) * size_t(w), sizeof(double) * size_t(w), size_t(w),
                                     cudaMemcpyDeviceToDevice, h->stream));
            if (kern::caqr(h->dev, sr, Stk, sr, w, R, 0, ws2, h->stream)) return CAGMRES_EINVAL;
            if (kern::gemm_rows(sdev(h), h->n_loc, P, ldp, w, P, ldp, w, Stk + size_t(h->rank) * w, sr, c0, h->stream))
                return CAGMRES_EINVAL;
            if (c0 == 1) CU(cudaMemcpyAsync(P, q0, sizeof(double) * size_t(h->n_loc), cudaMemcpyDeviceToDevice, h->stream));
        }
        h->bytes[PH_TSQR] += 8.0 * nl * (2.0 * w + double(w - c0));
    } else {
        CU(cudaMemsetAsync(R, 0, sizeof(double) * size_t(w) * size_t(w), h->stream));
        for (int k = 0; k < w; ++k) {
            double* pk = P + size_t(ldp) * k;
            if (k > 0) {
                if (kind == CAGMRES_CGS) {          // Fig. 9 right: r = V_{1:k-1}^T v_k
                    TRY(xty_global(h, P, ldp, k, pk, ldp, 1, R + size_t(w) * k, false, nullptr));
                    kern::update(sdev(h), h->n_loc, P, ldp, k, pk, ldp, 1, R + size_t(w) * k, h->stream);
                    h->bytes[PH_TSQR] += 8.0 * nl * (2.0 * k + 3.0);
                } else {                             // Fig. 9 left: one dot at a time
                    for (int l = 0; l < k; ++l) {
                        double* rl = R + l + size_t(w) * k;
                        TRY(xty_global(h, P + size_t(ldp) * l, ldp, 1, pk, ldp, 1, rl, false, nullptr));
                        kern::update(sdev(h), h->n_loc, P + size_t(ldp) * l, ldp, 1, pk, ldp, 1, rl, h->stream);
                        h->bytes[PH_TSQR] += 8.0 * nl * 5.0;
                    }
                }
            }
            double* rkk = R + k + size_t(w) * k;
            TRY(xty_global(h, pk, ldp, 1, pk, ldp, 1, h->gbuf, true, rkk));   // r_kk = ||v_k||
            if (k >= c0) kern::trsm(sdev(h), h->n_loc, pk, ldp, 1, rkk, 0, h->stream);
            h->bytes[PH_TSQR] += 8.0 * nl * (k >= c0 ? 3.0 : 1.0);
        }
    }
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

std::vector<Block> schedule(int s, int m) {
    std::vector<Block> bl;
    size_t off = 0;
    for (int j = 0; j < m;) {
        const int sb = std::min(s, m - j), w = sb + 1;
        Block b{j, sb, 0, 0, 0, 0};
        b.c1 = off; off += size_t(j) * size_t(sb);
        b.r1 = off; off += size_t(w) * size_t(w);
        b.c2 = off; off += size_t(j) * size_t(sb);
        b.r2 = off; off += size_t(w) * size_t(w);
        bl.push_back(b);
        j += sb;
    }
    return bl;
}

int diag_alloc(cagmres* h) {
    if (h->dg) return CAGMRES_OK;
    const size_t W = size_t(h->s) + 1;
    h->dg_cap = 2 * W * W * (size_t(h->m) + 1);
    CU(cudaMalloc(&h->dg, sizeof(double) * h->dg_cap));
    CU(cudaMemset(h->dg, 0, sizeof(double) * h->dg_cap));
    CU(cudaMallocHost(&h->h_dg, sizeof(double) * h->dg_cap));
    return CAGMRES_OK;
}

// Per-panel diagnostics of the cycle just copied to h_dg: max kappa_2(W^T W) and max
// ||I - Q_p^T Q_p||_2 over the blocks (Fig. 12).
void diag_reduce(cagmres* h, const std::vector<Block>& bl, double& max_orth, double& max_cond) {
    const size_t W = size_t(h->s) + 1;
    std::vector<double> ev(W), G(W * W);
    for (size_t bi = 0; bi < bl.size(); ++bi) {
        const int w = bl[bi].sb + 1;
        const double* g0 = h->h_dg + bi * 2 * W * W;
        host::sym_eigvals(g0, w, w, ev.data());
        const double cond = ev[0] > 0.0 ? ev[size_t(w - 1)] / ev[0] : INFINITY;
        max_cond = std::max(max_cond, cond);
        const double* g1 = g0 + W * W;
        for (int c = 0; c < w; ++c)
            for (int i = 0; i < w; ++i) G[size_t(i) + size_t(w) * c] = (i == c ? 1.0 : 0.0) - g1[size_t(i) + size_t(w) * c];
        host::sym_eigvals(G.data(), w, w, ev.data());
        max_orth = std::max(max_orth, std::max(std::fabs(ev[0]), std::fabs(ev[size_t(w - 1)])));
    }
}

// One CA cycle's GPU work: per block MPK -> BOrth -> TSQR [-> BOrth -> TSQR].
int ca_cycle(cagmres* h, const std::vector<Block>& bl) {
    const int kind = h->orth & CAGMRES_TSQR_MASK;
    const bool re2 = (h->orth & CAGMRES_REORTH) != 0, mgs = (h->orth & CAGMRES_BORTH_MGS) != 0;
    const size_t W2 = (size_t(h->s) + 1) * (size_t(h->s) + 1);
    size_t bi = 0;
    h->fold_kind = 0;
    for (const Block& b : bl) {
        const int j = b.j, sb = b.sb, w = sb + 1;
        const bool last_block = &b == &bl.back();
        const std::vector<host::Step> steps = h->basis == CAGMRES_MONOMIAL
            ? host::block_steps({}, {}, sb) : host::block_steps(h->sh_re, h->sh_im, sb);
        TRY(mpk_block(h, j, sb, steps));
        double* Pj = h->V + size_t(h->ldv) * j;                 // panel [q_j | W_1 .. W_sb]
        double* dgb = h->diag_on ? h->dg + 2 * W2 * bi++ : nullptr;
        if (dgb) {                                              // diagnostics: W^T W of the MPK output
            Scope sc(h, PH_OTHER);
            TRY(xty_global(h, Pj, h->ldv, w, Pj, h->ldv, w, dgb, false, nullptr));
        }
        for (int pass = 0; pass < (re2 ? 2 : 1); ++pass) {
            double* C = h->tab + (pass ? b.c2 : b.c1);
            double* R = h->tab + (pass ? b.r2 : b.r1);
            // fold this pass's panel update into x += V y (OPT_FOLD): last block, final pass
            const bool fold = h->fold && !h->diag_on && last_block && pass == (re2 ? 1 : 0);
            if (j > 0 && (h->orth & CAGMRES_ONEPASS) && j + w <= 64) {
                // one-pass BOrth + CholQR (NEXT-2): [Q P]^T P ; small step ; P := [Q P] M
                const double nl = double(h->n_loc);
                {
                    Scope sc(h, PH_BORTH);
                    TRY(xty_global(h, h->V, h->ldv, j + w, Pj, h->ldv, w, h->gbuf, false, nullptr));
                    h->bytes[PH_BORTH] += 8.0 * nl * (j + w);
                }
                Scope sc(h, PH_TSQR);
                kern::onepass_finalize(h->gbuf, j, w, C, R, h->op_M, h->status, h->stream);
                if (fold) { h->fold_kind = 2; h->fold_pass = pass; continue; }
                if (kern::gemm_rows(sdev(h), h->n_loc, h->V, h->ldv, j + w, Pj, h->ldv, w, h->op_M, j + w, 1,
                                    h->stream, true))
                    return CAGMRES_EINVAL;
                h->bytes[PH_TSQR] += 8.0 * nl * (j + w + (w - 1));
                continue;
            }
            if (j > 0 && !mgs && kind == CAGMRES_CHOLQR && h->fuse_borth_gram) {
                // BOrth pass 1, then [P -= Q C  fused with  B = [q_j P]^T [q_j P] (+ chol)]
                const double nl = double(h->n_loc);
                int fused = -1;
                {
                    Scope sc(h, PH_BORTH);
                    TRY(xty_global(h, h->V, h->ldv, j, Pj + h->ldv, h->ldv, sb, C, false, nullptr));
                    kern::UpdGramArgs ua{h->n_loc, h->V, h->ldv, j, Pj + h->ldv, h->ldv, sb, Pj, C, h->ws.part,
                                         h->gbuf, h->ws.counter, h->nranks == 1 ? 1 : 0, R, h->status};
                    fused = kern::update_gram(sdev(h), ua, h->stream);
                    if (fused == 0) h->bytes[PH_BORTH] += 8.0 * nl * (2.0 * j + 3.0 * sb);
                    else kern::update(sdev(h), h->n_loc, h->V, h->ldv, j, Pj + h->ldv, h->ldv, sb, C, h->stream);
                }
                if (fused == 0) {
                    Scope sc(h, PH_TSQR);
                    if (h->nranks > 1) {
                        TRY(allreduce(h, h->gbuf, size_t(w) * size_t(w)));
                        kern::chol(h->gbuf, w, R, h->status, h->stream);
                    }
                    if (fold) { h->fold_kind = 1; h->fold_pass = pass; continue; }
                    kern::trsm(sdev(h), h->n_loc, Pj, h->ldv, w, R, 1, h->stream);
                    h->bytes[PH_TSQR] += 8.0 * nl * (2.0 * w + double(w - 1));   // Gram bytes as if unfused
                    continue;
                }
                h->bytes[PH_BORTH] += 8.0 * nl * (2.0 * j + 3.0 * sb);
                TRY(tsqr_panel(h, Pj, h->ldv, w, R, kind, 1, (h->orth & CAGMRES_SVQR_RETRY) != 0, fold));
                if (fold) { h->fold_kind = 1; h->fold_pass = pass; }
                continue;
            }
            TRY(borth_panel(h, h->V, h->ldv, j, Pj + h->ldv, h->ldv, sb, C, mgs));
            const bool fold_tsqr = fold && (kind == CAGMRES_CHOLQR || kind == CAGMRES_SVQR);
            TRY(tsqr_panel(h, Pj, h->ldv, w, R, kind, 1, (h->orth & CAGMRES_SVQR_RETRY) != 0, fold_tsqr));
            if (fold_tsqr) { h->fold_kind = 1; h->fold_pass = pass; }
        }
        if (dgb) {                                              // ... and Q_p^T Q_p after the passes
            Scope sc(h, PH_OTHER);
            TRY(xty_global(h, Pj, h->ldv, w, Pj, h->ldv, w, dgb + W2, false, nullptr));
        }
    }
    return CAGMRES_OK;
}

// First Newton cycle = GMRES(m) with CGS Arnoldi, CGS2 with CAGMRES_REORTH (Fig. 14,
// DESIGN.md reading G12), on the same kernels with panel width 1; also the GMRES baseline.
// tab layout: per k: c1 (m+1), c2 (m+1, unused for CGS), r (1).
int arnoldi_cycle(cagmres* h, bool cgs2) {
    const int m = h->m;
    const size_t stride = 2 * size_t(m + 1) + 1;
    for (int k = 0; k < m; ++k) {
        double* vk = h->V + size_t(h->ldv) * k;
        double* v = h->V + size_t(h->ldv) * (k + 1);
        double* c1 = h->tab + stride * k;
        double* c2 = c1 + (m + 1);
        double* r = c2 + (m + 1);
        {
            Scope sc(h, PH_MPK);
            bool fused_q = false;
            TRY(start_halo(h, k, 1, fused_q));
            Scope sv(h, PH_SPMV);
            if (fused_q) {                 // v_k = S / ||S|| formed inside the SpMV (stored to V[:, k])
                if (kern::spmv_scaled(sdev(h), h->A, h->n_loc, h->S, h->pend_nrm, vk, v, 0.0, false, h->stream))
                    return CAGMRES_EINVAL;
                h->pend = false;
            } else {
                kern::spmv(sdev(h), h->A, h->n_loc, vk, v, nullptr, 0.0, nullptr, 0.0, h->stream);
            }
            const double by = spmv_bytes(h, h->n_loc, 1, false);
            h->bytes[PH_MPK] += by; h->bytes[PH_SPMV] += by; h->spmv_launches++;
        }
        if (h->arnoldi_fuse && k + 1 <= 32) {
            // c1 = Q^T v ; [v -= Q c1, c2 = Q^T v] ; [v -= Q c2, r = ||v||] ; v /= r
            const double nl = double(h->n_loc);
            kern::ArnoldiArgs aa{h->dev.panel_pf, h->n_loc, h->V, h->ldv, k + 1, v, nullptr, nullptr, h->arn_part,
                                 h->arn_counter, h->status, h->nranks == 1 ? 1 : 0};
            {
                Scope sc(h, PH_BORTH);
                aa.c_out = c1;
                if (kern::arnoldi_fused(sdev(h), aa, 0, h->stream)) return CAGMRES_EINVAL;
                TRY(allreduce(h, c1, size_t(k + 1)));
                if (cgs2) {
                    aa.c_in = c1; aa.c_out = c2;
                    if (kern::arnoldi_fused(sdev(h), aa, 1, h->stream)) return CAGMRES_EINVAL;
                    TRY(allreduce(h, c2, size_t(k + 1)));
                    h->bytes[PH_BORTH] += 8.0 * nl * (3.0 * (k + 1) + 4.0);
                } else {
                    h->bytes[PH_BORTH] += 8.0 * nl * ((k + 1) + 1.0);
                }
            }
            {
                Scope sc(h, PH_TSQR);
                aa.c_in = cgs2 ? c2 : c1; aa.c_out = r;
                aa.vout = h->fuse_scale ? h->S : nullptr;          // w -> S, normalised by the next SpMV
                if (kern::arnoldi_fused(sdev(h), aa, 2, h->stream)) return CAGMRES_EINVAL;
                aa.vout = nullptr;
                if (h->nranks > 1) {
                    TRY(allreduce(h, r, 1));
                    kern::chol(r, 1, r, h->status, h->stream);     // r = sqrt(r)
                }
                if (h->fuse_scale) {
                    h->pend = true; h->pend_nrm = r; h->pend_col = k + 1;
                    h->bytes[PH_TSQR] += 8.0 * nl * ((k + 1) + 2.0);
                } else {
                    kern::trsm(h->dev, h->n_loc, v, h->ldv, 1, r, 0, h->stream);   // (w = 1: no sweep order)
                    h->bytes[PH_TSQR] += 8.0 * nl * ((k + 1) + 2.0 + 2.0);
                }
            }
            continue;
        }
        TRY(borth_panel(h, h->V, h->ldv, k + 1, v, h->ldv, 1, c1, false));
        if (cgs2) TRY(borth_panel(h, h->V, h->ldv, k + 1, v, h->ldv, 1, c2, false));
        TRY(tsqr_panel(h, v, h->ldv, 1, r, CAGMRES_CHOLQR, 0));
    }
    h->pend = false;                       // V[:, m] (unnormalised, in S) is never read
    return CAGMRES_OK;
}

// residual r = b - A x into V[:,0]; returns ||r|| (host) and leaves r/||r|| in V[:,0].
// r = b - A x into V[:,0], beta = ||r|| (device), V[:,0] = r / beta, and an async copy of
// beta to the pinned h_beta followed by ev_beta — the caller waits only when it needs beta.
int residual_norm_async(cagmres* h, const double* b, const double* x) {
    Scope sc(h, PH_OTHER);
    const double* xx = x;
    if (h->nranks > 1) {
        CU(cudaMemcpyAsync(h->xe, x, sizeof(double) * size_t(h->n_loc), cudaMemcpyDeviceToDevice, h->stream));
        TRY(halo(h, h->xe, 1));
        xx = h->xe;
    }
    double* rv = h->fuse_scale ? h->S : h->V;          // r: unnormalised in S (fused) or in V[:, 0]
    kern::residual(sdev(h), h->A, h->n_loc, xx, b, rv, h->stream);
    double* rr = h->gbuf + 8;
    {   // ||r|| by the scalar reduction kernel (mode 2 with no Q columns)
        kern::ArnoldiArgs aa{h->dev.panel_pf, h->n_loc, h->V, h->ldv, 0, rv, nullptr, rr, h->arn_part, h->arn_counter,
                             h->status, h->nranks == 1 ? 1 : 0};
        if (kern::arnoldi_fused(sdev(h), aa, 2, h->stream)) return CAGMRES_EINVAL;
        if (h->nranks > 1) {
            TRY(allreduce(h, rr, 1));
            kern::chol(rr, 1, rr, h->status, h->stream);
        }
    }
    CU(cudaMemcpyAsync(h->h_beta, rr, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    CU(cudaEventRecord(h->ev_beta, h->stream));
    if (h->fuse_scale) {                                   // q_0 = r / beta formed by the next SpMV
        h->pend = true; h->pend_nrm = rr; h->pend_col = 0;
        h->bytes[PH_OTHER] += spmv_bytes(h, h->n_loc, 1, false) + 8.0 * double(h->n_loc);
    } else {
        kern::trsm(h->dev, h->n_loc, h->V, h->ldv, 1, rr, 0, h->stream);     // q_0 = r / beta (w = 1)
        h->bytes[PH_OTHER] += spmv_bytes(h, h->n_loc, 1, false) + 8.0 * double(h->n_loc) * 3.0;
    }
    return cudaGetLastError() == cudaSuccess ? CAGMRES_OK : CAGMRES_ECUDA;
}

// One restart cycle's GPU work plus the async copy of its coefficient table and status.
int enqueue_cycle(cagmres* h, bool arnoldi, const std::vector<Block>& bl) {
    h->dev.rev = 1;                        // the cycle's first streaming launch sweeps forward
    if (arnoldi) {
        // standard GMRES as the paper runs it: CGS Arnoldi (Fig. 14 "GMRES ... CGS" rows), CGS2
        // with CAGMRES_REORTH — for the shift-finding Newton cycle (G12) and the baseline
        TRY(arnoldi_cycle(h, (h->orth & CAGMRES_REORTH) != 0));
    } else {
        TRY(ca_cycle(h, bl));
    }
    CU(cudaMemcpyAsync(h->h_tab, h->tab, sizeof(double) * h->tab_cap, cudaMemcpyDeviceToHost, h->stream));
    if (h->diag_on && !arnoldi)
        CU(cudaMemcpyAsync(h->h_dg, h->dg, sizeof(double) * h->dg_cap, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaMemcpyAsync(h->h_stat, h->status, sizeof(int) * 2, cudaMemcpyDeviceToHost, h->stream));
    // under stream capture the record must become an external event node of the graph, so the
    // host can wait on it after each replay (a plain record is a capture-internal dependency)
    if (h->capturing) CU(cudaEventRecordWithFlags(h->ev_tab, h->stream, cudaEventRecordExternal));
    else CU(cudaEventRecord(h->ev_tab, h->stream));
    return CAGMRES_OK;
}

// One CA cycle through a CUDA graph (single rank; no timing events, diagnostics or temporally
// blocked MPK — their host-side state changes per launch): the cycle's ~45 launches, table
// copies and ev_tab record are captured on a private stream once per configuration and the
// executable graph is replayed on the handle's stream.  Programmatic dependent launch edges are
// kept by the capture.  Host-side accounting (algorithmic bytes, launch counts, the pending
// normalisation) is replayed from the capture's deltas.
bool graph_ok(const cagmres* h) {
    return h->use_graphs && h->nranks == 1 && !h->timer.on && !h->diag_on && !h->wave_on && !h->sweep_on &&
           (!h->pend || (h->pend_col == 0 && h->pend_nrm == h->gbuf + 8));
}

int enqueue_ca_cycle(cagmres* h, const std::vector<Block>& bl) {
    if (!graph_ok(h)) return enqueue_cycle(h, false, bl);
    const uint64_t key = h->cfg_version * 2 + (h->pend ? 1 : 0);   // the entry state is part of the graph
    if (h->cyc_exec == nullptr || h->cyc_version != key) {
        if (h->cyc_exec) { cudaGraphExecDestroy(h->cyc_exec); h->cyc_exec = nullptr; }
        if (!h->cap_stream) CU(cudaStreamCreateWithFlags(&h->cap_stream, cudaStreamNonBlocking));
        double b0[PH_N];
        std::memcpy(b0, h->bytes, sizeof(b0));
        const int s0 = h->spmv_launches;
        const long long l0 = kern::g_launches;
        cudaStream_t saved = h->stream;
        const bool pend0 = h->pend;
        h->stream = h->cap_stream;
        h->capturing = true;
        cudaError_t ce = cudaStreamBeginCapture(h->cap_stream, cudaStreamCaptureModeThreadLocal);
        int rc = ce == cudaSuccess ? enqueue_cycle(h, false, bl) : CAGMRES_ECUDA;
        cudaGraph_t g = nullptr;
        if (ce == cudaSuccess) ce = cudaStreamEndCapture(h->cap_stream, &g);
        h->capturing = false;
        h->stream = saved;
        if (rc == CAGMRES_OK && ce == cudaSuccess) {
            ce = cudaGraphInstantiate(&h->cyc_exec, g, 0);
            if (ce != cudaSuccess) h->cyc_exec = nullptr;
        }
        if (g) cudaGraphDestroy(g);
        if (rc != CAGMRES_OK || ce != cudaSuccess) {
            // capture not possible here: remember why, restore the host state, launch eagerly
            h->graph_err = ce != cudaSuccess ? int(ce) : -1;
            cudaGetLastError();
            std::memcpy(h->bytes, b0, sizeof(b0));
            h->spmv_launches = s0;
            kern::g_launches = l0;
            h->pend = pend0;
            h->use_graphs = false;
            return enqueue_cycle(h, false, bl);
        }
        for (int p = 0; p < PH_N; ++p) { h->cyc_bytes[p] = h->bytes[p] - b0[p]; h->bytes[p] = b0[p]; }
        h->cyc_spmv = h->spmv_launches - s0;
        h->spmv_launches = s0;
        h->cyc_launches = kern::g_launches - l0;
        kern::g_launches = l0;
        h->cyc_rev_end = h->dev.rev;
        h->cyc_version = key;
    }
    CU(cudaGraphLaunch(h->cyc_exec, h->stream));
    h->dev.rev = h->cyc_rev_end;           // the sweep state a stream-launched cycle ends in
    for (int p = 0; p < PH_N; ++p) h->bytes[p] += h->cyc_bytes[p];
    h->spmv_launches += h->cyc_spmv;
    kern::g_launches += h->cyc_launches;
    h->pend = false;                       // consumed by the cycle's first SpMV
    return CAGMRES_OK;
}

void collect_timing(cagmres* h, cagmres_stats* st) {
    double ms[PH_N] = {0, 0, 0, 0, 0};
    for (auto& r : h->timer.rec) {
        float t = 0.f;
        cudaEventElapsedTime(&t, r.second.first, r.second.second);
        ms[r.first] += double(t);
    }
    st->ms_mpk = ms[PH_MPK]; st->ms_borth = ms[PH_BORTH]; st->ms_tsqr = ms[PH_TSQR];
    st->ms_other = ms[PH_OTHER]; st->ms_spmv = ms[PH_SPMV];
    h->timer.reset();
}

}  // namespace

// =======================================================================================
// C ABI
// =======================================================================================
extern "C" {

const char* cagmres_strerror(int s) {
    switch (s) {
        case CAGMRES_OK: return "ok";
        case CAGMRES_NOT_CONVERGED: return "not converged within maxit restart cycles";
        case CAGMRES_EINVAL: return "invalid argument";
        case CAGMRES_ECUDA: return "CUDA error";
        case CAGMRES_ENCCL: return "communication error (NCCL call or in-process group collective failed)";
        case CAGMRES_EBREAKDOWN: return "numerical breakdown (Cholesky pivot <= 0 / zero norm)";
        case CAGMRES_ENOMEM: return "out of memory";
        case CAGMRES_EGHOST: return "supplied rows do not cover the ghost rows";
        case CAGMRES_ENOTSUP: return "option not supported by this build";
        default: return "unknown status";
    }
}

int64_t cagmres_kernel_launches(void) { return int64_t(kern::g_launches); }

int cagmres_create(cagmres_t* out, const cagmres_csr* A, int s, int m, int basis, int orth) {
    if (!out || !A) return CAGMRES_EINVAL;
    *out = nullptr;
    if (A->row_begin != 0 || A->row_end != A->n || A->own_begin != 0 || A->own_end != A->n)
        return CAGMRES_EINVAL;
    cagmres* h = new (std::nothrow) cagmres();
    if (!h) return CAGMRES_ENOMEM;
    const int64_t rs[2] = {0, A->n};
    const int st = init_common(h, A, rs, s, m, basis, orth);
    if (st != CAGMRES_OK) { delete h; return st; }
    *out = h;
    return CAGMRES_OK;
}

int cagmres_create_dist(cagmres_t* out, const cagmres_csr* A, const int64_t* row_starts,
                        int s, int m, int basis, int orth, const void* nccl_unique_id,
                        int rank, int nranks, int cuda_device) {
    if (!out || !A || !row_starts || !nccl_unique_id || nranks < 1 || rank < 0 || rank >= nranks)
        return CAGMRES_EINVAL;
    *out = nullptr;
    if (cudaSetDevice(cuda_device) != cudaSuccess) return CAGMRES_ECUDA;
    cagmres* h = new (std::nothrow) cagmres();
    if (!h) return CAGMRES_ENOMEM;
    h->rank = rank; h->nranks = nranks;
    if (nranks > 1) {
        h->tr.reset(make_nccl_transport(nccl_unique_id, rank, nranks));
        if (!h->tr) { delete h; return CAGMRES_ENCCL; }
    }
    const int st = init_common(h, A, row_starts, s, m, basis, orth);
    if (st != CAGMRES_OK) { delete h; return st; }
    *out = h;
    return CAGMRES_OK;
}

int cagmres_create_group(cagmres_t* out, const cagmres_csr* A, const int64_t* row_starts,
                         int s, int m, int basis, int orth, cagmres_group_t g, int rank) {
    if (!out || !A || !row_starts || !g || rank < 0 || rank >= g->P) return CAGMRES_EINVAL;
    *out = nullptr;
    if (cudaSetDevice(g->device[size_t(rank)]) != cudaSuccess) return CAGMRES_ECUDA;
    cagmres* h = new (std::nothrow) cagmres();
    if (!h) return CAGMRES_ENOMEM;
    h->rank = rank; h->nranks = g->P;
    if (g->P > 1) {
        h->tr.reset(make_group_transport(g, rank));
        if (!h->tr) { delete h; return CAGMRES_ENCCL; }
    }
    const int st = init_common(h, A, row_starts, s, m, basis, orth);
    if (st != CAGMRES_OK) { delete h; return st; }
    *out = h;
    return CAGMRES_OK;
}

int cagmres_destroy(cagmres_t h) {
    if (!h) return CAGMRES_OK;
    cudaStreamSynchronize(h->stream);
    delete h;
    return CAGMRES_OK;
}

int cagmres_set_stream(cagmres_t h, void* s) {
    if (!h) return CAGMRES_EINVAL;
    h->stream = s ? static_cast<cudaStream_t>(s) : h->own_stream;
    return CAGMRES_OK;
}

int cagmres_set_option(cagmres_t h, int opt, int64_t value) {
    if (!h) return CAGMRES_EINVAL;
    ++h->cfg_version;                      // any option may change the captured cycle
    switch (opt) {
        case CAGMRES_OPT_MPK_WAVE:
            if (value < 0 || value > 3) return CAGMRES_EINVAL;
            h->wave_on = value == 1 || value == 2; h->wave_force = value == 2; h->sweep_on = value == 3;
            if (h->sweep_on && !h->sweep_bar) {
                CU(cudaMalloc(&h->sweep_bar, sizeof(unsigned)));
                CU(cudaMemset(h->sweep_bar, 0, sizeof(unsigned)));
                h->sweep_base = 0;
            }
            return CAGMRES_OK;
        case CAGMRES_OPT_SPMV:
            if (value != -1 && value != 0 && value != 5 && value != 16 && value != 17) return CAGMRES_EINVAL;
            if (value == -1) return spmv_autotune(h);
            h->A.variant = int(value);
            return CAGMRES_OK;
        case CAGMRES_OPT_GRAM: if (value < 0 || value > 2) return CAGMRES_EINVAL; h->dev.gram = int(value); return CAGMRES_OK;
        case CAGMRES_OPT_ARNOLDI: if (value < 0 || value > 1) return CAGMRES_EINVAL; h->dev.arnoldi_ring = int(value); return CAGMRES_OK;
        case CAGMRES_OPT_PANEL_TW: if (value != 16 && value != 32) return CAGMRES_EINVAL; h->dev.panel_tw16 = value == 16; return CAGMRES_OK;
        case CAGMRES_OPT_TRSM: if (value < 0 || value > 4) return CAGMRES_EINVAL; h->dev.trsm_scalar = int(value); return CAGMRES_OK;
        case CAGMRES_OPT_PDL: if (value < 0 || value > 1) return CAGMRES_EINVAL; kern::g_pdl = int(value); return CAGMRES_OK;
        case CAGMRES_OPT_PANEL_PF: if (value < 0 || value > 1) return CAGMRES_EINVAL; h->dev.panel_pf = int(value); return CAGMRES_OK;
        case CAGMRES_OPT_GRAPH:
            if (value < 0 || value > 1) return CAGMRES_EINVAL;
            h->use_graphs = value != 0;
            return CAGMRES_OK;
        case CAGMRES_OPT_PEER:
            if (value < 0 || value > 1) return CAGMRES_EINVAL;
            h->peer_pull = value != 0;
            h->peer_ok = h->tr && h->tr->peer_capable() && h->peer_pull;
            return CAGMRES_OK;
        case CAGMRES_OPT_FUSE:
            h->fuse_borth_gram = (value & 1) != 0; h->arnoldi_fuse = (value & 2) != 0; h->fuse_scale = (value & 4) != 0;
            return CAGMRES_OK;
        case CAGMRES_OPT_FOLD: if (value < 0 || value > 1) return CAGMRES_EINVAL; h->fold = value != 0; return CAGMRES_OK;
        case CAGMRES_OPT_SERP: if (value < 0 || value > 1) return CAGMRES_EINVAL; h->serp = value != 0; return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_CHUNK:
            if (value < 256 || value % 256) return CAGMRES_EINVAL;
            h->wave_CH = int(value); wave_reset_pairs(h); return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_CTAS: h->wave_ctas = int(value); wave_reset_pairs(h); return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_LAG: h->wave_lag = int(value); wave_reset_pairs(h); return CAGMRES_OK;
        default: return CAGMRES_EINVAL;
    }
}

int cagmres_get_option(cagmres_t h, int opt, int64_t* value) {
    if (!h || !value) return CAGMRES_EINVAL;
    switch (opt) {
        case CAGMRES_OPT_MPK_WAVE: *value = h->sweep_on ? 3 : (h->wave_on ? (h->wave_force ? 2 : 1) : 0); return CAGMRES_OK;
        case CAGMRES_OPT_SPMV: *value = h->A.variant; return CAGMRES_OK;
        case CAGMRES_OPT_GRAM: *value = h->dev.gram; return CAGMRES_OK;
        case CAGMRES_OPT_ARNOLDI: *value = h->dev.arnoldi_ring; return CAGMRES_OK;
        case CAGMRES_OPT_PANEL_TW: *value = h->dev.panel_tw16 ? 16 : 32; return CAGMRES_OK;
        case CAGMRES_OPT_TRSM: *value = h->dev.trsm_scalar; return CAGMRES_OK;
        case CAGMRES_OPT_PDL: *value = kern::g_pdl; return CAGMRES_OK;
        case CAGMRES_OPT_PANEL_PF: *value = h->dev.panel_pf; return CAGMRES_OK;
        case CAGMRES_OPT_PEER: *value = h->peer_ok ? 1 : 0; return CAGMRES_OK;
        case CAGMRES_OPT_GRAPH: *value = h->graph_err ? -int64_t(h->graph_err) : (h->use_graphs ? 1 : 0); return CAGMRES_OK;
        case CAGMRES_OPT_FUSE:
            *value = (h->fuse_borth_gram ? 1 : 0) | (h->arnoldi_fuse ? 2 : 0) | (h->fuse_scale ? 4 : 0);
            return CAGMRES_OK;
        case CAGMRES_OPT_FOLD: *value = h->fold ? 1 : 0; return CAGMRES_OK;
        case CAGMRES_OPT_SERP: *value = h->serp ? 1 : 0; return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_CHUNK: *value = h->wave_CH; return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_CTAS: *value = h->wave_ctas; return CAGMRES_OK;
        case CAGMRES_OPT_WAVE_LAG: *value = h->wave_lag; return CAGMRES_OK;
        default: return CAGMRES_EINVAL;
    }
}

int cagmres_sizes(cagmres_t h, int64_t* n_loc, int64_t* n_ext, int64_t* ldv) {
    if (!h) return CAGMRES_EINVAL;
    if (n_loc) *n_loc = h->n_loc;
    if (n_ext) *n_ext = h->n_ext;
    if (ldv) *ldv = h->ldv;
    return CAGMRES_OK;
}

int cagmres_set_shifts(cagmres_t h, const double* re, const double* im, int count) {
    if (!h || count < 0) return CAGMRES_EINVAL;
    if (count == 0) {                        // forget the shifts: the next Newton solve starts
        h->sh_re.clear();                    // with the GMRES cycle again
        h->sh_im.clear();
        h->have_shifts = false;
        ++h->cfg_version;
        return CAGMRES_OK;
    }
    if (!re || !im) return CAGMRES_EINVAL;
    for (int k = 0; k < count; ++k) {
        if (im[k] > 0.0 && k + 1 < count && !(re[k + 1] == re[k] && im[k + 1] == -im[k])) return CAGMRES_EINVAL;
        if (im[k] < 0.0 && (k == 0 || !(re[k - 1] == re[k] && im[k - 1] == -im[k]))) return CAGMRES_EINVAL;
    }
    h->sh_re.assign(re, re + count);
    h->sh_im.assign(im, im + count);
    h->have_shifts = true;
    ++h->cfg_version;
    return CAGMRES_OK;
}

int cagmres_get_shifts(cagmres_t h, double* re, double* im, int cap, int* count) {
    if (!h || !count) return CAGMRES_EINVAL;
    *count = h->have_shifts ? int(h->sh_re.size()) : 0;
    for (int k = 0; k < std::min(cap, *count); ++k) { re[k] = h->sh_re[size_t(k)]; im[k] = h->sh_im[size_t(k)]; }
    return CAGMRES_OK;
}

int cagmres_mpk(cagmres_t h, const double* q, double* W, int64_t ldw, int sb) {
    if (!h || !q || !W || sb < 1 || sb > h->s || ldw < h->n_loc || sb > h->m) return CAGMRES_EINVAL;
    if (h->basis == CAGMRES_NEWTON && !h->have_shifts) return CAGMRES_EINVAL;
    h->pend = false;
    h->dev.rev = 1;                        // sweep order restarts with every call (deterministic)
    CU(cudaMemcpyAsync(h->V, q, sizeof(double) * size_t(h->n_loc), cudaMemcpyDeviceToDevice, h->stream));
    const std::vector<host::Step> steps = h->basis != CAGMRES_NEWTON
        ? host::block_steps({}, {}, sb) : host::block_steps(h->sh_re, h->sh_im, sb);
    TRY(mpk_block(h, 0, sb, steps));
    CU(cudaMemcpy2DAsync(W, sizeof(double) * size_t(ldw), h->V, sizeof(double) * size_t(h->ldv),
                         sizeof(double) * size_t(h->n_loc), size_t(sb) + 1, cudaMemcpyDeviceToDevice, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    h->timer.reset();
    return CAGMRES_OK;
}

int cagmres_borth(cagmres_t h, const double* Q, int64_t ldq, int j, double* P, int64_t ldp,
                  int w, double* C) {
    if (!h || j < 0 || w < 1 || w > 32 || ldq < h->n_loc || ldp < h->n_loc) return CAGMRES_EINVAL;
    if (j == 0) return CAGMRES_OK;
    if (!Q || !P || !C || j > int(h->tab_cap)) return CAGMRES_EINVAL;
    h->dev.rev = 1;
    TRY(borth_panel(h, Q, ldq, j, P, ldp, w, C, (h->orth & CAGMRES_BORTH_MGS) != 0));
    CU(cudaStreamSynchronize(h->stream));
    h->timer.reset();
    return CAGMRES_OK;
}

int cagmres_tsqr(cagmres_t h, double* P, int64_t ldp, int w, double* R, int orth) {
    if (!h || !P || !R || w < 1 || w > 32 || ldp < h->n_loc) return CAGMRES_EINVAL;
    const int kind = orth & CAGMRES_TSQR_MASK;
    if (kind > CAGMRES_CAQR) return CAGMRES_EINVAL;
    CU(cudaMemsetAsync(h->status, 0, sizeof(int), h->stream));
    const bool retry = (orth & CAGMRES_SVQR_RETRY) && kind == CAGMRES_CHOLQR;
    CU(cudaMemsetAsync(h->status, 0, sizeof(int) * 2, h->stream));
    h->dev.rev = 1;
    TRY(tsqr_panel(h, P, ldp, w, R, kind, 0, retry));
    if (orth & CAGMRES_REORTH) {
        double* R2 = h->tab;                        // scratch
        TRY(tsqr_panel(h, P, ldp, w, R2, kind, 0, retry));
        std::vector<double> r1(size_t(w) * w), r2(size_t(w) * w), rr(size_t(w) * w, 0.0);
        CU(cudaMemcpyAsync(r1.data(), R, sizeof(double) * r1.size(), cudaMemcpyDeviceToHost, h->stream));
        CU(cudaMemcpyAsync(r2.data(), R2, sizeof(double) * r2.size(), cudaMemcpyDeviceToHost, h->stream));
        CU(cudaStreamSynchronize(h->stream));
        for (int c = 0; c < w; ++c)
            for (int i = 0; i <= c; ++i) {
                double a = 0.0;
                for (int k = i; k <= c; ++k) a += r2[size_t(i) + size_t(w) * k] * r1[size_t(k) + size_t(w) * c];
                rr[size_t(i) + size_t(w) * c] = a;
            }
        CU(cudaMemcpyAsync(R, rr.data(), sizeof(double) * rr.size(), cudaMemcpyHostToDevice, h->stream));
    }
    int stat = 0;
    CU(cudaMemcpyAsync(&stat, h->status, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    h->timer.reset();
    return stat ? CAGMRES_EBREAKDOWN : CAGMRES_OK;
}

int cagmres_solve(cagmres_t h, const double* b, double* x, double tol, int maxit, cagmres_stats* st) {
    if (!h || !b || !x || maxit < 0 || !(tol >= 0.0)) return CAGMRES_EINVAL;
    const NvtxRange solve_range("cagmres_solve");
    const int m = h->m;
    h->timer.reset();
    h->timer.on = st && st->collect_timing;
    h->timer.light = st && st->collect_timing == 2;
    for (double& v : h->bytes) v = 0.0;
    h->spmv_launches = 0;
    if (st) { st->cycles = 0; st->iters = 0; st->hist_len = 0; }
    cudaEvent_t t0 = nullptr, t1 = nullptr;
    if (h->timer.on) { t0 = h->timer.get(); cudaEventRecord(t0, h->stream); }
    CU(cudaMemsetAsync(h->status, 0, sizeof(int) * 2, h->stream));
    h->h_stat[1] = 0;
    h->diag_on = st && st->collect_diag;
    double max_orth = 0.0, max_cond = 0.0;
    if (h->diag_on) TRY(diag_alloc(h));
    double rho0 = 0.0, beta = 0.0;
    h->dev.rev = 1;                        // sweep order: every solve starts the same way
    TRY(residual_norm_async(h, b, x));
    CU(cudaEventSynchronize(h->ev_beta));
    rho0 = *h->h_beta;
    beta = rho0;
    int rc = CAGMRES_NOT_CONVERGED;
    if (rho0 == 0.0) rc = CAGMRES_OK;
    std::vector<double> H(static_cast<size_t>(m + 1) * static_cast<size_t>(m)), y(static_cast<size_t>(m)),
        res(static_cast<size_t>(m));
    const double* htab = h->h_tab;
    const std::vector<Block> bl = schedule(h->s, m);
    int cyc = 0;
    bool pending = false;                    // next cycle already enqueued (speculation)
    for (; cyc < maxit && rc != CAGMRES_OK; ++cyc) {
        const bool first_newton = h->basis == CAGMRES_NEWTON && !h->have_shifts;
        const bool arnoldi = first_newton || h->basis == CAGMRES_GMRES;
        char rname[48];
        snprintf(rname, sizeof rname, "restart cycle %d (%s)", cyc + 1, arnoldi ? "GMRES" : "CA");
        const NvtxRange cycle_range(rname);
        const bool cgs2 = (h->orth & CAGMRES_REORTH) != 0;
        std::fill(H.begin(), H.end(), 0.0);
        if (!pending) TRY(arnoldi ? enqueue_cycle(h, true, bl) : enqueue_ca_cycle(h, bl));
        pending = false;
        CU(cudaEventSynchronize(h->ev_tab));
        if (*h->h_stat) { rc = CAGMRES_EBREAKDOWN; break; }
        if (h->diag_on && !arnoldi) diag_reduce(h, bl, max_orth, max_cond);
        // ---- Hessenberg matrix (host) ----
        if (arnoldi) {
            const size_t stride = 2 * size_t(m + 1) + 1;
            for (int k = 0; k < m; ++k) {
                const double* c1 = htab + stride * k;
                for (int i = 0; i <= k; ++i) H[size_t(i) + size_t(m + 1) * k] = c1[i] + (cgs2 ? c1[i + m + 1] : 0.0);
                H[size_t(k + 1) + size_t(m + 1) * k] = c1[2 * (m + 1)];
            }
        } else {
            const bool re2 = (h->orth & CAGMRES_REORTH) != 0;
            for (const Block& b0 : bl) {
                const int j = b0.j, sb = b0.sb, w = sb + 1, nr = j + sb + 1;
                std::vector<double> Rt(size_t(nr) * size_t(w), 0.0);
                const double* C1 = htab + b0.c1;
                const double* R1 = htab + b0.r1;
                for (int c = 0; c < w; ++c) {
                    for (int i = 0; i < j; ++i) Rt[size_t(i) + size_t(nr) * c] = c == 0 ? 0.0 : C1[size_t(i) + size_t(j) * (c - 1)];
                    for (int i = 0; i <= c; ++i) Rt[size_t(j + i) + size_t(nr) * c] = R1[size_t(i) + size_t(w) * c];
                }
                if (re2) {   // C = C1 + C2 R1, R = R2 R1 (reading G16)
                    const double* C2 = htab + b0.c2;
                    const double* R2 = htab + b0.r2;
                    std::vector<double> Rn(size_t(nr) * size_t(w), 0.0);
                    for (int c = 0; c < w; ++c) {
                        for (int i = 0; i < j; ++i) {
                            double a = Rt[size_t(i) + size_t(nr) * c];
                            for (int k = 1; k <= c; ++k) a += C2[size_t(i) + size_t(j) * (k - 1)] * R1[size_t(k) + size_t(w) * c];
                            Rn[size_t(i) + size_t(nr) * c] = a;
                        }
                        for (int i = 0; i <= c; ++i) {
                            double a = 0.0;
                            for (int k = i; k <= c; ++k) a += R2[size_t(i) + size_t(w) * k] * R1[size_t(k) + size_t(w) * c];
                            Rn[size_t(j + i) + size_t(nr) * c] = a;
                        }
                    }
                    Rt.swap(Rn);
                }
                const std::vector<host::Step> steps = h->basis == CAGMRES_MONOMIAL
                    ? host::block_steps({}, {}, sb) : host::block_steps(h->sh_re, h->sh_im, sb);
                std::vector<double> B(size_t(w) * size_t(sb));
                host::change_of_basis(steps, sb, B.data());
                if (host::hessenberg_update(H.data(), m + 1, j, sb, Rt.data(), nr, B.data()) != CAGMRES_OK) {
                    rc = CAGMRES_EBREAKDOWN;
                    break;
                }
            }
            if (rc == CAGMRES_EBREAKDOWN) break;
        }
        // ---- least squares + solution update ----
        if (host::givens_ls(H.data(), m + 1, m, beta, y.data(), res.data()) != CAGMRES_OK) { rc = CAGMRES_EBREAKDOWN; break; }
        int ncoef = m;
        for (int i = 0; i < m; ++i) h->h_y[i] = -y[size_t(i)];    // update() subtracts X C
        if (!arnoldi && h->fold_kind) {
            // OPT_FOLD: the last block's columns j+1..j+sb of V still hold the panel P (BOrth-
            // updated); Q_new[:, c] = (P R^{-1})[:, c] (c >= 1), or ([Q P] Mo)[:, c] with
            // Mo = [-Cf R^{-1}; R^{-1}] for one-pass.  So Q_new y_new = P z (- Q Cf z), with
            // z = R^{-1} [0; y_{j+1..j+sb}] (y_m := 0: the last column is not in the LS).
            const Block& b0 = bl.back();
            const int j = b0.j, sb = b0.sb, w = sb + 1;
            const double* Rf = htab + (h->fold_pass ? b0.r2 : b0.r1);
            std::vector<double> z(size_t(w), 0.0);
            for (int c = 1; c < w; ++c) z[size_t(c)] = j + c < m ? y[size_t(j + c)] : 0.0;
            for (int k = w - 1; k >= 0; --k) {                  // back substitution R z = [0; y]
                double a = z[size_t(k)];
                for (int l = k + 1; l < w; ++l) a -= Rf[size_t(k) + size_t(w) * l] * z[size_t(l)];
                z[size_t(k)] = a / Rf[size_t(k) + size_t(w) * k];
            }
            for (int k = 0; k < w; ++k) h->h_y[j + k] = (k == 0 ? -y[size_t(j)] : 0.0) - z[size_t(k)];
            if (h->fold_kind == 2) {
                const double* Cf = htab + (h->fold_pass ? b0.c2 : b0.c1);   // C[i, c-1], ld j
                for (int i = 0; i < j; ++i) {
                    double a = 0.0;
                    for (int c = 1; c < w; ++c) a += Cf[size_t(i) + size_t(j) * (c - 1)] * z[size_t(c)];
                    h->h_y[i] += a;
                }
            }
            ncoef = j + w;                                       // = m + 1
        }
        {
            Scope sc(h, PH_OTHER);
            CU(cudaMemcpyAsync(h->ybuf, h->h_y, sizeof(double) * size_t(ncoef), cudaMemcpyHostToDevice, h->stream));
            kern::update(sdev(h), h->n_loc, h->V, h->ldv, ncoef, x, h->n_loc, 1, h->ybuf, h->stream);
            h->bytes[PH_OTHER] += 8.0 * double(h->n_loc) * (ncoef + 2.0);
        }
        TRY(residual_norm_async(h, b, x));                        // r, beta, q_0 for the next cycle
        if (first_newton) {                                      // Ritz values -> Leja shifts
            std::vector<double> wr(static_cast<size_t>(m)), wi(static_cast<size_t>(m));
            if (host::hessenberg_eigvals(H.data(), m + 1, m, wr.data(), wi.data()) != CAGMRES_OK) { rc = CAGMRES_EBREAKDOWN; break; }
            host::modified_leja(wr.data(), wi.data(), m, h->s, h->sh_re, h->sh_im);
            h->have_shifts = true;
            ++h->cfg_version;
        }
        // Speculate: the next cycle needs only the device-resident q_0, so enqueue it before
        // waiting for beta unless the least-squares residual estimate says this cycle has
        // (almost) converged — hides the host round trip of the convergence test.
        if (cyc + 1 < maxit && res[size_t(m - 1)] > 2.0 * tol * rho0) {
            TRY(h->basis == CAGMRES_GMRES ? enqueue_cycle(h, true, bl) : enqueue_ca_cycle(h, bl));
            pending = true;
        }
        CU(cudaEventSynchronize(h->ev_beta));
        const double rho = *h->h_beta;
        beta = rho;
        if (st && st->rel_resid_hist && st->hist_len < st->hist_cap)
            st->rel_resid_hist[st->hist_len++] = rho0 > 0.0 ? rho / rho0 : 0.0;
        if (rho <= tol * rho0) rc = CAGMRES_OK;
    }
    if (h->timer.on) { t1 = h->timer.get(); cudaEventRecord(t1, h->stream); }
    CU(cudaStreamSynchronize(h->stream));
    if (st) {
        st->cycles = cyc;
        st->iters = cyc * m;
        st->bytes_mpk = h->bytes[PH_MPK]; st->bytes_borth = h->bytes[PH_BORTH];
        st->bytes_tsqr = h->bytes[PH_TSQR]; st->bytes_other = h->bytes[PH_OTHER];
        st->bytes_spmv = h->bytes[PH_SPMV]; st->spmv_launches = h->spmv_launches;
        st->ms_setup = h->ms_setup;
        st->retried_panels = h->h_stat[1];
        st->max_orth_err = max_orth;
        st->max_gram_cond = max_cond;
        st->ms_mpk = st->ms_borth = st->ms_tsqr = st->ms_other = st->ms_total = st->ms_spmv = 0.0;
        if (h->timer.on) {
            float tt = 0.f;
            cudaEventElapsedTime(&tt, t0, t1);
            st->ms_total = double(tt);
            collect_timing(h, st);
        }
    }
    h->timer.reset();
    h->timer.on = false;
    h->diag_on = false;
    return rc;
}

}  // extern "C"
