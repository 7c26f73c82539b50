// kernels.h — launchers of the sm_100a FP64 kernels of the CA-GMRES hot path.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace kern {

// Process-wide count of kernel launches issued by this library (bench.py gpu_launches).
extern long long g_launches;   // (approximate when several host threads launch)

// Programmatic dependent launch (PDL, sm_90+): the hot kernels are launched with
// programmaticStreamSerializationAllowed, so their CTAs are scheduled while the previous
// kernel in the stream drains (its tail / last-CTA reduction); each such kernel executes
// pdl_wait() (griddepcontrol.wait: the previous grid has completed and its memory is
// visible) before it touches any data a predecessor writes, then pdl_trigger().
// Process-wide switch (CAGMRES_OPT_PDL); 1 by default.
extern int g_pdl;
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
template <typename... KArgs, typename... Args>
inline void launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    // (not on the legacy default stream: programmatic serialisation needs an ordinary stream)
    const bool legacy = st == nullptr || st == cudaStreamLegacy;
    attr[0].val.programmaticStreamSerializationAllowed = (g_pdl && !legacy) ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}


// Device properties used for grid sizing (filled once per handle).
struct Dev {
    int sms = 148;
    int device = 0;
    int gram = 1;               // CholQR Gram kernel: 0 = FP64 tensor core (DMMA), 1 = scalar DFMA ring
    int arnoldi_ring = 1;       // first-cycle / GMRES Arnoldi passes: 1 = cp.async ring kernels
    int trsm_scalar = 1;        // CholQR/SVQR update: 1 = scalar DFMA ring (w <= 16), 0 = DMMA
    int panel_tw16 = 1;
    int panel_pf = 0;           // panel rings: L2 prefetch PF_DIST tiles beyond the cp.async window (off:
                                // with the serpentine order it costs more L2 than it hides)
    int rev = 0;                // direction of the next streaming launch (serpentine order, solver.cu)
};

// Tile order of the streaming kernels (DESIGN.md §6 "serpentine order").  Unit g of NU (a warp,
// or a warp pair) handles the tiles g, g + NU, g + 2 NU, ... of the T full tiles, so a band of NU
// consecutive tiles sweeps the panel and the temporal order is global, independent of the grid
// geometry; rev = 1 sweeps from the last tile down.  A kernel launched opposite to its
// predecessor first reads the rows the predecessor touched last — still in the 126 MB L2.
__host__ __device__ __forceinline__ int64_t band_count(int64_t T, int64_t NU, int64_t g) {
    return g < T ? (T - 1 - g) / NU + 1 : 0;
}
__host__ __device__ __forceinline__ int64_t band_tile(int64_t T, int64_t NU, int64_t g, int64_t i, int rev) {
    const int64_t t = g + i * NU;
    return rev ? T - 1 - t : t;
}

// Sliced ELLPACK, slice height 32 (one warp), column-major inside a slice, with per-slice
// diagonal-offset column compression: sinfo[sl] = dptr << 2 | clamp << 1 | dia.
//   dia == 1: entry t of row r has column r + dcol[dptr + t] (<= 32 diagonals; zero value if the
//             row lacks it; clamped into [0, ncols) only in slices flagged `clamp`)
//   dia == 0: entry t of lane l has column dcol[dptr + 32 t + l]
struct Sell {
    int64_t nrows = 0;          // stored rows (extended rows at distance <= s-1)
    int64_t nslices = 0;
    int variant = 0;            // SpMV kernel (CAGMRES_OPT_SPMV): 0, 5, 16, 17 (kernels.cu spmv)
    int64_t nstored = 0;        // stored values incl. padding
    int64_t nnz = 0;            // true nonzeros
    int64_t ncols = 0;          // valid x entries (clamp bound for DIA slices)
    int64_t ndcol = 0, ndia = 0;
    int dia_w = 0;              // most common width of the unclamped DIA slices (spmv_dia.cu)
    int64_t* sptr = nullptr;    // nslices+1 value offsets
    int64_t* sinfo = nullptr;   // nslices
    int32_t* dcol = nullptr;    // DIA offsets / explicit column ids
    double* val = nullptr;
};

// y_r = sum over the stored entries of row r (one lane of a 32-row slice), in stored order.
// All 32 lanes of the warp call it together with the 32 rows of one slice (r & 31 == lane,
// padding rows of the last slice included), because lane t loads the slice's DIA offset t.
// Loads of BATCH entries are issued before their FMAs; DIA offsets are loaded once per slice (lane
// t holds offset t) and broadcast with shuffles, so no column index is loaded per entry.
// SEL: load with selects (arrays always assigned) instead of guarded assignments; same FMAs.
// SCALE: every x operand is multiplied by xscale after its load (the fused q = w / ||w|| of the
// SX SpMV, spmv_dia.cu); otherwise xscale is ignored.
template <int BATCH, bool SEL = false, bool SCALE = false>
__device__ __forceinline__ double sell_slice_dot(int64_t r, int64_t b, int W, int64_t info, int myoff,
                                                 const int32_t* __restrict__ dcol, int64_t ncols,
                                                 const double* __restrict__ val,
                                                 const double* __restrict__ x, bool coherent,
                                                 double xscale = 1.0) {
    const int lane = int(r & 31);
    const int64_t dp = info >> 2;
    double acc = 0.0;
    auto ldx = [&](const double* p) {
        const double v = coherent ? __ldca(p) : __ldg(p);
        return SCALE ? v * xscale : v;
    };
    const double* vp = val + b + lane;              // entry t of this row: vp[32 t]
    if (info & 1) {
        if (!(info & 2)) {                          // no clamping: x address = x + r + offset
            const double* xr = x + r;
            for (int t0 = 0; t0 < W; t0 += BATCH, vp += 32 * BATCH) {
                double v[BATCH], xv[BATCH];
#pragma unroll
                for (int u = 0; u < BATCH; ++u) {
                    const int off = __shfl_sync(0xffffffffu, myoff, (t0 + u) & 31);
                    if (SEL) {                      // arrays fully assigned (stay in registers
                        const bool ok = t0 + u < W; //  inside the persistent kernel's loop)
                        v[u] = ok ? __ldg(vp + 32 * u) : 0.0;
                        xv[u] = ok ? ldx(xr + off) : 0.0;
                    } else if (t0 + u < W) {
                        v[u] = __ldg(vp + 32 * u);
                        xv[u] = ldx(xr + off);
                    }
                }
#pragma unroll
                for (int u = 0; u < BATCH; ++u)
                    if (t0 + u < W) acc = fma(v[u], xv[u], acc);
            }
        } else {
            for (int t0 = 0; t0 < W; t0 += BATCH, vp += 32 * BATCH) {
                double v[BATCH], xv[BATCH];
#pragma unroll
                for (int u = 0; u < BATCH; ++u) {
                    const int off = __shfl_sync(0xffffffffu, myoff, (t0 + u) & 31);
                    const bool ok = t0 + u < W;
                    int64_t c = r + off;
                    c = c < 0 ? 0 : (c >= ncols ? ncols - 1 : c);
                    if (SEL) {
                        v[u] = ok ? __ldg(vp + 32 * u) : 0.0;
                        xv[u] = ok ? ldx(x + c) : 0.0;
                    } else if (ok) {
                        v[u] = __ldg(vp + 32 * u);
                        xv[u] = ldx(x + c);
                    }
                }
#pragma unroll
                for (int u = 0; u < BATCH; ++u)
                    if (t0 + u < W) acc = fma(v[u], xv[u], acc);
            }
        }
    } else {
        const int32_t* cp = dcol + dp + lane;
        for (int t0 = 0; t0 < W; t0 += BATCH, vp += 32 * BATCH, cp += 32 * BATCH) {
            double v[BATCH];
            int c[BATCH];
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
                const bool ok = t0 + u < W;
                if (SEL) {
                    v[u] = ok ? __ldg(vp + 32 * u) : 0.0;
                    c[u] = ok ? __ldg(cp + 32 * u) : 0;
                } else if (ok) {
                    v[u] = __ldg(vp + 32 * u);
                    c[u] = __ldg(cp + 32 * u);
                }
            }
            double xv[BATCH];
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
                if (SEL) xv[u] = t0 + u < W ? ldx(x + c[u]) : 0.0;
                else if (t0 + u < W) xv[u] = ldx(x + c[u]);
            }
#pragma unroll
            for (int u = 0; u < BATCH; ++u)
                if (t0 + u < W) acc = fma(v[u], xv[u], acc);
        }
    }
    return acc;
}

// Slice descriptor of the slice holding row r: value offset b, width W (entries per row),
// sinfo word, and (DIA slices) this lane's diagonal offset (lane t holds offset t).
__device__ __forceinline__ void sell_slice_meta(int64_t sl, const int64_t* __restrict__ sptr,
                                                const int64_t* __restrict__ sinfo, int64_t& b, int& W,
                                                int64_t& info) {
    b = __ldg(sptr + sl);
    W = int((__ldg(sptr + sl + 1) - b) >> 5);
    info = __ldg(sinfo + sl);
}
__device__ __forceinline__ int sell_slice_off(int lane, int W, int64_t info, const int32_t* __restrict__ dcol) {
    return ((info & 1) && lane < W) ? __ldg(dcol + (info >> 2) + lane) : 0;
}

template <int BATCH>
__device__ __forceinline__ double sell_row_dot(int64_t r, const int64_t* __restrict__ sptr,
                                               const int64_t* __restrict__ sinfo,
                                               const int32_t* __restrict__ dcol, int64_t ncols,
                                               const double* __restrict__ val,
                                               const double* __restrict__ x, bool coherent) {
    int64_t b, info;
    int W;
    sell_slice_meta(r >> 5, sptr, sinfo, b, W, info);
    const int myoff = sell_slice_off(int(r & 31), W, info, dcol);
    return sell_slice_dot<BATCH>(r, b, W, info, myoff, dcol, ncols, val, x, coherent);
}

// Single-GPU temporally blocked MPK (mpk_wave.cu).
struct WaveArgs {
    const int64_t* sptr; const int64_t* sinfo; const int32_t* dcol; const double* val; int64_t ncols;
    double* V; int64_t ldv; int j;
    int64_t n; int64_t bw; int CH, nC;    // rows, half-bandwidth, rows per chunk, chunks
    const int2* pairs; int npairs;        // (chunk, step) items in wavefront order
    int* done;                            // (s+1) x nC epoch-stamped completion flags
    int* queue;                           // item ticket counter (zeroed before each launch)
    int epoch;
    int dia_w;                            // the matrix's dominant DIA width (fast row body)
    double theta[32], b2[32];
    int kind[32];
};
void mpk_wave(const Dev& d, const WaveArgs& a, int ctas_per_sm, cudaStream_t st);

// Single-GPU MPK block in one persistent launch with grid barriers between the steps
// (mpk_sweep.cu, CAGMRES_OPT_MPK_WAVE = 3).  bar: a device counter that only grows; bar_base
// its value before this launch, *next_base its value after.  Returns -1 if not applicable.
struct SweepArgs {
    const int64_t* sptr; const int64_t* sinfo; const int32_t* dcol; const double* val; int64_t ncols;
    double* V; int64_t ldv; int j; int sb;
    int64_t n;
    int dia_w;
    int rev0;                             // sweep direction of step 1 (then alternating)
    unsigned* bar; unsigned bar_base;
    double theta[32], b2[32];
    int kind[32];
};
int mpk_sweep(const Dev& d, const SweepArgs& a, cudaStream_t st, unsigned* next_base);

// Fused Arnoldi passes of the first (GMRES) cycle (arnoldi.cu).  mode 1: v -= Q c_in and
// c_out = Q^T v; mode 2: v -= Q c_in and c_out[0] = v^T v (sqrt if sqrt_out).  jx <= 32
// (returns -1 otherwise).  part: >= arnoldi_ws_doubles() doubles; counter: zeroed uint.
struct ArnoldiArgs {
    int pf;                     // L2 prefetch ahead of the ring (ring kernels)
    int64_t n;
    const double* Q; int64_t ldq; int jx;
    double* v;
    const double* c_in;
    double* c_out;
    double* part;
    unsigned int* counter;
    int* status;
    int sqrt_out;
    double* vout = nullptr;     // modes 1 / 2: write the updated v here instead of in place
    int rev = 0;                // tile order (band_tile); set from Dev::rev by the launcher
};
int arnoldi_fused(const Dev& d, const ArnoldiArgs& a, int mode, cudaStream_t st);
// p -= X c, p a single column (n), X n x jx (jx <= 32), c device jx-vector; -1 if not applicable
int update_w1(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* p, const double* c,
              cudaStream_t st);
size_t arnoldi_ws_doubles(const Dev& d);

// TSQR by CAQR (caqr.cu): P (n x w, w <= 32) := Q (columns >= c0 written), R (w x w, ld w,
// diag > 0).  ws: caqr_ws_doubles(n, w) doubles.  Returns -1 on bad sizes (n < w).
size_t caqr_ws_doubles(int64_t n, int w);
int caqr(const Dev& d, int64_t n, double* P, int64_t ldp, int w, double* R, int c0, double* ws,
         cudaStream_t st);

// BOrth pass 2 fused with the CholQR Gram (fused.cu): P := P - X C (P: n x w, X: n x jx,
// C: jx x w ld jx) and out = [q0 P]^T [q0 P] ((w+1) x (w+1), ld w+1), R = chol(out) if
// fin_chol.  Returns -1 when not applicable (unaligned, jx > 64, w + 1 > 16, tiny n).
struct UpdGramArgs {
    int64_t n;
    const double* X; int64_t ldx; int jx;
    double* P; int64_t ldp; int w;
    const double* q0;
    const double* C;
    double* part;
    double* out;
    unsigned int* counter;
    int fin_chol;
    double* R;
    int* status;
};
int update_gram(const Dev& d, const UpdGramArgs& a, cudaStream_t st);
size_t update_gram_ws_doubles(const Dev& d);

// Status bits written by device kernels into the handle's status word.
enum : int { ST_CHOL = 1, ST_SVQR = 2, ST_NORM = 4 };

// y[0:nrows) = A x + bu*u + bw*w  (u, w may be null).  Newton step: u = x, bu = -theta;
// second step of a complex pair: w = x_prev, bw = b^2.
void spmv(const Dev& d, const Sell& A, int64_t nrows, const double* x, double* y,
          const double* u, double bu, const double* w, double bw, cudaStream_t st);
// DIA-width-specialised SpMV (spmv_dia.cu), CAGMRES_OPT_SPMV 16 / 17; mode as k_spmv_sell32
// (3 = u - A x).
// mode 4 / 5 = modes 0 / 1 with the fused normalisation (SX): x is an unnormalised w with
// ||w|| = *xnrm (device), the operand is w * (1 / ||w||), and rows [0, nrows) of that normalised
// vector are also stored to xs (u is ignored: the shift operand is the normalised x).
void spmv_dia(const Dev& d, const Sell& A, int variant, int64_t nrows, const double* x, double* y,
              const double* u, double bu, const double* w, double bw, int mode, cudaStream_t st,
              const double* xnrm = nullptr, double* xs = nullptr);
// y = A (w / ||w||) [- theta (w / ||w||)] and xs = w / ||w|| on rows [0, nrows) in one launch
// (DIA variants 16 / 17 only; returns -1 otherwise and does nothing).
int spmv_scaled(const Dev& d, const Sell& A, int64_t nrows, const double* w, const double* wnrm, double* xs,
                double* y, double bu, bool shift, cudaStream_t st);
// xs[0:n) = w[0:n) * (1 / *wnrm)   (the same product as k_scale1)
void scale_copy(int64_t n, const double* w, const double* wnrm, double* xs, cudaStream_t st);
// r[0:nrows) = b - A x
void residual(const Dev& d, const Sell& A, int64_t nrows, const double* x, const double* b,
              double* r, cudaStream_t st);

// Partial + deterministic total of C = X^T Y (X: n x jx, ld ldx; Y: n x w, ld ldy), written
// to out (jx x w, ld jx).  fin_chol: out is the Gram (X == Y, jx == w) and R = chol(out)
// (upper, ld w) is computed in the same launch; breakdown sets ST_CHOL in *status.
// ws: workspace of at least xty_ws_doubles() doubles; counter: a zeroed device uint.
// counter: XTY_COUNTERS zeroed uints (tree_reduce tickets, reduce.cuh; left zeroed).
constexpr int XTY_COUNTERS = 4096;
struct XtyWs { double* part = nullptr; size_t cap = 0; unsigned int* counter = nullptr; };
size_t xty_ws_doubles(const Dev& d, int jx, int w);
int xty(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, const double* Y,
        int64_t ldy, int w, double* out, bool fin_chol, double* R, int* status,
        const XtyWs& ws, cudaStream_t st);

// Scalar-DFMA Gram G = P^T P (gram.cu; P 16-B aligned, ld even, w <= 12), same final
// reduction / in-launch Cholesky contract as xty with X == Y.  Returns -1 if not applicable.
struct GramArgs {
    int64_t n;
    const double* P; int64_t ldp; int w;
    int pf;                     // L2 prefetch ahead of the ring
    double* part;               // >= sms * w * w doubles
    double* out;                // w x w, ld w
    unsigned int* counter;
    int fin_chol;
    double* R;
    int* status;
    int rev = 0;                // tile order (band_tile); set from Dev::rev by the launcher
};
int gram_dfma(const Dev& d, const GramArgs& a, cudaStream_t st);

// R = chol(G) (upper, ld w), one tiny launch (used after a cross-rank allreduce of G).
void chol(const double* G, int w, double* R, int* status, cudaStream_t st);
// SVQR small factor: R from the Gram G (w x w), one CTA.
void svqr_factor(const double* G, int w, double* R, int* status, cudaStream_t st);
// G15 opt-in: if ST_CHOL is set in status[0], R := SVQR factor of G, clear ST_CHOL, ++status[1].
void svqr_retry(const double* G, int w, double* R, int* status, cudaStream_t st);

// P[:, 0:w] -= X C  (C: jx x w, ld jx)      (BOrth pass 2)
// early: the preceding kernel in the stream writes neither X nor P (only C): the ring kernel
// starts streaming X / P before griddepcontrol.wait (PDL overlap with that kernel's tail)
void update(const Dev& d, int64_t n, const double* X, int64_t ldx, int jx, double* P,
            int64_t ldp, int w, const double* C, cudaStream_t st, bool early = false);
// P[:, c0:w] = (X M)[:, c0:w]  (X: n x K, ld ldx, contiguous columns that contain P; M: K x w,
// ld ldm; P written in place)  — one-pass BOrth+CholQR update.  -1 if K > 64 or w > 32.
int gemm_rows(const Dev& d, int64_t n, const double* X, int64_t ldx, int K, double* P, int64_t ldp, int w,
              const double* M, int64_t ldm, int c0, cudaStream_t st, bool early = false);
// one-pass BOrth+CholQR small step (onepass.cu): from Mx = [Q P]^T P ((j+w) x w, ld j+w) write
// C (j x (w-1), ld j), R = chol(Mx[j:, :] - Cf^T Cf) (ld w), Mo = [-Cf R^{-1}; R^{-1}] (ld j+w).
void onepass_finalize(const double* Mx, int j, int w, double* C, double* R, double* Mo, int* status,
                      cudaStream_t st);
// P[:, c0:w] = (P R^{-1})[:, c0:w]   (R upper w x w, ld w)
// early: as for update (the preceding kernel only produced R)
void trsm(const Dev& d, int64_t n, double* P, int64_t ldp, int w, const double* R, int c0,
          cudaStream_t st, bool early = false);
// Halo pack / unpack over segments [off[i], off[i] + cnt[i]) of an index list (one segment per
// peer: the depth-limited prefix of that peer's level-sorted list).
struct Segs {
    int64_t off[32], cnt[32];
    int n = 0;
    void add(int64_t o, int64_t c) {
        if (c > 0 && n < 32) { off[n] = o; cnt[n] = c; ++n; }
    }
};
// gather_segs: dst[k] = src[idx[k]]   /   scatter_segs: dst[idx[k]] = src[k],   k in the segments.
// More than 32 segments: one launch per 32.
void gather_segs(const double* src, const int64_t* idx, const Segs& sg, double* dst, cudaStream_t st);
void scatter_segs(const double* src, const int64_t* idx, const Segs& sg, double* dst, cudaStream_t st);
// small device helpers
void add_small(const double* a, const double* b, double* c, int cnt, cudaStream_t st);

}  // namespace kern
