/*
 * cagmres.h — C ABI of the B200-native CA-GMRES(s, m) hot path.
 *
 * Method: Yamazaki, Anzt, Tomov, Hoemmen, Dongarra, "Improving the Performance of CA-GMRES
 * on Multicores with Multiple GPUs", IPDPS 2014.  "P:n" cites /root/reference/PAPER.md line n.
 * One restart cycle = MPK (Fig. 4) -> BOrth (CGS) -> TSQR (CholQR P:162-166 /
 * SVQR P:172; MGS/CGS comparators, Fig. 9) -> Hessenberg update per block of
 * s_b = min(s, m - j) basis vectors, then the least-squares solve on the host and
 * x := x + V_{1:m} y.
 *
 * Conventions (all functions):
 *   - return int status: 0 = CAGMRES_OK, > 0 warning, < 0 error.  Never abort, never print.
 *   - every double is IEEE fp64; matrices are COLUMN-MAJOR with explicit leading dimension.
 *   - "dev" pointers are CUDA device pointers on the handle's device (e.g. a torch tensor's
 *     data_ptr()); "host" pointers are ordinary CPU memory.  The caller owns every pointer it
 *     passes; the library never frees or retains them beyond the call.
 *   - all device work is enqueued on the handle's stream (cagmres_set_stream; default: a
 *     stream created by the handle).  Functions that return a value the host needs
 *     (tsqr breakdown, solve) synchronise that stream before returning.
 *   - multi-GPU: one process per GPU; collectives are NCCL over NVLink (P:45 block rows).
 *     A distributed function must be called by every rank with the same scalar arguments.
 *   - vectors and panels passed to mpk/borth/tsqr/solve hold this rank's OWNED rows only
 *     (n_loc = own_end - own_begin rows); ghost rows are managed inside the handle.
 */
#ifndef CAGMRES_H
#define CAGMRES_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------------------ */
#define CAGMRES_OK              0
#define CAGMRES_NOT_CONVERGED   1   /* solve: maxit cycles done, x holds the last iterate     */
#define CAGMRES_EINVAL         -1   /* bad argument, shape, leading dimension or alignment    */
#define CAGMRES_ECUDA          -2   /* a CUDA runtime call failed (no device, launch error)   */
#define CAGMRES_ENCCL          -3   /* an NCCL call (or an in-process group collective) failed  */
#define CAGMRES_EBREAKDOWN     -4   /* Cholesky pivot <= 0, zero norm, singular T     */
#define CAGMRES_ENOMEM         -5   /* device or host allocation failed                       */
#define CAGMRES_EGHOST         -6   /* supplied rows do not cover the (s-1)-hop ghost rows    */
#define CAGMRES_ENOTSUP        -7   /* option not supported by this build                     */

/* ---- options ----------------------------------------------------------------------- */
enum { CAGMRES_MONOMIAL = 0, CAGMRES_NEWTON = 1 };               /* MPK basis      */
/* Standard GMRES(m) baseline (the "GMRES" rows of Fig. 14/15): every
 * restart cycle is m Arnoldi steps, each one SpMV (1-deep halo) plus CGS orthogonalisation
 * of width 1 (CGS2 when CAGMRES_REORTH is set) on the same kernels; s is not used (pass 1).
 * Not a CA method — it is the comparator the paper's speedups are quoted against. */
#define CAGMRES_GMRES 2
enum { CAGMRES_CHOLQR = 0, CAGMRES_SVQR = 1, CAGMRES_CGS = 2,     /* TSQR, Fig. 9/10     */
       CAGMRES_MGS = 3, CAGMRES_CAQR = 4 };
#define CAGMRES_TSQR_MASK   0xff
#define CAGMRES_REORTH      0x100   /* "2x": BOrth+TSQR twice (Fig. 14)       */
#define CAGMRES_BORTH_MGS   0x200   /* BOrth by MGS instead of CGS      */
/* One-pass BOrth + CholQR (fused CGS; one-reduction kernels, P:275 fn 7):
 * for panels with j > 0, one pass [C; B] = [Q P]^T P, R = chol(B - C^T C) (Pythagoras, exact
 * when Q^T Q = I), then P := (P - Q C) R^{-1} in one pass.  Reads the panel twice instead of
 * four times and needs one reduction instead of two.  CholQR only (else EINVAL); less stable
 * than the two-pass method (use with CAGMRES_REORTH); j + s + 1 <= 64. */
#define CAGMRES_ONEPASS     0x400
/* CholQR breakdown (pivot <= 0) -> opt-in SVQR retry of that panel (SURVEY reading G15):
 * the panel's R is recomputed from the same Gram by SVQR on the device, counted
 * in cagmres_stats.retried_panels; without it a breakdown returns EBREAKDOWN.  CholQR only
 * (else EINVAL); two-pass BOrth+TSQR path (not with CAGMRES_ONEPASS / the fused Gram option). */
#define CAGMRES_SVQR_RETRY  0x800

typedef struct cagmres* cagmres_t;

/* Sparse matrix rows handed to create (host CSR, copied to the device by create).
 *   n                : global dimension (A is n x n, nonsymmetric allowed)
 *   row_begin/row_end: global ids of the rows described by rowptr (nrows = row_end-row_begin)
 *   rowptr           : host, nrows+1 entries, rowptr[0] == 0, int64
 *   colind           : host, global column ids in [0, n), int32.  A row's entries may be in
 *                      any order and may repeat a column: create canonicalises every row
 *                      (stable sort by column, repeated entries summed in input order), and the
 *                      device sums each row in increasing global column order
 *   val              : host, fp64 values
 *   own_begin/own_end: the rows this rank owns (block-row distribution);
 *                      must satisfy row_begin <= own_begin <= own_end <= row_end.
 * For the distributed handle the described rows must contain every row within graph
 * distance s-1 of the owned rows (the boundary sets delta^(d,k)); else EGHOST. */
typedef struct {
    int64_t n, nnz;
    const int64_t* rowptr;
    const int32_t* colind;
    const double*  val;
    int64_t row_begin, row_end;
    int64_t own_begin, own_end;
} cagmres_csr;

/* Statistics of a solve (Fig. 14 columns).  hist is caller-owned (host). */
typedef struct {
    int    cycles;          /* restart cycles executed                                      */
    int    iters;           /* basis vectors generated (cycles * m)                          */
    int    hist_cap;        /* capacity of rel_resid_hist                                    */
    int    hist_len;        /* entries written                                               */
    double* rel_resid_hist; /* ||b - A x_c|| / ||b - A x_0|| after each cycle (host)         */
    int    collect_timing;  /* in: 1 = time every phase with CUDA events; 2 = only the MPK     *
                             * kernel launches (ms_spmv) and ms_total; 0 = none               */
    double ms_mpk, ms_borth, ms_tsqr, ms_other, ms_total;   /* device time per phase (ms)   */
    double bytes_mpk, bytes_borth, bytes_tsqr, bytes_other; /* algorithmic bytes */
    int    spmv_launches;   /* SpMV launches timed in ms_spmv                                */
    double ms_spmv;         /* device time of the SpMV launches alone                        */
    double bytes_spmv;      /* algorithmic bytes of those launches                           */
    int    collect_diag;    /* in: 1 = per-panel numerical diagnostics below (two extra Gram     *
                             * passes per panel and a host sync per cycle: not for timing)     */
    double max_orth_err;    /* max over the CA panels of ||I - Q_p^T Q_p||_2, Q_p = [q_j, new     *
                             * columns] after BOrth+TSQR (0 if none / not collected)    */
    double max_gram_cond;   /* max over the CA panels of kappa_2(W^T W), W = the MPK output      *
                             * [q_j, W_1..W_sb] before BOrth (Fig. 12 "cond(B)")   */
    double ms_setup;        /* host wall time of the create call that built this handle (ms)  */
    int    retried_panels;  /* CholQR panels re-factored by SVQR (CAGMRES_SVQR_RETRY, G15)      */
} cagmres_stats;

/* ---- lifetime ---------------------------------------------------------------------- */
/* Single-GPU handle on the current CUDA device.  A: all n rows (row_begin=own_begin=0,
 * row_end=own_end=n).  s >= 1 block size, m >= 1 restart length, s <= m; basis
 * CAGMRES_MONOMIAL|NEWTON|GMRES; orth = TSQR kind | flags.  Copies A to the device (sliced-ELL
 * layout) and allocates the basis V (n x (m+1)) and all workspace.
 * Errors: EINVAL, ECUDA, ENOMEM. */
int cagmres_create(cagmres_t* h, const cagmres_csr* A, int s, int m, int basis, int orth);

/* Distributed handle: one per rank, NCCL communicator built from nccl_unique_id (128-byte
 * ncclUniqueId created by rank 0 and broadcast by the caller).  row_starts (host, nranks+1)
 * is the global block-row partition: rank p owns [row_starts[p], row_starts[p+1]), and
 * A->own_begin/own_end must equal this rank's range.  Computes the boundary sets
 * delta^(d,k) and the halo schedule (exchanging request lists over NCCL).
 * Errors: EINVAL, EGHOST, ECUDA, ENCCL, ENOMEM. */
int cagmres_create_dist(cagmres_t* h, const cagmres_csr* A, const int64_t* row_starts,
                        int s, int m, int basis, int orth,
                        const void* nccl_unique_id, int rank, int nranks, int cuda_device);

/* In-process group: P ranks of the distributed handle inside ONE process, one host thread
 * per rank (transport.h).  Rank p runs on devices[p] (NULL: every rank on device 0); ranks on
 * different devices exchange through peer memory (NVLink), ranks on the same device through
 * device copies — so the whole multi-rank device path (halo pack -> exchange -> unpack, the
 * cross-rank sums, the distributed residual) runs on a single GPU.  Sums over ranks are one
 * fixed-order kernel per rank (bitwise identical on every rank).  Every collective is a host
 * barrier across the P threads: each rank's calls (create_group, mpk, borth, tsqr, solve,
 * destroy) must be made from its own thread, concurrently with the other ranks', in the same
 * order.  A rank that stops calling makes the others fail with ENCCL after 600 s.
 * nranks in [1, 16].  destroy: EINVAL while a handle created from the group still exists. */
typedef struct cagmres_group* cagmres_group_t;
int cagmres_group_create(cagmres_group_t* g, int nranks, const int* devices);
int cagmres_group_destroy(cagmres_group_t g);
/* cagmres_create_dist over an in-process group instead of NCCL (same arguments otherwise;
 * the device is the group's devices[rank]).  Errors: as create_dist; ENCCL = group failure. */
int cagmres_create_group(cagmres_t* h, const cagmres_csr* A, const int64_t* row_starts,
                         int s, int m, int basis, int orth, cagmres_group_t g, int rank);

int cagmres_destroy(cagmres_t h);                 /* frees everything create allocated */
const char* cagmres_strerror(int status);         /* static string, never NULL         */

/* cudaStream_t to enqueue on (NULL = the handle's own non-blocking stream; cudaStreamLegacy for
 * the legacy default stream — the handle's work is then ordered with everything the caller
 * queues there, e.g. the copy of b).  Programmatic dependent launch is used on ordinary streams
 * only.  Not owned. */
int cagmres_set_stream(cagmres_t h, void* cuda_stream);

/* Tuning options (value semantics per option); EINVAL for an unknown option.
 *   CAGMRES_OPT_MPK_WAVE : 0 (default) = one SpMV launch per MPK step; 1 = single-GPU
 *                          temporally blocked MPK when A is banded enough and the reuse
 *                          window fits L2 ("reducing communication of MPK on a single
 *                          GPU"); 2 = force it whenever A is banded; 3 = every MPK block in
 *                          ONE persistent launch (DIA SpMV variants, one rank): the steps are
 *                          separated by grid barriers instead of kernel boundaries (needs
 *                          every CTA of the launch resident: do not run other kernels
 *                          concurrently on the device; measured slower, off).  All
 *                          settings give the same bits.  EINVAL for other values.
 *   CAGMRES_OPT_SPMV     : SpMV kernel (default: the fastest on this matrix, timed once at create;
 *                          -1 re-runs that selection): 0 = one SELL-32 slice per warp; 5 = persistent
 *                          grid, slice descriptors software-pipelined two slices ahead; 16, 17 = the
 *                          persistent kernel with a fully unrolled body for the matrix's most common
 *                          DIA slice width and an L2 prefetch of the next slice's values, >= 4 / 5
 *                          CTAs per SM.  All variants are bitwise identical.  Other values: EINVAL.
 *   CAGMRES_OPT_GRAM     : CholQR Gram kernel: 0 = FP64 tensor core (DMMA m8n8k4) on a per-warp
 *                          cp.async ring; 1 (default) = scalar DFMA on a deeper ring (w <= 12,
 *                          else the DMMA kernel).
 *   CAGMRES_OPT_ARNOLDI  : width-1 Arnoldi passes (first Newton cycle, GMRES baseline): 0 = one
 *                          thread per row, register loads; 1 (default) = per-warp cp.async ring.
 *   CAGMRES_OPT_FUSE     : bit 0 (default 0) = BOrth pass 2 fused with the CholQR Gram;
 *                          bit 1 (default 1) = fused first-cycle Arnoldi passes;
 *                          bit 2 (default 1) = the normalisations q = w / ||w|| (restart vector,
 *                          Arnoldi vectors) fused into the SpMV that consumes q (DIA SpMV variants;
 *                          bitwise identical to the separate scaling pass).
 *   CAGMRES_OPT_WAVE_CHUNK / _WAVE_CTAS / _WAVE_LAG : temporal-blocking tuning (rows per
 *                          chunk, multiple of 256; resident CTAs per SM; wavefront lag in
 *                          chunks, 0 = automatic). */
#define CAGMRES_OPT_MPK_WAVE   1
#define CAGMRES_OPT_WAVE_CHUNK 3
#define CAGMRES_OPT_WAVE_CTAS  4
#define CAGMRES_OPT_WAVE_LAG   5
#define CAGMRES_OPT_FUSE       6
#define CAGMRES_OPT_SPMV       7
#define CAGMRES_OPT_GRAM       8
#define CAGMRES_OPT_ARNOLDI    9
#define CAGMRES_OPT_PANEL_TW   10   /* wide panel kernels: 16 (default: 16-row ring tiles where
                                       measured faster) or 32 (always 32-row tiles) */
#define CAGMRES_OPT_PDL        12   /* process-wide: 1 (default) = programmatic dependent launch of
                                       the hot kernels (next kernel's CTAs scheduled while the
                                       previous one drains), 0 = plain stream order */
#define CAGMRES_OPT_PANEL_PF   13   /* 1 = panel ring kernels also prefetch tiles beyond their
                                       cp.async window into L2; 0 (default since the serpentine
                                       order: C2 27.06 vs 27.42 ms) = off */
#define CAGMRES_OPT_PEER       14   /* in-process group handles: 1 (default) = one-sided peer access —
                                       the MPK halo is ONE pull kernel reading the owners' vectors
                                       directly, and the cross-rank Gram sum + Cholesky is one
                                       launch; 0 = pack / peer copies / unpack and a separate sum.
                                       Must be set identically on every rank.  get: 1 if in use. */
#define CAGMRES_OPT_GRAPH      15   /* 1 = single-rank untimed solves replay each CA restart
                                       cycle as one captured CUDA graph (re-captured when the
                                       shifts or an option change); 0 (default: measured neutral,
                                       the host already runs ahead of the GPU) = stream launches.
                                       get: a negative value = the cudaError of a failed capture */
#define CAGMRES_OPT_TRSM       11   /* CholQR/SVQR panel update V R^{-1}: 1 (default) = scalar
                                       FP64 on a cp.async ring (w <= 16), 0 = FP64 tensor core */
#define CAGMRES_OPT_FOLD       16   /* 1 (default) = the last block's final panel update of a CA
                                       cycle (V := P R^{-1}; one-pass: P := [Q P] M) is not
                                       formed: those columns are read only by the solution update
                                       x += V y, and Q_new y = P (R^{-1} [0; y]), so the host
                                       folds R^{-1} (and -C R^{-1}) into the coefficients and one
                                       pass over V[:, 0:m+1] updates x.  Equal in exact arithmetic;
                                       off with collect_diag (it needs the final Q).  0 = form it. */
#define CAGMRES_OPT_SERP       17   /* 1 (default) = serpentine row order: every streaming kernel
                                       (SpMV, BOrth / Gram / TRSM / Arnoldi panel kernels) sweeps the
                                       rows opposite to the launch before it, so the rows that
                                       launch touched last — still in the 126 MB L2 — are read
                                       first; 0 = every launch sweeps forward.  Row-wise kernels
                                       give identical results either way; the reductions (xTy, Gram,
                                       norms) sum in another fixed order (deterministic). */
int cagmres_set_option(cagmres_t h, int opt, int64_t value);
/* Current value of an option (e.g. the SpMV variant the create-time selection picked).
 * EINVAL for a null handle / pointer or an unknown option. */
int cagmres_get_option(cagmres_t h, int opt, int64_t* value);

/* Sizes: n_loc owned rows, n_ext owned+ghost rows (P:60 i^(d,1)), ldv = leading dim of V. */
int cagmres_sizes(cagmres_t h, int64_t* n_loc, int64_t* n_ext, int64_t* ldv);

/* ---- shifts ------------------------------------------------------------------ */
/* Newton shifts theta_k = re[k] + i im[k], k < count, in application order, conjugate pairs
 * adjacent with +im first.  Replaces any shifts the first GMRES cycle would compute.
 * count >= 1 (extra entries beyond s are ignored).  count == 0 (re, im may be NULL) forgets
 * the shifts: a Newton solve keeps the Leja-ordered Ritz values of its first cycle for later
 * solves with the same matrix unless they are cleared this way.
 * Errors: EINVAL (pair not adjacent). */
int cagmres_set_shifts(cagmres_t h, const double* re, const double* im, int count);
/* Copies the current shifts (after a Newton solve: the Leja-ordered Ritz values) to host
 * arrays of capacity cap; *count = number available (0 if none). */
int cagmres_get_shifts(cagmres_t h, double* re, double* im, int cap, int* count);

/* ---- hot-path kernels (callable individually; "MPK, BOrth, and TSQR") ---------- */
/* MPK(s_b, q) of Fig. 4: W[:,0] = q, W[:,k] = (A - theta_k I) W[:,k-1] for
 * k = 1..sb (theta = 0 for the monomial basis; complex pairs in real arithmetic).
 * One halo exchange of q's ghost rows (distributed), then sb local SpMVs on shrinking row
 * sets i^(d,k+1) with no further communication.  Uses the handle's first sb shifts.
 *   q : dev, n_loc           W : dev, ldw x (sb+1), ldw >= n_loc, owned rows written
 * Errors: EINVAL (sb < 1 or sb > s, ldw < n_loc, Newton without shifts). */
int cagmres_mpk(cagmres_t h, const double* q, double* W, int64_t ldw, int sb);

/* BOrth by CGS: C = Q^T P (global sum over ranks), P := P - Q C.
 *   Q : dev, ldq x j (orthonormal columns)   P : dev, ldp x w, updated in place
 *   C : dev, j x w, leading dimension j (output)
 * j == 0 is a no-op.  Errors: EINVAL. */
int cagmres_borth(cagmres_t h, const double* Q, int64_t ldq, int j,
                  double* P, int64_t ldp, int w, double* C);

/* TSQR of the tall-skinny panel P (Fig. 9): P := Q with Q^T Q = I and P_in = Q R.
 *   P : dev, ldp x w (w <= 32), in place      R : dev, w x w col-major, upper, diag > 0
 *   orth: CAGMRES_CHOLQR | SVQR | CGS | MGS (| CAGMRES_REORTH for the "2x" variant).
 * Synchronises the stream.  Errors: EINVAL, EBREAKDOWN (CholQR pivot <= 0). */
int cagmres_tsqr(cagmres_t h, double* P, int64_t ldp, int w, double* R, int orth);

/* ---- solver -------------------------------------------------------------- */
/* Solves A x = b with CA-GMRES(s, m) restarted until ||b - A x|| <= tol ||b - A x0||
 * (explicit residual at each restart) or maxit cycles.  Newton basis without
 * preset shifts: the first cycle is GMRES(m) and its Ritz values, Leja-ordered, become the
 * shifts.
 *   b : dev, n_loc (owned rows)    x : dev, n_loc, in: x0, out: solution
 *   st: optional (may be NULL), host struct filled on return.
 * Returns OK, NOT_CONVERGED, or an error (EBREAKDOWN, ECUDA, ENCCL, EINVAL). */
int cagmres_solve(cagmres_t h, const double* b, double* x, double tol, int maxit,
                  cagmres_stats* st);

/* Process-wide number of CUDA kernel launches this library has issued (all handles).  Lets a
 * caller count the kernels inside a timed region (bench.py "gpu_launches"). */
int64_t cagmres_kernel_launches(void);

/* ---- host-only setup plan, exported for tests of the multi-GPU setup ------- */
/* Pure host functions (no CUDA, no NCCL): boundary sets, extended-row numbering
 * [owned | delta^(s) | ... | delta^(1)] (distance 1 first), halo request / send lists. */
typedef struct cagmres_plan* cagmres_plan_t;
int cagmres_plan_create(cagmres_plan_t* p, const cagmres_csr* A, const int64_t* row_starts,
                        int nranks, int rank, int s);
int cagmres_plan_destroy(cagmres_plan_t p);
/* n_loc, n_ext, n_mat (rows stored = distance <= s-1), level_len[h] (h = 0..s): number of
 * extended rows at distance <= h; nnz_mat: nonzeros of the stored extended rows. */
int cagmres_plan_info(cagmres_plan_t p, int64_t* n_loc, int64_t* n_ext, int64_t* n_mat,
                      int64_t* nnz_mat, int64_t* level_len);
/* global id of each extended row (host, n_ext). */
int cagmres_plan_ext_rows(cagmres_plan_t p, int64_t* gids);
/* extended local CSR of the n_mat stored rows (host; rowptr n_mat+1, colind/val nnz_mat). */
int cagmres_plan_ext_csr(cagmres_plan_t p, int64_t* rowptr, int32_t* colind, double* val);
/* Requests this rank makes: counts[nranks]; gids / levels concatenated by owner rank, each
 * owner's list sorted by (level, gid).  Pass NULL gids to query counts only. */
int cagmres_plan_requests(cagmres_plan_t p, int64_t* counts, int64_t* gids, int32_t* levels);
/* Receive position (extended row id) of each requested gid, same order as requests. */
int cagmres_plan_recv_index(cagmres_plan_t p, int64_t* ext_ids);
/* Install the requests other ranks made of this rank (counts[nranks], concatenated by
 * requester).  Errors: EINVAL (a gid not owned here). */
int cagmres_plan_set_sends(cagmres_plan_t p, const int64_t* counts, const int64_t* gids,
                           const int32_t* levels);
/* Send lists: owned local indices in request order (host, total = sum counts). */
int cagmres_plan_send_index(cagmres_plan_t p, int64_t* local_idx);

/* SELL-32 device layout of the plan's stored rows, built on the host exactly as create builds
 * it (lets tests check it without a GPU).  Query the sizes with NULL
 * arrays first: nslices, ndcol (entries of dcol), nstored (entries of val); then sptr
 * (nslices+1), sinfo (nslices), dcol, val.  sinfo[sl] = dptr << 2 | clamp << 1 | dia; a DIA
 * slice stores diagonal t of lane l at val[sptr[sl] + 32 t + l] with column row + dcol[dptr + t],
 * an explicit slice column dcol[dptr + 32 t + l].  Each row's nonzeros appear in increasing
 * GLOBAL column order (padding entries are exact zeros). */
int cagmres_plan_sell(cagmres_plan_t p, int64_t* nslices, int64_t* ndcol, int64_t* nstored,
                      int64_t* sptr, int64_t* sinfo, int32_t* dcol, double* val);

/* ---- host-only reordering for the row partition ------- */
/* Reverse Cuthill-McKee order of the symmetrised pattern of A (n x n CSR, host): perm[new] =
 * old.  Each connected component starts at a pseudo-peripheral node (repeated BFS from a
 * minimum-degree node of the deepest level); neighbours are visited by increasing (degree,
 * id); the Cuthill-McKee order is reversed.  Errors: EINVAL (column id out of range). */
int cagmres_host_rcm(int64_t n, const int64_t* rowptr, const int32_t* colind, int64_t* perm);
/* B = P A P^T: row i of B is row perm[i] of A with columns renumbered by the inverse
 * permutation and sorted.  Output arrays caller-owned (out_rowptr n+1, out_colind/out_val nnz).
 * Errors: EINVAL (perm not a permutation of 0..n-1, column out of range). */
int cagmres_host_permute(int64_t n, const int64_t* rowptr, const int32_t* colind, const double* val,
                         const int64_t* perm, int64_t* out_rowptr, int32_t* out_colind, double* out_val);

/* k-way partition of the symmetrised graph of A (n x n CSR, host) into nparts parts of
 * balanced row counts with a small edge cut (P:104 fn 3 "k-way partitioning ...
 * smaller surfaces and better load balances", Fig. 6/7 P:98-118): recursive bisection, each
 * bisection a breadth-first level-set split from a pseudo-peripheral vertex refined by
 * Fiduccia-Mattheyses passes; part sizes within (1 + imbalance) of n/nparts per bisection level.
 * part[v] in [0, nparts); *edge_cut = undirected edges between parts (may be NULL).
 * Deterministic.  Errors: EINVAL (column id out of range, nparts < 1, imbalance < 0). */
int cagmres_host_partition(int64_t n, const int64_t* rowptr, const int32_t* colind, int nparts,
                           double imbalance, int32_t* part, int64_t* edge_cut);
/* Permutation that makes every part a contiguous block of rows, for the block-row create_dist
 * (P:45): perm[new] = old, parts in order, original order kept inside a part; row_starts
 * (nparts + 1) = the block boundaries.  Apply with cagmres_host_permute. */
int cagmres_host_partition_order(int64_t n, const int32_t* part, int nparts, int64_t* perm,
                                 int64_t* row_starts);

/* ---- host-only small dense algorithms of the cycle (exported for tests) -------------- */
/* Eigenvalues (Ritz values) of the upper Hessenberg H (m x m, ld ldh), Francis
 * double-shift QR; conjugate pairs returned adjacent (+im first).  EBREAKDOWN if the QR
 * iteration does not converge. */
int cagmres_host_eigvals(const double* H, int ldh, int m, double* wr, double* wi);
/* Modified Leja ordering (reading G10) of cnt Ritz values; writes up to cap
 * shifts, *nout = number produced (>= s when cnt allows). */
int cagmres_host_leja(const double* wr, const double* wi, int cnt, int s, double* ore,
                      double* oim, int cap, int* nout);
/* Change-of-basis B ((sb+1) x sb, ld sb+1) of the Newton/monomial MPK: A W[:,0:sb] = W B. */
int cagmres_host_change_of_basis(const double* re, const double* im, int sb, double* B);
/* Hessenberg update of a block:
 * H[0:j+sb+1, j:j+sb] = (Rt B - [H[0:j+1,0:j] Rt[0:j,0:sb]; 0]) T^{-1}, T = Rt[j:j+sb,0:sb]. */
int cagmres_host_hessenberg_update(double* H, int ldh, int j, int sb, const double* Rt,
                                   int ldr, const double* B);
/* Eigenvalues (ascending) of the symmetric n x n matrix A (ld lda, upper triangle read),
 * cyclic Jacobi; used for the per-panel diagnostics (kappa_2 of a Gram, ||I - Q^T Q||_2). */
int cagmres_host_sym_eigvals(const double* A, int lda, int n, double* ev);
/* y = argmin ||beta e1 - H y|| (H (k+1) x k upper Hessenberg, Givens QR); res[i] =
 * residual estimate after i+1 columns (may be NULL). */
int cagmres_host_givens_ls(const double* H, int ldh, int k, double beta, double* y,
                           double* res);

#ifdef __cplusplus
}
#endif
#endif /* CAGMRES_H */
