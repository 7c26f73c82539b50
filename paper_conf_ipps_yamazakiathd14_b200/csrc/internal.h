// internal.h — shared declarations of the CA-GMRES B200 library (not part of the C ABI).
#pragma once
#include <cstdint>
#include <cstddef>
#include <vector>
#include "../../include/cagmres.h"

// ------------------------------------------------------------------------------------
// Setup plan: boundary sets, extended numbering, halo request/send lists.
// ------------------------------------------------------------------------------------
struct cagmres_plan {
    int nranks = 1, rank = 0, s = 1;
    int64_t n = 0, own_begin = 0, own_end = 0, n_loc = 0, n_ext = 0, n_mat = 0, nnz_mat = 0;
    std::vector<int64_t> level_len;        // s+1: ext rows with distance <= h
    std::vector<int64_t> ext_gid;          // n_ext
    std::vector<int32_t> ext_level;        // n_ext (0 = owned)
    std::vector<int64_t> rowptr;           // n_mat+1 (extended local CSR, stored rows)
    std::vector<int32_t> colind;           // local (extended) column ids
    std::vector<double>  val;
    // requests to owners (concatenated by owner rank; each sorted by (level, gid))
    std::vector<int64_t> req_counts;       // nranks
    std::vector<int64_t> req_gid;
    std::vector<int32_t> req_level;
    std::vector<int64_t> req_ext;          // ext row receiving each requested value
    // sends (requests other ranks made of me, concatenated by requester)
    std::vector<int64_t> send_counts;      // nranks
    std::vector<int64_t> send_idx;         // owned local index
    std::vector<int32_t> send_level;
    bool sends_set = false;
};

int plan_build(cagmres_plan* p, const cagmres_csr* A, const int64_t* row_starts,
               int nranks, int rank, int s);

// Host SELL-32 layout of the plan's stored rows (sell.cpp):
// sinfo[sl] = dptr << 2 | clamp << 1 | dia; DIA slices: dcol[dptr + t] = offset of diagonal t,
// else dcol[dptr + 32 t + lane] = column; values val[sptr[sl] + 32 t + lane].
struct SellHost {
    int64_t nslices = 0, ndia = 0;
    std::vector<int64_t> sptr, sinfo;
    std::vector<int32_t> dcol;
    std::vector<double> val;
};
void sell_build(const cagmres_plan& p, SellHost& out);   // throws std::bad_alloc

// count of entries of the (owner/requester) list `q` whose level <= depth
int64_t plan_prefix_count(const std::vector<int64_t>& counts, const std::vector<int32_t>& levels,
                          int q, int depth);

// symmetrised adjacency of a CSR pattern (A + A^T, no diagonal, sorted, unique) — reorder.cpp
void sym_graph(int64_t n, const int64_t* rp, const int32_t* ci, std::vector<int64_t>& gp,
               std::vector<int64_t>& gi);

// ------------------------------------------------------------------------------------
// Small dense host algorithms (P:41 LS and Hessenberg by-product; P:94 Ritz / Leja).
// All matrices column-major.
// ------------------------------------------------------------------------------------
namespace host {
// per-step shift description of a block (G10): kind 0 real, 1 first of pair, 2 second
struct Step { double a, b2; int kind; };
std::vector<Step> block_steps(const std::vector<double>& re, const std::vector<double>& im, int sb);
// change-of-basis B ((sb+1) x sb, ld sb+1)
void change_of_basis(const std::vector<Step>& st, int sb, double* B);
// H[0:j+sb+1, j:j+sb] = (Rt B - [H_prev Cs; 0]) T^{-1}; H ld = ldh; Rt ld = ldr
int hessenberg_update(double* H, int ldh, int j, int sb, const double* Rt, int ldr,
                      const double* B);
// y = argmin ||beta e1 - H y||, H (k+1) x k upper Hessenberg (ld ldh); res[i] estimates
int givens_ls(const double* H, int ldh, int k, double beta, double* y, double* res);
// eigenvalues of the upper Hessenberg m x m matrix (Francis double-shift QR)
int hessenberg_eigvals(const double* H, int ldh, int m, double* wr, double* wi);
// modified Leja order (G10); returns >= s shifts (or all available)
void modified_leja(const double* wr, const double* wi, int cnt, int s,
                   std::vector<double>& ore, std::vector<double>& oim);
// eigenvalues of a symmetric matrix (upper triangle read), ascending (cyclic Jacobi)
void sym_eigvals(const double* A, int lda, int n, double* ev);
}  // namespace host
