// plan.cpp — host setup of the distributed matrix powers kernel (§IV-A).
//
// Boundary sets by the recursion of P:62 (a BFS over the adjacency graph of A from the
// owned rows i^(d,s+1)): delta^(d,k) is the set of vertices at graph distance s-k+1.
// Extended numbering: [owned | distance 1 | distance 2 | ... | distance s], so every index
// set i^(d,k) is a PREFIX and MPK step k is a prefix-range SpMV.
// Rows at distance s are never computed (step 1 needs only distance <= s-1 rows), so only
// rows at distance <= s-1 are stored ("n_mat").  Within a level, ghosts are ordered by
// (owner rank, global id) so each owner's contribution to a level is one contiguous run.
#include <algorithm>
#include <cstring>
#include <unordered_map>

#include "internal.h"

static int owner_of(const int64_t* row_starts, int nranks, int64_t g) {
    // rank p owns [row_starts[p], row_starts[p+1])
    const int64_t* it = std::upper_bound(row_starts, row_starts + nranks + 1, g);
    return int(it - row_starts) - 1;
}

int plan_build(cagmres_plan* p, const cagmres_csr* A, const int64_t* row_starts,
               int nranks, int rank, int s) {
    if (!A || !row_starts || nranks < 1 || rank < 0 || rank >= nranks || s < 1)
        return CAGMRES_EINVAL;
    if (A->own_begin != row_starts[rank] || A->own_end != row_starts[rank + 1])
        return CAGMRES_EINVAL;
    if (A->row_begin > A->own_begin || A->own_end > A->row_end || A->n <= 0 ||
        A->own_begin > A->own_end || A->n >= (int64_t(1) << 31))
        return CAGMRES_EINVAL;
    if (row_starts[0] != 0 || row_starts[nranks] != A->n) return CAGMRES_EINVAL;
    p->nranks = nranks; p->rank = rank; p->s = s; p->n = A->n;
    p->own_begin = A->own_begin; p->own_end = A->own_end;
    p->n_loc = A->own_end - A->own_begin;
    const int64_t rb = A->row_begin, re = A->row_end;
    auto row_avail = [&](int64_t g) { return g >= rb && g < re; };
    auto in_own = [&](int64_t g) { return g >= A->own_begin && g < A->own_end; };

    // --- BFS levels -----------------------------------------------------------
    std::unordered_map<int64_t, int32_t> level;          // ghost gid -> distance
    std::vector<std::vector<int64_t>> lv(s + 1);
    std::vector<int64_t> frontier;
    frontier.reserve(size_t(p->n_loc));
    for (int64_t g = A->own_begin; g < A->own_end; ++g) frontier.push_back(g);
    for (int h = 1; h <= s; ++h) {
        std::vector<int64_t> next;
        for (int64_t g : frontier) {
            if (!row_avail(g)) return CAGMRES_EGHOST;
            const int64_t lr = g - rb;
            for (int64_t e = A->rowptr[lr]; e < A->rowptr[lr + 1]; ++e) {
                const int64_t c = A->colind[e];
                if (c < 0 || c >= A->n) return CAGMRES_EINVAL;
                if (in_own(c)) continue;
                if (level.find(c) != level.end()) continue;
                level.emplace(c, h);
                next.push_back(c);
            }
        }
        // order inside the level: (owner, gid) — owner ranges are contiguous in gid, so
        // plain gid order is (owner, gid) order
        std::sort(next.begin(), next.end());
        lv[h] = next;
        frontier.swap(next);
    }
    // --- extended numbering -------------------------------------------------------------
    p->level_len.assign(size_t(s) + 1, 0);
    p->ext_gid.clear();
    p->ext_level.clear();
    for (int64_t g = A->own_begin; g < A->own_end; ++g) { p->ext_gid.push_back(g); p->ext_level.push_back(0); }
    p->level_len[0] = p->n_loc;
    for (int h = 1; h <= s; ++h) {
        for (int64_t g : lv[h]) { p->ext_gid.push_back(g); p->ext_level.push_back(h); }
        p->level_len[h] = int64_t(p->ext_gid.size());
    }
    p->n_ext = int64_t(p->ext_gid.size());
    p->n_mat = p->level_len[s - 1];
    std::unordered_map<int64_t, int64_t> ext_of;
    ext_of.reserve(size_t(p->n_ext - p->n_loc) * 2 + 1);
    for (int64_t e = p->n_loc; e < p->n_ext; ++e) ext_of.emplace(p->ext_gid[e], e);
    auto ext_id = [&](int64_t g) -> int64_t {
        if (in_own(g)) return g - A->own_begin;
        auto it = ext_of.find(g);
        return it == ext_of.end() ? -1 : it->second;
    };
    // --- extended local CSR (rows at distance <= s-1) ----------------------------------------
    // Canonical rows: entries sorted by GLOBAL column id, duplicates summed in input order
    // (the CSR contract allows unsorted rows and repeated entries, include/cagmres.h).  Every
    // row is summed in global column order by the SpMV whatever the partition.
    p->rowptr.assign(size_t(p->n_mat) + 1, 0);
    p->colind.clear();
    p->val.clear();
    {
        int64_t tot = 0;
        for (int64_t r = 0; r < p->n_mat; ++r) {
            const int64_t g = p->ext_gid[r];
            if (!row_avail(g)) return CAGMRES_EGHOST;
            tot += A->rowptr[g - rb + 1] - A->rowptr[g - rb];
        }
        p->colind.reserve(size_t(tot));
        p->val.reserve(size_t(tot));
    }
    std::vector<std::pair<int64_t, int64_t>> ent;           // (global column, input position)
    for (int64_t r = 0; r < p->n_mat; ++r) {
        const int64_t g = p->ext_gid[r];
        const int64_t lr = g - rb;
        bool canon = true;                                  // already strictly increasing
        for (int64_t e = A->rowptr[lr] + 1; e < A->rowptr[lr + 1] && canon; ++e)
            canon = A->colind[e - 1] < A->colind[e];
        if (canon) {
            for (int64_t e = A->rowptr[lr]; e < A->rowptr[lr + 1]; ++e) {
                const int64_t c = ext_id(A->colind[e]);
                if (c < 0) return CAGMRES_EGHOST;
                p->colind.push_back(int32_t(c));
                p->val.push_back(A->val[e]);
            }
            p->rowptr[size_t(r) + 1] = int64_t(p->colind.size());
            continue;
        }
        ent.clear();
        for (int64_t e = A->rowptr[lr]; e < A->rowptr[lr + 1]; ++e) ent.push_back({A->colind[e], e});
        std::stable_sort(ent.begin(), ent.end(),
                         [](const std::pair<int64_t, int64_t>& a, const std::pair<int64_t, int64_t>& b) {
                             return a.first < b.first;
                         });
        for (size_t k = 0; k < ent.size(); ++k) {
            if (k > 0 && ent[k].first == ent[k - 1].first) {
                p->val.back() += A->val[ent[k].second];
                continue;
            }
            const int64_t c = ext_id(ent[k].first);
            if (c < 0) return CAGMRES_EGHOST;      // cannot happen for distance <= s-1 rows
            p->colind.push_back(int32_t(c));
            p->val.push_back(A->val[ent[k].second]);
        }
        p->rowptr[size_t(r) + 1] = int64_t(p->colind.size());
    }
    p->nnz_mat = int64_t(p->colind.size());
    // --- requests to owners, each sorted by (level, gid) -----------------------------------
    p->req_counts.assign(size_t(nranks), 0);
    std::vector<std::vector<int64_t>> byown(static_cast<size_t>(nranks));
    for (int64_t e = p->n_loc; e < p->n_ext; ++e) {
        const int o = owner_of(row_starts, nranks, p->ext_gid[e]);
        if (o < 0 || o >= nranks || o == rank) return CAGMRES_EINVAL;
        byown[size_t(o)].push_back(e);              // ext order is (level, owner, gid)
    }
    p->req_gid.clear(); p->req_level.clear(); p->req_ext.clear();
    for (int o = 0; o < nranks; ++o) {
        p->req_counts[size_t(o)] = int64_t(byown[size_t(o)].size());
        for (int64_t e : byown[size_t(o)]) {
            p->req_ext.push_back(e);
            p->req_gid.push_back(p->ext_gid[e]);
            p->req_level.push_back(p->ext_level[e]);
        }
    }
    p->send_counts.assign(size_t(nranks), 0);
    p->sends_set = (nranks == 1);
    return CAGMRES_OK;
}

int64_t plan_prefix_count(const std::vector<int64_t>& counts, const std::vector<int32_t>& levels,
                          int q, int depth) {
    int64_t off = 0;
    for (int i = 0; i < q; ++i) off += counts[size_t(i)];
    int64_t c = 0;
    for (int64_t k = 0; k < counts[size_t(q)]; ++k)
        if (levels[size_t(off + k)] <= depth) ++c;
        else break;                                 // lists are sorted by level
    return c;
}

// ---------------------------------------------------------------------------------------
// C ABI (host-only plan, for the multi-process CPU tests of the setup)
// ---------------------------------------------------------------------------------------
extern "C" {

int cagmres_plan_create(cagmres_plan_t* out, const cagmres_csr* A, const int64_t* row_starts,
                        int nranks, int rank, int s) {
    if (!out) return CAGMRES_EINVAL;
    *out = nullptr;
    cagmres_plan* p = new (std::nothrow) cagmres_plan();
    if (!p) return CAGMRES_ENOMEM;
    int st;
    try {
        st = plan_build(p, A, row_starts, nranks, rank, s);
    } catch (...) {
        st = CAGMRES_ENOMEM;
    }
    if (st != CAGMRES_OK) { delete p; return st; }
    *out = p;
    return CAGMRES_OK;
}

int cagmres_plan_destroy(cagmres_plan_t p) { delete p; return CAGMRES_OK; }

int cagmres_plan_info(cagmres_plan_t p, int64_t* n_loc, int64_t* n_ext, int64_t* n_mat,
                      int64_t* nnz_mat, int64_t* level_len) {
    if (!p) return CAGMRES_EINVAL;
    if (n_loc) *n_loc = p->n_loc;
    if (n_ext) *n_ext = p->n_ext;
    if (n_mat) *n_mat = p->n_mat;
    if (nnz_mat) *nnz_mat = p->nnz_mat;
    if (level_len) std::memcpy(level_len, p->level_len.data(), p->level_len.size() * sizeof(int64_t));
    return CAGMRES_OK;
}

int cagmres_plan_ext_rows(cagmres_plan_t p, int64_t* gids) {
    if (!p || !gids) return CAGMRES_EINVAL;
    std::memcpy(gids, p->ext_gid.data(), p->ext_gid.size() * sizeof(int64_t));
    return CAGMRES_OK;
}

int cagmres_plan_ext_csr(cagmres_plan_t p, int64_t* rowptr, int32_t* colind, double* val) {
    if (!p) return CAGMRES_EINVAL;
    if (rowptr) std::memcpy(rowptr, p->rowptr.data(), p->rowptr.size() * sizeof(int64_t));
    if (colind) std::memcpy(colind, p->colind.data(), p->colind.size() * sizeof(int32_t));
    if (val) std::memcpy(val, p->val.data(), p->val.size() * sizeof(double));
    return CAGMRES_OK;
}

int cagmres_plan_requests(cagmres_plan_t p, int64_t* counts, int64_t* gids, int32_t* levels) {
    if (!p || !counts) return CAGMRES_EINVAL;
    std::memcpy(counts, p->req_counts.data(), p->req_counts.size() * sizeof(int64_t));
    if (gids) std::memcpy(gids, p->req_gid.data(), p->req_gid.size() * sizeof(int64_t));
    if (levels) std::memcpy(levels, p->req_level.data(), p->req_level.size() * sizeof(int32_t));
    return CAGMRES_OK;
}

int cagmres_plan_recv_index(cagmres_plan_t p, int64_t* ext_ids) {
    if (!p || !ext_ids) return CAGMRES_EINVAL;
    std::memcpy(ext_ids, p->req_ext.data(), p->req_ext.size() * sizeof(int64_t));
    return CAGMRES_OK;
}

int cagmres_plan_set_sends(cagmres_plan_t p, const int64_t* counts, const int64_t* gids,
                           const int32_t* levels) {
    if (!p || !counts) return CAGMRES_EINVAL;
    int64_t tot = 0;
    for (int q = 0; q < p->nranks; ++q) {
        if (counts[q] < 0) return CAGMRES_EINVAL;
        tot += counts[q];
    }
    if (tot > 0 && (!gids || !levels)) return CAGMRES_EINVAL;
    p->send_counts.assign(counts, counts + p->nranks);
    p->send_idx.resize(size_t(tot));
    p->send_level.resize(size_t(tot));
    for (int64_t k = 0; k < tot; ++k) {
        const int64_t g = gids[k];
        if (g < p->own_begin || g >= p->own_end) return CAGMRES_EINVAL;
        if (k > 0 && levels[k] < 0) return CAGMRES_EINVAL;
        p->send_idx[size_t(k)] = g - p->own_begin;
        p->send_level[size_t(k)] = levels[k];
    }
    p->sends_set = true;
    return CAGMRES_OK;
}

int cagmres_plan_send_index(cagmres_plan_t p, int64_t* local_idx) {
    if (!p || !local_idx) return CAGMRES_EINVAL;
    std::memcpy(local_idx, p->send_idx.data(), p->send_idx.size() * sizeof(int64_t));
    return CAGMRES_OK;
}

}  // extern "C"
