// reorder.cpp — host-side matrix reordering for the row partition of the MPK (SURVEY §8(f)
// NEXT-4).  The paper orders its matrices with RCM (or METIS k-way) before the block-row
// distribution, because the MPK ghost sets delta^(d,k) — and so the redundant flops, the
// extended-matrix storage and the halo volume of Fig. 6/7 — grow with the number of
// rows within k hops of a partition boundary.  Reverse Cuthill-McKee keeps graph neighbours
// close in index, so contiguous block rows get small surfaces.
//   cagmres_host_rcm      : RCM permutation of the symmetrised pattern of A (perm[new] = old)
//   cagmres_host_permute  : B = P A P^T in CSR (columns sorted per row)
// Pure host code, no CUDA.
#include <algorithm>
#include <cstdint>
#include <vector>

#include "internal.h"

// symmetrised adjacency (pattern of A + A^T without the diagonal), CSR (also partition.cpp)
void sym_graph(int64_t n, const int64_t* rp, const int32_t* ci, std::vector<int64_t>& gp,
               std::vector<int64_t>& gi) {
    std::vector<int64_t> deg(size_t(n) + 1, 0);
    for (int64_t r = 0; r < n; ++r)
        for (int64_t e = rp[r]; e < rp[r + 1]; ++e) {
            const int64_t c = ci[e];
            if (c == r) continue;
            ++deg[size_t(r)];
            ++deg[size_t(c)];
        }
    gp.assign(size_t(n) + 1, 0);
    for (int64_t r = 0; r < n; ++r) gp[size_t(r) + 1] = gp[size_t(r)] + deg[size_t(r)];
    gi.assign(size_t(gp[size_t(n)]), 0);
    std::vector<int64_t> pos(gp.begin(), gp.end() - 1);
    for (int64_t r = 0; r < n; ++r)
        for (int64_t e = rp[r]; e < rp[r + 1]; ++e) {
            const int64_t c = ci[e];
            if (c == r) continue;
            gi[size_t(pos[size_t(r)]++)] = c;
            gi[size_t(pos[size_t(c)]++)] = r;
        }
    // sort + dedupe each adjacency list (A + A^T counts a symmetric pair twice)
    std::vector<int64_t> np(size_t(n) + 1, 0);
    int64_t w = 0;
    for (int64_t r = 0; r < n; ++r) {
        auto b = gi.begin() + gp[size_t(r)], e = gi.begin() + gp[size_t(r) + 1];
        std::sort(b, e);
        auto last = std::unique(b, e);
        np[size_t(r)] = w;
        for (auto it = b; it != last; ++it) gi[size_t(w++)] = *it;
    }
    np[size_t(n)] = w;
    gi.resize(size_t(w));
    gp.swap(np);
}

namespace {

// BFS from s over unvisited-in-`mark`-epoch nodes; returns the last level (the deepest nodes)
// and the number of levels.
int bfs_levels(int64_t s, const std::vector<int64_t>& gp, const std::vector<int64_t>& gi,
               std::vector<int>& mark, int epoch, std::vector<int64_t>& last,
               std::vector<int64_t>* all = nullptr) {
    std::vector<int64_t> cur{s}, nxt;
    mark[size_t(s)] = epoch;
    int levels = 0;
    while (!cur.empty()) {
        ++levels;
        if (all) all->insert(all->end(), cur.begin(), cur.end());
        nxt.clear();
        for (int64_t u : cur)
            for (int64_t e = gp[size_t(u)]; e < gp[size_t(u) + 1]; ++e) {
                const int64_t v = gi[size_t(e)];
                if (mark[size_t(v)] != epoch) {
                    mark[size_t(v)] = epoch;
                    nxt.push_back(v);
                }
            }
        if (nxt.empty()) last = cur;
        cur.swap(nxt);
    }
    return levels;
}

}  // namespace

extern "C" {

int cagmres_host_rcm(int64_t n, const int64_t* rowptr, const int32_t* colind, int64_t* perm) {
    if (n < 0 || (n > 0 && (!rowptr || !colind || !perm))) return CAGMRES_EINVAL;
    for (int64_t r = 0; r < n; ++r)
        for (int64_t e = rowptr[r]; e < rowptr[r + 1]; ++e)
            if (colind[e] < 0 || colind[e] >= n) return CAGMRES_EINVAL;
    std::vector<int64_t> gp, gi;
    sym_graph(n, rowptr, colind, gp, gi);
    auto deg = [&](int64_t v) { return gp[size_t(v) + 1] - gp[size_t(v)]; };
    std::vector<char> done(size_t(n), 0);
    std::vector<int> mark(size_t(n), 0);
    int epoch = 0;
    std::vector<int64_t> order;
    order.reserve(size_t(n));
    std::vector<int64_t> nb;
    for (int64_t seed = 0; seed < n; ++seed) {
        if (done[size_t(seed)]) continue;
        // component of `seed`: start at its minimum-degree node, then move to a min-degree node of
        // the deepest BFS level while the eccentricity grows (pseudo-peripheral node, GPS-style)
        std::vector<int64_t> comp, last;
        ++epoch;
        bfs_levels(seed, gp, gi, mark, epoch, last, &comp);
        int64_t start = comp[0];
        for (int64_t v : comp)
            if (deg(v) < deg(start)) start = v;
        int ecc = -1;
        for (int it = 0; it < 8; ++it) {
            ++epoch;
            const int lv = bfs_levels(start, gp, gi, mark, epoch, last);
            if (lv <= ecc) break;
            ecc = lv;
            int64_t nxt = last[0];
            for (int64_t v : last)
                if (deg(v) < deg(nxt) || (deg(v) == deg(nxt) && v < nxt)) nxt = v;
            if (nxt == start) break;
            start = nxt;
        }
        // Cuthill-McKee BFS: neighbours appended by increasing (degree, id)
        size_t head = order.size();
        order.push_back(start);
        done[size_t(start)] = 1;
        while (head < order.size()) {
            const int64_t u = order[head++];
            nb.clear();
            for (int64_t e = gp[size_t(u)]; e < gp[size_t(u) + 1]; ++e) {
                const int64_t v = gi[size_t(e)];
                if (!done[size_t(v)]) {
                    done[size_t(v)] = 1;
                    nb.push_back(v);
                }
            }
            std::sort(nb.begin(), nb.end(), [&](int64_t a, int64_t b) {
                return deg(a) != deg(b) ? deg(a) < deg(b) : a < b;
            });
            order.insert(order.end(), nb.begin(), nb.end());
        }
    }
    for (int64_t i = 0; i < n; ++i) perm[i] = order[size_t(n - 1 - i)];   // reverse
    return CAGMRES_OK;
}

int cagmres_host_permute(int64_t n, const int64_t* rowptr, const int32_t* colind, const double* val,
                         const int64_t* perm, int64_t* out_rowptr, int32_t* out_colind, double* out_val) {
    if (n < 0 || (n > 0 && (!rowptr || !colind || !val || !perm || !out_rowptr || !out_colind || !out_val)))
        return CAGMRES_EINVAL;
    std::vector<int64_t> iperm(size_t(n), -1);
    for (int64_t i = 0; i < n; ++i) {
        const int64_t o = perm[i];
        if (o < 0 || o >= n || iperm[size_t(o)] >= 0) return CAGMRES_EINVAL;   // not a permutation
        iperm[size_t(o)] = i;
    }
    out_rowptr[0] = 0;
    std::vector<std::pair<int32_t, double>> row;
    for (int64_t i = 0; i < n; ++i) {
        const int64_t o = perm[i];
        row.clear();
        for (int64_t e = rowptr[o]; e < rowptr[o + 1]; ++e) {
            if (colind[e] < 0 || colind[e] >= n) return CAGMRES_EINVAL;
            row.emplace_back(int32_t(iperm[size_t(colind[e])]), val[e]);
        }
        std::sort(row.begin(), row.end(), [](const auto& a, const auto& b) { return a.first < b.first; });
        int64_t w = out_rowptr[i];
        for (const auto& p : row) {
            out_colind[w] = p.first;
            out_val[w] = p.second;
            ++w;
        }
        out_rowptr[i + 1] = w;
    }
    return CAGMRES_OK;
}

}  // extern "C"
