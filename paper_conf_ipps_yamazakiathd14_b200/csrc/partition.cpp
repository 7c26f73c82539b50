// partition.cpp — host k-way graph partitioner for the row distribution (
// P:104 fn 3: "k-way partitioning ... often gave smaller surfaces and better load balances").
//
// The MPK ghost sets delta^(d,k) grow with the rows within k hops of a partition boundary
// (Fig. 6/7), so the row partition should minimise the boundary (edge cut) at a
// balanced number of rows per GPU.  METIS is an external library; this is a self-contained
// multilevel-free recursive bisection in the same spirit:
//   * initial bisection: a breadth-first (Cuthill-McKee) order of the sub-graph from a
//     pseudo-peripheral vertex, cut at the target size — a level-set split, contiguous in the
//     graph (restarted per connected component);
//   * Fiduccia-Mattheyses refinement: passes of single-vertex moves by best gain (lazy
//     max-heaps per side), each vertex moved at most once per pass, within the balance
//     tolerance; the pass is rolled back to its best prefix;
//   * k parts by recursive bisection with target sizes proportional to the part counts.
// The result is a part id per row; cagmres_host_partition_order turns it into the
// permutation that makes every part a contiguous block of rows, i.e. the input of the
// block-row create_dist.  Pure host code, no CUDA.
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdint>
#include <queue>
#include <vector>

#include "internal.h"

namespace {

struct Part {
    const std::vector<int64_t>& gp;
    const std::vector<int64_t>& gi;
    std::vector<int32_t>& part;         // final part ids
    std::vector<int32_t> side;          // 0 / 1 inside the current bisection; BFS marks 2 / 3
    std::vector<int64_t> stamp;         // subset membership: stamp[v] == cur
    std::vector<int64_t> dsub;          // degree inside the current subset
    std::vector<char> lock;             // moved in the current FM pass
    int64_t cur = 0;
    double eps;
    bool in(int64_t v) const { return stamp[size_t(v)] == cur; }
};

// Level-set order of the sub-graph vs: BFS from a pseudo-peripheral vertex of each component
// (two sweeps from a minimum-degree start), neighbours taken by increasing degree.
void bfs_order(Part& P, const std::vector<int64_t>& vs, std::vector<int64_t>& order) {
    const auto& gp = P.gp;
    const auto& gi = P.gi;
    order.clear();
    order.reserve(vs.size());
    auto by_deg = [&](int64_t a, int64_t b) { return P.dsub[size_t(a)] < P.dsub[size_t(b)]; };
    std::vector<int64_t> sorted(vs);
    std::stable_sort(sorted.begin(), sorted.end(), by_deg);
    std::vector<int64_t> lvl, nxt, tmp, visited, last;
    for (int64_t s0 : sorted) {
        if (P.side[size_t(s0)] == 2) continue;
        int64_t s = s0;
        for (int sweep = 0; sweep < 2; ++sweep) {
            lvl.assign(1, s);
            visited.assign(1, s);
            P.side[size_t(s)] = 3;
            last = lvl;
            while (!lvl.empty()) {
                nxt.clear();
                for (int64_t v : lvl)
                    for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e) {
                        const int64_t u = gi[size_t(e)];
                        if (P.in(u) && P.side[size_t(u)] < 2) {
                            P.side[size_t(u)] = 3;
                            nxt.push_back(u);
                            visited.push_back(u);
                        }
                    }
                if (!nxt.empty()) last = nxt;
                lvl.swap(nxt);
            }
            for (int64_t v : visited) P.side[size_t(v)] = -1;
            int64_t best = last[0];
            for (int64_t v : last)
                if (P.dsub[size_t(v)] < P.dsub[size_t(best)]) best = v;
            s = best;
        }
        lvl.assign(1, s);
        P.side[size_t(s)] = 2;
        order.push_back(s);
        while (!lvl.empty()) {
            nxt.clear();
            for (int64_t v : lvl) {
                tmp.clear();
                for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e) {
                    const int64_t u = gi[size_t(e)];
                    if (P.in(u) && P.side[size_t(u)] != 2) {
                        P.side[size_t(u)] = 2;
                        tmp.push_back(u);
                    }
                }
                std::stable_sort(tmp.begin(), tmp.end(), by_deg);
                for (int64_t u : tmp) { order.push_back(u); nxt.push_back(u); }
            }
            lvl.swap(nxt);
        }
    }
}

// Fiduccia-Mattheyses refinement of the bisection (side 0 / 1) of vs, target |side 0| = tl:
// a kept prefix deviates by at most `slack` = eps_level * min(tl, |vs| - tl); moves may pass
// through one more vertex of imbalance.
void fm_refine(Part& P, const std::vector<int64_t>& vs, int64_t tl) {
    const auto& gp = P.gp;
    const auto& gi = P.gi;
    const int64_t nv = int64_t(vs.size());
    const int64_t slack = int64_t(std::floor(P.eps * double(std::min(tl, nv - tl))));
    const int64_t mslack = std::max<int64_t>(1, slack);
    auto gain_of = [&](int64_t v) {                          // cut reduction if v changes side
        int64_t g = 0;
        for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e) {
            const int64_t u = gi[size_t(e)];
            if (P.in(u)) g += P.side[size_t(u)] != P.side[size_t(v)] ? 1 : -1;
        }
        return g;
    };
    int64_t size0 = 0;
    for (int64_t v : vs) size0 += P.side[size_t(v)] == 0;
    using Ent = std::pair<int64_t, int64_t>;                 // (gain, -v): ties -> smaller id
    std::vector<int64_t> moved;
    for (int pass = 0; pass < 12; ++pass) {
        std::priority_queue<Ent> heap[2];
        for (int64_t v : vs) heap[P.side[size_t(v)]].push({gain_of(v), -v});
        moved.clear();
        int64_t delta = 0, best_delta = 0, best_len = 0, s0 = size0, since_best = 0;
        const bool bal0 = std::llabs(size0 - tl) <= slack;
        if (!bal0) best_delta = INT64_MAX;                   // any balanced prefix is better
        const int64_t patience = std::max<int64_t>(64, nv / 50);
        while (since_best < patience) {
            int pick = -1;
            int64_t pg = 0, pv = -1;
            for (int sd = 0; sd < 2; ++sd) {
                const int64_t ns0 = sd == 0 ? s0 - 1 : s0 + 1;
                if (std::llabs(ns0 - tl) > mslack && std::llabs(ns0 - tl) >= std::llabs(s0 - tl)) continue;
                while (!heap[sd].empty()) {
                    const Ent t = heap[sd].top();
                    const int64_t v = -t.second;
                    if (P.lock[size_t(v)] || P.side[size_t(v)] != sd || t.first != gain_of(v)) { heap[sd].pop(); continue; }
                    if (pick < 0 || t.first > pg) { pick = sd; pg = t.first; pv = v; }
                    break;
                }
            }
            if (pick < 0) break;
            heap[pick].pop();
            P.side[size_t(pv)] = 1 - pick;
            P.lock[size_t(pv)] = 1;
            s0 += pick == 0 ? -1 : 1;
            delta -= pg;
            moved.push_back(pv);
            for (int64_t e = gp[size_t(pv)]; e < gp[size_t(pv) + 1]; ++e) {
                const int64_t u = gi[size_t(e)];
                if (P.in(u) && !P.lock[size_t(u)]) heap[P.side[size_t(u)]].push({gain_of(u), -u});
            }
            if (std::llabs(s0 - tl) <= slack && delta < best_delta) {
                best_delta = delta;
                best_len = int64_t(moved.size());
                since_best = 0;
            } else {
                ++since_best;
            }
        }
        for (int64_t v : moved) P.lock[size_t(v)] = 0;
        for (int64_t i = int64_t(moved.size()) - 1; i >= best_len; --i) {
            const int64_t v = moved[size_t(i)];
            P.side[size_t(v)] = 1 - P.side[size_t(v)];
        }
        size0 = 0;
        for (int64_t v : vs) size0 += P.side[size_t(v)] == 0;
        if (best_len == 0) break;                            // no improving prefix: converged
    }
}

// Greedy graph growing from seed s: repeatedly add the frontier vertex with the most edges into
// the region minus edges out of it (lazy max-heap), restarting from the smallest unreached
// vertex of vs when a component is exhausted; the first tl vertices form side 0.
void grow_order(Part& P, const std::vector<int64_t>& vs, int64_t s, std::vector<int64_t>& order) {
    const auto& gp = P.gp;
    const auto& gi = P.gi;
    order.clear();
    auto key = [&](int64_t v) {                               // into-region minus out-of-region
        int64_t in_r = 0, out = 0;
        for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e) {
            const int64_t u = gi[size_t(e)];
            if (!P.in(u)) continue;
            if (P.side[size_t(u)] == 2) ++in_r; else ++out;
        }
        return in_r - out;
    };
    using Ent = std::pair<int64_t, int64_t>;                  // (key, -v)
    std::priority_queue<Ent> heap;
    size_t next_seed = 0;
    heap.push({key(s), -s});
    while (order.size() < vs.size()) {
        if (heap.empty()) {
            while (P.side[size_t(vs[next_seed])] == 2) ++next_seed;
            heap.push({key(vs[next_seed]), -vs[next_seed]});
        }
        const Ent t = heap.top();
        heap.pop();
        const int64_t v = -t.second;
        if (P.side[size_t(v)] == 2 || t.first != key(v)) continue;
        P.side[size_t(v)] = 2;
        order.push_back(v);
        for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e) {
            const int64_t u = gi[size_t(e)];
            if (P.in(u) && P.side[size_t(u)] != 2) heap.push({key(u), -u});
        }
    }
}

int64_t sub_cut(const Part& P, const std::vector<int64_t>& vs) {
    int64_t c = 0;
    for (int64_t v : vs)
        for (int64_t e = P.gp[size_t(v)]; e < P.gp[size_t(v) + 1]; ++e) {
            const int64_t u = P.gi[size_t(e)];
            if (u > v && P.in(u) && P.side[size_t(u)] != P.side[size_t(v)]) ++c;
        }
    return c;
}

void rec_bisect(Part& P, std::vector<int64_t>& vs, int k, int first) {
    if (k <= 1 || vs.size() <= 1) {
        for (int64_t v : vs) P.part[size_t(v)] = first;
        return;
    }
    const int kl = k / 2;
    const int64_t tl = int64_t(std::llround(double(vs.size()) * double(kl) / double(k)));
    ++P.cur;
    for (int64_t v : vs) P.stamp[size_t(v)] = P.cur;
    for (int64_t v : vs) {
        int64_t d = 0;
        for (int64_t e = P.gp[size_t(v)]; e < P.gp[size_t(v) + 1]; ++e) d += P.in(P.gi[size_t(e)]);
        P.dsub[size_t(v)] = d;
    }
    // candidate initial bisections, each refined by FM; the smallest cut wins (ties: first):
    // the given row order (often already local), a breadth-first level-set order from a
    // pseudo-peripheral vertex, and greedy graph growing from that vertex
    std::vector<int64_t> order, best_side;
    int64_t best_cut = -1;
    for (int cand = 0; cand < 3; ++cand) {
        if (cand == 0) {
            order = vs;                                          // vs is in increasing id order
        } else {
            bfs_order(P, vs, order);
            if (cand == 2) {
                const int64_t s = order.front();
                for (int64_t v : vs) P.side[size_t(v)] = -1;
                grow_order(P, vs, s, order);
            }
        }
        for (size_t i = 0; i < order.size(); ++i) P.side[size_t(order[i])] = i < size_t(tl) ? 0 : 1;
        fm_refine(P, vs, tl);
        const int64_t c = sub_cut(P, vs);
        if (best_cut < 0 || c < best_cut) {
            best_cut = c;
            best_side.resize(vs.size());
            for (size_t i = 0; i < vs.size(); ++i) best_side[i] = P.side[size_t(vs[i])];
        }
    }
    for (size_t i = 0; i < vs.size(); ++i) P.side[size_t(vs[i])] = int32_t(best_side[i]);
    std::vector<int64_t> L, R;
    for (int64_t v : vs) (P.side[size_t(v)] == 0 ? L : R).push_back(v);
    for (int64_t v : vs) P.side[size_t(v)] = -1;
    std::vector<int64_t>().swap(vs);
    rec_bisect(P, L, kl, first);
    rec_bisect(P, R, k - kl, first + kl);
}

}  // namespace

extern "C" {

int cagmres_host_partition(int64_t n, const int64_t* rowptr, const int32_t* colind, int nparts,
                           double imbalance, int32_t* part, int64_t* edge_cut) {
    if (n < 0 || !rowptr || (n > 0 && !colind) || !part || nparts < 1 || !(imbalance >= 0.0)) return CAGMRES_EINVAL;
    for (int64_t e = 0; e < rowptr[n]; ++e)
        if (colind[e] < 0 || colind[e] >= n) return CAGMRES_EINVAL;
    try {
        std::vector<int64_t> gp, gi;
        sym_graph(n, rowptr, colind, gp, gi);
        std::vector<int32_t> pt(size_t(n), 0);
        int levels = 0;                                      // bisection levels: split the tolerance
        while ((1 << levels) < nparts) ++levels;
        Part P{gp, gi, pt, std::vector<int32_t>(size_t(n), -1), std::vector<int64_t>(size_t(n), 0),
               std::vector<int64_t>(size_t(n), 0), std::vector<char>(size_t(n), 0), 0,
               imbalance / double(std::max(levels, 1))};
        std::vector<int64_t> vs(static_cast<size_t>(n));
        for (int64_t v = 0; v < n; ++v) vs[size_t(v)] = v;
        rec_bisect(P, vs, nparts, 0);
        int64_t cut = 0;
        for (int64_t v = 0; v < n; ++v)
            for (int64_t e = gp[size_t(v)]; e < gp[size_t(v) + 1]; ++e)
                if (gi[size_t(e)] > v && pt[size_t(v)] != pt[size_t(gi[size_t(e)])]) ++cut;
        std::copy(pt.begin(), pt.end(), part);
        if (edge_cut) *edge_cut = cut;
    } catch (...) {
        return CAGMRES_ENOMEM;
    }
    return CAGMRES_OK;
}

int cagmres_host_partition_order(int64_t n, const int32_t* part, int nparts, int64_t* perm,
                                 int64_t* row_starts) {
    if (n < 0 || !part || nparts < 1 || !perm || !row_starts) return CAGMRES_EINVAL;
    std::vector<int64_t> cnt(size_t(nparts) + 1, 0);
    for (int64_t v = 0; v < n; ++v) {
        if (part[v] < 0 || part[v] >= nparts) return CAGMRES_EINVAL;
        ++cnt[size_t(part[v]) + 1];
    }
    for (int p = 0; p < nparts; ++p) cnt[size_t(p) + 1] += cnt[size_t(p)];
    for (int p = 0; p <= nparts; ++p) row_starts[p] = cnt[size_t(p)];
    for (int64_t v = 0; v < n; ++v) perm[cnt[size_t(part[v])]++] = v;    // stable within a part
    return CAGMRES_OK;
}

}  // extern "C"
