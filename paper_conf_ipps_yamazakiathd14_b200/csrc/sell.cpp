// sell.cpp — host construction of the SELL-32 matrix layout; pure
// host code (no CUDA), also exported through the C ABI so the layout can be checked on a CPU.
#include <algorithm>
#include <climits>
#include <cstring>

#include "internal.h"

// SELL-32 with per-slice diagonal-offset column compression.  A slice
// (32 consecutive rows, one warp) whose rows' column offsets col - row take few distinct
// values (stencils, banded and most PDE matrices) is stored DIA-style: one int32 offset per
// stored "diagonal" plus 32 values per diagonal (exact zeros where a row lacks it), so the
// column stream drops from 4 B to ~4/32 B per stored entry.  Other slices keep explicit
// column indices.  Every row is summed in GLOBAL column order in both modes (the plan's rows
// are in global column order): in a DIA slice the diagonals are ordered by a topological
// sort of the per-row orders — on a single GPU that is increasing offset, on a rank > 0 the
// ghost columns (extended ids >= n_loc) that precede the owned ones globally come first — and
// a slice whose rows admit no common order keeps explicit columns.  So a row's value does not
// depend on the partition (tests: multi-rank MPK bitwise equal to the single-GPU MPK).
namespace {
// Diagonal order of one slice consistent with every row's entry order; false if none exists.
bool dia_order(const cagmres_plan& p, int64_t r0, int64_t r1, const std::vector<int64_t>& u,
               std::vector<int32_t>& order) {
    const size_t k = u.size();
    std::vector<uint32_t> succ(k, 0);                  // bitmask of successors (k <= 32)
    std::vector<int> indeg(k, 0);
    auto slot = [&](int64_t o) { return size_t(std::lower_bound(u.begin(), u.end(), o) - u.begin()); };
    for (int64_t r = r0; r < r1; ++r) {
        size_t prev = k;
        for (int64_t e = p.rowptr[size_t(r)]; e < p.rowptr[size_t(r) + 1]; ++e) {
            const size_t c = slot(int64_t(p.colind[size_t(e)]) - r);
            if (prev < k && !(succ[prev] >> c & 1u)) { succ[prev] |= 1u << c; ++indeg[c]; }
            prev = c;
        }
    }
    order.clear();
    uint32_t used = 0;
    for (size_t it = 0; it < k; ++it) {                 // Kahn: smallest available offset first
        size_t pick = k;
        for (size_t c = 0; c < k; ++c)
            if (!(used >> c & 1u) && indeg[c] == 0) { pick = c; break; }
        if (pick == k) return false;                    // cycle: no common order
        used |= 1u << pick;
        order.push_back(int32_t(u[pick]));
        for (size_t c = 0; c < k; ++c)
            if (succ[pick] >> c & 1u) --indeg[c];
    }
    return true;
}
}  // namespace

void sell_build(const cagmres_plan& p, SellHost& out) {
    const int64_t nr = p.n_mat;
    const int64_t ns = (nr + 31) / 32;
    std::vector<int64_t> sptr(size_t(ns) + 1, 0), sinfo(static_cast<size_t>(ns));
    std::vector<std::vector<int32_t>> offs(static_cast<size_t>(ns));
    std::vector<char> dia(static_cast<size_t>(ns), 0);
    int64_t ndcol = 0, ndia = 0;
    std::vector<int64_t> o;
    std::vector<int32_t> order;
    for (int64_t sl = 0; sl < ns; ++sl) {
        int64_t wmax = 0;
        o.clear();
        const int64_t r0 = sl * 32, r1 = std::min(nr, sl * 32 + 32);
        for (int64_t r = r0; r < r1; ++r) {
            wmax = std::max(wmax, p.rowptr[size_t(r) + 1] - p.rowptr[size_t(r)]);
            for (int64_t e = p.rowptr[size_t(r)]; e < p.rowptr[size_t(r) + 1]; ++e)
                o.push_back(int64_t(p.colind[size_t(e)]) - r);
        }
        std::sort(o.begin(), o.end());
        o.erase(std::unique(o.begin(), o.end()), o.end());
        const bool use_dia = int64_t(o.size()) <= wmax + (wmax + 3) / 4 && o.size() <= 32 &&
                             (o.empty() || (o.front() > INT32_MIN / 2 && o.back() < INT32_MAX / 2)) &&
                             dia_order(p, r0, r1, o, order);
        int64_t wdt = wmax;
        if (use_dia) {
            dia[size_t(sl)] = 1;
            ++ndia;
            wdt = int64_t(o.size());
            offs[size_t(sl)] = order;
            // clamp flag: some row + offset of this slice (padding lanes included) leaves [0, n_ext)
            const bool clamp = !o.empty() && (r0 + o.front() < 0 || sl * 32 + 31 + o.back() >= p.n_ext);
            sinfo[size_t(sl)] = (ndcol << 2) | (clamp ? 2 : 0) | 1;
            ndcol += wdt;
        } else {
            sinfo[size_t(sl)] = ndcol << 2;
            ndcol += 32 * wdt;
        }
        sptr[size_t(sl) + 1] = sptr[size_t(sl)] + 32 * wdt;
    }
    const int64_t tot = sptr[size_t(ns)];
    std::vector<int32_t> dcol(static_cast<size_t>(ndcol));
    std::vector<double> val(static_cast<size_t>(tot), 0.0);
    for (int64_t sl = 0; sl < ns; ++sl) {
        const int64_t wdt = (sptr[size_t(sl) + 1] - sptr[size_t(sl)]) / 32;
        const int64_t dp = sinfo[size_t(sl)] >> 2;
        if (dia[size_t(sl)]) {
            const std::vector<int32_t>& of = offs[size_t(sl)];
            for (int64_t t = 0; t < wdt; ++t) dcol[size_t(dp + t)] = of[size_t(t)];
            for (int lane = 0; lane < 32; ++lane) {
                const int64_t r = sl * 32 + lane;
                if (r >= nr) continue;
                for (int64_t e = p.rowptr[size_t(r)]; e < p.rowptr[size_t(r) + 1]; ++e) {
                    const int64_t off = int64_t(p.colind[size_t(e)]) - r;
                    int64_t t = 0;
                    while (of[size_t(t)] != off) ++t;          // present: of holds every offset of the slice
                    val[size_t(sptr[size_t(sl)] + 32 * t + lane)] = p.val[size_t(e)];
                }
            }
        } else {
            for (int lane = 0; lane < 32; ++lane) {
                const int64_t r = sl * 32 + lane;
                const int64_t b = r < nr ? p.rowptr[size_t(r)] : 0, e = r < nr ? p.rowptr[size_t(r) + 1] : 0;
                for (int64_t t = 0; t < wdt; ++t) {
                    const int64_t o = sptr[size_t(sl)] + 32 * t + lane;
                    if (b + t < e) {
                        dcol[size_t(dp + 32 * t + lane)] = p.colind[size_t(b + t)];
                        val[size_t(o)] = p.val[size_t(b + t)];
                    } else {
                        dcol[size_t(dp + 32 * t + lane)] = int32_t(r < nr ? r : 0);
                    }
                }
            }
        }
    }
    out.nslices = ns;
    out.ndia = ndia;
    out.sptr.swap(sptr);
    out.sinfo.swap(sinfo);
    out.dcol.swap(dcol);
    out.val.swap(val);
}

extern "C" {

int cagmres_plan_sell(cagmres_plan_t p, int64_t* nslices, int64_t* ndcol, int64_t* nstored,
                      int64_t* sptr, int64_t* sinfo, int32_t* dcol, double* val) {
    if (!p) return CAGMRES_EINVAL;
    SellHost sh;
    try {
        sell_build(*p, sh);
    } catch (...) {
        return CAGMRES_ENOMEM;
    }
    if (nslices) *nslices = sh.nslices;
    if (ndcol) *ndcol = int64_t(sh.dcol.size());
    if (nstored) *nstored = int64_t(sh.val.size());
    if (sptr) std::memcpy(sptr, sh.sptr.data(), sizeof(int64_t) * sh.sptr.size());
    if (sinfo) std::memcpy(sinfo, sh.sinfo.data(), sizeof(int64_t) * sh.sinfo.size());
    if (dcol) std::memcpy(dcol, sh.dcol.data(), sizeof(int32_t) * sh.dcol.size());
    if (val) std::memcpy(val, sh.val.data(), sizeof(double) * sh.val.size());
    return CAGMRES_OK;
}

}  // extern "C"
