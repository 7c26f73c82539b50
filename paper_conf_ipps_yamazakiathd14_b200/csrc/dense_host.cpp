// dense_host.cpp — the tiny host work of one restart cycle:
// change-of-basis B, Hessenberg update, Givens least squares, Ritz values (Francis
// double-shift QR on the Hessenberg matrix) and modified Leja ordering of the shifts.
// All O(m^2)-O(m^3) with m <= a few hundred; column-major.
#include <algorithm>
#include <cfloat>
#include <cmath>
#include <cstring>

#include "internal.h"

namespace host {

std::vector<Step> block_steps(const std::vector<double>& re, const std::vector<double>& im, int sb) {
    // G10: first sb shifts; a conjugate pair a +- ib occupies two consecutive steps; a pair
    // truncated at the block end is replaced by its real part.
    std::vector<Step> st;
    int k = 0;
    while (k < sb) {
        const double a = k < int(re.size()) ? re[size_t(k)] : 0.0;
        const double b = k < int(im.size()) ? im[size_t(k)] : 0.0;
        if (b > 0.0 && k + 1 < sb) {
            st.push_back({a, 0.0, 1});
            st.push_back({a, b * b, 2});
            k += 2;
        } else {
            st.push_back({a, 0.0, 0});
            k += 1;
        }
    }
    return st;
}

void change_of_basis(const std::vector<Step>& st, int sb, double* B) {
    // A W[:,0:sb] = W B  (P:94 via [4]): real theta: B[c,c] = theta, B[c+1,c] = 1;
    // second step of a pair: additionally B[c-1,c] = -b^2.
    const int ld = sb + 1;
    std::memset(B, 0, sizeof(double) * size_t(ld) * size_t(sb));
    for (int c = 0; c < sb; ++c) {
        B[c + ld * c] = st[size_t(c)].a;
        B[c + 1 + ld * c] = 1.0;
        if (st[size_t(c)].kind == 2) B[c - 1 + ld * c] = -st[size_t(c)].b2;
    }
}

int hessenberg_update(double* H, int ldh, int j, int sb, const double* Rt, int ldr,
                      const double* B) {
    // H[0:j+sb+1, j:j+sb] = (Rt B - [H[0:j+1,0:j] Rt[0:j,0:sb] ; 0]) T^{-1},
    // T = Rt[j:j+sb, 0:sb] upper triangular.
    const int nr = j + sb + 1, ldb = sb + 1;
    std::vector<double> M(size_t(nr) * size_t(sb), 0.0);
    for (int c = 0; c < sb; ++c)
        for (int i = 0; i < nr; ++i) {
            double acc = 0.0;
            for (int k = 0; k <= sb; ++k) acc += Rt[i + size_t(ldr) * k] * B[k + size_t(ldb) * c];
            M[i + size_t(nr) * c] = acc;
        }
    for (int c = 0; c < sb; ++c)
        for (int i = 0; i <= j && j > 0; ++i) {
            double acc = 0.0;
            for (int k = 0; k < j; ++k) acc += H[i + size_t(ldh) * k] * Rt[k + size_t(ldr) * c];
            M[i + size_t(nr) * c] -= acc;
        }
    for (int i = 0; i < nr; ++i) {
        for (int c = 0; c < sb; ++c) {
            double x = M[i + size_t(nr) * c];
            for (int k = 0; k < c; ++k) x -= H[i + size_t(ldh) * (j + k)] * Rt[j + k + size_t(ldr) * c];
            const double t = Rt[j + c + size_t(ldr) * c];
            if (t == 0.0 || !std::isfinite(t)) return CAGMRES_EBREAKDOWN;
            H[i + size_t(ldh) * (j + c)] = x / t;
        }
    }
    return CAGMRES_OK;
}

int givens_ls(const double* Hin, int ldh, int k, double beta, double* y, double* res) {
    std::vector<double> H(size_t(k + 1) * size_t(k));
    for (int c = 0; c < k; ++c)
        for (int i = 0; i <= k; ++i) H[i + size_t(k + 1) * c] = Hin[i + size_t(ldh) * c];
    auto h = [&](int i, int c) -> double& { return H[i + size_t(k + 1) * c]; };
    std::vector<double> g(size_t(k) + 1, 0.0);
    g[0] = beta;
    for (int i = 0; i < k; ++i) {
        const double a = h(i, i), b = h(i + 1, i);
        const double r = std::hypot(a, b);
        const double cs = r == 0.0 ? 1.0 : a / r, sn = r == 0.0 ? 0.0 : b / r;
        for (int c = i; c < k; ++c) {
            const double u = h(i, c), v = h(i + 1, c);
            h(i, c) = cs * u + sn * v;
            h(i + 1, c) = -sn * u + cs * v;
        }
        const double gi = g[size_t(i)];
        g[size_t(i)] = cs * gi;
        g[size_t(i) + 1] = -sn * gi;
        if (res) res[i] = std::fabs(g[size_t(i) + 1]);
    }
    for (int i = k - 1; i >= 0; --i) {
        double x = g[size_t(i)];
        for (int c = i + 1; c < k; ++c) x -= h(i, c) * y[c];
        if (h(i, i) == 0.0) return CAGMRES_EBREAKDOWN;
        y[i] = x / h(i, i);
    }
    return CAGMRES_OK;
}

static void eig2(double a, double b, double c, double d, double* r1, double* i1, double* r2, double* i2) {
    const double p = 0.5 * (a - d);
    const double q = p * p + b * c;
    if (q >= 0.0) {
        const double z = p + std::copysign(std::sqrt(q), p);
        *r1 = d + z;
        *r2 = (z != 0.0) ? d - b * c / z : d + z;
        *i1 = *i2 = 0.0;
    } else {
        *r1 = *r2 = d + p;
        *i1 = std::sqrt(-q);
        *i2 = -*i1;
    }
}

int hessenberg_eigvals(const double* Hin, int ldh, int m, double* wr, double* wi) {
    // Francis implicit double-shift QR (Golub & Van Loan, Alg. 7.5.1) with deflation,
    // eigenvalues only: transforms are confined to the active window [lo, hi].
    if (m <= 0) return CAGMRES_OK;
    std::vector<double> a(size_t(m) * size_t(m), 0.0);
    auto A = [&](int i, int j) -> double& { return a[size_t(i) + size_t(m) * size_t(j)]; };
    double nrm = 0.0;
    for (int j = 0; j < m; ++j)
        for (int i = 0; i <= std::min(j + 1, m - 1); ++i) {
            A(i, j) = Hin[i + size_t(ldh) * j];
            nrm += std::fabs(A(i, j));
        }
    if (nrm == 0.0) nrm = 1.0;
    int hi = m - 1, its = 0, total = 0;
    while (hi >= 0) {
        int lo = hi;
        while (lo > 0) {
            double s = std::fabs(A(lo - 1, lo - 1)) + std::fabs(A(lo, lo));
            if (s == 0.0) s = nrm;
            if (std::fabs(A(lo, lo - 1)) <= DBL_EPSILON * s) { A(lo, lo - 1) = 0.0; break; }
            --lo;
        }
        if (lo == hi) { wr[hi] = A(hi, hi); wi[hi] = 0.0; --hi; its = 0; continue; }
        if (lo == hi - 1) {
            eig2(A(hi - 1, hi - 1), A(hi - 1, hi), A(hi, hi - 1), A(hi, hi),
                 &wr[hi - 1], &wi[hi - 1], &wr[hi], &wi[hi]);
            hi -= 2; its = 0; continue;
        }
        if (++total > 60 * m) return CAGMRES_EBREAKDOWN;
        ++its;
        double s, t;
        if (its % 11 == 10) {                      // exceptional shift
            const double w = std::fabs(A(hi, hi - 1)) + std::fabs(A(hi - 1, hi - 2));
            s = 1.5 * w;
            t = w * w;
        } else {
            s = A(hi - 1, hi - 1) + A(hi, hi);
            t = A(hi - 1, hi - 1) * A(hi, hi) - A(hi - 1, hi) * A(hi, hi - 1);
        }
        double x = A(lo, lo) * A(lo, lo) + A(lo, lo + 1) * A(lo + 1, lo) - s * A(lo, lo) + t;
        double y = A(lo + 1, lo) * (A(lo, lo) + A(lo + 1, lo + 1) - s);
        double z = A(lo + 1, lo) * A(lo + 2, lo + 1);
        for (int k = lo; k <= hi - 2; ++k) {
            const double nv = std::sqrt(x * x + y * y + z * z);
            if (nv != 0.0) {
                const double alpha = -std::copysign(nv, x);
                const double v0 = x - alpha, v1 = y, v2 = z;
                const double beta = 2.0 / (v0 * v0 + v1 * v1 + v2 * v2);
                for (int c = std::max(lo, k - 1); c <= hi; ++c) {
                    const double d = beta * (v0 * A(k, c) + v1 * A(k + 1, c) + v2 * A(k + 2, c));
                    A(k, c) -= d * v0; A(k + 1, c) -= d * v1; A(k + 2, c) -= d * v2;
                }
                for (int r = lo; r <= std::min(k + 3, hi); ++r) {
                    const double d = beta * (A(r, k) * v0 + A(r, k + 1) * v1 + A(r, k + 2) * v2);
                    A(r, k) -= d * v0; A(r, k + 1) -= d * v1; A(r, k + 2) -= d * v2;
                }
            }
            x = A(k + 1, k);
            y = A(k + 2, k);
            if (k < hi - 2) z = A(k + 3, k);
        }
        {
            const int k = hi - 1;
            const double nv = std::hypot(x, y);
            if (nv != 0.0) {
                const double alpha = -std::copysign(nv, x);
                const double v0 = x - alpha, v1 = y;
                const double beta = 2.0 / (v0 * v0 + v1 * v1);
                for (int c = std::max(lo, k - 1); c <= hi; ++c) {
                    const double d = beta * (v0 * A(k, c) + v1 * A(k + 1, c));
                    A(k, c) -= d * v0; A(k + 1, c) -= d * v1;
                }
                for (int r = lo; r <= hi; ++r) {
                    const double d = beta * (A(r, k) * v0 + A(r, k + 1) * v1);
                    A(r, k) -= d * v0; A(r, k + 1) -= d * v1;
                }
            }
        }
    }
    return CAGMRES_OK;
}

void modified_leja(const double* wr, const double* wi, int cnt, int s,
                   std::vector<double>& ore, std::vector<double>& oim) {
    // G10: candidates = Ritz values with im >= 0 sorted by (re, im); first = max modulus
    // (tie: larger re); then argmax sum log|z - chosen| (ties: first in sorted order);
    // a complex choice is followed by its conjugate.
    struct C { double re, im; };
    std::vector<C> cand;
    for (int i = 0; i < cnt; ++i)
        if (wi[i] >= 0.0) cand.push_back({wr[i], wi[i]});
    std::stable_sort(cand.begin(), cand.end(), [](const C& x, const C& y) {
        return x.re < y.re || (x.re == y.re && x.im < y.im);
    });
    ore.clear(); oim.clear();
    if (cand.empty()) return;
    std::vector<char> used(cand.size(), 0);
    std::vector<C> chosen;
    auto push = [&](size_t i) {
        used[i] = 1;
        ore.push_back(cand[i].re); oim.push_back(cand[i].im); chosen.push_back(cand[i]);
        if (cand[i].im > 0.0) {
            ore.push_back(cand[i].re); oim.push_back(-cand[i].im); chosen.push_back({cand[i].re, -cand[i].im});
        }
    };
    size_t first = 0;
    for (size_t i = 1; i < cand.size(); ++i) {
        const double mi = std::hypot(cand[i].re, cand[i].im), mf = std::hypot(cand[first].re, cand[first].im);
        if (mi > mf || (mi == mf && cand[i].re > cand[first].re)) first = i;
    }
    push(first);
    while (int(ore.size()) < s) {
        bool any = false;
        size_t best = 0;
        double bsc = 0.0;
        for (size_t i = 0; i < cand.size(); ++i) {
            if (used[i]) continue;
            double sc = 0.0;
            for (const C& c : chosen) sc += std::log(std::hypot(cand[i].re - c.re, cand[i].im - c.im));
            if (!any || sc > bsc) { any = true; best = i; bsc = sc; }
        }
        if (!any) break;
        push(best);
    }
}

// Eigenvalues of the symmetric n x n matrix A (ld lda; only the upper triangle is read) by
// cyclic Jacobi rotations (Golub & Van Loan 8.5); ascending.  For the per-panel diagnostics:
// kappa_2 of a Gram matrix and ||I - Q^T Q||_2.
void sym_eigvals(const double* A, int lda, int n, double* ev) {
    std::vector<double> M(size_t(n) * size_t(n));
    for (int c = 0; c < n; ++c)
        for (int i = 0; i < n; ++i)
            M[size_t(i) + size_t(n) * c] = i <= c ? A[size_t(i) + size_t(lda) * c] : A[size_t(c) + size_t(lda) * i];
    auto at = [&](int i, int c) -> double& { return M[size_t(i) + size_t(n) * c]; };
    for (int sweep = 0; sweep < 100; ++sweep) {
        double off = 0.0, tot = 0.0;
        for (int c = 0; c < n; ++c)
            for (int i = 0; i < n; ++i) {
                tot += at(i, c) * at(i, c);
                if (i != c) off += at(i, c) * at(i, c);
            }
        if (off <= 1e-34 * tot || off == 0.0) break;
        for (int p = 0; p < n - 1; ++p)
            for (int q = p + 1; q < n; ++q) {
                const double apq = at(p, q);
                if (apq == 0.0) continue;
                const double theta = (at(q, q) - at(p, p)) / (2.0 * apq);
                const double t = (theta >= 0.0 ? 1.0 : -1.0) / (std::fabs(theta) + std::sqrt(theta * theta + 1.0));
                const double cs = 1.0 / std::sqrt(t * t + 1.0), sn = t * cs;
                for (int k = 0; k < n; ++k) {            // columns p, q
                    const double akp = at(k, p), akq = at(k, q);
                    at(k, p) = cs * akp - sn * akq;
                    at(k, q) = sn * akp + cs * akq;
                }
                for (int k = 0; k < n; ++k) {            // rows p, q
                    const double apk = at(p, k), aqk = at(q, k);
                    at(p, k) = cs * apk - sn * aqk;
                    at(q, k) = sn * apk + cs * aqk;
                }
            }
    }
    for (int i = 0; i < n; ++i) ev[i] = at(i, i);
    std::sort(ev, ev + n);
}

}  // namespace host

// ---------------------------------------------------------------------------------------
// C ABI wrappers of the host algorithms (used by the solver and by the CPU tests)
// ---------------------------------------------------------------------------------------
extern "C" {

int cagmres_host_eigvals(const double* H, int ldh, int m, double* wr, double* wi) {
    if (!H || !wr || !wi || m < 0 || ldh < m) return CAGMRES_EINVAL;
    return host::hessenberg_eigvals(H, ldh, m, wr, wi);
}

int cagmres_host_leja(const double* wr, const double* wi, int cnt, int s, double* ore,
                      double* oim, int cap, int* nout) {
    if (!wr || !wi || !ore || !oim || !nout || cnt < 0) return CAGMRES_EINVAL;
    std::vector<double> r, i;
    host::modified_leja(wr, wi, cnt, s, r, i);
    const int n = std::min(int(r.size()), cap);
    for (int k = 0; k < n; ++k) { ore[k] = r[size_t(k)]; oim[k] = i[size_t(k)]; }
    *nout = int(r.size());
    return CAGMRES_OK;
}

int cagmres_host_change_of_basis(const double* re, const double* im, int sb, double* B) {
    if (!re || !im || !B || sb < 1) return CAGMRES_EINVAL;
    std::vector<double> r(re, re + sb), i(im, im + sb);
    host::change_of_basis(host::block_steps(r, i, sb), sb, B);
    return CAGMRES_OK;
}

int cagmres_host_hessenberg_update(double* H, int ldh, int j, int sb, const double* Rt,
                                   int ldr, const double* B) {
    if (!H || !Rt || !B || j < 0 || sb < 1 || ldh < j + sb + 1 || ldr < j + sb + 1)
        return CAGMRES_EINVAL;
    return host::hessenberg_update(H, ldh, j, sb, Rt, ldr, B);
}

int cagmres_host_sym_eigvals(const double* A, int lda, int n, double* ev) {
    if (!A || !ev || n < 1 || lda < n) return CAGMRES_EINVAL;
    host::sym_eigvals(A, lda, n, ev);
    return CAGMRES_OK;
}

int cagmres_host_givens_ls(const double* H, int ldh, int k, double beta, double* y, double* res) {
    if (!H || !y || k < 1 || ldh < k + 1) return CAGMRES_EINVAL;
    return host::givens_ls(H, ldh, k, beta, y, res);
}

}  // extern "C"
