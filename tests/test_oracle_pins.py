"""Pins of the oracle (oracle/cagmres_oracle.py) against things other than itself:
dense linear algebra, closed forms, brute force, invariants the paper states.
Each test names the passage it pins (P:n = /root/reference/PAPER.md line n)."""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp

from oracle import cagmres_oracle as O
from synth import generators as G


@pytest.fixture(scope="module")
def cd2():
    return G.convection_diffusion(32, 2, 5).to_scipy()


@pytest.fixture(scope="module")
def small():
    return G.convection_diffusion(6, 2, 5).to_scipy()          # n = 36, dense-friendly


# ----------------------------------------------------------------------------- MPK
def test_mpk_monomial_equals_dense_powers(small):
    A = small.toarray()
    q = G.u(3, np.arange(36))
    W = O.mpk(small, q, 6)
    for k in range(7):
        ref = np.linalg.matrix_power(A, k) @ q
        assert np.allclose(W[:, k], ref, rtol=1e-13, atol=1e-13 * np.abs(ref).max())


def test_mpk_newton_real_and_complex_pairs_equal_dense_product(small):
    A = small.toarray()
    q = G.u(4, np.arange(36))
    re = np.array([1.5, 3.0, 3.0, 0.25, 6.0])
    im = np.array([0.0, 0.7, -0.7, 0.0, 0.0])
    W = O.mpk(small, q, 5, re, im)
    acc = q.astype(np.complex128)
    I = np.eye(36)
    for k in range(5):
        acc = (A - complex(re[k], im[k]) * I) @ acc
        if k != 1:  # after the first half of a pair the Newton vector is not the complex product
            assert np.allclose(W[:, k + 1], acc.real, rtol=1e-12, atol=1e-12 * np.abs(acc).max())
            assert np.abs(acc.imag).max() < 1e-9 * np.abs(acc).max()
    # truncated pair at the end of a block -> real part (G10)
    W3 = O.mpk(small, q, 2, np.array([1.5, 3.0, 3.0]), np.array([0.0, 0.7, -0.7]))
    ref = (A - 3.0 * I) @ ((A - 1.5 * I) @ q)
    assert np.allclose(W3[:, 2], ref, rtol=1e-13)


@pytest.mark.parametrize("shifts", [None, ([2.0, 5.0, 5.0, 1.0], [0.0, 1.5, -1.5, 0.0])])
def test_change_of_basis_relation(cd2, shifts):
    q = G.u(5, np.arange(cd2.shape[0]))
    re, im = (None, None) if shifts is None else map(np.array, shifts)
    sb = 4
    W = O.mpk(cd2, q, sb, re, im)
    B = O.change_of_basis(sb, re, im)
    lhs = cd2 @ W[:, :sb]
    err = np.linalg.norm(lhs - W @ B) / (sp.linalg.norm(cd2) * np.linalg.norm(W))
    assert err < 1e-15 * 50


def test_newton_with_zero_shifts_is_monomial_bitwise(cd2):
    q = G.u(6, np.arange(cd2.shape[0]))
    W0 = O.mpk(cd2, q, 5)
    W1 = O.mpk(cd2, q, 5, np.zeros(5), np.zeros(5))
    assert np.array_equal(W0, W1)


# ----------------------------------------------------------------------------- BOrth
@pytest.mark.parametrize("kind", ["cgs", "mgs"])
def test_borth_projects_out(kind):
    Q, _ = np.linalg.qr(G.random_panel(500, 12, 1))
    P = G.random_panel(500, 5, 2)
    C, Pn = O.BORTH[kind](Q, P)
    assert np.abs(Q.T @ Pn).max() < 1e-13
    assert np.allclose(Q @ C + Pn, P, atol=1e-13)
    assert np.allclose(C, Q.T @ P, atol=1e-13)


def test_onepass_borth_cholqr_equals_two_pass():
    """One-pass BOrth+CholQR (NEXT-2) equals CGS BOrth followed by CholQR when Q^T Q = I
    (Pythagoras); pinned against the two-pass composition and against Householder QR of the
    explicitly projected panel."""
    Q, _ = np.linalg.qr(G.random_panel(3000, 20, 4))
    P = G.random_panel(3000, 6, 5)
    P[:, 0] = np.linalg.qr(np.column_stack([Q, P[:, 0]]))[0][:, -1]      # q_j orthonormal, _|_ Q
    P[:, 2] += 0.3 * Q[:, 5] + 0.2 * P[:, 1]
    C1, Qh1, R1 = O.borth_cholqr_onepass(Q, P)
    Cp, Pp = O.borth_cgs(Q, P[:, 1:])
    Qh2, R2 = O.tsqr_cholqr(np.column_stack([P[:, 0], Pp]))
    assert np.abs(C1 - Q.T @ P[:, 1:]).max() < 1e-13
    assert np.abs(C1 - Cp).max() < 1e-13
    assert np.abs(R1 - R2).max() < 1e-12 * np.abs(R2).max()
    assert np.abs(Qh1 - Qh2).max() < 1e-11
    Qr, Rr = _ref_qr(np.column_stack([P[:, 0], P[:, 1:] - Q @ (Q.T @ P[:, 1:])]))
    assert np.abs(R1 - Rr).max() < 1e-12 * np.abs(Rr).max()
    assert O.orth_error(np.column_stack([Q, Qh1])) < 1e-12


# ----------------------------------------------------------------------------- TSQR (Fig. 9/10)
def _ref_qr(P):
    Q, R = np.linalg.qr(P)
    s = np.sign(np.diag(R))
    return Q * s, s[:, None] * R


@pytest.mark.parametrize("kind", ["cholqr", "svqr", "mgs", "cgs", "caqr"])
def test_tsqr_matches_householder(kind):
    P = G.random_panel(2000, 11, 3)
    P[:, 3] += 0.5 * P[:, 2]                      # mildly correlated columns
    Q, R = O.TSQR[kind](P)
    Qr, Rr = _ref_qr(P)
    assert np.allclose(np.triu(R), R)
    assert np.all(np.diag(R) > 0)
    assert np.abs(R - Rr).max() < 1e-12 * np.abs(Rr).max()
    assert O.fact_error(P, Q, R) < 1e-14
    assert O.orth_error(Q) < 1e-13


def test_caqr_row_blocks_equal_single_block():
    P = G.random_panel(3001, 7, 4)
    Q1, R1 = O.tsqr_caqr(P, 1)
    Q3, R3 = O.tsqr_caqr(P, 3)
    assert np.abs(R1 - R3).max() < 1e-13 * np.abs(R1).max()
    assert np.abs(Q1 - Q3).max() < 1e-13


def test_cholqr_breaks_down_on_rank_deficient_panel():
    """'one of the column vectors is a linear combination ... Cholesky may fail'."""
    P = G.random_panel(300, 5, 5)
    P[:, 4] = P[:, 0] - 2.0 * P[:, 1]
    with pytest.raises(O.Breakdown):
        O.tsqr_cholqr(P)
    Q, R = O.tsqr_svqr(P)                         # SVQR still returns a finite R
    assert np.all(np.isfinite(R))


def test_cholqr_svqr_retry_factors_the_panel_cholqr_cannot():
    """G15 opt-in retry: where CholQR breaks down the panel is factored by SVQR —
    checked against the factorisation itself (P = QR, R upper, diag > 0), not against the
    oracle's own SVQR; a well-conditioned panel keeps the CholQR factor (Householder R)."""
    P = G.random_panel(300, 5, 5)
    P[:, 4] = P[:, 0] - 2.0 * P[:, 1]                          # rank deficient: pivot < 0 here
    with pytest.raises(O.Breakdown):
        O.tsqr_cholqr(P)
    Q, R = O.tsqr_cholqr_svqr_retry(P)
    assert np.allclose(np.tril(R, -1), 0.0) and np.all(np.diag(R) > 0)
    assert O.fact_error(P, Q, R) < 1e-12
    assert np.allclose(Q[:, :4].T @ Q[:, :4], np.eye(4), atol=1e-12)   # the independent part
    Pw = G.random_panel(3000, 6, 9)
    Qw, Rw = O.tsqr_cholqr_svqr_retry(Pw)
    _, Rh = np.linalg.qr(Pw)
    Rh = np.sign(np.diag(Rh))[:, None] * Rh
    assert np.allclose(Rw, Rh, rtol=1e-12, atol=1e-12 * np.abs(Rh).max())


def test_orthogonality_ordering_fig10():
    """Fig. 10: ||I-Q^TQ|| is O(eps k^2) CholQR/SVQR, O(eps k) MGS, O(eps) CAQR."""
    rng_panel = G.random_panel(4000, 8, 6)
    U, _ = np.linalg.qr(rng_panel)
    V, _ = np.linalg.qr(G.random_panel(8, 8, 7))
    P = U @ np.diag(np.logspace(0, -6, 8)) @ V.T      # kappa = 1e6
    e = {k: O.orth_error(O.TSQR[k](P)[0]) for k in ("cholqr", "svqr", "mgs", "caqr")}
    assert e["caqr"] < 1e-14
    assert e["mgs"] < 1e-8 and e["mgs"] > 10 * e["caqr"]
    assert e["cholqr"] > 10 * e["mgs"] and e["svqr"] > 10 * e["mgs"]
    # CholQR twice ("2x") restores orthogonality
    Q1, R1 = O.tsqr_cholqr(P)
    Q2, R2 = O.tsqr_cholqr(Q1)
    assert O.orth_error(Q2) < 1e-14
    assert O.fact_error(P, Q2, R2 @ R1) < 1e-14


# ----------------------------------------------------------------------------- LS
def test_givens_ls_matches_lstsq():
    m = 12
    H = np.triu(G.random_panel(m + 1, m, 8), -1)
    H[np.arange(1, m + 1), np.arange(m)] = np.abs(H[np.arange(1, m + 1), np.arange(m)]) + 0.1
    y, res = O.givens_ls(H, 2.5)
    rhs = np.zeros(m + 1); rhs[0] = 2.5
    yr = np.linalg.lstsq(H, rhs, rcond=None)[0]
    assert np.allclose(y, yr, rtol=1e-12, atol=1e-12)
    assert res[-1] == pytest.approx(np.linalg.norm(rhs - H @ yr), rel=1e-10)
    assert np.all(np.diff(res) <= 1e-15)              # residual estimates non-increasing


# ----------------------------------------------------------------------------- H update (G1)
@pytest.mark.parametrize("tsqr,reorth,onepass", [("cholqr", False, False), ("cholqr", True, False),
                                                 ("svqr", False, False), ("mgs", False, False),
                                                 ("caqr", False, False), ("cgs", True, False),
                                                 ("cholqr", False, True), ("cholqr", True, True)])
def test_ca_cycle_arnoldi_relation_and_gmres_equivalence(cd2, tsqr, reorth, onepass):
    n = cd2.shape[0]
    b = G.rhs(n)
    m, s = 30, 5
    re, im = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(cd2, b, m)[1], m), s)
    Q = np.zeros((n, m + 1), order="F"); Q[:, 0] = b / np.linalg.norm(b)
    H = np.zeros((m + 1, m))
    O.ca_cycle(cd2, Q, H, s, m, re, im, tsqr=tsqr, reorth=reorth, onepass=onepass)
    Aop = sp.linalg.norm(cd2)
    assert np.linalg.norm(cd2 @ Q[:, :m] - Q @ H) / Aop < 1e-12
    assert np.allclose(np.tril(H, -2), 0.0)            # exactly upper Hessenberg
    Qg, Hg, _ = O.arnoldi_mgs(cd2, b, m)
    assert np.linalg.norm(H - Hg) / np.linalg.norm(Hg) < 1e-10
    assert O.orth_error(Q) < 1e-10


def test_first_cycle_equals_brute_force_krylov_least_squares(cd2):
    """GMRES minimises ||b - A x|| over x in K_m(A, b) ([3]); brute force with a
    dense orthonormalised power basis and lstsq."""
    n = cd2.shape[0]
    b = G.rhs(n)
    m = 8
    K = np.zeros((n, m))
    v = b.copy()
    for k in range(m):
        K[:, k] = v / np.linalg.norm(v)
        v = cd2 @ K[:, k]
    Kq, _ = np.linalg.qr(K)
    y = np.linalg.lstsq(cd2 @ Kq, b, rcond=None)[0]
    rho_bf = np.linalg.norm(b - cd2 @ (Kq @ y)) / np.linalg.norm(b)
    for kw in (dict(basis="monomial", s=4), dict(basis="newton", s=4),
               dict(basis="newton", s=3, tsqr="mgs", reorth=True)):
        r = O.cagmres(cd2, b, kw.pop("s"), m, maxcyc=1, **kw)
        assert r["hist"][0] == pytest.approx(rho_bf, rel=1e-8)
    g = O.gmres(cd2, b, m, maxcyc=1)
    assert g["hist"][0] == pytest.approx(rho_bf, rel=1e-8)


def test_s1_is_gmres(cd2):
    """CA-GMRES(1, m) == GMRES(m) in exact arithmetic."""
    b = G.rhs(cd2.shape[0])
    ca = O.cagmres(cd2, b, 1, 30, basis="monomial", reorth=True, maxcyc=4, tol=0)
    g = O.gmres(cd2, b, 30, maxcyc=4, tol=0)
    assert np.allclose(ca["hist"], g["hist"], rtol=1e-8)


# ----------------------------------------------------------------------------- whole solve
@pytest.mark.parametrize("basis,tsqr,reorth,onepass", [("newton", "cholqr", False, False),
                                                       ("monomial", "cholqr", False, False),
                                                       ("newton", "cholqr", True, False),
                                                       ("newton", "svqr", False, False),
                                                       ("newton", "cholqr", True, True)])
def test_solve_matches_dense_direct(cd2, basis, tsqr, reorth, onepass):
    b = G.rhs(cd2.shape[0])
    r = O.cagmres(cd2, b, 5, 30, basis=basis, tsqr=tsqr, reorth=reorth, tol=1e-8, onepass=onepass)
    xs = np.linalg.solve(cd2.toarray(), b)
    kappa = np.linalg.cond(cd2.toarray())
    assert r["hist"][-1] <= 1e-8
    assert np.linalg.norm(r["x"] - xs) / np.linalg.norm(xs) <= kappa * 1e-8
    assert np.all(np.diff(r["hist"]) <= 0)             # monotone
    g = O.gmres(cd2, b, 30, tol=1e-8)
    assert abs(r["cycles"] - g["cycles"]) <= 1         # same restarts


# ----------------------------------------------------------------------------- Leja (G10)
def test_modified_leja_greedy_product_bruteforce():
    """Partial pin: each chosen point maximises the product of distances (direct product,
    not the oracle's log-sum) over the remaining candidates; pairs adjacent, +im first."""
    pts = np.array([3.0, -1.0 + 2.0j, -1.0 - 2.0j, 0.5, 2.0 + 0.5j, 2.0 - 0.5j, -2.5])
    re, im = O.modified_leja(pts, 7)
    out = re + 1j * im
    assert sorted(np.round(out, 12), key=lambda z: (z.real, z.imag)) == \
        sorted(np.round(pts, 12), key=lambda z: (z.real, z.imag))
    assert abs(out[0]) == max(abs(pts))
    i = 0
    chosen = []
    reps = [z for z in pts if z.imag >= 0]
    while i < len(out):
        z = out[i]
        remaining = [c for c in reps if not any(abs(c - x) == 0 for x in chosen)]
        if chosen:
            prod = {c: np.prod([abs(c - x) for x in chosen]) for c in remaining}
            assert prod[complex(z)] == max(prod.values())
        chosen.append(complex(z))
        if z.imag > 0:
            assert out[i + 1] == np.conj(z)
            chosen.append(complex(np.conj(z)))
            i += 2
        else:
            i += 1


def test_leja_exhaustive_first_pair_maximises_distance():
    pts = np.array([1.0, 4.0, -3.0, 0.5, 2.5, -1.0, 3.5, -2.0])
    re, _ = O.modified_leja(pts, 8)
    best = max(itertools.permutations(pts, 2),
               key=lambda p: (abs(p[0]) == max(abs(pts))) * 100 + abs(p[0] - p[1]))
    assert (re[0], re[1]) == best


@pytest.mark.parametrize("pts,want_re,want_im", [
    # first point: |3| == |-3| -> the larger real part (G10); then the farther point
    ([-3.0, 3.0, 1.0], [3.0, -3.0, 1.0], [0.0, 0.0, 0.0]),
    # max modulus is the pair 0 +- 5i (+im first); then -1 and 1 score log 26 each: tie ->
    # the first in (re, im) order, i.e. -1
    ([-1.0, 1.0, 5j, -5j], [0.0, 0.0, -1.0, 1.0], [5.0, -5.0, 0.0, 0.0]),
    # a repeated value stays a separate candidate with score -inf: it goes last
    ([2.0, 2.0, -1.0], [2.0, -1.0, 2.0], [0.0, 0.0, 0.0]),
    # two pairs of equal modulus: larger real part first; the other pair follows its partner
    ([1 + 1j, 1 - 1j, -1 + 1j, -1 - 1j], [1.0, 1.0, -1.0, -1.0], [1.0, -1.0, 1.0, -1.0]),
])
def test_modified_leja_tie_breaking_by_hand(pts, want_re, want_im):
    """Ties resolved by hand from the G10 reading, not from the oracle: first
    point max |theta| with ties to the larger real part; then argmax of the log-distance sum with
    ties to the first candidate in (re, im) order; repeats score -inf."""
    re, im = O.modified_leja(np.array(pts, dtype=np.complex128), len(pts))
    assert np.array_equal(re, np.array(want_re)) and np.array_equal(im, np.array(want_im))


def test_ritz_values_full_krylov_space_recover_known_spectrum():
    """Pin of ritz_values (+ the CGS Arnoldi that feeds it): with m = n the Krylov space is the
    whole space, so the Ritz values of H[0:n,0:n] are the eigenvalues of A.  A is a
    dense orthogonal similarity of a block-diagonal matrix with KNOWN eigenvalues (real ones
    and a +- i b pairs from 2x2 rotation-scaling blocks)."""
    lam_real = [3.0, -1.5, 0.75, 5.0]
    pairs = [(1.0, 2.0), (-2.0, 0.5)]
    n = len(lam_real) + 2 * len(pairs)
    D = np.zeros((n, n))
    for i, lr in enumerate(lam_real):
        D[i, i] = lr
    k = len(lam_real)
    for a, b in pairs:
        D[k:k + 2, k:k + 2] = [[a, b], [-b, a]]
        k += 2
    Qm, _ = np.linalg.qr(G.random_panel(n, n, 5))
    A = Qm @ D @ Qm.T
    import scipy.sparse as sp
    _, H, _ = O.arnoldi_cgs2(sp.csr_matrix(A), G.u(3, np.arange(n)), n)
    ritz = np.sort_complex(O.ritz_values(H, n))
    want = np.sort_complex(np.array(lam_real + [complex(a, s * b) for a, b in pairs for s in (1, -1)]))
    assert np.allclose(ritz, want, rtol=0, atol=1e-10)


# ----------------------------------------------------------------------------- boundary sets
def test_boundary_sets_vs_dense_reachability():
    A = G.g3_shaped(n=400, width=20).to_scipy()
    D = (A.toarray() != 0).astype(np.int64)
    own = (120, 260)
    s = 4
    lv = O.boundary_sets(A, *own, s)
    reach = np.zeros(400, dtype=bool); reach[own[0]:own[1]] = True
    for h in range(1, s + 1):
        nxt = (D[reach].sum(axis=0) > 0) | reach
        ref = np.flatnonzero(nxt & ~reach)
        assert np.array_equal(lv[h - 1], ref)
        reach = nxt


def test_boundary_sets_slab_closed_form():
    """Natural-ordered 5-point grid split in row blocks: level h is one grid row per side."""
    N = 10
    A = G.convection_diffusion(N, 2, 5).to_scipy()
    lv = O.boundary_sets(A, 4 * N, 6 * N, 3)
    for h in range(1, 4):
        ref = np.r_[np.arange((4 - h) * N, (5 - h) * N), np.arange((5 + h) * N, (6 + h) * N)]
        assert np.array_equal(lv[h - 1], ref)
    starts = O.block_rows(1001, 8)
    assert starts[0] == 0 and starts[-1] == 1001 and np.ptp(np.diff(starts)) <= 1
