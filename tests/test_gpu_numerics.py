"""GPU numerics beyond the well-conditioned parity cases (VERDICT r1 "Next round" 2, 3, 8):

  * C4 (banded-27, n = 4,194,304, monomial basis): the TSQR variants on the IDENTICAL
    ill-conditioned MPK panel vs the oracle's — Fig. 10 ordering, CholQR2 /
    reorth ||I - Q^T Q||_2 <= 1e-8 (north_star), monomial s = 15 CholQR breakdown
    and the opt-in SVQR retry (G15);
  * the per-panel diagnostics of cagmres_stats (collect_diag: kappa_2(W^T W), Fig. 12
    P:260-267; ||I - Q_p^T Q_p||_2) vs the oracle's ca_cycle(diag=...);
  * TSQR R of graded panels vs the oracle's own TSQR variants (not only Householder);
  * C3 (G3_circuit-shaped, n = 1,585,478) full-size solve parity.
"""
import numpy as np
import pytest

from oracle import cagmres_oracle as O
from synth import generators as G

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from test_gpu_parity import colmajor, dev, hist_within_envelope, rounding_envelope  # noqa: E402

EPS = np.finfo(np.float64).eps


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_yamazakiathd14_b200 import _lib
    _lib.load()
    torch.cuda.set_device(0)


def Solver(*a, **k):
    from paper_conf_ipps_yamazakiathd14_b200.solver import Solver as S
    return S(*a, **k)


@pytest.fixture(scope="module")
def c4():
    A = G.banded()                                   # C4: n = 4,194,304, 27 diagonals
    return A, A.to_scipy()


def _c4_panel(c4, s):
    A, As = c4
    q = G.rhs(A.n)
    q /= np.linalg.norm(q)
    return q, O.mpk(As, q, s)


def test_c4_mpk_monomial_matches_oracle(c4):
    A, As = c4
    q, Wo = _c4_panel(c4, 10)
    S = Solver(A, s=15, m=30, basis="monomial")
    W = S.mpk(dev(q), 10).cpu().numpy()
    for k in range(11):
        assert np.max(np.abs(W[:, k] - Wo[:, k])) <= 1e-13 * np.max(np.abs(Wo[:, k])), k


def test_c4_tsqr_variants_on_identical_panel_fig10(c4):
    """Fig. 10 on the C4 monomial s = 10 panel, GPU vs oracle on the same input:
    every variant's ||I - Q^T Q||_2 no worse than 10x the oracle's and inside its Fig. 10 bound,
    the ordering CholQR ~ SVQR >> MGS >> CholQR2 ~ CAQR on both sides, and the
    north-star bound ||I - Q^T Q|| <= 1e-8 for CholQR with reorthogonalisation."""
    A, _ = c4
    _, Wo = _c4_panel(c4, 10)
    S = Solver(A, s=15, m=30, basis="monomial")
    w = Wo.shape[1]
    ref = {"cholqr": O.orth_error(O.tsqr_cholqr(Wo)[0]),
           "svqr": O.orth_error(O.tsqr_svqr(Wo)[0]),
           "mgs": O.orth_error(O.tsqr_mgs(Wo)[0]),
           "caqr": O.orth_error(O.tsqr_caqr(Wo)[0])}
    Q1 = O.tsqr_cholqr(Wo)[0]
    ref["cholqr2"] = O.orth_error(O.tsqr_cholqr(Q1)[0])
    got = {}
    for kind, reorth, key in (("cholqr", False, "cholqr"), ("svqr", False, "svqr"), ("mgs", False, "mgs"),
                              ("caqr", False, "caqr"), ("cholqr", True, "cholqr2")):
        Pd = colmajor(Wo)
        R = S.tsqr(Pd, w, kind, reorth).cpu().numpy()
        Q = Pd.cpu().numpy()
        got[key] = O.orth_error(Q)
        assert O.fact_error(Wo, Q, R) < 1e-12, key
    kappa = np.linalg.cond(Wo)
    bound = {"cholqr": kappa ** 2, "svqr": kappa ** 2, "mgs": kappa, "caqr": 1.0, "cholqr2": 1.0}
    for k in ref:
        # never worse than 10x the oracle on the same panel, and inside the Fig. 10 bound
        # (O(eps kappa^2) CholQR / SVQR, O(eps kappa) MGS, O(eps) CAQR / CholQR2); the GPU may be
        # MORE accurate: its Gram is summed in a blocked tree (148 x 16-warp partials), the
        # BLAS product P^T P of the oracle in long running sums
        assert got[k] <= 10 * max(ref[k], 1e-14), (k, got[k], ref[k])
        assert got[k] <= 100 * EPS * bound[k], (k, got[k], kappa)
    assert got["cholqr2"] <= 1e-8 and got["caqr"] <= 1e-13
    assert got["cholqr"] > 10 * got["mgs"] and got["svqr"] > 10 * got["mgs"]
    assert got["mgs"] > 10 * got["cholqr2"]
    assert ref["cholqr"] > 10 * ref["mgs"] > 100 * ref["cholqr2"]


def test_c4_monomial_s15_cholqr_breakdown_and_svqr_retry(c4):
    """Monomial s = 15: the Gram of the C4 panel is numerically singular, CholQR returns
    EBREAKDOWN (oracle raises too); with CAGMRES_SVQR_RETRY the same panel is factored by SVQR
    on the device (G15) and matches the oracle's retry within the Fig. 10 SVQR level."""
    from paper_conf_ipps_yamazakiathd14_b200 import _lib as L
    A, _ = c4
    _, Wo = _c4_panel(c4, 15)
    with pytest.raises(O.Breakdown):
        O.tsqr_cholqr(Wo)
    S = Solver(A, s=15, m=30, basis="monomial")
    with pytest.raises(L.CagmresError) as e:
        S.tsqr(colmajor(Wo), 16, "cholqr")
    assert e.value.status == L.EBREAKDOWN
    Sr = Solver(A, s=15, m=30, basis="monomial")
    Pd = colmajor(Wo)
    R = Sr.tsqr(Pd, 16, "cholqr", svqr_retry=True)
    Qo, Ro = O.tsqr_cholqr_svqr_retry(Wo)
    Q = Pd.cpu().numpy()
    eg, eo = O.orth_error(Q), O.orth_error(Qo)
    assert eg <= 10 * eo                                    # not worse than the oracle's retry
    assert O.fact_error(Wo, Q, R.cpu().numpy()) < 1e-12


def test_c4_solve_svqr_retry_counts_panels(c4):
    """A monomial s = 15 CA cycle on C4: without the flag the solve stops with EBREAKDOWN;
    with CAGMRES_SVQR_RETRY it completes and reports the retried panels."""
    from paper_conf_ipps_yamazakiathd14_b200 import _lib as L
    A, _ = c4
    b = dev(G.rhs(A.n))
    S = Solver(A, s=15, m=30, basis="monomial")
    with pytest.raises(L.CagmresError) as e:
        S.solve(b, tol=1e-8, maxit=1)
    assert e.value.status == L.EBREAKDOWN
    Sr = Solver(A, s=15, m=30, basis="monomial", svqr_retry=True)
    _, st = Sr.solve(b, tol=1e-8, maxit=1)
    assert st.retried_panels >= 1 and st.cycles == 1
    assert st.hist[0] < 1.0


@pytest.mark.parametrize("gen,s,m,basis,tsqr,reorth,cyc", [
    ("C1", 5, 30, "newton", "cholqr", False, 4), ("C1", 5, 30, "monomial", "cholqr", True, 3),
    ("C4", 10, 30, "monomial", "cholqr", True, 1), ("C4", 10, 30, "monomial", "svqr", False, 1)])
def test_collect_diag_matches_oracle(gen, s, m, basis, tsqr, reorth, cyc, c4):
    """cagmres_stats.max_gram_cond / max_orth_err (collect_diag) vs the oracle's per-panel
    cond(W^T W) and ||I - Q_p^T Q_p||_2 (ca_cycle(diag=...)): kappa within 5 % where it is
    below 1e13 (fp64 resolves it); the orthogonality error never worse than 10x the oracle's."""
    if gen == "C1":
        A = G.convection_diffusion(32, 2, 5)
        As = A.to_scipy()
    else:
        A, As = c4
    b = G.rhs(A.n)
    sh = None
    if basis == "newton":
        sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, m)[1], m), s)
    S = Solver(A, s=s, m=m, basis=basis, tsqr=tsqr, reorth=reorth)
    if sh is not None:
        S.set_shifts(*sh)
    _, st = S.solve(dev(b), tol=0.0, maxit=cyc, diag=True)
    dg = []
    O.cagmres(As, b, s, m, basis=basis, tsqr=tsqr, reorth=reorth, tol=0.0, maxcyc=cyc, shifts=sh, diag=dg)
    kref = max(d["cond_gram"] for d in dg)
    oref = max(d["orth"] for d in dg)
    assert st.ms_setup > 0.0
    if kref < 1e13:
        assert abs(st.max_gram_cond - kref) <= 0.05 * kref, (st.max_gram_cond, kref)
    else:
        assert st.max_gram_cond > 1e12
    # not worse than 10x the oracle's (the GPU Gram is summed more accurately, see the Fig. 10
    # test); rounding-level values floored at 1e-14
    assert st.max_orth_err <= 10 * max(oref, 1e-14), (st.max_orth_err, oref)
    if oref > 1e-10:                                        # an ill-conditioned case stays one
        assert st.max_orth_err > 1e-3 * oref


@pytest.mark.parametrize("kind", ["cholqr", "svqr", "cgs", "mgs", "caqr"])
@pytest.mark.parametrize("kappa", [1e2, 1e5])
def test_tsqr_graded_panels_vs_oracle_variant(kind, kappa):
    """R of the GPU variant vs R of the SAME variant in the oracle on graded panels
    P = U diag(logspace(0, -log10 kappa)) V^T (n = 200,003, w = 11): relative kappa^2 * 1e-14
    for the Gram-based CholQR / SVQR, kappa * 1e-13 for CGS / MGS / CAQR; ||I - Q^T Q|| within
    10x of the oracle's (one-sided: the GPU CGS, with fixed-order tree reductions, measured
    20-50x MORE orthogonal than NumPy's on these panels)."""
    n, w = 200003, 11
    S = Solver(G.banded(n=n), s=1, m=2, basis="monomial")
    U, _ = np.linalg.qr(G.random_panel(n, w, 51))
    V, _ = np.linalg.qr(G.random_panel(w, w, 52))
    P = U @ np.diag(np.logspace(0, -np.log10(kappa), w)) @ V.T
    Qo, Ro = O.TSQR[kind](P)
    Pd = colmajor(P)
    R = S.tsqr(Pd, w, kind).cpu().numpy()
    Q = Pd.cpu().numpy()
    tol = kappa ** 2 * 1e-14 if kind in ("cholqr", "svqr") else kappa * 1e-13
    assert np.max(np.abs(R - Ro)) <= tol * np.abs(Ro).max(), kind
    eg, eo = O.orth_error(Q), O.orth_error(Qo)
    assert eg <= 10 * max(eo, 1e-14)                       # not worse than the oracle's variant


def test_solve_full_size_C3():
    """Config C3 (G3_circuit-shaped, n = 1,585,478, s = 5, m = 60, Newton, CholQR) at full
    size: restart cycles +-1 and per-cycle residuals vs the oracle under the DESIGN §8 rule."""
    A = G.g3_shaped()
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=5, m=60, basis="newton")
    x, st = S.solve(dev(b), tol=1e-8, maxit=120)
    ref, env = rounding_envelope(As, b, nperm=1, s=5, m=60, basis="newton", tol=1e-8, maxcyc=120)
    assert st.status == 0
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)
    r = b - As @ x.cpu().numpy()
    assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)
