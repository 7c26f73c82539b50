"""GPU parity: the CUDA path (through the C ABI) vs the oracle on identical seeded inputs.

Tolerances (DESIGN.md §8 "Parity tolerances", from BASELINE.json north_star + SURVEY §8(c)):
  MPK columns: |W_gpu - W_orc| <= 1e-13 * max|W_orc[:,k]| (FMA contraction only; measured
    <= 8e-15, profiles/r2_parity_margins.json)
  R, C (well conditioned): relative 1e-10
  per-cycle rho: |rho_gpu - rho_orc| <= max(1e-10, 10 env_c) rho_orc + 1e-15 (units of ||r0||),
    env_c = the oracle's own deviation under symmetric permutations (its rounding noise);
    measured GPU deviation <= 3.1 env_c over six configs (profiles/r2_parity_margins.json)
  restart cycles to 1e-8: +-1
"""
import numpy as np
import pytest

from oracle import cagmres_oracle as O
from synth import generators as G

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


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


def dev(x):
    return torch.tensor(np.ascontiguousarray(x), dtype=torch.float64, device="cuda")


def colmajor(M):
    """device column-major copy of a 2-D numpy array (stride(0) == 1)."""
    return dev(np.asarray(M).T).t()


def hist_close(h, ref, rtol=1e-10, atol=1e-15):
    k = min(len(h), len(ref))
    return np.all(np.abs(h[:k] - ref[:k]) <= rtol * ref[:k] + atol)


def rounding_envelope(As, b, nperm=2, **kw):
    """The oracle's own sensitivity to summation order: rerun it on symmetric permutations
    P A P^T, P b (identical in exact arithmetic, different rounding) and return
    (reference history, running max of the relative deviation per cycle).
    SVQR additionally: its R is the Cholesky factor of the Gram in exact arithmetic,
    computed through a symmetric eigendecomposition whose algorithm differs between the sides
    (LAPACK dsyevd vs the device's Jacobi sweeps); the oracle's own SVQR-vs-CholQR difference
    measures that algorithm noise and joins the envelope."""
    ref = O.cagmres(As, b, **kw)["hist"]
    dev_ = np.zeros(len(ref))
    alts = [dict(kw, tsqr="cholqr")] if kw.get("tsqr") == "svqr" else []
    for s in range(nperm):
        p = np.argsort(G.u(1000 + s, np.arange(As.shape[0])))
        hp = O.cagmres(As[p][:, p], b[p], **kw)["hist"]
        k = min(len(hp), len(ref))
        dev_[:k] = np.maximum(dev_[:k], np.abs(hp[:k] - ref[:k]) / ref[:k])
    for kw2 in alts:
        hp = O.cagmres(As, b, **kw2)["hist"]
        k = min(len(hp), len(ref))
        dev_[:k] = np.maximum(dev_[:k], np.abs(hp[:k] - ref[:k]) / ref[:k])
    return ref, np.maximum.accumulate(dev_)


def hist_within_envelope(h, ref, env, factor=10.0):
    """|rho_gpu - rho_orc| <= max(1e-10, factor * env_c) * rho_orc + 1e-15 per cycle: the
    north-star relative 1e-10 where the problem is well conditioned, else a multiple of the
    oracle's own rounding noise."""
    k = min(len(h), len(ref))
    tol = np.maximum(1e-10, factor * env[:k]) * ref[:k] + 1e-15
    return np.all(np.abs(h[:k] - ref[:k]) <= tol)


SHIFTS = (np.array([7.9, 7.9, 0.09, 0.09, 3.8, 5.5, 1.2, 6.6, 2.5, 4.4]),
          np.array([0.02, -0.02, 0.03, -0.03, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0]))


# ----------------------------------------------------------------------------- MPK
@pytest.mark.parametrize("basis", ["monomial", "newton"])
@pytest.mark.parametrize("gen", ["C1", "cd27_ragged", "g3_small", "banded_1row_tail", "cd7_ragged"])
def test_mpk_parity(basis, gen):
    """Last-slice cases: banded n = 300001 leaves ONE valid row in a DIA slice of 14 diagonals
    (lanes 1..13 must still load their offsets), 2025 = 63*32 + 9 rows for the 5-pt stencil."""
    A = {"C1": lambda: G.convection_diffusion(32, 2, 5),
         "cd27_ragged": lambda: G.convection_diffusion(13, 3, 27),       # n = 2197, ragged tail
         "g3_small": lambda: G.g3_shaped(n=50001, width=250),
         "banded_1row_tail": lambda: G.banded(n=300001),
         "cd7_ragged": lambda: G.convection_diffusion(45, 2, 5)}[gen]()
    As = A.to_scipy()
    s = 6
    S = Solver(A, s=s, m=12, basis=basis)
    re, im = (None, None)
    if basis == "newton":
        re, im = SHIFTS[0][:s], SHIFTS[1][:s]
        S.set_shifts(re, im)
    q = G.u(11, np.arange(A.n))
    for sb in (1, 3, s):
        W = S.mpk(dev(q), sb).cpu().numpy()
        Wo = O.mpk(As, q, sb, re, im)
        for k in range(sb + 1):
            assert np.max(np.abs(W[:, k] - Wo[:, k])) <= 1e-13 * np.max(np.abs(Wo[:, k])), (sb, k)


def test_mpk_newton_zero_shifts_bitwise_equals_monomial():
    A = G.convection_diffusion(20, 3, 7)
    q = dev(G.u(3, np.arange(A.n)))
    S1 = Solver(A, s=5, m=10, basis="monomial")
    S2 = Solver(A, s=5, m=10, basis="newton")
    S2.set_shifts(np.zeros(5))
    assert torch.equal(S1.mpk(q, 5), S2.mpk(q, 5))


@pytest.mark.parametrize("gen", ["C2", "cd27_40", "banded"])
def test_mpk_wave_bitwise_equals_stepwise(gen):
    """Temporally blocked single-GPU MPK (NEXT-3) computes every row exactly as the
    one-launch-per-step MPK: the results must be bitwise identical."""
    A = {"C2": lambda: G.convection_diffusion(128, 3, 7),
         "cd27_40": lambda: G.convection_diffusion(40, 3, 27),
         "banded": lambda: G.banded(n=300001)}[gen]()
    q = dev(G.u(5, np.arange(A.n)))
    S1 = Solver(A, s=10, m=30, basis="newton")
    S2 = Solver(A, s=10, m=30, basis="newton")
    S1.set_option("mpk_wave", 2)                   # forced on (off by default)
    S2.set_option("mpk_wave", 0)
    for S in (S1, S2):
        S.set_shifts(*SHIFTS)
    for sb in (10, 4, 2):
        W1, W2 = S1.mpk(q, sb), S2.mpk(q, sb)
        assert torch.equal(W1, W2), (gen, sb)
    if gen == "cd27_40":                          # and directly against the oracle (Fig. 4)
        Wo = O.mpk(A.to_scipy(), q.cpu().numpy(), 10, *SHIFTS)
        W1 = S1.mpk(q, 10).cpu().numpy()
        for k in range(11):
            assert np.max(np.abs(W1[:, k] - Wo[:, k])) <= 1e-13 * np.max(np.abs(Wo[:, k])), k


@pytest.mark.parametrize("gen", ["C2", "cd27_ragged", "g3_small", "banded", "cd7_ragged"])
def test_mpk_sweep_bitwise_equals_stepwise(gen):
    """CAGMRES_OPT_MPK_WAVE = 3: the whole MPK block in one persistent launch (grid barriers
    between the steps, alternating sweep direction) computes every row as the stepwise MPK —
    bitwise identical bases for every block size, including complex-conjugate pairs (SHIFTS
    has two) and a block ending inside a pair; then whole solves, bit for bit, and directly
    against the oracle's MPK."""
    A = {"C2": lambda: G.convection_diffusion(128, 3, 7),
         "cd27_ragged": lambda: G.convection_diffusion(17, 3, 27),
         "g3_small": lambda: G.g3_shaped(n=40000, width=200),
         "banded": lambda: G.banded(n=300001),
         "cd7_ragged": lambda: G.convection_diffusion(45, 3, 7)}[gen]()
    q = dev(G.u(5, np.arange(A.n)))
    S1 = Solver(A, s=10, m=30, basis="newton")
    S2 = Solver(A, s=10, m=30, basis="newton")
    S1.set_option("mpk_wave", 3)
    assert S1.get_option("mpk_wave") == 3
    S2.set_option("mpk_wave", 0)
    for S in (S1, S2):
        S.set_option("spmv", 16)
        S.set_shifts(*SHIFTS)
    for sb in (10, 7, 4, 2, 1):
        W1, W2 = S1.mpk(q, sb), S2.mpk(q, sb)
        assert torch.equal(W1, W2), (gen, sb)
    if gen in ("cd27_ragged", "g3_small"):
        Wo = O.mpk(A.to_scipy(), q.cpu().numpy(), 10, *SHIFTS)
        W1 = S1.mpk(q, 10).cpu().numpy()
        for k in range(11):
            assert np.max(np.abs(W1[:, k] - Wo[:, k])) <= 1e-13 * np.max(np.abs(Wo[:, k])), k
    if gen in ("cd7_ragged", "g3_small"):
        b = dev(G.rhs(A.n))
        m = 60 if gen == "g3_small" else 30
        out = []
        for wave in (3, 0):
            S = Solver(A, s=5, m=m, basis="newton")
            S.set_option("spmv", 16)
            S.set_option("mpk_wave", wave)
            x, st = S.solve(b, tol=1e-8, maxit=100)
            assert st.status == 0
            out.append((x, st))
        assert np.array_equal(out[0][1].hist, out[1][1].hist) and torch.equal(out[0][0], out[1][0])


@pytest.mark.parametrize("gen", ["cd27_ragged", "g3_small", "banded", "cd7_ragged"])
def test_spmv_variants_bitwise(gen):
    """Every SpMV kernel variant (CAGMRES_OPT_SPMV: one or two SELL-32 slices per warp, load
    batches 4/8, persistent with pipelined slice descriptors) sums each row in the same order: the MPK bases are bitwise identical; the
    parity of variant 0 against the oracle is test_mpk_parity."""
    A = {"cd27_ragged": lambda: G.convection_diffusion(17, 3, 27),
         "g3_small": lambda: G.g3_shaped(n=40000, width=200),
         "banded": lambda: G.banded(n=300001),
         "cd7_ragged": lambda: G.convection_diffusion(45, 3, 7)}[gen]()
    q = dev(G.u(6, np.arange(A.n)))
    S = Solver(A, s=6, m=30, basis="newton")
    S.set_shifts(*SHIFTS)
    Ws = []
    variants = [0, 5, 16, 17]
    for v in variants:
        S.set_option("spmv", v)
        Ws.append(S.mpk(q, 6))
    for i, v in enumerate(variants[1:], 1):
        assert torch.equal(Ws[i], Ws[0]), v


@pytest.mark.parametrize("gen", ["cd7_ragged", "g3_small"])
def test_serpentine_order(gen):
    """CAGMRES_OPT_SERP: every streaming kernel sweeps the rows opposite to its
    predecessor (band order, kern::band_tile).  Row-wise kernels are unchanged: the MPK basis is
    bitwise that of the all-forward order for every SpMV variant.  The reductions (Gram, xTy,
    norms) sum the same products in another fixed order: R and Q agree to rounding, and the
    solve matches the oracle under the §8 rule either way (and reproduces itself bit for bit)."""
    A = {"g3_small": lambda: G.g3_shaped(n=40000, width=200),
         "cd7_ragged": lambda: G.convection_diffusion(45, 3, 7)}[gen]()
    As = A.to_scipy()
    q = dev(G.u(6, np.arange(A.n)))
    W = {}
    for serp in (0, 1):
        for v in (16, 0):
            S = Solver(A, s=6, m=30, basis="newton")
            S.set_option("serp", serp)
            assert S.get_option("serp") == serp
            S.set_option("spmv", v)
            S.set_shifts(*SHIFTS)
            W[serp, v] = S.mpk(q, 6)
    for key in W:
        assert torch.equal(W[key], W[0, 16]), key
    P = G.random_panel(A.n, 11, 31)
    QR = {}
    for serp in (0, 1):
        S = Solver(A, s=6, m=30, basis="newton")
        S.set_option("serp", serp)
        Q = colmajor(P)
        R = S.tsqr(Q, 11, "cholqr")
        QR[serp] = (Q.cpu().numpy(), R.cpu().numpy())
    (Q0, R0), (Q1, R1) = QR[0], QR[1]
    assert np.max(np.abs(R1 - R0)) <= 1e-13 * np.max(np.abs(R0))
    assert np.max(np.abs(Q1 - Q0)) <= 1e-13 * np.max(np.abs(Q0))
    assert O.fact_error(P, Q1, R1) < 1e-13 and O.orth_error(Q1) < 1e-12
    b = G.rhs(A.n)
    m = 60 if gen == "g3_small" else 30
    sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, m)[1], m), 5)
    ref, env = rounding_envelope(As, b, nperm=1, s=5, m=m, basis="newton", tol=1e-8, maxcyc=100, shifts=sh)
    hist = {}
    for serp in (0, 1, 1):
        S = Solver(A, s=5, m=m, basis="newton")
        S.set_option("serp", serp)
        S.set_shifts(*sh)
        x, st = S.solve(dev(b), tol=1e-8, maxit=100)
        assert st.status == 0 and abs(st.cycles - len(ref)) <= 1
        assert hist_within_envelope(st.hist, ref, env)
        if serp in hist:
            assert np.array_equal(hist[serp][0], st.hist) and torch.equal(hist[serp][1], x)
        hist[serp] = (st.hist, x)


def test_mpk_full_size_C2():
    """Config C2 at full size (n = 2,097,152) in the launch configuration bench.py times."""
    A = G.convection_diffusion(128, 3, 7)
    As = A.to_scipy()
    S = Solver(A, s=10, m=30, basis="newton")
    S.set_shifts(*SHIFTS)
    q = G.rhs(A.n)
    q /= np.linalg.norm(q)
    W = S.mpk(dev(q), 10).cpu().numpy()
    Wo = O.mpk(As, q, 10, *SHIFTS)
    for k in range(11):
        assert np.max(np.abs(W[:, k] - Wo[:, k])) <= 1e-13 * np.max(np.abs(Wo[:, k]))


def test_mpk_full_size_C5_sampled():
    """Config C5 at full size (400^3 27-pt, n = 64M, 1.72e9 nnz), the launch configuration
    bench.py times, checked on sampled z-planes.  Step k at a row depends only on rows within k
    hops, so the oracle runs on the principal sub-block of the planes within s = 10
    of the sample: its values on the sample plane are exact for every k <= 10."""
    N, s = 400, 10
    P = N * N
    A = G.convection_diffusion_stream(N, 3, 27)
    S = Solver(A, s=s, m=30, basis="newton")
    del A
    S.set_shifts(*SHIFTS)
    q = G.rhs(N ** 3)
    q /= np.linalg.norm(q)
    W = S.mpk(dev(q), s)
    for z0 in (0, 217, N - 1):                                  # both boundary planes and one inside
        lo, hi = max(0, z0 - s) * P, min(N, z0 + s + 1) * P
        sub = G.convection_diffusion_stream(N, 3, 27, rows=(lo, hi)).to_scipy()[:, lo:hi]
        Wo = O.mpk(sub.tocsr(), q[lo:hi], s, *SHIFTS)
        a, b = z0 * P - lo, (z0 + 1) * P - lo
        Wg = W[z0 * P:(z0 + 1) * P].cpu().numpy()
        for k in range(s + 1):
            ref = Wo[a:b, k]
            assert np.max(np.abs(Wg[:, k] - ref)) <= 1e-13 * np.max(np.abs(ref)), (z0, k)


# ----------------------------------------------------------------------------- BOrth / TSQR
@pytest.mark.parametrize("n,j,w", [(5000, 12, 6), (70002, 55, 5), (3000, 1, 1), (40000, 30, 11),
                                   (1000, 70, 3), (70001, 7, 4), (262144, 20, 10)])
def test_borth_parity(n, j, w):
    A = G.banded(n=n)                                            # any matrix with n rows
    S = Solver(A, s=1, m=max(j, 1), basis="monomial")
    Q, _ = np.linalg.qr(G.random_panel(n, j, 21))
    P = G.random_panel(n, w, 22)
    Qd, Pd = colmajor(Q), colmajor(P)
    C = S.borth(Qd, j, Pd, w).cpu().numpy()
    Co, Po = O.borth_cgs(Q, P)
    assert np.allclose(C, Co, rtol=1e-10, atol=1e-12)
    assert np.allclose(Pd.cpu().numpy(), Po, rtol=1e-10, atol=1e-12)


@pytest.mark.parametrize("kind,reorth", [("cholqr", False), ("cholqr", True), ("svqr", False),
                                         ("cgs", False), ("mgs", False), ("caqr", False)])
@pytest.mark.parametrize("n,w", [(100002, 11), (100003, 11), (777, 6), (4096, 1), (20000, 16), (65538, 13)])
@pytest.mark.parametrize("gram", [0, 1, 2])
def test_tsqr_parity(kind, reorth, n, w, gram):
    """gram: CAGMRES_OPT_GRAM (0 = DMMA tensor-core Gram, 1 = scalar DFMA ring Gram)."""
    A = G.banded(n=n)
    S = Solver(A, s=1, m=2, basis="monomial")
    S.set_option("gram", gram)
    P = G.random_panel(n, w, 31)
    if w > 2:
        P[:, 2] += 0.3 * P[:, 1]
    Pd = colmajor(P)
    R = S.tsqr(Pd, w, kind, reorth).cpu().numpy()
    Q = Pd.cpu().numpy()
    _, Rr = np.linalg.qr(P)
    Rr = np.sign(np.diag(Rr))[:, None] * Rr
    assert np.allclose(R, Rr, rtol=1e-10, atol=1e-10 * np.abs(Rr).max())
    assert O.orth_error(Q) < 1e-12
    assert O.fact_error(P, Q, R) < 1e-13


def test_caqr_is_unconditionally_orthogonal():
    """Fig. 10: CAQR ||I - Q^T Q|| = O(eps) even where CholQR breaks down."""
    n, w = 60000, 12
    S = Solver(G.banded(n=n), s=1, m=2, basis="monomial")
    U, _ = np.linalg.qr(G.random_panel(n, w, 41))
    Vv, _ = np.linalg.qr(G.random_panel(w, w, 42))
    P = U @ np.diag(np.logspace(0, -9, w)) @ Vv.T                # kappa = 1e9
    Pd = colmajor(P)
    R = S.tsqr(Pd, w, "caqr").cpu().numpy()
    Q = Pd.cpu().numpy()
    assert O.orth_error(Q) < 1e-13
    assert O.fact_error(P, Q, R) < 1e-14
    assert np.all(np.diag(R) > 0)


def test_tsqr_cholqr_breakdown_reported():
    from paper_conf_ipps_yamazakiathd14_b200 import _lib as L
    n = 5000
    S = Solver(G.banded(n=n), s=1, m=2, basis="monomial")
    P = G.random_panel(n, 4, 5)
    P[:, 3] = 0.0                                  # pivot exactly 0 (a rounding-free breakdown)
    with pytest.raises(L.CagmresError) as e:
        S.tsqr(colmajor(P), 4, "cholqr")
    assert e.value.status == L.EBREAKDOWN


# ----------------------------------------------------------------------------- solve
@pytest.mark.parametrize("basis,tsqr,reorth,borth", [
    ("newton", "cholqr", False, "cgs"), ("monomial", "cholqr", False, "cgs"),
    ("newton", "cholqr", True, "cgs"), ("newton", "svqr", False, "cgs"),
    ("newton", "cgs", True, "cgs"), ("newton", "mgs", False, "mgs"), ("newton", "caqr", False, "cgs")])
def test_solve_C1_injected_shifts(basis, tsqr, reorth, borth):
    A = G.convection_diffusion(32, 2, 5)
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=5, m=30, basis=basis, tsqr=tsqr, reorth=reorth, borth=borth)
    sh = None
    if basis == "newton":
        sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, 30)[1], 30), 5)
        S.set_shifts(*sh)
    x, st = S.solve(dev(b), tol=1e-8, maxit=40)
    ref, env = rounding_envelope(As, b, s=5, m=30, basis=basis, tsqr=tsqr, reorth=reorth,
                                 borth=borth, tol=1e-8, shifts=sh)
    assert st.status == 0
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)
    xs = np.linalg.solve(As.toarray(), b)
    assert np.linalg.norm(x.cpu().numpy() - xs) <= 1e-6 * np.linalg.norm(xs)


def test_solve_C1_newton_first_cycle_gmres():
    """Newton without preset shifts: cycle 1 is GMRES(m) on the GPU, its Ritz values (host
    Francis QR) in Leja order become the shifts."""
    A = G.convection_diffusion(32, 2, 5)
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=5, m=30, basis="newton")
    x, st = S.solve(dev(b), tol=1e-8, maxit=40)
    ref = O.cagmres(As, b, 5, 30, basis="newton", tol=1e-8)
    re, im = S.get_shifts()
    assert np.allclose(re[:5], ref["shifts"][0][:5], rtol=1e-8)
    assert np.allclose(im[:5], ref["shifts"][1][:5], rtol=1e-8, atol=1e-12)
    assert abs(st.cycles - ref["cycles"]) <= 1
    _, env = rounding_envelope(As, b, s=5, m=30, basis="newton", tol=1e-8)
    assert hist_within_envelope(st.hist, ref["hist"], env)
    g = O.gmres(As, b, 30, tol=1e-8)
    assert abs(st.cycles - g["cycles"]) <= 1
    assert np.all(np.diff(st.hist) <= 0)


def test_solve_partial_last_block_and_ragged_n():
    """(s, m) = (7, 30) -> blocks 7,7,7,7,2 (P:273 'generates 20 and then 10'); n = 2197."""
    A = G.convection_diffusion(13, 3, 27)
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=7, m=30, basis="monomial", reorth=True)
    x, st = S.solve(dev(b), tol=1e-10, maxit=20)
    ref, env = rounding_envelope(As, b, s=7, m=30, basis="monomial", reorth=True, tol=1e-10)
    assert abs(st.cycles - len(ref)) <= 1 and hist_within_envelope(st.hist, ref, env)


def test_solve_g3_shaped_small():
    A = G.g3_shaped(n=40000, width=200)
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=5, m=60, basis="newton")
    x, st = S.solve(dev(b), tol=1e-8, maxit=200)
    ref, env = rounding_envelope(As, b, nperm=1, s=5, m=60, basis="newton", tol=1e-8, maxcyc=200)
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)


def test_solve_full_size_C2():
    """Config C2 (bench workload) at full size: per-cycle residuals vs the oracle."""
    A = G.convection_diffusion(128, 3, 7)
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=10, m=30, basis="newton")
    x, st = S.solve(dev(b), tol=1e-8, maxit=60)
    ref, env = rounding_envelope(As, b, nperm=1, s=10, m=30, basis="newton", tol=1e-8, maxcyc=60)
    assert st.status == 0
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)
    r = b - As @ x.cpu().numpy()
    assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)


@pytest.mark.parametrize("fuse", [0, 1])
@pytest.mark.parametrize("s,m,reorth", [(5, 30, False), (15, 60, True), (10, 80, False)])
def test_solve_fused_borth_gram(fuse, s, m, reorth):
    """BOrth pass 2 fused with the CholQR Gram (fused.cu; j up to 60 -> 16 k-tiles, w+1 = 16)
    against the unfused path, both vs the oracle; m = 80 exceeds the fused kernel's j <= 64
    and falls back to the separate update + Gram inside a cycle.  n = 2500 (ragged tail)."""
    A = G.convection_diffusion(50, 2, 5)
    As = A.to_scipy()
    b = G.rhs(A.n)
    sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, m)[1], m), s)
    S = Solver(A, s=s, m=m, basis="newton", reorth=reorth)
    S.set_option("fuse", fuse | 2)
    S.set_shifts(*sh)
    x, st = S.solve(dev(b), tol=1e-8, maxit=40)
    ref, env = rounding_envelope(As, b, s=s, m=m, basis="newton", reorth=reorth, tol=1e-8, shifts=sh)
    assert st.status == 0
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)


@pytest.mark.parametrize("spmv,gram", [(16, 1), (5, 0), (0, 1)])
def test_solve_kernel_options(spmv, gram):
    """Solve with the persistent SpMVs (CAGMRES_OPT_SPMV 16 / 5) and the scalar-DFMA Gram
    (CAGMRES_OPT_GRAM 1) against the oracle: 3D 7-point 40^3 (n = 64,000), s = 10, m = 30."""
    A = G.convection_diffusion(40, 3, 7)
    As = A.to_scipy()
    b = G.rhs(A.n)
    sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, 30)[1], 30), 10)
    S = Solver(A, s=10, m=30, basis="newton")
    S.set_option("spmv", spmv)
    S.set_option("gram", gram)
    S.set_shifts(*sh)
    x, st = S.solve(dev(b), tol=1e-8, maxit=40)
    ref, env = rounding_envelope(As, b, s=10, m=30, basis="newton", tol=1e-8, shifts=sh)
    assert st.status == 0
    assert abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)
    r = b - As @ x.cpu().numpy()
    assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)


# ----------------------------------------------------------------------------- GMRES baseline
@pytest.mark.parametrize("reorth,arnoldi", [(False, 1), (True, 1), (False, 0)])
@pytest.mark.parametrize("gen", ["C1", "g3_small"])
def test_solve_gmres_baseline(gen, reorth, arnoldi):
    """basis="gmres": the standard GMRES(m) comparator of Fig. 14/15 on the GPU —
    SpMV + CGS (CGS2 with reorth) per iteration.  Restarted GMRES's per-cycle residuals are
    fixed by the Krylov space, so they must match the oracle's MGS GMRES(m) [3] to rounding
    (its own sensitivity to summation order measured by symmetric permutations)."""
    if gen == "C1":
        A, m = G.convection_diffusion(32, 2, 5), 30
    else:
        A, m = G.g3_shaped(n=40000, width=200), 60
    As = A.to_scipy()
    b = G.rhs(A.n)
    S = Solver(A, s=1, m=m, basis="gmres", reorth=reorth)
    S.set_option("arnoldi", arnoldi)          # 1: cp.async ring Arnoldi passes (n >= 2048), 0: register kernel
    x, st = S.solve(dev(b), tol=1e-8, maxit=200)
    ref = O.gmres(As, b, m, tol=1e-8, maxcyc=200)["hist"]
    env = np.zeros(len(ref))
    p = np.argsort(G.u(1000, np.arange(A.n)))
    hp = O.gmres(As[p][:, p], b[p], m, tol=1e-8, maxcyc=200)["hist"]
    k = min(len(hp), len(ref))
    env[:k] = np.abs(hp[:k] - ref[:k]) / ref[:k]
    env = np.maximum.accumulate(env)
    assert st.status == 0 and abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env, factor=100.0)
    assert np.all(np.diff(st.hist) <= 1e-14)                      # restarted GMRES is monotone
    r = b - As @ x.cpu().numpy()
    assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)


# ----------------------------------------------------------------------------- one-pass BOrth+CholQR
@pytest.mark.parametrize("s,m,reorth,gen", [(5, 30, False, "C1"), (5, 30, True, "C1"), (10, 30, True, "cd7"),
                                             (5, 60, False, "g3_small"), (7, 30, True, "cd27_ragged")])
def test_solve_onepass(s, m, reorth, gen):
    """CAGMRES_ONEPASS (NEXT-2): per-cycle residuals vs oracle cagmres(onepass=True) with the same
    injected shifts; rounding envelope of the oracle as in the other solve tests."""
    A = {"C1": lambda: G.convection_diffusion(32, 2, 5),
         "cd7": lambda: G.convection_diffusion(40, 3, 7),
         "g3_small": lambda: G.g3_shaped(n=40000, width=200),
         "cd27_ragged": lambda: G.convection_diffusion(13, 3, 27)}[gen]()
    As = A.to_scipy()
    b = G.rhs(A.n)
    re, im = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, m)[1], m), s)
    S = Solver(A, s=s, m=m, basis="newton", reorth=reorth, onepass=True)
    S.set_shifts(re, im)
    x, st = S.solve(dev(b), tol=1e-8, maxit=200)
    ref, env = rounding_envelope(As, b, nperm=1, s=s, m=m, basis="newton", reorth=reorth, tol=1e-8,
                                 maxcyc=200, shifts=(re, im), onepass=True)
    assert st.status == 0 and abs(st.cycles - len(ref)) <= 1
    assert hist_within_envelope(st.hist, ref, env)
    r = b - As @ x.cpu().numpy()
    assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)


@pytest.mark.parametrize("kw", [dict(), dict(reorth=True), dict(onepass=True), dict(onepass=True, reorth=True),
                                dict(tsqr="svqr"), dict(basis="monomial")])
def test_fold_last_panel_update_into_solution_update(kw):
    """CAGMRES_OPT_FOLD: the last block's final panel update is not formed and x += V y uses
    the panel P with coefficients R^{-1}[0; y] (and -C R^{-1}[0; y] for one-pass).  Equal in exact
    arithmetic: both settings must match the oracle (same rule as every solve test) and each
    other to rounding; the folded cycle launches one panel kernel less."""
    A = G.convection_diffusion(40, 3, 7)
    As = A.to_scipy()
    b = G.rhs(A.n)
    kw = dict(kw)
    basis = kw.pop("basis", "newton")
    sv = 10 if basis == "newton" else 5
    sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, 30)[1], 30), sv) if basis == "newton" else None
    ref, env = rounding_envelope(As, b, nperm=1, s=sv, m=30, basis=basis, tol=1e-8, maxcyc=60, shifts=sh,
                                 reorth=kw.get("reorth", False), onepass=kw.get("onepass", False),
                                 tsqr=kw.get("tsqr", "cholqr"))
    out = {}
    for fold in (0, 1):
        S = Solver(A, s=sv, m=30, basis=basis, **kw)
        S.set_option("fold", fold)
        assert S.get_option("fold") == fold
        if sh is not None:
            S.set_shifts(*sh)
        x, st = S.solve(dev(b), tol=1e-8, maxit=60)
        assert st.status == 0 and abs(st.cycles - len(ref)) <= 1
        assert hist_within_envelope(st.hist, ref, env)
        r = b - As @ x.cpu().numpy()
        assert np.linalg.norm(r) <= 1.01e-8 * np.linalg.norm(b)
        out[fold] = (x.cpu().numpy(), st)
    (x0, s0), (x1, s1) = out[0], out[1]
    assert s0.cycles == s1.cycles
    assert np.allclose(s0.hist, s1.hist, rtol=1e-6, atol=1e-15)
    assert np.linalg.norm(x0 - x1) <= 1e-9 * np.linalg.norm(x0)


def test_onepass_cycle_basis_matches_two_pass():
    """One cycle, same shifts: the one-pass basis spans the same space as the two-pass one —
    residual histories agree to rounding (Pythagoras exact when Q^T Q = I)."""
    A = G.convection_diffusion(64, 3, 7)
    b = G.rhs(A.n)
    out = []
    for op in (False, True):
        S = Solver(A, s=10, m=30, basis="newton", reorth=True, onepass=op)
        S.set_shifts(*SHIFTS)
        _, st = S.solve(dev(b), tol=0.0, maxit=3)
        out.append(st.hist)
    assert np.allclose(out[0], out[1], rtol=1e-8)


@pytest.mark.parametrize("gen,basis", [("C1", "newton"), ("cd7_40", "newton"), ("cd7_40", "gmres"),
                                       ("cd27_ragged", "monomial")])
def test_fused_normalisation_is_bitwise_the_separate_scaling(gen, basis):
    """CAGMRES_OPT_FUSE bit 2: q = w / ||w|| formed inside the consuming SpMV (restart vector and
    Arnoldi vectors) gives bit-for-bit the histories and solution of the separate scaling pass."""
    A = {"C1": lambda: G.convection_diffusion(32, 2, 5), "cd7_40": lambda: G.convection_diffusion(40, 3, 7),
         "cd27_ragged": lambda: G.convection_diffusion(13, 3, 27)}[gen]()
    b = dev(G.rhs(A.n))
    out = []
    for fuse in (6, 2):
        for spmv in (16, 17, 5, 0):                  # 16 / 17 fuse; 0 / 5 form q separately
            S = Solver(A, s=5 if basis != "gmres" else 1, m=30, basis=basis)
            S.set_option("fuse", fuse)
            S.set_option("spmv", spmv)
            assert S.get_option("fuse") == fuse
            x, st = S.solve(b, tol=1e-10, maxit=60)
            out.append((x, st))
    for x, st in out[1:]:
        assert np.array_equal(out[0][1].hist, st.hist) and torch.equal(out[0][0], x)


@pytest.mark.parametrize("gen,kw", [("cd7_40", dict(basis="newton")), ("C1", dict(basis="monomial", reorth=True)),
                                    ("cd7_40", dict(basis="newton", onepass=True)),
                                    ("g3_small", dict(basis="newton", tsqr="svqr"))])
def test_cuda_graph_cycles_are_bitwise_the_stream_launches(gen, kw):
    """CAGMRES_OPT_GRAPH: every CA cycle replayed from one captured CUDA graph gives the bits of
    the stream-launched cycles; re-capture after new shifts (second solve with cleared shifts)
    and after an option change; also with the separate normalisation (different entry state)."""
    A = {"C1": lambda: G.convection_diffusion(32, 2, 5), "cd7_40": lambda: G.convection_diffusion(40, 3, 7),
         "g3_small": lambda: G.g3_shaped(n=40000, width=200)}[gen]()
    b = dev(G.rhs(A.n))
    out = {}
    for graph in (1, 0):
        S = Solver(A, s=5, m=30 if gen != "g3_small" else 60, **kw)
        S.set_option("graph", graph)
        res = []
        for fuse in (6, 2):
            S.set_option("fuse", fuse)
            S.clear_shifts()
            x, st = S.solve(b, tol=1e-10, maxit=80)
            res.append((x.clone(), st))
        assert S.get_option("graph") == graph            # (negative: the capture failed)
        out[graph] = res
    for (xa, sa), (xb, sb) in zip(out[1], out[0]):
        assert sa.status == 0 and sa.cycles == sb.cycles
        assert np.array_equal(sa.hist, sb.hist) and torch.equal(xa, xb)
        assert sa.spmv_launches == sb.spmv_launches


def test_clear_shifts_reruns_first_cycle_bitwise():
    """set_shifts(count = 0): the next Newton solve runs its own GMRES shift cycle again
    and, the reductions being deterministic, reproduces the first solve bit for bit."""
    A = G.convection_diffusion(40, 3, 7)
    b = dev(G.rhs(A.n))
    S = Solver(A, s=10, m=30, basis="newton")
    x1, st1 = S.solve(b, tol=1e-8, maxit=60)
    sh1 = S.get_shifts()
    x2, st2 = S.solve(b, tol=1e-8, maxit=60)            # reuses the shifts: no GMRES cycle
    S.clear_shifts()
    x3, st3 = S.solve(b, tol=1e-8, maxit=60)
    assert np.array_equal(st3.hist, st1.hist) and torch.equal(x3, x1)
    assert np.array_equal(S.get_shifts()[0], sh1[0])
    assert st2.cycles >= 1


def test_distributed_handle_single_rank_nccl_matches_single_gpu():
    """cagmres_create_dist through a real NCCL communicator (one rank; this box has one GPU):
    unique-id broadcast, plan, request exchange over NCCL, then a full Newton solve — bitwise
    equal to the single-GPU handle (the multi-rank host logic is covered by test_dist_gloo)."""
    import os
    import torch.distributed as dist
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29533")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        A = G.convection_diffusion(40, 3, 7)
        b = dev(G.rhs(A.n))
        S1 = Solver(A, s=5, m=30, basis="newton")
        x1, st1 = S1.solve(b, tol=1e-8, maxit=60)
        S2 = Solver(A, s=5, m=30, basis="newton", group=dist.group.WORLD,
                    row_starts=np.array([0, A.n], dtype=np.int64))
        x2, st2 = S2.solve(b, tol=1e-8, maxit=60)
        assert st2.status == 0 and st2.cycles == st1.cycles
        assert np.array_equal(st2.hist, st1.hist) and torch.equal(x2, x1)
    finally:
        dist.destroy_process_group()
