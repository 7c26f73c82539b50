"""ORACLE for CA-GMRES(s, m) — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementation (NumPy/SciPy, IEEE fp64) of what the
B200 hot path computes.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import it.  It shares no code with the CUDA
library (paper_conf_ipps_yamazakiathd14_b200/) and never imports it.

Citations: "P:n" = /root/reference/PAPER.md line n.  Readings of garbled / silent passages
("G#") are SURVEY.md §8(c) readings, restated in DESIGN.md "Readings".

Pinning (tests/test_oracle_pins.py): every function below is pinned by something other
than itself — dense direct solve, dense matrix powers, numpy Householder QR, brute-force
Krylov least squares, Arnoldi relation, brute-force BFS.  Exception noted inline:
  * modified_leja: pinned by the brute-force greedy-product check on <= 8 points, the
    conjugate-adjacency invariant and hand-derived tie cases of the G10 reading (equal moduli,
    equal log-distance sums, repeated values); GPU solve parity tests still inject shifts
    where near-ties of computed Ritz values could reorder them (G19).
  * ritz_values: pinned with the CGS Arnoldi by recovering a known spectrum from a full Krylov
    space (m = n).
"""
from __future__ import annotations

import numpy as np
import scipy.linalg as sla
import scipy.sparse as sp

EPS = np.finfo(np.float64).eps


class Breakdown(RuntimeError):
    """Cholesky pivot <= 0 / zero norm (G15: no silent fallback)."""


# ---------------------------------------------------------------------------------------
# Shifts and change of basis (complex pairs in real arithmetic per [4] §7.3.2, G10)
# ---------------------------------------------------------------------------------------
def block_shifts(re, im, sb):
    """Shifts used by a block of sb MPK steps: the first sb of the Leja-ordered list.
    If position sb-1 holds the first half of a conjugate pair (im > 0), its real part is
    used instead (G10).  Returns a list of (a, b2, kind) per step: kind 'r' = real shift a,
    'p1' = first step of a pair (A - aI), 'p2' = second step ((A - aI)v + b^2 v_prev)."""
    re = np.asarray(re, dtype=np.float64)
    im = np.asarray(im, dtype=np.float64)
    steps = []
    k = 0
    while k < sb:
        a, b = float(re[k]), float(im[k])
        if b > 0.0 and k + 1 < sb:
            steps.append((a, 0.0, "p1"))
            steps.append((a, b * b, "p2"))
            k += 2
        else:
            steps.append((a, 0.0, "r"))   # real shift, or truncated pair -> real part
            k += 1
    return steps


def mpk(A, q, sb, re=None, im=None):
    """Matrix powers kernel, MPK(s, v) of Fig. 4 in its global (1-partition) form.
    W[:,0] = q;  W[:,k] = (A - theta_k I) W[:,k-1]  (Newton basis);  monomial when
    all theta = 0.  Complex pair a +- ib at steps k, k+1:
        W[:,k]   = (A - aI) W[:,k-1]
        W[:,k+1] = (A - aI) W[:,k] + b^2 W[:,k-1]      ([4] §7.3.2 via P:94)."""
    n = A.shape[0]
    if re is None:
        re = np.zeros(sb)
        im = np.zeros(sb)
    W = np.zeros((n, sb + 1), order="F")
    W[:, 0] = q
    for k, (a, b2, kind) in enumerate(block_shifts(re, im, sb), start=1):
        W[:, k] = A @ W[:, k - 1] - a * W[:, k - 1]
        if kind == "p2":
            W[:, k] += b2 * W[:, k - 2]
    return W


def change_of_basis(sb, re=None, im=None):
    """B ((sb+1) x sb) with A W[:,0:sb] = W B for the W of mpk() (from [4] via P:94):
    real theta_k: B[k-1,k-1] = theta_k, B[k,k-1] = 1;  pair at (k,k+1): columns
    [a, 1, 0]^T and [-b^2, a, 1]^T."""
    if re is None:
        re = np.zeros(sb)
        im = np.zeros(sb)
    B = np.zeros((sb + 1, sb))
    for k, (a, b2, kind) in enumerate(block_shifts(re, im, sb), start=1):
        c = k - 1                      # column of B for A W[:,k-1]
        B[c, c] = a
        B[c + 1, c] = 1.0
        if kind == "p2":
            B[c - 1, c] = -b2
    return B


# ---------------------------------------------------------------------------------------
# Block orthogonalisation (P:142-146 MGS, P:156 CGS)
# ---------------------------------------------------------------------------------------
def borth_cgs(Q, P):
    """BOrth by CGS: C = Q^T P ; P := P - Q C.  Returns (C, P_new)."""
    C = Q.T @ P
    return C, P - Q @ C


def borth_mgs(Q, P):
    """BOrth by MGS: for l = 1..j:  P := P - q_l (q_l^T P)."""
    P = P.copy()
    C = np.zeros((Q.shape[1], P.shape[1]))
    for l in range(Q.shape[1]):
        C[l, :] = Q[:, l] @ P
        P -= np.outer(Q[:, l], C[l, :])
    return C, P


# ---------------------------------------------------------------------------------------
# TSQR variants (Fig. 9, Fig. 10); all return (Q, R), R upper with
# positive diagonal.
# ---------------------------------------------------------------------------------------
def _trsm_right(P, R):
    """P R^{-1} by triangular solve (the DTRSM of P:166 / P:275)."""
    return sla.solve_triangular(R, P.T, trans="T", lower=False).T


def tsqr_cholqr(P):
    """CholQR: B = P^T P ; R = chol(B) (R^T R = B) ; Q = P R^{-1}."""
    B = P.T @ P
    try:
        L = np.linalg.cholesky(B)
    except np.linalg.LinAlgError as e:
        raise Breakdown("CholQR: Gram matrix not positive definite") from e
    R = L.T.copy()
    return _trsm_right(P, R), R


def borth_cholqr_onepass(Q, P):
    """One-pass BOrth + CholQR (the fused-CGS direction of P:176 and
    the one-reduction tall-skinny kernels of P:275 fn 7).  P = [q_j, W_1..W_sb]:
      M  = [Q P]^T P                       (one product: C and the Gram of the raw panel)
      Cf = M[0:j, :] with column 0 := 0     (q_j is not re-orthogonalised, G2)
      G  = M[j:, :] - Cf^T Cf               (Pythagoras: = (P - Q Cf)^T (P - Q Cf) when Q^T Q = I)
      R  = chol(G) ;  Q_hat = (P - Q Cf) R^{-1}
    Returns (C = Cf[:, 1:], Q_hat, R).  Equal to borth_cgs + tsqr_cholqr in exact arithmetic
    when Q has orthonormal columns."""
    j = Q.shape[1]
    M = np.column_stack([Q, P]).T @ P
    Cf = M[:j, :].copy()
    Cf[:, 0] = 0.0
    G = M[j:, :] - Cf.T @ Cf
    try:
        L = np.linalg.cholesky(G)
    except np.linalg.LinAlgError as e:
        raise Breakdown("one-pass CholQR: Gram matrix not positive definite") from e
    R = L.T.copy()
    return Cf[:, 1:], _trsm_right(P - Q @ Cf, R), R


def tsqr_svqr(P):
    """SVQR (G14): B = P^T P ; D = diag(B)^{-1/2} ; D B D = U S U^T ;
    s_i <- max(s_i, eps*s_max) ; R_hat = R of qr(S^{1/2} U^T) with positive diagonal ;
    R = R_hat D^{-1} ; Q = P R^{-1}."""
    B = P.T @ P
    dB = np.diag(B)
    if np.any(dB <= 0.0):
        raise Breakdown("SVQR: zero column")
    d = 1.0 / np.sqrt(dB)
    Bh = d[:, None] * B * d[None, :]
    s, U = np.linalg.eigh(Bh)
    s = np.maximum(s, EPS * s.max())
    M = np.sqrt(s)[:, None] * U.T
    _, Rh = np.linalg.qr(M)
    sg = np.sign(np.diag(Rh))
    sg[sg == 0] = 1.0
    Rh = sg[:, None] * Rh
    R = Rh / d[None, :]
    return _trsm_right(P, R), R


def tsqr_mgs(P):
    """TSQR by MGS (Fig. 9 left): column by column dot products."""
    V = P.copy()
    w = V.shape[1]
    R = np.zeros((w, w))
    for k in range(w):
        for l in range(k):
            R[l, k] = V[:, l] @ V[:, k]
            V[:, k] -= R[l, k] * V[:, l]
        R[k, k] = np.sqrt(V[:, k] @ V[:, k])
        if R[k, k] == 0.0:
            raise Breakdown("MGS: zero column")
        V[:, k] /= R[k, k]
    return V, R


def tsqr_cgs(P):
    """TSQR by CGS (Fig. 9 right): per column r = V_{1:k-1}^T v_k."""
    V = P.copy()
    w = V.shape[1]
    R = np.zeros((w, w))
    for k in range(w):
        r = V[:, :k].T @ V[:, k]
        V[:, k] -= V[:, :k] @ r
        R[:k, k] = r
        R[k, k] = np.sqrt(V[:, k] @ V[:, k])
        if R[k, k] == 0.0:
            raise Breakdown("CGS: zero column")
        V[:, k] /= R[k, k]
    return V, R


def tsqr_caqr(P, row_blocks=1):
    """CAQR (Fig. 9 bottom right): local QR of each row block, QR of the stacked
    R's, V^(d) := V^(d) Q^(d).  Q formed explicitly (P:245 fn 6); signs normalised so
    diag(R) > 0 (G19)."""
    n, w = P.shape
    edges = [(b * n) // row_blocks for b in range(row_blocks + 1)]
    Ql, Rs = [], []
    for b in range(row_blocks):
        q, r = np.linalg.qr(P[edges[b]:edges[b + 1]])
        Ql.append(q)
        Rs.append(r)
    Qs, R = np.linalg.qr(np.vstack(Rs))
    Q = np.zeros_like(P)
    off = 0
    for b in range(row_blocks):
        kb = Rs[b].shape[0]
        Q[edges[b]:edges[b + 1]] = Ql[b] @ Qs[off:off + kb]
        off += kb
    sg = np.sign(np.diag(R))
    sg[sg == 0] = 1.0
    return Q * sg[None, :], sg[:, None] * R


def tsqr_cholqr_svqr_retry(P):
    """CholQR, and on its breakdown (non-positive pivot) the same panel by SVQR
     — the opt-in retry of reading G15 (no silent fallback without the flag)."""
    try:
        return tsqr_cholqr(P)
    except Breakdown:
        return tsqr_svqr(P)


TSQR = {"cholqr": tsqr_cholqr, "svqr": tsqr_svqr, "mgs": tsqr_mgs, "cgs": tsqr_cgs,
        "caqr": tsqr_caqr, "cholqr_retry": tsqr_cholqr_svqr_retry}
BORTH = {"cgs": borth_cgs, "mgs": borth_mgs}


# ---------------------------------------------------------------------------------------
# Hessenberg update ("H obtained as a by-product"; formula lost with Fig. 2, G1)
# ---------------------------------------------------------------------------------------
def hessenberg_update(H, j, sb, Rt, B):
    """H[0:j+sb+1, j:j+sb] = (Rt B - [H[0:j+1,0:j] Cs ; 0]) T^{-1}
    with Rt = [C; R] ((j+sb+1) x (sb+1)), Cs = Rt[0:j, 0:sb], T = Rt[j:j+sb, 0:sb].
    Derivation: A Q[:,0:j] = Q[:,0:j+1] H_prev and A W[:,0:sb] = W B with
    W = Q[:,0:j+sb+1] Rt."""
    M = Rt @ B                                   # (j+sb+1) x sb
    if j > 0:
        M[0:j + 1, :] -= H[0:j + 1, 0:j] @ Rt[0:j, 0:sb]
    T = Rt[j:j + sb, 0:sb]
    # M T^{-1} by triangular solve
    H[0:j + sb + 1, j:j + sb] = sla.solve_triangular(T, M.T, trans="T", lower=False).T
    return H


# ---------------------------------------------------------------------------------------
# Least squares by Givens rotations (y = argmin ||c - H z||, ~3(m+1)^2 flops)
# ---------------------------------------------------------------------------------------
def givens_ls(H, beta):
    """Solve min_y || beta e1 - H y ||_2 for upper Hessenberg H ((k+1) x k) by Givens QR.
    Returns (y, res) with res[i] = |g_{i+1}| the residual estimate after i+1 columns."""
    H = np.array(H, dtype=np.float64, copy=True)
    kp1, k = H.shape
    g = np.zeros(kp1)
    g[0] = beta
    res = np.zeros(k)
    for i in range(k):
        a, b = H[i, i], H[i + 1, i]
        r = np.hypot(a, b)
        c, s = (1.0, 0.0) if r == 0.0 else (a / r, b / r)
        Hi = H[i, i:].copy()
        H[i, i:] = c * Hi + s * H[i + 1, i:]
        H[i + 1, i:] = -s * Hi + c * H[i + 1, i:]
        g[i], g[i + 1] = c * g[i], -s * g[i]
        res[i] = abs(g[i + 1])
    y = sla.solve_triangular(H[:k, :k], g[:k], lower=False)
    return y, res


# ---------------------------------------------------------------------------------------
# Ritz values and (modified) Leja ordering (ref [17]; G10)
# ---------------------------------------------------------------------------------------
def ritz_values(H, m):
    """Eigenvalues of the square part H[0:m, 0:m] of the first restart's Hessenberg."""
    return np.linalg.eigvals(H[:m, :m])


def modified_leja(theta, s):
    """Leja order ('distance between two consecutive shifts is maximized'; G10):
    candidates = values with im >= 0 (a complex one stands for its conjugate pair), sorted by
    (re, im) ascending.  First: max |theta| (tie: larger re).  Next: argmax of
    sum_i log|theta - theta_i| over all chosen points (conjugates included), ties -> first in
    sorted order; a chosen complex point is followed by its conjugate.  Stops once >= s
    shifts are listed.  Returns (re, im) arrays of length >= s."""
    theta = np.asarray(theta, dtype=np.complex128)
    # keep multiplicity: duplicates stay as separate candidates (score -inf -> last)
    cand = sorted([(float(t.real), float(t.imag)) for t in theta if t.imag >= 0.0],
                  key=lambda t: (t[0], t[1]))
    chosen = []          # full list of chosen points incl. conjugates
    out_re, out_im = [], []
    remaining = list(range(len(cand)))
    # first point: max modulus, ties -> larger re
    best = None
    for idx in remaining:
        a, b = cand[idx]
        key = (np.hypot(a, b), a)
        if best is None or key > best[0]:
            best = (key, idx)
    order = [best[1]]
    remaining.remove(best[1])

    def push(idx):
        a, b = cand[idx]
        out_re.append(a); out_im.append(b); chosen.append(complex(a, b))
        if b > 0.0:
            out_re.append(a); out_im.append(-b); chosen.append(complex(a, -b))

    push(order[0])
    while len(out_re) < s and remaining:
        best = None
        for idx in remaining:
            z = complex(*cand[idx])
            with np.errstate(divide="ignore"):
                sc = float(np.sum(np.log(np.abs(z - np.asarray(chosen)))))
            if best is None or sc > best[0]:
                best = (sc, idx)
        remaining.remove(best[1])
        push(best[1])
    return np.asarray(out_re), np.asarray(out_im)


# ---------------------------------------------------------------------------------------
# GMRES(m) (Saad-Schultz [3]) — independent second method for the CA == GMRES pin
# ---------------------------------------------------------------------------------------
def arnoldi_mgs(A, r, m):
    n = A.shape[0]
    beta = np.linalg.norm(r)
    Q = np.zeros((n, m + 1), order="F")
    H = np.zeros((m + 1, m))
    Q[:, 0] = r / beta
    for k in range(m):
        w = A @ Q[:, k]
        for i in range(k + 1):
            H[i, k] = Q[:, i] @ w
            w = w - H[i, k] * Q[:, i]
        H[k + 1, k] = np.linalg.norm(w)
        if H[k + 1, k] == 0.0:
            raise Breakdown("Arnoldi breakdown")
        Q[:, k + 1] = w / H[k + 1, k]
    return Q, H, beta


def arnoldi_cgs(A, r, m, reorth=False):
    """First (shift-finding) cycle of Newton CA-GMRES: the standard GMRES iterations as
    the paper runs GMRES — Arnoldi with CGS (the "GMRES ... CGS" rows of Fig. 14),
    plus one reorthogonalisation pass ("2x", CGS2) when reorth (reading G12)."""
    n = A.shape[0]
    beta = np.linalg.norm(r)
    Q = np.zeros((n, m + 1), order="F")
    H = np.zeros((m + 1, m))
    Q[:, 0] = r / beta
    for k in range(m):
        w = A @ Q[:, k]
        c = Q[:, :k + 1].T @ w
        w = w - Q[:, :k + 1] @ c
        if reorth:
            c2 = Q[:, :k + 1].T @ w
            w = w - Q[:, :k + 1] @ c2
            c = c + c2
        H[:k + 1, k] = c
        H[k + 1, k] = np.sqrt(w @ w)
        if H[k + 1, k] == 0.0:
            raise Breakdown("Arnoldi breakdown")
        Q[:, k + 1] = w / H[k + 1, k]
    return Q, H, beta


def arnoldi_cgs2(A, r, m):
    """arnoldi_cgs with one reorthogonalisation (CGS2)."""
    return arnoldi_cgs(A, r, m, reorth=True)


def gmres(A, b, m, tol=1e-8, maxcyc=100, x0=None):
    """Restarted GMRES(m), MGS Arnoldi, Givens LS; explicit residual at restarts."""
    A = sp.csr_matrix(A)
    x = np.zeros(A.shape[0]) if x0 is None else np.array(x0, dtype=np.float64)
    rho0 = np.linalg.norm(b - A @ x)
    hist = []
    for _ in range(maxcyc):
        r = b - A @ x
        Q, H, beta = arnoldi_mgs(A, r, m)
        y, _ = givens_ls(H, beta)
        x = x + Q[:, :m] @ y
        rho = np.linalg.norm(b - A @ x)
        hist.append(rho / rho0)
        if rho <= tol * rho0:
            break
    return dict(x=x, hist=np.asarray(hist), cycles=len(hist))


# ---------------------------------------------------------------------------------------
# CA-GMRES(s, m) (Fig. 2 reconstructed per SURVEY §8(c) / DESIGN.md)
# ---------------------------------------------------------------------------------------
def ca_cycle(A, Q, H, s, m, re, im, tsqr="cholqr", borth="cgs", reorth=False,
             caqr_blocks=1, diag=None, onepass=False):
    """One restart cycle's basis generation: fills Q[:,1:m+1] and H ((m+1) x m) given
    Q[:,0] = r/beta.  Blocks of sb = min(s, m-j).  onepass: panels with j > 0 use
    borth_cholqr_onepass (CholQR only) for each BOrth+TSQR pass."""
    j = 0
    tsqr_f = TSQR[tsqr]
    borth_f = BORTH[borth]
    if onepass and (tsqr != "cholqr" or borth != "cgs"):
        raise ValueError("onepass needs tsqr='cholqr', borth='cgs'")

    def bt_pass(P):                                          # one BOrth + TSQR pass on P
        Cc = np.zeros((j, P.shape[1]))
        if onepass and j > 0:
            Cc[:, 1:], Qh_, R_ = borth_cholqr_onepass(Q[:, :j], P)
            return Cc, Qh_, R_
        P = P.copy()
        if j > 0:                                            # BOrth, col 0 skipped
            Cp, P1 = borth_f(Q[:, :j], P[:, 1:])
            Cc[:, 1:] = Cp
            P[:, 1:] = P1
        Qh_, R_ = tsqr_caqr(P, caqr_blocks) if tsqr == "caqr" else tsqr_f(P)   # TSQR (Fig. 9)
        return Cc, Qh_, R_

    while j < m:
        sb = min(s, m - j)
        W = mpk(A, Q[:, j], sb, re, im)                          # MPK (Fig. 4)
        B = change_of_basis(sb, re, im)
        C, Qh, R = bt_pass(W)
        if reorth:                                               # "2x" (G16)
            C2, Qh, R2 = bt_pass(np.column_stack([Q[:, j], Qh[:, 1:]]))
            C = C + C2 @ R
            R = R2 @ R
        Q[:, j + 1:j + sb + 1] = Qh[:, 1:]                       # q_j kept (G2)
        if diag is not None:
            diag.append(dict(j=j, sb=sb, R=R.copy(), C=C.copy(),
                             orth=np.linalg.norm(np.eye(sb + 1) - np.column_stack(
                                 [Q[:, j], Qh[:, 1:]]).T @ np.column_stack([Q[:, j], Qh[:, 1:]]), 2),
                             cond_gram=np.linalg.cond(W.T @ W)))
        Rt = np.vstack([C, R])
        hessenberg_update(H, j, sb, Rt, B)
        j += sb
    return Q, H


def cagmres(A, b, s, m, basis="newton", tsqr="cholqr", borth="cgs", reorth=False,
            tol=1e-8, maxcyc=100, x0=None, shifts=None, caqr_blocks=1, diag=None,
            keep_last=False, onepass=False):
    """CA-GMRES(s, m) solve.  x0 = 0 by default (G17).
    basis 'newton': first cycle is GMRES(m) (Arnoldi CGS, CGS2 if reorth) unless shifts are given; its
    Ritz values in modified Leja order become the shifts.  'monomial': theta = 0
    from cycle 1 (G18).  Returns dict(x, hist (rho_c / rho_0 per cycle), cycles, shifts)."""
    A = sp.csr_matrix(A)
    n = A.shape[0]
    x = np.zeros(n) if x0 is None else np.array(x0, dtype=np.float64)
    rho0 = np.linalg.norm(b - A @ x)
    out = dict(x=x, hist=np.zeros(0), cycles=0, shifts=None)
    if rho0 == 0.0:
        return out
    if basis == "monomial":
        re, im = np.zeros(s), np.zeros(s)
    elif shifts is not None:
        re, im = (np.asarray(shifts[0], dtype=np.float64), np.asarray(shifts[1], dtype=np.float64))
    else:
        re = im = None
    hist = []
    last = None
    for c in range(maxcyc):
        r = b - A @ x
        beta = np.linalg.norm(r)
        Q = np.zeros((n, m + 1), order="F")
        Q[:, 0] = r / beta
        H = np.zeros((m + 1, m))
        if re is None:                                   # first Newton cycle = GMRES(m)
            Q, H, _ = arnoldi_cgs(A, r, m, reorth=reorth)
            re, im = modified_leja(ritz_values(H, m), s)
        else:
            ca_cycle(A, Q, H, s, m, re, im, tsqr, borth, reorth, caqr_blocks, diag, onepass)
        y, _ = givens_ls(H, beta)                        # LS on the CPU
        x = x + Q[:, :m] @ y                             # x := x + V_{1:m} y
        rho = np.linalg.norm(b - A @ x)                  # explicit residual (G17)
        hist.append(rho / rho0)
        if keep_last:
            last = dict(Q=Q, H=H, beta=beta)
        if rho <= tol * rho0:
            break
    out.update(x=x, hist=np.asarray(hist), cycles=len(hist),
               shifts=(np.asarray(re), np.asarray(im)), last=last)
    return out


# ---------------------------------------------------------------------------------------
# Multi-GPU setup pieces (P:45 block rows; P:60-64 boundary-set recursion)
# ---------------------------------------------------------------------------------------
def block_rows(n, nranks):
    """Contiguous block-row distribution with about equal rows per GPU (P:45, P:104 fn 2)."""
    return np.array([(p * n) // nranks for p in range(nranks + 1)], dtype=np.int64)


def boundary_sets(A, own_begin, own_end, s):
    """delta^(d,k) for k = s..1 by the recursion of P:62:
        delta^(d,k) = U_{i in i^(d,k+1)} str(a_i,:) \\ i^(d,k+1),  i^(d,k) = i^(d,k+1) U delta^(d,k)
    with i^(d,s+1) = owned rows.  Returned as a list indexed by distance h = s-k+1 = 1..s
    (delta^(d,s) is distance 1), each a sorted int64 array of global row ids."""
    A = sp.csr_matrix(A)
    cur = set(range(own_begin, own_end))
    frontier = sorted(cur)
    levels = []
    for _ in range(s):
        nxt = set()
        for i in frontier:
            nxt.update(A.indices[A.indptr[i]:A.indptr[i + 1]].tolist())
        nxt -= cur
        levels.append(np.array(sorted(nxt), dtype=np.int64))
        cur |= nxt
        frontier = sorted(nxt)
    return levels


def orth_error(Q):
    """||I - Q^T Q||_2 (G6)."""
    return np.linalg.norm(np.eye(Q.shape[1]) - Q.T @ Q, 2)


def fact_error(P, Q, R):
    """||P - QR||_F / ||P||_F (G6)."""
    return np.linalg.norm(P - Q @ R) / np.linalg.norm(P)
