"""C4 study (banded-27, n = 4,194,304, monomial basis, a fixed number of
cycles): the TSQR variants of Fig. 9 / Fig. 10 on the identical ill-conditioned MPK panel — time,
achieved HBM GB/s against the algorithmic bytes of DESIGN.md §6, the paper's "effective Gflop/s"
(4 n w^2 - 4 w^3 / 3) / t (DGEQRF + DORGQR flops), ||I - Q^T Q||_2 (GPU and oracle) — and a
3-cycle CholQR2 solve with per-phase GB/s and the per-panel diagnostics (kappa(W^T W)).

    python tools/c4_study.py > profiles/r2_c4_study.json
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import cagmres_oracle as O  # noqa: E402
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402


def colmajor(M):
    return torch.tensor(np.ascontiguousarray(np.asarray(M).T), dtype=torch.float64, device="cuda").t()


def main():
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())     # ordinary stream, as bench.py (PDL on)
    A = G.banded()
    As = A.to_scipy()
    n, s = A.n, 10
    w = s + 1
    S = Solver(A, s=15, m=30, basis="monomial")
    q = torch.tensor(G.rhs(n), device="cuda")
    q /= q.norm()
    W = S.mpk(q, s)
    Wh = W.cpu().numpy()
    kappa = float(np.linalg.cond(Wh))
    # bytes per variant (DESIGN.md §6 algorithmic model): Gram read + TRSM read/write per pass;
    # column passes of MGS / CGS as the solver counts them; CAQR reads twice, writes once
    nb = 8.0 * n
    model = {"cholqr": nb * 3 * w, "svqr": nb * 3 * w, "cholqr2": 2 * nb * 3 * w,      # (the API writes all w columns)
             "mgs": nb * sum(5 * k + 3 for k in range(w)), "cgs": nb * sum((2 * k + 3 if k else 0) + 3 for k in range(w)),
             "caqr": nb * 3 * w}
    out = {"config": "C4 banded-27, n = 4,194,304, monomial MPK panel s = 10 (w = 11)", "kappa_W": kappa, "variants": {}}
    for name, kind, reorth in (("cholqr", "cholqr", False), ("cholqr2", "cholqr", True), ("svqr", "svqr", False),
                               ("mgs", "mgs", False), ("cgs", "cgs", False), ("caqr", "caqr", False)):
        ts = []
        for rep in range(6):
            P = W.clone()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            R = S.tsqr(P, w, kind, reorth)
            e1.record()
            torch.cuda.synchronize()
            if rep:
                ts.append(e0.elapsed_time(e1))
        t = float(np.median(ts)) * 1e-3
        Q = P.cpu().numpy()
        orc = {"cholqr": lambda X: O.tsqr_cholqr(X), "svqr": O.tsqr_svqr, "mgs": O.tsqr_mgs, "cgs": O.tsqr_cgs,
               "caqr": O.tsqr_caqr, "cholqr2": lambda X: O.tsqr_cholqr(O.tsqr_cholqr(X)[0])}[name]
        try:
            eo = float(O.orth_error(orc(Wh)[0]))
        except O.Breakdown:
            eo = None
        out["variants"][name] = {
            "ms": round(t * 1e3, 4), "gbs": round(model[name] / t / 1e9, 1),
            "eff_gflops": round((4 * n * w * w - 4 * w ** 3 / 3) / t / 1e9, 1),
            "orth_err_gpu": float(O.orth_error(Q)), "orth_err_oracle": eo,
            "fact_err_gpu": float(O.fact_error(Wh, Q, R.cpu().numpy()))}
        print(name, json.dumps(out["variants"][name]), file=sys.stderr, flush=True)
    S2 = Solver(A, s=10, m=30, basis="monomial", reorth=True)
    b = torch.tensor(G.rhs(n), device="cuda")
    S2.solve(b, tol=0.0, maxit=1)
    _, st = S2.solve(b, tol=0.0, maxit=3, timing=True)
    _, sd = S2.solve(b, tol=0.0, maxit=3, diag=True)
    out["solve_3_cycles_cholqr2"] = {
        "ms": st.ms, "phase_gbs": {k: round(st.bytes[k] / (st.ms[k] * 1e-3) / 1e9, 1) for k in ("mpk", "borth", "tsqr")
                                   if st.ms[k] > 0},
        "hist": [float(x) for x in st.hist], "max_orth_err": sd.max_orth_err, "max_gram_cond": sd.max_gram_cond}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
