"""TSQR comparison on config C4 (ill-conditioned banded-27, n = 4,194,304), the B200 analog of
PAPER.md Fig. 10 / Fig. 13: MPK panels W = [q, Aq, ..., A^s q] (monomial
s = 10 and s = 15, and the Newton basis), factored by every TSQR variant of the library.

Reports per variant: ||I - Q^T Q||_2, ||W - QR||_F / ||W||_F, cond(W) (from R of CAQR),
device time of one call after a warm-up call (includes the call's host synchronisation), algorithmic GB/s and the paper's "effective Gflop/s" = (4 n w^2 - 4 w^3 / 3) / t
(DGEQRF + DORGQR flops).  Breakdowns are reported, not hidden.

    python tools/tsqr_study.py [--n 4194304] > profiles/r1_tsqr_study_C4.json
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200 import _lib as L  # noqa: E402
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402


def measure(S, W, w, kind, reorth):
    try:                                                  # warm-up (first-call set-up, caches)
        S.tsqr(W.clone(), w, kind, reorth)
    except L.CagmresError:
        pass
    P = W.clone()
    torch.cuda.synchronize()
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    try:
        R = S.tsqr(P, w, kind, reorth)
    except L.CagmresError as e:
        return {"breakdown": str(e)}
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    n = P.shape[0]
    QtQ = P.t() @ P
    orth = float(torch.linalg.matrix_norm(torch.eye(w, dtype=torch.float64, device="cuda") - QtQ, ord=2))
    fact = float(torch.linalg.matrix_norm(W - P @ R) / torch.linalg.matrix_norm(W))
    passes = 2 if reorth else 1
    by = 8.0 * n * 3 * w * passes
    flops = (4.0 * n * w * w - 4.0 * w ** 3 / 3.0)
    return {"orth_err": orth, "fact_err": fact, "ms": round(ms, 4), "gbs": round(by / ms / 1e6, 1),
            "eff_gflops": round(flops / ms / 1e6, 1)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=4194304)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    A = G.banded(n=args.n)
    q = torch.tensor(G.rhs(args.n), device="cuda")
    q /= q.norm()
    out = {"config": f"C4 banded-27 n={args.n}", "variants": {}}
    # Newton shifts from one GMRES(30) cycle of the library
    Sn = Solver(A, s=15, m=30, basis="newton")
    Sn.solve(torch.tensor(G.rhs(args.n), device="cuda"), tol=0.0, maxit=1)
    re, im = Sn.get_shifts()
    for label, basis, s in [("monomial s=10", "monomial", 10), ("monomial s=15", "monomial", 15),
                            ("newton s=10", "newton", 10)]:
        S = Solver(A, s=s, m=30, basis=basis)
        if basis == "newton":
            S.set_shifts(re, im)
        W = S.mpk(q, s)                                              # column-major (stride(0) == 1)
        w = s + 1
        res = {}
        _, Rh = torch.linalg.qr(W)
        sv = torch.linalg.svdvals(Rh)
        res["cond_W"] = float(sv[0] / sv[-1])
        for kind, reorth in [("cholqr", False), ("cholqr", True), ("svqr", False), ("mgs", False),
                             ("cgs", True), ("caqr", False)]:
            res[kind + ("2" if reorth else "")] = measure(S, W, w, kind, reorth)
        out["variants"][label] = res
        print(label, json.dumps(res), file=sys.stderr, flush=True)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
