"""Measure the margins behind the DESIGN.md §8 parity tolerances (run on a GPU box):

  * MPK: max_k max|W_gpu[:,k] - W_orc[:,k]| / max|W_orc[:,k]| on the parity generators;
  * solve: per cycle, the GPU's relative residual deviation from the oracle,
    d_c = |rho_gpu - rho_orc| / rho_orc, next to the oracle's own rounding envelope env_c
    (its deviation from itself under symmetric permutations P A P^T, P b) — reported as
    max_c d_c / max(env_c, 1e-16) and the largest d_c where env_c < 1e-10.

    python tools/parity_margins.py > profiles/r2_parity_margins.json
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402

from oracle import cagmres_oracle as O  # noqa: E402
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402
from test_gpu_parity import SHIFTS, rounding_envelope  # noqa: E402


def dev(x):
    return torch.tensor(np.ascontiguousarray(x), dtype=torch.float64, device="cuda")


def mpk_margins():
    gens = {"C1": lambda: G.convection_diffusion(32, 2, 5),
            "cd27_ragged": lambda: G.convection_diffusion(13, 3, 27),
            "g3_small": lambda: G.g3_shaped(n=50001, width=250),
            "banded": lambda: G.banded(n=300001),
            "C2": lambda: G.convection_diffusion(128, 3, 7)}
    out = {}
    for name, f in gens.items():
        A = f()
        As = A.to_scipy()
        for basis in ("monomial", "newton"):
            S = Solver(A, s=10, m=30, basis=basis)
            re = im = None
            if basis == "newton":
                re, im = SHIFTS
                S.set_shifts(re, im)
            q = G.u(11, np.arange(A.n))
            q /= np.linalg.norm(q)
            W = S.mpk(dev(q), 10).cpu().numpy()
            Wo = O.mpk(As, q, 10, re, im)
            rel = [float(np.max(np.abs(W[:, k] - Wo[:, k])) / np.max(np.abs(Wo[:, k]))) for k in range(11)]
            out[f"{name}/{basis}"] = {"max_rel": max(rel), "per_k": rel}
            S.close()
    return out


def solve_margins():
    cases = {
        "C1_newton_injected": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton"), True),
        "C1_monomial": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="monomial"), False),
        "C1_newton_first_cycle": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton"), False),
        "cd7_40_s10": (lambda: G.convection_diffusion(40, 3, 7), dict(s=10, m=30, basis="newton"), True),
        "g3_40k": (lambda: G.g3_shaped(n=40000, width=200), dict(s=5, m=60, basis="newton"), False),
        "C2_full": (lambda: G.convection_diffusion(128, 3, 7), dict(s=10, m=30, basis="newton"), False),
        "C1_svqr": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton", tsqr="svqr"), True),
        "C1_cholqr2": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton", reorth=True), True),
        "C1_cgs2": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton", tsqr="cgs", reorth=True), True),
        "C1_mgs": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton", tsqr="mgs", borth="mgs"), True),
        "C1_caqr": (lambda: G.convection_diffusion(32, 2, 5), dict(s=5, m=30, basis="newton", tsqr="caqr"), True),
    }
    only = os.environ.get("MARGINS_ONLY")
    if only:
        cases = {k: v for k, v in cases.items() if k in only.split(",")}
    out = {}
    for name, (f, kw, inject) in cases.items():
        A = f()
        As = A.to_scipy()
        b = G.rhs(A.n)
        sh = None
        if inject:
            sh = O.modified_leja(O.ritz_values(O.arnoldi_cgs2(As, b, kw["m"])[1], kw["m"]), kw["s"])
        S = Solver(A, **kw)
        if sh is not None:
            S.set_shifts(*sh)
        _, st = S.solve(dev(b), tol=1e-8, maxit=200)
        ref, env = rounding_envelope(As, b, nperm=2, tol=1e-8, maxcyc=200, shifts=sh, **kw)
        k = min(len(ref), len(st.hist))
        d = np.abs(st.hist[:k] - ref[:k]) / ref[:k]
        ratio = d / np.maximum(env[:k], 1e-16)
        out[name] = {"cycles_gpu": int(st.cycles), "cycles_oracle": int(len(ref)),
                     "max_rel_dev": float(d.max()), "max_ratio_to_env": float(ratio.max()),
                     "per_cycle_rel_dev": [float(x) for x in d], "per_cycle_env": [float(x) for x in env[:k]],
                     "rho": [float(x) for x in ref[:k]]}
        S.close()
    return out


if __name__ == "__main__":
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())     # ordinary stream, as bench.py (PDL on)
    out = {"solve": solve_margins()}
    if not os.environ.get("MARGINS_ONLY"):
        out["mpk"] = mpk_margins()
    print(json.dumps(out, indent=1))
