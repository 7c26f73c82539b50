"""Sweep the temporal-blocking MPK parameters (chunk rows, CTAs/SM, lag) and compare with one
SpMV launch per step.  Device time of cagmres_mpk (sb = s = 10; includes the copy of q in and
of the 11 basis columns out, the same for both).

    python tools/wave_tune.py [C2|C5s|band] > profiles/r2_wave_tune.json
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402
from tools.microbench import timeit  # noqa: E402

torch.cuda.set_device(0)
which = sys.argv[1:] or ["C2"]
mats = {"C2": lambda: G.convection_diffusion(128, 3, 7),
        "C5s": lambda: G.convection_diffusion(200, 3, 27),
        "band": lambda: G.banded()}
res = {}
for name in which:
    A = mats[name]()
    S = Solver(A, s=10, m=30, basis="newton")
    S.set_shifts(np.array([7.9, 7.9, 0.09, 0.09, 3.8, 5.5, 1.2, 6.6, 2.5, 4.4]),
                 np.array([0.02, -0.02, 0.03, -0.03, 0, 0, 0, 0, 0, 0]))
    q = torch.tensor(G.rhs(A.n), device="cuda")
    q /= q.norm()
    W = torch.empty(11, A.n, dtype=torch.float64, device="cuda").t()
    S.set_option("mpk_wave", 0)
    base = timeit(lambda: S.mpk(q, 10, out=W))
    one = timeit(lambda: S.mpk(q, 1, out=W[:, :2]))
    S.mpk(q, 10, out=W)
    ref = W.clone()
    r = {"stepwise_ms": round(base, 4), "sb1_ms": round(one, 4)}
    S.set_option("mpk_wave", 2)                      # force (skip the L2-fit heuristic)
    for ch in (512, 1024, 2048):
        for ctas in (2, 3, 4):
            for lag in (0, 24, 48, 96, 192):
                S.set_option("wave_chunk", ch)
                S.set_option("wave_ctas", ctas)
                S.set_option("wave_lag", lag)
                t = timeit(lambda: S.mpk(q, 10, out=W))
                ok = bool(torch.equal(W, ref))
                r[f"ch{ch}_c{ctas}_L{lag}"] = (round(t, 4), ok)
                print(name, ch, ctas, lag, round(t, 4), ok, file=sys.stderr, flush=True)
    res[name] = r
print(json.dumps(res, indent=1))
