"""Panel-kernel fixed costs: one CholQR TSQR (Gram + Cholesky + TRSM) and one BOrth at
several n, for an ncu launch list (gpu__time_duration per kernel vs n separates the
per-launch fixed cost — final reduction, Cholesky, tail — from the streaming part).

    ncu --metrics gpu__time_duration.sum python tools/panel_scaling.py [--gram 1]
"""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--gram", type=int, default=1)
ap.add_argument("--w", type=int, default=11)
ap.add_argument("--pad", type=int, default=0, help="extra rows in the leading dimension")
args = ap.parse_args()
torch.cuda.set_device(0)
for n in [1 << 16, 1 << 18, 1 << 20, 1 << 21]:
    S = Solver(G.banded(n=n), s=1, m=32, basis="monomial")
    S.set_option("gram", args.gram)
    ld = n + args.pad
    V = torch.randn(args.w + 20, ld, dtype=torch.float64, device="cuda").t()[:n]
    P = V[:, 20:20 + args.w]
    for _ in range(2):
        S.tsqr(P, args.w, "cholqr")
        S.borth(V[:, :20], 20, P, args.w)
    torch.cuda.synchronize()
    print("n", n, flush=True)
