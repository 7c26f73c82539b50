"""One C2 solve (for ncu --set full captures of single kernels).

    ncu --set full -k regex:NAME -s SKIP -c 1 -o OUT python tools/kprof.py [--opt spmv=5 ...]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--opt", action="append", default=[])
ap.add_argument("--config", default="C2")
ap.add_argument("--mpk-only", action="store_true", help="three MPK blocks instead of a solve")
args = ap.parse_args()
torch.cuda.set_device(0)
torch.cuda.set_stream(torch.cuda.Stream())     # an ordinary stream, as in bench.py (PDL on)
if args.config == "C2":
    A, s, m = G.convection_diffusion(128, 3, 7), 10, 30
else:
    A, s, m = G.g3_shaped(), 5, 60
S = Solver(A, s=s, m=m, basis="newton")
for kv in args.opt:
    k, v = kv.split("=")
    S.set_option(k, int(v))
b = torch.tensor(G.rhs(A.n), device="cuda")
if args.mpk_only:
    import numpy as np
    S.set_shifts(np.linspace(0.5, 3.0, s), np.zeros(s))
    q = b / b.norm()
    for _ in range(6):
        S.mpk(q, s)
    torch.cuda.synchronize()
    print("mpk done, spmv variant", S.get_option("spmv"))
else:
    x, st = S.solve(b, tol=1e-8, maxit=200)
    torch.cuda.synchronize()
    print("cycles", st.cycles, "spmv variant", S.get_option("spmv"))
