"""Run the temporally blocked MPK (forced) on C2 a few times — target for `ncu -k regex:mpk_wave`."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402

ch = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
ctas = int(sys.argv[2]) if len(sys.argv) > 2 else 2
lag = int(sys.argv[3]) if len(sys.argv) > 3 else 0
torch.cuda.set_device(0)
A = G.convection_diffusion(128, 3, 7)
S = Solver(A, s=10, m=30, basis="monomial")
S.set_option("mpk_wave", 2)
S2 = Solver(A, s=10, m=30, basis="monomial")   # stepwise reference (spmv kernel)
S.set_option("wave_chunk", ch)
S.set_option("wave_ctas", ctas)
S.set_option("wave_lag", lag)
q = torch.tensor(G.rhs(A.n) / np.linalg.norm(G.rhs(A.n)), device="cuda")
W = torch.empty(11, A.n, dtype=torch.float64, device="cuda").t()
for _ in range(4):
    S.mpk(q, 10, out=W)
    S2.mpk(q, 10, out=W)
torch.cuda.synchronize()
print("done")
