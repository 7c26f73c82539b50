"""Per-kernel microbenchmarks at bench sizes through the C ABI (device time, CUDA events).

    python tools/microbench.py [--n 2097152]

Reports achieved GB/s against the algorithmic bytes of DESIGN.md §6 for BOrth (xTy +
update), TSQR (Gram+Cholesky + TRSM) and one MPK step, plus the split between the two
halves of BOrth/TSQR (timed via the standalone kernels' API calls).
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402


def timeit(fn, reps=10):
    st = torch.cuda.current_stream()
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        fn()
        e1.record(st)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=128 ** 3)
    args = ap.parse_args()
    n = args.n
    torch.cuda.set_device(0)
    A = G.convection_diffusion(128, 3, 7) if n == 128 ** 3 else G.banded(n=n)
    S = Solver(A, s=10, m=64, basis="monomial")
    ld = (n + 31) // 32 * 32
    out = {}
    V = torch.randn(66, ld, dtype=torch.float64, device="cuda").t()   # col-major n x 66, ld
    V = V[:n]
    for (j, w) in [(1, 1), (10, 1), (30, 1), (10, 10), (20, 10), (55, 5), (30, 6)]:
        Q = V[:, :j]
        P = V[:, 66 - w:66]                      # disjoint from Q (j <= 55)
        t = timeit(lambda: S.borth(Q, j, P, w))
        by = 8.0 * n * (2 * j + 3 * w)
        out[f"borth j={j} w={w}"] = dict(ms=round(t, 4), gbs=round(by / t / 1e6, 1))
    for w, gram in [(1, 0), (6, 0), (11, 0), (16, 0), (1, 1), (6, 1), (11, 1), (12, 1)]:
        S.set_option("gram", gram)
        Pt = torch.randn(w, ld, dtype=torch.float64, device="cuda")
        P = Pt.t()[:n]                           # fresh column-major panel, ld = ld

        def f():
            S.tsqr(P, w, "cholqr")
        try:
            t = timeit(f)
            by = 8.0 * n * (3 * w)
            out[f"tsqr cholqr w={w} gram={gram}"] = dict(ms=round(t, 4), gbs=round(by / t / 1e6, 1))
        except Exception as e:                   # report, keep going
            out[f"tsqr cholqr w={w} gram={gram}"] = dict(error=str(e), norms=[float(P[:, c].norm()) for c in range(w)])
    q = torch.tensor(G.rhs(n), device="cuda")
    W = torch.empty(11, n, dtype=torch.float64, device="cuda").t()
    t = timeit(lambda: S.mpk(q, 10, out=W))
    by = 10 * (12.0 * A.nnz + 4 * (n + 1) + 16.0 * n) + 16.0 * n * 11
    out["mpk sb=10 (incl. copies)"] = dict(ms=round(t, 4), gbs=round(by / t / 1e6, 1))
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
