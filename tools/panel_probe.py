"""Device time of single panel kernels on C2-sized panels (n = 2,097,152) through the C ABI
(cagmres_tsqr / cagmres_borth), per kernel option, CUDA events, median of R runs.

    python tools/panel_probe.py
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402


def med(fn, reps=15):
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
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts))


def main():
    torch.cuda.set_device(0)
    n, w = 128 ** 3, 11
    A = G.convection_diffusion(128, 3, 7)
    S = Solver(A, s=10, m=30, basis="monomial")
    g = torch.Generator(device="cuda").manual_seed(0)
    P0 = torch.randn(w, n, dtype=torch.float64, device="cuda", generator=g).t()   # column-major n x w
    P = P0.clone()
    out = {}
    for opt, vals in (("gram", [0, 1, 2]), ("trsm", [0, 1])):
        for v in vals:
            S.set_option(opt, v)

            def f():
                P.copy_(P0)
                S.tsqr(P, w)
            t_copy = med(lambda: P.copy_(P0))
            t = med(f) - t_copy
            out[f"tsqr {opt}={v}"] = round(t, 1)
            print(opt, v, round(t, 1), file=sys.stderr, flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
