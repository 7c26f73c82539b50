"""SpMV kernel variants (CAGMRES_OPT_SPMV) on the bench matrices: device time of one MPK
block (s SpMV steps, CUDA events) per variant, and a bitwise check of the basis against
variant 0 (one slice per warp).

    python tools/spmv_variants.py [--s 10]
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


def timeit(fn, reps=20):
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
    ap.add_argument("--s", type=int, default=10)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    mats = {"C2 cd7 128^3": G.convection_diffusion(128, 3, 7),
            "C3 g3-shaped": G.g3_shaped(),
            "C4 banded-27": G.banded()}
    out = {}
    for name, A in mats.items():
        q = torch.tensor(G.rhs(A.n), device="cuda")
        q /= q.norm()
        S = Solver(A, s=args.s, m=30, basis="monomial")
        res = {}
        W0 = None
        for v in (0, 5, 16, 17):
            S.set_option("spmv", v)
            W = S.mpk(q, args.s)
            if W0 is None:
                W0 = W.clone()
            ms = timeit(lambda: S.mpk(q, args.s))
            res[f"v{v}"] = {"us_per_step": round(1000 * ms / args.s, 2),
                            "bitwise_eq_v0": bool(torch.equal(W, W0))}
        out[name] = res
        print(name, json.dumps(res), file=sys.stderr, flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
