"""Where does the end-to-end solve (host b -> device, solve, x -> host) lose time against the
device-resident solve?  Times K solves of a bench config per variant (CUDA events, the
solve's own stream), same handle:
  dev      b, x resident (x zeroed in place)            — bench.py's `value`
  newx     b resident, a new x tensor per solve
  h2d      b copied from pinned host memory per solve, x resident
  e2e      bench.py's e2e: pinned b -> new device b, new x, solve, x -> pinned host

    python tools/e2e_probe.py [C2|C3] [K]
"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_yamazakiathd14_b200.solver import Solver  # noqa: E402
from synth import generators as G  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "C3"
K = int(sys.argv[2]) if len(sys.argv) > 2 else 5
cfg = bench.CFG[cfg_name]
torch.cuda.set_device(0)
torch.cuda.set_stream(torch.cuda.Stream())     # an ordinary stream, as in bench.py (PDL on)
A = cfg["build"]()
S = Solver(A, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"])
b_host = G.rhs(cfg["n"])
b = torch.tensor(b_host, device="cuda")
x = torch.zeros_like(b)
b_pin = torch.tensor(b_host).pin_memory()
x_pin = torch.empty_like(b_pin).pin_memory()
stream = torch.cuda.current_stream()
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")


def run(kind):
    S.clear_shifts()
    if kind == "dev":
        x.zero_()
        S.solve(b, x, tol=1e-8, maxit=200)
    elif kind == "newx":
        S.solve(b, torch.zeros_like(b), tol=1e-8, maxit=200)
    elif kind == "h2d":
        bd = b_pin.to("cuda", non_blocking=True)
        x.zero_()
        S.solve(bd, x, tol=1e-8, maxit=200)
    else:
        bd = b_pin.to("cuda", non_blocking=True)
        xd = torch.zeros_like(bd)
        S.solve(bd, xd, tol=1e-8, maxit=200)
        x_pin.copy_(xd, non_blocking=True)


for kind in ("dev", "newx", "h2d", "e2e", "dev"):
    for _ in range(2):
        run(kind)
    torch.cuda.synchronize()
    ev, wall = [], []
    for k in range(K):
        flush.fill_(float(k))
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(stream)
        run(kind)
        e1.record(stream)
        torch.cuda.synchronize()
        wall.append((time.perf_counter() - t0) * 1e3)
        ev.append(e0.elapsed_time(e1))
    print(f"{cfg_name} {kind:5s} events ms {np.round(ev, 2).tolist()}  wall ms {np.round(wall, 2).tolist()}", flush=True)
