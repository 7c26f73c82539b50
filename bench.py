"""bench.py — CA-GMRES(s, m) time-to-solution on B200 (BASELINE.json metric), one JSON line.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C2]

A step = one full cagmres_solve (all SURVEY §8(a) rows: MPK, BOrth, TSQR, small factor,
Hessenberg update, LS, x update, explicit residual; the first Newton cycle is GMRES(m))
from x0 = 0 to ||r|| <= 1e-8 ||r0|| on the N=1 workload, config C2 (BASELINE.json
configs[1]: 3D convection-diffusion 7-point 128^3, s=10, m=30, Newton, CholQR).
Inputs are resident in HBM before timing (A 175 MB + V 520 MB, larger than the 126 MB L2;
an L2 flush buffer is also written between steps).  value = mean device time per solve (ms,
lower is better); e2e = the same solve through the C ABI with b copied from pinned host
memory and x copied back inside the timed region.

Multi-GPU (torchrun, one process per GPU): the rows of the same matrix are partitioned in
contiguous blocks and solved with NCCL halo exchange + allreduces (strong scaling);
the time is the max over ranks.  --impl reference times the CPU oracle (oracle/) on a
bounded sample (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import generators as G  # noqa: E402

CFG = {"C2": dict(build=lambda rows=None: G.convection_diffusion(128, 3, 7, rows=rows), n=128 ** 3,
                  s=10, m=30, basis="newton", tsqr="cholqr", reorth=False,
                  workload="C2: 3D convection-diffusion 7-pt 128^3 (n=2,097,152), s=10, m=30, Newton, CholQR"),
       "C3": dict(build=lambda rows=None: G.g3_shaped(rows=rows), n=1585478, s=5, m=60, basis="newton",
                  tsqr="cholqr", reorth=False,
                  workload="C3: G3_circuit-shaped (n=1,585,478), s=5, m=60, Newton, CholQR"),
       "C1": dict(build=lambda rows=None: G.convection_diffusion(32, 2, 5, rows=rows), n=1024, s=5, m=30,
                  basis="newton", tsqr="cholqr", reorth=False,
                  workload="C1: 2D convection-diffusion 5-pt 32^2 (n=1024), s=5, m=30, Newton, CholQR"),
       # the metric's large configuration (BASELINE.json configs[4]); fits one B200 (A 21 GB CSR,
       # V 16 GB); built by the sort-free stencil generator (identical CSR, tests/test_inputs.py)
       "C5": dict(build=lambda rows=None: G.convection_diffusion_stream(400, 3, 27, rows=rows), n=400 ** 3,
                  s=10, m=30, basis="newton", tsqr="cholqr", reorth=False,
                  workload="C5: 3D convection-diffusion 27-pt 400^3 (n=64,000,000), s=10, m=30, Newton, CholQR")}
TOL = 1e-8
METRIC = "CA-GMRES time-to-solution (rel. residual 1e-8)"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class Clocks:
    """SM clock / throttle-reason sampler running during the timed region: NVML from a thread
    every 10 ms (starts at once, so even a short timed region gets samples); nvidia-smi -lms 100
    as the fallback."""

    NAMES = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20, "sw_power_cap": 0x4}

    def __init__(self, idx):
        self.idx = idx
        self.path = os.path.join("/tmp", f"clocks_{os.getpid()}.csv")
        self.p = None
        self.th = None
        self.samples = []

    def _nvml_loop(self, nv, hnd):
        while not self.stop.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(hnd, nv.NVML_CLOCK_SM)
                mx = nv.nvmlDeviceGetMaxClockInfo(hnd, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(hnd)
                self.samples.append((float(sm), float(mx), int(rs)))
            except Exception:
                pass
            self.stop.wait(0.01)

    def __enter__(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            hnd = nv.nvmlDeviceGetHandleByIndex(self.idx)
            self.stop = threading.Event()
            self.th = threading.Thread(target=self._nvml_loop, args=(nv, hnd), daemon=True)
            self.th.start()
            return self
        except Exception:
            self.th = None
        try:
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "100"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        if self.th is not None:
            self.stop.set()
            self.th.join(timeout=5)
        if self.p is not None:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()
            self.f.close()

    def summary(self):
        sm, mx, reasons = [], [], set()
        if self.th is not None:
            for a, b, r in self.samples:
                sm.append(a); mx.append(b)
                for nm, bit in self.NAMES.items():
                    if r & bit:
                        reasons.add(nm)
            src = "nvml"
        else:
            if self.p is None or not os.path.exists(self.path):
                return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
            names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
            for line in open(self.path):
                parts = [x.strip() for x in line.split(",")]
                if len(parts) < 7:
                    continue
                try:
                    sm.append(float(parts[0])); mx.append(float(parts[1]))
                except ValueError:
                    continue
                for nm, v in zip(names, parts[3:7]):
                    if v.lower().startswith("active"):
                        reasons.add(nm)
            src = "nvidia-smi"
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": float(max(mx)), "reasons": sorted(reasons),
                "samples": len(sm), "source": src}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    lrank = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, lrank


def ghost_rows(cfg, row_starts, rank, s):
    """Rows this rank needs: owned rows plus every row within s-1 hops.  For the
    naturally ordered configs a contiguous band suffices; found by BFS on generated rows."""
    n = cfg["n"]
    lo, hi = int(row_starts[rank]), int(row_starts[rank + 1])
    A = cfg["build"]((lo, hi))
    rows = np.repeat(np.arange(lo, hi), np.diff(A.rowptr))
    bw = int(np.abs(A.colind.astype(np.int64) - rows).max()) if A.nnz else 0
    clo, chi = max(0, lo - (s - 1) * bw), min(n, hi + (s - 1) * bw)
    return cfg["build"]((clo, chi))


def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_yamazakiathd14_b200 import _lib as L
    from paper_conf_ipps_yamazakiathd14_b200.solver import Solver

    ws, rank, lrank = dist_env()
    torch.cuda.set_device(lrank)
    # one ordinary (non-default) stream for everything: the solver binds torch's current stream,
    # so the copies of b / x and the flush are ordered with its kernels, and programmatic
    # dependent launch applies (it is not used on the legacy default stream)
    torch.cuda.set_stream(torch.cuda.Stream())
    group = None
    cfg = CFG[args.config]
    if ws > 1:
        if torch.cuda.device_count() < ws:
            raise RuntimeError(f"{ws} ranks but only {torch.cuda.device_count()} CUDA devices on this node")
        dist.init_process_group("nccl", device_id=torch.device("cuda", lrank))
        group = dist.group.WORLD
        if dist.get_world_size() != args.gpus:
            raise RuntimeError(f"NCCL world has {dist.get_world_size()} ranks, --gpus {args.gpus}")
    t0 = time.time()
    if ws == 1:
        A = cfg["build"]()
        print(f"[bench] A built: n={A.n} nnz={A.nnz} ({time.time() - t0:.1f} s)", file=sys.stderr, flush=True)
        S = Solver(A, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"] or args.reorth,
                   onepass=args.onepass)
        b_host = G.rhs(cfg["n"])
    elif args.order == "natural":
        rs = np.array([(p * cfg["n"]) // ws for p in range(ws + 1)], dtype=np.int64)
        A = ghost_rows(cfg, rs, rank, cfg["s"])
        S = Solver(A, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"] or args.reorth,
                   group=group, row_starts=rs, onepass=args.onepass)
        b_host = G.rhs(cfg["n"], rows=(rs[rank], rs[rank + 1]))
    else:
        # NEXT-4 row distribution: every rank builds the same permutation of the whole
        # matrix (k-way partition or RCM, host library, deterministic) and owns a block of B = P A P^T
        from paper_conf_ipps_yamazakiathd14_b200 import host
        A, perm, rs = host.distribute(cfg["build"](), ws, args.order)
        S = Solver(A, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"] or args.reorth,
                   group=group, row_starts=rs, onepass=args.onepass)
        b_host = G.rhs(cfg["n"])[perm][rs[rank]:rs[rank + 1]]
    for kv in args.opt:
        k_, v_ = kv.split("=")
        S.set_option(k_, int(v_))
    setup_s = time.time() - t0
    print(f"[bench] setup done ({setup_s:.1f} s)", file=sys.stderr, flush=True)
    stream = torch.cuda.current_stream()
    b = torch.tensor(b_host, device="cuda")
    x = torch.zeros_like(b)
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")   # 256 MB > L2

    def one(timing):
        # every timed solve is a complete one: the Newton shifts of a previous solve are
        # forgotten, so each solve runs its own first GMRES cycle — host flag, no GPU work
        x.zero_()
        S.clear_shifts()
        return S.solve(b, x, tol=TOL, maxit=200, timing=timing)

    for _ in range(args.warmup):
        one(False)
    # ---- timed region: device events on the solver's stream, barrier + sync both sides ----
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    stats = []
    l0 = l1 = None
    with Clocks(lrank) as clk:
        for k in range(args.steps):
            flush.fill_(float(k))
            if group is not None:
                dist.barrier()
            torch.cuda.synchronize()
            if l0 is None:
                l0 = L.load().cagmres_kernel_launches()
            ev[k][0].record(stream)
            _, st = one(0)
            ev[k][1].record(stream)
            torch.cuda.synchronize()
            l1 = L.load().cagmres_kernel_launches()      # after the last timed solve
            stats.append(st)
        # ---- kernel roofline pass: the same solves with CUDA events around every MPK SpMV
        # launch (on the solver's stream); these solves are not part of `value` ----
        kstats = []
        for k in range(args.steps):
            flush.fill_(float(k))
            torch.cuda.synchronize()
            _, st = one(2)
            kstats.append(st)
    launches_total = l1 - l0                         # all K timed solves
    ms = np.array([e[0].elapsed_time(e[1]) for e in ev])
    ms_step = float(ms.mean())
    if group is not None:
        t = torch.tensor([ms_step], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_step = float(t.item())
    st0 = kstats[-1]
    _, stp = one(1)                            # untimed: per-phase breakdown (all phases evented)
    # ---- dominant kernel (MPK SpMV) roofline, measured live inside the timed region ----
    spmv_ms = np.mean([s.ms["spmv"] / max(s.spmv_launches, 1) for s in kstats])
    spmv_bytes = st0.bytes["spmv"] / max(st0.spmv_launches, 1)
    peak, peak_kind = peaks()
    achieved = spmv_bytes / (spmv_ms * 1e-3) / 1e9
    phase = {k: float(stp.ms[k]) for k in ("mpk", "borth", "tsqr", "other", "total")}
    phase_gbs = {k: (stp.bytes[k] / (phase[k] * 1e-3) / 1e9 if phase[k] > 0 else None)
                 for k in ("mpk", "borth", "tsqr", "other")}
    traffic = None
    tf = os.path.join(ROOT, "profiles", "spmv_traffic.json")
    if os.path.exists(tf):
        with open(tf) as f:
            traffic = json.load(f).get(args.config)
    # ---- e2e: host b (pinned) -> device, solve via the C ABI, x -> host, all timed ----
    b_pin = torch.tensor(b_host).pin_memory()
    x_pin = torch.empty_like(b_pin).pin_memory()
    for _ in range(2):                               # e2e warm-up (first pinned transfers)
        S.clear_shifts()
        bd = b_pin.to("cuda", non_blocking=True)
        S.solve(bd, torch.zeros_like(bd), tol=TOL, maxit=200)
        x_pin.copy_(bd, non_blocking=True)
    torch.cuda.synchronize()
    e2e_ms, e2e_cycles = [], []
    for k in range(args.steps):
        flush.fill_(float(k))
        if group is not None:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        S.clear_shifts()
        bd = b_pin.to("cuda", non_blocking=True)
        xd = torch.zeros_like(bd)
        _, st_e = S.solve(bd, xd, tol=TOL, maxit=200)
        x_pin.copy_(xd, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))
        e2e_cycles.append(st_e.cycles)
    e2e = float(np.median(e2e_ms))          # median: robust to a rare host-side stall (each_ms kept)
    if group is not None:
        t = torch.tensor([e2e], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e = float(t.item())
    # ---- comparators on the same GPU kernels, timed like `value` (not part of it) ----
    def time_other(S2, maxit):
        x2 = torch.zeros_like(b)
        S2.clear_shifts()
        S2.solve(b, x2, tol=TOL, maxit=maxit)
        o_ms, o_st = [], None
        for k in range(max(1, min(args.steps, 3))):
            flush.fill_(float(k))
            if group is not None:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            x2.zero_()
            S2.clear_shifts()
            e0.record(stream)
            _, o_st = S2.solve(b, x2, tol=TOL, maxit=maxit)
            e1.record(stream)
            torch.cuda.synchronize()
            o_ms.append(e0.elapsed_time(e1))
        v = float(np.mean(o_ms))
        if group is not None:
            t = torch.tensor([v], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            v = float(t.item())
        S2.close()
        return v, o_st

    kw = {} if ws == 1 else dict(group=group, row_starts=rs)
    gm = None
    if not args.no_gmres:      # the paper's comparator (Fig. 14/15): standard GMRES(m)
        gv, g_st = time_other(Solver(A, 1, cfg["m"], basis="gmres", tsqr="cholqr", reorth=False, **kw), 400)
        gm = {"value": round(gv, 4), "unit": "ms", "cycles": int(g_st.cycles),
              "method": f"GMRES({cfg['m']}) with CGS, one SpMV + CGS pass per iteration (basis='gmres')",
              "ca_speedup": round(gv / ms_step, 3)}
    op = None
    if not args.no_gmres and not args.onepass:   # SURVEY NEXT-2 variant of the same solve
        ov, o_st = time_other(Solver(A, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"],
                                     reorth=cfg["reorth"] or args.reorth, onepass=True, **kw), 200)
        op = {"value": round(ov, 4), "unit": "ms", "cycles": int(o_st.cycles),
              "method": "one-pass BOrth+CholQR (CAGMRES_ONEPASS: [Q P]^T P, Pythagorean Gram, (P-QC)R^-1 in one pass)"}
    clocks = clk.summary()
    out = None
    if rank == 0:
        cpu = cpu_baseline(cfg, stats[-1].cycles, ws) if (ws == 1 and not args.no_cpu) else None
        out = {
            "metric": METRIC, "value": round(ms_step, 4), "unit": "ms", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 4),
            "higher_is_better": False, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg["workload"], "n": cfg["n"], "s": cfg["s"], "m": cfg["m"],
                       "tol": TOL, "cycles": stats[-1].cycles, "parallelism": f"rows{ws}",
                       "row_order": args.order if ws > 1 else "natural",
                       "l2": f"inputs larger than L2 (A {12 * A.nnz / 1e6:.0f} MB as CSR, V {8 * S.ldv * (cfg['m'] + 1) / 1e6:.0f} MB)"
                             " + 256 MB flush between steps",
                       "setup_s": round(setup_s, 2), "options": args.opt,
                       "orth": ("CholQR" + ("2 (reorth)" if (cfg["reorth"] or args.reorth) else "")
                                + (", one-pass BOrth+CholQR (NEXT-2)" if args.onepass else ", BOrth CGS")),
                       "kernels": {k_: S.get_option(k_) for k_ in ("spmv", "gram", "fuse", "mpk_wave", "graph")}},
            "e2e": {"value": round(e2e, 4), "unit": "ms", "stat": "median of K", "h2d_bytes_per_step": 8 * len(b_host),
                    "d2h_bytes_per_step": 8 * len(b_host), "each_ms": [round(v, 3) for v in e2e_ms],
                    "cycles": sorted(set(e2e_cycles))},
            "value_each_ms": [round(float(v), 3) for v in ms],
            "gpu_launches": int(launches_total),
            "gpu_launches_per_step": round(launches_total / args.steps, 1),
            "roofline": {"bound": "hbm", "kernel": f"SELL-32 SpMV (MPK step), CAGMRES_OPT_SPMV variant {S.get_option('spmv')}",
                         "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "dram_gbs": round(traffic / (spmv_ms * 1e-3) / 1e9, 1) if traffic else None,
                         "dram_frac": round(traffic / (spmv_ms * 1e-3) / 1e9 / peak, 4) if traffic else None,
                         "note": "achieved/frac use the paper's CSR byte model (12 B/nnz + vectors); the "
                                 "DIA-compressed SELL format moves fewer bytes (traffic = ncu DRAM bytes per "
                                 "launch), so frac can exceed 1; dram_frac = real DRAM bytes / time / peak",
                         "peak_source": peak_kind, "bytes_per_launch": spmv_bytes,
                         "avg_launch_us": round(spmv_ms * 1e3, 2), "launches_per_step": st0.spmv_launches,
                         "timing": "CUDA events around every SpMV launch on the solver stream, "
                                   "in K extra solves of the same workload after the timed ones"},
            "phases_ms": {k: round(v, 3) for k, v in phase.items()},
            "phases_note": "one extra untimed solve with CUDA events around every phase",
            "phases_gbs": {k: (round(v, 1) if v else None) for k, v in phase_gbs.items()},
            "gmres_baseline": gm,
            "onepass_variant": op,
            "clocks": clocks,
            "cpu_baseline": cpu,
        }
        print(json.dumps(out), flush=True)
    S.close()
    if group is not None:
        dist.barrier()
        dist.destroy_process_group()
    return out


def _cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


def cpu_baseline(cfg, gpu_cycles, ws):
    """The oracle as it stands, on this host's cores, on a bounded sample: 2 restart cycles of
    the same workload (cycle 1 = GMRES(m) shift cycle, cycle 2 = CA), time per cycle
    extrapolated to the GPU-measured cycle count."""
    from oracle import cagmres_oracle as O
    A = cfg["build"]().to_scipy()
    b = G.rhs(cfg["n"])
    t0 = time.perf_counter()
    r1 = O.cagmres(A, b, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"],
                   tol=TOL, maxcyc=1)                     # cycle 1: GMRES(m), finds the shifts
    t1 = time.perf_counter() - t0
    t0 = time.perf_counter()
    O.cagmres(A, b, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"],
              tol=0.0, maxcyc=1, shifts=r1["shifts"])     # one CA cycle
    t2 = time.perf_counter() - t0
    dt = t1 + t2
    threads = _cores()
    try:
        from threadpoolctl import threadpool_info
        threads = max([i.get("num_threads", 1) for i in threadpool_info()] + [1])
    except Exception:
        pass
    return {"value": round((t1 + t2 * max(gpu_cycles - 1, 0)) * 1e3, 1), "unit": "ms", "cores": threads,
            "kind": "oracle",
            "sample": f"2 restart cycles of {cfg['workload']} on the host (NumPy/SciPy fp64): the GMRES "
                      f"shift cycle ({t1:.2f} s) + one CA cycle ({t2:.2f} s) x {gpu_cycles - 1} "
                      f"(GPU cycle count - 1), extrapolated"}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return None
    from oracle import cagmres_oracle as O
    cfg = CFG[args.config]
    A = cfg["build"]().to_scipy()
    b = G.rhs(cfg["n"])
    # warm-up steps also establish the oracle's own cycle count to tolerance (one full solve)
    t0 = time.perf_counter()
    full = O.cagmres(A, b, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"],
                     tol=TOL, maxcyc=200)
    t_full = time.perf_counter() - t0
    cycles = full["cycles"]
    re, im = full["shifts"]
    t0 = time.perf_counter()                    # the solve's first cycle: GMRES(m) finding the shifts
    O.cagmres(A, b, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"],
              tol=0.0, maxcyc=1)
    t_first = time.perf_counter() - t0
    times = []
    for k in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        O.cagmres(A, b, cfg["s"], cfg["m"], basis=cfg["basis"], tsqr=cfg["tsqr"], reorth=cfg["reorth"],
                  tol=0.0, maxcyc=1, shifts=(re, im))
        if k >= args.warmup:
            times.append(time.perf_counter() - t0)
    per = float(np.mean(times))
    val = (t_first + per * (cycles - 1)) * 1e3
    cores = _cores()
    out = {"metric": METRIC, "value": round(val, 1), "unit": "ms", "n_gpus": ws, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(per * 1e3, 1), "higher_is_better": False,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
           "config": {"workload": cfg["workload"], "n": cfg["n"], "s": cfg["s"], "m": cfg["m"], "tol": TOL,
                      "cycles": cycles, "full_oracle_solve_s": round(t_full, 2)},
           "cpu_baseline": {"value": round(val, 1), "unit": "ms", "cores": cores, "kind": "oracle",
                            "sample": f"each step = 1 CA restart cycle (shifts from the oracle's own "
                                      f"first cycle); value = first (GMRES) cycle {t_first:.2f} s + mean "
                                      f"CA cycle time x {cycles - 1} cycles"},
           "e2e": {"value": round(val, 1), "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return out


def _free_port():
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    return port


def launch_ranks(args):
    """--gpus N without a torchrun environment: re-launch this script as N ranks (one process
    per GPU) under torch.distributed.run.  Refuses (exit 2, one JSON line) when this node has
    fewer than N GPUs — never a silent 1-GPU number for an N-GPU request."""
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        print(json.dumps({"metric": METRIC, "error": f"--gpus {args.gpus} requested but this node has {have} "
                                                     f"CUDA device(s)", "n_gpus": args.gpus}), flush=True)
        sys.exit(2)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2", choices=sorted(CFG))
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-gmres", action="store_true", help="skip the GPU GMRES(m) comparator")
    ap.add_argument("--reorth", action="store_true", help="2x BOrth+TSQR (CholQR2)")
    ap.add_argument("--onepass", action="store_true", help="one-pass BOrth+CholQR (CAGMRES_ONEPASS, NEXT-2)")
    ap.add_argument("--order", default="natural", choices=["natural", "rcm", "kway"],
                    help="row distribution for --gpus N > 1 (NEXT-4): natural block rows, RCM, or the "
                         "library's k-way partition made contiguous")
    ap.add_argument("--opt", action="append", default=[],
                    help="solver option NAME=VALUE (CAGMRES_OPT_*: spmv, gram, fuse, mpk_wave, ...); "
                         "default: the library's defaults")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    ws, _, _ = dist_env()
    if "WORLD_SIZE" in os.environ and ws != args.gpus:
        print(json.dumps({"metric": METRIC, "error": f"--gpus {args.gpus} but WORLD_SIZE={ws}"}), flush=True)
        sys.exit(2)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        launch_ranks(args)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
