"""MPK surface-to-volume and halo-volume study (the quantities of the paper's Fig. 6/7,
P:98-118) for contiguous block-row partitions: natural vs RCM order vs
the library's k-way partition (cagmres_host_partition, parts made contiguous).
Host only (the setup plan of libcagmres.so, cagmres_plan_* / cagmres_host_rcm); no GPU.

For P ranks and depth s, rank d's MPK needs the ghost rows within s hops of its owned rows
(delta^(d,1:s)): halo words per block = n_ext - n_loc, and step k recomputes the
ghost rows within s - k hops: redundant SpMV rows = sum_{k=1..s} (L[s-k] - n_loc), where
L[h] = rows within h hops (level_len).  Reported as fractions of n_loc, max over ranks.

    python tools/surface_volume.py > profiles/r2_mpk_surface_volume.json
"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_yamazakiathd14_b200 import host  # noqa: E402
from synth import generators as G  # noqa: E402

S_MAX = 10


def study(A, P, rs=None):
    if rs is None:
        rs = np.array([(p * A.n) // P for p in range(P + 1)], dtype=np.int64)
    per = []
    for d in range(P):
        pl = host.Plan(A, rs, d, S_MAX)
        L = pl.level_len.astype(np.float64)
        nl = float(pl.n_loc)
        per.append({s: ((L[s] - nl) / nl, sum(L[s - k] - nl for k in range(1, s + 1)) / (s * nl))
                    for s in (1, 2, 3, 5, 10)})
    return {f"s={s}": {"halo_frac_max": round(max(p[s][0] for p in per), 5),
                       "redundant_spmv_frac_max": round(max(p[s][1] for p in per), 5)}
            for s in (1, 2, 3, 5, 10)}


def main():
    mats = {"C3 G3-shaped (n=1,585,478)": G.g3_shaped(),
            "C5-shaped 27-pt 100^3 (n=1,000,000)": G.convection_diffusion(100, 3, 27)}
    out = {}
    for name, A in mats.items():
        t0 = time.time()
        p = host.rcm(A)
        Ar = host.permute(A, p)
        t_rcm = time.time() - t0
        As = host.permute(A, np.argsort(G.u(99, np.arange(A.n))))       # arbitrary (scrambled) order
        Asr = host.permute(As, host.rcm(As))                            # ... then RCM
        for order, M in (("natural", A), ("rcm", Ar), ("scrambled", As), ("scrambled+rcm", Asr),
                         ("kway", A), ("scrambled+kway", As)):
            for P in (2, 4, 8):
                rs = None
                if order.endswith("kway"):
                    t0 = time.time()
                    M2, _, rs = host.distribute(M, P, "kway")
                    out[f"{name} | {order} | P={P} | partition_seconds"] = round(time.time() - t0, 2)
                else:
                    M2 = M
                out[f"{name} | {order} | P={P}"] = study(M2, P, rs)
                print(name, order, P, json.dumps(out[f"{name} | {order} | P={P}"]["s=10"]),
                      file=sys.stderr, flush=True)
        out[f"{name} | rcm_seconds"] = round(t_rcm, 2)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
