"""Multi-process CPU test (gloo) of the multi-GPU setup path: each rank builds the library's
host plan (boundary sets P:60-64, extended numbering, halo request lists), the ranks exchange
requests over torch.distributed (the role NCCL plays in cagmres_create_dist), and then run
the matrix powers kernel on the extended rows exactly as the device does — one halo
exchange of the start vector limited to depth sb, then sb prefix SpMVs — in NumPy.  Ghost
rows deeper than sb are poisoned with NaN to prove the prefix schedule never reads them.
The owned rows must equal the oracle's global MPK (Fig. 4)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, gen, s, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import cagmres_oracle as O
        from paper_conf_ipps_yamazakiathd14_b200.host import Plan
        from synth import generators as G
        build = {"cd7": lambda rows=None: G.convection_diffusion(12, 3, 7, rows=rows),
                 "g3": lambda rows=None: G.g3_shaped(n=6000, width=80, rows=rows),
                 "band": lambda rows=None: G.banded(n=3001, rows=rows)}[gen]
        full = build()
        n = full.n
        rs = O.block_rows(n, world)
        lo, hi = rs[rank], rs[rank + 1]
        # rows within s-1 hops (superset: the whole matrix for g3's long-range edges)
        Aloc = full if gen == "g3" else build((max(0, lo - s * 200), min(n, hi + s * 200)))
        plan = Plan(Aloc, rs, rank, s)
        cnt, gids, lvls, ext = plan.requests()
        allreq = [None] * world
        dist.all_gather_object(allreq, (cnt.tolist(), gids.tolist(), lvls.tolist()))
        inc = [allreq[p][0][rank] for p in range(world)]
        g_in, l_in = [], []
        for p in range(world):
            c, g, lv = allreq[p]
            off = sum(c[:rank])
            g_in += g[off:off + c[rank]]
            l_in += lv[off:off + c[rank]]
        plan.set_sends(np.array(inc), np.array(g_in, dtype=np.int64), np.array(l_in, dtype=np.int32))
        sidx = plan.send_index()
        qv = G.u(99, np.arange(n))
        rp, ci, va = plan.ext_csr()
        ll = plan.level_len
        re_ = np.array([0.7, 2.0, 2.0, 0.3, 5.0, 1.0])
        im_ = np.array([0.0, 0.6, -0.6, 0.0, 0.0, 0.0])
        As = full.to_scipy()
        for sb in range(1, s + 1):
            # halo exchange of depth sb (prefix of each (level-sorted) send list)
            qloc = qv[lo:hi]
            send = {}
            off = 0
            for p in range(world):
                lv = np.array(l_in[off:off + inc[p]], dtype=np.int32)
                k = int((lv <= sb).sum())
                assert np.all(lv[:k] <= sb) and np.all(lv[k:] > sb)       # level-sorted
                send[p] = qloc[sidx[off:off + k]]
                off += inc[p]
            got = [None] * world
            dist.all_gather_object(got, send)
            z = np.full(plan.n_ext, np.nan)
            z[:plan.n_loc] = qloc
            roff = 0
            for p in range(world):
                vals = got[p][rank]
                z[ext[roff:roff + len(vals)]] = vals
                roff += cnt[p]
            assert not np.any(np.isnan(z[:ll[sb]]))
            W = [z]
            steps = O.block_shifts(re_, im_, sb)
            for k, (a, b2, kind) in enumerate(steps, start=1):
                rows = ll[sb - k]
                y = np.full(plan.n_ext, np.nan)
                for r in range(rows):
                    acc = 0.0
                    for e in range(rp[r], rp[r + 1]):
                        acc += va[e] * W[-1][ci[e]]
                    y[r] = acc - a * W[-1][r] + (b2 * W[-2][r] if kind == "p2" else 0.0)
                W.append(y)
            ref = O.mpk(As, qv, sb, re_, im_)
            for k in range(sb + 1):
                got_k = W[k][:plan.n_loc]
                assert np.all(np.isfinite(got_k))
                assert np.allclose(got_k, ref[lo:hi, k], rtol=1e-12, atol=1e-12 * np.abs(ref[:, k]).max())
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("gen,world,s", [("cd7", 2, 3), ("g3", 3, 3), ("band", 2, 4)])
def test_distributed_plan_and_halo_mpk_gloo(gen, world, s):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, gen, s, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert res[r] == "ok", res[r]
