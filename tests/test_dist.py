"""Outer-axis decomposition (DESIGN.md a10): host geometry on CPU and a
world_size-2 gloo run of the halo-exchange protocol the library's NCCL path follows.

The slab geometry comes from the C ABI's host plan builder (fftstencil_describe_dist);
the exchange moves exactly the rows the library sends (top r*T owned rows to rank-1,
bottom r*T owned rows to rank+1); each pass is modelled by direct steps on the rank's
slab + halo buffer (the oracle), which is exact on the owned rows because a halo of
r*T rows covers the dependency cone of t <= T steps.  The gathered result must equal the
undecomposed oracle bitwise.
"""
import os
import socket

import numpy as np
import pytest

import oracle
from synth import workloads as wl

fs = pytest.importorskip("paper_conf_ppopp_hanlcbzyczcy25_b200")


def geometry(ext, w, r, T, n):
    return [fs.describe_dist(ext, w, r, T, n, k) for k in range(n)]


@pytest.mark.parametrize("ext,shape,r,T,n", [((10240, 10240), "box", 1, 8, 8), ((300, 170), "star", 1, 4, 3),
                                             ((513,), "star", 2, 3, 4), ((60, 40, 50), "box", 1, 2, 2),
                                             ((400, 97), "star", 3, 2, 5), ((40960, 640), "box", 1, 16, 8)])
def test_slabs_partition_rows_and_pairs(ext, shape, r, T, n):
    w = wl.seeded_weights(shape, len(ext), r)
    gs = geometry(ext, w, r, T, n)
    single = fs.describe(ext, w, r, T)
    h = single["halo"]
    assert gs[0]["row_begin"] == 0 and gs[-1]["row_end"] == ext[0]
    for a, b in zip(gs, gs[1:]):
        assert a["row_end"] == b["row_begin"]
        assert a["pair_end"] == b["pair_begin"]
    assert gs[0]["pair_begin"] == 0 and gs[-1]["pair_end"] == single["pairs"]
    for k, g in enumerate(gs):
        assert g["nranks"] == n and g["rank"] == k
        assert g["row_end"] - g["row_begin"] >= h
        assert g["pair_begin"] <= g["interior_begin"] <= g["interior_end"] <= g["pair_end"]
        assert g["ghost_lo"] == (0 if k == 0 else h)
        assert g["ghost_hi"] == (0 if k == n - 1 else h)
        assert g["T"] == single["T"] and g["tile"] == single["tile"]
    # balance: whole tile rows per rank, at most one unit apart
    nunits = single["pairs"] if len(ext) == 1 else -(-(ext[0] - 2 * h) // single["valid"][0])
    ppu = single["pairs"] // nunits
    per = [g["pair_end"] - g["pair_begin"] for g in gs]
    assert all(p % ppu == 0 for p in per)
    assert max(per) - min(per) <= ppu


def test_too_many_ranks_rejected():
    w = wl.seeded_weights("box", 2, 1)
    with pytest.raises(fs.FftStencilError):
        fs.describe_dist((40, 40), w, 1, 8, 8, 0)
    with pytest.raises(fs.FftStencilError):
        fs.describe_dist((400, 40), w, 1, 8, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, case, q):
    import torch.distributed as dist
    import torch
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        ext, shape, r, T, steps = case
        nd = len(ext)
        w = wl.seeded_weights(shape, nd, r)
        u = wl.grid(ext, 31)
        g = fs.describe_dist(ext, w, r, T, world, rank)
        h, Tp = g["halo"], g["T"]
        s, e = g["row_begin"], g["row_end"]
        g0, g1 = s - g["ghost_lo"], e + g["ghost_hi"]
        buf = u[g0:g1].copy()                       # slab + halos (halos refreshed per pass)
        done = 0
        while done < steps:
            t = min(Tp, steps - done)
            # ---- the library's exchange: top h owned rows -> rank-1, bottom h -> rank+1 ----
            reqs = []
            own = buf[s - g0:e - g0]
            if rank > 0:
                reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(own[:h])), rank - 1))
                top = torch.empty((s - g0,) + own.shape[1:], dtype=torch.float64)
                reqs.append(dist.irecv(top, rank - 1))
            if rank < world - 1:
                reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(own[-h:])), rank + 1))
                bot = torch.empty((g1 - e,) + own.shape[1:], dtype=torch.float64)
                reqs.append(dist.irecv(bot, rank + 1))
            for rq in reqs:
                rq.wait()
            if rank > 0:
                buf[:s - g0] = top.numpy()
            if rank < world - 1:
                buf[e - g0:] = bot.numpy()
            # ---- one pass of t steps; exact on the owned rows (cone within the halo) ----
            nxt = oracle.stencil_run(buf, w, r, t)
            # global ring rows stay fixed: the buffer's own edge rows are ring only at the grid edge
            buf[s - g0:e - g0] = nxt[s - g0:e - g0]
            done += t
        owned = torch.from_numpy(np.ascontiguousarray(buf[s - g0:e - g0]))
        sizes = [None] * world
        dist.all_gather_object(sizes, (s, e))
        if rank == 0:
            parts = [owned]
            for k in range(1, world):
                sk, ek = sizes[k]
                t_ = torch.empty((ek - sk,) + tuple(ext[1:]), dtype=torch.float64)
                dist.recv(t_, k)
                parts.append(t_)
            full = torch.cat(parts).numpy()
            ref = oracle.stencil_run(u, w, r, steps)
            q.put(("ok", bool(np.array_equal(full, ref)), float(np.abs(full - ref).max())))
        else:
            dist.send(owned, 0)
    except Exception as ex:  # pragma: no cover - surfaced through the queue
        q.put(("err", repr(ex), 0.0))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", [((90, 37), "box", 1, 4, 11), ((200,), "star", 2, 3, 10),
                                  ((41, 20, 18), "star", 1, 2, 5), ((120, 60), "star", 3, 2, 7)])
def test_gloo_two_rank_halo_protocol(case):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, 2, port, case, q)) for k in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=120)
    assert res[0] == "ok", res
    assert res[1], f"decomposed result differs from the oracle (max abs {res[2]})"
    assert all(p.exitcode == 0 for p in procs)
