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


# ---------------------------------------------------------------- peer transport protocol replay
def _peer_replay(ext, shape, r, T, n, runs, fused, seed):
    """Replays the op lists the library executes for a peer-transport group (fftstencil_peer_schedule,
    the same list capi.cu run_dist_peer runs) under one random interleaving of the ranks' streams
    (a stream blocks only at WAIT).  Row versions are tracked per rank, buffer and outer row:
    every read must see the previous pass's data (so a neighbour's write that lands before the read
    it must follow -- a race -- shows up as a wrong version), halo rows must carry the fixed-ring
    cells (a full-row copy has landed), and the copy-out must see the last pass."""
    rng = np.random.default_rng(seed)
    w = wl.seeded_weights(shape, len(ext), r)
    geo = [fs.describe_dist(ext, w, r, T, n, k) for k in range(n)]
    h, n0 = geo[0]["halo"], ext[0]
    lo = [g["row_begin"] for g in geo]
    hi = [g["row_end"] for g in geo]
    g0 = [max(0, lo[k] - h) if k > 0 else 0 for k in range(n)]
    g1 = [min(n0, hi[k] + h) if k < n - 1 else n0 for k in range(n)]
    ver = np.full((n, 2, n0), -1)      # version = run * 10^6 + pass (0 = the run's input)
    ring = np.zeros((n, 2, n0), bool)  # full rows (with their fixed-ring cells) in place
    sig = [0] * n
    progs, epoch = [], [0] * n
    plan_T = geo[0]["T"]
    for k in range(n):
        ops, e = [], 0
        for ri, steps in enumerate(runs):
            sch = fs.peer_schedule(ext, w, r, T, n, k, steps, fused, e)
            ops += [(ri, tuple(int(x) for x in op)) for op in sch]
            e = max([e] + [int(op[1]) for op in sch if op[0] == 3])
        progs.append(ops)
    pc = [0] * n
    nbrs = lambda k: [q for q in (k - 1, k + 1) if 0 <= q < n]  # noqa: E731
    bnd = lambda k: (np.arange(lo[k], lo[k] + h), np.arange(hi[k] - h, hi[k]))  # noqa: E731
    while True:
        live = [k for k in range(n) if pc[k] < len(progs[k])]
        if not live:
            break
        ready = [k for k in live if progs[k][pc[k]][1][0] != 0 or all(sig[q] >= progs[k][pc[k]][1][1] for q in nbrs(k))]
        assert ready, f"deadlock: {[progs[k][pc[k]] for k in live]}"
        k = int(rng.choice(ready))
        ri, (op, a, b, c) = progs[k][pc[k]]
        pc[k] += 1
        base = ri * 10**6
        P = -(-runs[ri] // plan_T)
        if op == 1:        # COPYIN: input into buffer 0, fixed ring into buffer 1 (owned rows)
            ver[k, 0, lo[k]:hi[k]] = base
            ring[k, :, lo[k]:hi[k]] = True
        elif op == 2:      # PUSH a -> b: own boundary rows into the neighbours' halo rows
            for q in nbrs(k):
                rows = bnd(k)[0] if q < k else bnd(k)[1]
                ver[q, b, rows] = ver[k, a, rows]
                ring[q, b, rows] = True
        elif op == 3:
            sig[k] = a
        elif op == 4:      # INTERIOR: reads owned rows of b, writes [lo + h, hi - h) of b ^ 1
            assert (ver[k, b, lo[k]:hi[k]] == base + a - 1).all(), f"rank {k} pass {a}: interior read a stale row"
            ver[k, b ^ 1, lo[k] + h:hi[k] - h] = base + a
        elif op == 5:      # EDGE: reads [g0, g1) of b, writes the boundary rows (+ the neighbours')
            rows = slice(g0[k], g1[k])
            assert (ver[k, b, rows] == base + a - 1).all(), f"rank {k} pass {a}: edge read a stale / overwritten row"
            assert ring[k, b, rows].all(), f"rank {k} pass {a}: halo row without its fixed-ring cells"
            for side, rr in zip((0, 1), bnd(k)):
                ver[k, b ^ 1, rr] = base + a
                q = k - 1 if side == 0 else k + 1
                if c and 0 <= q < n:
                    ver[q, b ^ 1, rr] = base + a
        elif op == 6:      # COPYOUT
            assert (ver[k, a, lo[k]:hi[k]] == base + P).all(), f"rank {k} run {ri}: copy-out before the last pass"
    return progs


PEER_CASES = [((300, 170), "box", 1, 4, 3), ((257, 129), "star", 3, 2, 2), ((60, 40, 50), "box", 1, 2, 2),
              ((5000,), "star", 1, 8, 4), ((2048, 256), "box", 1, 0, 4), ((90, 30, 34), "star", 1, 3, 3)]


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("ext,shape,r,T,n", PEER_CASES)
def test_peer_schedule_replays_race_free(ext, shape, r, T, n, fused):
    """50 random interleavings of the ranks' streams, three chained runs (the second a single
    pass, the last with a remainder pass): every read sees exactly the previous pass."""
    Tp = fs.describe(ext, wl.seeded_weights(shape, len(ext), r), r, T)["T"]
    runs = (3 * Tp + 1, Tp, 2 * Tp)
    for seed in range(50):
        _peer_replay(ext, shape, r, T, n, runs, fused, seed)


def test_peer_replay_catches_a_missing_wait():
    """Mutation check: dropping the WAIT before a pass's edge work lets a rank read its halo rows
    before the neighbour's data for that pass arrived -- some interleaving must fail."""
    orig = fs.peer_schedule

    def no_edge_wait(*a, **k):
        ops = orig(*a, **k)
        keep = [i for i in range(len(ops)) if not (ops[i][0] == 0 and i + 1 < len(ops) and ops[i + 1][0] == 5)]
        return ops[keep]

    fs.peer_schedule = no_edge_wait
    try:
        failed = 0
        for seed in range(200):
            try:
                _peer_replay((300, 170), "box", 1, 4, 3, (13,), True, seed)
            except AssertionError:
                failed += 1
        assert failed > 0
    finally:
        fs.peer_schedule = orig


def test_peer_replay_catches_a_missing_ring_push():
    """Mutation check: without the begin-of-run push into buffer 1, fused stores leave buffer 1's
    halo rows without their fixed-ring cells."""
    orig = fs.peer_schedule

    def no_second_push(*a, **k):
        ops = orig(*a, **k)
        keep = [i for i in range(len(ops)) if not (ops[i][0] == 2 and ops[i][2] == 1 and ops[i][1] == 0)]
        return ops[keep]

    fs.peer_schedule = no_second_push
    try:
        with pytest.raises(AssertionError):
            _peer_replay((300, 170), "box", 1, 4, 2, (13,), True, 0)
    finally:
        fs.peer_schedule = orig
