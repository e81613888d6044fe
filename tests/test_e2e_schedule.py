"""CPU: the pipelined run_host schedule (plan.cpp build_e2e_schedule, exported as
fftstencil_e2e_schedule) replayed row by row against the data it must read.

Model: a pass writes each interior row once and reads the previous pass's
rows within h = r*T of it (the fused tile of unit u reads rows [uS, uS+L) = its output rows
+- h; band rows read their +- h cone).  Pass k reads `in` (k = 1) or buffer (k-2) % 2 and
writes buffer (k-1) % 2.  The replay checks that every read row holds exactly pass k-1's
version in the buffer read (an overwrite by pass k+1 before the read shows as k+1, so this
also checks the ping-pong anti-dependency), that ring rows are in place before use, that
copies-out see pass P, and that chunks and items partition rows and units exactly.
"""
import numpy as np
import pytest

import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs
from synth import workloads as wl


def replay(ext, shape, r, T, steps, K, Q, mutate=None, check_cover=True):
    w = wl.seeded_weights(shape, len(ext), r)
    info = fs.describe(ext, w, r, T)
    h, S, n0 = info["halo"], info["valid"][0], ext[0]
    U = -(-(n0 - 2 * h) // S)
    T_used = info["T"]
    P = steps // T_used + (1 if steps % T_used else 0)
    ops = fs.e2e_schedule(ext, w, r, T, steps, K, Q)
    if mutate is not None:
        ops = mutate(ops)
    row = lambda u: 0 if u <= 0 else (n0 if u >= U else u * S + h)  # noqa: E731
    in_ok = np.zeros(n0, bool)
    ring_ok = np.zeros((2, n0), bool)
    ver = np.full((2, n0), -1)
    out_buf = 0 if P % 2 else 1          # dsts[0] = out when P is odd
    h2d, d2h = np.zeros(n0, int), np.zeros(n0, int)
    cover = np.zeros((P + 1, U), int)
    # rows of the output buffer already queued for copy-out: the D2H runs asynchronously on the
    # copy stream while later items keep writing the same buffer, so none may touch them again
    frozen = np.zeros(n0, bool)
    for op, x, y, z in ops:
        if op == 0:
            h2d[x:y] += 1
            in_ok[x:y] = True
        elif op == 1:
            assert in_ok[x:y].all(), "ring rows copied before they arrived"
            ring_ok[:, x:y] = True
        elif op == 2:
            k, u0, u1 = x, y, z
            assert 1 <= k <= P and 0 <= u0 < u1 <= U
            cover[k, u0:u1] += 1
            src, dst = (k - 2) % 2, (k - 1) % 2
            lo, hi = row(u0), row(u1)
            rlo, rhi = max(0, lo - h), min(n0, hi + h)
            if k == 1:
                assert in_ok[rlo:rhi].all(), f"pass 1 units [{u0},{u1}) read rows not yet copied in"
            else:
                assert (ver[src, rlo:rhi] == k - 1).all(), \
                    f"pass {k} units [{u0},{u1}) read rows not holding pass {k - 1}"
                assert ring_ok[src, rlo:rhi].all()
            if dst == out_buf:
                assert not frozen[lo:hi].any(), f"pass {k} units [{u0},{u1}) write rows queued for copy-out"
            ver[dst, lo:hi] = k
        else:
            assert (ver[out_buf, x:y] == P).all(), "rows copied out before the last pass"
            assert ring_ok[out_buf, x:y].all()
            d2h[x:y] += 1
            frozen[x:y] = True
    assert (h2d == 1).all() and (d2h == 1).all()
    if check_cover:
        assert (cover[1:] == 1).all(), "every pass must produce every unit exactly once"
    return ops, U, P


CASES = [
    # extents, shape, r, T, steps, K, Q
    ((10240, 10240), "star", 1, 11, 1000, 6, 16),   # the bench line's schedule
    ((10240, 10240), "star", 1, 11, 1000, 16, 20),
    ((10240, 10240), "box", 3, 4, 1000, 6, 16),     # Box-2D49P (h = 12, S = 40)
    ((1024, 64, 64), "star", 1, 2, 100, 6, 16),     # 3D (h = 2, S = 12)
    ((1500, 200), "star", 1, 11, 100, 16, 16),      # P = 10 < Q
    ((800, 150), "box", 1, 4, 103, 4, 3),           # P > 2Q, remainder pass
    ((700, 130), "box", 3, 4, 50, 4, 2),
    ((420, 36, 40), "star", 1, 2, 9, 16, 16),
    ((200, 30, 33), "box", 1, 2, 12, 2, 1),         # K = 2, Q = 1
    ((600, 97), "star", 1, 8, 1, 2, 4),             # one pass
    ((2000, 64), "star", 1, 8, 8 * 40, 12, 12),     # P = 40 passes, no remainder
]


@pytest.mark.parametrize("ext,shape,r,T,steps,K,Q", CASES)
def test_schedule_replays(ext, shape, r, T, steps, K, Q):
    ops, U, P = replay(ext, shape, r, T, steps, K, Q)
    n_items = int((ops[:, 0] == 2).sum())
    assert n_items >= P                 # at least one item per pass
    # at most K + 2 input and K + 2 output pieces (plan.cpp: ramp 1 splits the first input and
    # the last output chunk 1/4 + 3/4, ramp 2 also the last input and the first output chunk)
    assert n_items <= P + 2 * (K + 2) * min(Q, P)


def test_head_overlaps_copies():
    """The first Q passes start before the input has fully arrived, and the first result
    chunk is copied out before the last pass is done."""
    ops, U, P = replay((10240, 10240), "star", 1, 11, 1000, 6, 16)
    kinds = list(ops[:, 0])
    last_h2d = max(i for i, k in enumerate(kinds) if k == 0)
    first_d2h = kinds.index(3)
    assert any(k == 2 for k in kinds[:last_h2d]), "no pass issued before the last input chunk"
    last_item = max(i for i, k in enumerate(kinds) if k == 2)
    assert first_d2h < last_item, "no copy-out before the last item"


@pytest.mark.parametrize("ext,shape,r,T,steps,K", [
    ((4096,), "star", 1, 8, 64, 6),          # 1D: not pipelined
    ((300, 120), "box", 1, 8, 20, 6),        # 6 outer tile rows < 2K
    ((1500, 200), "star", 1, 11, 0, 6),      # no steps
    ((1500, 200), "star", 1, 11, 100, 1),    # K < 2
])
def test_ineligible(ext, shape, r, T, steps, K):
    w = wl.seeded_weights(shape, len(ext), r)
    with pytest.raises(fs.FftStencilError):
        fs.e2e_schedule(ext, w, r, T, steps, K, 16)


def _swap_first(ops, pred):
    """Move the first op satisfying pred(prev, op) one slot earlier."""
    ops = ops.copy()
    for i in range(1, len(ops)):
        if pred(ops[i - 1], ops[i]):
            ops[[i - 1, i]] = ops[[i, i - 1]]
            return ops
    raise RuntimeError("no op to swap")


@pytest.mark.parametrize("pred", [
    lambda a, b: a[0] == 2 and b[0] == 2 and b[1] == a[1] + 1,   # pass k+1 before the pass-k item it needs
    lambda a, b: a[0] == 0 and b[0] == 1,                         # ring before its input chunk
    lambda a, b: a[0] == 2 and b[0] == 3,                         # copy-out before the last item
])
def test_replay_catches_reordering(pred):
    """The replay is not vacuous: moving one op before something it depends on fails it."""
    with pytest.raises(AssertionError):
        replay((1500, 200), "star", 1, 11, 100, 4, 6, mutate=lambda o: _swap_first(o, pred))


def test_replay_catches_item_before_its_input_chunk():
    def mutate(ops):
        ops = ops.copy()
        c2 = [i for i in range(len(ops)) if ops[i, 0] == 0][1]       # second input chunk
        it = next(i for i in range(c2, len(ops)) if ops[i, 0] == 2)  # first item after it
        return np.concatenate([ops[:c2], ops[it:it + 1], ops[c2:it], ops[it + 1:]])
    with pytest.raises(AssertionError):
        replay((1500, 200), "star", 1, 11, 100, 4, 6, mutate=mutate)


def test_replay_catches_write_after_copy_out():
    """A later item that rewrites rows already queued for copy-out (the D2H reads them
    asynchronously) fails the frozen-rows check even where every version check passes: here a
    pass-P item re-issued after the first copy-out on the units that copy covered."""
    def mutate(ops):
        i3 = next(i for i in range(len(ops)) if ops[i, 0] == 3)
        P = int(ops[ops[:, 0] == 2, 1].max())
        it = next(i for i in range(i3) if ops[i, 0] == 2 and ops[i, 1] == P)   # a pass-P item before it
        return np.concatenate([ops[:i3 + 1], ops[it:it + 1], ops[i3 + 1:]])
    replay((1500, 200), "star", 1, 11, 100, 4, 6, check_cover=False)          # the clean schedule passes
    with pytest.raises(AssertionError, match="queued for copy-out"):
        replay((1500, 200), "star", 1, 11, 100, 4, 6, mutate=mutate, check_cover=False)


@pytest.mark.parametrize("ramp,tail", [(1, None), (2, 24), (2, 3), (1, 30)])
@pytest.mark.parametrize("ext,shape,r,T,steps,K,Q", [CASES[0], CASES[3], CASES[5], CASES[8]])
def test_schedule_replays_ramp_and_tail_depth(monkeypatch, ramp, tail, ext, shape, r, T, steps, K, Q):
    """The schedule knobs the A/B runs use (FFTSTENCIL_E2E_RAMP, FFTSTENCIL_E2E_DEPTH_TAIL) keep
    every replay invariant."""
    monkeypatch.setenv("FFTSTENCIL_E2E_RAMP", str(ramp))
    if tail is not None:
        monkeypatch.setenv("FFTSTENCIL_E2E_DEPTH_TAIL", str(tail))
    replay(ext, shape, r, T, steps, K, Q)
