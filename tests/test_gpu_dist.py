"""GPU test of the outer-axis decomposition on one device (loopback transport).

NCCL refuses two ranks on one GPU, so the decomposition is exercised here with loopback
ranks (fftstencil_plan_create_dist with no NCCL id) run together by fftstencil_run_group,
whose halo exchange is a device copy of exactly the rows the NCCL path sends.  Because
slabs are whole tile rows and tile pairs never straddle them, the decomposed result must
equal the single-GPU result BITWISE, and the oracle within tolerance.
"""
import numpy as np
import pytest

import oracle
from synth import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def fs():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ppopp_hanlcbzyczcy25_b200 as mod
    return mod


CASES = [
    ((300, 170), "box", 1, 4, 11, 3),
    ((257, 129), "star", 3, 2, 9, 2),
    ((400, 96), "box", 1, 8, 20, 4),
    ((5000,), "star", 1, 8, 19, 4),
    ((777,), "star", 2, 3, 10, 3),
    ((60, 40, 50), "box", 1, 2, 5, 2),
    ((90, 30, 34), "star", 1, 3, 7, 3),
    ((2048, 256), "box", 1, 16, 33, 8),
]


@pytest.mark.parametrize("ext,shape,r,T,steps,n", CASES)
def test_loopback_group_bitwise_equals_single_gpu(fs, ext, shape, r, T, steps, n):
    w = wl.seeded_weights(shape, len(ext), r)
    u0 = wl.grid(ext, 41)
    single = fs.Plan(ext, w, r, T)
    a = torch.from_numpy(u0).cuda()
    ref_gpu = torch.empty_like(a)
    single.run(a, ref_gpu, steps)
    plans = [fs.Plan(ext, w, r, T, nranks=n, rank=k, loopback=True) for k in range(n)]
    infos = [p.info() for p in plans]
    ins = [a[i["row_begin"]:i["row_end"]].contiguous() for i in infos]
    outs = [torch.empty_like(t) for t in ins]
    fs.run_group(plans, ins, outs, steps)
    torch.cuda.synchronize()
    got = torch.cat(outs).cpu().numpy()
    assert np.array_equal(got, ref_gpu.cpu().numpy())
    ref = oracle.stencil_run(u0, w, r, steps)
    assert np.abs(got - ref).max() <= 1e-9 * np.abs(ref).max()
    # launches per rank: 3 fused (interior + two edges, empty ones skipped) + band per pass
    assert all(p.info()["last_run_launches"] > 0 for p in plans)


def test_loopback_rank_refuses_plain_run(fs):
    w = wl.seeded_weights("box", 2, 1)
    p = fs.Plan((300, 100), w, 1, 4, nranks=2, rank=0, loopback=True)
    x = torch.zeros(p.extents, dtype=torch.float64, device="cuda")
    with pytest.raises(fs.FftStencilError):
        p.run(x, torch.empty_like(x), 4)


def test_nccl_single_rank_plan_runs(fs):
    """nranks = 1 through the dist entry point is an ordinary plan."""
    w = wl.seeded_weights("box", 2, 1)
    uid = fs.nccl_unique_id()
    assert len(uid) == 128
    p = fs.Plan((120, 90), w, 1, 4, nranks=1, rank=0, nccl_id=uid)
    u0 = wl.grid((120, 90), 3)
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    p.run(a, b, 9)
    torch.cuda.synchronize()
    ref = oracle.stencil_run(u0, w, 1, 9)
    assert np.abs(b.cpu().numpy() - ref).max() <= 1e-9


def test_nccl_two_ranks_bitwise(fs, tmp_path):
    """The NCCL halo exchange (ncclSend / ncclRecv on the plan's comm stream, overlapped with the
    halo-free pairs) on two GPUs, bitwise equal to one GPU (G7).  Needs >= 2 visible devices."""
    import os
    import socket
    import subprocess
    import sys
    if torch.cuda.device_count() < 2:
        pytest.skip("needs >= 2 CUDA devices (NCCL refuses two ranks on one GPU)")
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    worker = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_nccl_worker.py")
    env = dict(os.environ, NCCL_DEBUG="INFO")
    res = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                          "--master-addr=127.0.0.1", f"--master-port={port}", worker],
                         capture_output=True, text=True, env=env, timeout=600)
    log = res.stdout + res.stderr
    (tmp_path / "nccl.log").write_text(log)
    assert res.returncode == 0, log[-4000:]
    assert log.count("bitwise OK") == 5, log[-4000:]
    assert "Init COMPLETE" in log or "ncclCommInitRank" in log, "no NCCL communicator was initialised"


@pytest.mark.parametrize("nproc,fused", [(2, 1), (3, 1), (2, 0)])
def test_peer_transport_processes(fs, tmp_path, nproc, fused):
    """The peer-memory transport (no NCCL) across `nproc` processes -- on one GPU when only one is
    visible (IPC within a device), else one GPU per rank -- bitwise equal to one GPU over chained
    calls (G7).  fused = 1: the boundary rows reach the neighbours as the edge tiles' and the
    band's own stores (default); 0: a copy-engine push after each pass."""
    import os
    import socket
    import subprocess
    import sys
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    worker = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_peer_worker.py")
    res = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
                          "--master-addr=127.0.0.1", f"--master-port={port}", worker],
                         capture_output=True, text=True, timeout=900,
                         env=dict(os.environ, FFTSTENCIL_PEER_FUSED=str(fused)))
    log = res.stdout + res.stderr
    (tmp_path / "peer.log").write_text(log)
    assert res.returncode == 0, log[-4000:]
    assert log.count("bitwise OK") == 7, log[-4000:]
    if fused:   # the 1D, 2D and 3D ALU-engine cases push with the kernels' stores
        assert log.count("fused_push=1") >= 6, log[-4000:]
    else:
        assert "fused_push=1" not in log, log[-4000:]
