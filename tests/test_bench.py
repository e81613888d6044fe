"""Host-side accounting of bench.py (no GPU): the whole-job GStencils/s of a weak-scaled run.

bench.py stacks the N=1 workload's rows N times along axis 0 (the global grid the library
decomposes back into per-rank slabs), so the throughput is global cells x time steps / the
max-over-ranks time -- with no extra factor of the world size (reading Q18).
"""
import pytest
import bench
from synth import workloads as wl


def test_gstencils_definition():
    # 10240^2 cells x 1000 steps in 100 ms = 1048.576 GStencils/s
    assert abs(bench.gstencils(10240 * 10240, 1000, 100.0) - 1048.576) < 1e-9


def test_weak_scaling_counts_each_slab_once():
    wk = wl.CONFIGS["box2d9p_weak"]
    per_gpu = 1
    for e in wk.extents:
        per_gpu *= e
    one = bench.gstencils(per_gpu, 1000, 50.0)
    for world in (2, 4, 8):
        glob = (wk.extents[0] * world,) + tuple(wk.extents[1:])
        cells = 1
        for e in glob:
            cells *= e
        # perfect weak scaling (same time per rank) reports exactly world x the 1-GPU value
        assert abs(bench.gstencils(cells, 1000, 50.0) / one - world) < 1e-12


def test_smem_wavefront_model():
    # 2D five passes (4 read + write, 1 read) + S_T; 3D cropped inverse passes
    assert bench.smem_wavefronts_per_pair({"ndim": 2}) == 10 * 512
    assert bench.smem_wavefronts_per_pair({"ndim": 3, "valid": [12, 12, 12]}) == 4416
    assert bench.smem_wavefronts_per_pair({"ndim": 3, "valid": [16, 16, 16]}) == 10 * 512
    assert bench.smem_wavefronts_per_pair({"ndim": 1}) == 14 * 512
    assert abs(bench.SMEM_PEAK_TBPS - 37.22496) < 1e-9


def _sass_mix(obj):
    """(DADD, DMUL, DFMA) static counts of the TMA instantiation (<true, false[, false]>) in `obj`,
    without the band-folding subroutine (the CALL right before the kernel's final EXIT, up to
    its RET): the mix weights the FP64 peak of the tile passes, which is what bench.py reports."""
    import re
    import subprocess
    out = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
    lines, inside = [], False
    for ln in out.splitlines():
        if "Function" in ln:
            # the TMA, non-periodic, single-GPU instantiation (not the peer-store one, <1, 0, 1>)
            inside = "ILb1ELb0E" in ln and "ILb1ELb0ELb1E" not in ln
            continue
        m = re.match(r"\s*/\*([0-9a-f]+)\*/\s+(.*)", ln)
        if inside and m:
            lines.append((int(m.group(1), 16), m.group(2)))
    skip = None
    for k, (addr, txt) in enumerate(lines):
        if re.match(r"EXIT\b", txt):                     # the kernel's final, unconditional EXIT
            call = next((t for _, t in reversed(lines[max(0, k - 4):k]) if "CALL" in t), None)
            if call:
                lo = int(re.search(r"0x([0-9a-f]+)", call).group(1), 16)
                hi = next(a for a, t in lines if a > lo and t.startswith("RET"))
                skip = (lo, hi)
            break
    counts = {"DADD": 0, "DMUL": 0, "DFMA": 0}
    for addr, txt in lines:
        if skip and skip[0] <= addr <= skip[1]:
            continue
        for mm in re.finditer(r"\b(DADD|DMUL|DFMA)\b", txt):
            counts[mm.group(1)] += 1
    return counts["DADD"], counts["DMUL"], counts["DFMA"]


def test_alu_kernel_mix_matches_build():
    """bench.py's FP64 mixes (the weights of the ALU peak) are those of the built kernels."""
    import os
    import shutil

    import pytest
    build = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                         "paper_conf_ppopp_hanlcbzyczcy25_b200", "_build")
    if shutil.which("cuobjdump") is None or not os.path.isdir(build):
        pytest.skip("needs cuobjdump and a built tree")
    for name, mix in bench.ALU_KERNEL_MIX.items():
        obj = os.path.join(build, name + ".cu.o")
        if not os.path.exists(obj):
            pytest.skip(f"{obj} not built")
        assert _sass_mix(obj) == mix, name


def test_alu_peak_between_opcode_rates():
    for mix in bench.ALU_KERNEL_MIX.values():
        p = bench.alu_peak_tops(mix)
        assert min(bench.FP64_RATES_TOPS.values()) < p < max(bench.FP64_RATES_TOPS.values())


def test_default_workloads_and_per_config_cover_baseline():
    """N = 1 headline = the largest single-GPU BASELINE config (Heat-3D 1024^3, configs[3]);
    N > 1 = configs[4]'s weak slab; every BASELINE config appears in the per_config list."""
    assert bench.default_workload(1) == "heat3d"
    assert all(bench.default_workload(n) == "heat3d_weak" for n in (2, 4, 8))
    labels = {lab.split()[0] for _, _, _, lab in bench.PER_CONFIG}
    assert {"configs[0]", "configs[1]", "configs[2]", "configs[3]", "configs[4]"} <= labels
    names = {n for n, *_ in bench.PER_CONFIG}
    for n in names:
        assert n in wl.CONFIGS
    # configs[1]'s T sweep covers 1..16 for both stencils
    sweep = {(n, t) for n, t, _, lab in bench.PER_CONFIG if "sweep" in lab}
    assert {t for _, t in sweep} >= {1, 2, 4, 8, 16}


def test_gpus_without_torchrun_relaunches(monkeypatch):
    """`bench.py --gpus N > 1` outside torch.distributed re-executes itself under
    torch.distributed.run with N ranks on 127.0.0.1 (it must not silently measure one GPU)."""
    import subprocess
    calls = []
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(subprocess, "call", lambda cmd: calls.append(cmd) or 0)
    assert bench.main(["--gpus", "4", "--steps", "2"]) == 0
    (cmd,) = calls
    assert "torch.distributed.run" in cmd and "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd
    assert cmd[-3:] == ["--gpus", "4", "--steps", "2"][-3:]


def test_world_size_mismatch_is_an_error(monkeypatch):
    import pytest
    monkeypatch.setenv("WORLD_SIZE", "2")
    monkeypatch.setenv("RANK", "0")
    with pytest.raises(SystemExit):
        bench.main(["--gpus", "4"])


def _peer_plan_worker(rank, port, fail_rank, fail_stage, out):
    import os

    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)

    class FakePlan:
        closed = False

        def __init__(self, *a, **k):
            if rank == fail_rank and fail_stage == "create":
                raise RuntimeError("no peer access")
            self.extents = (4, 4)

        def peer_handle(self):
            return bytes([rank]) * 256

        def peer_connect(self, lower, upper):
            if rank == fail_rank and fail_stage == "connect":
                raise RuntimeError("cudaIpcOpenMemHandle failed")
            assert (lower is None) == (rank == 0) and (upper is None) == (rank == 1)

        def close(self):
            FakePlan.closed = True

    class FakeFs:
        Plan = FakePlan

    bench.TRANSPORT_NOTE.clear()
    plan = bench.peer_plan(FakeFs, dist, 2, rank, (8, 4), None, 1, 2)
    out.put((rank, plan is not None, list(bench.TRANSPORT_NOTE)))
    dist.destroy_process_group()


@pytest.mark.parametrize("fail_rank,fail_stage", [(-1, ""), (1, "create"), (0, "connect")])
def test_peer_plan_falls_back_together(fail_rank, fail_stage):
    """bench.peer_plan: either every rank gets a connected peer plan, or -- when any rank fails to
    create / export / map -- every rank gets None (the group falls back to NCCL together), without
    a rank stuck in a collective the others skipped (gloo, world size 2, CPU)."""
    import multiprocessing as mp
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_peer_plan_worker, args=(r, port, fail_rank, fail_stage, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    ok = fail_rank < 0
    assert all(r[1] == ok for r in res)
    assert all(bool(r[2]) == (not ok) for r in res)
