"""Worker of tests/test_gpu_dist.py::test_peer_transport_two_processes (run under torchrun): the
peer-memory halo transport of fftstencil_run (capi.cu run_dist_peer: CUDA IPC buffers, copy-engine
pushes, stream-memory signal / wait) across processes -- one GPU per rank when there are enough
devices, else the ranks share device 0.  Handles travel over a gloo group; rank 0 compares the
gathered slabs with a single-GPU run, bitwise, for several calls in a row (the ranks' lockstep
epochs carry across calls)."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

CASES = [((300, 170), "box", 1, 4, (11, 4)), ((257, 129), "star", 3, 2, (9,)), ((60, 40, 50), "box", 1, 2, (5, 2)),
         ((5000,), "star", 1, 8, (19,)), ((2048, 256), "box", 1, 0, (40, 13)), ((90, 30, 34), "star", 1, 3, (7,)),
         ((300000,), "star", 1, 0, (2100,))]   # 1D factored ALU engine (4096-cell tiles, T = 1024)


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    ndev = torch.cuda.device_count()
    dev = rank if ndev >= world else 0
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo")
    bad = 0
    for ext, shape, r, T, runs in CASES:
        w = wl.seeded_weights(shape, len(ext), r)
        u0 = wl.grid(ext, 91)
        p = fs.Plan(ext, w, r, T, nranks=world, rank=rank, transport="peer")
        p.connect_peers()
        inf = p.info()
        a = torch.from_numpy(np.ascontiguousarray(u0[inf["row_begin"]:inf["row_end"]])).cuda()
        for steps in runs:      # successive calls chain: the input of each is the last output
            b = torch.empty_like(a)
            p.run(a, b, steps)
            torch.cuda.synchronize()
            a = b
        fused = p.info()["last_run_peer_fused"]
        slabs = [None] * world
        dist.all_gather_object(slabs, a.cpu().numpy())
        if rank == 0:
            got = np.concatenate(slabs)
            q = fs.Plan(ext, w, r, T)
            x = torch.from_numpy(u0).cuda()
            for steps in runs:   # the same chain of calls (a different pass split rounds differently)
                y = torch.empty_like(x)
                q.run(x, y, steps)
                x = y
            torch.cuda.synchronize()
            ok = np.array_equal(got, y.cpu().numpy())
            print(f"case {ext} r={r} T={inf['T']} ranks={world} devices={min(ndev, world)} runs={runs} "
                  f"engine={inf['engine']} fused_push={int(fused)}: bitwise {'OK' if ok else 'MISMATCH'}", flush=True)
            bad += not ok
            q.close()
        dist.barrier()   # every rank done with its plan before any closes its IPC-shared buffers
        p.close()
        dist.barrier()
    dist.destroy_process_group()
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
