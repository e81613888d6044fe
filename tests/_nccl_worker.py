"""Worker of tests/test_gpu_dist.py::test_nccl_two_ranks_bitwise (run under torchrun, one rank
per GPU): the NCCL halo-exchange path of fftstencil_run (capi.cu nccl_exchange) on a real
process group; rank 0 compares the gathered slabs with a single-GPU run, bitwise."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

CASES = [((300, 170), "box", 1, 4, 11), ((257, 129), "star", 3, 2, 9), ((60, 40, 50), "box", 1, 2, 5),
         ((5000,), "star", 1, 8, 19), ((2048, 256), "box", 1, 0, 40)]


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", rank))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    bad = 0
    for ext, shape, r, T, steps in CASES:
        w = wl.seeded_weights(shape, len(ext), r)
        u0 = wl.grid(ext, 77)
        obj = [fs.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        p = fs.Plan(ext, w, r, T, nranks=world, rank=rank, nccl_id=obj[0])
        inf = p.info()
        a = torch.from_numpy(np.ascontiguousarray(u0[inf["row_begin"]:inf["row_end"]])).cuda()
        b = torch.empty_like(a)
        p.run(a, b, steps)
        torch.cuda.synchronize()
        slabs = [None] * world
        dist.all_gather_object(slabs, b.cpu().numpy())
        if rank == 0:
            got = np.concatenate(slabs)
            q = fs.Plan(ext, w, r, T)
            x = torch.from_numpy(u0).cuda()
            y = torch.empty_like(x)
            q.run(x, y, steps)
            torch.cuda.synchronize()
            ok = np.array_equal(got, y.cpu().numpy())
            print(f"case {ext} r={r} T={inf['T']} ranks={world}: bitwise {'OK' if ok else 'MISMATCH'}", flush=True)
            bad += not ok
            q.close()
        p.close()
    dist.barrier()
    dist.destroy_process_group()
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
