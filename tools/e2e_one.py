"""One pipelined run_host call on Heat-2D 10240^2 (1000 steps), for an ncu launch list of the
e2e schedule (`ncu --metrics gpu__time_duration.sum ... python tools/e2e_one.py`)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs  # noqa: E402
from synth import workloads as wl  # noqa: E402

ext = (10240, 10240)
p = fs.Plan(ext, wl.seeded_weights("star", 2, 1), 1, 0)
h_in = torch.from_numpy(wl.grid(ext, 1)).pin_memory()
h_out = torch.empty(ext, dtype=torch.float64).pin_memory()
p.run_host(h_in, h_out, int(sys.argv[1]) if len(sys.argv) > 1 else 1000)
torch.cuda.synchronize()
print("launches", p.info()["last_run_launches"])
