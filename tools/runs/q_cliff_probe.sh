mkdir -p gpurun_out
for Q in 12 16; do
  nvidia-smi --query-gpu=clocks.sm,power.draw,clocks_throttle_reasons.active --format=csv,noheader -lms 10 > gpurun_out/s4_q${Q}_clocks.txt &
  SMI=$!
  FFTSTENCIL_E2E_PIPE=4 FFTSTENCIL_E2E_DEPTH=$Q python - <<'PY' >> gpurun_out/s4_q_cliff.txt 2>&1
import os, sys, time, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs
from synth import workloads as wl
ext = (10240, 10240)
p = fs.Plan(ext, wl.seeded_weights("star", 2, 1), 1, 0)
h_in = torch.from_numpy(wl.grid(ext, 1)).pin_memory(); h_out = torch.empty(ext, dtype=torch.float64).pin_memory()
for i in range(6):
    t0 = time.perf_counter(); p.run_host(h_in, h_out, 1000); t = (time.perf_counter() - t0) * 1e3
    print("Q", os.environ["FFTSTENCIL_E2E_DEPTH"], "call", i, "ms", round(t, 2), flush=True)
PY
  kill $SMI
done
for Q in 12 16; do echo "Q=$Q"; sort gpurun_out/s4_q${Q}_clocks.txt | uniq -c | sort -rn | head -5; done
cat gpurun_out/s4_q_cliff.txt
