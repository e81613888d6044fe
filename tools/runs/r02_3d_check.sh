# 3D pair-shuffle kernel: parity, sanitizers, speed vs the line kernel
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "3d or vs_oracle" 2>&1 | tail -4
timeout 600 python -m pytest tests/test_gpu_steady_state.py -q -x -m gpu -k "60 or 52 or 49 or 120 or 130 or 44" 2>&1 | tail -4
cat > /tmp/san3d.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs
from synth import workloads as wl
import oracle
for ext, shape, r, T, steps, env in [((60, 50, 45), "star", 1, 2, 5, {"FFTSTENCIL_MAX_CTAS": "1"}),
                                     ((40, 36, 34), "box", 1, 1, 3, {}), ((33, 35, 37), "star", 1, 2, 3, {"FFTSTENCIL_TMA": "0"})]:
    os.environ.update(env)
    w = wl.seeded_weights(shape, 3, r); u0 = wl.grid(ext, 3)
    p = fs.Plan(ext, w, r, T); a = torch.from_numpy(u0).cuda(); b = torch.empty_like(a)
    p.run(a, b, steps); torch.cuda.synchronize()
    ref = oracle.stencil_run(u0, w, r, steps)
    print("ok", ext, env, float(np.abs(b.cpu().numpy() - ref).max()))
    for k in env: del os.environ[k]
PY
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san3d.py > gpurun_out/r02_san3d_$tool.log 2>&1; echo "$tool rc=$?"; grep -E "^ok|ERROR SUMMARY" gpurun_out/r02_san3d_$tool.log | tail -4
done
for k in pairs lines; do
  FFTSTENCIL_3D_KERNEL=$k timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_3d_$k.jsonl 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02_3d_$k.jsonl').read().strip().splitlines()[-1]);print('$k', round(d['value'],1), 'GSt/s', 'frac', round(d['roofline']['frac'],3), 'fused ms', round(d['roofline']['fused_ms_avg'],3))" || tail -5 gpurun_out/r02_3d_$k.jsonl
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft3d_b3 -s 2 -c 1 -o gpurun_out/r02_fft3d_b3 python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_ncu3d.log 2>&1; echo ncu rc=$?
