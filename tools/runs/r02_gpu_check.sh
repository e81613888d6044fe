# round 2: steady-state parity tests + sanitizers on the capped multi-pair cases + 3D bench baseline
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests/test_gpu_steady_state.py -q -x -m gpu 2>&1 | tail -15 > gpurun_out/r02_steady.txt
cat gpurun_out/r02_steady.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "full_size or engines" 2>&1 | tail -8 > gpurun_out/r02_parity_sel.txt
cat gpurun_out/r02_parity_sel.txt
for tool in memcheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/r02_san_$tool.log 2>&1; echo "$tool rc=$?"; tail -3 gpurun_out/r02_san_$tool.log
done
timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02_heat3d_base.jsonl 2>&1; tail -c 600 gpurun_out/r02_heat3d_base.jsonl
