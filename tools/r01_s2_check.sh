# session-2 re-entry check: GPU tests, default bench, 3D bench
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err; echo bench $?
timeout 600 python bench.py --workload heat3d --no-cpu-baseline > gpurun_out/bench_heat3d.jsonl 2>&1; echo b3 $?
cat gpurun_out/bench_default.jsonl
