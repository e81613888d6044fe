python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "3d or 3D or periodic" > gpurun_out/pytest_3d.log 2>&1; echo pytest $?
tail -5 gpurun_out/pytest_3d.log
FFTSTENCIL_ENGINE=alu timeout 600 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/b3_alu.jsonl 2>&1; echo b3 $?
tail -1 gpurun_out/b3_alu.jsonl | cut -c1-1500
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft3d_bf -c 1 -o gpurun_out/r01_fft3d_bf_b python bench.py --workload heat3d --steps 1 --warmup 0 --time-steps 2 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
