# full GPU suite + default bench line + launch list (ncu --metrics gpu__time_duration.sum)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err; echo bench $?
cat gpurun_out/bench_default.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_s2.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1; echo ncu $?
timeout 600 ncu --set full --clock-control none -k regex:fft2d_bf -c 1 --csv --page raw --metrics dram__bytes_read.sum,dram__bytes_write.sum python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > gpurun_out/traffic2d.csv 2>&1; echo tr $?
