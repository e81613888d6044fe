# session 3 closing run: smoke, all GPU tests, default bench line, reference arm, launch list
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/s3z_smoke.log 2>&1; echo smoke $?; cat gpurun_out/s3z_smoke.log | tail -4
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/s3z_gpu_tests.log 2>&1; echo tests $?; tail -1 gpurun_out/s3z_gpu_tests.log
timeout 600 python bench.py > gpurun_out/s3z_bench_default.jsonl 2> gpurun_out/s3z_bench_default.err; echo bench $?
cat gpurun_out/s3z_bench_default.jsonl
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/s3z_bench_ref.jsonl 2>&1; echo ref $?
timeout 300 python bench.py --workload heat1d > gpurun_out/s3z_bench_heat1d.jsonl 2>&1; echo heat1d $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3z_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
