# session 3: re-verify the restored tree on a fresh box (GPU tests + default bench line)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/s3_gpu_tests.log 2>&1; echo tests $?
tail -3 gpurun_out/s3_gpu_tests.log
timeout 600 python bench.py > gpurun_out/s3_bench_default.jsonl 2> gpurun_out/s3_bench_default.err; echo bench $?
cat gpurun_out/s3_bench_default.jsonl
