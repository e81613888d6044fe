# full GPU test suite + default bench line (per_config included) + reference arm
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4
timeout 2400 python -m pytest tests -q -m gpu -x 2>&1 | tail -5 > gpurun_out/r02_gpu_tests.txt; cat gpurun_out/r02_gpu_tests.txt
( time timeout 900 python bench.py > gpurun_out/r02_bench_default.jsonl 2> gpurun_out/r02_bench_default.err ) 2>&1 | tail -3
tail -c 3000 gpurun_out/r02_bench_default.jsonl; tail -5 gpurun_out/r02_bench_default.err
( time timeout 600 python bench.py --impl reference > gpurun_out/r02_bench_reference.jsonl ) 2>&1 | tail -3
