# round-2 re-entry: confirm HEAD on a fresh box (smoke, GPU tests, default bench line)
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4 | tee gpurun_out/r02c_smoke.txt
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -4 | tee gpurun_out/r02c_gpu_tests.txt
( time timeout 900 python bench.py > gpurun_out/r02c_bench.jsonl 2> gpurun_out/r02c_bench.err ) 2>&1 | tail -3
head -c 600 gpurun_out/r02c_bench.jsonl
