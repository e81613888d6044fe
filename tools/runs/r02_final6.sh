# closing run: 3D device band serialised, pipelined run_host items with the band concurrent
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4 | tee gpurun_out/r02k_smoke.txt
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -4 | tee gpurun_out/r02k_gpu_tests.txt
( time timeout 900 python bench.py > gpurun_out/r02k_bench.jsonl 2> gpurun_out/r02k_bench.err ) 2>&1 | tail -3
for rep in 1 2; do for b in 0 1; do
  FFTSTENCIL_E2E_BAND_STREAM=$b timeout 600 python bench.py --no-per-config --no-cpu-baseline --steps 5 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('e2e_band_stream=$b', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done; done | tee gpurun_out/r02k_e2e_band_ab.txt
