# full GPU suite, 1D benches after the band SM reservation, default bench, sanitizers (ALU kernels)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms', r['bound'], 'frac', round(r['frac'],3), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],3))" $1 "$2" 2>&1 | tail -1; }
for w in heat1d_512m 1d5p_512m 1d7p_512m heat1d; do
  timeout 600 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/s2_$w.jsonl 2>&1
  summ gpurun_out/s2_$w.jsonl "$w"
done
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err; echo bench $?
summ gpurun_out/bench_default.jsonl default
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/san_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/san_$tool.log
done
