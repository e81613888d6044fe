python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "engines or periodic or full_size" > gpurun_out/pytest_st.log 2>&1; echo pytest $?
tail -2 gpurun_out/pytest_st.log
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms', r['bound'], 'frac', round(r['frac'],3), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],3))" $1 "$2" 2>&1 | tail -1; }
for w in heat2d box2d49p heat3d heat1d_512m; do
  timeout 600 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/st_$w.jsonl 2>&1
  summ gpurun_out/st_$w.jsonl "$w"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -c 1 -o gpurun_out/r01_fft2d_bf_st python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu2 $?
