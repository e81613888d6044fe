# 1D ALU engine: parity, Table 3 benches, ncu
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "1d or 1D or periodic or parity_vs_oracle" > gpurun_out/pytest_1d.log 2>&1; echo pytest $?
tail -5 gpurun_out/pytest_1d.log
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms', r['bound'], 'frac', round(r['frac'],3), 'share', round(r['fused_share_of_step'],3), r['kernel'])" $1 "$2" 2>&1 | tail -1; }
for w in heat1d_512m 1d5p_512m 1d7p_512m heat1d; do
  timeout 600 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/s1_$w.jsonl 2>&1
  summ gpurun_out/s1_$w.jsonl "$w"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft1d_bf -c 1 -o gpurun_out/r01_fft1d_bf python bench.py --workload heat1d_512m --steps 1 --warmup 0 --time-steps 1024 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
