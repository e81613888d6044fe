# run-to-run variance of the default headline line (no per_config), three back-to-back runs
for i in 1 2 3; do
  timeout 600 python bench.py --no-per-config --no-cpu-baseline --steps 8 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('run', $i, round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done
