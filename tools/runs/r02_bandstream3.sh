# 3D band serialised (FFTSTENCIL_BAND_STREAM=0) vs concurrent (default now), bench lines with clocks
for rep in 1 2 3; do
  for b in 0 1; do
    FFTSTENCIL_BAND_STREAM=$b timeout 600 python bench.py --no-per-config --no-cpu-baseline --steps 8 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('band_stream=$b', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
  done
done
nvidia-smi --query-gpu=power.draw,power.limit,clocks.sm --format=csv
