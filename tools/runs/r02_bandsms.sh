# SMs reserved for the concurrent band kernel in fftstencil_run (FFTSTENCIL_BAND_SMS), one box
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
run() {  # R workload
  FFTSTENCIL_BAND_SMS=$1 timeout 300 python bench.py --workload $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('R=$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band_ms', round(r['band_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
}
for w in heat3d heat2d box3d27p box2d49p; do
  for R in 0 1 2 4 8; do run $R $w; done
done
for R in 0 2; do run $R heat3d; run $R heat2d; done
