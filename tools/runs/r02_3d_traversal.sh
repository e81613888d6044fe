# 3D ALU kernel traversal order (FFTSTENCIL_3D_TRAV = block side in tile lines, 0 = natural order):
# parity subset, bench A/B, and DRAM bytes per fused launch under ncu.
set -u
FFTSTENCIL_3D_TRAV=6 timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py tests/test_gpu_e2e_pipe.py tests/test_gpu_dist.py -k "3d or heat3d or box3d or ENGINE or engine" 2>&1 | tail -3
run() {  # blk workload
  FFTSTENCIL_3D_TRAV=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('trav=$1 $2', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r['band_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2))"
}
for w in heat3d box3d27p; do for b in 0 6 0 6 4 8 12; do run $b $w; done; done
for b in 0 6 8; do
  FFTSTENCIL_3D_TRAV=$b timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:fft3d_bf -s 2 -c 2 --csv python bench.py --workload heat3d --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/trav_ncu_$b.csv 2>/dev/null
  echo "ncu trav=$b"; grep -E "dram__bytes|gpu__time|hit_rate" gpurun_out/trav_ncu_$b.csv | awk -F'","' '{print $(NF-3), $(NF-2), $NF}'
done
