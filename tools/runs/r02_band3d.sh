# band cone kernel: warp-parallel tap table + flattened region load / store
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "band or vs_oracle or full_size_3d or engines" 2>&1 | tail -2
run() {  # stream workload
  FFTSTENCIL_BAND_STREAM=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('stream=$1 $2', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r['band_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2))"
}
for w in heat3d box3d27p heat2d box2d49p box2d9p star2d13p; do run 0 $w; run 1 $w; done
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize.py > gpurun_out/r02_san_band_memcheck.log 2>&1; echo "memcheck rc=$?"
