# band folded into the 2D / 3D ALU fused kernels: parity (fold on / off), sanitizers, A/B bench
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_e2e_pipe.py tests/test_gpu_steady_state.py tests/test_gpu_dist.py -q -x -m gpu 2>&1 | tail -3
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/r02_san_fold_$tool.log 2>&1; echo "$tool rc=$?"; grep -E "ERROR SUMMARY" gpurun_out/r02_san_fold_$tool.log | tail -1
done
D=paper_conf_ppopp_hanlcbzyczcy25_b200
run() {  # lib fold workload
  FFTSTENCIL_LIB=$D/$1 FFTSTENCIL_BAND_FOLD=$2 timeout 300 python bench.py --workload $3 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1 fold=$2 $3', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
}
for rep in 1 2; do
  for w in heat2d heat3d box2d49p; do
    run libfftstencil_ab_old.so 1 $w; run libfftstencil.so 0 $w; run libfftstencil.so 1 $w
  done
done
timeout 300 python bench.py --workload heat3d --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('heat3d fold e2e', round(d['value'],1), round(d['e2e']['value'],1), d['e2e']['ms_per_step'])"
timeout 300 python bench.py --workload heat2d --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('heat2d fold e2e', round(d['value'],1), round(d['e2e']['value'],1), d['e2e']['ms_per_step'])"
