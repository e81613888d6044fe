# 3D ALU kernel: S_t evaluated in P3 from per-line symbol coefficients (FFTSTENCIL_ONFLY=1, default)
# vs the staged 64 KB S_t table (FFTSTENCIL_ONFLY=0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py -k "3d or heat3d or box3d" 2>&1 | tail -2
run() {  # onfly workload
  FFTSTENCIL_ONFLY=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('onfly=$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
}
for rep in 1 2; do for w in heat3d box3d27p; do run 0 $w; run 1 $w; done; done
for b in 0 1; do
  FFTSTENCIL_ONFLY=$b timeout 600 ncu --metrics gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:fft3d_bf -s 1 -c 1 --csv python bench.py --workload heat3d --time-steps 6 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | grep -E "wavefronts|fp64|inst_exec|dram|duration" | awk -F'","' '{print "ncu onfly='$b'", $(NF-2), $NF}'
done
