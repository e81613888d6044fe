# Table 4-style with / without analysis of the fused kernels on B200:
# ALU (butterfly) vs DMMA line engine, TMA SWIZZLE_128B staging vs per-thread cp.async, for
# 1D3P (Heat-1D 512M), 2D9P (Box-2D9P 10240^2), 3D27P (Box-3D27P 1024^3).  One ncu report per
# case (one steady-state fused launch, SourceCounters for the uncoalesced-access rule) + a short
# bench run for GSt/s.  Reports land in gpurun_out/t4/ and are summarised by tools/table4_summary.py.
mkdir -p gpurun_out/t4
M=gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,sm__sass_inst_executed_op_shared_st.sum,sm__sass_inst_executed_op_shared_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum,l1tex__t_requests_pipe_lsu_mem_global_op_st.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ldgsts_cache_access.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ldgsts_cache_access.sum,l1tex__m_xbar2l1tex_read_sectors_mem_global_op_tma_ld.sum,dram__bytes_read.sum,dram__bytes_write.sum
case_run() {  # tag workload steps env...
  tag=$1; w=$2; ts=$3; shift 3
  env "$@" timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('BENCH $tag $w', round(d['value'],2), d['unit'], 'fused_ms', round(r['fused_ms_avg'],4), 'T', d['config'].get('T'))"
  env "$@" timeout 900 ncu --section SourceCounters --metrics $M --clock-control none -k regex:fft[123]d -s 1 -c 1 -f -o gpurun_out/t4/${tag}_${w} python bench.py --workload $w --time-steps $ts --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1 || echo "NCU FAILED $tag $w"
}
for w in heat1d_512m box2d9p box3d27p; do
  ts=30; [ $w = box3d27p ] && ts=6
  case_run alu_tma $w $ts FFTSTENCIL_ENGINE=alu
  case_run alu_cpasync $w $ts FFTSTENCIL_ENGINE=alu FFTSTENCIL_TMA=0
  case_run dmma_tma $w $ts FFTSTENCIL_ENGINE=dmma
  case_run dmma_cpasync $w $ts FFTSTENCIL_ENGINE=dmma FFTSTENCIL_TMA=0
done
ls -la gpurun_out/t4
