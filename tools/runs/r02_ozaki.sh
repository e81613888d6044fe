# NEXT-4 microbenchmark: Ozaki-sliced INT8 tcgen05 DFT-16 vs the FP64 butterfly FFT-16
mkdir -p gpurun_out
/usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo \
  -I paper_conf_ppopp_hanlcbzyczcy25_b200/csrc tools/ozaki_dft16.cu -o /tmp/ozaki_dft16 || exit 1
timeout 300 /tmp/ozaki_dft16 2>&1 | tee gpurun_out/r02_ozaki.txt
# per-kernel pipe counters of the compute-bound (R = 16) butterfly and full Ozaki launches
timeout 600 ncu --metrics gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fp64.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_uniform.sum,smsp__inst_executed.sum --clock-control none -s 126 -c 22 /tmp/ozaki_dft16 > gpurun_out/r02_ozaki_ncu.txt 2>&1
grep -E "bf_kernel|ozaki_kernel|duration|fp64|tensor|inst_executed" gpurun_out/r02_ozaki_ncu.txt | awk 'NR<=7 || (NR>=133 && NR<=139)'
