# ncu --set full (source-level) of one Heat-2D fused launch of the default 2D ALU kernel (final code)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fft2d_bf" -c 1 -o gpurun_out/s3_fft2d_bf_final python bench.py --workload heat2d --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > gpurun_out/s3_ncu2d_final.log 2>&1; echo ncu $?
