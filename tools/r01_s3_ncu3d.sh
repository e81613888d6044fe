# ncu --set full (source-level) of one Heat-3D fused launch of the 3D ALU kernel
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fft3d_bf" -c 1 -o gpurun_out/s3_fft3d_bf python bench.py --workload heat3d --steps 1 --warmup 0 --time-steps 2 --no-e2e --no-cpu-baseline > gpurun_out/s3_ncu3d.log 2>&1; echo ncu $?
