python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -c 1 -o gpurun_out/r01_fft2d_bf_b python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu2 $?
