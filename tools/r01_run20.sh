timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft2d_ct -c 1 -o gpurun_out/r01_fft2d_ct_3m python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft3d_ct -c 1 -o gpurun_out/r01_fft3d_ct_b python bench.py --workload heat3d --steps 1 --warmup 0 --time-steps 2 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out/
