for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/san_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/san_$tool.log
done
ncu --set full --clock-control none --import-source on -k regex:fft2d_ct -s 2 -c 1 -o gpurun_out/r01_fft2d_ct_tma python bench.py --steps 1 --warmup 1 --time-steps 33 --no-e2e --no-cpu-baseline > gpurun_out/ncu_ct2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:fft3d_ct -s 2 -c 1 -o gpurun_out/r01_fft3d_ct python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 6 --no-e2e --no-cpu-baseline > gpurun_out/ncu_3d.log 2>&1
tail -n1 gpurun_out/ncu_ct2.log; tail -n1 gpurun_out/ncu_3d.log
