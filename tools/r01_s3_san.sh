# compute-sanitizer memcheck / racecheck / synccheck of every kernel on small cases (final code)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/s3_san_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/s3_san_$tool.log
done
