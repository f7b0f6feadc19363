for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/r02san2_$tool.txt 2>&1; echo "$tool exit $?" >> gpurun_out/r02san2_summary.txt
done
echo done
