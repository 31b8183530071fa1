# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_run.py (every kernel path).
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "== $tool (exit $?)"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run done|Error|error" gpurun_out/sanitize_$tool.log | tail -5
done
