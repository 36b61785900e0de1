# compute-sanitizer over the whole C ABI (tools/sanitize_run.py); logs -> gpurun_out/sanitizer_*.log
export DP_GRAPH=0
for tool in memcheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_run.py \
     > gpurun_out/sanitizer_$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/sanitizer_summary.txt
done
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report all --error-exitcode 9 --print-limit 50 \
   python tools/sanitize_run.py --tiny > gpurun_out/sanitizer_racecheck.log 2>&1; echo "racecheck(tiny) rc=$?" >> gpurun_out/sanitizer_summary.txt
tail -3 gpurun_out/sanitizer_*.log >> gpurun_out/sanitizer_summary.txt
