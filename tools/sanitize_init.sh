export DP_GRAPH=0
timeout 1500 compute-sanitizer --tool initcheck --error-exitcode 9 --print-limit 100000 python tools/sanitize_run.py \
  > gpurun_out/sanitizer_initcheck.log 2>&1; echo "initcheck rc=$?" > gpurun_out/sanitizer_summary2.txt
grep "Host Frame\|Kernel\|at 0x" gpurun_out/sanitizer_initcheck.log | sed 's/0x[0-9a-f]*//g' | sort | uniq -c | sort -rn | head -20 >> gpurun_out/sanitizer_summary2.txt
tail -2 gpurun_out/sanitizer_initcheck.log >> gpurun_out/sanitizer_summary2.txt
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report all --error-exitcode 9 --print-limit 50 \
   python tools/sanitize_run.py > gpurun_out/sanitizer_racecheck_adaptec1.log 2>&1; echo "racecheck(tiny+adaptec1) rc=$?" >> gpurun_out/sanitizer_summary2.txt
tail -2 gpurun_out/sanitizer_racecheck_adaptec1.log >> gpurun_out/sanitizer_summary2.txt
