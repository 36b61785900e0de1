# sort reuse: new GPU tests, the whole GPU suite, and the headline A/B (fixed positions: reuse = no sort)
python -m pytest tests/test_gpu_sort_reuse.py -q -x 2>&1 | tail -15 > gpurun_out/reuse_tests.log
python -m pytest tests -m gpu -q 2>&1 | tail -8 > gpurun_out/reuse_all_tests.log
bash tools/ab_quick.sh "DP_REUSE_SORT=0" "DP_REUSE_SORT=1" "DP_SCHED=1" "DP_SCHED=0" > gpurun_out/reuse_ab.log 2>&1
bash tools/launch_list.sh > /dev/null 2>&1; cp gpurun_out/launches.txt gpurun_out/reuse_launches.txt 2>/dev/null
