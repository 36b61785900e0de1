# fused combine / recomputing gather: tests and headline A/B (walk)
python -m pytest tests/test_gpu_sort_reuse.py tests/test_gpu_parity.py -q -x -k "stale or switches or host" 2>&1 | tail -3 > gpurun_out/rc_tests.log
bash tools/ab_quick.sh "DP_X=0" "DP_FUSE_COMBINE=1" "DP_GATHER_RC=1" "DP_GATHER_RC=1 DP_FUSE_COMBINE=1" "DP_X=1" > gpurun_out/rc_ab.log 2>&1
for v in "DP_X=0" "DP_GATHER_RC=1 DP_FUSE_COMBINE=1"; do echo "== $v"; env $v python tools/gp_prof.py bigblue4 600; done >> gpurun_out/rc_ab.log 2>&1
