# parity subset + headline A/B of the current build (arguments: env settings for ab_quick)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gp.py tests/test_gpu_det.py -x -q -k "not adaptec1" > gpurun_out/t_quick.log 2>&1; tail -2 gpurun_out/t_quick.log
bash tools/ab_quick.sh "$@" > gpurun_out/ab_quick.txt 2>&1
