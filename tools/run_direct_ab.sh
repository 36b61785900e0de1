python -m pytest tests/test_gpu_gp.py -x -q -k "not adaptec1" > gpurun_out/t_gp.log 2>&1; tail -2 gpurun_out/t_gp.log
DP_DIRECT=1 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lse.py tests/test_gpu_gp.py -x -q -k "not slow and not adaptec1" > gpurun_out/t_direct.log 2>&1; tail -2 gpurun_out/t_direct.log
bash tools/ab_quick.sh "DP_DIRECT=1" "DP_DIRECT=0" "DP_DIRECT=1" "DP_DIRECT=0" > gpurun_out/ab_direct.txt 2>&1
python bench.py --steps 300 --warmup 10 --no-cpu-baseline --e2e-steps 2 2>&1 | tail -1 > gpurun_out/bench_gp.json
