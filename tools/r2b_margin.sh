# margin + IF-node sort: tests, GP trajectories, headline A/B
python -m pytest tests/test_gpu_sort_reuse.py -q -x 2>&1 | tail -4 > gpurun_out/m_tests.log
python -m pytest tests -m gpu -q -x 2>&1 | tail -4 >> gpurun_out/m_tests.log
python tools/gp_motion.py adaptec1 bigblue4 --iters 1500 --every 300 --json gpurun_out/gp_motion_m.json > gpurun_out/gp_motion_m.txt 2>&1
for v in "DP_REUSE_SORT=0" "DP_SORT_COND=0" "DP_SORT_COND=1"; do echo "== $v"; env $v python tools/gp_prof.py bigblue4 20; env $v python tools/gp_prof.py bigblue4 600; done > gpurun_out/m_gp.txt 2>&1
bash tools/ab_quick.sh "DP_REUSE_SORT=0" "DP_SORT_COND=0" "DP_SORT_COND=1" > gpurun_out/m_ab.log 2>&1
