# A/B of the persistent double-buffered WA pipeline (DP_WA_PIPE=1) against the default chunk launch
mkdir -p gpurun_out
bash tools/ab_quick.sh DP_WA_PIPE=0 "DP_WA_PIPE=1 DP_WA_PIPE_RESERVE=16" "DP_WA_PIPE=1 DP_WA_PIPE_RESERVE=40" "DP_WA_PIPE=1 DP_WA_PIPE_RESERVE=74" "DP_WA_PIPE=1 DP_WA_PIPE_RESERVE=0 DP_PRIO=0"
