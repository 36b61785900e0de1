# GP iteration time vs the re-sort threshold / IF node (adaptec1 and bigblue4 at iteration 600)
for v in "DP_REUSE_SORT=0" "DP_RESORT_PCT=0.5" "DP_RESORT_PCT=2" "DP_RESORT_PCT=5" "DP_RESORT_PCT=20" "DP_SORT_COND=0"; do
  echo "== $v"; env $v python tools/gp_prof.py adaptec1 600; env $v python tools/gp_prof.py adaptec1 1200; env $v python tools/gp_prof.py bigblue4 600
done
