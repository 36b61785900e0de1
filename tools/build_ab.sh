# build libdp.so of git revision $1 into paper_conf_dac_lindlrkp19_b200/lib_ab/$2.so (A/B runs: DP_LIB_AB=...)
set -e
rev=$1; name=$2
wt=/tmp/dp_ab_$name
rm -rf $wt; git worktree add -f $wt $rev > /dev/null 2>&1
(cd $wt && python -c "import sys; sys.path.insert(0,'.'); from paper_conf_dac_lindlrkp19_b200.build import build; build(force=True)" > /dev/null)
mkdir -p paper_conf_dac_lindlrkp19_b200/lib_ab
cp $wt/paper_conf_dac_lindlrkp19_b200/lib/libdp.so paper_conf_dac_lindlrkp19_b200/lib_ab/$name.so
git worktree remove --force $wt
echo paper_conf_dac_lindlrkp19_b200/lib_ab/$name.so
