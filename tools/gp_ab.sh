# GP loop A/B of in-tree builds (lib_ab/*.so): GP iterations/s from the initial placement and the bench headline
L=paper_conf_dac_lindlrkp19_b200/lib_ab
for lib in "$@"; do echo "== $lib"; DP_LIB_AB=$L/$lib.so python tools/gp_prof.py bigblue4 20; DP_LIB_AB=$L/$lib.so python tools/gp_prof.py bigblue4 300; done
