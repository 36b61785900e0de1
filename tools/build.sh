#!/bin/bash
# Build libdp.so in-tree and print register/spill lines of the named kernels.
cd "$(dirname "$0")/.." && python -m paper_conf_dac_lindlrkp19_b200.build 2>&1 | grep -v Warn | tail -1
for k in "$@"; do grep -A2 "$k" paper_conf_dac_lindlrkp19_b200/lib/build.log | grep -E "registers|spill" | sed "s/^/$k: /"; done
