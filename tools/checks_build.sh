#!/bin/bash
# Rebuild libens.so with the device checks on (ENS_CHECKS=1: bounds / invariant traps in the
# cross-CTA paths) and run the given pytest selection against it; the product build is restored after.
set -e
FL="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo --fmad=false -std=c++17 -Xcompiler -fPIC -DENS_CHECKS=1"
(cd paper_conf_icppw_tiancd23_b200/csrc && rm -f kernels.o kernels_items.o kernels_sub.o api.o && make -s -j16 NVFLAGS="$FL" > /dev/null)
set +e
python -m pytest "$@"
rc=$?
(cd paper_conf_icppw_tiancd23_b200/csrc && rm -f kernels.o kernels_items.o kernels_sub.o api.o && make -s -j16 > /dev/null)
exit $rc
