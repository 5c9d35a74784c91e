#!/bin/bash
# Rebuild libens.so with larger unionized sort buckets (ENS_XS_UBKT_DIV=D records per bucket on
# average, device checks on) so that the bucket sort's local-array (9..64) and in-place (> 64)
# paths run, then the given pytest selection; the product build is restored after.
# usage: bash tools/ubkt_check.sh D [pytest args...]
D=$1
shift
FL="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo --fmad=false -std=c++17 -Xcompiler -fPIC -DENS_CHECKS=1 -DENS_XS_UBKT_DIV=$D"
(cd paper_conf_icppw_tiancd23_b200/csrc && rm -f kernels.o kernels_items.o kernels_sub.o api.o && make -s -j16 NVFLAGS="$FL" > /dev/null) || exit 1
python -m pytest "$@"
rc=$?
(cd paper_conf_icppw_tiancd23_b200/csrc && rm -f kernels.o kernels_items.o kernels_sub.o api.o && make -s -j16 > /dev/null)
exit $rc
