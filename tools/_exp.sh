FL="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo --fmad=false -std=c++17 -Xcompiler -fPIC"
for V in "-DENS_MAX_TEAM=8" "-DENS_MAX_TEAM=16"; do
  (cd paper_conf_icppw_tiancd23_b200/csrc && rm -f kernels.o kernels_sub.o kernels_items.o api.o && make -s -j16 NVFLAGS="$FL $V" > /dev/null 2>&1)
  echo "VARIANT $V"; for w in C1 C3 C2; do python tools/ktimes.py $w 5 2>&1 | grep "best\|phase 1 "; done
done
