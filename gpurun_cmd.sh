P="python tools/probe.py"
C=paper_conf_icppw_tiancd23_b200/csrc
for cfg in "512 2" "1024 1" "1024 2" "512 1" "512 4"; do
  set -- $cfg
  rm -f $C/kernels.o
  make -s -C $C NVFLAGS="-gencode arch=compute_100a,code=sm_100a -O3 --fmad=false -std=c++17 -Xcompiler -fPIC -DENS_MINB_NUM=$1 -DENS_XS_U=$2" > /dev/null 2>&1
  echo "== MINB_NUM=$1 U=$2"
  $P "xsbench -s small -g 1000 -G unionized -l 10000 -r {i}" 1024 256 2
  $P "xsbench -s small -g 1000 -G unionized -l 10000 -r {i}" 1024 512 2
  $P "xsbench -s small -g 1000 -G unionized -l 10000 -r {i}" 1024 128 2
  $P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 64 512 2
  $P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 64 256 2
done
