P="python tools/probe.py"
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -m gpu 2>&1 | tail -3
$P "xsbench -s large -g 11303 -G hash -h 10000 -l 0 -r {i}" 64 512 2
$P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 64 512 2
$P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 1 512 2
$P "xsbench -s small -g 1000 -G unionized -l 10000 -r {i}" 1024 256 2
