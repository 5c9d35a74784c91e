P="python tools/probe.py"
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -m gpu 2>&1 | tail -1
$P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 64 512 2 --phases | head -1
$P "xsbench -s large -g 11303 -G hash -h 10000 -l 1000000 -r {i}" 64 512 2 --team 1 | head -1
