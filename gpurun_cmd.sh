P="python tools/probe.py"
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "xs or thread or more" 2>&1 | tail -1
$P "xsbench -s small -g 1000 -G unionized -l 0 -r {i}" 1024 256 2
$P "xsbench -s small -g 1000 -G unionized -l 10000 -r {i}" 1024 256 2
