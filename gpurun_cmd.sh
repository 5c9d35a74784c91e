timeout 600 python bench.py > gpurun_out/bench3.json 2> gpurun_out/bench3.err; echo bench=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 2 --warmup 3 --no-extras > /dev/null 2>&1; echo list=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ens_kernel -s 1 -c 1 -o gpurun_out/c2_r1b python bench.py --steps 1 --warmup 3 --no-extras > /dev/null 2>&1; echo full=$?
