#!/bin/bash
# session-7: cfg1 with the flush write-back moved out of the step; launch list + full capture of cfg1's kernel
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s7; mkdir -p $O
timeout 600 python bench.py --config 1 > $O/bench_cfg1.log 2>&1
timeout 600 python bench.py --config 1 --steps 500 --no-cpu-baseline > $O/bench_cfg1_500.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg1.csv python bench.py --config 1 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg1 python bench.py --config 1 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full1.log 2>&1
echo done
