#!/bin/bash
# consolidated measurement session: every bench line + ncu launch lists / full captures
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/intpipe tools/intpipe.cu && /tmp/intpipe > $O/intpipe.json 2>&1
for c in 2 1 3 4 5; do timeout 900 python bench.py --config $c > $O/bench_cfg$c.log 2>&1; done
timeout 900 python bench.py --config 3 --p 500 --rows 2000000 > $O/bench_cfg3_p500.log 2>&1
timeout 900 python bench.py --config 3 --p 1000 --rows 1000000 > $O/bench_cfg3_p1000.log 2>&1
timeout 900 python bench.py --config 4 --bits 2048 > $O/bench_cfg4_2048.log 2>&1
timeout 900 python bench.py --config 4 --e 3 > $O/bench_cfg4_e3.log 2>&1
timeout 900 python bench.py --config 5 --P 500 > $O/bench_cfg5_P500.log 2>&1
timeout 900 python bench.py --config 5 --P 5000 --rows 100000 > $O/bench_cfg5_P5000.log 2>&1
timeout 900 python bench.py --config 5 --P 20000 --rows 10000 > $O/bench_cfg5_P20000.log 2>&1
timeout 600 python bench.py --impl reference > $O/bench_reference_cfg2.log 2>&1
for c in 2 3 4; do
  R=""; [ $c = 4 ] && R="--rows 1000000"
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg$c.csv python bench.py --config $c $R --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 2 > $O/ncu_launch$c.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg$c python bench.py --config $c $R --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full$c.log 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg5.csv python bench.py --config 5 --rows 100000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg5 python bench.py --config 5 --rows 100000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full5.log 2>&1
echo done
