#!/bin/bash
# session-8: cfg1 with the flush write-back moved out of the step (+ ncu of its kernel);
# sin_P v3 block size 32/64/128 (UP_SIN_NT): parity tests + cfg5 bench lines
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s8; mkdir -p $O
timeout 600 python bench.py --config 1 > $O/bench_cfg1.log 2>&1
for nt in 32 64; do
  UP_SIN_NT=$nt timeout 900 python -m pytest tests/test_gpu_sin.py -q -p no:cacheprovider -x > $O/pytest_sin_nt$nt.log 2>&1
  UP_SIN_NT=$nt timeout 600 python bench.py --config 5 --no-cpu-baseline > $O/bench_cfg5_nt$nt.log 2>&1
done
timeout 600 python bench.py --config 5 --no-cpu-baseline > $O/bench_cfg5_nt128.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg1.csv python bench.py --config 1 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg1 python bench.py --config 1 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full1.log 2>&1
echo done
