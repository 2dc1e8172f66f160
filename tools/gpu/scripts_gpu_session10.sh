#!/bin/bash
# session-10 (final): smoke, full GPU suite, default bench + cfg5 with the one-warp sin_P v3 blocks
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s10; mkdir -p $O
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -q -p no:cacheprovider -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_cfg2.log 2>&1
timeout 600 python bench.py --config 5 > $O/bench_cfg5.log 2>&1
timeout 600 python bench.py --config 5 --P 500 --no-cpu-baseline > $O/bench_cfg5_P500.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg5.csv python bench.py --config 5 --rows 100000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg5 python bench.py --config 5 --rows 100000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full5.log 2>&1
echo done
