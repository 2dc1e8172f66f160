#!/bin/bash
# one GPU session: smoke, parity tests, bench lines, ncu launch lists + full captures
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
timeout 300 python -c 'import __graft_entry__ as g; g.build(); g.smoke()' > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --maxfail=40 -p no:cacheprovider -x ${PYTEST_K} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in ${BENCH_CONFIGS:-2 4 5 3 1}; do
  timeout 900 python bench.py --config $c > gpurun_out/bench_cfg$c.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_cfg$c.log
done
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg4.csv python bench.py --config 4 --rows 1000000 --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_launch4.log 2>&1
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg5.csv python bench.py --config 5 --rows 100000 --steps 3 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_launch5.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 2 -c 1 -o gpurun_out/prof_cfg4 python bench.py --config 4 --rows 1000000 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full4.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 2 -c 1 -o gpurun_out/prof_cfg5 python bench.py --config 5 --rows 100000 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full5.log 2>&1
fi
echo done
