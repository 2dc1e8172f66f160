#!/bin/bash
# session-3 measurement: full GPU suite, every bench line, ncu launch lists + full captures
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s6; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1800 python -m pytest tests -q -p no:cacheprovider -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
O=$O/bench PARTS=1 ./tools/gpu/scripts_gpu_bench_all.sh
timeout 600 python bench.py --impl reference > $O/bench_reference_cfg2.log 2>&1
for c in 2 3 4 5; do
  R=""; [ $c = 4 ] && R="--rows 1000000"; [ $c = 5 ] && R="--rows 100000"
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg$c.csv python bench.py --config $c $R --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_launch$c.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg2 python bench.py --config 2 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:contract -s 2 -c 1 -o $O/prof_cfg3_tc python bench.py --config 3 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 2 -c 1 -o $O/prof_cfg3_rest python bench.py --config 3 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full3r.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg4 python bench.py --config 4 --rows 1000000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:upk -s 4 -c 1 -o $O/prof_cfg5 python bench.py --config 5 --rows 100000 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_full5.log 2>&1
echo done
