#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/ncu_tc; mkdir -p $O
P=${P:-200}; R=${R:-2000000}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_p$P.csv python bench.py --config 3 --p $P --rows $R --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > $O/launch_p$P.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:contract -s 1 -c 1 -o $O/prof_tc_p$P python bench.py --config 3 --p $P --rows $R --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > $O/full_p$P.log 2>&1
echo done
