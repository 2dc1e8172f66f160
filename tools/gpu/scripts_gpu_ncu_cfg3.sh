cd "$GRAFT_REPO_ROOT"
O=gpurun_out/s4; mkdir -p $O
for P in 200 1000; do R=""; [ $P = 1000 ] && R="--rows 1000000"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg3_p$P.csv python bench.py --config 3 --p $P $R --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/launch_p$P.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:contract -s 2 -c 1 -o $O/prof_tc_p$P python bench.py --config 3 --p $P $R --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/full_p$P.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:upk -s 2 -c 1 -o $O/prof_rest_p200 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/full_rest.log 2>&1
