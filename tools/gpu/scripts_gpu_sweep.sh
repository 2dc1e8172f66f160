#!/bin/bash
# remaining bench lines: sin_P sweep, RSA e=3, cfg3 precisions
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/sweep; mkdir -p $O
timeout 600 python bench.py --config 5 --P 500 > $O/bench_cfg5_P500.log 2>&1
timeout 600 python bench.py --config 5 --P 5000 --rows 100000 > $O/bench_cfg5_P5000.log 2>&1
timeout 600 python bench.py --config 5 --P 20000 --rows 10000 > $O/bench_cfg5_P20000.log 2>&1
timeout 600 python bench.py --config 4 --e 3 > $O/bench_cfg4_e3.log 2>&1
timeout 600 python bench.py --config 3 > $O/bench_cfg3.log 2>&1
timeout 600 python bench.py --config 3 --p 500 --rows 2000000 > $O/bench_cfg3_p500.log 2>&1
timeout 600 python bench.py --config 3 --p 1000 --rows 1000000 > $O/bench_cfg3_p1000.log 2>&1
UP_NO_TC=1 timeout 600 python bench.py --config 3 --no-cpu-baseline > $O/bench_cfg3_cudacore.log 2>&1
echo done
