#!/bin/bash
# bench lines: default + cfg3 (p 200/500/1000) + cfg4 + cfg5; $O from env
cd "$GRAFT_REPO_ROOT" || exit 1
O=${O:-gpurun_out/bench}; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
timeout 600 python bench.py > $O/bench_cfg2.log 2>&1
timeout 600 python bench.py --config 1 > $O/bench_cfg1.log 2>&1
timeout 600 python bench.py --config 3 > $O/bench_cfg3.log 2>&1
timeout 600 python bench.py --config 3 --p 500 --rows 2000000 > $O/bench_cfg3_p500.log 2>&1
timeout 600 python bench.py --config 3 --p 1000 --rows 1000000 > $O/bench_cfg3_p1000.log 2>&1
timeout 600 python bench.py --config 4 > $O/bench_cfg4.log 2>&1
timeout 600 python bench.py --config 4 --bits 2048 > $O/bench_cfg4_2048.log 2>&1
timeout 600 python bench.py --config 5 > $O/bench_cfg5.log 2>&1
[ -n "$PARTS" ] && timeout 400 python tools/bench_cfg3_parts.py > $O/parts.log 2>&1
echo done
