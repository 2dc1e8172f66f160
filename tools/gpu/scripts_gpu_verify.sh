#!/bin/bash
# session-start verification: full GPU suite + the bench lines touched by the latest commits
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/verify; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -q -p no:cacheprovider -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_default.log 2>&1
timeout 600 python bench.py --config 3 > $O/bench_cfg3.log 2>&1
timeout 600 python bench.py --config 3 --p 1000 --rows 1000000 > $O/bench_cfg3_p1000.log 2>&1
timeout 600 python bench.py --config 4 > $O/bench_cfg4.log 2>&1
timeout 600 python bench.py --config 4 --bits 2048 > $O/bench_cfg4_2048.log 2>&1
timeout 600 python bench.py --config 5 > $O/bench_cfg5.log 2>&1
echo done
