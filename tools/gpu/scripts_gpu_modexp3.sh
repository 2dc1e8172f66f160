#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/mx3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_modexp.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python bench.py --config 4 --no-cpu-baseline > $O/bench_cfg4.log 2>&1
timeout 300 python bench.py --config 4 --e 3 --no-cpu-baseline > $O/bench_cfg4_e3.log 2>&1
timeout 300 python bench.py --config 4 --bits 2048 --no-cpu-baseline > $O/bench_2048.log 2>&1
