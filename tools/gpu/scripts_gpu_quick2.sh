#!/bin/bash
# correctness subset + cfg3 bench lines
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/q2; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_contract_tc.py tests/test_gpu_wide.py tests/test_gpu_divtop.py tests/test_gpu_parity.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for p in 200 500 1000; do R=""; [ $p = 500 ] && R="--rows 2000000"; [ $p = 1000 ] && R="--rows 1000000"; timeout 300 python bench.py --config 3 --p $p $R --no-cpu-baseline > $O/bench_cfg3_p$p.log 2>&1; done
UP_OVERLAP=1 timeout 300 python bench.py --config 3 --no-cpu-baseline > $O/bench_cfg3_p200_overlap.log 2>&1
