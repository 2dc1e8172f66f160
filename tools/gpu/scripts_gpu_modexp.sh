#!/bin/bash
# modexp parity + bench lines
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/mx; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_modexp.py tests/test_gpu_fullsize.py -q -p no:cacheprovider -x -k "modexp or cfg4 or rsa or RSA or pow" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python bench.py --config 4 --no-cpu-baseline > $O/bench_cfg4.log 2>&1
timeout 300 python bench.py --config 4 --e 3 --no-cpu-baseline > $O/bench_cfg4_e3.log 2>&1
UP_MODEXP_OUTCONV=1 timeout 300 python bench.py --config 4 --e 3 --no-cpu-baseline > $O/bench_cfg4_e3_outconv.log 2>&1
