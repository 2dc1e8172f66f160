#!/bin/bash
# session-11: block size of the grouped sin_P kernel (UP_SIN_GT): parity tests at 32/64, P=5000/20000 bench lines at 32/64/128/256
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s11; mkdir -p $O
for gt in 32 64; do
  UP_SIN_GT=$gt timeout 900 python -m pytest tests/test_gpu_sin.py -q -p no:cacheprovider -x > $O/pytest_sin_gt$gt.log 2>&1
done
for gt in 32 64 128 256; do
  UP_SIN_GT=$gt timeout 600 python bench.py --config 5 --P 5000 --rows 100000 --no-cpu-baseline --e2e-steps 1 > $O/bench_cfg5_P5000_gt$gt.log 2>&1
  UP_SIN_GT=$gt timeout 600 python bench.py --config 5 --P 20000 --rows 10000 --no-cpu-baseline --e2e-steps 1 > $O/bench_cfg5_P20000_gt$gt.log 2>&1
done
echo done
