#!/bin/bash
# focused GPU session: selected tests + selected bench configs (+ intpipe microbenchmark)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
if [ -n "$INTPIPE" ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/intpipe tools/intpipe.cu && /tmp/intpipe > gpurun_out/intpipe.json 2>&1
fi
if [ -n "$TESTS" ]; then
  timeout 2400 python -m pytest $TESTS -q -p no:cacheprovider -x > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
fi
for c in $BENCH; do
  timeout 900 python bench.py $BENCH_ARGS --config $c > gpurun_out/bench_q_cfg$c.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_q_cfg$c.log
done
if [ -n "$Q1" ]; then
  timeout 900 python tools/bench_q1.py > gpurun_out/q1.log 2>&1; echo "q1 rc=$?" >> gpurun_out/q1.log
fi
if [ -n "$OPS" ]; then
  timeout 900 python tools/bench_operators.py > gpurun_out/ops.log 2>&1; echo "ops rc=$?" >> gpurun_out/ops.log
fi
echo done
