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
echo done
