#!/bin/bash
# full GPU test suite (+ optional bench configs in $BENCH)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/tests; mkdir -p $O
timeout 1800 python -m pytest tests -q -p no:cacheprovider -m gpu $PYTEST_ARGS > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
for c in $BENCH; do timeout 600 python bench.py --config $c $BENCH_ARGS > $O/bench_cfg$c.log 2>&1; done
if [ -n "$PARTS" ]; then timeout 600 python tools/bench_cfg3_parts.py > $O/parts.log 2>&1; fi
echo done
