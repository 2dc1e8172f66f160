#!/bin/bash
# stage-depth experiment for the tensor-core contraction (UP_TC_KC)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/kc; mkdir -p $O
UP_TC_KC=256 timeout 300 python tools/tc_smoke.py > $O/smoke256.log 2>&1
for kc in 256 64; do
  UP_TC_KC=$kc timeout 300 python bench.py --config 3 --no-cpu-baseline > $O/bench_p200_kc$kc.log 2>&1
  UP_TC_KC=$kc timeout 300 python bench.py --config 3 --p 500 --rows 2000000 --no-cpu-baseline > $O/bench_p500_kc$kc.log 2>&1
done
