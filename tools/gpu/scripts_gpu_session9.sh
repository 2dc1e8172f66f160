#!/bin/bash
# session-9: occupancy of the narrow (R = 4) SUM kernels: default vs UP_MINBLOCKS=8 on cfg1 / cfg2
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/s9; mkdir -p $O
for mb in 8 0; do
  for c in 1 2; do
    if [ $mb = 0 ]; then timeout 600 python bench.py --config $c --no-cpu-baseline > $O/bench_cfg${c}_mbdef.log 2>&1
    else UP_MINBLOCKS=$mb timeout 600 python bench.py --config $c --no-cpu-baseline > $O/bench_cfg${c}_mb$mb.log 2>&1; fi
  done
done
echo done
