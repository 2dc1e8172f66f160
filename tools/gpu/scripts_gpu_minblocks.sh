cd "$GRAFT_REPO_ROOT"
O=gpurun_out/mb; mkdir -p $O
for mb in ${MBS:-2 3 4}; do UP_MINBLOCKS=$mb timeout 300 python bench.py --config 3 --no-cpu-baseline > $O/bench_mb$mb.log 2>&1; done
