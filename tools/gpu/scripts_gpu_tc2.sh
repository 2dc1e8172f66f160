cd "$GRAFT_REPO_ROOT"
timeout 200 python tools/tc_smoke.py > gpurun_out/tc_smoke.log 2>&1; echo rc=$? >> gpurun_out/tc_smoke.log
timeout 300 python tools/bench_cfg3_parts.py > gpurun_out/tc_parts.log 2>&1
P=200 R=2000000 ./tools/gpu/scripts_gpu_ncu_tc.sh
