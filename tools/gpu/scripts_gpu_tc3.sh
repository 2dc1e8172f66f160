cd "$GRAFT_REPO_ROOT"
timeout 900 python -m pytest tests/test_gpu_contract_tc.py tests/test_gpu_wide.py -q -p no:cacheprovider -x > gpurun_out/tc_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/tc_pytest.log
P=1000 R=1000000 ./tools/gpu/scripts_gpu_ncu_tc.sh
