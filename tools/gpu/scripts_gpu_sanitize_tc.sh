#!/bin/bash
# compute-sanitizer over the tensor-core contraction and the top-limb division (small cases)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/san_tc; mkdir -p $O
S=/usr/local/cuda/bin/compute-sanitizer
K='(test_tc_contraction_shapes and (129 or -1-)) or test_tc_contraction_empty'
timeout 1200 $S --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_contract_tc.py -q -p no:cacheprovider -k "$K" > $O/memcheck_tc.log 2>&1; echo "rc=$?" >> $O/memcheck_tc.log
timeout 1200 $S --tool racecheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_contract_tc.py -q -p no:cacheprovider -k "test_tc_contraction_shapes and 129 and (200-200 or 1000-1000)" > $O/racecheck_tc.log 2>&1; echo "rc=$?" >> $O/racecheck_tc.log
timeout 1200 $S --tool synccheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_contract_tc.py -q -p no:cacheprovider -k "test_tc_contraction_shapes and 129 and (200-200 or 1000-1000)" > $O/synccheck_tc.log 2>&1; echo "rc=$?" >> $O/synccheck_tc.log
timeout 1200 $S --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_divtop.py -q -p no:cacheprovider > $O/memcheck_divtop.log 2>&1; echo "rc=$?" >> $O/memcheck_divtop.log
echo done
