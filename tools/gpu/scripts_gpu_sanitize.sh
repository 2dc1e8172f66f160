#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over small parity cases + the full-size tests
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out/san
S=/usr/local/cuda/bin/compute-sanitizer
K='test_eval_expr_parity or test_sum_expr_parity or test_textbook or test_sin_rows_parity or test_cfg3_wide_sum_parity or test_compact_round_trip'
timeout 1800 $S --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py tests/test_gpu_modexp.py tests/test_gpu_sin.py tests/test_gpu_wide.py tests/test_compact_codec.py -q -p no:cacheprovider -k "$K and not 2051 and not 3001 and not 1000 and not 5000" > gpurun_out/san/memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/san/memcheck.log
timeout 1800 $S --tool racecheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sin.py -q -p no:cacheprovider -k "test_sum_expr_parity and (7) or test_sin_rows_parity and 500" > gpurun_out/san/racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/san/racecheck.log
timeout 1800 $S --tool synccheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sin.py -q -p no:cacheprovider -k "test_sum_expr_parity and (7) or test_sin_rows_parity and 500" > gpurun_out/san/synccheck.log 2>&1; echo "rc=$?" >> gpurun_out/san/synccheck.log
timeout 2400 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider > gpurun_out/san/fullsize.log 2>&1; echo "rc=$?" >> gpurun_out/san/fullsize.log
echo done
