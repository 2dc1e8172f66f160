cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out/divtop; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_divtop.py tests/test_gpu_parity.py tests/test_gpu_wide.py tests/test_gpu_fullsize.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python tools/bench_cfg3_parts.py > $O/parts.log 2>&1
UP_NO_DIVTOP=1 EXPRS="c3/c4;c1*c2 - c3/c4" timeout 600 python tools/bench_cfg3_parts.py > $O/parts_nodivtop.log 2>&1
timeout 600 python bench.py --config 3 > $O/bench_cfg3.log 2>&1
