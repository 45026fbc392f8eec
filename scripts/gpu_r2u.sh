TAG=${1:-r2u}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool synccheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "test_aggregate_parity and hub" > gpurun_out/sanitizer_synccheck_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_synccheck_$TAG.txt
timeout 900 compute-sanitizer --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "gat_transform or straddling or chunks or agg1 or agg2" > gpurun_out/sanitizer_memcheck2_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_memcheck2_$TAG.txt
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
