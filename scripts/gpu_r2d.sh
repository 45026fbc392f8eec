TAG=${1:-r2d}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/gemm_ab.py > gpurun_out/gemm_ab_$TAG.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_parity.py tests/test_gpu_plan_io.py -q -k "gat or gemm or c5_step or plan" -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_$TAG.log 2>&1
