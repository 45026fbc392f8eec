# iteration session: GEMM check, aggregation, GPU tests, bench
set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/kbench.py gemm > gpurun_out/kb_gemm.log 2>&1; echo "rc=$?" >> gpurun_out/kb_gemm.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench3.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench3.log
