# round-2 GPU session: new parity tests, full GPU suite, bench
# usage: bash scripts/gpu_r2.sh TAG
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi_$TAG.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_bench_configs.py -q -p no:cacheprovider > gpurun_out/pytest_new_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_new_$TAG.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --ignore=tests/test_gpu_bench_configs.py > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/bench_$TAG.log
