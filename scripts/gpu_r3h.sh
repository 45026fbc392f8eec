# full validation: NEXT-2 tests first, then the whole GPU suite, smoke, bench, launch list
TAG=${1:-r3h}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_next2.py tests/test_gpu_multirank.py -q -p no:cacheprovider > gpurun_out/pytest_next2_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_next2_$TAG.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_launch_$TAG.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_launch_$TAG.log
