# cp.async ring S2 = 8 for NV = 2: full GPU suite + C3 + bench
TAG=${1:-r3v}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
(timeout 900 python scripts/c3_ab.py s2_8; timeout 300 python scripts/c3_ab.py s2_8; timeout 300 python scripts/agg_ab.py s2_8) > gpurun_out/c3_ab_$TAG.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
