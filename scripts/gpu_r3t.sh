# hot-row L2 residency at plan level (default) vs off (GNN_L2_PIN=0): parity, C5 / C3 A/B, bench
TAG=${1:-r3t}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
(for r in 1 2; do
timeout 600 python scripts/agg_ab.py pin
GNN_L2_PIN=0 timeout 300 python scripts/agg_ab.py nopin
done
timeout 900 python scripts/c3_ab.py pin
GNN_L2_PIN=0 timeout 300 python scripts/c3_ab.py nopin
timeout 300 python scripts/c3_ab.py pin --prescaled
GNN_L2_PIN=0 timeout 300 python scripts/c3_ab.py nopin --prescaled) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
GNN_L2_PIN=0 timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/bench_nopin_$TAG.log 2>&1
