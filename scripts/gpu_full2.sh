# full GPU suite + aggregation A/B + bench
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
(timeout 600 python scripts/agg_ab.py default
GNN_AGG_CP=1 timeout 300 python scripts/agg_ab.py cp_chain
GNN_AGG_CP=0 timeout 300 python scripts/agg_ab.py reg_kernel) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/bench_$TAG.log
