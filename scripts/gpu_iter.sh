# iteration session: GPU tests, aggregation kbench, bench
set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python scripts/kbench.py agg --cfg C5 > gpurun_out/kb_agg_v3.log 2>&1; echo "rc=$?" >> gpurun_out/kb_agg_v3.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench4.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench4.log
