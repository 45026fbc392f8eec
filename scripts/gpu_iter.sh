# iteration session: GEMM check, aggregation A/B, GPU tests, bench
set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/kbench.py gemm > gpurun_out/kb_gemm.log 2>&1; echo "rc=$?" >> gpurun_out/kb_gemm.log
timeout 400 python scripts/kbench.py agg --cfg C5 > gpurun_out/kb_agg_mb4.log 2>&1; echo "rc=$?" >> gpurun_out/kb_agg_mb4.log
GNN_LIB_PATH=$GRAFT_REPO_ROOT/paper_conf_ppopp_huangzzys21_b200/libgnn_mb3.so timeout 400 python scripts/kbench.py agg --cfg C5 > gpurun_out/kb_agg_mb3.log 2>&1; echo "rc=$?" >> gpurun_out/kb_agg_mb3.log
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/bench2.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench2.log
