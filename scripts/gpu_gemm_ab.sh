# GEMM ring-depth / column-block A/B at the C5 shapes + GEMM parity tests
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for cfg in "GNN_GEMM_CB=1" "GNN_GEMM_CB=2" "GNN_GEMM_CB=1 GNN_GEMM_SA=3" "GNN_GEMM_CB=1 GNN_GEMM_SA=4" "GNN_GEMM_CB=2 GNN_GEMM_SA=4" "GNN_GEMM_CB=0"; do
  env $cfg timeout 300 python scripts/gemm_ab.py
done) > gpurun_out/gemm_ab_$TAG.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_parity.py -q -k "gemm" -p no:cacheprovider > gpurun_out/pytest_gemm_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gemm_$TAG.log
