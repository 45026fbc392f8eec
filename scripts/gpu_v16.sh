# round-end refresh: GEMM A/B log, full GPU suite, bench, launch list, ncu, smoke
TAG=${1:-v16}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GNN_GEMM_CB=0 timeout 300 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_nocb_$TAG.log 2>&1
timeout 300 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_$TAG.log 2>&1
bash scripts/gpu_full.sh $TAG
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
