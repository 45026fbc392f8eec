# quick GEMM A/B: TMA-fed vs register-fed X tiles (parity + timing); column blocks on/off
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "gemm or gat or attn" -p no:cacheprovider > gpurun_out/pytest_gemm_tma.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gemm_tma.log
timeout 400 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_tma.log 2>&1
echo "kbench rc=$?" >> gpurun_out/kbench_gemm_tma.log
GNN_GEMM_CB=0 timeout 400 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_nocb.log 2>&1
