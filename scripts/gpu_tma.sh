# quick GEMM A/B: TMA-fed vs register-fed X tiles (parity + timing); 8 vs 4 epilogue warps
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k gemm -p no:cacheprovider > gpurun_out/pytest_gemm_tma.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gemm_tma.log
timeout 400 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_tma.log 2>&1
echo "kbench rc=$?" >> gpurun_out/kbench_gemm_tma.log
GNN_GEMM_EPI8=0 timeout 400 python scripts/kbench.py gemm > gpurun_out/kbench_gemm_epi4.log 2>&1
