# does the tcgen05 kind::tf32 MMA truncate raw fp32 exactly like hi_of()? (bitwise test) + timing
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GNN_GEMM_HISTORE=0 timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "gemm_tma_matches" -p no:cacheprovider > gpurun_out/hs_test.log 2>&1
echo "rc=$?" >> gpurun_out/hs_test.log
timeout 300 python scripts/kbench.py gemm > gpurun_out/hs_on.log 2>&1
GNN_GEMM_HISTORE=0 timeout 300 python scripts/kbench.py gemm > gpurun_out/hs_off.log 2>&1
