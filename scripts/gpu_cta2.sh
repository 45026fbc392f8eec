# CTA-pair GEMM A/B (GNN_GEMM_CTA2) + the register-store epilogue diag + GEMM parity under the pair
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 300 python scripts/gemm_ab.py
 GNN_GEMM_CTA2=1 timeout 120 python scripts/gemm_ab.py
 GNN_LIB_PATH=$PWD/diag/libgnn_REGSTORE.so timeout 300 python scripts/gemm_ab.py) > gpurun_out/gemm_cta2_$TAG.txt 2>&1
GNN_GEMM_CTA2=1 timeout 600 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_parity.py -q -x -k "gemm or gat_transform" -p no:cacheprovider > gpurun_out/pytest_cta2_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_cta2_$TAG.log
