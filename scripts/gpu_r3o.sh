# GEMM: skip the padded K steps of the last K block (GEMM1 K = 100): parity + A/B
TAG=${1:-r3o}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_next2.py tests/test_gpu_lstm.py -q -x -p no:cacheprovider -k "gemm or gcn_layer or gat_layer or edgeconv or gat_transform or c5_step or mirrored or lstm" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do
timeout 600 python scripts/gemm_ab.py
GNN_LIB_PATH=$PWD/$V/kfull/libgnn.so timeout 600 python scripts/gemm_ab.py
done) > gpurun_out/gemm_ab_$TAG.txt 2>&1
