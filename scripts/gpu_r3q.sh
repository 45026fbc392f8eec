# unit claims two ahead (default) vs one ahead (claim1): parity + A/B (agg1 / C3 and the register kernels via --maps)
TAG=${1:-r3q}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "aggregate or agg1 or c5_step_layer1 or nondeterministic or integer or strided or full_size or tuner or edgeconv or gcn_layer or gat or trace or attn or score" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do
timeout 600 python scripts/agg_ab.py claim2
GNN_LIB_PATH=$PWD/$V/claim1/libgnn.so timeout 300 python scripts/agg_ab.py claim1
done
GNN_G4_GAT=0 timeout 300 python scripts/agg_ab.py claim2_gatreg
GNN_G4_GAT=0 GNN_LIB_PATH=$PWD/$V/claim1/libgnn.so timeout 300 python scripts/agg_ab.py claim1_gatreg
timeout 900 python scripts/c3_ab.py claim2
GNN_LIB_PATH=$PWD/$V/claim1/libgnn.so timeout 300 python scripts/c3_ab.py claim1) > gpurun_out/agg_ab_$TAG.txt 2>&1
