# lean chain: next unit's index line prefetched to L2 + ndst early (pf) vs not (pf0); source-level ncu of agg1
TAG=${1:-r3p}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or c5_step_layer1 or nondeterministic or integer or strided or full_size or tuner or edgeconv or gcn_layer" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do
timeout 600 python scripts/agg_ab.py pf
GNN_LIB_PATH=$PWD/$V/pf0/libgnn.so timeout 300 python scripts/agg_ab.py pf0
done
timeout 900 python scripts/c3_ab.py pf
GNN_LIB_PATH=$PWD/$V/pf0/libgnn.so timeout 300 python scripts/c3_ab.py pf0) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 ncu --section SourceCounters --section WarpStateStats --section InstructionStats --import-source on --clock-control none -k regex:"k_aggregate" -c 1 -o gpurun_out/prof_agg1src_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_agg1src_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_agg1src_$TAG.log
