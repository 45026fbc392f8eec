# lean chain: weights one window ahead (default) vs at window entry (wa0): parity + A/B
TAG=${1:-r3n}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or c5_step_layer1 or nondeterministic or integer or strided or full_size or tuner or edgeconv" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do
timeout 600 python scripts/agg_ab.py wahead
GNN_LIB_PATH=$PWD/$V/wa0/libgnn.so timeout 300 python scripts/agg_ab.py wa0
done
timeout 900 python scripts/c3_ab.py wahead
GNN_LIB_PATH=$PWD/$V/wa0/libgnn.so timeout 300 python scripts/c3_ab.py wa0) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 ncu --section SpeedOfLight --section WarpStateStats --section InstructionStats --section SchedulerStats --section MemoryWorkloadAnalysis --clock-control none -k regex:"k_aggregate" -c 1 -o gpurun_out/prof_agg1_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_agg1_$TAG.log 2>&1
