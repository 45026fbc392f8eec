# streaming lean chain across units: parity + A/B (stream/64 regs, stream/80 regs, per-unit)
TAG=${1:-r3i}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or agg2 or c5_step or nondeterministic or mapping or integer or strided or full_size or wide or tuner or trace or gat or GAT or straddl or chunks" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(timeout 600 python scripts/agg_ab.py stream
GNN_LIB_PATH=$PWD/$V/minb3/libgnn.so timeout 300 python scripts/agg_ab.py stream_minb3
GNN_LIB_PATH=$PWD/$V/nostream/libgnn.so timeout 300 python scripts/agg_ab.py perunit
timeout 300 python scripts/agg_ab.py stream
GNN_LIB_PATH=$PWD/$V/minb3/libgnn.so timeout 300 python scripts/agg_ab.py stream_minb3
GNN_LIB_PATH=$PWD/$V/nostream/libgnn.so timeout 300 python scripts/agg_ab.py perunit
timeout 900 python scripts/c3_ab.py stream
GNN_LIB_PATH=$PWD/$V/minb3/libgnn.so timeout 300 python scripts/c3_ab.py stream_minb3
GNN_LIB_PATH=$PWD/$V/nostream/libgnn.so timeout 300 python scripts/c3_ab.py perunit
GNN_AGG_CP=1 timeout 300 python scripts/agg_ab.py stream_cpall
GNN_AGG_CP=1 GNN_LIB_PATH=$PWD/$V/minb3/libgnn.so timeout 300 python scripts/agg_ab.py stream_minb3_cpall) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 ncu --section SpeedOfLight --section WarpStateStats --section InstructionStats --section SchedulerStats --section MemoryWorkloadAnalysis --clock-control none -k regex:"k_aggregate" -c 1 -o gpurun_out/prof_agg1_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_agg1_$TAG.log 2>&1
