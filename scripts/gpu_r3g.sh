# lean chain v2 (IMAD.WIDE row addresses, full-batch fast path): parity + A/B + ncu
TAG=${1:-r3g}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or agg2 or c5_step or nondeterministic or mapping or integer or strided or full_size or wide or tuner" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(timeout 600 python scripts/agg_ab.py lean2
timeout 300 python scripts/agg_ab.py lean2
timeout 900 python scripts/c3_ab.py lean2
timeout 300 python scripts/c3_ab.py lean2) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 ncu --section SpeedOfLight --section WarpStateStats --section InstructionStats --section SchedulerStats --section MemoryWorkloadAnalysis --clock-control none -k regex:"k_aggregate" -c 1 -o gpurun_out/prof_agg1_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_agg1_$TAG.log 2>&1
