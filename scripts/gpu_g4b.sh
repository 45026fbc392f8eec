TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or gat or agg2 or integer or rerun or chunks" > gpurun_out/pytest_g4b_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_g4b_$TAG.log
(timeout 600 python scripts/agg_ab.py g4b) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section InstructionStats --section SourceCounters --import-source on --clock-control none -k regex:"k_stream_g4" -o gpurun_out/prof_g4b_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_g4b_$TAG.log 2>&1
