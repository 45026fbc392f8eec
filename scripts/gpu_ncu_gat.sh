TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/agg_ab.py prep --once > /dev/null 2>&1
timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section InstructionStats --section SourceCounters --import-source on --clock-control none -k regex:"k_stream_g4" -o gpurun_out/prof_g4gat_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_g4gat_$TAG.log 2>&1
