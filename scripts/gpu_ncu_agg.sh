# ncu of the aggregation kernels (gather4 vs register) on C5
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/agg_ab.py prep --once > /dev/null 2>&1   # builds the /tmp graph + plan cache
timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section LaunchStats --section Occupancy --section SourceCounters --import-source on --clock-control none -k regex:"k_stream_g4|k_aggregate" -o gpurun_out/prof_g4_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_g4_$TAG.log 2>&1
GNN_AGG_CP=0 timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section LaunchStats --section Occupancy --section SourceCounters --import-source on --clock-control none -k regex:"k_aggregate" -o gpurun_out/prof_reg_$TAG -f python scripts/agg_ab.py reg --once > gpurun_out/ncu_reg_$TAG.log 2>&1
