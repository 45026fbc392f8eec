# GAT on the gather4 kernel: merged score gather + quad fast path vs register kernel (same box)
TAG=${1:-r3b}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GNN_G4_GAT=1 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "gat or GAT" > gpurun_out/pytest_g4gat_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_g4gat_$TAG.log
(timeout 600 python scripts/agg_ab.py default
GNN_G4_GAT=1 timeout 300 python scripts/agg_ab.py g4gat_merged
GNN_G4_GAT=1 GNN_G4_MERGED=0 timeout 300 python scripts/agg_ab.py g4gat_two
timeout 300 python scripts/agg_ab.py default
GNN_G4_GAT=1 timeout 300 python scripts/agg_ab.py g4gat_merged) > gpurun_out/agg_ab_$TAG.txt 2>&1
GNN_G4_GAT=1 timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section InstructionStats --section LaunchStats --section Occupancy --clock-control none -k regex:"k_stream_g4" -c 2 -o gpurun_out/prof_g4_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_g4_$TAG.log 2>&1
timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section WarpStateStats --section SchedulerStats --section InstructionStats --section LaunchStats --section Occupancy --clock-control none -k regex:"k_aggregate" -c 2 -o gpurun_out/prof_reg_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_reg_$TAG.log 2>&1
