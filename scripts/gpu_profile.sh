# profile session: ncu --set full of the aggregation kernels + the tcgen05 GEMM of one bench step
set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_aggregate|k_gemm_tc" -c 6 -o gpurun_out/prof_v2 -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_v2.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_full_v2.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v2.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_v2.log 2>&1
