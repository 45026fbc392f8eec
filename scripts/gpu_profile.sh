# profile session: ncu --set full of the aggregation kernels + GEMMs of one bench step, and the launch list
set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_aggregate|k_gemm_tc" -c 6 -o gpurun_out/prof_v8 -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_v8.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_full_v8.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v8.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_v8.log 2>&1
