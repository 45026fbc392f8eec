# final code of round 2: full GPU suite, smoke, A/B, bench, launch list, ncu of the aggregation kernels and the step
TAG=${1:-r4f}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
(for r in 1 2; do timeout 600 python scripts/agg_ab.py final; GNN_G4_GAT=1 GNN_G4_SUM=1 timeout 600 python scripts/agg_ab.py g4_all; done) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_aggregate|k_gemm_tc|k_stream_g4" -c 6 -o gpurun_out/prof_step_$TAG -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_full_$TAG.log 2>&1
