# sum / mean / max on the cp.async chain for every width: full GPU suite, A/B, bench, F sweep
TAG=${1:-r4a}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
(for r in 1 2; do timeout 600 python scripts/agg_ab.py cp_all; GNN_G4_SUM=1 timeout 600 python scripts/agg_ab.py g4_sum; done
timeout 600 python scripts/fsweep_ab.py cp_all) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
GNN_G4_SUM=1 timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/bench_g4sum_$TAG.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_aggregate|k_stream_g4" -c 3 -o gpurun_out/prof_aggs_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_full_$TAG.log 2>&1
