TAG=${1:-r2s}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
timeout 600 python scripts/las_upside.py > gpurun_out/las_upside_$TAG.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 > gpurun_out/ncu_launch_$TAG.log 2>&1
