# gather4 LDS fast path: sanitizer on the gather4 GAT / sum cases, full GPU suite, A/B, bench, launch list, ncu
TAG=${1:-r3j}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "straddling or gat_aggregate_parity or (aggregate_parity and hub and 256)" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
(timeout 600 python scripts/agg_ab.py g4lds
timeout 300 python scripts/agg_ab.py g4lds
timeout 900 python scripts/c3_ab.py g4lds --prescaled
timeout 300 python scripts/c3_ab.py g4lds) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_stream_g4|k_aggregate" -c 3 -o gpurun_out/prof_aggs_$TAG -f python scripts/agg_ab.py g4 --once > gpurun_out/ncu_full_$TAG.log 2>&1
