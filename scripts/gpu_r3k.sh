# agg1 input pitch 100 vs 104 (sector-aligned rows) A/B + the bench-step parity with the padded Xs
TAG=${1:-r3k}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_multirank.py tests/test_gpu_next2.py -q -p no:cacheprovider -k "c5_step or two_ranks or mirrored" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(timeout 600 python scripts/agg_ab.py ld100
AGG_AB_LDX1=104 timeout 300 python scripts/agg_ab.py ld104
timeout 300 python scripts/agg_ab.py ld100
AGG_AB_LDX1=104 timeout 300 python scripts/agg_ab.py ld104
AGG_AB_LDX1=128 timeout 300 python scripts/agg_ab.py ld128) > gpurun_out/agg_ab_$TAG.txt 2>&1
AGG_AB_LDX1=104 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_aggregate" -c 1 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_ld104_$TAG.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_aggregate" -c 1 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_ld100_$TAG.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
