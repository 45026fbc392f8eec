# GAT on the lean cp.async chain (GNN_CP_GAT=1) vs gather4: parity + A/B; bench with the fixed GAT routing
TAG=${1:-r4b}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GNN_CP_GAT=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "gat or GAT or straddl or attn" > gpurun_out/pytest_cpgat_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_cpgat_$TAG.log
(for r in 1 2; do timeout 600 python scripts/agg_ab.py g4gat; GNN_CP_GAT=1 timeout 600 python scripts/agg_ab.py cpgat; done) > gpurun_out/agg_ab_$TAG.txt 2>&1
GNN_CP_GAT=1 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_aggregate" -c 3 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_cpgat_$TAG.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
