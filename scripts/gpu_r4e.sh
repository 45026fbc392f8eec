# NV = 2 cp.async kernels: launch bounds 3 CTAs/SM (80 registers, default) vs 4 (minb4): parity + A/B
TAG=${1:-r4e}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "aggregate or agg2 or c5_step or gat or GAT or straddl or full_size or wide or chunks" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do timeout 600 python scripts/agg_ab.py minb3; GNN_LIB_PATH=$PWD/$V/minb4/libgnn.so timeout 600 python scripts/agg_ab.py minb4; done
timeout 900 python scripts/c3_ab.py minb3; GNN_LIB_PATH=$PWD/$V/minb4/libgnn.so timeout 300 python scripts/c3_ab.py minb4) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_aggregate" -c 3 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_minb3_$TAG.log 2>&1
