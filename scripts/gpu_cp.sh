# cp.async aggregation: parity tests, then A/B vs the register kernel and ring-depth variants
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or gat or agg1 or agg2 or mapping or integer or rerun or nondeterministic or strided or edgeconv or chunks" > gpurun_out/pytest_cp_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_cp_$TAG.log
V=paper_conf_ppopp_huangzzys21_b200/_variants
(timeout 600 python scripts/agg_ab.py cp_default
GNN_AGG_CP=0 timeout 300 python scripts/agg_ab.py reg_kernel
for v in cp4 cp6 cp5b; do
  GNN_LIB_PATH=$PWD/$V/$v/libgnn.so timeout 300 python scripts/agg_ab.py $v
done) > gpurun_out/agg_ab_$TAG.txt 2>&1
