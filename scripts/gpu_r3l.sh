# lean chain with compact ring slots (400 B at F=100): parity + ring depth A/B (S = 12 / 16 / 20 / 24)
TAG=${1:-r3l}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or agg2 or c5_step or nondeterministic or mapping or integer or strided or full_size or wide or tuner or trace or edgeconv" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
(for r in 1 2; do
AGG_AB_LDX1=104 timeout 600 python scripts/agg_ab.py compact_s12
for S in 16 20 24; do AGG_AB_LDX1=104 GNN_LIB_PATH=$PWD/$V/s$S/libgnn.so timeout 300 python scripts/agg_ab.py compact_s$S; done
done
timeout 900 python scripts/c3_ab.py compact) > gpurun_out/agg_ab_$TAG.txt 2>&1
