TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "aggregate or gat or agg1 or agg2 or mapping or integer or rerun or nondeterministic or strided or edgeconv or chunks or attn" > gpurun_out/pytest_g4_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_g4_$TAG.log
(timeout 600 python scripts/agg_ab.py g4
GNN_AGG_CP=1 timeout 300 python scripts/agg_ab.py cp_chain
GNN_AGG_CP=0 timeout 300 python scripts/agg_ab.py reg_kernel) > gpurun_out/agg_ab_$TAG.txt 2>&1
