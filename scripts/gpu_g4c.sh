TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py tests/test_gpu_attn.py -q -x -p no:cacheprovider -k "aggregate or gat or agg2 or integer or rerun or chunks or attn" > gpurun_out/pytest_g4c_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_g4c_$TAG.log
(timeout 600 python scripts/agg_ab.py g4v8
GNN_G4_VEC=4 timeout 300 python scripts/agg_ab.py g4v4) > gpurun_out/agg_ab_$TAG.txt 2>&1
