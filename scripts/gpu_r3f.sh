# gather4 with GCN weights (F > 128 default; F <= 128 opt-in): parity + C5 / C3 A/B
TAG=${1:-r3f}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or agg1 or agg2 or c5_step or nondeterministic or mapping or integer or strided or full_size or wide" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
GNN_G4_NARROW=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate_parity or agg1 or c5_step_layer1 or integer or strided" > gpurun_out/pytest_narrow_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_narrow_$TAG.log
(timeout 600 python scripts/agg_ab.py default
GNN_G4_NARROW=1 timeout 300 python scripts/agg_ab.py g4narrow
GNN_G4_NARROW=1 GNN_G4_PROMO=64 timeout 300 python scripts/agg_ab.py g4narrow_p64
timeout 300 python scripts/agg_ab.py default
GNN_G4_NARROW=1 timeout 300 python scripts/agg_ab.py g4narrow
timeout 900 python scripts/c3_ab.py g4gcn
GNN_AGG_CP=1 timeout 300 python scripts/c3_ab.py cpchain
timeout 300 python scripts/c3_ab.py g4gcn
GNN_AGG_CP=1 timeout 300 python scripts/c3_ab.py cpchain) > gpurun_out/agg_ab_$TAG.txt 2>&1
