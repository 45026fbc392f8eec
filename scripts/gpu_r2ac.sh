# lean cp chain: edges per commit group (U) and ring depth (S) A/B on C5 agg1 + parity
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 600 python scripts/agg_ab.py U2
 for v in NOXB U1 U4 S16U4 S16U2 CPLEGACY; do GNN_LIB_PATH=$PWD/diag/libgnn_$v.so timeout 300 python scripts/agg_ab.py $v; done
 timeout 300 python scripts/agg_ab.py U2) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench_configs.py -q -x -p no:cacheprovider -k "aggregate or cp or sum or mean or max or agg1 or prescaled or gat or att or edgeconv" > gpurun_out/pytest_lean_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_lean_$TAG.log
