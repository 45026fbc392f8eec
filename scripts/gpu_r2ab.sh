# lean cp chain A/B (agg1) vs the legacy chain + GAT bound-slack diagnosis on the bench's own inputs
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 600 python scripts/agg_ab.py lean
 GNN_LIB_PATH=$PWD/diag/libgnn_CPLEGACY.so timeout 300 python scripts/agg_ab.py legacy
 timeout 300 python scripts/agg_ab.py lean) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 python scripts/gat_slack.py > gpurun_out/gat_slack_$TAG.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "aggregate or cp or sum or mean or max" > gpurun_out/pytest_lean_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_lean_$TAG.log
