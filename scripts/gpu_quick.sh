# quick dev session: a subset of GPU tests (-k EXPR) + a kbench mode
# usage: bash scripts/gpu_quick.sh TAG "pytest -k expr" "kbench args"
TAG=${1:-q}; K=${2:-gat}; KB=${3:-map100}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "$K" > gpurun_out/pytest_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 900 python scripts/kbench.py $KB > gpurun_out/kb_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/kb_$TAG.log
