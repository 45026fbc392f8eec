# mapping sweep session (dev)
TAG=${1:-map}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "mapping" > gpurun_out/pytest_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 900 python scripts/kbench.py map --cfg C5 > gpurun_out/kb_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/kb_$TAG.log
