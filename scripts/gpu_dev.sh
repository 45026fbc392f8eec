# dev session: GPU tests + kernel comparison
TAG=${1:-dev}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 600 python scripts/kbench.py impl --cfg C5 > gpurun_out/kb_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/kb_$TAG.log
