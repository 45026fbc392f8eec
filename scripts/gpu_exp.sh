set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python scripts/stream_bench.py > gpurun_out/stream_bench.log 2>&1; echo "rc=$?" >> gpurun_out/stream_bench.log
