# dev session: kbench mode + bench line (no e2e/cpu legs)
TAG=${1:-b}; KB=${2:-map100}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python scripts/kbench.py $KB > gpurun_out/kb_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/kb_$TAG.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$TAG.log
