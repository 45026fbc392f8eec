# compact ring slots: full GPU suite, smoke (extended), C5 / C3 A/B
TAG=${1:-r3m}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
(timeout 600 python scripts/agg_ab.py compact
timeout 300 python scripts/agg_ab.py compact
timeout 900 python scripts/c3_ab.py compact
timeout 300 python scripts/c3_ab.py compact --prescaled) > gpurun_out/agg_ab_$TAG.txt 2>&1
