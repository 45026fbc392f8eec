# source-level local-memory (spill) counters of the GAT kernel + ncu full of agg1 (lean chain) + new GPU tests
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/agg_ab.py warm --once > /dev/null 2>&1
timeout 900 ncu --section SourceCounters --section WarpStateStats --import-source on --clock-control none -k regex:"k_aggregate<3" -c 1 \
  -o gpurun_out/prof_gatsrc_$TAG -f python scripts/agg_ab.py src --once > gpurun_out/ncu_gatsrc_$TAG.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_aggregate<0" -c 1 \
  -o gpurun_out/prof_agg1_$TAG -f python scripts/agg_ab.py src --once > gpurun_out/ncu_agg1_$TAG.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "trace" > gpurun_out/pytest_trace_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_trace_$TAG.log
