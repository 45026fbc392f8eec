# aux: load-balance report (Fig 8 analogue), compute-sanitizer memcheck / racecheck on small parity cases
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python scripts/balance_report.py C5 C3 > gpurun_out/balance_$TAG.txt 2>&1
timeout 1200 compute-sanitizer --tool memcheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "cora or small or hub" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck --racecheck-report all --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "test_aggregate_parity and hub" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_racecheck_$TAG.txt
timeout 600 compute-sanitizer --tool synccheck --target-processes all --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "test_aggregate_parity and hub" > gpurun_out/sanitizer_synccheck_$TAG.txt 2>&1
echo "rc=$?" >> gpurun_out/sanitizer_synccheck_$TAG.txt
