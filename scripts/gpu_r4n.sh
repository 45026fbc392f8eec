TAG=${1:-r4n}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_attn.py tests/test_gpu_bench_configs.py tests/test_gpu_kernel_equivalence.py -q -p no:cacheprovider -k "gat or GAT or attn or c5_step or straddl or equivalence or bit_identical" > gpurun_out/pytest_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
