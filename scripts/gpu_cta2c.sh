# CTA-pair GEMM defaults: A/B (pair off / default / EB=2 / SA=6) + GEMM parity + bench
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for cfg in "GNN_GEMM_CTA2=0" "GNN_GEMM_CTA2=1" "GNN_GEMM_EB=2" "GNN_GEMM_SL=3" "GNN_GEMM_SB=4"; do
  echo "== $cfg"; env $cfg timeout 120 python scripts/gemm_ab.py
done) > gpurun_out/gemm_cta2c_$TAG.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_bench_configs.py tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x -p no:cacheprovider > gpurun_out/pytest_cta2c_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_cta2c_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
