# bench A/B on one box: GEMM column blocks on (default) vs GNN_GEMM_CB=0, alternating
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for i in 1 2; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/cbab_on_$i.log 2>&1
  GNN_GEMM_CB=0 timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/cbab_off_$i.log 2>&1
done
