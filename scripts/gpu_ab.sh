# bench A/B: in-tree libgnn.so vs a scratch variant (GNN_LIB_PATH), alternating
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=${1:-scratch/minb3/libgnn.so}
for i in 1 2; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_base_$i.log 2>&1
  GNN_LIB_PATH=$V timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_var_$i.log 2>&1
done
