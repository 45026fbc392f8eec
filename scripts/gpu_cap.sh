TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for cap in 4 3 2 1; do
  GNN_AGG_CP=0 GNN_AGG_CTAS_PER_SM=$cap timeout 300 python scripts/agg_ab.py reg_cap$cap
  GNN_AGG_CP=1 GNN_AGG_CTAS_PER_SM=$cap timeout 300 python scripts/agg_ab.py cp_cap$cap
done
GNN_AGG_CP=0 timeout 300 python scripts/agg_ab.py reg_maps --maps) > gpurun_out/agg_cap_$TAG.txt 2>&1
