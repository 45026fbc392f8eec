# aggregation A/B: default build vs variant builds (cache policy, launch bounds) on C5
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
(timeout 600 python scripts/agg_ab.py default --maps
for v in off na minb5 minb6 minb3; do
  GNN_LIB_PATH=$PWD/$V/$v/libgnn.so timeout 300 python scripts/agg_ab.py $v
done
timeout 300 python scripts/agg_ab.py default) > gpurun_out/agg_ab_$TAG.txt 2>&1
