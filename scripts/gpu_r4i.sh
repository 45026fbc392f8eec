# agg1 ring depth S1 = 12 (default) vs 8, three same-box pairs
TAG=${1:-r4i}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
(for r in 1 2 3; do timeout 600 python scripts/agg_ab.py s1_12; GNN_LIB_PATH=$PWD/$V/s1_8/libgnn.so timeout 600 python scripts/agg_ab.py s1_8; done) > gpurun_out/agg_ab_$TAG.txt 2>&1
