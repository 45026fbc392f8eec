# C3 (F=256, GCN weights: the cp.async chain with NV = 2): ring depth S2 = 6 (default) / 4 / 8 / 12
TAG=${1:-r3u}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
(timeout 900 python scripts/c3_ab.py s2_6
for r in 1 2; do
for S in 4 8 12; do GNN_LIB_PATH=$PWD/$V/s2_$S/libgnn.so timeout 300 python scripts/c3_ab.py s2_$S; done
timeout 300 python scripts/c3_ab.py s2_6
done) > gpurun_out/c3_ab_$TAG.txt 2>&1
