# CTA-pair GEMM: ring-depth A/B + one ncu --set full capture of gat_transform under the pair
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for cfg in "GNN_GEMM_CTA2=0" "GNN_GEMM_CTA2=1" "GNN_GEMM_CTA2=1 GNN_GEMM_SB=3" "GNN_GEMM_CTA2=1 GNN_GEMM_SL=3" "GNN_GEMM_CTA2=1 GNN_GEMM_SB=3 GNN_GEMM_SL=3" "GNN_GEMM_CTA2=1 GNN_GEMM_SA=3" "GNN_GEMM_CTA2=1 GNN_GEMM_EPI8=0" "GNN_GEMM_CTA2=1 GNN_GEMM_CB=2"; do
  echo "== $cfg"; env $cfg timeout 120 python scripts/gemm_ab.py
done) > gpurun_out/gemm_cta2b_$TAG.txt 2>&1
GNN_GEMM_CTA2=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 1 -c 1 -o gpurun_out/prof_gemm3pair_$TAG -f \
  python scripts/gemm_one.py gat 2 > gpurun_out/ncu_gemm3pair_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_gemm3pair_$TAG.log
