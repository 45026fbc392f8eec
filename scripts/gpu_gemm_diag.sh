# GEMM bottleneck diagnosis: time the C5 GEMM shapes with parts of the
# pipeline compiled out (diag/libgnn_*.so built with -DGNN_GEMM_DBG_*)
TAG=${1:-r2}
VARIANTS=${2:-"NOMMA NOEPI NOSPLIT NOW LOADONLY"}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 300 python scripts/gemm_ab.py
for v in $VARIANTS; do
  GNN_LIB_PATH=$PWD/diag/libgnn_$v.so timeout 300 python scripts/gemm_ab.py
done) > gpurun_out/gemm_diag_$TAG.txt 2>&1
