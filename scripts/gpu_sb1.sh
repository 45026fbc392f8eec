# GEMM A/B: W ring 1 stage + deeper X ring (GNN_GEMM_SB1=1) vs default
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/kbench.py gemm > gpurun_out/kb_def.log 2>&1
GNN_GEMM_SB1=1 timeout 300 python scripts/kbench.py gemm > gpurun_out/kb_sb1.log 2>&1
timeout 300 python scripts/kbench.py gemm > gpurun_out/kb_def2.log 2>&1
