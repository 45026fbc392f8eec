# a4 rule for 128 < F < 256: gather4 (default) vs the cp.async chain (GNN_AGG_CP=1), weight one, C5
TAG=${1:-r3y}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for r in 1 2; do timeout 600 python scripts/fsweep_ab.py g4; GNN_AGG_CP=1 timeout 600 python scripts/fsweep_ab.py cpchain; done) > gpurun_out/fsweep_ab_$TAG.txt 2>&1
