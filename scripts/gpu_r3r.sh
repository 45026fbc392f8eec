TAG=${1:-r3r}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 600 python scripts/agg_ab.py default; timeout 600 python scripts/fpitch_ab.py; timeout 600 python scripts/fpitch_ab.py) > gpurun_out/fpitch_$TAG.txt 2>&1
