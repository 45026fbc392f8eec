# agg2 (F=256 prescaled) on the cp.async chain (8-slot ring) vs gather4
TAG=${1:-r3z}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for r in 1 2 3; do timeout 600 python scripts/agg_ab.py g4; GNN_AGG_CP=1 timeout 600 python scripts/agg_ab.py cpchain_agg2; done) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_aggregate" -c 2 env GNN_AGG_CP=1 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_cpagg2_$TAG.log 2>&1
