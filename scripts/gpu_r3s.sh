# experiment: hot source rows (top-K by out-degree) pinned evict_last in L2 around each aggregation
TAG=${1:-r3s}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(for r in 1 2; do for K in 0 30000 60000 120000; do AGG_AB_PIN=$K timeout 600 python scripts/agg_ab.py pin; done; done) > gpurun_out/agg_ab_$TAG.txt 2>&1
for K in 0 60000; do AGG_AB_PIN=$K timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_stream_g4|k_aggregate" python scripts/agg_ab.py g4 --once > gpurun_out/ncu_pin${K}_$TAG.log 2>&1; done
