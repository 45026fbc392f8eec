# gather4 L2 promotion A/B (GAT merged on gather4, agg2) + DRAM bytes per variant
TAG=${1:-r3d}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 600 python scripts/agg_ab.py default
GNN_G4_GAT=1 timeout 300 python scripts/agg_ab.py g4gat_auto
GNN_G4_GAT=1 GNN_G4_PROMO=0 timeout 300 python scripts/agg_ab.py g4gat_p0
GNN_G4_GAT=1 GNN_G4_PROMO=128 timeout 300 python scripts/agg_ab.py g4gat_p128
GNN_G4_GAT=1 GNN_G4_PROMO=256 timeout 300 python scripts/agg_ab.py g4gat_p256
GNN_G4_GAT=1 GNN_G4_MERGED=0 timeout 300 python scripts/agg_ab.py g4gat_two_auto
GNN_AGG_CP=1 timeout 300 python scripts/agg_ab.py cpchain_all
timeout 300 python scripts/agg_ab.py default
GNN_G4_GAT=1 timeout 300 python scripts/agg_ab.py g4gat_auto) > gpurun_out/agg_ab_$TAG.txt 2>&1
for v in auto:-1 p0:0 p256:256; do n=${v%%:*}; pr=${v##*:}; [ $pr = -1 ] && unset GNN_G4_PROMO || export GNN_G4_PROMO=$pr
GNN_G4_GAT=1 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_stream_g4" -c 2 python scripts/agg_ab.py g4 --once > gpurun_out/ncu_promo_${n}_$TAG.log 2>&1; done
