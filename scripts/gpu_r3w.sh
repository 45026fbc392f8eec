# agg1 (NV = 1 cp.async ring): S1 = 12 (default) / 8 / 4
TAG=${1:-r3w}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=paper_conf_ppopp_huangzzys21_b200/_variants
(for r in 1 2; do
timeout 600 python scripts/agg_ab.py s1_12
for S in 8 4; do GNN_LIB_PATH=$PWD/$V/s1_$S/libgnn.so timeout 300 python scripts/agg_ab.py s1_$S; done
done) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 1800 python scripts/configs_report.py --cfg C3 --out gpurun_out/configs_c3_$TAG.json > gpurun_out/configs_c3_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/configs_c3_$TAG.log
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
  --clock-control none -k regex:k_aggregate --csv --log-file gpurun_out/c3_ncu_$TAG.csv \
  python scripts/configs_report.py --ncu-pass > gpurun_out/c3_ncu_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/c3_ncu_$TAG.log
