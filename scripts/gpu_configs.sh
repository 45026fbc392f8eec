# per-config report session: C1-C4 + F sweep, C3 ncu DRAM pass, GAT/agg ncu full
TAG=${1:-cfg}; CFG=${2:-C1,C2,C4,C3,FS}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt; grep -m1 "model name" /proc/cpuinfo >> gpurun_out/nproc.txt
timeout 1500 python scripts/configs_report.py --cfg $CFG --out gpurun_out/configs_$TAG.json > gpurun_out/configs_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/configs_$TAG.log
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
  --clock-control none -k regex:k_aggregate --csv --log-file gpurun_out/c3_ncu_$TAG.csv \
  python scripts/configs_report.py --ncu-pass > gpurun_out/c3_ncu_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/c3_ncu_$TAG.log
