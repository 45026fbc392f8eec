# round-2 closing session: full GPU suite, smoke, bench (all legs), launch list, ncu of the step's kernels,
# per-config report (C1-C4 + F sweep) with the C3 ncu DRAM pass
TAG=${1:-fin}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi_$TAG.txt 2>&1
nproc > gpurun_out/nproc_$TAG.txt; grep -m1 "model name" /proc/cpuinfo >> gpurun_out/nproc_$TAG.txt
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$TAG.log 2>&1
echo "ref rc=$?" >> gpurun_out/bench_ref_$TAG.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_aggregate|k_gemm_tc|k_stream_g4" -c 6 -o gpurun_out/prof_step_$TAG -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-rho0 --no-traffic > gpurun_out/ncu_full_$TAG.log 2>&1
timeout 3600 python scripts/configs_report.py --cfg C1,C2,C4,C3,FS,LSTM,ATT --out gpurun_out/configs_$TAG.json > gpurun_out/configs_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/configs_$TAG.log
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
  --clock-control none -k regex:k_aggregate --csv --log-file gpurun_out/c3_ncu_$TAG.csv \
  python scripts/configs_report.py --ncu-pass > gpurun_out/c3_ncu_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/c3_ncu_$TAG.log
