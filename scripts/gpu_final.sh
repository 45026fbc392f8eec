# round-end session: full GPU tests, bench (all legs), launch list, ncu of the bench kernels,
# ncu of the NEXT-3/4 kernels, per-config report for the small configs
TAG=${1:-final}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash scripts/gpu_full.sh $TAG
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_sage_lstm$" -c 1 -o gpurun_out/prof_lstm_$TAG -f \
  python scripts/kbench.py lstm > gpurun_out/ncu_lstm_$TAG.log 2>&1
timeout 1500 python scripts/configs_report.py --cfg C1,C2,C4,LSTM --out gpurun_out/configs_$TAG.json > gpurun_out/configs_$TAG.log 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
