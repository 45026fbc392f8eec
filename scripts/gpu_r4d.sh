# per-config report refresh with the final defaults: F sweep, Table 2 scores (C2, C5), GraphSAGE-LSTM, C4, C1, C2
TAG=${1:-r4d}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python scripts/configs_report.py --cfg C1,C2,C4,FS,ATT,LSTM --out gpurun_out/configs_$TAG.json > gpurun_out/configs_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/configs_$TAG.log
