# GAT rows of 64..128 features on the lean chain (GNN_CP_GAT_NARROW=1) vs the register kernel: C2 layer, C5-graph F=128
TAG=${1:-r4m}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 900 python scripts/configs_report.py --cfg C2 --out gpurun_out/c2_reg_$TAG.json > /dev/null 2>&1; echo reg $?
GNN_CP_GAT_NARROW=1 timeout 900 python scripts/configs_report.py --cfg C2 --out gpurun_out/c2_cp_$TAG.json > /dev/null 2>&1; echo cp $?) > gpurun_out/c2_ab_$TAG.txt 2>&1
python - >> gpurun_out/c2_ab_$TAG.txt 2>&1 <<'PY'
import json
for k in ("reg", "cp"):
    d = json.load(open(f"gpurun_out/c2_{k}_r4m.json"))["C2"]
    print(k, json.dumps({kk: vv for kk, vv in d.items() if "ms" in kk or "variants" in kk})[:1500])
PY
