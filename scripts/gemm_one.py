"""Launch one C5 GEMM shape a few times (for ncu captures; dev tool).
    python scripts/gemm_one.py gat|gemm1|gemm2 [reps]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

M = 2449029
which = sys.argv[1] if len(sys.argv) > 1 else "gat"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
torch.manual_seed(0)
k = 100 if which == "gemm1" else 256
X = torch.rand(M, k, device="cuda") * 2 - 1
W = (torch.rand(k, 256, device="cuda") * 2 - 1) * float(np.sqrt(6 / (k + 256)))
if which == "gat":
    a_s = torch.rand(256, device="cuda") - 0.5
    a_d = torch.rand(256, device="cuda") - 0.5
    Z = G.gat_transform(X, W, a_s, a_d, 8, 32)
    for _ in range(reps):
        G.gat_transform(X, W, a_s, a_d, 8, 32, out=Z)
else:
    rs = (torch.rand(M, device="cuda") + 0.1) if which == "gemm2" else None
    H = G.gemm(X, W, row_scale=rs, relu=which == "gemm1")
    for _ in range(reps):
        G.gemm(X, W, row_scale=rs, relu=which == "gemm1", out=H)
torch.cuda.synchronize()
print("ok", which)
