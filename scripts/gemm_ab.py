"""GEMM A/B at the C5 step's shapes (dev tool): time the tcgen05 kernel under
the env knobs GNN_GEMM_CB / GNN_GEMM_SA / GNN_GEMM_EPI8 (read once per
process) and check it against the register-fed path bit for bit and the oracle
on sampled rows.   GNN_GEMM_SA=6 python scripts/gemm_ab.py"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

M = 2449029
SHAPES = [("gemm1", M, 100, 256, True, False), ("gemm2", M, 256, 256, False, True), ("gemm3", M, 256, 272, False, False)]


def timeit(fn, iters=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(iters):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / iters


tag = " ".join(f"{k}={os.path.basename(os.environ[k])}" for k in ("GNN_GEMM_CB", "GNN_GEMM_SA", "GNN_GEMM_EPI8", "GNN_LIB_PATH") if k in os.environ)
torch.manual_seed(0)
for name, m, k, n, relu, scale in SHAPES:
    X = torch.rand(m, k, device="cuda") * 2 - 1
    W = (torch.rand(k, n, device="cuda") * 2 - 1) * float(np.sqrt(6 / (k + n)))
    rs = (torch.rand(m, device="cuda") + 0.1) if scale else None
    H = G.gemm(X, W, row_scale=rs, relu=relu)
    ms = timeit(lambda: G.gemm(X, W, row_scale=rs, relu=relu, out=H))
    G.set_gemm_impl(3)
    H3 = G.gemm(X, W, row_scale=rs, relu=relu)
    G.set_gemm_impl(0)
    torch.cuda.synchronize()
    same = bool(torch.equal(H.view(torch.int32), H3.view(torch.int32)))
    rows = torch.randint(0, m, (1024,), device="cuda")
    ref = oracle.gemm(X[rows].cpu().numpy(), W.cpu().numpy(),
                      None if rs is None else rs[rows].cpu().numpy())
    if relu:
        ref = np.maximum(ref, 0)
    err = np.abs(H[rows].cpu().numpy() - ref)
    ok = bool(np.all(err <= 1e-5 + 1e-4 * np.abs(ref)))
    tf = 2 * m * k * n / (ms * 1e-3) / 1e12
    print(f"[{tag}] {name} {m}x{k}x{n}: {ms:.3f} ms ({tf:.0f} TF/s useful, {3 * tf:.0f} issued) "
          f"tma==reg {same} oracle_ok {ok}", flush=True)
    del X, W, H, H3
    torch.cuda.empty_cache()

# GEMM3 as the bench runs it now: [Z | s | t] = Y2 W3 with the score epilogue
X = torch.rand(M, 256, device="cuda") * 2 - 1
W = (torch.rand(256, 256, device="cuda") * 2 - 1) * float(np.sqrt(6 / 512))
a_s = torch.rand(256, device="cuda") - 0.5
a_d = torch.rand(256, device="cuda") - 0.5
Z = G.gat_transform(X, W, a_s, a_d, 8, 32)
ms = timeit(lambda: G.gat_transform(X, W, a_s, a_d, 8, 32, out=Z))
print(f"[{tag}] gat_transform {M}x256x(8x32 + scores): {ms:.3f} ms", flush=True)
