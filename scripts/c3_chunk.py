"""C3 (Reddit-shaped, n = 233K, avg degree 492) aggregation at F = 256 with
the feature columns processed in chunks whose source slice fits L2 (dev
tool): n x Fc x 4 B <= ~60 MB makes every source row come from DRAM about
once per chunk (the N*Feat bytes of P:443-449) instead of ~190 times.  Each
feature's R9 chain is independent of the others, so chunked output must be
bit-identical to the one-shot launch.
    python scripts/c3_chunk.py"""
import hashlib
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
g = gs.config_graph(cfg)
plan = G.Plan(g.rowptr, g.colidx, reorder=1)
n = g.n
F = 256
gen = torch.Generator(device="cuda")
gen.manual_seed(3)
X = torch.rand(n, F, device="cuda", generator=gen) * 2 - 1
Y = torch.empty_like(X)


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


def fp(t):
    torch.cuda.synchronize()
    return hashlib.sha1(t.cpu().numpy().tobytes()).hexdigest()[:10]


for weight in ("gcn", "one"):
    for fc in (256, 128, 64, 32):
        def run():
            for c0 in range(0, F, fc):
                G.aggregate(plan, X[:, c0:c0 + fc], "sum", weight, out=Y[:, c0:c0 + fc])
        Y.zero_()
        ms = timeit(run)
        print(f"[{cfg} n={n} nnz={g.nnz}] weight={weight} chunk {fc:3d} ({F // fc} launches, "
              f"{n * fc * 4 / 1e6:.0f} MB source slice): {ms:.3f} ms  fp {fp(Y)}", flush=True)
    for m in [(4, 16, 1), (4, 32, 1), (8, 8, 1), (4, 8, 2)]:
        G.set_agg_mapping(*m)

        def run64():
            for c0 in range(0, F, 64):
                G.aggregate(plan, X[:, c0:c0 + 64], "sum", weight, out=Y[:, c0:c0 + 64])
        ms = timeit(run64)
        print(f"  weight={weight} chunk 64 mapping {m}: {ms:.3f} ms  fp {fp(Y)}", flush=True)
        G.set_agg_mapping(0, 0, 0)
