"""F sweep A/B on the C5 graph (dev tool): sum aggregation, weight one, for
F = 64..256 under this process's env (e.g. GNN_AGG_CP=1: cp.async chain for
F > 128 instead of gather4).  Uses agg_ab.py's cached graph/plan."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

GPATH, PPATH = "/tmp/agg_ab_c5_sym.npz", "/tmp/agg_ab_c5_sym.gnnplan"
if os.path.exists(GPATH):
    z = np.load(GPATH)
    rowptr, colidx = z["rowptr"], z["colidx"]
else:
    g = gs.config_graph("C5")
    rowptr, colidx = g.rowptr, g.colidx
    np.savez(GPATH, rowptr=rowptr, colidx=colidx)
n = len(rowptr) - 1
plan = G.Plan.load(PPATH) if os.path.exists(PPATH) else G.Plan(rowptr, colidx, reorder=1)
if not os.path.exists(PPATH):
    plan.save(PPATH)
tag = sys.argv[1] if len(sys.argv) > 1 else "default"


def timeit(fn, iters=5, warm=2):
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


out = []
for F in range(128, 257, 16):
    X = torch.rand((n, F), device="cuda")
    Y = torch.empty_like(X)
    out.append(f"{F}:{timeit(lambda: G.aggregate(plan, X, 'sum', 'one', out=Y)):.2f}")
    del X, Y
print(f"[{tag}] " + " ".join(out), flush=True)
