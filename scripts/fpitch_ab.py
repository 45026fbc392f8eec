"""F x row-pitch A/B on the C5 graph (dev tool): sum aggregation (weight one
and GCN weights) for F in {96, 100, 112, 128} at pitch F and at pitch 128,
to separate row width from row alignment.  Uses agg_ab.py's cached graph/plan."""
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


for F in (96, 100, 112, 128):
    for pitch in sorted({F, 128}):
        X = torch.rand((n, pitch), device="cuda")[:, :F]
        Y = torch.empty((n, F), device="cuda")
        t1 = timeit(lambda: G.aggregate(plan, X, "sum", "one", out=Y))
        t2 = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y))
        print(f"F={F} pitch={pitch}: one {t1:.3f} ms | gcn {t2:.3f} ms", flush=True)
        del X, Y
