"""How much locality a better task order could buy (dev experiment): the C5
graph's aggregation with (a) identity order, (b) LAS, (c) the generator's
planted community order (pre-relabel ids, unknown to LAS), via
gnn_plan_create_perm.  Prints kernel times."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402


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


g = gs.config_graph("C5", with_relabel=True)
rel = g.stats["relabel"]          # new id of pre-relabel node v
community_order = np.argsort(np.argsort(rel)).astype(np.int32)  # placeholder, replaced below
inv = np.empty_like(rel)
inv[rel] = np.arange(len(rel))   # pre-relabel id of new node
community_order = rel.astype(np.int32)  # task i = new id of pre-relabel node i (communities contiguous)
X2 = torch.rand(g.n, 256, device="cuda")
Y2 = torch.empty_like(X2)
Zs = torch.rand(g.n, 272, device="cuda")
Yg = torch.empty(g.n, 256, device="cuda")
X1 = torch.rand(g.n, 100, device="cuda")
Y1 = torch.empty_like(X1)
for name, kw in [("identity", dict(reorder=0)), ("LAS", dict(reorder=1)),
                 ("planted communities", dict(perm=community_order))]:
    plan = G.Plan(g.rowptr, g.colidx, **kw)
    a = timeit(lambda: G.aggregate(plan, X1, "sum", "gcn", out=Y1))
    b = timeit(lambda: G.aggregate(plan, X2, "sum", "one", out=Y2))
    c = timeit(lambda: G.gat_aggregate(plan, Zs, Zs[:, 264:], 8, 32, out=Yg))
    print(f"{name:22s}: agg F=100 gcn {a:.3f} ms | sum F=256 {b:.3f} ms | GAT 8x32 {c:.3f} ms", flush=True)
    del plan
