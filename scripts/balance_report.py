"""Fig 8 analogue: load balance of the graph operations with and
without neighbour grouping.  "Balanced" = total worker busy time / number of
workers (perfect balance: every persistent worker busy until the end);
"Actual" = kernel span; both from gnn_set_agg_trace (%globaltimer in the
kernel).  Base = rows never split (group_size 0, one worker per row, as a
warp-per-row implementation); NG = the plan's neighbour groups.
    python scripts/balance_report.py [C5] [C3] > profiles/r02_balance.txt"""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

cfgs = [a for a in sys.argv[1:] if a.startswith("C")] or ["C5"]
trace = torch.zeros(8, dtype=torch.int64, device="cuda")
G.gnn.gnn_set_agg_trace(trace.data_ptr())


def measure(fn):
    fn()
    torch.cuda.synchronize()
    t = trace.cpu().tolist()
    busy, workers, t0, t1, units, longest = t[:6]
    return busy / workers / 1e6, (t1 - t0) / 1e6, longest / 1e6, units, workers


for cfg in cfgs:
    t = time.time()
    g = gs.config_graph(cfg)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    ng_default = plan.info["group_size"]
    print(f"{cfg}: n={g.n} nnz={g.nnz} max degree {int((g.rowptr[1:] - g.rowptr[:-1]).max())} "
          f"(gen+plan {time.time() - t:.0f}s); NG bound {ng_default}", flush=True)
    widths = [("F=100 GCN sum", 100, None), ("F=256 sum", 256, None), ("GAT 8x32", 256, (8, 32))]
    for label, ng in [("Base (no NG)", 0), ("NG", ng_default)]:
        G.set_group_size(plan, ng)
        for name, F, gat in widths:
            if gat:
                Zs = torch.rand(g.n, 272, device="cuda")
                Y = torch.empty(g.n, 256, device="cuda")
                fn = lambda: G.gat_aggregate(plan, Zs, Zs[:, 264:], 8, 32, out=Y)  # noqa: E731
            else:
                X = torch.rand(g.n, F, device="cuda")
                Y = torch.empty_like(X)
                fn = lambda: G.aggregate(plan, X, "sum", "gcn", out=Y)  # noqa: E731
            bal, act, longest, units, workers = measure(fn)
            print(f"  {label:13s} {name:14s}: balanced {bal:7.3f} ms  actual {act:7.3f} ms  "
                  f"(actual/balanced {act / bal:5.2f}; longest worker {longest:7.3f} ms; {units} units, "
                  f"{workers} workers)", flush=True)
            del Y
    del plan
    torch.cuda.empty_cache()
G.gnn.gnn_set_agg_trace(None)
