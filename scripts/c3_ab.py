"""C3 aggregation A/B (dev tool): the Reddit-shaped graph (rho 0.8, LAS + NG
plan) aggregated at F=256 with GCN weights, as configs_report.py's C3 row,
under the library / env of this process; prints ms and an output fingerprint.
The graph and plan are cached under /tmp for the next variant process."""
import hashlib
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else "default"
GPATH, PPATH = "/tmp/c3_ab.npz", "/tmp/c3_ab.gnnplan"
t0 = time.time()
if os.path.exists(GPATH):
    z = np.load(GPATH)
    rowptr, colidx = z["rowptr"], z["colidx"]
else:
    g = gs.config_graph("C3", rho=0.8)
    rowptr, colidx = g.rowptr, g.colidx
    np.savez(GPATH, rowptr=rowptr, colidx=colidx)
n = len(rowptr) - 1
plan = G.Plan.load(PPATH) if os.path.exists(PPATH) else G.Plan(rowptr, colidx, reorder=1)
if not os.path.exists(PPATH):
    plan.save(PPATH)
prep = time.time() - t0
gen = torch.Generator(device="cuda")
gen.manual_seed(3)
Hs = torch.rand((n, 256), device="cuda", generator=gen) * 2 - 1
H1 = torch.empty_like(Hs)
if "--prescaled" in sys.argv:  # the transform-first layer's form: rows pre-scaled by nsrc, x ndst in the epilogue
    import ctypes
    ws, wb = plan.workspace(G.gnn.GNN_OP_AGGREGATE, 0, 256, 0, Hs.device)
    P = lambda t: ctypes.c_void_p(t.data_ptr())  # noqa: E731
    fn = lambda: G.gnn._lib.gnn_gcn_aggregate_prescaled(plan.handle, P(Hs), 256, 256, P(H1), 256, 0, P(ws), wb,  # noqa
                                                      None)
    tag += " prescaled"
else:
    fn = lambda: G.aggregate(plan, Hs, "sum", "gcn", out=H1)  # noqa: E731
if "--once" in sys.argv:
    fn()
    torch.cuda.synchronize()
    sys.exit(0)
for _ in range(3):
    fn()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10):
    fn()
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b) / 10
fp = hashlib.sha1(H1.cpu().numpy().tobytes()).hexdigest()[:10]
print(f"[{tag}] C3 agg F=256 gcn {ms:.3f} ms | fp {fp} (prep {prep:.0f}s)", flush=True)
