"""One launch of the bench step's dominant graph kernel on the bench's own
graph and plan (saved by bench.py under /tmp), for an ncu DRAM-traffic
capture that bench.py runs as a subprocess:
    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum ... python scripts/traffic_probe.py DIR KERNEL
KERNEL: gat_agg_8x32 | agg2_F256 | agg1_F100.  Values are random: the traffic
depends on the access pattern and the cache, not on the values."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

d, kernel = sys.argv[1], sys.argv[2]
meta = np.load(os.path.join(d, "meta.npz"))
n, F_in, F, H, Fh = (int(meta[k]) for k in ("n", "F_in", "F", "H", "Fh"))
plan = G.Plan.load(os.path.join(d, "plan.gnnplan"))
ldwe = (H * Fh + 2 * H + 7) // 8 * 8
if kernel == "gat_agg_8x32":
    Z = torch.rand(n, ldwe, device="cuda")
    Y = torch.empty(n, H * Fh, device="cuda")
    fn = lambda: G.gat_aggregate(plan, Z, Z[:, H * Fh + H:], H, Fh, out=Y)  # noqa: E731
elif kernel == "agg2_F256":
    X = torch.rand(n, F, device="cuda")
    Y = torch.empty_like(X)
    ws, wb = plan.workspace(G.gnn.GNN_OP_AGGREGATE, 0, F, 0, X.device)
    import ctypes
    fn = lambda: G.gnn._lib.gnn_gcn_aggregate_prescaled(plan.handle, ctypes.c_void_p(X.data_ptr()), F, F,  # noqa: E731
                                                       ctypes.c_void_p(Y.data_ptr()), F, 0,
                                                       ctypes.c_void_p(ws.data_ptr()), wb, None)
else:
    X = torch.rand(n, F_in, device="cuda")
    Y = torch.empty_like(X)
    fn = lambda: G.aggregate(plan, X, "sum", "gcn", out=Y)  # noqa: E731
fn()
fn()
torch.cuda.synchronize()
