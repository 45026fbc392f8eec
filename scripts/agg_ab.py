"""Aggregation A/B on the C5 graph (dev tool): times the three graph kernels
of the bench step (agg1 F=100 GCN, agg2 F=256 prescaled, GAT 8x32) with the
library in GNN_LIB_PATH (variant builds) and prints an output fingerprint, so
variants can be compared for speed and bit-identity.  The C5 graph and its
LAS plan are cached under /tmp (gnn_plan_save / gnn_plan_load) for the next
variant process of the same session.
    GNN_LIB_PATH=.../libgnn.so python scripts/agg_ab.py [tag] [--maps]"""
import ctypes
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

tag = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("--") else os.path.basename(
    os.path.dirname(G.gnn.LIB_PATH))
GPATH, PPATH = "/tmp/agg_ab_c5_sym.npz", "/tmp/agg_ab_c5_sym.gnnplan"
t0 = time.time()
if os.path.exists(GPATH):
    z = np.load(GPATH)
    rowptr, colidx = z["rowptr"], z["colidx"]
else:
    g = gs.config_graph("C5")
    rowptr, colidx = g.rowptr, g.colidx
    np.savez(GPATH, rowptr=rowptr, colidx=colidx)
n, nnz = len(rowptr) - 1, int(rowptr[-1])
if os.path.exists(PPATH):
    plan = G.Plan.load(PPATH)
else:
    plan = G.Plan(rowptr, colidx, reorder=1)
    plan.save(PPATH)
prep = time.time() - t0


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


def fp(t):
    torch.cuda.synchronize()
    return hashlib.sha1(t.cpu().numpy().tobytes()).hexdigest()[:10]


gen = torch.Generator(device="cuda")
gen.manual_seed(1)
LDX1 = int(os.environ.get("AGG_AB_LDX1", "100"))  # row pitch of agg1's X (the bench pads 100 -> 104)
X1 = (torch.rand(n, LDX1, device="cuda", generator=gen) * 2 - 1)[:, :100]
Y1 = torch.empty((n, 100), device="cuda")
X2 = torch.rand(n, 256, device="cuda", generator=gen) * 2 - 1
Y2 = torch.empty_like(X2)
Hh, Fh = 8, 32
Zs = torch.rand(n, 272, device="cuda", generator=gen) * 2 - 1
Yg = torch.empty(n, 256, device="cuda")
ws, wb = plan.workspace(G.gnn.GNN_OP_AGGREGATE, 0, 256, 0, torch.device("cuda"))
lib = G.gnn._lib
P = lambda t: ctypes.c_void_p(t.data_ptr())  # noqa: E731


def agg2():
    assert lib.gnn_gcn_aggregate_prescaled(plan.handle, P(X2), 256, 256, P(Y2), 256, 0, P(ws), wb, None) == 0


def run(label):
    a = timeit(lambda: G.aggregate(plan, X1, "sum", "gcn", out=Y1))
    b = timeit(agg2)
    c = timeit(lambda: G.gat_aggregate(plan, Zs, Zs[:, 264:], Hh, Fh, out=Yg))
    print(f"[{tag}{label}] agg1 F=100 {a:.3f} ms | agg2 F=256 {b:.3f} ms | GAT 8x32 {c:.3f} ms | "
          f"fp {fp(Y1)} {fp(Y2)} {fp(Yg)} (prep {prep:.0f}s)", flush=True)


if "--once" in sys.argv:  # one call of each kernel (for ncu)
    G.aggregate(plan, X1, "sum", "gcn", out=Y1)
    agg2()
    G.gat_aggregate(plan, Zs, Zs[:, 264:], Hh, Fh, out=Yg)
    torch.cuda.synchronize()
    sys.exit(0)
run("")
if "--maps" in sys.argv:
    for m in [(8, 32, 1), (8, 16, 2), (4, 32, 2), (4, 16, 2), (4, 32, 1), (8, 8, 4)]:
        G.set_agg_mapping(*m)
        run(f" map{m}")
    G.set_agg_mapping(0, 0, 0)
