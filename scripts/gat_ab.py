"""dev A/B: GAT 8x32 aggregation time with the current library vs another build
(GNN_LIB_PATH), same inputs (C5 graph)."""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

g = gs.config_graph("C5")
plan = G.Plan(g.rowptr, g.colidx, reorder=1)
H, Fh = 8, 32
HF = H * Fh
torch.manual_seed(0)
Zs = (torch.rand((g.n, HF + 2 * H), device="cuda") * 2 - 1)
Y = torch.empty((g.n, HF), device="cuda")
t = Zs[:, HF + H:]
for _ in range(3):
    G.gat_aggregate(plan, Zs, t, H, Fh, out=Y)
torch.cuda.synchronize()
a = torch.cuda.Event(enable_timing=True)
b = torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10):
    G.gat_aggregate(plan, Zs, t, H, Fh, out=Y)
b.record()
torch.cuda.synchronize()
print(f"{os.environ.get('GNN_LIB_PATH', 'current')}: GAT 8x32 {a.elapsed_time(b) / 10:.3f} ms  checksum {float(Y.double().sum()):.6e}")
