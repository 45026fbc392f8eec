"""L2 residency of hot source rows: on a graph whose source
rows exceed L2 the aggregation launches the pin / unpin kernels around the
main kernel, and the output is bit-identical to a process with GNN_L2_PIN=0
(cache hints only)."""
import os
import subprocess
import sys

import numpy as np
import pytest

import gnn_synth as gs

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import gnn_synth as gs
import paper_conf_ppopp_huangzzys21_b200 as G
g = gs.powerlaw(300000, 6000000, 20, 4000, 3000, comm=64, rho=0.8, seed=11)
plan = G.Plan(g.rowptr, g.colidx, reorder=1)
X = torch.from_numpy(gs.uniform(g.n, 256, seed=3)).cuda()        # 307 MB of source rows > L2
Zs = torch.from_numpy(gs.uniform(g.n, 8 * 32 + 8, seed=4)).cuda()
t = torch.from_numpy(gs.uniform(g.n, 8, lo=-2, hi=2, seed=5)).cuda()
c0 = G.launch_count()
Y = G.aggregate(plan, X, "sum", "gcn")
c1 = G.launch_count()
Yg = G.gat_aggregate(plan, Zs, t, 8, 32)
torch.cuda.synchronize()
np.save(sys.argv[2], np.concatenate([Y.cpu().numpy().view(np.uint32).ravel(), Yg.cpu().numpy().view(np.uint32).ravel()]))
print(c1 - c0)
"""


def _run(tmp_path, pin):
    out = tmp_path / f"y{pin}.npy"
    env = dict(os.environ, GNN_L2_PIN=str(pin))
    r = subprocess.run([sys.executable, "-c", SCRIPT, ROOT, str(out)], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    return np.load(out), int(r.stdout.strip().splitlines()[-1])


def test_l2_residency_is_bit_identical_and_runs(tmp_path):
    y1, n1 = _run(tmp_path, 1)
    y0, n0 = _run(tmp_path, 0)
    assert np.array_equal(y1, y0)
    assert n1 == n0 + 2, (n1, n0)  # pin + unpin around the aggregation kernel
