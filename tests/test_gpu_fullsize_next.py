"""Full-size (BASELINE.json C5, products-shaped: 2.45M nodes, 123.7M CSR
entries) parity of the fused attention aggregations (a7 GAT 8x32 as in the
bench, NEXT-4 Table 2 scores) and the NEXT-3 GraphSAGE-LSTM layer, in the
bench's launch configuration (LAS plan, automatic mapping), on sampled rows
(2,048 random + the 32 largest; rows are independent) vs the oracle."""
import numpy as np
import pytest

import gnn_synth as gs
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover - CPU box
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402

RTOL, ATOL = 1e-4, 1e-5


def close(got, ref, what):
    err = np.abs(got.astype(np.float64) - ref)
    bad = err > ATOL + RTOL * np.abs(ref)
    assert not bad.any(), f"{what}: {bad.sum()} / {bad.size} outside tol, max abs err {err.max():.3e}"


@pytest.fixture(scope="module")
def c5():
    g = gs.config_graph("C5")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    rng = np.random.default_rng(0)
    deg = np.diff(g.rowptr)
    rows = np.unique(np.concatenate([rng.choice(g.n, 2048, replace=False), np.argsort(deg)[-32:]]))
    yield g, plan, rows
    del plan


@pytest.mark.parametrize("score", ["gat", "sym", "gaan"])
def test_c5_attention_full(c5, score):
    g, plan, rows = c5
    H, Fh = 8, 32
    F = H * Fh
    extra = {"gat": H, "sym": 2 * H, "gaan": F}[score]
    Zs = gs.uniform(g.n, F + extra, seed=31)
    Tv = {"gat": gs.uniform(g.n, H, seed=32), "sym": None, "gaan": gs.uniform(g.n, F, lo=-0.3, hi=0.3, seed=33)}[score]
    Zd = torch.from_numpy(Zs).cuda()
    Td = None if Tv is None else torch.from_numpy(Tv).cuda()
    if score == "gat":
        Y = G.gat_aggregate(plan, Zd, Td, H, Fh, 0.2).cpu().numpy()
    else:
        Y = G.attn_aggregate(plan, score, Zd, H, Fh, Td).cpu().numpy()
    del Zd, Td
    ref = oracle.attn_aggregate(g.rowptr, g.colidx, score, Zs, H, Fh, Tv=Tv, rows=rows)
    close(Y[rows], ref, f"C5 {score} 8x32")


def test_c5_sage_lstm_full(c5):
    g, plan, rows = c5
    f_in, F, F_out, T = 32, 32, 32, 16
    rng = np.random.default_rng(4)
    P = {k: rng.uniform(-0.3, 0.3, size=s).astype(np.float32) for k, s in
         dict(W_ih=(4 * F, f_in), W_hh=(4 * F, F), b_ih=(4 * F,), b_hh=(4 * F,), W_self=(F_out, f_in),
              W_neigh=(F_out, F), bias=(F_out,)).items()}
    X = gs.uniform(g.n, f_in, seed=5)
    Pd = [torch.from_numpy(P[k]).cuda() for k in ("W_ih", "W_hh", "b_ih", "b_hh", "W_self", "W_neigh", "bias")]
    Y = G.sage_lstm_layer(plan, torch.from_numpy(X).cuda(), *Pd, T=T, seed=9).cpu().numpy()
    table = oracle.sample_neighbors(g.rowptr, g.colidx, T, 9)
    ref = oracle.sage_lstm(X, table, **P, rows=rows)
    close(Y[rows], ref, "C5 GraphSAGE-LSTM")
