"""NEXT-3 GraphSAGE-LSTM on the GPU (through the C-ABI) vs the oracle
(Fig 6; reading R13).  Sampling is integer work: bit-exact.  The
layer is fp32 (3xTF32 pre-transform, fp32 cells) vs the fp64 oracle within
the north_star tolerance |g - r| <= 1e-5 + 1e-4 |r|."""
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


def T_(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def close(got, ref, what):
    err = np.abs(got.astype(np.float64) - ref)
    bad = err > ATOL + RTOL * np.abs(ref)
    assert not bad.any(), f"{what}: {bad.sum()} outside tol, max abs err {err.max():.3e}"


def params(f_in, F, F_out, seed, scale=0.3):
    rng = np.random.default_rng(seed)
    u = lambda *s: rng.uniform(-scale, scale, size=s).astype(np.float32)  # noqa: E731
    return dict(W_ih=u(4 * F, f_in), W_hh=u(4 * F, F), b_ih=u(4 * F), b_hh=u(4 * F), W_self=u(F_out, f_in),
                W_neigh=u(F_out, F), bias=u(F_out))


def hub_graph():
    rng = np.random.default_rng(0)
    rows = []
    for v in range(500):
        if v % 13 == 0:
            rows.append([])
        elif v == 7:
            rows.append(sorted(rng.integers(0, 500, size=3000).tolist()))
        else:
            rows.append(sorted(rng.integers(0, 500, size=int(rng.integers(1, 40))).tolist()))
    return gs.from_rows(rows)


GRAPHS = {"hub": hub_graph, "cora": lambda: gs.config_graph("C1"),
          "small": lambda: gs.random_small(300, avg_deg=5, seed=8, allow_empty=True)}


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("T,seed", [(16, 0), (1, 3), (32, 12345678901234)])
def test_sample_neighbors_bit_exact(gname, T, seed):
    g = GRAPHS[gname]()
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    tab = G.sample_neighbors(plan, T, seed).cpu().numpy()
    assert np.array_equal(tab, oracle.sample_neighbors(g.rowptr, g.colidx, T, seed))


@pytest.fixture
def impl():
    return 0  # the SIMT cells (the tcgen05 / mma.sync cell variants measured slower and were removed in r02)


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("f_in,F_out,T", [(32, 32, 16), (37, 7, 5), (8, 32, 1)])
def test_sage_lstm_layer_parity(gname, f_in, F_out, T, impl):
    g = GRAPHS[gname]()
    P = params(f_in, 32, F_out, 21)
    X = gs.uniform(g.n, f_in, seed=22)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    Y = G.sage_lstm_layer(plan, T_(X), *(T_(P[k]) for k in ("W_ih", "W_hh", "b_ih", "b_hh", "W_self", "W_neigh",
                                                             "bias")), T=T, seed=99)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, T, 99)
    ref = oracle.sage_lstm(X, table, **P)
    close(Y.cpu().numpy(), ref, f"sage lstm {gname} f_in={f_in} F_out={F_out} T={T}")


def test_sage_lstm_aggregate_from_host_pretransform(impl):
    """The fused cell kernel alone: GS (gates interleaved per unit, then the
    self term) prepared on the host in fp64 from the oracle's definition."""
    g = GRAPHS["small"]()
    f_in, F, F_out, T = 32, 32, 32, 16
    P = params(f_in, F, F_out, 5, scale=1.0)
    X = gs.uniform(g.n, f_in, seed=6)
    Xd = X.astype(np.float64)
    G4 = Xd @ P["W_ih"].astype(np.float64).T + P["b_ih"] + P["b_hh"]        # [n, 4F] blocks i, f, z, o
    inter = G4.reshape(g.n, 4, F).transpose(0, 2, 1).reshape(g.n, 4 * F)  # column 4j+g
    S = Xd @ P["W_self"].astype(np.float64).T + P["bias"]
    GS = np.concatenate([inter, S], axis=1).astype(np.float32)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, T, 4)
    plan = G.Plan(g.rowptr, g.colidx)
    Y = G.sage_lstm_aggregate(plan, T_(table), T_(GS), T_(P["W_hh"]), T_(P["W_neigh"]))
    close(Y.cpu().numpy(), oracle.sage_lstm(X, table, **P), "sage lstm aggregate")


def test_sage_lstm_rejects_unsupported_hidden_size():
    g = GRAPHS["small"]()
    plan = G.Plan(g.rowptr, g.colidx)
    P = params(8, 16, 8, 1)
    with pytest.raises(G.GnnError) as e:
        G.sage_lstm_layer(plan, T_(gs.uniform(g.n, 8, seed=1)), *(T_(P[k]) for k in ("W_ih", "W_hh", "b_ih", "b_hh",
                                                                                   "W_self", "W_neigh", "bias")))
    assert e.value.status == 6


def test_sage_lstm_rerun_identical(impl):
    g = GRAPHS["hub"]()
    P = params(32, 32, 32, 2)
    X = T_(gs.uniform(g.n, 32, seed=3))
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    args = [T_(P[k]) for k in ("W_ih", "W_hh", "b_ih", "b_hh", "W_self", "W_neigh", "bias")]
    a = G.sage_lstm_layer(plan, X, *args, T=16, seed=5).cpu()
    b = G.sage_lstm_layer(plan, X, *args, T=16, seed=5).cpu()
    assert torch.equal(a, b)
