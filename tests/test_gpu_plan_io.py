"""Plan persistence (LAS runs once offline and is reused):
gnn_plan_save / gnn_plan_load / gnn_plan_create_perm on the GPU."""
import numpy as np
import pytest

import gnn_synth as gs
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402


def _agg(plan, X):
    Y = G.aggregate(plan, torch.from_numpy(X).cuda(), "sum", "gcn", relu=True)
    Z = G.gat_aggregate(plan, torch.from_numpy(X).cuda(), torch.from_numpy(X[:, :4].copy()).cuda(), 4, 8)
    torch.cuda.synchronize()
    return Y.cpu().numpy(), Z.cpu().numpy()


@pytest.mark.parametrize("with_las", [0, 1])
def test_save_load_roundtrip_bit_identical(tmp_path, with_las):
    g = gs.powerlaw(6000, 120000, 20, 2000, 1500, comm=32, rho=0.8, seed=2)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1, group_size=32, seed=5)
    path = str(tmp_path / "p.gnnplan")
    plan.save(path, with_las=bool(with_las))
    p2 = G.Plan.load(path)
    a, b = plan.export(), p2.export()
    for x, y in zip(a, b):
        assert np.array_equal(x, y)
    i1, i2 = plan.info, p2.info
    for k in ("n", "n_src", "nnz", "n_groups", "n_tiles", "n_split_rows", "n_empty_rows", "n_clusters",
              "group_size", "reorder"):
        assert i1[k] == i2[k], k
    if with_las:
        for x, y in zip(plan.export_las(), p2.export_las()):
            assert np.array_equal(x, y)
        assert i2["n_pairs"] == i1["n_pairs"]
    else:
        with pytest.raises(G.GnnError):
            p2.export_las()
    X = gs.uniform(g.n, 36, seed=1)
    for x, y in zip(_agg(plan, X), _agg(p2, X)):
        assert np.array_equal(x.view(np.uint32), y.view(np.uint32))
    # the loaded schedule is the oracle's LAS schedule
    operm, _ = oracle.las_schedule(g.rowptr, g.colidx, seed=5)
    assert np.array_equal(b[0], operm)


def test_load_rejects_corrupt_and_truncated(tmp_path):
    g = gs.random_small(300, avg_deg=5, seed=1)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    path = tmp_path / "p.gnnplan"
    plan.save(str(path))
    raw = bytearray(path.read_bytes())
    bad = tmp_path / "bad.gnnplan"
    raw2 = bytearray(raw)
    raw2[len(raw2) // 2] ^= 0x40
    bad.write_bytes(bytes(raw2))
    with pytest.raises(G.GnnError):
        G.Plan.load(str(bad))
    short = tmp_path / "short.gnnplan"
    short.write_bytes(bytes(raw[:-20]))
    with pytest.raises(G.GnnError):
        G.Plan.load(str(short))


def test_create_perm_matches_las_plan_and_rejects_non_permutation():
    g = gs.powerlaw(3000, 50000, 16, 900, 700, comm=32, rho=0.8, seed=4)
    las = G.Plan(g.rowptr, g.colidx, reorder=1, group_size=16)
    perm = las.export()[0]
    p2 = G.Plan(g.rowptr, g.colidx, perm=perm, reorder=1, group_size=16)
    for x, y in zip(las.export(), p2.export()):
        assert np.array_equal(x, y)
    X = gs.uniform(g.n, 36, seed=3)
    for x, y in zip(_agg(las, X), _agg(p2, X)):
        assert np.array_equal(x.view(np.uint32), y.view(np.uint32))
    bad = perm.copy()
    bad[0] = bad[1]
    with pytest.raises(G.GnnError):
        G.Plan(g.rowptr, g.colidx, perm=bad)
