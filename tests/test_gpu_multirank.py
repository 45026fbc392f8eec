"""a10 on the GPU: the row-partitioned C5-style step (model.RowPartitionedGCNGAT)
with P = 2 ranks sharing one B200 (gloo, exchange staged through host memory,
since this environment has one GPU) is bit-identical to P = 1, and P = 1
matches the oracle on sampled rows (R10, c10)."""
import os
import socket

import numpy as np
import pytest

import gnn_synth as gs

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)


def _inputs(Fh=16):
    g = gs.powerlaw(30000, 600000, 20, 4000, 3000, comm=64, rho=0.8, seed=5)
    F_in, F, Hh = 100, 64, 4
    X = gs.uniform(g.n, F_in, seed=1)
    W1 = gs.uniform(F_in, F, lo=-0.2, hi=0.2, seed=2)
    W2 = gs.uniform(F, F, lo=-0.25, hi=0.25, seed=3)
    W3 = gs.uniform(F, Hh * Fh, lo=-0.25, hi=0.25, seed=4)
    a_s = gs.uniform(1, Hh * Fh, lo=-0.5, hi=0.5, seed=5)[0]
    a_d = gs.uniform(1, Hh * Fh, lo=-0.5, hi=0.5, seed=6)[0]
    return g, X, W1, W2, W3, a_s, a_d, Hh, Fh


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, overlap=False, exchange="nccl", Fh=16):
    try:
        import torch.distributed as dist
        from paper_conf_ppopp_huangzzys21_b200.model import RowPartitionedGCNGAT
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        g, X, W1, W2, W3, a_s, a_d, Hh, Fh = _inputs(Fh)
        m = RowPartitionedGCNGAT(g.rowptr, g.colidx, W1, W2, W3, a_s, a_d, Hh, Fh, rank=rank, world=world,
                                 reorder=1, staged_allgather=True, overlap=overlap, exchange=exchange)
        m.load_input(torch.from_numpy(X), non_blocking=False)
        Y = m.step().cpu().numpy()
        if exchange == "peer":  # a second step over the same IPC buffers, then unmap / free
            Y2 = m.step().cpu().numpy()
            assert np.array_equal(Y.view(np.uint32), Y2.view(np.uint32)), "peer exchange rerun differs"
            m.close()
        if overlap:  # layer outputs too (the overlapped path is checked layer by layer)
            Y = (m.Y1.cpu().numpy(), m.Y2.cpu().numpy(), Y, m.step().cpu().numpy())
        parts = [None] * world
        dist.all_gather_object(parts, Y)
        if rank == 0:
            q.put(tuple(np.concatenate([pp[i] for pp in parts]) for i in range(4)) if overlap
                  else np.concatenate(parts))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put(repr(e))


def test_two_ranks_bit_identical_to_one_and_oracle():
    import torch.multiprocessing as mp

    import oracle
    from paper_conf_ppopp_huangzzys21_b200.model import RowPartitionedGCNGAT
    g, X, W1, W2, W3, a_s, a_d, Hh, Fh = _inputs()
    m1 = RowPartitionedGCNGAT(g.rowptr, g.colidx, W1, W2, W3, a_s, a_d, Hh, Fh, reorder=0)
    m1.load_input(torch.from_numpy(X), non_blocking=False)
    Y1 = m1.step().cpu().numpy()
    L1, L2 = m1.Y1.cpu().numpy(), m1.Y2.cpu().numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    Y2 = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
    assert not isinstance(Y2, str), Y2
    assert np.array_equal(Y1.view(np.uint32), Y2.view(np.uint32))
    # P = 1 vs the oracle layer by layer on sampled rows, each layer fed the
    # GPU's own input to it, at the north_star tolerance (R11)
    rows = np.sort(np.random.default_rng(0).choice(g.n, 300, replace=False))
    tol = lambda r: 1e-5 + 1e-4 * np.abs(r)  # noqa: E731
    r1 = oracle.gcn_layer(g.rowptr, g.colidx, X, W1, relu=True, rows=rows)
    assert np.all(np.abs(L1[rows] - r1.astype(np.float64)) <= tol(r1)), "layer 1"
    r2 = oracle.gcn_layer(g.rowptr, g.colidx, L1, W2, relu=False, rows=rows)
    assert np.all(np.abs(L2[rows] - r2.astype(np.float64)) <= tol(r2)), "layer 2"
    r3 = oracle.gat_layer(g.rowptr, g.colidx, L2, W3, a_s, a_d, Hh, Fh, 0.2, rows=rows)
    assert np.all(np.abs(Y1[rows] - r3.astype(np.float64)) <= tol(r3)), "layer 3"


@pytest.mark.parametrize("Fh", [16, 32])
def test_two_ranks_peer_exchange_bit_identical_to_one(Fh):
    """NEXT-2: the exchange fused into the producers -- each rank's GEMM2 and
    GAT-transform epilogues also store their rows into the peer's replica
    buffer (CUDA IPC mapping, gnn_gemm_mirrored / gnn_gat_transform_mirrored),
    then a barrier -- is bit-identical to P = 1.  Two processes share this
    B200 (no kernel waits on the other rank: the barrier is on the host).
    Fh = 16 takes the folded-score GEMM, Fh = 32 the score epilogue."""
    import torch.multiprocessing as mp

    from paper_conf_ppopp_huangzzys21_b200.model import RowPartitionedGCNGAT
    g, X, W1, W2, W3, a_s, a_d, Hh, Fh = _inputs(Fh)
    m1 = RowPartitionedGCNGAT(g.rowptr, g.colidx, W1, W2, W3, a_s, a_d, Hh, Fh, reorder=0)
    m1.load_input(torch.from_numpy(X), non_blocking=False)
    Y1 = m1.step().cpu().numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, False, "peer", Fh)) for r in range(2)]
    for p in procs:
        p.start()
    Y2 = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
    assert not isinstance(Y2, str), Y2
    assert np.array_equal(Y1.view(np.uint32), Y2.view(np.uint32))


def test_two_ranks_overlapped_exchange_vs_oracle():
    """NEXT-2 groundwork: layer 2's exchange as a ring of P - 1 steps with the
    aggregation of each arrived source block (gnn_aggregate_accumulate in ring
    order, then x ndst).  Not bit-identical to P = 1 (block partial sums), so
    it is checked layer by layer against the oracle at the north_star
    tolerance, and reruns are bit-identical."""
    import torch.multiprocessing as mp

    import oracle
    g, X, W1, W2, W3, a_s, a_d, Hh, Fh = _inputs()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, True)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
    assert not isinstance(res, str), res
    L1, L2, Y3, Y3b = res
    assert np.array_equal(Y3.view(np.uint32), Y3b.view(np.uint32))  # rerun identical
    rows = np.sort(np.random.default_rng(1).choice(g.n, 300, replace=False))
    tol = lambda r: 1e-5 + 1e-4 * np.abs(r)  # noqa: E731
    r1 = oracle.gcn_layer(g.rowptr, g.colidx, X, W1, relu=True, rows=rows)
    assert np.all(np.abs(L1[rows] - r1.astype(np.float64)) <= tol(r1)), "layer 1"
    r2 = oracle.gcn_layer(g.rowptr, g.colidx, L1, W2, relu=False, rows=rows)
    assert np.all(np.abs(L2[rows] - r2.astype(np.float64)) <= tol(r2)), "layer 2 (overlapped exchange)"
    r3 = oracle.gat_layer(g.rowptr, g.colidx, L2, W3, a_s, a_d, Hh, Fh, 0.2, rows=rows)
    assert np.all(np.abs(Y3[rows] - r3.astype(np.float64)) <= tol(r3)), "layer 3"


@pytest.mark.parametrize("nparts", [3, 4])
def test_source_block_accumulation_single_process(nparts):
    """All ranks of a P-way partition simulated in one process (no exchange):
    each rank's layer-2 aggregation as ring-ordered source blocks
    (gnn_aggregate_accumulate + gnn_scale_rows) vs the oracle's GCN
    aggregation, at the north_star tolerance."""
    import oracle
    import paper_conf_ppopp_huangzzys21_b200 as G
    g = gs.powerlaw(20000, 400000, 20, 3000, 2500, comm=64, rho=0.8, seed=9)
    F = 64
    X = gs.uniform(g.n, F, seed=4)
    deg_out = np.bincount(g.colidx, minlength=g.n).astype(np.float32)
    nsrc = np.where(deg_out > 0, 1.0 / np.sqrt(np.maximum(deg_out, 1)), 0).astype(np.float32)
    Hs = torch.from_numpy((X * nsrc[:, None]).astype(np.float32)).cuda()
    ref = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn")
    b = G.partition_rows(g.rowptr, nparts)
    for rank in range(nparts):
        lo, hi = int(b[rank]), int(b[rank + 1])
        lrp, lci, sdeg, rmax = G.local_csr(g.rowptr, g.colidx, b, rank)
        full = G.Plan(lrp, lci, n_src=nparts * rmax, src_degree=sdeg, reorder=1)
        perm = full.export()[0]
        _, ndst = full.normalizers()
        Y = torch.empty((hi - lo, F), device="cuda")
        outs = []
        for rep in range(2):
            for s in range(nparts):
                qb = (rank - s) % nparts
                brp, bci = G.local_csr_block(g.rowptr, g.colidx, b, rank, qb)
                bp = G.Plan(brp, bci, n_src=max(1, int(b[qb + 1] - b[qb])), perm=perm)
                G.aggregate_accumulate(bp, Hs[int(b[qb]):int(b[qb + 1])], Y, accumulate=s > 0)
            G.scale_rows(Y, ndst)
            torch.cuda.synchronize()
            outs.append(Y.cpu().numpy().copy())
        assert np.array_equal(outs[0].view(np.uint32), outs[1].view(np.uint32))
        err = np.abs(outs[0].astype(np.float64) - ref[lo:hi])
        assert np.all(err <= 1e-5 + 1e-4 * np.abs(ref[lo:hi])), err.max()
