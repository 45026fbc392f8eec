"""a10 multi-GPU row partitioning, exercised with world_size 2 (and 3) over
`gloo` on CPU.  The host logic under test is the product's
(gnn_partition_rows, gnn_local_csr: padded all-gather layout, global source
degrees); the per-rank compute stands in with the oracle because this box has
no GPU.  Concatenating the ranks' outputs must reproduce the single-process
result bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gnn_synth as gs
import oracle

P = pytest.importorskip("paper_conf_ppopp_huangzzys21_b200")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        g = gs.powerlaw(3000, 45000, 15, 900, 700, comm=32, rho=0.5, seed=11)
        F = 12
        X = gs.integer_features(g.n, F, seed=3)
        d_in = np.diff(g.rowptr)
        d_out = np.bincount(g.colidx, minlength=g.n)
        bounds = P.partition_rows(g.rowptr, world)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        lrp, lci, sdeg, rmax = P.local_csr(g.rowptr, g.colidx, bounds, rank)
        # rank's owned rows into its slot of the padded layout, then all-gather
        slot = torch.zeros((rmax, F), dtype=torch.float32)
        slot[:hi - lo] = torch.from_numpy(X[lo:hi])
        Hpad = torch.empty((world * rmax, F), dtype=torch.float32)
        dist.all_gather_into_tensor(Hpad, slot)
        Hpad = Hpad.numpy()
        for qq in range(world):
            a, b = int(bounds[qq]), int(bounds[qq + 1])
            assert np.array_equal(Hpad[qq * rmax:qq * rmax + (b - a)], X[a:b])
        # source degrees in the padded layout are the GLOBAL out-degrees
        for qq in range(world):
            a, b = int(bounds[qq]), int(bounds[qq + 1])
            assert np.array_equal(sdeg[qq * rmax:qq * rmax + (b - a)], d_out[a:b])
        # local aggregation (GCN weights from global degrees, integer sum exact)
        src = lci
        owner = src // rmax
        gsrc = bounds[owner] + (src - owner * rmax)
        dst = np.repeat(np.arange(lo, hi), np.diff(lrp))
        w = (1.0 / np.sqrt(d_out[gsrc].astype(np.float64) * d_in[dst])).astype(np.float32)
        Yl = oracle.aggregate(lrp, lci, Hpad, "sum", "edge", w)
        Yi = oracle.aggregate(lrp, lci, Hpad, "sum", "one")
        parts = [None] * world
        dist.all_gather_object(parts, (Yl, Yi))
        if rank == 0:
            Y = np.concatenate([p[0] for p in parts])
            Yint = np.concatenate([p[1] for p in parts])
            gw = (1.0 / np.sqrt(d_out[g.colidx].astype(np.float64) *
                                np.repeat(d_in, d_in))).astype(np.float32)
            ref = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "edge", gw)
            q.put((np.array_equal(Y, ref), np.array_equal(Yint, oracle.aggregate(g.rowptr, g.colidx, X, "sum"))))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put(repr(e))


@pytest.mark.parametrize("world", [2, 3])
def test_row_partition_allgather_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
    assert res == (True, True), res


# --------------------------------------------------------------------------- #
# NEXT-2 groundwork: ring all-gather in P - 1 steps with a per-block callback,
# and the source-block decomposition of a rank's CSR (host logic)
# --------------------------------------------------------------------------- #
def _ring_worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_ppopp_huangzzys21_b200.model import ring_allgather_blocks
        rmax, F = 5, 3
        buf = torch.full((world * rmax, F), -1.0)
        buf[rank * rmax:(rank + 1) * rmax] = torch.arange(rmax * F, dtype=torch.float32).view(rmax, F) + 100 * rank
        seen = []

        def on_block(b):  # the block must be complete when it is handed over
            want = torch.arange(rmax * F, dtype=torch.float32).view(rmax, F) + 100 * b
            seen.append((b, bool(torch.equal(buf[b * rmax:(b + 1) * rmax], want))))

        ring_allgather_blocks(buf, rmax, rank, world, None, on_block)
        q.put((rank, seen))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))


@pytest.mark.parametrize("world", [2, 3, 4])
def test_ring_allgather_blocks_order_and_contents(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ring_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
        order = [b for b, _ in res[r]]
        assert order == [(r - s) % world for s in range(world)]  # own block, then r-1, r-2, ...
        assert all(ok for _, ok in res[r])


@pytest.mark.parametrize("nparts", [2, 3, 5])
def test_source_blocks_partition_each_row(nparts):
    """gnn_local_csr_block: the P blocks of a rank's rows partition its CSR;
    per row, block q holds exactly the entries with sources in block q, in CSR
    order, so the block sums add up to the row sums (integer features: exact)."""
    g = gs.powerlaw(2500, 30000, 12, 400, 400, comm=32, rho=0.5, seed=nparts)
    X = gs.integer_features(g.n, 6, seed=2)
    b = P.partition_rows(g.rowptr, nparts)
    full = oracle.aggregate(g.rowptr, g.colidx, X, "sum")
    for rank in range(nparts):
        lo, hi = int(b[rank]), int(b[rank + 1])
        acc = np.zeros((hi - lo, 6), np.float64)
        for qb in range(nparts):
            brp, bci = P.local_csr_block(g.rowptr, g.colidx, b, rank, qb)
            assert brp[0] == 0 and len(brp) == hi - lo + 1
            # the block's entries, back in global ids, are the row's entries in [b_q, b_q+1), in order
            for v in range(lo, hi, max(1, (hi - lo) // 40)):
                row = g.colidx[g.rowptr[v]:g.rowptr[v + 1]]
                want = row[(row >= b[qb]) & (row < b[qb + 1])]
                got = bci[brp[v - lo]:brp[v - lo + 1]] + b[qb]
                assert np.array_equal(got, want)
            Xq = X[int(b[qb]):int(b[qb + 1])]
            if len(Xq) == 0:
                continue
            acc += oracle.aggregate(brp, bci, Xq, "sum")
        assert np.array_equal(acc.astype(np.float32), full[lo:hi])
