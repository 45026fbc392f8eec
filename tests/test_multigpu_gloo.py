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
