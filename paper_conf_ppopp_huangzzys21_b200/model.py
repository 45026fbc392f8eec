"""The C5 forward step on 1..P GPUs (a10: destination-row partitioning with a
per-layer all-gather of transformed source rows, reading R10).

Every arithmetic step runs in libgnn.so kernels through the C-ABI; this module
only owns buffers, the order of calls and the collective.

    layer 1  Y1 = ReLU((A_gcn X) W1)   aggregate-first (X replicated: no exchange)
    layer 2  Y2 = A_gcn (Y1 W2)        transform-first: Hs = (Y1 W2) * nsrc, all-gather, aggregate * ndst
    layer 3  Y3 = GAT_HxFh(Y2)         [Z|s|t] = Y2 W', all-gather, fused edge-softmax aggregation

Rank p owns destination rows [bounds[p], bounds[p+1]); sources live in the
padded layout u -> owner(u) * r_max + (u - bounds[owner]).  With the
deterministic plan option the concatenated P-rank output is bit-identical to
P = 1 (the per-row arithmetic depends only on (CSR, ng, F), R9).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import gnn as _g


def ring_allgather_blocks(buf, rmax, rank, world, group=None, on_block=None, staged=False):
    """All-gather of the padded layout buf [world * rmax, F] as P - 1 ring steps
    (NEXT-2 groundwork, SURVEY §8(e) lever ii): step s sends block (rank - s + 1)
    mod P to rank + 1 and receives block (rank - s) mod P from rank - 1, so rank
    r holds its blocks in the order r, r - 1, ..., r + 1 (mod P).  on_block(q) is
    called as soon as block q is present -- the caller enqueues that block's
    aggregation, which overlaps the next step's transfer (NCCL runs the P2P
    on its own stream; `wait()` only orders the caller's stream).  staged: move
    the blocks through host memory (gloo tests)."""
    import torch.distributed as dist
    if on_block:
        on_block(rank)
    for s in range(1, world):
        sq, rq = (rank - s + 1) % world, (rank - s) % world
        send = buf[sq * rmax:(sq + 1) * rmax]
        recv = buf[rq * rmax:(rq + 1) * rmax]
        if staged:
            sbuf, rbuf = send.cpu(), torch.empty(recv.shape, dtype=recv.dtype)
        else:
            sbuf, rbuf = send.contiguous(), recv
        ops = [dist.P2POp(dist.isend, sbuf, (rank + 1) % world, group),
               dist.P2POp(dist.irecv, rbuf, (rank - 1) % world, group)]
        for req in dist.batch_isend_irecv(ops):
            req.wait()
        if staged:
            recv.copy_(rbuf)
        if on_block:
            on_block(rq)


class RowPartitionedGCNGAT:
    def __init__(self, rowptr, colidx, W1, W2, W3, a_src, a_dst, heads, head_dim, neg_slope=0.2,
                 rank=0, world=1, group=None, reorder=1, device=None, plan_opts=None, staged_allgather=False,
                 overlap=False, exchange="nccl"):
        self.rank, self.world, self.group = rank, world, group
        self.dev = device or torch.device("cuda", torch.cuda.current_device())
        self.staged = staged_allgather  # gloo: exchange through host memory (tests only)
        # layer 2 exchange pipelined with the aggregation over source blocks (world > 1)
        self.overlap = bool(overlap) and world > 1
        # exchange of layers 2 and 3: "nccl" (all_gather_into_tensor, or the ring
        # with overlap) or "peer" (NEXT-2: the GEMM epilogue stores its rows into
        # every peer's replica buffer through CUDA IPC, then a barrier)
        if exchange not in ("nccl", "peer"):
            raise ValueError("exchange must be 'nccl' or 'peer'")
        self.peer = exchange == "peer" and world > 1
        if self.peer and self.overlap:
            raise ValueError("exchange='peer' replaces the ring exchange (overlap)")
        n = len(rowptr) - 1
        self.n = n
        opts = dict(reorder=reorder, **(plan_opts or {}))
        if world == 1:
            self.bounds = np.array([0, n], np.int64)
            self.rmax = n
            self.plan = _g.Plan(rowptr, colidx, **opts)
        else:
            self.bounds = _g.partition_rows(rowptr, world)
            lrp, lci, sdeg, rmax = _g.local_csr(rowptr, colidx, self.bounds, rank)
            self.rmax = rmax
            self.plan = _g.Plan(lrp, lci, n_src=world * rmax, src_degree=sdeg, **opts)
            if self.overlap:
                # one plan per source block, in the local plan's task order (LAS runs once)
                perm = self.plan.export()[0]
                bopts = dict(opts)
                bopts.pop("reorder", None)
                self.block_plans = []
                for q in range(world):
                    brp, bci = _g.local_csr_block(rowptr, colidx, self.bounds, rank, q)
                    self.block_plans.append(_g.Plan(brp, bci, n_src=rmax, perm=perm, reorder=0, **bopts))
        self.lo, self.hi = int(self.bounds[rank]), int(self.bounds[rank + 1])
        self.rows = self.hi - self.lo
        self.nnz_local = int(rowptr[self.hi] - rowptr[self.lo])
        d = self.dev
        self.W1 = torch.as_tensor(W1, device=d).contiguous()
        self.W2 = torch.as_tensor(W2, device=d).contiguous()
        self.W3 = torch.as_tensor(W3, device=d).contiguous()
        self.a_s = torch.as_tensor(a_src, device=d).contiguous()
        self.a_d = torch.as_tensor(a_dst, device=d).contiguous()
        self.F_in, self.F = self.W1.shape
        self.H, self.Fh = heads, head_dim
        self.HF = heads * head_dim
        self.slope = float(neg_slope)
        self.ldwe = (self.HF + 2 * heads + 7) // 8 * 8
        R, P = self.rows, world * self.rmax
        self.Xs = torch.zeros((P, self.F_in), device=d)          # replicated input, padded layout
        self.A1 = torch.empty((R, self.F_in), device=d)
        self.Y1 = torch.empty((R, self.F), device=d)
        self.Y2 = torch.empty((R, self.F), device=d)
        if self.peer:
            self._setup_peer(P, d)
        else:
            self.Hs2 = torch.zeros((P, self.F), device=d)
            self.Zst = torch.zeros((P, self.ldwe), device=d)
        self.Y3 = torch.empty((R, self.HF), device=d)
        self.nsrc_ptr, self.ndst_ptr = self.plan.normalizers()
        self.ws_agg, self.ws_agg_b = self.plan.workspace(_g.GNN_OP_AGGREGATE, 0, max(self.F, self.F_in), 0, d)
        self.ws_gat, self.ws_gat_b = self.plan.workspace(_g.GNN_OP_GAT_AGGREGATE, 0, self.HF, heads, d)
        self.names = ["agg1", "gemm1", "gemm2+xchg", "agg2", "gemm3+xchg", "gat_agg"]
        gw = max(_g._lib.gnn_gemm_workspace_size(R, self.F_in, self.F), _g._lib.gnn_gemm_workspace_size(R, self.F, self.F),
                 _g._lib.gnn_gat_transform_workspace_size(R, self.F, heads, head_dim))
        self.ws_gemm = torch.empty(max(gw, 256), dtype=torch.uint8, device=d)
        self.ws_gemm_b = gw

    # -- end to end over a stream of inputs ---------------------------------
    def run_pipelined(self, X_host, Y_host, steps, stream=None):
        """`steps` forward passes from pinned host input to pinned host output.

        Three streams overlap the host links with compute: the input of step
        k+1 is uploaded once step k's layer-1 aggregation has consumed the
        previous input, and the output of step k is downloaded while step k+1
        computes (the GAT output alternates between two device buffers).
        Returns the device-side events (start, end) bracketing the whole run.
        """
        dev = self.dev
        comp = torch.cuda.current_stream(dev) if stream is None else stream
        cin = torch.cuda.Stream(device=dev)
        cout = torch.cuda.Stream(device=dev)
        if not hasattr(self, "Y3b"):
            self.Y3b = [self.Y3, torch.empty_like(self.Y3)]
        E = lambda: torch.cuda.Event()  # noqa: E731
        start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        start.record(comp)
        cin.wait_event(start)
        cout.wait_event(start)
        consumed = None  # layer 1 of the previous step has read Xs
        downloaded = [None, None]
        for k in range(steps):
            with torch.cuda.stream(cin):
                if consumed is not None:
                    cin.wait_event(consumed)
                self.load_input(X_host, non_blocking=True)
                up = E()
                up.record(cin)
            comp.wait_event(up)
            b = k % 2
            if downloaded[b] is not None:
                comp.wait_event(downloaded[b])
            self.Y3 = self.Y3b[b]
            evs = [E() for _ in range(7)]
            self.step(stream=comp, events=evs)
            consumed = evs[1]
            with torch.cuda.stream(cout):
                cout.wait_event(evs[6])
                Y_host.copy_(self.Y3b[b], non_blocking=True)
                dl = E()
                dl.record(cout)
                downloaded[b] = dl
        comp.wait_stream(cout)
        end.record(comp)
        return start, end

    # -- inputs -------------------------------------------------------------
    def load_input(self, X_host_or_dev, non_blocking=True):
        """X [n, F_in] (host pinned or device) -> the replicated padded buffer."""
        for q in range(self.world):
            a, b = int(self.bounds[q]), int(self.bounds[q + 1])
            self.Xs[q * self.rmax:q * self.rmax + (b - a)].copy_(X_host_or_dev[a:b], non_blocking=non_blocking)

    # -- exchange -----------------------------------------------------------
    def _setup_peer(self, P, d):
        """NEXT-2: the replica buffers Hs2 / Zst live in IPC-shareable memory;
        every rank maps its peers' buffers and keeps, per layer, the list of
        peer addresses of its own row block (the GEMM epilogue's mirrors)."""
        import torch.distributed as dist
        self._ipc = [_g.IpcBuffer((P, self.F), d), _g.IpcBuffer((P, self.ldwe), d)]
        self.Hs2, self.Zst = self._ipc[0].tensor, self._ipc[1].tensor
        self.Hs2.zero_()
        self.Zst.zero_()
        handles = [None] * self.world
        dist.all_gather_object(handles, [b.handle_bytes() for b in self._ipc], group=self.group)
        self._peer_ptrs = []
        off = self.rank * self.rmax
        self.mirrors2, self.mirrors3 = [], []
        with torch.cuda.device(d):
            for q in range(self.world):
                if q == self.rank:
                    continue
                p2, p3 = _g.ipc_open(handles[q][0]), _g.ipc_open(handles[q][1])
                self._peer_ptrs += [p2, p3]
                self.mirrors2.append(p2 + 4 * off * self.F)
                self.mirrors3.append(p3 + 4 * off * self.ldwe)
        self._mir2 = _g._ptr_array(self.mirrors2)
        self._mir3 = _g._ptr_array(self.mirrors3)
        self._flag = torch.zeros(1, device=d)
        torch.cuda.synchronize(d)
        dist.barrier(group=self.group)

    def _peer_barrier(self):
        """Every rank's mirrored GEMM has finished (its stores are performed and
        fenced at system scope) before any rank reads its replica: a
        stream-ordered NCCL all_reduce of a flag (the aggregation queued after
        it waits on the device, not the host); gloo: host barrier."""
        import torch.distributed as dist
        if dist.get_backend(self.group) == "nccl":
            dist.all_reduce(self._flag, group=self.group)
        else:
            torch.cuda.synchronize(self.dev)
            dist.barrier(group=self.group)

    def close(self):
        """Unmap the peers' buffers and free the IPC buffers (peer exchange)."""
        if getattr(self, "_peer_ptrs", None):
            import torch.distributed as dist
            torch.cuda.synchronize(self.dev)
            dist.barrier(group=self.group)  # no peer still writes into our buffers
            for ptr in self._peer_ptrs:
                _g.ipc_close(ptr)
            self._peer_ptrs = []
            dist.barrier(group=self.group)  # every peer has unmapped ours
            self.Hs2 = self.Zst = None
            for b in self._ipc:
                b.free()
            self._ipc = []

    def _allgather(self, buf):
        if self.world == 1:
            return
        import torch.distributed as dist
        mine = buf[self.rank * self.rmax:(self.rank + 1) * self.rmax]
        if self.staged:
            out = torch.empty((self.world * self.rmax, buf.shape[1]), dtype=buf.dtype)
            dist.all_gather_into_tensor(out, mine.cpu(), group=self.group)
            buf.copy_(out)
        else:
            dist.all_gather_into_tensor(buf, mine.clone(), group=self.group)

    # -- the step -----------------------------------------------------------
    def step(self, stream=None, events=None):
        lib = _g._lib
        s = torch.cuda.current_stream(self.dev) if stream is None else stream
        sp = ctypes.c_void_p(s.cuda_stream)
        P = lambda t: ctypes.c_void_p(t.data_ptr())  # noqa: E731
        rec = (lambda i: events[i].record(s)) if events else (lambda i: None)
        R, F, Fi, HF, H = self.rows, self.F, self.F_in, self.HF, self.H
        off = self.rank * self.rmax

        def chk(st, what):
            if st != 0:
                raise _g.GnnError(what, st)

        rec(0)
        chk(lib.gnn_aggregate(self.plan.handle, _g.GNN_SUM, _g.GNN_W_GCN, None, P(self.Xs), Fi, Fi, P(self.A1), Fi,
                              0, None, 0, P(self.ws_agg), self.ws_agg_b, sp), "agg1")
        rec(1)
        gws = (P(self.ws_gemm), self.ws_gemm_b) if self.ws_gemm_b else (None, 0)
        chk(lib.gnn_gemm(P(self.A1), Fi, P(self.W1), F, P(self.Y1), F, R, Fi, F, None, None, 1, *gws, sp), "gemm1")
        rec(2)
        h_loc = self.Hs2[off:off + R]
        if self.peer:  # NEXT-2: the epilogue writes the rows into every peer's replica too
            chk(lib.gnn_gemm_mirrored(P(self.Y1), F, P(self.W2), F, P(h_loc), F, R, F, F,
                                      ctypes.c_void_p(self.nsrc_ptr + 4 * off), None, 0, self._mir2[0],
                                      self._mir2[1], *gws, sp), "gemm2 (mirrored)")
        else:
            chk(lib.gnn_gemm(P(self.Y1), F, P(self.W2), F, P(h_loc), F, R, F, F,
                             ctypes.c_void_p(self.nsrc_ptr + 4 * off), None, 0, *gws, sp), "gemm2")
        if self.overlap:
            # source-block pipeline: aggregate each rank's block of Hs2 as it arrives
            # (own block first), raw sums accumulated in ring order, then x ndst
            def on_block(q):
                bp = self.block_plans[q]
                ws, wb = bp.workspace(_g.GNN_OP_AGGREGATE, 0, F, 0, self.dev)
                chk(lib.gnn_aggregate_accumulate(bp.handle, _g.GNN_W_ONE, None,
                                                 P(self.Hs2[q * self.rmax:(q + 1) * self.rmax]), F, F, P(self.Y2), F,
                                                 int(q != self.rank), P(ws), wb, sp), "agg2 block")
            rec(3)
            ring_allgather_blocks(self.Hs2, self.rmax, self.rank, self.world, self.group, on_block, self.staged)
            chk(lib.gnn_scale_rows(P(self.Y2), F, R, F, ctypes.c_void_p(self.ndst_ptr), 0, sp), "agg2 scale")
        else:
            if self.peer:
                self._peer_barrier()
            else:
                self._allgather(self.Hs2)
            rec(3)
            chk(lib.gnn_gcn_aggregate_prescaled(self.plan.handle, P(self.Hs2), F, F, P(self.Y2), F, 0,
                                                P(self.ws_agg), self.ws_agg_b, sp), "agg2")
        rec(4)
        z_loc = self.Zst[off:off + R]
        # [Z | s | t] = Y2 W3 with the GAT scores from the GEMM epilogue (R5)
        if self.peer:
            chk(lib.gnn_gat_transform_mirrored(P(self.Y2), F, R, F, P(self.W3), HF, P(self.a_s), P(self.a_d), H,
                                               self.Fh, P(z_loc), self.ldwe, self._mir3[0], self._mir3[1], *gws, sp),
                "gemm3 (gat transform, mirrored)")
            self._peer_barrier()
        else:
            chk(lib.gnn_gat_transform(P(self.Y2), F, R, F, P(self.W3), HF, P(self.a_s), P(self.a_d), H, self.Fh,
                                      P(z_loc), self.ldwe, *gws, sp), "gemm3 (gat transform)")
            self._allgather(self.Zst)
        rec(5)
        tptr = ctypes.c_void_p(z_loc.data_ptr() + 4 * (HF + H))
        chk(lib.gnn_gat_aggregate(self.plan.handle, P(self.Zst), self.ldwe, tptr, self.ldwe, H, self.Fh,
                                  ctypes.c_float(self.slope), P(self.Y3), HF, P(self.ws_gat), self.ws_gat_b, sp),
            "gat agg")
        rec(6)
        return self.Y3
