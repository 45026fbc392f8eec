"""Per-config measurements of SURVEY.md §8(d) ("What is reported" column) for
the BASELINE.json configs C1-C4 (C5 is bench.py's workload), with parity
against the oracle on the same seeded inputs, and the Table 6 / Fig 8-9
style ablations (±LAS, ±NG, deterministic vs atomic, fused vs unfused GAT,
factorised vs per-edge EdgeConv).

    python scripts/configs_report.py [--cfg C1,C2,C3,C4,FS] [--out FILE]
    python scripts/configs_report.py --cfg C3 --ncu-pass     # under ncu: one launch per variant
    python scripts/configs_report.py --merge-ncu CSV --out FILE   # add ncu DRAM bytes to FILE

Timing: CUDA events on the launching stream after warm-up; µs-scale calls
(C1) are timed as CUDA-graph replays.  "cold" = a 2xL2 buffer is written
before each call.  Unfused / per-edge ablation arms are plain torch ops
(they stand for the frameworks' multi-kernel pipelines); they
are comparison arms, not the product path.  The oracle is timed on 1 host
core.  Outputs are JSON (one object per config).
"""
import argparse
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import oracle  # noqa: E402  (test infrastructure: parity + the CPU timing only)
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402
from paper_conf_ppopp_huangzzys21_b200 import gnn as GN  # noqa: E402

DEV = "cuda"
RTOL, ATOL = 1e-4, 1e-5


def sync():
    torch.cuda.synchronize()


def events_ms(fn, iters=20, warm=3, flush=None):
    """median / min ms of single calls (events around each call)."""
    for _ in range(warm):
        fn()
    sync()
    ts = []
    for _ in range(iters):
        if flush is not None:
            flush()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts), min(ts)


def graph_us(fn, calls=100, reps=10):
    """µs per call from CUDA-graph replays of `calls` back-to-back calls."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    sync()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(calls):
            fn()
    g.replay()
    sync()
    ts = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e3 / calls)
    return statistics.median(ts), min(ts)


_FLUSH = {}


def flush_l2():
    if "buf" not in _FLUSH:
        l2 = torch.cuda.get_device_properties(0).L2_cache_size
        _FLUSH["buf"] = torch.empty(2 * l2 // 4, dtype=torch.float32, device=DEV)
    _FLUSH["buf"].fill_(1.0)


def cpu_ms(fn, reps=3):
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        r = fn()
        ts.append((time.perf_counter() - t0) * 1e3)
    return statistics.median(ts), r


def close(got, ref, rtol=RTOL, atol=ATOL):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    err = np.abs(got - ref)
    ok = bool(np.all(err <= atol + rtol * np.abs(ref)))
    return {"pass": ok, "max_abs_err": float(err.max()) if err.size else 0.0,
            "max_rel_err": float((err / np.maximum(np.abs(ref), 1e-30)).max()) if err.size else 0.0}


def T(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def glorot(fi, fo, seed):
    lim = np.sqrt(6.0 / (fi + fo))
    return gs.uniform(fi, fo, lo=-lim, hi=lim, seed=seed)


def agg_bytes(nnz, n, F, per_edge_extra=0, extra_row=0):
    return nnz * (4 + 4 * F + per_edge_extra) + n * (8 + 4 * F + extra_row)


def sample_rows(g, k=2048, top=64, seed=7):
    deg = np.diff(g.rowptr)
    rng = np.random.default_rng(seed)
    r = set(rng.choice(g.n, size=min(k, g.n), replace=False).tolist())
    r.update(np.argsort(-deg, kind="stable")[:top].tolist())
    return np.array(sorted(r), dtype=np.int64)


# --------------------------------------------------------------------------- #
def c1():
    """Cora-shaped GCN sum aggregation, F=16: launch-bound; µs per call."""
    g = gs.config_graph("C1")
    X = gs.uniform(g.n, 16, seed=gs.seed_of("C1", 1))
    out = {"graph": {"n": g.n, "nnz": g.nnz}}
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    Xd = T(X)
    Y = torch.empty_like(Xd)
    out["aggregate_us"], out["aggregate_us_min"] = graph_us(lambda: G.aggregate(plan, Xd, "sum", "gcn", relu=True,
                                                                                 out=Y))
    ref = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn", relu=True)
    out["parity_aggregate_all_rows"] = close(Y.cpu().numpy(), ref)
    out["oracle_aggregate_us"] = cpu_ms(lambda: oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn", relu=True),
                                        reps=5)[0] * 1e3
    # full layer on the secondary Cora input (1433 -> 16, Bernoulli(0.0127) features)
    rng = np.random.default_rng(gs.seed_of("C1", 1) + 7)
    X0 = (rng.random((g.n, 1433)) < 0.0127).astype(np.float32)
    W = glorot(1433, 16, gs.seed_of("C1", 2))
    X0d, Wd = T(X0), T(W)
    Yl = torch.empty((g.n, 16), device=DEV)
    out["gcn_layer_us"], _ = graph_us(lambda: G.gcn_layer(plan, X0d, Wd, relu=True, out=Yl), calls=50)
    refl = oracle.gcn_layer(g.rowptr, g.colidx, X0, W, relu=True)
    out["parity_gcn_layer_all_rows"] = close(Yl.cpu().numpy(), refl)
    out["oracle_gcn_layer_us"] = cpu_ms(lambda: oracle.gcn_layer(g.rowptr, g.colidx, X0, W, relu=True), reps=3)[0] * 1e3
    out["speedup_aggregate_vs_oracle"] = out["oracle_aggregate_us"] / out["aggregate_us"]
    out["speedup_layer_vs_oracle"] = out["oracle_gcn_layer_us"] / out["gcn_layer_us"]
    return out


def gat_unfused(row, col, n, Zs, t, H, Fh, slope):
    """The frameworks' multi-kernel edge-softmax pipeline, torch ops:
    u_add_v -> LeakyReLU -> reduce max -> exp -> reduce sum -> divide -> u_mul_e + sum."""
    HF = H * Fh
    z = Zs[:, :HF].view(-1, H, Fh)
    s = Zs[:, HF:HF + H]
    e = torch.nn.functional.leaky_relu(s[col] + t[row], slope)
    m = torch.full((n, H), -float("inf"), device=DEV).scatter_reduce(0, row[:, None].expand(-1, H), e, "amax")
    ex = torch.exp(e - m[row])
    l_ = torch.zeros((n, H), device=DEV).index_add_(0, row, ex)
    alpha = ex / l_[row]
    y = torch.zeros((n, H, Fh), device=DEV).index_add_(0, row, alpha[:, :, None] * z[col])
    return y.view(n, HF)


def c2():
    """arxiv-shaped GAT layer 128 -> 8 x 8 (fused score/softmax/aggregate)."""
    c = gs.CONFIGS["C2"]
    g = gs.config_graph("C2")
    Hh, Fh, F_in = c["H"], c["Fh"], c["F_in"]
    HF = Hh * Fh
    X = gs.uniform(g.n, F_in, seed=gs.seed_of("C2", 1))
    W = glorot(F_in, HF, gs.seed_of("C2", 2))
    al = np.sqrt(6.0 / (Fh + 1))
    a_s = gs.uniform(1, HF, lo=-al, hi=al, seed=gs.seed_of("C2", 3))[0]
    a_d = gs.uniform(1, HF, lo=-al, hi=al, seed=gs.seed_of("C2", 3) + 1)[0]
    deg = np.diff(g.rowptr)
    out = {"graph": {"n": g.n, "nnz": g.nnz, "max_deg": int(deg.max()), "zero_in_deg": int((deg == 0).sum())}}
    Xd, Wd, asd, add = T(X), T(W), T(a_s), T(a_d)
    Y = torch.empty((g.n, HF), device=DEV)
    res = {}
    for name, kw in [("las_ng", dict(reorder=1)), ("ng_only", dict(reorder=0)),
                     ("las_only", dict(reorder=1, group_size=0)), ("base", dict(reorder=0, group_size=0))]:
        plan = G.Plan(g.rowptr, g.colidx, **kw)
        warm = events_ms(lambda: G.gat_layer(plan, Xd, Wd, asd, add, Hh, Fh, 0.2, out=Y), iters=30)
        cold = events_ms(lambda: G.gat_layer(plan, Xd, Wd, asd, add, Hh, Fh, 0.2, out=Y), iters=20, flush=flush_l2)
        res[name] = {"layer_ms_warm": warm[0], "layer_ms_cold": cold[0], "n_units": plan.info["n_groups"]}
        if name == "las_ng":
            ref = oracle.gat_layer(g.rowptr, g.colidx, X, W, a_s, a_d, Hh, Fh, 0.2)
            out["parity_gat_layer_all_rows"] = close(Y.cpu().numpy(), ref)
            out["oracle_gat_layer_ms"] = cpu_ms(lambda: oracle.gat_layer(g.rowptr, g.colidx, X, W, a_s, a_d, Hh, Fh,
                                                                         0.2), reps=1)[0]
            # the aggregation alone (fused kernel) vs the 7-step unfused pipeline
            Wext = torch.empty((F_in, HF + 2 * Hh), device=DEV)
            GN._call("gnn_gat_fold_weights", Wd.data_ptr(), asd.data_ptr(), add.data_ptr(), F_in, Hh, Fh,
                     Wext.data_ptr(), HF + 2 * Hh, None)
            Zs = G.gemm(Xd, Wext)
            t = Zs[:, HF + Hh:]
            Ya = torch.empty((g.n, HF), device=DEV)
            fa = events_ms(lambda: G.gat_aggregate(plan, Zs, t, Hh, Fh, 0.2, out=Ya), iters=30)
            row = torch.from_numpy(np.repeat(np.arange(g.n), deg)).to(DEV)
            col = torch.from_numpy(g.colidx.astype(np.int64)).to(DEV)
            tt = t.contiguous()
            ua = events_ms(lambda: gat_unfused(row, col, g.n, Zs, tt, Hh, Fh, 0.2), iters=10)
            yu = gat_unfused(row, col, g.n, Zs, tt, Hh, Fh, 0.2)
            out["fused_vs_unfused"] = {"fused_aggregate_ms": fa[0], "unfused_7step_torch_ms": ua[0],
                                       "speedup": ua[0] / fa[0],
                                       "fused_vs_unfused_max_abs_diff": float((yu - Ya).abs().max())}
            out["edges_HFh_per_s_aggregate"] = g.nnz * HF / (fa[0] * 1e-3)
            out["aggregate_alg_GBps"] = agg_bytes(g.nnz, g.n, HF, 4 * Hh, 4 * Hh) / (fa[0] * 1e-3) / 1e9
        del plan
    out["ablation_gat_layer"] = res
    # deterministic vs atomic split-row combine (sum aggregation, F = 64)
    X64 = T(gs.uniform(g.n, 64, seed=3))
    Y64 = torch.empty_like(X64)
    det = {}
    for d in (1, 0):
        plan = G.Plan(g.rowptr, g.colidx, reorder=1, deterministic=d)
        det["deterministic" if d else "atomic"] = events_ms(lambda: G.aggregate(plan, X64, "sum", "gcn", out=Y64),
                                                            iters=30)[0]
        del plan
    out["sum_F64_det_vs_atomic_ms"] = det
    return out


def c3(rho, ncu_pass=False):
    """Reddit-shaped 2-layer GCN (602 -> 256 -> 256), transform-first."""
    c = gs.CONFIGS["C3"]
    t0 = time.time()
    g = gs.config_graph("C3", rho=rho)
    gen_s = time.time() - t0
    F_in, F = c["F_in"], c["F"]
    out = {"rho": rho, "graph": {"n": g.n, "nnz": g.nnz, "max_deg": int(np.diff(g.rowptr).max()), "gen_s": gen_s}}
    X = gs.uniform(g.n, F_in, ld=604, seed=gs.seed_of("C3", 1))
    Xd = T(X)[:, :F_in]
    W1 = glorot(F_in, F, gs.seed_of("C3", 2))
    W2 = glorot(F, F, gs.seed_of("C3", 2) + 1)
    W1d, W2d = T(W1), T(W2)
    H1 = torch.empty((g.n, F), device=DEV)
    variants = [("las_ng", dict(reorder=1)), ("ng_only", dict(reorder=0)), ("las_only", dict(reorder=1, group_size=0)),
                ("base", dict(reorder=0, group_size=0))]
    res = {}
    Hs = torch.rand((g.n, F), device=DEV) * 2 - 1
    for name, kw in variants:
        t0 = time.time()
        plan = G.Plan(g.rowptr, g.colidx, **kw)
        build_s = time.time() - t0
        info = plan.info
        if ncu_pass:  # one aggregation launch per variant, in this order
            G.aggregate(plan, Hs, "sum", "gcn", out=H1)
            sync()
            del plan
            continue
        agg = events_ms(lambda: G.aggregate(plan, Hs, "sum", "gcn", out=H1), iters=10)
        agg_cold = events_ms(lambda: G.aggregate(plan, Hs, "sum", "gcn", out=H1), iters=5, flush=flush_l2)
        # the transform-first layer's form: rows pre-scaled by nsrc in the GEMM
        # epilogue, weight 1 in the loop, x ndst in the epilogue (gather4 kernel)
        ws_p, nb_p = plan.workspace(GN.GNN_OP_AGGREGATE, 0, F, 0, DEV)
        pres = events_ms(lambda: GN._call("gnn_gcn_aggregate_prescaled", plan.handle, GN._tp(Hs), F, F, GN._tp(H1), F, 0,
                                          GN._tp(ws_p), nb_p, None), iters=10)
        alg = agg_bytes(g.nnz, g.n, F, per_edge_extra=4)
        r = {"plan_build_s": build_s, "ms_minhash": info["ms_minhash"], "ms_lsh": info["ms_lsh"],
             "ms_merge": info["ms_merge"], "ms_ng": info["ms_ng"], "n_units": info["n_groups"],
             "group_size": info["group_size"], "aggregate_F256_ms": agg[0], "aggregate_F256_ms_cold": agg_cold[0],
             "aggregate_prescaled_F256_ms": pres[0],
             "aggregate_alg_GBps": alg / (agg[0] * 1e-3) / 1e9,
             "effective_gather_GBps": g.nnz * F * 4 / (agg[0] * 1e-3) / 1e9,
             "edges_F_per_s": g.nnz * F / (agg[0] * 1e-3)}
        if name == "las_ng":
            Y1 = torch.empty((g.n, F), device=DEV)
            Y2 = torch.empty((g.n, F), device=DEV)
            l1 = events_ms(lambda: G.gcn_layer(plan, Xd, W1d, relu=True, order=1, out=Y1), iters=5)
            l2 = events_ms(lambda: G.gcn_layer(plan, Y1, W2d, relu=False, order=1, out=Y2), iters=5)
            gm1 = events_ms(lambda: G.gemm(Xd, W1d, out=H1), iters=5)
            gm2 = events_ms(lambda: G.gemm(Y1, W2d, out=H1), iters=5)
            r.update({"layer1_ms": l1[0], "layer2_ms": l2[0], "gemm1_ms": gm1[0], "gemm2_ms": gm2[0],
                      "gemm1_TFLOPs": 2 * g.n * F_in * F / (gm1[0] * 1e-3) / 1e12,
                      "gemm2_TFLOPs": 2 * g.n * F * F / (gm2[0] * 1e-3) / 1e12})
            # parity: sampled rows + the 64 largest, both layers, vs the oracle
            rows = sample_rows(g, k=1024, top=32)
            Xh = np.ascontiguousarray(X[:, :F_in])
            ref1 = oracle.gcn_layer(g.rowptr, g.colidx, Xh, W1, relu=True, rows=rows)
            r["parity_layer1_sampled"] = close(Y1.cpu().numpy()[rows], ref1)
            # epilogue fused vs separate (linear-property postponement):
            # ndst scaling + ReLU in the aggregation's epilogue vs an extra
            # elementwise pass over Y (torch op standing for the separate kernel)
            Hs2 = torch.rand((g.n, F), device=DEV) - 0.5
            Yf = torch.empty((g.n, F), device=DEV)
            ws_f, nb_f = plan.workspace(GN.GNN_OP_AGGREGATE, 0, F, 0, DEV)
            deg = np.diff(g.rowptr).astype(np.float32)
            ndst = torch.from_numpy(np.where(deg > 0, 1.0 / np.sqrt(np.maximum(deg, 1)), 0).astype(np.float32)).to(DEV)

            def fused():
                GN._call("gnn_gcn_aggregate_prescaled", plan.handle, GN._tp(Hs2), F, F, GN._tp(Yf), F, 1,
                         GN._tp(ws_f), nb_f, None)

            def separate():
                G.aggregate(plan, Hs2, "sum", "one", out=Yf)
                Yf.mul_(ndst[:, None]).relu_()
            r["epilogue_fused_ms"] = events_ms(fused, iters=5)[0]
            r["epilogue_separate_ms"] = events_ms(separate, iters=5)[0]
            del Hs2, Yf
            # layer 2 as a standalone layer on its own seeded input (no oracle
            # input ever comes from the GPU path)
            X2 = gs.uniform(g.n, F, lo=0.0, hi=1.0, seed=gs.seed_of("C3", 1) + 1)
            G.gcn_layer(plan, T(X2), W2d, relu=False, order=1, out=Y2)
            ref2 = oracle.gcn_layer(g.rowptr, g.colidx, X2, W2, relu=False, rows=rows)
            r["parity_layer2_sampled"] = close(Y2.cpu().numpy()[rows], ref2)
            r["parity_rows"] = int(len(rows))
        res[name] = r
        del plan
    out["variants"] = res
    return out


def c4():
    """kNN point clouds (32 x 1024, k=20) EdgeConv max, F 64 -> 64."""
    g = gs.config_graph("C4")
    F = 64
    X = gs.uniform(g.n, F, seed=gs.seed_of("C4", 1))
    th = glorot(F, F, gs.seed_of("C4", 2))
    ph = glorot(F, F, gs.seed_of("C4", 2) + 1)
    b = gs.uniform(1, F, lo=-0.1, hi=0.1, seed=gs.seed_of("C4", 3))[0]
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    Xd, thd, phd, bd = T(X), T(th), T(ph), T(b)
    Y = torch.empty((g.n, F), device=DEV)
    out = {"graph": {"n": g.n, "nnz": g.nnz}}
    out["edgeconv_layer_ms"] = events_ms(lambda: G.edgeconv(plan, Xd, thd, phd, bd, out=Y), iters=30)[0]
    ref = oracle.edgeconv(g.rowptr, g.colidx, X, th, ph, b)
    out["parity_edgeconv_all_rows"] = close(Y.cpu().numpy(), ref)
    Wcat = torch.cat([thd.t(), (phd - thd).t()], dim=1).contiguous()  # [64, 128] = [Θᵀ ‖ (Φ−Θ)ᵀ]
    PQ = G.gemm(Xd, Wcat, col_bias=torch.cat([torch.zeros_like(bd), bd]))
    Ya = torch.empty((g.n, F), device=DEV)
    out["max_aggregate_ms"] = events_ms(lambda: G.edgeconv_aggregate(plan, PQ, F, out=Ya), iters=30)[0]
    out["max_aggregate_us_graph"] = graph_us(lambda: G.edgeconv_aggregate(plan, PQ, F, out=Ya))[0]
    # per-edge MLP (no redundancy bypass): E x [x_u - x_v, x_v] x [Θ; Φ]ᵀ, then max
    deg = np.diff(g.rowptr)
    row = torch.from_numpy(np.repeat(np.arange(g.n), deg)).to(DEV)
    col = torch.from_numpy(g.colidx.astype(np.int64)).to(DEV)
    Wpe = torch.cat([thd, phd], dim=1).t().contiguous()  # [128, 64]

    def per_edge():
        h = torch.cat([Xd[col] - Xd[row], Xd[row]], dim=1) @ Wpe + bd
        h = torch.relu(h)
        return torch.full((g.n, F), -float("inf"), device=DEV).scatter_reduce(0, row[:, None].expand(-1, F), h, "amax")

    torch.backends.cuda.matmul.allow_tf32 = False
    out["per_edge_mlp_torch_ms"] = events_ms(per_edge, iters=10)[0]
    ype = per_edge()
    out["per_edge_vs_factorised_max_abs_diff"] = float((ype - Y).abs().max())
    out["factorised_gemm_GFLOP"] = 2 * g.n * F * 2 * F / 1e9
    out["per_edge_gemm_GFLOP"] = 2 * g.nnz * 2 * F * F / 1e9
    out["speedup_factorised_vs_per_edge"] = out["per_edge_mlp_torch_ms"] / out["edgeconv_layer_ms"]
    out["oracle_edgeconv_ms"] = cpu_ms(lambda: oracle.edgeconv(g.rowptr, g.colidx, X, th, ph, b), reps=1)[0]
    return out


def lstm_base_torch(X, table, P, T):
    """Fig 6 base implementation (torch ops): per cell gather the neighbour
    feature matrix X[u_t], transform it (no redundancy bypass), then the cell."""
    n = X.shape[0]
    F = P["W_hh"].shape[1]
    h = torch.zeros((n, F), device=DEV)
    c = torch.zeros((n, F), device=DEV)
    has = (table[:, 0] >= 0)[:, None]
    idx = table.clamp(min=0).long()
    b = P["b_ih"] + P["b_hh"]
    for t in range(T):
        xg = X[idx[:, t]]                                  # graph op: neighbour feature matrix
        a = xg @ P["W_ih"].t() + h @ P["W_hh"].t() + b     # neural op on the expanded data
        i, f, z, o = a.split(F, dim=1)
        c2 = torch.sigmoid(f) * c + torch.sigmoid(i) * torch.tanh(z)
        h2 = torch.sigmoid(o) * torch.tanh(c2)
        c = torch.where(has, c2, c)
        h = torch.where(has, h2, h)
    return X @ P["W_self"].t() + h @ P["W_neigh"].t() + P["bias"]


def lstm(cfg="C5"):
    """NEXT-3 GraphSAGE-LSTM layer (32 -> 32, 16 sampled neighbours)
    on a config graph: layer / cell-kernel ms, rooflines, Fig 11 analogue."""
    g = gs.config_graph(cfg)
    f_in, F, F_out, nT = 32, 32, 32, 16
    rng = np.random.default_rng(gs.seed_of(cfg, 4))
    Ph = {k: rng.uniform(-0.3, 0.3, size=s).astype(np.float32) for k, s in
          dict(W_ih=(4 * F, f_in), W_hh=(4 * F, F), b_ih=(4 * F,), b_hh=(4 * F,), W_self=(F_out, f_in),
               W_neigh=(F_out, F), bias=(F_out,)).items()}
    P = {k: T(v) for k, v in Ph.items()}
    X = gs.uniform(g.n, f_in, seed=gs.seed_of(cfg, 1) + 5)
    Xd = T(X)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    args = [P[k] for k in ("W_ih", "W_hh", "b_ih", "b_hh", "W_self", "W_neigh", "bias")]
    Y = torch.empty((g.n, F_out), device=DEV)
    out = {"graph": cfg, "n": g.n, "nnz": g.nnz, "T": nT, "f_in": f_in, "F": F, "F_out": F_out}
    out["layer_ms"] = events_ms(lambda: G.sage_lstm_layer(plan, Xd, *args, T=nT, seed=7, out=Y), iters=10)[0]
    # the parts: sampling, pre-transform GEMM (redundancy bypass), fused cells
    tab = G.sample_neighbors(plan, nT, 7)
    out["sample_ms"] = events_ms(lambda: G.sample_neighbors(plan, nT, 7, out=tab), iters=10)[0]
    Wcat = torch.cat([P["W_ih"].view(4, F, f_in).permute(1, 0, 2).reshape(4 * F, f_in), P["W_self"]], 0).t()
    bcat = torch.cat([(P["b_ih"] + P["b_hh"]).view(4, F).t().reshape(-1), P["bias"]])
    GS = torch.empty((g.n, 4 * F + F_out), device=DEV)
    out["pretransform_gemm_ms"] = events_ms(lambda: G.gemm(Xd, Wcat.contiguous(), col_bias=bcat, out=GS), iters=10)[0]
    Ya = torch.empty_like(Y)
    cell = events_ms(lambda: G.sage_lstm_aggregate(plan, tab, GS, P["W_hh"], P["W_neigh"], out=Ya), iters=10)[0]
    out["cell_kernel_ms"] = cell
    out["cell_vs_layer_max_abs_diff"] = float((Ya - Y).abs().max())
    flop = 2.0 * g.n * nT * (4 * F * F) + 2.0 * g.n * F * F_out
    byts = g.n * nT * (4 * (4 * F) + 4) + g.n * (4 * F_out * 2 + 4)
    clk = 1.965e9
    fp32_peak = 148 * 128 * 2 * clk / 1e12
    out["cell_roofline"] = {"flop": flop, "algorithmic_bytes": byts, "TFLOPs": flop / (cell * 1e-3) / 1e12,
                            "fp32_fma_peak_TFLOPs": fp32_peak, "frac_fp32": flop / (cell * 1e-3) / 1e12 / fp32_peak,
                            "GBps": byts / (cell * 1e-3) / 1e9}
    # parity on sampled rows (oracle on the same counter-based table)
    rows = sample_rows(g, k=1024, top=16)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, nT, 7)
    ref = oracle.sage_lstm(X, table, **Ph, rows=rows)
    out["parity_sampled"] = close(Y.cpu().numpy()[rows], ref)
    out["parity_rows"] = int(len(rows))
    # Fig 11 analogue: base implementation (expand + transform every cell), torch ops
    torch.backends.cuda.matmul.allow_tf32 = False
    base = events_ms(lambda: lstm_base_torch(Xd, tab, P, nT), iters=3, warm=1)[0]
    out["base_impl_torch_ms"] = base
    out["speedup_vs_base"] = base / out["layer_ms"]
    out["base_vs_ours_max_abs_diff"] = float((lstm_base_torch(Xd, tab, P, nT) - Y).abs().max())
    del plan
    return out


def attn(cfg="C5", H=8, Fh=32):
    """NEXT-4 Table 2 scores + softmax aggregation on a config graph: ms,
    algorithmic GB/s, sampled parity; GaAN also against an unfused torch
    SDDMM -> edge softmax -> SpMM pipeline."""
    g = gs.config_graph(cfg)
    F = H * Fh
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    rng = np.random.default_rng(3)
    rows = sample_rows(g, k=512, top=16)
    out = {"graph": cfg, "n": g.n, "nnz": g.nnz, "H": H, "Fh": Fh, "scores": {}}
    extra_edge = {"gat": 4 * H, "sym": 8 * H, "linear": 4 * H, "gaan": 4 * F, "gene": 4 * F}
    extra_row = {"gat": 4 * H, "sym": 8 * H, "linear": 0, "gaan": 4 * F, "gene": 4 * F}
    for score in ("gat", "sym", "linear", "gaan", "gene"):
        w = F + (H if score in ("gat", "linear") else 2 * H if score == "sym" else F)
        Zs = torch.rand((g.n, w), device=DEV) * 2 - 1
        Tv = None
        if score == "gat":
            Tv = torch.rand((g.n, H), device=DEV) * 2 - 1
        elif score in ("gaan", "gene"):
            Tv = (torch.rand((g.n, F), device=DEV) * 2 - 1) * 0.5
        Wa = torch.from_numpy(rng.uniform(-0.5, 0.5, size=(H, Fh)).astype(np.float32)).to(DEV) if score == "gene" else None
        Y = torch.empty((g.n, F), device=DEV)
        ms = events_ms(lambda: G.attn_aggregate(plan, score, Zs, H, Fh, Tv, Wa, out=Y), iters=5, warm=2)[0]
        alg = g.nnz * (4 + 4 * F + extra_edge[score]) + g.n * (8 + 4 * F + extra_row[score])
        ref = oracle.attn_aggregate(g.rowptr, g.colidx, score, Zs.cpu().numpy(), H, Fh,
                                    Tv=None if Tv is None else Tv.cpu().numpy(),
                                    Wa=None if Wa is None else Wa.cpu().numpy(), rows=rows)
        r = {"ms": ms, "alg_GBps": alg / (ms * 1e-3) / 1e9, "parity_sampled": close(Y.cpu().numpy()[rows], ref)}
        if score == "gaan":  # unfused: SDDMM (per-edge dot) -> edge softmax -> SpMM, torch ops
            deg = np.diff(g.rowptr)
            row_t = torch.from_numpy(np.repeat(np.arange(g.n), deg)).to(DEV)
            col_t = torch.from_numpy(g.colidx.astype(np.int64)).to(DEV)

            def unfused():
                q = Zs[:, F:].view(-1, H, Fh)
                e = (q[col_t] * Tv.view(-1, H, Fh)[row_t]).sum(-1)
                m = torch.full((g.n, H), -float("inf"), device=DEV).scatter_reduce(
                    0, row_t[:, None].expand(-1, H), e, "amax")
                ex = torch.exp(e - m[row_t])
                l_ = torch.zeros((g.n, H), device=DEV).index_add_(0, row_t, ex)
                return torch.zeros((g.n, H, Fh), device=DEV).index_add_(
                    0, row_t, (ex / l_[row_t])[:, :, None] * Zs[:, :F].view(-1, H, Fh)[col_t]).view(g.n, F)
            try:
                r["unfused_torch_ms"] = events_ms(unfused, iters=3, warm=1)[0]
                r["speedup_vs_unfused"] = r["unfused_torch_ms"] / ms
            except RuntimeError as exc:  # the expanded [E, H, Fh] tensors may not fit
                r["unfused_torch_ms"] = f"failed: {str(exc)[:80]}"
        out["scores"][score] = r
        print(f"  {score}: {ms:.3f} ms", flush=True)
        del Zs, Tv, Y
        torch.cuda.empty_cache()
    del plan
    return out


def fsweep():
    """F sweep (Fig 4 / Fig 12 analogue, NEXT-1): sum-aggregation throughput vs
    feature length on the C5 graph with the automatic a4 mapping."""
    g = gs.config_graph("C5")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    res = []
    for F in list(range(16, 257, 16)) + [100, 602 // 2]:
        X = torch.rand((g.n, F), device=DEV)
        Y = torch.empty_like(X)
        ms = events_ms(lambda: G.aggregate(plan, X, "sum", "one", out=Y), iters=5, warm=2)[0]
        res.append({"F": F, "ms": ms, "Gedge_F_per_s": g.nnz * F / (ms * 1e-3) / 1e9,
                    "alg_GBps": agg_bytes(g.nnz, g.n, F) / (ms * 1e-3) / 1e9})
        print(f"  F={F}: {ms:.3f} ms", flush=True)
        del X, Y
    return {"graph": "C5", "nnz": g.nnz, "points": res}


def merge_ncu(csv_path, out_path):
    """Attach ncu DRAM bytes / hit rates of the C3 --ncu-pass launches (order:
    rho 0.8 then 0; variants las_ng, ng_only, las_only, base) to the report."""
    import csv
    rows = [r for r in csv.reader(open(csv_path)) if r]
    hdr_i = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    hdr = rows[hdr_i]
    ki, mi, vi, ii = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
    launches = {}
    for r in rows[hdr_i + 1:]:
        if "k_aggregate" not in r[ki]:
            continue
        launches.setdefault(int(r[ii]), {})[r[mi]] = float(r[vi].replace(",", ""))
    ids = sorted(launches)
    rep = json.load(open(out_path))
    names = ["las_ng", "ng_only", "las_only", "base"]
    k = 0
    for key in ("C3_rho0.8", "C3_rho0.0"):
        if key not in rep:
            continue
        for nm in names:
            if k >= len(ids):
                break
            m = launches[ids[k]]
            k += 1
            v = rep[key]["variants"].get(nm)
            if v is None:
                continue
            dram = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
            dur = m.get("gpu__time_duration.sum", 0) * 1e-9
            v["ncu"] = {"dram_bytes": dram, "duration_ms": dur * 1e3, "dram_GBps": dram / dur / 1e9 if dur else None,
                        "l2_hit_pct": m.get("lts__t_sector_hit_rate.pct"),
                        "dram_frac_of_8TBps": dram / dur / 8e12 if dur else None}
    json.dump(rep, open(out_path, "w"), indent=1)


def summary(path):
    """Markdown digest of a report JSON (profiles/rNN_configs.md)."""
    d = json.load(open(path))
    L = [f"# Per-config report ({d['device']['name']}, {d['device']['sms']} SMs, L2 {d['device']['l2_bytes'] / 2**20:.0f} MiB)",
         "", "Generated by `scripts/configs_report.py` (+ `--merge-ncu` for the C3 DRAM columns). "
         "Oracle = 1 host core, fp64. Parity = |g-r| <= 1e-5 + 1e-4|r| (R11).", ""]
    if "C1" in d:
        c = d["C1"]
        L += ["## C1 Cora-shaped GCN, F=16 (launch-bound)", "",
              f"- gnn_aggregate (sum, GCN weights, ReLU): **{c['aggregate_us']:.1f} µs**/call (CUDA-graph replay); "
              f"oracle {c['oracle_aggregate_us']:.0f} µs; parity all rows: {c['parity_aggregate_all_rows']['pass']}",
              f"- full GCN layer 1433->16 (Bernoulli features): **{c['gcn_layer_us']:.1f} µs**; oracle "
              f"{c['oracle_gcn_layer_us'] / 1e3:.1f} ms; parity all rows: {c['parity_gcn_layer_all_rows']['pass']}", ""]
    if "C2" in d:
        c = d["C2"]
        a = c["ablation_gat_layer"]
        f = c["fused_vs_unfused"]
        L += ["## C2 arxiv-shaped GAT layer 128 -> 8x8", "",
              f"graph: n={c['graph']['n']}, nnz={c['graph']['nnz']}, max in-degree {c['graph']['max_deg']}, "
              f"{c['graph']['zero_in_deg']} empty rows; parity all rows: {c['parity_gat_layer_all_rows']['pass']} "
              f"(oracle {c['oracle_gat_layer_ms']:.0f} ms)", "",
              "| variant | layer ms (warm) | layer ms (cold L2) | work units |", "|---|---|---|---|"]
        for k, v in a.items():
            L.append(f"| {k} | {v['layer_ms_warm']:.3f} | {v['layer_ms_cold']:.3f} | {v['n_units']} |")
        L += ["", f"- fused aggregate {f['fused_aggregate_ms']:.3f} ms vs unfused 7-step (torch ops) "
              f"{f['unfused_7step_torch_ms']:.3f} ms: **{f['speedup']:.1f}x**",
              f"- sum F=64 split-row combine: deterministic {c['sum_F64_det_vs_atomic_ms']['deterministic']:.3f} ms, "
              f"atomic {c['sum_F64_det_vs_atomic_ms']['atomic']:.3f} ms", ""]
    for key in ("C3_rho0.8", "C3_rho0.0"):
        if key not in d:
            continue
        c = d[key]
        L += [f"## C3 Reddit-shaped 2-layer GCN 602->256->256, rho={c['rho']}", "",
              f"graph: nnz={c['graph']['nnz']}, max degree {c['graph']['max_deg']}", "",
              "| variant | agg F=256 ms (GCN weights) | cold ms | alg GB/s | ncu DRAM GB | ncu DRAM GB/s | L2 hit % | "
              "prescaled agg ms (layer form) | plan s |",
              "|---|---|---|---|---|---|---|---|---|"]
        for k, v in c["variants"].items():
            n = v.get("ncu", {})
            L.append(f"| {k} | {v['aggregate_F256_ms']:.2f} | {v['aggregate_F256_ms_cold']:.2f} | "
                     f"{v['aggregate_alg_GBps']:.0f} | {n.get('dram_bytes', 0) / 1e9:.1f} | "
                     f"{n.get('dram_GBps') or 0:.0f} | {n.get('l2_hit_pct')} | "
                     f"{v.get('aggregate_prescaled_F256_ms', float('nan')):.2f} | {v['plan_build_s']:.2f} |")
        v = c["variants"]["las_ng"]
        if "epilogue_fused_ms" in v:
            L += ["", f"- epilogue (x ndst, ReLU) fused into the aggregation {v['epilogue_fused_ms']:.2f} ms vs a "
                  f"separate elementwise pass {v['epilogue_separate_ms']:.2f} ms"]
        L += ["", f"- layers: L1 {v['layer1_ms']:.2f} ms, L2 {v['layer2_ms']:.2f} ms; GEMM1 {v['gemm1_ms']:.3f} ms "
              f"({v['gemm1_TFLOPs']:.0f} TF/s), GEMM2 {v['gemm2_ms']:.3f} ms ({v['gemm2_TFLOPs']:.0f} TF/s)",
              f"- parity ({v['parity_rows']} sampled rows incl. the 32 largest): L1 {v['parity_layer1_sampled']['pass']}, "
              f"L2 {v['parity_layer2_sampled']['pass']}", ""]
    if "C4" in d:
        c = d["C4"]
        L += ["## C4 EdgeConv max, kNN 32x1024, k=20, F=64", "",
              f"- full layer (GEMM [P|Q] + max aggregate): **{c['edgeconv_layer_ms']:.3f} ms**; max aggregate "
              f"{c['max_aggregate_ms']:.3f} ms ({c['max_aggregate_us_graph']:.1f} µs graph-replayed); parity all rows: "
              f"{c['parity_edgeconv_all_rows']['pass']}",
              f"- per-edge MLP (torch, no redundancy bypass) {c['per_edge_mlp_torch_ms']:.3f} ms -> factorised "
              f"**{c['speedup_factorised_vs_per_edge']:.1f}x** ({c['factorised_gemm_GFLOP']:.2f} vs "
              f"{c['per_edge_gemm_GFLOP']:.1f} GFLOP); oracle {c['oracle_edgeconv_ms']:.0f} ms", ""]
    if "LSTM_C5" in d:
        c = d["LSTM_C5"]
        r = c["cell_roofline"]
        L += [f"## GraphSAGE-LSTM (NEXT-3), {c['graph']}-shaped graph, {c['f_in']}->{c['F_out']}, T={c['T']}", "",
              f"- layer **{c['layer_ms']:.2f} ms** = sampling {c['sample_ms']:.3f} + pre-transform GEMM "
              f"{c['pretransform_gemm_ms']:.3f} + fused cells {c['cell_kernel_ms']:.2f} ms",
              f"- cells: {r['TFLOPs']:.1f} TFLOP/s = {100 * r['frac_fp32']:.0f}% of the fp32 FMA peak "
              f"({r['fp32_fma_peak_TFLOPs']:.1f}); {r['GBps']:.0f} GB/s algorithmic",
              f"- base implementation (gather + transform every cell, torch) {c['base_impl_torch_ms']:.1f} ms -> "
              f"**{c['speedup_vs_base']:.1f}x**; parity ({c['parity_rows']} sampled rows): "
              f"{c['parity_sampled']['pass']}", ""]
    for key in ("ATTN_C2", "ATTN_C5"):
        if key not in d:
            continue
        c = d[key]
        L += [f"## Table 2 edge functions (NEXT-4), {c['graph']}-shaped graph, {c['H']} heads x {c['Fh']}", "",
              "| score | ms | alg GB/s | sampled parity | unfused torch ms |", "|---|---|---|---|---|"]
        for k, v in c["scores"].items():
            L.append(f"| {k} | {v['ms']:.3f} | {v['alg_GBps']:.0f} | {v['parity_sampled']['pass']} | "
                     f"{v.get('unfused_torch_ms', '')} |")
        L.append("")
    if "F_sweep" in d:
        L += ["## F sweep (C5 graph, sum, automatic a4 mapping)", "", "| F | ms | Gedge*F/s | alg GB/s |",
              "|---|---|---|---|"]
        for p_ in d["F_sweep"]["points"]:
            L.append(f"| {p_['F']} | {p_['ms']:.2f} | {p_['Gedge_F_per_s']:.0f} | {p_['alg_GBps']:.0f} |")
    return "\n".join(L) + "\n"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", default="C1,C2,C3,C4")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "configs.json"))
    ap.add_argument("--ncu-pass", action="store_true")
    ap.add_argument("--merge-ncu", default=None)
    ap.add_argument("--rhos", default="0.8,0.0")
    ap.add_argument("--summary", default=None, help="render a report JSON as markdown")
    args = ap.parse_args()
    if args.summary:
        print(summary(args.summary), end="")
        return
    if args.merge_ncu:
        merge_ncu(args.merge_ncu, args.out)
        return
    torch.cuda.set_device(0)
    if args.ncu_pass:
        for rho in [float(x) for x in args.rhos.split(",")]:
            c3(rho, ncu_pass=True)
        return
    rep = {}
    if os.path.exists(args.out):
        rep = json.load(open(args.out))
    props = torch.cuda.get_device_properties(0)
    rep["device"] = {"name": props.name, "sms": props.multi_processor_count, "l2_bytes": props.L2_cache_size,
                     "host_cpu_cores_used_by_oracle": 1}
    for c in args.cfg.split(","):
        t0 = time.time()
        if c == "C1":
            rep["C1"] = c1()
        elif c == "C2":
            rep["C2"] = c2()
        elif c == "C3":
            for rho in [float(x) for x in args.rhos.split(",")]:
                rep[f"C3_rho{rho}"] = c3(rho)
        elif c == "C4":
            rep["C4"] = c4()
        elif c == "LSTM":
            rep["LSTM_C5"] = lstm("C5")
        elif c == "ATT":
            rep["ATTN_C5"] = attn("C5")
            rep["ATTN_C2"] = attn("C2", H=8, Fh=8)
        elif c == "FS":
            rep["F_sweep"] = fsweep()
        print(f"{c} done in {time.time() - t0:.1f}s", flush=True)
        os.makedirs(os.path.dirname(args.out), exist_ok=True)
        json.dump(rep, open(args.out, "w"), indent=1)
    print(json.dumps(rep, indent=1))


if __name__ == "__main__":
    main()
