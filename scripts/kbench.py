"""Kernel micro-benchmarks on the GPU (dev tool, not the bench contract).

    python scripts/kbench.py gemm            # SIMT vs tcgen05 3xTF32 at the C5 shapes (+ parity)
    python scripts/kbench.py agg [--cfg C5]  # aggregation kernels on a config graph
"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs  # noqa: E402
import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402


def timeit(fn, iters=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(iters):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / iters


def gemm():
    import oracle
    shapes = [(2449029, 100, 256), (2449029, 256, 256), (2449029, 256, 272), (232965, 602, 256),
              (169343, 128, 80), (32768, 64, 128), (4099, 602, 256), (1000, 37, 5)]
    for (m, k, n) in shapes:
        X = torch.rand(m, k, device="cuda") * 2 - 1
        W = (torch.rand(k, n, device="cuda") * 2 - 1) * float(np.sqrt(6 / (k + n)))
        rs = torch.rand(m, device="cuda") + 0.1
        res = {}
        for impl, name in [(1, "simt"), (2, "tc"), (3, "tc_reg")]:
            G.set_gemm_impl(impl)
            try:
                H = G.gemm(X, W, row_scale=rs, simt=(impl == 1))
                torch.cuda.synchronize()
                ms = timeit(lambda: G.gemm(X, W, row_scale=rs, out=H, simt=(impl == 1)))
                res[name] = (ms, H.clone())
            except Exception as e:  # noqa: BLE001
                res[name] = (None, repr(e))
        G.set_gemm_impl(0)
        rows = torch.randint(0, m, (512,), device="cuda")
        ref = oracle.gemm(X[rows].cpu().numpy(), W.cpu().numpy(), rs[rows].cpu().numpy())
        line = f"m={m} k={k} n={n}"
        for name, (ms, H) in res.items():
            if ms is None:
                line += f" | {name}: FAILED {H}"
                continue
            got = H[rows].cpu().numpy()
            err = np.abs(got - ref)
            ok = np.all(err <= 1e-5 + 1e-4 * np.abs(ref))
            tf = 2 * m * k * n / (ms * 1e-3) / 1e12
            gbs = 4 * (m * k + k * n + m * n) / (ms * 1e-3) / 1e9
            line += f" | {name}: {ms:.3f} ms {tf:.1f} TF/s {gbs:.0f} GB/s maxerr {err.max():.2e} ok={ok}"
        print(line, flush=True)


def agg(cfg="C5"):
    t0 = time.time()
    g = gs.config_graph(cfg)
    print(f"{cfg}: n={g.n} nnz={g.nnz} gen {time.time() - t0:.1f}s", flush=True)
    for reorder in (0, 1):
        t0 = time.time()
        plan = G.Plan(g.rowptr, g.colidx, reorder=reorder)
        print(f" plan reorder={reorder}: {time.time() - t0:.1f}s info={plan.info}", flush=True)
        for F in (64, 100, 256):
            X = torch.rand(g.n, F, device="cuda")
            Y = torch.empty_like(X)
            ms = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y), iters=5, warm=2)
            alg = g.nnz * (4 + 4 * F + 4) + g.n * (8 + 4 * F)
            print(f"  F={F}: {ms:.3f} ms  {alg / ms / 1e6:.0f} GB/s algorithmic  "
                  f"{g.nnz * F / ms / 1e6:.1f} Gedge*F/s", flush=True)
        Hh, Fh = 8, 32
        Zs = torch.rand(g.n, Hh * Fh + 2 * Hh, device="cuda")
        Y = torch.empty(g.n, Hh * Fh, device="cuda")
        t = Zs[:, Hh * Fh + Hh:]
        ms = timeit(lambda: G.gat_aggregate(plan, Zs, t, Hh, Fh, out=Y), iters=5, warm=2)
        alg = g.nnz * (4 + 4 * (Hh * Fh + Hh)) + g.n * (8 + 4 * Hh * Fh + 4 * Hh)
        print(f"  GAT 8x32: {ms:.3f} ms  {alg / ms / 1e6:.0f} GB/s algorithmic", flush=True)


def mapsweep(cfg="C5"):
    """a4 mapping sweep: feature chunk width vs time (sum at F=256, GAT 8x32)."""
    t0 = time.time()
    g = gs.config_graph(cfg)
    print(f"{cfg}: n={g.n} nnz={g.nnz} gen {time.time() - t0:.1f}s", flush=True)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    print(f" plan: {plan.info}", flush=True)
    F = 256
    X = torch.rand(g.n, F, device="cuda")
    Y = torch.empty_like(X)
    Hh, Fh = 8, 32
    Zs = torch.rand(g.n, Hh * Fh + 2 * Hh, device="cuda")
    Yg = torch.empty(g.n, Hh * Fh, device="cuda")
    t = Zs[:, Hh * Fh + Hh:]
    maps = [(0, 0, 0), (8, 32, 1), (4, 32, 2), (8, 16, 1), (4, 32, 1), (8, 8, 1), (4, 16, 1), (4, 8, 1), (8, 4, 1),
            (2, 32, 1), (4, 4, 1)]
    for (v, l, nv) in maps:
        G.set_agg_mapping(v, l, nv)
        ms = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y), iters=5, warm=2)
        msg = timeit(lambda: G.gat_aggregate(plan, Zs, t, Hh, Fh, out=Yg), iters=5, warm=2)
        print(f" map vec={v} lanes={l} nv={nv} cw={v * l * nv}: sum F=256 {ms:.3f} ms | GAT 8x32 {msg:.3f} ms",
              flush=True)
    G.set_agg_mapping(0, 0, 0)


def map100(cfg="C5"):
    """a4 sweep at the bench's layer-1 width (F=100, GCN weights) and GAT 8x32."""
    g = gs.config_graph(cfg)
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    X1 = torch.rand(g.n, 100, device="cuda")
    Y1 = torch.empty_like(X1)
    ref = None
    for (v, l, nv) in [(0, 0, 0), (4, 16, 2), (4, 8, 4), (2, 16, 2), (4, 32, 1), (0, 0, 0)]:
        G.set_agg_mapping(v, l, nv)
        ms = timeit(lambda: G.aggregate(plan, X1, "sum", "gcn", out=Y1), iters=5, warm=2)
        same = None if ref is None else bool(torch.equal(ref, Y1))
        ref = Y1.clone() if ref is None else ref
        print(f" F=100 map vec={v} lanes={l} nv={nv}: {ms:.3f} ms identical={same}", flush=True)
    G.set_agg_mapping(0, 0, 0)
    Hh, Fh = 8, 32
    Zs = torch.rand(g.n, Hh * Fh + 2 * Hh, device="cuda") * 2 - 1
    Yg = torch.empty(g.n, Hh * Fh, device="cuda")
    t = Zs[:, Hh * Fh + Hh:]
    for (v, l, nv) in [(0, 0, 0), (8, 16, 2), (8, 8, 4), (4, 16, 2)]:
        G.set_agg_mapping(v, l, nv)
        ms = timeit(lambda: G.gat_aggregate(plan, Zs, t, Hh, Fh, out=Yg), iters=5, warm=2)
        print(f" GAT 8x32 map vec={v} lanes={l} nv={nv}: {ms:.3f} ms", flush=True)
    X2 = torch.rand(g.n, 256, device="cuda")
    Y2 = torch.empty_like(X2)
    for (v, l, nv) in [(0, 0, 0), (8, 16, 2), (8, 8, 4), (4, 16, 2)]:
        G.set_agg_mapping(v, l, nv)
        ms = timeit(lambda: G.aggregate(plan, X2, "sum", "one", out=Y2), iters=5, warm=2)
        print(f" sum F=256 map vec={v} lanes={l} nv={nv}: {ms:.3f} ms", flush=True)
    G.set_agg_mapping(0, 0, 0)


def tune():
    """NEXT-1 tuner on the config graphs: default vs tuned (bound, mapping)."""
    for cfg, F in [("C1", 16), ("C2", 64), ("C5", 100), ("C5", 256)]:
        g = gs.config_graph(cfg)
        plan = G.Plan(g.rowptr, g.colidx, reorder=1)
        X = torch.rand(g.n, F, device="cuda")
        t0 = time.time()
        r = G.tune_aggregate(plan, X, "sum", "gcn")
        print(f" {cfg} F={F}: {r} in {time.time() - t0:.1f}s", flush=True)
        del plan


def c2gat():
    """GAT mappings on the arxiv-shaped graph (C2, 8 heads x 8)."""
    g = gs.config_graph("C2")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    H, Fh = 8, 8
    HF = H * Fh
    Zs = torch.rand((g.n, HF + 2 * H), device="cuda") * 2 - 1
    t = Zs[:, HF + H:]
    Y = torch.empty((g.n, HF), device="cuda")
    ref = None
    X = torch.rand((g.n, HF), device="cuda")
    for m in [(0, 0, 0), (4, 32, 1), (2, 32, 1), (1, 32, 1)]:
        G.set_agg_mapping(*m)
        ms = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y), iters=20, warm=3)
        print(f" C2 sum F=64 map {m}: {ms * 1e3:.1f} us", flush=True)
    g1 = gs.config_graph("C1")
    p1 = G.Plan(g1.rowptr, g1.colidx, reorder=1)
    X1 = torch.rand((g1.n, 16), device="cuda")
    Y1 = torch.empty_like(X1)
    for m in [(0, 0, 0), (4, 32, 1), (2, 32, 1), (1, 32, 1), (8, 4, 1)]:
        G.set_agg_mapping(*m)
        ms = timeit(lambda: G.aggregate(p1, X1, "sum", "gcn", out=Y1), iters=50, warm=5)
        print(f" C1 sum F=16 map {m}: {ms * 1e3:.1f} us", flush=True)
    for m in [(0, 0, 0), (4, 32, 1), (8, 32, 1), (2, 32, 1), (4, 16, 1), (8, 8, 1)]:
        G.set_agg_mapping(*m)
        ms = timeit(lambda: G.gat_aggregate(plan, Zs, t, H, Fh, out=Y), iters=20, warm=3)
        d = 0.0 if ref is None else float((Y - ref).abs().max())
        ref = Y.clone() if ref is None else ref
        print(f" C2 GAT map {m}: {ms * 1e3:.1f} us  max|diff| {d:.2e}", flush=True)
    G.set_agg_mapping(0, 0, 0)


def c4map():
    """EdgeConv max aggregation mappings on the kNN graph (C4, F=64, k=20)."""
    g = gs.config_graph("C4")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    PQ = torch.rand((g.n, 128), device="cuda") * 2 - 1
    Y = torch.empty((g.n, 64), device="cuda")
    X = torch.rand((g.n, 64), device="cuda")
    for m in [(0, 0, 0), (2, 32, 1), (4, 32, 1), (8, 8, 1), (4, 16, 1)]:
        G.set_agg_mapping(*m)
        a = timeit(lambda: G.edgeconv_aggregate(plan, PQ, 64, out=Y), iters=50, warm=5)
        b = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y), iters=50, warm=5)
        print(f" C4 map {m}: edgeconv max {a * 1e3:.1f} us | sum gcn {b * 1e3:.1f} us", flush=True)
    G.set_agg_mapping(0, 0, 0)


def pad104():
    """agg1 of the bench (GCN weights) at F=100 vs the same rows padded to 104."""
    g = gs.config_graph("C5")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    X = torch.rand((g.n, 104), device="cuda")
    X[:, 100:] = 0
    Y = torch.empty_like(X)
    Y100 = torch.empty((g.n, 100), device="cuda")
    X100 = X[:, :100].contiguous()
    print(f" F=100 (ld 100): {timeit(lambda: G.aggregate(plan, X100, 'sum', 'gcn', out=Y100)):.3f} ms", flush=True)
    for m in [(0, 0, 0), (8, 32, 1), (4, 16, 2), (4, 32, 1)]:
        G.set_agg_mapping(*m)
        ms = timeit(lambda: G.aggregate(plan, X, "sum", "gcn", out=Y))
        print(f" F=104 map {m}: {ms:.3f} ms  same as F=100 {bool(torch.equal(Y[:, :100], Y100))}", flush=True)
    G.set_agg_mapping(0, 0, 0)


def c1probe():
    """C1 (Cora) aggregate calls for an ncu launch list (launch-bound config)."""
    g = gs.config_graph("C1")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    X = torch.rand(g.n, 16, device="cuda")
    Y = torch.empty_like(X)
    for _ in range(5):
        G.aggregate(plan, X, "sum", "gcn", relu=True, out=Y)
    torch.cuda.synchronize()
    print(plan.info, flush=True)


def lstm_probe():
    """GraphSAGE-LSTM cell kernel on the C5 graph (for ncu / quick timing)."""
    g = gs.config_graph("C5")
    plan = G.Plan(g.rowptr, g.colidx, reorder=1)
    F, T = 32, 16
    rng = np.random.default_rng(1)
    P = {k: torch.from_numpy(rng.uniform(-0.3, 0.3, size=s).astype(np.float32)).cuda() for k, s in
         dict(W_hh=(4 * F, F), W_neigh=(F, F)).items()}
    GS = torch.rand((g.n, 5 * F), device="cuda") - 0.5
    tab = G.sample_neighbors(plan, T, 7)
    Y = torch.empty((g.n, F), device="cuda")
    ms = timeit(lambda: G.sage_lstm_aggregate(plan, tab, GS, P["W_hh"], P["W_neigh"], out=Y), iters=5, warm=2)
    print(f" lstm cells: {ms:.3f} ms", flush=True)

if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "gemm"
    if what == "gemm":
        gemm()
    elif what == "tune":
        tune()
    elif what == "lstm":
        lstm_probe()
    elif what == "c2gat":
        c2gat()
    elif what == "c4map":
        c4map()
    elif what == "pad104":
        pad104()
    elif what == "c1":
        c1probe()
    elif what == "map100":
        map100(sys.argv[sys.argv.index("--cfg") + 1] if "--cfg" in sys.argv else "C5")
    elif what == "map":
        mapsweep(sys.argv[sys.argv.index("--cfg") + 1] if "--cfg" in sys.argv else "C5")
    else:
        agg(sys.argv[sys.argv.index("--cfg") + 1] if "--cfg" in sys.argv else "C5")
