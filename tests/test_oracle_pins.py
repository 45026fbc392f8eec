"""Pins for the oracle (CPU only, `-m "not gpu"`).

Every oracle function is checked against something other than itself: values
the paper prints or a hand computation (tests/golden/), closed forms,
invariants, textbook special cases, or an independent brute-force formulation
(dense adjacency matmul, edge-list scatter) on tiny inputs.  Each test names
the PAPER.md passage (P:<line>) it pins.
"""
import math

import numpy as np
import pytest

import gnn_synth as gs
import oracle
from conftest import golden_path

RTOL, ATOL = 1e-4, 1e-5  # BASELINE.json north_star tolerance


def read_golden(name):
    out = {}
    rows = []
    for line in open(golden_path(name)):
        line = line.split("#")[0].strip()
        if not line:
            continue
        key, _, val = line.partition(":")
        if key.strip().isdigit():
            rows.append([int(x) for x in val.split()])
        else:
            out[key.strip()] = val.split()
    out["rows"] = rows
    return out


def dense_adj(g, weight="one", edge_w=None):
    """Independent formulation: dense fp64 adjacency A[v, u] += e_uv."""
    n = g.n
    A = np.zeros((n, n), np.float64)
    d_in = np.diff(g.rowptr).astype(np.float64)
    d_out = np.bincount(g.colidx, minlength=n).astype(np.float64)
    for v in range(n):
        for k in range(g.rowptr[v], g.rowptr[v + 1]):
            u = g.colidx[k]
            if weight == "one":
                e = 1.0
            elif weight == "gcn":
                e = 1.0 / math.sqrt(d_out[u] * d_in[v])
            else:
                e = float(edge_w[k])
            A[v, u] += e
    return A, d_in


def edge_list_max(g, X, weight="one", edge_w=None):
    """Independent formulation (edge-wise expand + scatter-max, Fig 2 upper)."""
    n = g.n
    dst = np.repeat(np.arange(n), np.diff(g.rowptr))
    src = g.colidx.astype(np.int64)
    if weight == "one":
        e = np.ones(len(src))
    elif weight == "gcn":
        d_in = np.diff(g.rowptr).astype(np.float64)
        d_out = np.bincount(src, minlength=n).astype(np.float64)
        e = 1.0 / np.sqrt(d_out[src] * d_in[dst])
    else:
        e = edge_w.astype(np.float64)
    msg = e[:, None] * X.astype(np.float64)[src]
    Y = np.full((n, X.shape[1]), -np.inf)
    np.maximum.at(Y, dst, msg)
    Y[np.diff(g.rowptr) == 0] = 0.0
    return Y


def close(a, b, rtol=RTOL, atol=ATOL):
    return np.all(np.abs(a.astype(np.float64) - b) <= atol + rtol * np.abs(b))


# --------------------------------------------------------------------------- #
# a6 aggregation: Table 1 x Table 2
# --------------------------------------------------------------------------- #
def test_fig2_hand_graph():
    """Fig 2 toy graph (reading R2) by hand: golden sum/mean/max."""
    gd = read_golden("fig2_graph.txt")
    g = gs.from_rows(gd["rows"])
    X = np.arange(5, dtype=np.float32)[:, None]
    for red in ("sum", "mean", "max"):
        Y = oracle.aggregate(g.rowptr, g.colidx, X, reduce=red)
        want = np.array([float(x) for x in gd[red]], np.float32)
        assert np.array_equal(Y[:, 0], want), (red, Y[:, 0], want)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("weight", ["one", "gcn", "edge"])
def test_sum_mean_vs_dense_adjacency(seed, weight):
    """sum/mean == dense fp64 A @ X (independent brute force), incl. empty rows,
    self loops and multi-edges (reading R1)."""
    g = gs.random_small(40 + seed * 7, avg_deg=3 + seed, seed=seed, self_loops=seed % 2 == 1,
                        multi=seed % 3 == 2)
    X = gs.uniform(g.n, 5 + seed, seed=seed + 100)
    ew = gs.uniform(g.nnz, 1, seed=seed + 200)[:, 0] if weight == "edge" else None
    A, d_in = dense_adj(g, weight, ew)
    ref = A @ X.astype(np.float64)
    Y = oracle.aggregate(g.rowptr, g.colidx, X, "sum", weight, ew)
    assert close(Y, ref, 1e-6, 1e-7)
    Ym = oracle.aggregate(g.rowptr, g.colidx, X, "mean", weight, ew)
    refm = np.where(d_in[:, None] > 0, ref / np.maximum(d_in, 1)[:, None], 0.0)
    assert close(Ym, refm, 1e-6, 1e-7)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("weight", ["one", "gcn", "edge"])
def test_max_vs_edge_scatter(seed, weight):
    """max == edge-wise expand + scatter-max (PyG formulation); exact."""
    g = gs.random_small(50, avg_deg=4, seed=seed, multi=seed % 2 == 0)
    X = gs.uniform(g.n, 7, seed=seed)
    ew = gs.uniform(g.nnz, 1, seed=seed + 9)[:, 0] if weight == "edge" else None
    Y = oracle.aggregate(g.rowptr, g.colidx, X, "max", weight, ew)
    assert np.array_equal(Y, edge_list_max(g, X, weight, ew).astype(np.float32))


def test_integer_features_exact():
    """Integer-valued X with const weights: every partial sum is an exact
    integer, so sum/mean/max equal exact integer arithmetic."""
    g = gs.random_small(200, avg_deg=12, seed=3)
    Xi = np.random.default_rng(1).integers(-8, 9, size=(g.n, 9))
    A, d_in = dense_adj(g)
    s = (A.astype(np.int64) @ Xi)
    Y = oracle.aggregate(g.rowptr, g.colidx, Xi.astype(np.float32), "sum")
    assert np.array_equal(Y, s.astype(np.float32))
    Ym = oracle.aggregate(g.rowptr, g.colidx, Xi.astype(np.float32), "mean")
    want = np.where(d_in[:, None] > 0, s / np.maximum(d_in, 1)[:, None], 0).astype(np.float32)
    assert np.array_equal(Ym, want)


def test_gcn_complete_graph_closed_form():
    """K_n without self loops, GCN weights 1/sqrt((n-1)(n-1)): row v =
    (SUM_{u != v} x_u)/(n-1) (Table 2 GCN)."""
    n = 9
    g = gs.from_rows([[u for u in range(n) if u != v] for v in range(n)])
    X = gs.uniform(n, 4, seed=5)
    tot = X.astype(np.float64).sum(0)
    want = (tot[None, :] - X) / (n - 1)
    Y = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn")
    assert close(Y, want, 1e-6, 1e-7)


def test_gcn_regular_equals_mean():
    """d-regular (in == out degree d): e_gcn = 1/d, so GCN-sum == mean."""
    n, d = 30, 4
    g = gs.from_rows([sorted((v + k) % n for k in range(1, d + 1)) for v in range(n)])
    X = gs.uniform(n, 6, seed=2)
    a = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn")
    b = oracle.aggregate(g.rowptr, g.colidx, X, "mean", "one")
    assert close(a, b.astype(np.float64), 1e-6, 1e-7)


def test_star_graph_and_empty_rows_relu():
    """Star: hub row 0 gathers leaves 1..n-1, leaves are empty -> 0 for every
    reducer (reading R3-i); ReLU clamps the hub (Eq 1 ACT)."""
    n = 6
    g = gs.from_rows([list(range(1, n))] + [[] for _ in range(n - 1)])
    X = -np.ones((n, 3), np.float32)
    for red in ("sum", "mean", "max"):
        Y = oracle.aggregate(g.rowptr, g.colidx, X, red)
        assert np.all(Y[1:] == 0)
        assert np.all(Y[0] == {"sum": -5, "mean": -1, "max": -1}[red])
        Yr = oracle.aggregate(g.rowptr, g.colidx, X, red, relu=True)
        assert np.all(Yr == 0)


def test_row_sampling_matches_full():
    g = gs.random_small(80, avg_deg=5, seed=8)
    X = gs.uniform(g.n, 8, seed=8)
    full = oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn")
    rows = np.array([5, 0, 79, 33])
    assert np.array_equal(oracle.aggregate(g.rowptr, g.colidx, X, "sum", "gcn", rows=rows), full[rows])


@pytest.mark.parametrize("ng", [0, 1, 3, 16])
@pytest.mark.parametrize("red", ["sum", "mean", "max"])
@pytest.mark.parametrize("weight", ["one", "gcn", "edge"])
def test_ng_f32_order_replica(ng, red, weight):
    """The deterministic-order fp32 replica (R9) agrees with the fp64
    definition within the north_star tolerance, and exactly on integers."""
    g = gs.random_small(120, avg_deg=20, seed=ng + 1)
    X = gs.uniform(g.n, 11, seed=ng)
    ew = gs.uniform(g.nnz, 1, seed=3)[:, 0] if weight == "edge" else None
    ref = oracle.aggregate(g.rowptr, g.colidx, X, red, weight, ew)
    Y = oracle.aggregate_ng_f32(g.rowptr, g.colidx, X, ng, red, weight, ew)
    assert close(Y, ref.astype(np.float64))
    if red == "max" and weight == "one":
        assert np.array_equal(Y, ref)
    Xi = gs.integer_features(g.n, 5, seed=2)
    if weight == "one":
        assert np.array_equal(oracle.aggregate_ng_f32(g.rowptr, g.colidx, Xi, ng, red),
                              oracle.aggregate(g.rowptr, g.colidx, Xi, red))


# --------------------------------------------------------------------------- #
# a5 dense transform and the GCN layer (Eq 1)
# --------------------------------------------------------------------------- #
def test_gemm_vs_numpy():
    X = gs.uniform(37, 29, seed=1)
    W = gs.uniform(29, 13, seed=2)
    rs = gs.uniform(37, 1, lo=0.1, hi=2.0, seed=3)[:, 0]
    ref = (X.astype(np.float64) @ W.astype(np.float64)) * rs[:, None].astype(np.float64)
    assert close(oracle.gemm(X, W, rs), ref, 1e-6, 1e-7)


def test_gcn_layer_vs_dense():
    """Eq 1: ReLU((A_gcn X) W) == numpy fp64 A_hat @ X @ W (textbook GCN)."""
    g = gs.random_small(60, avg_deg=5, seed=4)
    X = gs.uniform(g.n, 17, seed=1)
    W = gs.uniform(17, 6, seed=2)
    A, _ = dense_adj(g, "gcn")
    ref = np.maximum(A @ X.astype(np.float64) @ W.astype(np.float64), 0)
    assert close(oracle.gcn_layer(g.rowptr, g.colidx, X, W, relu=True), ref, 1e-6, 1e-7)
    ref2 = A @ X.astype(np.float64) @ W.astype(np.float64)
    assert close(oracle.gcn_layer(g.rowptr, g.colidx, X, W, relu=False), ref2, 1e-6, 1e-7)


# --------------------------------------------------------------------------- #
# a7 GAT: Eq 2, Listing 1, Table 2 GAT
# --------------------------------------------------------------------------- #
def dense_gat(g, Z, s, t, H, Fh, slope):
    """Independent formulation: dense masked softmax over the adjacency."""
    n = g.n
    mask = np.zeros((n, n), bool)
    cnt = np.zeros((n, n))
    for v in range(n):
        for k in range(g.rowptr[v], g.rowptr[v + 1]):
            mask[v, g.colidx[k]] = True
            cnt[v, g.colidx[k]] += 1
    Y = np.zeros((n, H * Fh))
    for h in range(H):
        e = s[None, :, h] + t[:, None, h]
        e = np.where(e > 0, e, slope * e)
        e = np.where(mask, e, -np.inf)
        m = e.max(1, keepdims=True)
        m[~np.isfinite(m)] = 0
        p = np.exp(e - m) * cnt
        den = p.sum(1, keepdims=True)
        a = np.where(den > 0, p / np.where(den > 0, den, 1), 0)
        Y[:, h * Fh:(h + 1) * Fh] = a @ Z[:, h * Fh:(h + 1) * Fh]
    return Y


def make_zs(Z, s):
    return np.concatenate([Z, s], 1).astype(np.float32)


@pytest.mark.parametrize("seed", range(4))
def test_gat_aggregate_vs_dense_softmax(seed):
    g = gs.random_small(45, avg_deg=5, seed=seed, multi=seed == 3)
    H, Fh = 3, 4
    Z = gs.uniform(g.n, H * Fh, seed=seed)
    s = gs.uniform(g.n, H, lo=-3, hi=3, seed=seed + 1)
    t = gs.uniform(g.n, H, lo=-3, hi=3, seed=seed + 2)
    Y = oracle.gat_aggregate(g.rowptr, g.colidx, make_zs(Z, s), t, H, Fh, 0.2)
    ref = dense_gat(g, Z.astype(np.float64), s.astype(np.float64), t.astype(np.float64), H, Fh, 0.2)
    assert close(Y, ref, 1e-6, 1e-7)


def test_gat_uniform_attention_is_mean():
    """a_src = a_dst = 0 -> all scores 0 -> uniform softmax -> mean.  alpha = 1/d
    is inexact in binary, so the match is to fp64 rounding, not bitwise."""
    g = gs.random_small(70, avg_deg=6, seed=1)
    H, Fh = 2, 3
    Z = gs.integer_features(g.n, H * Fh, seed=4)
    zeros = np.zeros((g.n, H), np.float32)
    Y = oracle.gat_aggregate(g.rowptr, g.colidx, make_zs(Z, zeros), zeros, H, Fh)
    assert close(Y, oracle.aggregate(g.rowptr, g.colidx, Z, "mean").astype(np.float64), 1e-6, 1e-7)


def test_gat_single_neighbor_identity():
    g = gs.from_rows([[2], [0], [1]])
    Z = gs.uniform(3, 4, seed=3)
    s = gs.uniform(3, 2, lo=-50, hi=50, seed=1)
    t = gs.uniform(3, 2, lo=-50, hi=50, seed=2)
    Y = oracle.gat_aggregate(g.rowptr, g.colidx, make_zs(Z, s), t, 2, 2)
    assert np.array_equal(Y, Z[[2, 0, 1]])


def test_gat_two_neighbors_hand():
    gd = read_golden("gat_two_neighbors.txt")
    g = gs.from_rows([[1, 2], [], []])
    z = np.array([[0], [8], [-4]], np.float32)
    s = np.array([[0], [math.log(3)], [0]], np.float32)
    t = np.array([[1], [0], [0]], np.float32)
    Y = oracle.gat_aggregate(g.rowptr, g.colidx, make_zs(z, s), t, 1, 1)
    assert abs(Y[0, 0] - float(gd["y"][0])) < 1e-6
    assert Y[1, 0] == 0 and Y[2, 0] == 0


def test_gat_softmax_rows_sum_to_one_and_large_scores():
    """Append a ones column to z: the output column is sum(alpha) = 1; huge
    |e| ~ 1e4 stays finite (max shift, reading R5-ii)."""
    g = gs.random_small(60, avg_deg=7, seed=2, allow_empty=False)
    H, Fh = 1, 3
    Z = gs.uniform(g.n, Fh, seed=1)
    Z[:, -1] = 1.0
    s = gs.uniform(g.n, 1, lo=-1e4, hi=1e4, seed=2)
    t = gs.uniform(g.n, 1, lo=-1e4, hi=1e4, seed=3)
    Y = oracle.gat_aggregate(g.rowptr, g.colidx, make_zs(Z, s), t, H, Fh)
    assert np.all(np.isfinite(Y))
    assert np.allclose(Y[:, -1], 1.0, atol=1e-6)


def test_gat_layer_vs_dense():
    """Full layer: Z = XW, s/t per head, then Eq 2 (dense formulation)."""
    g = gs.random_small(40, avg_deg=5, seed=6)
    H, Fh, fin = 2, 3, 7
    X = gs.uniform(g.n, fin, seed=1)
    W = gs.uniform(fin, H * Fh, seed=2)
    a_s = gs.uniform(1, H * Fh, seed=3)[0]
    a_d = gs.uniform(1, H * Fh, seed=4)[0]
    Z = X.astype(np.float64) @ W.astype(np.float64)
    s = np.stack([Z[:, h * Fh:(h + 1) * Fh] @ a_s[h * Fh:(h + 1) * Fh] for h in range(H)], 1)
    t = np.stack([Z[:, h * Fh:(h + 1) * Fh] @ a_d[h * Fh:(h + 1) * Fh] for h in range(H)], 1)
    ref = dense_gat(g, Z, s, t, H, Fh, 0.2)
    Y = oracle.gat_layer(g.rowptr, g.colidx, X, W, a_s, a_d, H, Fh, 0.2)
    assert close(Y, ref, 1e-6, 1e-7)


# --------------------------------------------------------------------------- #
# a8 EdgeConv (reading R6; pooling P:236-237, redundancy bypass P:1014-1021)
# --------------------------------------------------------------------------- #
def dense_edgeconv(g, X, th, ph, b):
    n = g.n
    X = X.astype(np.float64)
    Y = np.zeros((n, th.shape[0]))
    for v in range(n):
        nb = g.colidx[g.rowptr[v]:g.rowptr[v + 1]]
        if len(nb) == 0:
            continue
        h = (X[nb] - X[v]) @ th.T.astype(np.float64) + X[v] @ ph.T.astype(np.float64) + b
        Y[v] = np.maximum(h, 0).max(0)
    return Y


def test_edgeconv_vs_dense_and_special_cases():
    g = gs.random_small(50, avg_deg=4, seed=1)
    fin, fout = 6, 5
    X = gs.uniform(g.n, fin, seed=1)
    th = gs.uniform(fout, fin, seed=2)
    ph = gs.uniform(fout, fin, seed=3)
    b = gs.uniform(1, fout, lo=-0.1, hi=0.1, seed=4)[0]
    Y = oracle.edgeconv(g.rowptr, g.colidx, X, th, ph, b)
    assert close(Y, dense_edgeconv(g, X, th, ph, b.astype(np.float64)), 1e-6, 1e-7)
    nonempty = np.diff(g.rowptr) > 0
    # theta = 0 -> y_v = ReLU(phi x_v + b) for d_v >= 1
    Y0 = oracle.edgeconv(g.rowptr, g.colidx, X, np.zeros_like(th), ph, b)
    want0 = np.maximum(X.astype(np.float64) @ ph.T.astype(np.float64) + b, 0)
    assert close(Y0[nonempty], want0[nonempty], 1e-6, 1e-7)
    assert np.all(Y0[~nonempty] == 0)
    # phi = theta -> y_v = ReLU(b + max_u theta x_u) (GraphSAGE-pool form)
    Y1 = oracle.edgeconv(g.rowptr, g.colidx, X, th, th, b)
    P = X.astype(np.float64) @ th.T.astype(np.float64)
    for v in np.nonzero(nonempty)[0]:
        nb = g.colidx[g.rowptr[v]:g.rowptr[v + 1]]
        assert close(Y1[v], np.maximum(b + P[nb].max(0), 0), 1e-6, 1e-7)


# --------------------------------------------------------------------------- #
# a2 LAS, reading R7
# --------------------------------------------------------------------------- #
def test_splitmix64_known_answers():
    gd = read_golden("splitmix64.txt")
    want = [int(x, 16) for x in gd["seed 0"]]
    assert oracle.splitmix64_stream(0, 2) == want


def test_fmix64_bijection_sample():
    vals = {oracle.fmix64(x) for x in range(5000)}
    assert len(vals) == 5000
    assert oracle.fmix64(0) == 0  # fixed point of the xor-shift-multiply finalizer


def test_minhash_estimates_jaccard():
    """P[sig agree] = Jaccard (Min-Hashing, MMDS [24]): {0..99} vs
    {50..149}, J = 1/3; mean over seeds within 3 sigma."""
    g = gs.from_rows([list(range(100)), list(range(50, 150))] + [[] for _ in range(148)])
    K = 32
    est = []
    for seed in range(300):
        sig = oracle.minhash(g.rowptr, g.colidx, K, seed)
        est.append(np.mean(sig[0] == sig[1]))
    J = 1 / 3
    sd = math.sqrt(J * (1 - J) / (K * 300))
    assert abs(np.mean(est) - J) < 3 * sd


def test_minhash_definition_small():
    """sig[v][k] == min over neighbours of h_k(u), h_k(u) = fmix64(u + c_k)."""
    g = gs.from_rows([[3, 7, 9], [], [1]])
    sig = oracle.minhash(g.rowptr, g.colidx, 4, seed=11)
    c = oracle.splitmix64_stream(11, 4)
    M = (1 << 64) - 1
    for k in range(4):
        assert sig[0, k] == min(oracle.fmix64((u + c[k]) & M) for u in (3, 7, 9))
        assert sig[1, k] == M
        assert sig[2, k] == oracle.fmix64((1 + c[k]) & M)


def test_las_identical_neighborhoods_blocks_of_32():
    """Hand trace (1): 100 rows with identical neighbour sets -> clusters of
    32 (cap) = {0..31},{32..63},{64..95},{96..99}; perm = identity."""
    g = gs.from_rows([[100, 101, 102, 103, 104] for _ in range(100)] + [[] for _ in range(5)])
    perm, info = oracle.las_schedule(g.rowptr, g.colidx, seed=3)
    cl = info["cluster_of"]
    assert np.array_equal(perm, np.arange(105))
    for lo, hi in [(0, 32), (32, 64), (64, 96), (96, 100)]:
        assert len(set(cl[lo:hi])) == 1
    assert len(set(cl[:100])) == 4
    assert info["n_clusters"] == 4 + 5


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_las_recovers_planted_groups(seed):
    """Hand trace (2): planted groups (<= 32 members) sharing one neighbour set,
    sets disjoint, other rows empty, random relabel -> each group is one
    cluster, listed contiguously in perm."""
    rng = np.random.default_rng(seed)
    sizes = [32, 5, 17, 2, 32, 9]
    n = sum(sizes) + 400
    relabel = rng.permutation(n)
    rows = [[] for _ in range(n)]
    groups = []
    base = 0
    for gi, sz in enumerate(sizes):
        members = [int(relabel[base + j]) for j in range(sz)]
        nbrs = sorted(int(x) for x in relabel[sum(sizes) + 40 * gi: sum(sizes) + 40 * gi + 12])
        for m in members:
            rows[m] = nbrs
        groups.append(sorted(members))
        base += sz
    g = gs.from_rows(rows)
    perm, info = oracle.las_schedule(g.rowptr, g.colidx, seed=seed)
    cl = info["cluster_of"]
    pos = np.empty(n, np.int64)
    pos[perm] = np.arange(n)
    for members in groups:
        assert len({cl[m] for m in members}) == 1
        assert sum(cl == cl[members[0]]) == len(members)
        p = sorted(pos[members])
        assert p[-1] - p[0] == len(members) - 1


@pytest.mark.parametrize("seed", [0, 1])
def test_las_invariants_powerlaw(seed):
    g = gs.powerlaw(3000, 30000, 10, 300, 400, comm=32, rho=0.8, seed=seed)
    perm, info = oracle.las_schedule(g.rowptr, g.colidx, seed=seed)
    n = g.n
    assert np.array_equal(np.sort(perm), np.arange(n))
    cl = info["cluster_of"]
    sizes = np.bincount(cl, minlength=n)
    assert sizes.max() <= 32
    # members of a cluster are contiguous in perm and ascending; clusters ordered by
    # (representative signature, min member) (R7)
    sig_ = info["sig"]
    seen = []
    i = 0
    while i < n:
        c = cl[perm[i]]
        j = i
        while j < n and cl[perm[j]] == c:
            j += 1
        assert j - i == sizes[c]
        assert np.all(np.diff(perm[i:j]) > 0)
        seen.append((tuple(int(x) for x in sig_[c]), int(perm[i])))
        i = j
    assert seen == sorted(seen)
    # the smallest-member order (cluster_order 0) is the other option
    perm0, _, _, _ = oracle.las_merge(info["sig"], info["pairs"], 32, 2, cluster_order=0)
    heads = [int(v) for k, v in enumerate(perm0) if k == 0 or cl[perm0[k - 1]] != cl[v]]
    assert heads == sorted(heads)
    # every candidate pair shares a full band (LSH bucket); sim >= r
    sig, pairs = info["sig"], info["pairs"]
    for a, b in pairs[:2000]:
        agree = sig[a] == sig[b]
        assert agree.reshape(16, 2).all(1).any()
    # every merge grouped rows with a common band: clusters are connected via >= r agreement
    assert info["merges"] == n - info["n_clusters"]
    # deterministic
    perm2, _ = oracle.las_schedule(g.rowptr, g.colidx, seed=seed)
    assert np.array_equal(perm, perm2)


# --------------------------------------------------------------------------- #
# a3 neighbor grouping (reading R8)
# --------------------------------------------------------------------------- #
@pytest.mark.parametrize("ng", [0, 1, 4, 16, 64])
def test_neighbor_groups_cover_edges(ng):
    g = gs.random_small(300, avg_deg=9, seed=ng)
    perm = np.random.default_rng(ng).permutation(g.n).astype(np.int32)
    gr, gb = oracle.neighbor_groups(g.rowptr, ng, perm)
    deg = np.diff(g.rowptr)
    expect_G = int(np.sum(np.ceil(deg / ng))) if ng > 0 else int(np.sum(deg > 0))
    assert len(gr) == expect_G
    covered = np.zeros(g.nnz, np.int64)
    ends = np.minimum(gb + (ng if ng > 0 else 10 ** 9), g.rowptr[gr + 1])
    for r, b, e in zip(gr, gb, ends):
        assert g.rowptr[r] <= b < e <= g.rowptr[r + 1]
        if ng > 0:
            assert e - b <= ng
        covered[b:e] += 1
    assert np.all(covered == 1)
    # schedule order: rows appear in perm order
    order = [r for i, r in enumerate(gr) if i == 0 or gr[i - 1] != r]
    assert order == [int(v) for v in perm if deg[v] > 0]


def test_partition_rows():
    g = gs.powerlaw(5000, 80000, 16, 900, 700, comm=32, rho=0.0, seed=4)
    E = g.nnz
    maxd = np.diff(g.rowptr).max()
    for P in (1, 2, 4, 8):
        b = oracle.partition_rows(g.rowptr, P)
        assert b[0] == 0 and b[-1] == g.n and np.all(np.diff(b) >= 0)
        nnz = np.diff(g.rowptr[b])
        assert nnz.sum() == E
        assert np.all(nnz <= E / P + maxd)


# --------------------------------------------------------------------------- #
# NEXT-3 GraphSAGE-LSTM (Fig 6; reading R13)
# --------------------------------------------------------------------------- #
def _lstm_params(f_in, F, F_out, seed, scale=0.3):
    rng = np.random.default_rng(seed)
    u = lambda *s: (rng.uniform(-scale, scale, size=s)).astype(np.float32)  # noqa: E731
    return dict(W_ih=u(4 * F, f_in), W_hh=u(4 * F, F), b_ih=u(4 * F), b_hh=u(4 * F), W_self=u(F_out, f_in),
                W_neigh=u(F_out, F), bias=u(F_out))


def test_sage_lstm_matches_torch_lstm():
    """The LSTM cell chain (Fig 6, gate blocks i, f, z, o) against PyTorch's
    nn.LSTM in fp64 on the same sampled sequences (a library routine), then
    the SAGE combine y = W_self x_v + W_neigh h_T + b by numpy."""
    torch = pytest.importorskip("torch")
    g = gs.random_small(60, avg_deg=6, seed=11)
    f_in, F, F_out, T = 12, 8, 5, 7
    X = gs.uniform(g.n, f_in, seed=12)
    P = _lstm_params(f_in, F, F_out, 13)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, T, seed=5)
    Y = oracle.sage_lstm(X, table, **P)
    lstm = torch.nn.LSTM(f_in, F, batch_first=True).double()
    with torch.no_grad():
        lstm.weight_ih_l0.copy_(torch.from_numpy(P["W_ih"].astype(np.float64)))
        lstm.weight_hh_l0.copy_(torch.from_numpy(P["W_hh"].astype(np.float64)))
        lstm.bias_ih_l0.copy_(torch.from_numpy(P["b_ih"].astype(np.float64)))
        lstm.bias_hh_l0.copy_(torch.from_numpy(P["b_hh"].astype(np.float64)))
    deg = np.diff(g.rowptr)
    ref = np.empty_like(Y, dtype=np.float64)
    for v in range(g.n):
        h = np.zeros(F)
        if deg[v] > 0:
            seq = torch.from_numpy(X[table[v]].astype(np.float64))[None]
            with torch.no_grad():
                _, (hT, _) = lstm(seq)
            h = hT[0, 0].numpy()
        ref[v] = P["W_self"].astype(np.float64) @ X[v] + P["W_neigh"].astype(np.float64) @ h + P["bias"]
    assert np.allclose(Y, ref, rtol=1e-6, atol=1e-7)


def test_sage_lstm_zero_weights_closed_form():
    """W = R = 0: every cell sees only its biases, c_t = s_f c_{t-1} + s_i tanh(b_z),
    so c_T = s_i tanh(b_z) (1 - s_f^T) / (1 - s_f) and h_T = s_o tanh(c_T)."""
    g = gs.random_small(40, avg_deg=3, seed=2, allow_empty=True)
    f_in, F, T = 6, 4, 16
    P = _lstm_params(f_in, F, F, 3, scale=1.0)
    P["W_ih"][:] = 0
    P["W_hh"][:] = 0
    P["W_self"][:] = 0
    P["W_neigh"] = np.eye(F, dtype=np.float32)
    P["bias"][:] = 0
    X = gs.uniform(g.n, f_in, seed=4)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, T, seed=1)
    Y = oracle.sage_lstm(X, table, **P)
    b = P["b_ih"].astype(np.float64) + P["b_hh"]
    sig = lambda x: 1 / (1 + np.exp(-x))  # noqa: E731
    si, sf, sz, so = sig(b[:F]), sig(b[F:2 * F]), np.tanh(b[2 * F:3 * F]), sig(b[3 * F:])
    cT = si * sz * (1 - sf ** T) / (1 - sf)
    hT = so * np.tanh(cT)
    deg = np.diff(g.rowptr)
    assert np.allclose(Y[deg > 0], hT[None, :], rtol=1e-6, atol=1e-7)
    assert np.all(Y[deg == 0] == 0)


def test_sage_lstm_empty_rows_and_single_step():
    """Empty rows: h_T = 0, y = W_self x_v + b.  T = 1: h_1 = s(o) tanh(s(i) tanh(z))
    with the gate pre-activations computed by a dense matmul of the one neighbour."""
    g = gs.from_rows([[1], [], [0], [2]])
    f_in, F, F_out = 3, 2, 2
    P = _lstm_params(f_in, F, F_out, 9, scale=0.8)
    X = gs.uniform(g.n, f_in, seed=10)
    table = oracle.sample_neighbors(g.rowptr, g.colidx, 1, seed=0)
    assert table.ravel().tolist() == [1, -1, 0, 2]
    Y = oracle.sage_lstm(X, table, **P)
    W = {k: v.astype(np.float64) for k, v in P.items()}
    assert np.allclose(Y[1], W["W_self"] @ X[1] + W["bias"], rtol=1e-6, atol=1e-7)
    sig = lambda x: 1 / (1 + np.exp(-x))  # noqa: E731
    for v, u in ((0, 1), (2, 0), (3, 2)):
        a = W["W_ih"] @ X[u] + W["b_ih"] + W["b_hh"]
        h = sig(a[3 * F:]) * np.tanh(sig(a[:F]) * np.tanh(a[2 * F:3 * F]))
        assert np.allclose(Y[v], W["W_self"] @ X[v] + W["W_neigh"] @ h + W["bias"], rtol=1e-6, atol=1e-7)


def test_sample_neighbors_uniform_with_replacement():
    """Reading R13: every sample is a neighbour of its row; degree-1 rows repeat
    their neighbour; on a degree-4 row, T = 4000 samples hit each neighbour
    with frequency 1/4 (within 5 sigma); different seeds give different tables."""
    g = gs.from_rows([[3, 5, 7, 9], [2], []])
    t = oracle.sample_neighbors(g.rowptr, g.colidx, 4000, seed=123)
    cnt = np.array([(t[0] == u).sum() for u in (3, 5, 7, 9)])
    assert cnt.sum() == 4000
    assert np.all(np.abs(cnt - 1000) < 5 * math.sqrt(4000 * 0.25 * 0.75))
    assert np.all(t[1] == 2) and np.all(t[2] == -1)
    g2 = gs.random_small(200, avg_deg=8, seed=5)
    a = oracle.sample_neighbors(g2.rowptr, g2.colidx, 16, seed=1)
    b = oracle.sample_neighbors(g2.rowptr, g2.colidx, 16, seed=2)
    for v in range(g2.n):
        nb = set(g2.colidx[g2.rowptr[v]:g2.rowptr[v + 1]].tolist())
        assert set(a[v].tolist()) <= (nb if nb else {-1})
    assert (a != b).mean() > 0.5


# --------------------------------------------------------------------------- #
# NEXT-4 Table 2 edge functions + Softmax_aggr (R14)
# --------------------------------------------------------------------------- #
def _dense_softmax_aggr(A, E, Z):
    """Dense masked softmax (multiplicity weights A[v,u]) then the weighted sum."""
    out = np.zeros((A.shape[0], Z.shape[1]))
    for v in range(A.shape[0]):
        m = A[v] > 0
        if not m.any():
            continue
        ev = np.where(m, E[v], -np.inf)
        w = A[v] * np.exp(ev - ev[m].max())
        out[v] = (w / w.sum()) @ Z
    return out


def _dense_adj(g):
    A = np.zeros((g.n, g.n))
    for v in range(g.n):
        for u in g.colidx[g.rowptr[v]:g.rowptr[v + 1]]:
            A[v, u] += 1
    return A


@pytest.mark.parametrize("score", ["gat", "sym", "linear", "gaan", "gene"])
def test_attn_scores_vs_dense(score):
    """Every Table 2 score, evaluated per edge by the oracle, against a dense
    all-pairs formulation (N x N score matrix, adjacency-masked softmax)."""
    g = gs.random_small(40, avg_deg=5, seed=17, self_loops=True, multi=True)
    H, Fh = 3, 4
    F = H * Fh
    rng = np.random.default_rng(18)
    Z = rng.uniform(-2, 2, size=(g.n, F)).astype(np.float32)
    s = rng.uniform(-2, 2, size=(g.n, H)).astype(np.float32)
    t = rng.uniform(-2, 2, size=(g.n, H)).astype(np.float32)
    q = rng.uniform(-1, 1, size=(g.n, F)).astype(np.float32)
    k = rng.uniform(-1, 1, size=(g.n, F)).astype(np.float32)
    Wa = rng.uniform(-1, 1, size=(H, Fh)).astype(np.float32)
    A = _dense_adj(g)
    lk = lambda x: np.where(x > 0, x, 0.2 * x)  # noqa: E731
    Tv = None
    if score == "gat":
        Zs, Tv = np.concatenate([Z, s], 1), t
        E = [lk(s[None, :, h].astype(np.float64) + t[:, None, h]) for h in range(H)]
    elif score == "sym":
        Zs = np.concatenate([Z, s, t], 1)
        E = [lk(s[None, :, h].astype(np.float64) + t[:, None, h]) + lk(s[:, None, h].astype(np.float64) + t[None, :, h])
             for h in range(H)]
    elif score == "linear":
        Zs = np.concatenate([Z, s], 1)
        E = [np.tanh(np.broadcast_to(s[None, :, h].astype(np.float64), (g.n, g.n))) for h in range(H)]
    elif score == "gaan":
        Zs, Tv = np.concatenate([Z, q], 1), k
        E = [k[:, h * Fh:(h + 1) * Fh].astype(np.float64) @ q[:, h * Fh:(h + 1) * Fh].T.astype(np.float64)
             for h in range(H)]
    else:
        Zs, Tv = np.concatenate([Z, q], 1), k
        E = [np.tanh(q[None, :, h * Fh:(h + 1) * Fh].astype(np.float64) + k[:, None, h * Fh:(h + 1) * Fh]) @
             Wa[h].astype(np.float64) for h in range(H)]
    Y = oracle.attn_aggregate(g.rowptr, g.colidx, score, Zs, H, Fh, Tv=Tv, Wa=Wa)
    ref = np.concatenate([_dense_softmax_aggr(A, E[h], Z[:, h * Fh:(h + 1) * Fh].astype(np.float64))
                          for h in range(H)], 1)
    assert np.allclose(Y, ref, rtol=1e-6, atol=1e-6)
    Ym = oracle.attn_aggregate(g.rowptr, g.colidx, score, Zs, H, Fh, Tv=Tv, Wa=Wa, head_mean=True)
    assert np.allclose(Ym, ref.reshape(g.n, H, Fh).mean(1), rtol=1e-6, atol=1e-6)


def test_attn_special_cases():
    """Zero attention parameters give uniform weights (= mean aggregation,
    pinned above by the dense adjacency); the GAT score path equals the
    separately written GAT oracle (Listing 1 order)."""
    g = gs.random_small(80, avg_deg=6, seed=19)
    H, Fh = 2, 3
    F = H * Fh
    rng = np.random.default_rng(20)
    Z = rng.uniform(-1, 1, size=(g.n, F)).astype(np.float32)
    zeros = np.zeros((g.n, F), np.float32)
    mean = oracle.aggregate(g.rowptr, g.colidx, Z, "mean")
    for score, Zs, Tv, Wa in [("gaan", np.concatenate([Z, zeros], 1), rng.uniform(-1, 1, (g.n, F)), None),
                              ("gene", np.concatenate([Z, rng.uniform(-1, 1, (g.n, F))], 1),
                               rng.uniform(-1, 1, (g.n, F)), np.zeros((H, Fh))),
                              ("linear", np.concatenate([Z, np.zeros((g.n, H), np.float32)], 1), None, None)]:
        Y = oracle.attn_aggregate(g.rowptr, g.colidx, score, Zs, H, Fh, Tv=Tv, Wa=Wa)
        assert np.allclose(Y, mean, rtol=1e-6, atol=1e-7), score
    s = rng.uniform(-3, 3, size=(g.n, H)).astype(np.float32)
    t = rng.uniform(-3, 3, size=(g.n, H)).astype(np.float32)
    Zs = np.concatenate([Z, s], 1)
    a = oracle.attn_aggregate(g.rowptr, g.colidx, "gat", Zs, H, Fh, Tv=t)
    b = oracle.gat_aggregate(g.rowptr, g.colidx, Zs, t, H, Fh, 0.2)
    assert np.allclose(a, b, rtol=1e-6, atol=1e-7)
