"""oracle — TEST INFRASTRUCTURE ONLY.

Thin ctypes wrapper over ``oracle.c``: a plain, slow, single-threaded fp64 CPU
implementation of the paper's definitions (Huang et al., PPoPP'21; PAPER.md
lines cited in oracle.c).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with ``paper_conf_ppopp_huangzzys21_b200`` and
never imports it.

Parity status per function (DESIGN.md §4 lists the pins):
  aggregate, aggregate_ng_f32, gemm, gcn_layer, gat_aggregate, gat_layer,
  edgeconv, minhash, lsh_pairs, las_merge, neighbor_groups,
  partition_rows: pinned by tests/test_oracle_pins.py; the LSH window and
  within-bucket order, pair completeness/dedup, the merge's re-enqueue branch
  and the hash family's known answers by tests/test_oracle_pins_las.py
  (hand traces, tests/golden/fmix64_minhash.txt, the LSH S-curve).
  LAS *quality* (how much L2 reuse the schedule buys) is "parity unpinned":
  the paper's real graphs are unavailable.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

SUM, MEAN, MAX = 0, 1, 2
W_ONE, W_GCN, W_EDGE = 0, 1, 2
_RED = {"sum": SUM, "mean": MEAN, "max": MAX}
_WGT = {"one": W_ONE, "gcn": W_GCN, "edge": W_EDGE}

_p = ctypes.c_void_p
_i64 = ctypes.c_int64
_i32 = ctypes.c_int32


def build() -> str:
    """gcc -O2, no -ffast-math, no OpenMP (SURVEY §8(c) General)."""
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fno-fast-math", "-ffp-contract=off",
                               "-shared", "-fPIC", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        sig = {
            "orc_degrees": (None, [_i64, _p, _p, _p, _p]),
            "orc_aggregate": (ctypes.c_int, [_i64, _p, _p, ctypes.c_int, ctypes.c_int, _p, _p, _i64, _i32,
                                             ctypes.c_int, _p, _i64, _p, _i64, _p]),
            "orc_aggregate_ng_f32": (ctypes.c_int, [_i64, _p, _p, ctypes.c_int, ctypes.c_int, _p, _p, _i64,
                                                    _i32, ctypes.c_int, _i32, _p, _i64]),
            "orc_gemm": (ctypes.c_int, [_i64, _i32, _i32, _p, _i64, _p, _i64, _p, _p, _i64]),
            "orc_gcn_layer": (ctypes.c_int, [_i64, _p, _p, _p, _i64, _i32, _p, _i64, _i32, ctypes.c_int,
                                             _p, _i64, _p, _i64]),
            "orc_gat_aggregate": (ctypes.c_int, [_i64, _p, _p, _p, _i64, _p, _i64, _i32, _i32, ctypes.c_float,
                                                 _p, _i64, _p, _i64]),
            "orc_gat_layer": (ctypes.c_int, [_i64, _p, _p, _p, _i64, _i32, _p, _p, _p, _i32, _i32,
                                             ctypes.c_float, _p, _i64, _p, _i64]),
            "orc_edgeconv": (ctypes.c_int, [_i64, _p, _p, _p, _i64, _i32, _p, _p, _p, _i32, _p, _i64, _p, _i64]),
            "orc_splitmix64": (ctypes.c_uint64, [_p]),
            "orc_fmix64": (ctypes.c_uint64, [ctypes.c_uint64]),
            "orc_minhash": (None, [_i64, _p, _p, _i32, ctypes.c_uint64, _p]),
            "orc_sim": (_i32, [_p, _i32, _i64, _i64]),
            "orc_lsh_pairs": (_i64, [_i64, _p, _p, _i32, _i32, _i32, _p, _i64]),
            "orc_las_merge": (_i64, [_i64, _p, _i32, _p, _i64, _i32, _i32, _i32, _p, _p, _p]),
            "orc_neighbor_groups": (_i64, [_i64, _p, _p, _i32, _p, _p]),
            "orc_partition_rows": (None, [_i64, _p, _i32, _p]),
            "orc_forget_degrees": (None, []),
            "orc_attn_aggregate": (ctypes.c_int, [_i64, _p, _p, _i32, _p, _i64, _p, _i64, _p, _i32, _i32,
                                                  ctypes.c_float, _i32, _p, _i64, _p, _i64]),
            "orc_sample_neighbors": (None, [_i64, _p, _p, _i32, ctypes.c_uint64, _p]),
            "orc_sage_lstm": (ctypes.c_int, [_i64, _p, _i64, _i32, _p, _i32, _p, _p, _p, _p, _i32, _p, _p, _p,
                                             _i32, _p, _i64, _p, _i64]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


def _csr(rowptr, colidx):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    return rowptr, colidx


def _rows(rows):
    if rows is None:
        return None, 0
    r = np.ascontiguousarray(rows, dtype=np.int64)
    return r, len(r)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def degrees(rowptr, colidx):
    rowptr, colidx = _csr(rowptr, colidx)
    n = len(rowptr) - 1
    d_in = np.empty(n, np.int32)
    d_out = np.empty(n, np.int32)
    lib().orc_degrees(n, _ptr(rowptr), _ptr(colidx), _ptr(d_in), _ptr(d_out))
    return d_in, d_out


def aggregate(rowptr, colidx, X, reduce="sum", weight="one", edge_w=None, relu=False, rows=None,
              return_abs=False):
    """Table 1 reducer x Table 2 weight, fp64 accumulate (oracle.c orc_aggregate)."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _f32(X)
    n = len(rowptr) - 1
    F = X.shape[1]
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, F), np.float32)
    S = np.empty((m, F), np.float64) if return_abs else None
    ew = _f32(edge_w) if edge_w is not None else None
    lib().orc_forget_degrees()
    rc = lib().orc_aggregate(n, _ptr(rowptr), _ptr(colidx), _RED[reduce], _WGT[weight], _ptr(ew),
                             _ptr(X), X.shape[1], F, int(relu), _ptr(r), nr, _ptr(Y), F, _ptr(S))
    assert rc == 0
    return (Y, S) if return_abs else Y


def aggregate_ng_f32(rowptr, colidx, X, ng, reduce="sum", weight="one", edge_w=None, relu=False):
    """Replica of the deterministic fp32 order (R9) for the bit-exact pin."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _f32(X)
    n = len(rowptr) - 1
    F = X.shape[1]
    Y = np.empty((n, F), np.float32)
    ew = _f32(edge_w) if edge_w is not None else None
    lib().orc_forget_degrees()
    rc = lib().orc_aggregate_ng_f32(n, _ptr(rowptr), _ptr(colidx), _RED[reduce], _WGT[weight], _ptr(ew),
                                    _ptr(X), F, F, int(relu), int(ng), _ptr(Y), F)
    assert rc == 0
    return Y


def gemm(X, W, row_scale=None):
    X = _f32(X)
    W = _f32(W)
    m, k = X.shape
    n = W.shape[1]
    H = np.empty((m, n), np.float32)
    rs = _f32(row_scale) if row_scale is not None else None
    assert lib().orc_gemm(m, k, n, _ptr(X), k, _ptr(W), n, _ptr(rs), _ptr(H), n) == 0
    return H


def gcn_layer(rowptr, colidx, X, W, relu=True, rows=None):
    rowptr, colidx = _csr(rowptr, colidx)
    X = _f32(X)
    W = _f32(W)
    n = len(rowptr) - 1
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, W.shape[1]), np.float32)
    lib().orc_forget_degrees()
    assert lib().orc_gcn_layer(n, _ptr(rowptr), _ptr(colidx), _ptr(X), X.shape[1], X.shape[1], _ptr(W),
                               W.shape[1], W.shape[1], int(relu), _ptr(r), nr, _ptr(Y), W.shape[1]) == 0
    return Y


def gat_aggregate(rowptr, colidx, Zs, t, H, Fh, neg_slope=0.2, rows=None):
    rowptr, colidx = _csr(rowptr, colidx)
    Zs = _f32(Zs)
    t = _f32(t)
    n = len(rowptr) - 1
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, H * Fh), np.float32)
    assert lib().orc_gat_aggregate(n, _ptr(rowptr), _ptr(colidx), _ptr(Zs), Zs.shape[1], _ptr(t), t.shape[1],
                                   H, Fh, neg_slope, _ptr(r), nr, _ptr(Y), H * Fh) == 0
    return Y


def gat_layer(rowptr, colidx, X, W, a_src, a_dst, H, Fh, neg_slope=0.2, rows=None):
    rowptr, colidx = _csr(rowptr, colidx)
    X = _f32(X)
    W = _f32(W)
    n = len(rowptr) - 1
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, H * Fh), np.float32)
    assert lib().orc_gat_layer(n, _ptr(rowptr), _ptr(colidx), _ptr(X), X.shape[1], X.shape[1], _ptr(W),
                               _ptr(_f32(a_src)), _ptr(_f32(a_dst)), H, Fh, neg_slope, _ptr(r), nr,
                               _ptr(Y), H * Fh) == 0
    return Y


def edgeconv(rowptr, colidx, X, theta, phi, bias=None, rows=None):
    rowptr, colidx = _csr(rowptr, colidx)
    X = _f32(X)
    theta = _f32(theta)
    phi = _f32(phi)
    n = len(rowptr) - 1
    f_out, f_in = theta.shape
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, f_out), np.float32)
    b = _f32(bias) if bias is not None else None
    assert lib().orc_edgeconv(n, _ptr(rowptr), _ptr(colidx), _ptr(X), X.shape[1], f_in, _ptr(theta),
                              _ptr(phi), _ptr(b), f_out, _ptr(r), nr, _ptr(Y), f_out) == 0
    return Y


def splitmix64_stream(seed, count):
    st = ctypes.c_uint64(seed)
    return [lib().orc_splitmix64(ctypes.byref(st)) for _ in range(count)]


def fmix64(z):
    return lib().orc_fmix64(z)


def minhash(rowptr, colidx, K=32, seed=0):
    rowptr, colidx = _csr(rowptr, colidx)
    n = len(rowptr) - 1
    sig = np.empty((n, K), np.uint64)
    lib().orc_minhash(n, _ptr(rowptr), _ptr(colidx), K, seed, _ptr(sig))
    return sig


def lsh_pairs(rowptr, sig, r=2, W=8):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    sig = np.ascontiguousarray(sig, dtype=np.uint64)
    n, K = sig.shape
    cnt = lib().orc_lsh_pairs(n, _ptr(rowptr), _ptr(sig), K, r, W, None, 0)
    pairs = np.empty((max(cnt, 1), 2), np.int32)
    lib().orc_lsh_pairs(n, _ptr(rowptr), _ptr(sig), K, r, W, _ptr(pairs), cnt)
    return pairs[:cnt]


def las_merge(sig, pairs, cap=32, min_sim=2, cluster_order=1):
    sig = np.ascontiguousarray(sig, dtype=np.uint64)
    pairs = np.ascontiguousarray(pairs, dtype=np.int32)
    n, K = sig.shape
    perm = np.empty(n, np.int32)
    cl = np.empty(n, np.int32)
    st = np.zeros(3, np.int64)
    nc = lib().orc_las_merge(n, _ptr(sig), K, _ptr(pairs), len(pairs), cap, min_sim, cluster_order, _ptr(perm),
                             _ptr(cl), _ptr(st))
    return perm, cl, int(nc), {"merges": int(st[0]), "pops": int(st[1]), "repush": int(st[2])}


def las_schedule(rowptr, colidx, K=32, r=2, W=8, cap=32, min_sim=None, seed=0, cluster_order=1):
    """Full a2 pipeline: MinHash -> LSH -> merge -> schedule."""
    sig = minhash(rowptr, colidx, K, seed)
    pairs = lsh_pairs(rowptr, sig, r, W)
    perm, cl, nc, st = las_merge(sig, pairs, cap, r if min_sim is None else min_sim, cluster_order)
    return perm, {"sig": sig, "pairs": pairs, "cluster_of": cl, "n_clusters": nc, **st}


def neighbor_groups(rowptr, ng, perm=None):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    n = len(rowptr) - 1
    p = np.ascontiguousarray(perm, dtype=np.int32) if perm is not None else None
    G = lib().orc_neighbor_groups(n, _ptr(rowptr), _ptr(p), ng, None, None)
    grp_row = np.empty(max(G, 1), np.int32)
    grp_beg = np.empty(max(G, 1), np.int64)
    lib().orc_neighbor_groups(n, _ptr(rowptr), _ptr(p), ng, _ptr(grp_row), _ptr(grp_beg))
    return grp_row[:G], grp_beg[:G]


def partition_rows(rowptr, P):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    b = np.empty(P + 1, np.int64)
    lib().orc_partition_rows(len(rowptr) - 1, _ptr(rowptr), P, _ptr(b))
    return b


def sample_neighbors(rowptr, colidx, T=16, seed=0):
    """NEXT-3 sampling (reading R13): [n, T] int32 node ids, -1 for empty rows."""
    rowptr, colidx = _csr(rowptr, colidx)
    n = len(rowptr) - 1
    table = np.empty((n, T), np.int32)
    lib().orc_sample_neighbors(n, _ptr(rowptr), _ptr(colidx), T, seed, _ptr(table))
    return table


def sage_lstm(X, table, W_ih, W_hh, b_ih, b_hh, W_self, W_neigh, bias=None, rows=None):
    """NEXT-3 GraphSAGE-LSTM layer, fp64 (Fig 6 base implementation): returns [n or len(rows), F_out]."""
    X = _f32(X)
    table = np.ascontiguousarray(table, dtype=np.int32)
    n, T = table.shape
    F4, f_in = W_ih.shape
    F = F4 // 4
    F_out = W_self.shape[0]
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    Y = np.empty((m, F_out), np.float32)
    W_ih, W_hh, b_ih, b_hh, W_self, W_neigh = (_f32(a) for a in (W_ih, W_hh, b_ih, b_hh, W_self, W_neigh))
    b = _f32(bias) if bias is not None else None
    assert lib().orc_sage_lstm(n, _ptr(X), X.shape[1], f_in, _ptr(table), T, _ptr(W_ih), _ptr(W_hh), _ptr(b_ih),
                               _ptr(b_hh), F, _ptr(W_self), _ptr(W_neigh), _ptr(b), F_out, _ptr(r), nr, _ptr(Y),
                               F_out) == 0
    return Y


SCORES = {"gat": 0, "sym": 1, "linear": 2, "gaan": 3, "gene": 4}


def attn_aggregate(rowptr, colidx, score, Zs, H, Fh, Tv=None, Wa=None, neg_slope=0.2, head_mean=False, rows=None):
    """NEXT-4 Table 2 edge functions + softmax aggregation (reading R14), fp64."""
    rowptr, colidx = _csr(rowptr, colidx)
    Zs = _f32(Zs)
    n = len(rowptr) - 1
    Tv = _f32(Tv) if Tv is not None else None
    Wa = _f32(Wa) if Wa is not None else None
    r, nr = _rows(rows)
    m = nr if rows is not None else n
    width = Fh if head_mean else H * Fh
    Y = np.empty((m, width), np.float32)
    assert lib().orc_attn_aggregate(n, _ptr(rowptr), _ptr(colidx), SCORES[score], _ptr(Zs), Zs.shape[1], _ptr(Tv),
                                    0 if Tv is None else Tv.shape[1], _ptr(Wa), H, Fh, neg_slope, int(head_mean),
                                    _ptr(r), nr, _ptr(Y), width) == 0
    return Y
