"""Seeded synthetic inputs shared by the oracle tests, GPU parity tests and bench.py.

This module holds none of the method's arithmetic: it draws graphs and
features only (DESIGN.md §3 "input recipe").  The power-law generator is plain
C (``synth.c``) so that the full-size Reddit/products shapes generate in
seconds on the bench host; kNN point clouds are numpy.

Configs follow BASELINE.json ``configs`` (C1..C5) and SURVEY.md §8(d); the
graph statistics are PAPER.md Table 3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_SO = os.path.join(_HERE, "libsynth.so")
_lib = None


def build() -> str:
    """Compile synth.c -> libsynth.so (gcc -O2, no fast-math)."""
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.synth_powerlaw.restype = ctypes.c_int
        lib.synth_powerlaw.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                       ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_uint64,
                                       ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.synth_powerlaw_ex.restype = ctypes.c_int
        lib.synth_powerlaw_ex.argtypes = lib.synth_powerlaw.argtypes + [ctypes.c_void_p]
        lib.synth_powerlaw_sym.restype = ctypes.c_int
        lib.synth_powerlaw_sym.argtypes = lib.synth_powerlaw_ex.argtypes
        lib.synth_uniform_f32.restype = None
        lib.synth_uniform_f32.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_float,
                                          ctypes.c_float, ctypes.c_uint64, ctypes.c_void_p]
        _lib = lib
    return _lib


@dataclass
class Graph:
    """CSR by destination: row v lists the sources u of edges u->v."""
    n: int
    rowptr: np.ndarray  # int64[n+1]
    colidx: np.ndarray  # int32[nnz]
    stats: dict

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])


def powerlaw(n, nnz, mean, var, cap, comm=32, rho=0.8, seed=1, with_relabel=False, sym=False) -> Graph:
    """GEN-PL graph (directed; sym=True: the undirected recipe of SURVEY §8(d),
    nnz/2 pairs symmetrised, min degree 1).  with_relabel=True also returns
    (in stats["relabel"]) the relabel permutation (new id of pre-relabel node v)."""
    lib = _load()
    rowptr = np.empty(n + 1, dtype=np.int64)
    colidx = np.empty(max(nnz, 1), dtype=np.int32)
    st = np.zeros(4, dtype=np.int64)
    rel = np.empty(n, dtype=np.int64) if with_relabel else None
    fn = lib.synth_powerlaw_sym if sym else lib.synth_powerlaw_ex
    rc = fn(n, nnz, float(mean), float(var), cap, comm, float(rho), seed, rowptr.ctypes.data, colidx.ctypes.data,
            st.ctypes.data, None if rel is None else rel.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"synth_powerlaw failed rc={rc}")
    stats = {"max": int(st[0]), "mean": st[1] / 1e6, "var": st[2] / 1e3, "zero_rows": int(st[3])}
    if rel is not None:
        stats["relabel"] = rel
    return Graph(n, rowptr, colidx[:nnz], stats)


def uniform(rows, cols, ld=None, lo=-1.0, hi=1.0, seed=1) -> np.ndarray:
    """fp32 [rows, ld] with U(lo, hi) in the first `cols` columns and zero padding."""
    ld = cols if ld is None else ld
    out = np.empty((rows, ld), dtype=np.float32)
    _load().synth_uniform_f32(rows, cols, ld, lo, hi, seed, out.ctypes.data)
    return out


def integer_features(rows, cols, lo=-8, hi=8, seed=1) -> np.ndarray:
    """Integer-valued fp32 features: every partial sum is exact."""
    rng = np.random.default_rng(seed)
    return rng.integers(lo, hi + 1, size=(rows, cols)).astype(np.float32)


def knn_clouds(batch=32, points=1024, k=20, seed=1) -> Graph:
    """GEN-KNN: `batch` clouds of U[0,1)^3 points, exact fp64 kNN (no self,
    distance ties -> smaller id), block-diagonal ids.  Row v lists its k nearest
    neighbours as sources (EdgeConv's N(v))."""
    n = batch * points
    rowptr = np.arange(n + 1, dtype=np.int64) * k
    colidx = np.empty(n * k, dtype=np.int32)
    idx = np.arange(points)
    for b in range(batch):
        rng = np.random.default_rng([seed, b])
        p = rng.random((points, 3))
        d = ((p[:, None, :] - p[None, :, :]) ** 2).sum(-1)
        d[idx, idx] = np.inf
        order = np.lexsort((np.broadcast_to(idx, d.shape), d), axis=1)[:, :k]
        order.sort(axis=1)
        colidx[b * points * k:(b + 1) * points * k] = (order + b * points).reshape(-1)
    return Graph(n, rowptr, colidx, {"max": k, "mean": float(k), "var": 0.0, "zero_rows": 0})


def random_small(n, avg_deg=4.0, seed=0, allow_empty=True, self_loops=False, multi=False) -> Graph:
    """Tiny uniform random CSR graphs for property tests (numpy)."""
    rng = np.random.default_rng(seed)
    deg = rng.poisson(avg_deg, size=n)
    if not allow_empty:
        deg = np.maximum(deg, 1)
    rows = []
    for v in range(n):
        d = int(deg[v])
        if multi:
            c = rng.integers(0, n, size=d)
        else:
            pool = np.arange(n) if self_loops else np.delete(np.arange(n), v)
            d = min(d, len(pool))
            c = rng.choice(pool, size=d, replace=False)
        rows.append(np.sort(c).astype(np.int32))
    rowptr = np.zeros(n + 1, dtype=np.int64)
    rowptr[1:] = np.cumsum([len(r) for r in rows])
    colidx = np.concatenate(rows) if rows and rowptr[-1] > 0 else np.zeros(0, dtype=np.int32)
    return Graph(n, rowptr, colidx.astype(np.int32), {})


def from_rows(rows) -> Graph:
    n = len(rows)
    rowptr = np.zeros(n + 1, dtype=np.int64)
    rowptr[1:] = np.cumsum([len(r) for r in rows])
    colidx = np.array([u for r in rows for u in r], dtype=np.int32)
    return Graph(n, rowptr, colidx, {})


# BASELINE.json configs; seeds = 20210227 + 10*cfg + {0 graph, 1 X, 2 W, 3 a/theta/phi/b}
CONFIGS = {
    # C1: Cora-shaped, 2,708 nodes, 10,556 CSR entries, F=16
    "C1": dict(n=2708, nnz=10556, mean=3.9, var=27.0, cap=168, comm=32, F=16, sym=True),
    # C2: ogbn-arxiv-shaped (Table 3): 169,343 nodes, 1,166,243 edges, max 13,155, var 4.6K
    "C2": dict(n=169343, nnz=1166243, mean=6.89, var=4600.0, cap=13155, comm=32, F_in=128, H=8, Fh=8),
    # C3: Reddit-shaped: 232,965 nodes, 114.6M entries, max 21,657, var 640K
    "C3": dict(n=232965, nnz=114615892, mean=492.0, var=640000.0, cap=21657, comm=1024, F_in=602, F=256, sym=True),
    # C4: kNN point clouds 32 x 1024, k=20, F=64
    "C4": dict(batch=32, points=1024, k=20, F=64),
    # C5: ogbn-products-shaped: 2,449,029 nodes, 123,718,280 entries, max 17,481, var 9.1K
    "C5": dict(n=2449029, nnz=123718280, mean=50.5, var=9100.0, cap=17481, comm=256, F_in=100, F=256, H=8, Fh=32,
               sym=True),
}


def seed_of(cfg: str, what: int) -> int:
    return 20210227 + 10 * int(cfg[1]) + what


def config_graph(cfg: str, rho: float = 0.8, scale: float = 1.0, with_relabel: bool = False) -> Graph:
    c = CONFIGS[cfg]
    if cfg == "C4":
        return knn_clouds(c["batch"], c["points"], c["k"], seed=seed_of(cfg, 0))
    n = max(64, int(c["n"] * scale))
    nnz = max(n, int(c["nnz"] * scale))
    cap = min(c["cap"], n - 1)
    # Cora, Reddit and products are undirected: SURVEY §8(d) GEN-PL draws
    # nnz/2 pairs and symmetrises them (min degree 1); arxiv (C2) is directed
    sym = c.get("sym", False)
    if sym:
        nnz -= nnz % 2
    return powerlaw(n, nnz, c["mean"], c["var"], cap, c["comm"], rho, seed_of(cfg, 0) + int(rho * 100),
                    with_relabel=with_relabel, sym=sym)
