"""Thin Python binding of libgnn.so (include/gnn.h) — argument marshalling only.

Every C entry point is exposed under its C name (``gnn_plan_create``,
``gnn_aggregate``, ...) taking raw pointers/ints exactly like the C-ABI.  On
top sit small torch-tensor conveniences (``Plan``, ``aggregate``,
``gat_aggregate``, ...) that only read ``data_ptr()``/``stride()`` and allocate
outputs/workspace with torch; every step of the path runs in the library's
sm_100a kernels.  There is NO CPU or Python fallback: if libgnn.so is missing
or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GNN_LIB_PATH") or os.path.join(_PKG, "libgnn.so")  # override: dev A/B builds only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_ppopp_huangzzys21_b200.build` "
                      "(or __graft_entry__.build()); there is no fallback path")
_lib = ctypes.CDLL(LIB_PATH)

GNN_OK = 0
STATUS = {0: "GNN_OK", 1: "GNN_ERR_INVALID_ARG", 2: "GNN_ERR_INVALID_GRAPH", 3: "GNN_ERR_WORKSPACE",
          4: "GNN_ERR_CUDA", 5: "GNN_ERR_NOMEM", 6: "GNN_ERR_UNSUPPORTED", 7: "GNN_ERR_INTERNAL"}
GNN_SUM, GNN_MEAN, GNN_MAX = 0, 1, 2
GNN_W_ONE, GNN_W_GCN, GNN_W_EDGE = 0, 1, 2
GNN_OP_AGGREGATE, GNN_OP_GAT_AGGREGATE, GNN_OP_EDGECONV, GNN_OP_GCN_LAYER, GNN_OP_GAT_LAYER, \
    GNN_OP_SAGE_LSTM_LAYER, GNN_OP_ATTN_AGGREGATE, GNN_OP_ATTN_AGGREGATE_MEAN = range(8)
SCORES = {"gat": 0, "sym": 1, "linear": 2, "gaan": 3, "gene": 4}
REDUCE = {"sum": GNN_SUM, "mean": GNN_MEAN, "max": GNN_MAX}
WEIGHT = {"one": GNN_W_ONE, "gcn": GNN_W_GCN, "edge": GNN_W_EDGE}


class GnnError(RuntimeError):
    def __init__(self, fn, status):
        self.status = status
        super().__init__(f"{fn} -> {STATUS.get(status, status)}: {gnn_last_error()}")


class gnn_plan_opts(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("reorder", ctypes.c_int32), ("group_size", ctypes.c_int32),
                ("tile_groups", ctypes.c_int32), ("cluster_cap", ctypes.c_int32), ("minhash_k", ctypes.c_int32),
                ("lsh_rows", ctypes.c_int32), ("pair_window", ctypes.c_int32), ("min_sim", ctypes.c_int32),
                ("deterministic", ctypes.c_int32), ("cluster_order", ctypes.c_int32), ("seed", ctypes.c_uint64)]


class gnn_plan_info(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int64) for k in ("n", "n_src", "nnz", "n_groups", "n_tiles", "n_split_rows",
                                                "n_empty_rows", "n_clusters", "n_pairs")] + \
               [(k, ctypes.c_int32) for k in ("group_size", "tile_groups", "max_degree", "reorder")] + \
               [(k, ctypes.c_double) for k in ("ms_validate", "ms_upload", "ms_degrees", "ms_minhash", "ms_lsh",
                                                 "ms_merge", "ms_ng")]


class gnn_tune_result(ctypes.Structure):
    _fields_ = [("group_size", ctypes.c_int32), ("vec", ctypes.c_int32), ("lanes", ctypes.c_int32),
                ("nv", ctypes.c_int32), ("ms", ctypes.c_float), ("ms_default", ctypes.c_float),
                ("rounds", ctypes.c_int32), ("mappings_tried", ctypes.c_int32)]


_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32
_SZ = ctypes.c_size_t
_F = ctypes.c_float

_SIGS = {
    "gnn_plan_opts_default": (None, [ctypes.POINTER(gnn_plan_opts)]),
    "gnn_plan_create": (ctypes.c_int, [_I64, _I64, _P, _P, ctypes.POINTER(gnn_plan_opts), ctypes.POINTER(_P)]),
    "gnn_plan_create_ex": (ctypes.c_int, [_I64, _I64, _I64, _P, _P, _P, ctypes.POINTER(gnn_plan_opts),
                                          ctypes.POINTER(_P)]),
    "gnn_plan_create_perm": (ctypes.c_int, [_I64, _I64, _I64, _P, _P, _P, _P, ctypes.POINTER(gnn_plan_opts),
                                            ctypes.POINTER(_P)]),
    "gnn_plan_save": (ctypes.c_int, [_P, ctypes.c_char_p, _I32]),
    "gnn_plan_load": (ctypes.c_int, [ctypes.c_char_p, ctypes.POINTER(_P)]),
    "gnn_plan_get_info": (ctypes.c_int, [_P, ctypes.POINTER(gnn_plan_info)]),
    "gnn_plan_export": (ctypes.c_int, [_P, _P, _P, _P]),
    "gnn_plan_export_las": (ctypes.c_int, [_P, _P, _P, _P]),
    "gnn_plan_normalizers": (ctypes.c_int, [_P, ctypes.POINTER(_P), ctypes.POINTER(_P)]),
    "gnn_plan_destroy": (ctypes.c_int, [_P]),
    "gnn_workspace_size": (_SZ, [_P, ctypes.c_int, _I32, _I32, _I32]),
    "gnn_aggregate": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int, _P, _P, _I64, _I32, _P, _I64, _I32, _P, _I64,
                                     _P, _SZ, _P]),
    "gnn_gat_aggregate": (ctypes.c_int, [_P, _P, _I64, _P, _I64, _I32, _I32, _F, _P, _I64, _P, _SZ, _P]),
    "gnn_aggregate_accumulate": (ctypes.c_int, [_P, ctypes.c_int, _P, _P, _I64, _I32, _P, _I64, _I32, _P, _SZ, _P]),
    "gnn_scale_rows": (ctypes.c_int, [_P, _I64, _I64, _I32, _P, _I32, _P]),
    "gnn_gat_layer": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _P, _P, _I32, _I32, _F, _P, _I64, _P, _SZ, _P]),
    "gnn_edgeconv_aggregate": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _I64, _P, _SZ, _P]),
    "gnn_edgeconv": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _P, _P, _I32, _P, _I64, _P, _SZ, _P]),
    "gnn_gemm": (ctypes.c_int, [_P, _I64, _P, _I64, _P, _I64, _I64, _I32, _I32, _P, _P, _I32, _P, _SZ, _P]),
    "gnn_gemm_workspace_size": (_SZ, [_I64, _I32, _I32]),
    "gnn_set_gemm_impl": (ctypes.c_int, [ctypes.c_int]),
    "gnn_set_agg_mapping": (ctypes.c_int, [_I32, _I32, _I32]),
    "gnn_set_agg_trace": (None, [_P]),
    "gnn_gcn_layer": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _I64, _I32, _I32, _I32, _P, _I64, _P, _SZ, _P]),
    "gnn_gcn_aggregate_prescaled": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _I64, _I32, _P, _SZ, _P]),
    "gnn_gat_fold_weights": (ctypes.c_int, [_P, _P, _P, _I32, _I32, _I32, _P, _I64, _P]),
    "gnn_gat_transform": (ctypes.c_int, [_P, _I64, _I64, _I32, _P, _I64, _P, _P, _I32, _I32, _P, _I64, _P, _SZ, _P]),
    "gnn_gat_transform_workspace_size": (_SZ, [_I64, _I32, _I32, _I32]),
    "gnn_partition_rows": (ctypes.c_int, [_I64, _P, _I32, _P]),
    "gnn_local_csr": (ctypes.c_int, [_I64, _P, _P, _P, _I32, _I32, ctypes.POINTER(_I64), ctypes.POINTER(_I64),
                                     _P, _P, _P]),
    "gnn_local_csr_block": (ctypes.c_int, [_I64, _P, _P, _P, _I32, _I32, _I32, ctypes.POINTER(_I64), _P, _P]),
    "gnn_las_host": (ctypes.c_int, [_I64, _P, _P, _I32, _I32, _I32, _I32, _I32, _I32, _P, _P, ctypes.POINTER(_I64),
                                    ctypes.POINTER(_I64)]),
    "gnn_groups_host": (ctypes.c_int, [_I64, _P, _P, _I32, ctypes.POINTER(_I64), _P, _P]),
    "gnn_launch_count": (ctypes.c_uint64, []),
    "gnn_plan_set_group_size": (ctypes.c_int, [_P, _I32]),
    "gnn_attn_aggregate": (ctypes.c_int, [_P, ctypes.c_int, _P, _I64, _P, _I64, _P, _I32, _I32, _F, _I32, _P, _I64,
                                          _P, _SZ, _P]),
    "gnn_sample_neighbors": (ctypes.c_int, [_P, _I32, ctypes.c_uint64, _P, _P]),
    "gnn_sage_lstm_aggregate": (ctypes.c_int, [_P, _P, _I32, _P, _I64, _I32, _P, _P, _I32, _P, _I64, _P]),
    "gnn_sage_lstm_layer": (ctypes.c_int, [_P, _P, _I64, _I32, _P, _P, _P, _P, _P, _P, _P, _I32, _I32, _I32,
                                           ctypes.c_uint64, _P, _I64, _P, _SZ, _P]),
    "gnn_tune_aggregate": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int, _P, _P, _I64, _I32, _P, _I64, _I32,
                                          ctypes.POINTER(gnn_tune_result), _P]),
    "gnn_gemm_mirrored": (ctypes.c_int, [_P, _I64, _P, _I64, _P, _I64, _I64, _I32, _I32, _P, _P, _I32, _P, _I32, _P,
                                         _SZ, _P]),
    "gnn_gat_transform_mirrored": (ctypes.c_int, [_P, _I64, _I64, _I32, _P, _I64, _P, _P, _I32, _I32, _P, _I64, _P,
                                                  _I32, _P, _SZ, _P]),
    "gnn_ipc_alloc": (ctypes.c_int, [_SZ, ctypes.POINTER(_P), _P]),
    "gnn_ipc_free": (ctypes.c_int, [_P]),
    "gnn_ipc_open": (ctypes.c_int, [_P, ctypes.POINTER(_P)]),
    "gnn_ipc_close": (ctypes.c_int, [_P]),
    "gnn_last_error": (ctypes.c_char_p, []),
    "gnn_version": (ctypes.c_char_p, []),
}

EXPORTED = sorted(_SIGS)

for _name, (_res, _args) in _SIGS.items():
    if os.environ.get("GNN_LIB_PATH") and not hasattr(_lib, _name):
        continue  # dev A/B against an older build: symbols it predates stay unbound
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args
    globals()[_name] = _f


def gnn_last_error() -> str:  # noqa: F811 — decode the C string
    return _lib.gnn_last_error().decode()


def gnn_version() -> str:  # noqa: F811
    return _lib.gnn_version().decode()


def _call(name, *args):
    st = getattr(_lib, name)(*args)
    if st != GNN_OK:
        raise GnnError(name, st)


# --------------------------------------------------------------------------- #
# torch conveniences (marshalling only)
# --------------------------------------------------------------------------- #
def _torch():
    import torch
    return torch


def _np_ptr(a):
    return None if a is None else a.ctypes.data


def _tp(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _ld(t, width):
    assert t.dtype == _torch().float32, "fp32 tensors only"
    assert t.dim() == 2 and t.stride(1) == 1, "row-major 2-D tensors only"
    assert t.shape[1] >= width
    return t.stride(0)


def _stream(stream):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def default_opts(**kw) -> gnn_plan_opts:
    o = gnn_plan_opts()
    _lib.gnn_plan_opts_default(ctypes.byref(o))
    for k, v in kw.items():
        setattr(o, k, v)
    return o


class Plan:
    """Owns a gnn_plan_t built from a host CSR (numpy int64 rowptr, int32 colidx)."""

    def __init__(self, rowptr, colidx, n_src=None, src_degree=None, perm=None, **opts):
        """gnn_plan_create_ex, or gnn_plan_create_perm when a task order `perm`
        (e.g. a LAS schedule computed earlier) is given."""
        rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
        colidx = np.ascontiguousarray(colidx, dtype=np.int32)
        self.n = len(rowptr) - 1
        self.nnz = int(rowptr[-1])
        self.n_src = self.n if n_src is None else int(n_src)
        self.opts = default_opts(**opts)
        h = ctypes.c_void_p()
        sd = None if src_degree is None else np.ascontiguousarray(src_degree, dtype=np.int32)
        if perm is None:
            _call("gnn_plan_create_ex", self.n, self.n_src, self.nnz, _np_ptr(rowptr), _np_ptr(colidx), _np_ptr(sd),
                  ctypes.byref(self.opts), ctypes.byref(h))
        else:
            pm = np.ascontiguousarray(perm, dtype=np.int32)
            _call("gnn_plan_create_perm", self.n, self.n_src, self.nnz, _np_ptr(rowptr), _np_ptr(colidx),
                  _np_ptr(sd), _np_ptr(pm), ctypes.byref(self.opts), ctypes.byref(h))
        self.handle = h
        self._ws = {}

    @classmethod
    def load(cls, path):
        """gnn_plan_load: a plan saved by Plan.save (no LAS rerun)."""
        self = cls.__new__(cls)
        h = ctypes.c_void_p()
        _call("gnn_plan_load", os.fsencode(path), ctypes.byref(h))
        self.handle = h
        self._ws = {}
        i = self.info
        self.n, self.n_src, self.nnz = i["n"], i["n_src"], i["nnz"]
        self.opts = default_opts(reorder=i["reorder"])
        return self

    def save(self, path, with_las=False):
        """gnn_plan_save: CSR, degrees, task order (+ LAS intermediates)."""
        _call("gnn_plan_save", self.handle, os.fsencode(path), int(with_las))

    @property
    def info(self) -> dict:
        i = gnn_plan_info()
        _call("gnn_plan_get_info", self.handle, ctypes.byref(i))
        return {k: getattr(i, k) for k, _ in gnn_plan_info._fields_}

    def export(self):
        """(perm, grp_row, grp_beg); CTA tile t = groups [t*T, (t+1)*T)."""
        G = self.info["n_groups"]
        perm = np.empty(self.n, np.int32)
        gr = np.empty(max(G, 1), np.int32)
        gb = np.empty(max(G, 1), np.int64)
        _call("gnn_plan_export", self.handle, _np_ptr(perm), _np_ptr(gr), _np_ptr(gb))
        return perm, gr[:G], gb[:G]

    def export_las(self):
        info = self.info
        K = self.opts.minhash_k
        sig = np.empty((self.n, K), np.uint64)
        pairs = np.empty((max(info["n_pairs"], 1), 2), np.int32)
        cl = np.empty(self.n, np.int32)
        _call("gnn_plan_export_las", self.handle, _np_ptr(sig), _np_ptr(pairs), _np_ptr(cl))
        return sig, pairs[:info["n_pairs"]], cl

    def normalizers(self):
        a, b = ctypes.c_void_p(), ctypes.c_void_p()
        _call("gnn_plan_normalizers", self.handle, ctypes.byref(a), ctypes.byref(b))
        return a.value, b.value

    def workspace(self, op, f_in=0, f_out=0, heads=0, device=None):
        nbytes = _lib.gnn_workspace_size(self.handle, op, f_in, f_out, heads)
        if nbytes == 0:
            return None, 0
        key = (op, f_in, f_out, heads)
        ws = self._ws.get(key)
        if ws is None:
            torch = _torch()
            ws = torch.empty(nbytes, dtype=torch.uint8, device=device or "cuda")
            self._ws[key] = ws
        return ws, nbytes

    def destroy(self):
        if getattr(self, "handle", None):
            _lib.gnn_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def aggregate(plan: Plan, X, reduce="sum", weight="one", edge_w=None, relu=False, add_row=None, out=None,
              stream=None):
    torch = _torch()
    F = X.shape[1]
    Y = out if out is not None else torch.empty((plan.n, F), dtype=torch.float32, device=X.device)
    ws, nb = plan.workspace(GNN_OP_AGGREGATE, 0, F, 0, X.device)
    _call("gnn_aggregate", plan.handle, REDUCE[reduce], WEIGHT[weight], _tp(edge_w), _tp(X), _ld(X, F), F, _tp(Y),
          _ld(Y, F), int(relu), _tp(add_row), 0 if add_row is None else _ld(add_row, F), _tp(ws), nb,
          _stream(stream))
    return Y


def aggregate_accumulate(plan: Plan, X, Y, accumulate=True, weight="one", edge_w=None, stream=None):
    """gnn_aggregate_accumulate: Y (+)= raw sums of this (source-block) plan."""
    F = X.shape[1]
    ws, nb = plan.workspace(GNN_OP_AGGREGATE, 0, F, 0, X.device)
    _call("gnn_aggregate_accumulate", plan.handle, WEIGHT[weight], _tp(edge_w), _tp(X), _ld(X, F), F, _tp(Y),
          _ld(Y, F), int(accumulate), _tp(ws), nb, _stream(stream))
    return Y


def scale_rows(Y, scale, relu=False, stream=None):
    """gnn_scale_rows: Y[v] = ReLU?(Y[v] * scale[v]) (scale: device tensor or pointer)."""
    sp = scale if isinstance(scale, int) else scale.data_ptr()
    _call("gnn_scale_rows", _tp(Y), _ld(Y, Y.shape[1]), Y.shape[0], Y.shape[1], ctypes.c_void_p(sp), int(relu),
          _stream(stream))
    return Y


def gat_aggregate(plan: Plan, Zs, t, H, Fh, neg_slope=0.2, out=None, stream=None):
    torch = _torch()
    F = H * Fh
    Y = out if out is not None else torch.empty((plan.n, F), dtype=torch.float32, device=Zs.device)
    ws, nb = plan.workspace(GNN_OP_GAT_AGGREGATE, 0, F, H, Zs.device)
    _call("gnn_gat_aggregate", plan.handle, _tp(Zs), _ld(Zs, F + H), _tp(t), _ld(t, H), H, Fh, float(neg_slope),
          _tp(Y), _ld(Y, F), _tp(ws), nb, _stream(stream))
    return Y


def gat_layer(plan: Plan, X, W, a_src, a_dst, H, Fh, neg_slope=0.2, out=None, stream=None):
    torch = _torch()
    F = H * Fh
    f_in = X.shape[1]
    Y = out if out is not None else torch.empty((plan.n, F), dtype=torch.float32, device=X.device)
    ws, nb = plan.workspace(GNN_OP_GAT_LAYER, f_in, F, H, X.device)
    _call("gnn_gat_layer", plan.handle, _tp(X), _ld(X, f_in), f_in, _tp(W.contiguous()), _tp(a_src.contiguous()),
          _tp(a_dst.contiguous()), H, Fh, float(neg_slope), _tp(Y), _ld(Y, F), _tp(ws), nb, _stream(stream))
    return Y


def gat_transform(X, W, a_src, a_dst, H, Fh, out=None, stream=None):
    """gnn_gat_transform: [Z | s | t] = X W with the GAT scores (reading R5)."""
    torch = _torch()
    m, f_in = X.shape
    ldz = (H * Fh + 2 * H + 7) // 8 * 8
    Z = out if out is not None else torch.empty((m, ldz), dtype=torch.float32, device=X.device)
    nb = _lib.gnn_gat_transform_workspace_size(m, f_in, H, Fh)
    ws = torch.empty(max(nb, 256), dtype=torch.uint8, device=X.device)
    _call("gnn_gat_transform", _tp(X), _ld(X, f_in), m, f_in, _tp(W.contiguous()), H * Fh, _tp(a_src.contiguous()),
          _tp(a_dst.contiguous()), H, Fh, _tp(Z), Z.stride(0), _tp(ws), nb, _stream(stream))
    return Z


def edgeconv_aggregate(plan: Plan, PQ, f_out, out=None, stream=None):
    torch = _torch()
    Y = out if out is not None else torch.empty((plan.n, f_out), dtype=torch.float32, device=PQ.device)
    ws, nb = plan.workspace(GNN_OP_AGGREGATE, 0, f_out, 0, PQ.device)
    _call("gnn_edgeconv_aggregate", plan.handle, _tp(PQ), _ld(PQ, 2 * f_out), f_out, _tp(Y), _ld(Y, f_out),
          _tp(ws), nb, _stream(stream))
    return Y


def edgeconv(plan: Plan, X, theta, phi, bias=None, out=None, stream=None):
    torch = _torch()
    f_out, f_in = theta.shape
    Y = out if out is not None else torch.empty((plan.n, f_out), dtype=torch.float32, device=X.device)
    ws, nb = plan.workspace(GNN_OP_EDGECONV, f_in, f_out, 0, X.device)
    _call("gnn_edgeconv", plan.handle, _tp(X), _ld(X, f_in), f_in, _tp(theta.contiguous()), _tp(phi.contiguous()),
          _tp(bias), f_out, _tp(Y), _ld(Y, f_out), _tp(ws), nb, _stream(stream))
    return Y


_GEMM_WS = {}


def gemm_workspace(m, k, n, device):
    """Workspace for the tcgen05 path (the split, swizzled W image); cached per device/size."""
    nbytes = _lib.gnn_gemm_workspace_size(m, k, n)
    if nbytes == 0:
        return None, 0
    torch = _torch()
    key = (str(device), nbytes)
    ws = _GEMM_WS.get(key)
    if ws is None:
        ws = torch.empty(nbytes, dtype=torch.uint8, device=device)
        _GEMM_WS[key] = ws
    return ws, nbytes


def gemm(X, W, row_scale=None, col_bias=None, relu=False, out=None, stream=None, simt=False):
    torch = _torch()
    m, k = X.shape
    n = W.shape[1]
    H = out if out is not None else torch.empty((m, n), dtype=torch.float32, device=X.device)
    ws, nb = (None, 0) if simt else gemm_workspace(m, k, n, X.device)
    _call("gnn_gemm", _tp(X), _ld(X, k), _tp(W), _ld(W, n), _tp(H), _ld(H, n), m, k, n, _tp(row_scale),
          _tp(col_bias), int(relu), _tp(ws), nb, _stream(stream))
    return H


def _ptr_array(ptrs):
    arr = (ctypes.c_void_p * max(1, len(ptrs)))(*[int(p) for p in ptrs])
    return arr, len(ptrs)


def gemm_mirrored(X, W, mirrors, row_scale=None, col_bias=None, relu=False, out=None, stream=None):
    """gnn_gemm_mirrored: H = X W written to `out` and to every mirror (device
    pointers laid out like `out`: the same rows of peer replicas; NEXT-2)."""
    torch = _torch()
    m, k = X.shape
    n = W.shape[1]
    H = out if out is not None else torch.empty((m, n), dtype=torch.float32, device=X.device)
    ws, nb = gemm_workspace(m, k, n, X.device)
    arr, cnt = _ptr_array(mirrors)
    _call("gnn_gemm_mirrored", _tp(X), _ld(X, k), _tp(W), _ld(W, n), _tp(H), _ld(H, n), m, k, n, _tp(row_scale),
          _tp(col_bias), int(relu), arr, cnt, _tp(ws), nb, _stream(stream))
    return H


class IpcBuffer:
    """A device buffer shareable across processes (gnn_ipc_alloc), viewed as a
    torch fp32 tensor of `shape` (zero-copy, __cuda_array_interface__)."""

    def __init__(self, shape, device):
        torch = _torch()
        self.shape = tuple(int(x) for x in shape)
        nbytes = int(np.prod(self.shape)) * 4
        self.handle = ctypes.create_string_buffer(64)
        p = ctypes.c_void_p()
        with torch.cuda.device(device):
            _call("gnn_ipc_alloc", nbytes, ctypes.byref(p), self.handle)
        self.ptr = p.value
        self.__cuda_array_interface__ = {"shape": self.shape, "typestr": "<f4", "data": (self.ptr, False),
                                         "version": 3, "strides": None}
        self.tensor = torch.as_tensor(self, device=device)

    def handle_bytes(self) -> bytes:
        return self.handle.raw

    def free(self):
        if self.ptr:
            self.tensor = None
            _call("gnn_ipc_free", ctypes.c_void_p(self.ptr))
            self.ptr = None


def ipc_open(handle: bytes) -> int:
    """Map a peer process's gnn_ipc_alloc buffer; returns the device pointer."""
    p = ctypes.c_void_p()
    hb = ctypes.create_string_buffer(handle, 64)
    _call("gnn_ipc_open", hb, ctypes.byref(p))
    return p.value


def ipc_close(ptr: int) -> None:
    _call("gnn_ipc_close", ctypes.c_void_p(ptr))


def set_gemm_impl(impl: int) -> int:
    return _lib.gnn_set_gemm_impl(impl)


def set_agg_mapping(vec: int = 0, lanes: int = 0, nv: int = 0) -> None:
    """a4 mapping override (gnn_set_agg_mapping); all zero = automatic rule."""
    _call("gnn_set_agg_mapping", vec, lanes, nv)


def gcn_layer(plan: Plan, X, W, relu=True, order=0, out=None, stream=None):
    torch = _torch()
    f_in = X.shape[1]
    f_out = W.shape[1]
    Y = out if out is not None else torch.empty((plan.n, f_out), dtype=torch.float32, device=X.device)
    ws, nb = plan.workspace(GNN_OP_GCN_LAYER, f_in, f_out, 0, X.device)
    _call("gnn_gcn_layer", plan.handle, _tp(X), _ld(X, f_in), f_in, _tp(W), _ld(W, f_out), f_out, int(relu),
          int(order), _tp(Y), _ld(Y, f_out), _tp(ws), nb, _stream(stream))
    return Y


def partition_rows(rowptr, nparts):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    b = np.empty(nparts + 1, np.int64)
    _call("gnn_partition_rows", len(rowptr) - 1, _np_ptr(rowptr), nparts, _np_ptr(b))
    return b


def local_csr(rowptr, colidx, bounds, rank):
    """Rank-local CSR in the padded all-gather layout (host only)."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    bounds = np.ascontiguousarray(bounds, dtype=np.int64)
    n = len(rowptr) - 1
    P = len(bounds) - 1
    rmax, lnnz = ctypes.c_int64(), ctypes.c_int64()
    _call("gnn_local_csr", n, _np_ptr(rowptr), _np_ptr(colidx), _np_ptr(bounds), P, rank, ctypes.byref(rmax),
          ctypes.byref(lnnz), None, None, None)
    rows = int(bounds[rank + 1] - bounds[rank])
    lrp = np.empty(rows + 1, np.int64)
    lci = np.empty(max(lnnz.value, 1), np.int32)
    sdeg = np.empty(max(P * rmax.value, 1), np.int32)
    _call("gnn_local_csr", n, _np_ptr(rowptr), _np_ptr(colidx), _np_ptr(bounds), P, rank, ctypes.byref(rmax),
          ctypes.byref(lnnz), _np_ptr(lrp), _np_ptr(lci), _np_ptr(sdeg))
    return lrp, lci[:lnnz.value], sdeg[:P * rmax.value], rmax.value


def local_csr_block(rowptr, colidx, bounds, rank, q):
    """gnn_local_csr_block: rank's rows restricted to sources of block q, sources relative to the block."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    b = np.ascontiguousarray(bounds, dtype=np.int64)
    n, P = len(rowptr) - 1, len(b) - 1
    cnt = ctypes.c_int64()
    _call("gnn_local_csr_block", n, _np_ptr(rowptr), _np_ptr(colidx), _np_ptr(b), P, rank, q, ctypes.byref(cnt),
          None, None)
    rows = int(b[rank + 1] - b[rank])
    brp = np.empty(rows + 1, np.int64)
    bci = np.empty(max(cnt.value, 1), np.int32)
    _call("gnn_local_csr_block", n, _np_ptr(rowptr), _np_ptr(colidx), _np_ptr(b), P, rank, q, ctypes.byref(cnt),
          _np_ptr(brp), _np_ptr(bci))
    return brp, bci[:cnt.value]


def las_host(rowptr, sig, r=2, W=8, cap=32, min_sim=-1, cluster_order=1):
    """a2 steps 2-5 on the host from given MinHash signatures (no GPU)."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    sig = np.ascontiguousarray(sig, dtype=np.uint64)
    n, K = sig.shape
    perm = np.empty(n, np.int32)
    cl = np.empty(n, np.int32)
    npairs, nc = ctypes.c_int64(), ctypes.c_int64()
    _call("gnn_las_host", n, _np_ptr(rowptr), _np_ptr(sig), K, r, W, cap, min_sim, cluster_order, _np_ptr(perm),
          _np_ptr(cl),
          ctypes.byref(npairs), ctypes.byref(nc))
    return perm, cl, npairs.value, nc.value


def groups_host(rowptr, ng, perm=None):
    """a3 neighbor groups in task order on the host (no GPU): (grp_row, grp_beg)."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    n = len(rowptr) - 1
    p = None if perm is None else np.ascontiguousarray(perm, dtype=np.int32)
    G = ctypes.c_int64()
    _call("gnn_groups_host", n, _np_ptr(rowptr), _np_ptr(p), ng, ctypes.byref(G), None, None)
    gr = np.empty(max(G.value, 1), np.int32)
    gb = np.empty(max(G.value, 1), np.int64)
    _call("gnn_groups_host", n, _np_ptr(rowptr), _np_ptr(p), ng, ctypes.byref(G), _np_ptr(gr), _np_ptr(gb))
    return gr[:G.value], gb[:G.value]


def set_group_size(plan: Plan, group_size: int) -> None:
    """gnn_plan_set_group_size: rebuild the plan's NG schedule for another bound."""
    _call("gnn_plan_set_group_size", plan.handle, int(group_size))
    plan._ws = {}


def tune_aggregate(plan: Plan, X, reduce="sum", weight="one", edge_w=None, out=None, max_rounds=20,
                   stream=None) -> dict:
    """gnn_tune_aggregate: the online tuner (mapping templates, then NG bound)."""
    torch = _torch()
    F = X.shape[1]
    Y = out if out is not None else torch.empty((plan.n, F), dtype=torch.float32, device=X.device)
    r = gnn_tune_result()
    _call("gnn_tune_aggregate", plan.handle, REDUCE[reduce], WEIGHT[weight], _tp(edge_w), _tp(X), _ld(X, F), F,
          _tp(Y), _ld(Y, F), int(max_rounds), ctypes.byref(r), _stream(stream))
    plan._ws = {}
    return {k: getattr(r, k) for k, _ in gnn_tune_result._fields_}


def attn_aggregate(plan: Plan, score, Zs, H, Fh, Tv=None, Wa=None, neg_slope=0.2, head_mean=False, out=None,
                   stream=None):
    """gnn_attn_aggregate: a Table 2 score + softmax aggregation, fused (reading R14)."""
    torch = _torch()
    F = H * Fh
    width = Fh if head_mean else F
    Y = out if out is not None else torch.empty((plan.n, width), dtype=torch.float32, device=Zs.device)
    op = GNN_OP_ATTN_AGGREGATE_MEAN if head_mean else GNN_OP_ATTN_AGGREGATE
    ws, nb = plan.workspace(op, 0, F, H, Zs.device)
    _call("gnn_attn_aggregate", plan.handle, SCORES[score], _tp(Zs), Zs.stride(0), _tp(Tv),
          0 if Tv is None else Tv.stride(0), _tp(Wa), H, Fh, neg_slope, int(head_mean), _tp(Y), _ld(Y, width),
          _tp(ws), nb, _stream(stream))
    return Y


def sample_neighbors(plan: Plan, T=16, seed=0, out=None, stream=None):
    """gnn_sample_neighbors -> [n, T] int32 device table (reading R13)."""
    torch = _torch()
    tab = out if out is not None else torch.empty((plan.n, T), dtype=torch.int32, device="cuda")
    _call("gnn_sample_neighbors", plan.handle, int(T), ctypes.c_uint64(seed), _tp(tab), _stream(stream))
    return tab


def sage_lstm_aggregate(plan: Plan, table, GS, R, W_neigh, out=None, stream=None):
    """gnn_sage_lstm_aggregate: fused LSTM cells over pre-transformed rows GS + SAGE combine."""
    torch = _torch()
    T = table.shape[1]
    F_out = W_neigh.shape[0]
    F = R.shape[1]
    Y = out if out is not None else torch.empty((plan.n, F_out), dtype=torch.float32, device=GS.device)
    _call("gnn_sage_lstm_aggregate", plan.handle, _tp(table), T, _tp(GS), GS.stride(0), F, _tp(R), _tp(W_neigh),
          F_out, _tp(Y), _ld(Y, F_out), _stream(stream))
    return Y


def sage_lstm_layer(plan: Plan, X, W_ih, W_hh, b_ih, b_hh, W_self, W_neigh, bias=None, T=16, seed=0, out=None,
                    stream=None):
    """gnn_sage_lstm_layer: y = W_self x_v + W_neigh LSTM(sampled neighbours) + b."""
    torch = _torch()
    f_in = X.shape[1]
    F = W_hh.shape[1]
    F_out = W_self.shape[0]
    Y = out if out is not None else torch.empty((plan.n, F_out), dtype=torch.float32, device=X.device)
    ws, nb = plan.workspace(GNN_OP_SAGE_LSTM_LAYER, f_in, F_out, T, X.device)
    _call("gnn_sage_lstm_layer", plan.handle, _tp(X), _ld(X, f_in), f_in, _tp(W_ih), _tp(W_hh), _tp(b_ih), _tp(b_hh),
          _tp(W_self), _tp(W_neigh), _tp(bias), F, F_out, int(T), ctypes.c_uint64(seed), _tp(Y), _ld(Y, F_out),
          _tp(ws), nb, _stream(stream))
    return Y


def launch_count() -> int:
    return int(_lib.gnn_launch_count())
