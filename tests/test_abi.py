"""C-ABI boundary checks that need no GPU (`-m "not gpu"`):
libgnn.so loads, exports every symbol include/gnn.h declares, and its host-only
logic (validation, LAS merge, neighbor groups/tiles, row partition, local CSR)
is bit-identical to the oracle."""
import ctypes
import os
import re

import numpy as np
import pytest

import gnn_synth as gs
import oracle
from conftest import ROOT

P = pytest.importorskip("paper_conf_ppopp_huangzzys21_b200")


def header_functions():
    src = open(os.path.join(ROOT, "include", "gnn.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(gnn_[a-z0-9_]+)\s*\(", src)
    return sorted(set(names))


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(P.gnn.LIB_PATH)
    declared = header_functions()
    assert len(declared) >= 20
    missing = [n for n in declared if not hasattr(lib, n)]
    assert not missing, missing
    # the binding wraps every declared function under the same name
    assert set(declared) <= set(P.gnn.EXPORTED), set(declared) - set(P.gnn.EXPORTED)


def test_library_is_sm100a_and_not_fast_math():
    out = os.popen(f"cuobjdump --list-elf {P.gnn.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out, out


def test_version_and_defaults():
    assert "sm_100a" in P.gnn.gnn_version()
    o = P.gnn.default_opts()
    assert (o.reorder, o.group_size, o.tile_groups, o.cluster_cap, o.minhash_k, o.lsh_rows, o.pair_window,
            o.min_sim, o.deterministic, o.cluster_order) == (0, -1, 32, 32, 32, 2, 8, -1, 1, 1)


def _create(rowptr, colidx, n=None, **kw):
    rowptr = np.ascontiguousarray(rowptr, np.int64)
    colidx = np.ascontiguousarray(colidx, np.int32)
    n = len(rowptr) - 1 if n is None else n
    h = ctypes.c_void_p()
    o = P.gnn.default_opts(**kw)
    st = P.gnn.gnn_plan_create(n, len(colidx), rowptr.ctypes.data,
                               colidx.ctypes.data if len(colidx) else None, ctypes.byref(o), ctypes.byref(h))
    return st, h


@pytest.mark.parametrize("case", ["rowptr0", "rowptr_end", "decreasing", "col_neg", "col_big"])
def test_plan_create_rejects_invalid_csr(case):
    """Validation happens on the host before any device work (gnn.h, gnn_plan_create)."""
    rp = np.array([0, 2, 3, 5], np.int64)
    ci = np.array([1, 2, 0, 0, 1], np.int32)
    if case == "rowptr0":
        rp = rp + 1
    elif case == "rowptr_end":
        rp = np.array([0, 2, 3, 4], np.int64)
    elif case == "decreasing":
        rp = np.array([0, 3, 2, 5], np.int64)
    elif case == "col_neg":
        ci[1] = -1
    else:
        ci[1] = 3
    st, h = _create(rp, ci, n=3)
    assert st == 2, P.gnn.gnn_last_error()
    assert h.value is None
    assert P.gnn.gnn_last_error()


def test_invalid_args_return_status_not_crash():
    assert P.gnn.gnn_aggregate(None, 0, 0, None, None, 1, 1, None, 1, 0, None, 0, None, 0, None) == 1
    assert P.gnn.gnn_gemm(None, 1, None, 1, None, 1, 4, 4, 4, None, None, 0, None, 0, None) == 1
    assert P.gnn.gnn_plan_destroy(None) == 0


@pytest.mark.parametrize("vec,lanes,nv", [(3, 32, 1), (8, 2, 1), (8, 32, 4), (1, 16, 2), (2, 8, 4), (4, 4, 2),
                                          (0, 32, 1)])
def test_agg_mapping_rejects_unsupported(vec, lanes, nv):
    assert P.gnn.gnn_set_agg_mapping(vec, lanes, nv) == 1
    assert P.gnn.gnn_set_agg_mapping(0, 0, 0) == 0


def test_agg_mapping_accepts_supported():
    for m in [(8, 32, 1), (8, 32, 2), (4, 32, 4), (8, 8, 1), (1, 4, 1), (4, 16, 2), (8, 16, 2), (2, 16, 2),
              (8, 8, 4), (4, 8, 4)]:
        assert P.gnn.gnn_set_agg_mapping(*m) == 0
    assert P.gnn.gnn_set_agg_mapping(0, 0, 0) == 0


@pytest.mark.parametrize("ng", [0, 1, 5, 16, 64])
def test_groups_host_bit_exact_vs_oracle(ng):
    g = gs.powerlaw(1500, 25000, 16, 1500, 900, comm=32, rho=0.5, seed=ng)
    perm = np.random.default_rng(ng).permutation(g.n).astype(np.int32)
    gr, gb = P.groups_host(g.rowptr, ng, perm)
    ogr, ogb = oracle.neighbor_groups(g.rowptr, ng, perm)
    assert np.array_equal(gr, ogr) and np.array_equal(gb, ogb)


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("rho", [0.0, 0.8])
def test_las_host_bit_exact_vs_oracle(seed, rho):
    """a2 steps 2-5 (R7) from the oracle's signatures: perm and
    clusters identical to the oracle (independent implementations)."""
    g = gs.powerlaw(4000, 40000, 10, 600, 500, comm=32, rho=rho, seed=seed)
    perm_o, info = oracle.las_schedule(g.rowptr, g.colidx, seed=seed)
    perm, cl, npairs, nc = P.las_host(g.rowptr, info["sig"])
    assert npairs == len(info["pairs"])
    assert nc == info["n_clusters"]
    assert np.array_equal(perm, perm_o)
    assert np.array_equal(cl, info["cluster_of"])
    perm0, _, _, _ = P.las_host(g.rowptr, info["sig"], cluster_order=0)
    operm0, _, _, _ = oracle.las_merge(info["sig"], info["pairs"], 32, 2, cluster_order=0)
    assert np.array_equal(perm0, operm0)


def test_las_host_other_parameters():
    g = gs.powerlaw(2000, 30000, 15, 500, 400, comm=16, rho=0.9, seed=4)
    for (K, r, W, cap) in [(16, 1, 3, 8), (24, 3, 8, 32), (32, 4, 2, 16)]:
        perm_o, info = oracle.las_schedule(g.rowptr, g.colidx, K=K, r=r, W=W, cap=cap, seed=9)
        perm, cl, npairs, nc = P.las_host(g.rowptr, info["sig"], r=r, W=W, cap=cap)
        assert np.array_equal(perm, perm_o) and np.array_equal(cl, info["cluster_of"]), (K, r, W, cap)


@pytest.mark.parametrize("P_", [1, 2, 3, 4, 8])
def test_partition_rows_vs_oracle(P_):
    g = gs.powerlaw(5000, 70000, 14, 800, 600, comm=32, rho=0.0, seed=P_)
    assert np.array_equal(P.partition_rows(g.rowptr, P_), oracle.partition_rows(g.rowptr, P_))


def test_partition_rows_with_empty_tail():
    g = gs.from_rows([[1], [0, 2], [1]] + [[] for _ in range(10)])
    for P_ in (1, 2, 4, 8):
        assert np.array_equal(P.partition_rows(g.rowptr, P_), oracle.partition_rows(g.rowptr, P_))


@pytest.mark.parametrize("nparts", [2, 3, 4])
def test_local_csr_translation(nparts):
    """Padded all-gather layout (R10): u -> owner(u)*r_max + (u - bounds[owner])."""
    g = gs.powerlaw(3000, 40000, 13, 500, 500, comm=32, rho=0.3, seed=nparts)
    b = P.partition_rows(g.rowptr, nparts)
    d_out = np.bincount(g.colidx, minlength=g.n)
    for rank in range(nparts):
        lrp, lci, sdeg, rmax = P.local_csr(g.rowptr, g.colidx, b, rank)
        lo, hi = b[rank], b[rank + 1]
        assert rmax == np.diff(b).max()
        assert np.array_equal(lrp, g.rowptr[lo:hi + 1] - g.rowptr[lo])
        owner = np.searchsorted(b, g.colidx[g.rowptr[lo]:g.rowptr[hi]], side="right") - 1
        src = g.colidx[g.rowptr[lo]:g.rowptr[hi]]
        assert np.array_equal(lci, owner * rmax + (src - b[owner]))
        # global out-degree in padded slots; pads are 0
        want = np.zeros(nparts * rmax, np.int64)
        for q in range(nparts):
            want[q * rmax: q * rmax + (b[q + 1] - b[q])] = d_out[b[q]:b[q + 1]]
        assert np.array_equal(sdeg, want)


def test_new_entry_points_reject_null_plans():
    """NEXT-1/3/4 entry points validate before touching the device."""
    g = P.gnn
    r = g.gnn_tune_result()
    assert g.gnn_tune_aggregate(None, 0, 0, None, None, 1, 1, None, 1, 0, ctypes.byref(r), None) == 1
    assert g.gnn_plan_set_group_size(None, 16) == 1
    assert g.gnn_sample_neighbors(None, 16, 0, None, None) == 1
    assert g.gnn_sage_lstm_aggregate(None, None, 16, None, 160, 32, None, None, 32, None, 32, None) == 1
    assert g.gnn_sage_lstm_layer(None, None, 32, 32, None, None, None, None, None, None, None, 32, 32, 16, 0, None, 32,
                                 None, 0, None) == 1
    assert g.gnn_attn_aggregate(None, 0, None, 9, None, 1, None, 1, 8, 0.2, 0, None, 8, None, 0, None) == 1
    assert g.gnn_workspace_size(None, 6, 0, 64, 8) == 0


def test_accumulate_and_scale_validate_before_device_work():
    g = P.gnn
    assert g.gnn_aggregate_accumulate(None, 0, None, None, 1, 1, None, 1, 0, None, 0, None) == 1
    assert g.gnn_scale_rows(None, 4, 2, 8, None, 0, None) == 1  # ldy < F
    assert g.gnn_gat_transform(None, 1, 4, 1, None, 1, None, None, 1, 1, None, 3, None, 0, None) == 1


def test_plan_load_rejects_missing_and_foreign_files(tmp_path):
    """gnn_plan_load validates the file on the host before any device work."""
    h = ctypes.c_void_p()
    assert P.gnn.gnn_plan_load(str(tmp_path / "none").encode(), ctypes.byref(h)) == 1
    assert h.value is None
    f = tmp_path / "foreign"
    f.write_bytes(b"NOTAPLAN" + bytes(100))
    assert P.gnn.gnn_plan_load(str(f).encode(), ctypes.byref(h)) == 1
    assert "not a gnn plan" in P.gnn.gnn_last_error()
    assert P.gnn.gnn_plan_save(None, b"/tmp/x", 0) == 1


def test_mirrored_entry_points_validate_before_device_work():
    """NEXT-2 entry points (gnn_gemm_mirrored, gnn_gat_transform_mirrored,
    gnn_ipc_*) reject bad arguments on the host, with fake device pointers."""
    g = P.gnn
    fake = lambda off: ctypes.c_void_p(0x7f0000000000 + off)  # noqa: E731 (never dereferenced)
    X, W, H, ws = fake(0), fake(1 << 30), fake(2 << 30), fake(3 << 30)
    m, k, n = 1000, 64, 64
    arr8, _ = g._ptr_array([0x7f1000000000 + 4096 * i for i in range(8)])
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, k, n, None, None, 0, arr8, 8, ws, 1 << 20, None) == 1  # > 7
    assert "n_mirrors" in g.gnn_last_error()
    bad, _ = g._ptr_array([0x7f1000000004])
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, k, n, None, None, 0, bad, 1, ws, 1 << 20, None) == 1  # misaligned
    null, _ = g._ptr_array([0])
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, k, n, None, None, 0, null, 1, ws, 1 << 20, None) == 1
    ok, _ = g._ptr_array([0x7f1000000000])
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, k, n, None, None, 0, ok, 1, None, 0, None) == 1  # no workspace
    assert g.gnn_gemm_mirrored(X, k, W, n, X, n, m, k, n, None, None, 0, ok, 1, ws, 1 << 20, None) == 1  # H == X
    over, _ = g._ptr_array([0x7f0000000000 + 64])  # inside X
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, k, n, None, None, 0, over, 1, ws, 1 << 20, None) == 1
    assert g.gnn_gemm_mirrored(X, k, W, n, H, n, m, 0, n, None, None, 0, ok, 1, ws, 1 << 20, None) == 1  # k < 1
    assert g.gnn_gat_transform_mirrored(X, 64, m, 64, W, 256, fake(5 << 30), fake(6 << 30), 8, 32, H, 272, arr8, 8,
                                        ws, 1 << 20, None) == 1
    assert g.gnn_ipc_alloc(0, None, None) == 1
    assert g.gnn_ipc_open(None, None) == 1
    assert g.gnn_ipc_free(None) == 0 and g.gnn_ipc_close(None) == 0
