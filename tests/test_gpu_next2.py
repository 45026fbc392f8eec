"""NEXT-2 on one GPU: the mirrored GEMM epilogue (gnn_gemm_mirrored /
gnn_gat_transform_mirrored) writes bit-identical copies of its output to
every mirror -- here local buffers standing in for the peer replicas that
the multi-process exchange maps through CUDA IPC (test_gpu_multirank.py) --
and refuses what it cannot mirror instead of running unmirrored."""
import ctypes

import numpy as np
import pytest

import gnn_synth as gs

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ppopp_huangzzys21_b200 as G  # noqa: E402
from paper_conf_ppopp_huangzzys21_b200 import gnn as _g  # noqa: E402


def T(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).cuda()


def bits(t):
    return t.cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("m,k,n", [(1000, 64, 64), (100003, 256, 256), (5000, 100, 272), (7001, 256, 400)])
@pytest.mark.parametrize("nmir", [1, 3, 7])
def test_gemm_mirrored_bit_identical(m, k, n, nmir):
    X = T(gs.uniform(m, k, seed=1))
    W = T(gs.uniform(k, n, lo=-0.2, hi=0.2, seed=2))
    rs = T(gs.uniform(m, 1, lo=0.1, hi=1.0, seed=3)[:, 0])
    ref = G.gemm(X, W, row_scale=rs, relu=True)
    # mirrors inside one big buffer at different row offsets (like peer replicas' row blocks)
    big = torch.full((nmir, m + 5, n), -7.0, device="cuda")
    mirrors = [big[q, q % 5:q % 5 + m] for q in range(nmir)]
    H = G.gemm_mirrored(X, W, [t.data_ptr() for t in mirrors], row_scale=rs, relu=True)
    torch.cuda.synchronize()
    assert np.array_equal(bits(H), bits(ref))
    for q, t in enumerate(mirrors):
        assert np.array_equal(bits(t), bits(ref)), f"mirror {q}"
        # nothing outside the mirrored rows was touched
        assert torch.all(big[q, :q % 5] == -7.0) and torch.all(big[q, q % 5 + m:] == -7.0)


@pytest.mark.parametrize("Hh,Fh", [(8, 32), (4, 16), (3, 12)])
def test_gat_transform_mirrored_bit_identical(Hh, Fh):
    m, f_in = 20011, 128
    X = T(gs.uniform(m, f_in, seed=4))
    W = T(gs.uniform(f_in, Hh * Fh, lo=-0.2, hi=0.2, seed=5))
    a_s = T(gs.uniform(1, Hh * Fh, lo=-0.5, hi=0.5, seed=6)[0])
    a_d = T(gs.uniform(1, Hh * Fh, lo=-0.5, hi=0.5, seed=7)[0])
    ref = G.gat_transform(X, W, a_s, a_d, Hh, Fh)
    ldz = ref.shape[1]
    Z = torch.zeros_like(ref)
    mir = [torch.zeros_like(ref) for _ in range(2)]
    nb = _g._lib.gnn_gat_transform_workspace_size(m, f_in, Hh, Fh)
    ws = torch.empty(max(nb, 256), dtype=torch.uint8, device="cuda")
    arr, cnt = _g._ptr_array([t.data_ptr() for t in mir])
    P = lambda t: ctypes.c_void_p(t.data_ptr())  # noqa: E731
    st = _g._lib.gnn_gat_transform_mirrored(P(X), f_in, m, f_in, P(W), Hh * Fh, P(a_s), P(a_d), Hh, Fh, P(Z), ldz,
                                            arr, cnt, P(ws), nb, None)
    assert st == 0, _g.gnn_last_error()
    torch.cuda.synchronize()
    w = Hh * Fh + 2 * Hh  # z | s | t
    assert np.array_equal(bits(Z[:, :w]), bits(ref[:, :w]))
    for t in mir:
        assert np.array_equal(bits(t[:, :w]), bits(ref[:, :w]))


def test_gemm_mirrored_refuses_what_it_cannot_mirror():
    m, k, n = 300, 17, 40
    X = T(gs.uniform(m, k, seed=1))  # ldx = 17: rows not 16-byte aligned -> no TMA epilogue
    W = T(gs.uniform(k, n, seed=2))
    H = torch.empty((m, n), device="cuda")
    mir = torch.empty((m, n), device="cuda")
    ws, nb = _g.gemm_workspace(m, k, n, X.device)
    arr, cnt = _g._ptr_array([mir.data_ptr()])
    P = lambda t: ctypes.c_void_p(t.data_ptr())  # noqa: E731
    st = _g._lib.gnn_gemm_mirrored(P(X), k, P(W), n, P(H), n, m, k, n, None, None, 0, arr, cnt, P(ws), nb, None)
    assert st == 6, "misaligned X rows: GNN_ERR_UNSUPPORTED, not an unmirrored run"
    st = _g._lib.gnn_gemm_mirrored(P(X), k, P(W), n, P(H), n, m, k, n, None, None, 0, arr, cnt, None, 0, None)
    assert st != 0, "no workspace: refused"
    bad, _ = _g._ptr_array([mir.data_ptr() + 4])
    st = _g._lib.gnn_gemm_mirrored(P(X), k, P(W), n, P(H), n, m, k, n, None, None, 0, bad, 1, P(ws), nb, None)
    assert st == 1, "misaligned mirror: GNN_ERR_INVALID_ARG"
    arr8, _ = _g._ptr_array([mir.data_ptr()] * 8)
    st = _g._lib.gnn_gemm_mirrored(P(X), k, P(W), n, P(H), n, m, k, n, None, None, 0, arr8, 8, P(ws), nb, None)
    assert st == 1, "more than 7 mirrors: GNN_ERR_INVALID_ARG"


def test_ipc_buffer_roundtrip_same_process():
    buf = _g.IpcBuffer((1000, 64), torch.device("cuda", 0))
    buf.tensor.copy_(torch.arange(64000, dtype=torch.float32, device="cuda").view(1000, 64))
    assert len(buf.handle_bytes()) == 64
    torch.cuda.synchronize()
    assert float(buf.tensor[999, 63]) == 63999.0
    buf.free()
