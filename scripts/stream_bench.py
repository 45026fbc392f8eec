"""dev experiment: memory-system bound of the C5 gather stream (see stream_bench_k.cu)."""
import ctypes, os, sys, time
import numpy as np
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs
import paper_conf_ppopp_huangzzys21_b200 as G
L = ctypes.CDLL(os.path.join(ROOT, "scripts", "libstreambench.so"))
P = ctypes.c_void_p
L.sb_run_stream.argtypes = [P, P, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int, P]
L.sb_run_rows.argtypes = [P, P, P, P, ctypes.c_int64, P, ctypes.c_int, ctypes.c_int, P]
g = gs.config_graph("C5")
X = torch.rand(g.n, 256, device="cuda")
Y = torch.empty_like(X)
out = torch.zeros(1, device="cuda")
ctr = torch.zeros(1, dtype=torch.int32, device="cuda")
def ev(fn, it=3):
    fn(); torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it
for reorder in (0, 1):
    if reorder:
        plan = G.Plan(g.rowptr, g.colidx, reorder=1)
        perm = plan.export()[0]
    else:
        perm = np.arange(g.n, dtype=np.int32)
    deg = np.diff(g.rowptr)[perm]
    tptr = np.zeros(g.n + 1, np.int64); tptr[1:] = np.cumsum(deg)
    # task-ordered colidx
    idx = np.concatenate([g.colidx[g.rowptr[v]:g.rowptr[v + 1]] for v in perm[:0]] + [np.zeros(0, np.int32)])
    order = np.repeat(g.rowptr[perm], deg) + (np.arange(g.nnz) - np.repeat(tptr[:-1], deg))
    idx = torch.from_numpy(np.ascontiguousarray(g.colidx[order])).cuda()
    tp = torch.from_numpy(tptr).cuda(); tr = torch.from_numpy(perm.astype(np.int32)).cuda()
    for U in (2, 4, 8):
        for occ in (4, 8):
            blocks = 148 * occ
            warps = blocks * 8
            chunk = (g.nnz + warps - 1) // warps
            ms = ev(lambda: L.sb_run_stream(X.data_ptr(), idx.data_ptr(), g.nnz, chunk, U, blocks, out.data_ptr()))
            ms2 = ev(lambda: L.sb_run_rows(X.data_ptr(), idx.data_ptr(), tp.data_ptr(), tr.data_ptr(), g.n,
                                            ctr.data_ptr(), U, blocks, Y.data_ptr()))
            print(f"reorder={reorder} U={U} blocks/SM={occ}: stream {ms:.2f} ms ({g.nnz*1024/ms/1e9:.0f} GB/s)"
                  f" | rows(dynamic) {ms2:.2f} ms", flush=True)
