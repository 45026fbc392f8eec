"""dev experiment: feature-chunked sweeps of the C5 gather stream (see chunk_bench_k.cu)."""
import ctypes, os, sys, subprocess
import numpy as np
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gnn_synth as gs
import paper_conf_ppopp_huangzzys21_b200 as G
so = os.path.join(ROOT, "scripts", "libchunkbench.so")
if not os.path.exists(so):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler",
                           "-fPIC", os.path.join(ROOT, "scripts", "chunk_bench_k.cu"), "-o", so])
L = ctypes.CDLL(so)
P = ctypes.c_void_p
L.cb_run.argtypes = [ctypes.c_int] * 4 + [P, ctypes.c_int64, P, P, P, ctypes.c_int64, ctypes.c_int, P, P]
cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
g = gs.config_graph(cfg)
F = 256
X = torch.rand(g.n, F, device="cuda")
Y = torch.empty_like(X)
ctr = torch.zeros(64, dtype=torch.int32, device="cuda")
plan = G.Plan(g.rowptr, g.colidx, reorder=1)
perm = plan.export()[0]
deg = np.diff(g.rowptr)[perm]
tptr = np.zeros(g.n + 1, np.int64); tptr[1:] = np.cumsum(deg)
order = np.repeat(g.rowptr[perm], deg) + (np.arange(g.nnz) - np.repeat(tptr[:-1], deg))
idx = torch.from_numpy(np.ascontiguousarray(g.colidx[order])).cuda()
tp = torch.from_numpy(tptr).cuda(); tr = torch.from_numpy(perm.astype(np.int32)).cuda()

def run(kind, cw, p1, p2):
    return L.cb_run(kind, cw, p1, p2, X.data_ptr(), F, idx.data_ptr(), tp.data_ptr(), tr.data_ptr(), g.n, F,
                    ctr.data_ptr(), Y.data_ptr())

def ev(fn, it=3):
    rc = fn(); torch.cuda.synchronize()
    if rc != 0:
        return None
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

ref = None
cases = [(0, 256, 4, 4), (0, 256, 2, 4), (0, 128, 4, 4), (0, 128, 8, 4), (0, 64, 8, 4), (0, 64, 16, 4),
         (1, 128, 8, 2), (1, 128, 12, 2), (1, 128, 16, 1), (1, 64, 8, 4), (1, 64, 12, 4), (1, 128, 4, 4),
         (2, 256, 6, 4), (2, 256, 8, 2), (2, 128, 8, 4), (2, 128, 16, 2), (2, 64, 16, 4), (2, 64, 24, 4), (2, 64, 8, 8)]
names = {0: "reg", 1: "ldgsts", 2: "bulk"}
if len(sys.argv) > 2:  # explicit cases "kind,cw,p1,p2;..."
    cases = [tuple(int(x) for x in c.split(",")) for c in sys.argv[2].split(";")]
it = int(os.environ.get("CB_IT", "3"))
for (kind, cw, p1, p2) in cases:
    Y.zero_()
    ms = ev(lambda: run(kind, cw, p1, p2), it)
    if ms is None:
        print(f"{names[kind]} cw={cw} p1={p1} blocks/SM={p2}: launch failed {torch.cuda.synchronize()}", flush=True)
        continue
    if ref is None:
        ref = Y.clone()
    same = bool(torch.equal(Y, ref))
    print(f"{names[kind]:6s} cw={cw:3d} p1={p1:2d} blocks/SM={p2}: {ms:7.3f} ms  "
          f"{g.nnz * F * 4 / ms / 1e6:6.0f} GB/s gathered  bit-identical={same}", flush=True)
