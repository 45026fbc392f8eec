"""bench.py — BASELINE.json metric on the products-shaped config (C5).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config C5] [--rho 0.8] [--reorder 1]

One step = one forward pass of the whole hot path over the C5 graph
(BASELINE.json configs[4]: 2,449,029 nodes, 123,718,280 CSR entries,
F = 100 -> 256):
    layer 1  Y1 = ReLU((A_gcn X) W1)        aggregate-first at F=100, then X.W
    layer 2  Y2 = A_gcn (Y1 W2)             transform-first, aggregate at F=256
    layer 3  Y3 = GAT_8x32(Y2)              X.W' -> fused edge-softmax aggregate
with the plan (LAS reorder + neighbor groups + tiles) built once before timing
(offline).  value = aggregated edge-features per second
(sum over layers of nnz * F_agg / step time, all ranks) — "edge*F/s".
N > 1: destination rows are partitioned (nnz-balanced) and every layer
all-gathers its transformed source rows over NCCL (torch.distributed).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gnn_synth as gs  # noqa: E402

METRIC = "GCN/GAT layer aggregation ms and HBM GB/s vs roofline at 1/2/4/8 B200"
UNIT = "Gedge*feat/s"
WORKLOAD = "C5: 2-layer GCN (100->256->256) + GAT 8x32 layer on ogbn-products-shaped synthetic graph"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--rho", type=float, default=0.8)
    ap.add_argument("--reorder", type=int, default=1)
    ap.add_argument("--scale", type=float, default=1.0, help="graph scale (1.0 = BASELINE size; <1 only for dev)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-rho0", action="store_true", help="skip the rho = 0 control graph (SURVEY §8(d))")
    ap.add_argument("--no-traffic", action="store_true", help="skip the ncu DRAM-traffic capture of the dominant kernel")
    ap.add_argument("--overlap", type=int, default=0,
                    help="N > 1: pipeline layer 2's exchange with its aggregation over source blocks (NEXT-2)")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "peer"],
                    help="N > 1: layer 2/3 exchange by NCCL all-gather, or fused into the GEMM epilogues as "
                         "stores into the peers' replicas through CUDA IPC (NEXT-2)")
    ap.add_argument("--cpu-rows", type=int, default=0, help="oracle sample rows (0 = auto)")
    return ap.parse_args()


# --------------------------------------------------------------------------- #
# clocks sampling (B200_PROFILING.md clocks line)
# --------------------------------------------------------------------------- #
class ClockSampler:
    FIELDS = "clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown," \
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown," \
             "clocks_event_reasons.sw_power_cap"

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------------------- #
# workload
# --------------------------------------------------------------------------- #
def glorot(fi, fo, seed):
    lim = np.sqrt(6.0 / (fi + fo))
    return gs.uniform(fi, fo, lo=-lim, hi=lim, seed=seed)


def make_inputs(cfg, rho, scale):
    c = gs.CONFIGS[cfg]
    t0 = time.time()
    g = gs.config_graph(cfg, rho=rho, scale=scale)
    gen_s = time.time() - t0
    F_in, F = c["F_in"], c["F"]
    Hh, Fh = c.get("H", 8), c.get("Fh", 32)
    X = gs.uniform(g.n, F_in, seed=gs.seed_of(cfg, 1))
    W1 = glorot(F_in, F, gs.seed_of(cfg, 2))
    W2 = glorot(F, F, gs.seed_of(cfg, 2) + 1)
    W3 = glorot(F, Hh * Fh, gs.seed_of(cfg, 2) + 2)
    al = np.sqrt(6.0 / (Fh + 1))
    a_s = gs.uniform(1, Hh * Fh, lo=-al, hi=al, seed=gs.seed_of(cfg, 3))[0]
    a_d = gs.uniform(1, Hh * Fh, lo=-al, hi=al, seed=gs.seed_of(cfg, 3) + 1)[0]
    return g, dict(X=X, W1=W1, W2=W2, W3=W3, a_src=a_s, a_dst=a_d, F_in=F_in, F=F, H=Hh, Fh=Fh, gen_s=gen_s)


def agg_bytes(nnz, n, F, extra_row=0, per_edge_extra=0):
    """Algorithmic bytes of one aggregation launch: per edge a
    4 B index + the gathered F*4 B row; per row 8 B rowptr/group + F*4 B out."""
    return nnz * (4 + 4 * F + per_edge_extra) + n * (8 + 4 * F + extra_row)


# --------------------------------------------------------------------------- #
# our arm
# --------------------------------------------------------------------------- #
def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_huangzzys21_b200 as G
    from paper_conf_ppopp_huangzzys21_b200.model import RowPartitionedGCNGAT

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")  # the communicator lines show the rank count
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        dist.init_process_group("nccl", device_id=dev)
    g, inp = make_inputs(args.config, args.rho, args.scale)
    n, nnz = g.n, g.nnz
    F_in, F, Hh, Fh = inp["F_in"], inp["F"], inp["H"], inp["Fh"]
    HF = Hh * Fh
    t0 = time.time()
    model = RowPartitionedGCNGAT(g.rowptr, g.colidx, inp["W1"], inp["W2"], inp["W3"], inp["a_src"], inp["a_dst"],
                                 Hh, Fh, rank=rank, world=world, reorder=args.reorder, device=dev,
                                 overlap=bool(args.overlap), exchange=args.exchange)
    plan_s = time.time() - t0
    info = model.plan.info
    rows, lnnz = model.rows, model.nnz_local
    model.load_input(torch.from_numpy(inp["X"]), non_blocking=False)  # inputs resident in HBM
    stream = torch.cuda.current_stream(dev)
    for _ in range(args.warmup):
        model.step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    nev = 7
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(nev)] for _ in range(args.steps)]
    clk = ClockSampler(local)
    clk.start()
    time.sleep(0.3)
    launches0 = G.launch_count()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for k in range(args.steps):
        model.step(events=evs[k])
    t_end.record(stream)
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    launches = G.launch_count() - launches0
    clocks = clk.stop()
    ms = torch.tensor([t_start.elapsed_time(t_end)], device=dev)
    if world > 1:
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_step = float(ms.item()) / args.steps
    parts = np.zeros(nev - 1)
    for k in range(args.steps):
        for i in range(nev - 1):
            parts[i] += evs[k][i].elapsed_time(evs[k][i + 1])
    parts /= args.steps
    names = ["agg1_F100", "gemm1", "gemm2+allgather", "agg2_F256", "gemm3+allgather", "gat_agg_8x32"]
    edge_feats = float(nnz) * (F_in + F + HF)  # whole job (all ranks)
    value = edge_feats / (ms_step * 1e-3) / 1e9

    # roofline of the dominant graph kernel (algorithmic bytes per launch / event time)
    per_launch = {
        "agg1_F100": agg_bytes(lnnz, rows, F_in, per_edge_extra=4),                # + nsrc[u] gather
        "agg2_F256": agg_bytes(lnnz, rows, F, extra_row=4),                        # + ndst[v]
        "gat_agg_8x32": agg_bytes(lnnz, rows, HF, per_edge_extra=4 * Hh, extra_row=4 * Hh),
    }
    dom_name = max(per_launch, key=lambda k: parts[names.index(k)])
    dom = names.index(dom_name)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = float(peaks.get("hbm_gbs", 6650.0))
    achieved = per_launch[dom_name] / (parts[dom] * 1e-3) / 1e9
    traffic, traffic_src = None, "not measured"
    if world == 1 and not args.no_traffic:
        traffic, traffic_src = measure_traffic(g, inp, model, dom_name)
    roofline = {"bound": "hbm", "kernel": dom_name, "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic,
                "dram_gbs": round(traffic / (parts[dom] * 1e-3) / 1e9, 1) if traffic else None,
                "dram_frac": round(traffic / (parts[dom] * 1e-3) / 1e9 / peak, 4) if traffic else None,
                "note": "achieved = SURVEY §8(d) no-reuse algorithmic bytes (every gathered row counted) / the "
                        "launch's event time; LAS + L2 serve part of them, so it can exceed the HBM peak. "
                        "dram_gbs = ncu DRAM bytes (traffic, cold-cache capture) / the same time.",
                "algorithmic_bytes": int(per_launch[dom_name]), "launch_ms": round(float(parts[dom]), 4),
                "traffic_source": traffic_src,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)" if "hbm_gbs" in peaks else "fallback 6650"}

    # e2e: the same steps through the public API from pinned host input to
    # pinned host output, the copies inside the timed region (pipelined over
    # the host links: input of step k+1 and output of step k overlap compute)
    e2e = None
    if not args.no_e2e:
        numa = bind_to_gpu_numa_node(dev)  # pinned buffers on the GPU's side of the host
        Xh = torch.from_numpy(inp["X"]).pin_memory()
        Yh = torch.empty((rows, HF), dtype=torch.float32).pin_memory()
        h2d = Xh.numel() * 4
        d2h = Yh.numel() * 4
        s0, s1 = model.run_pipelined(Xh, Yh, 2)
        torch.cuda.synchronize(dev)
        ke = max(2, args.steps)  # the same K as the device-timed value (pipeline fill / drain amortised alike)
        e_s, e_e = model.run_pipelined(Xh, Yh, ke)
        torch.cuda.synchronize(dev)
        me = torch.tensor([e_s.elapsed_time(e_e) / ke], device=dev)
        if world > 1:
            dist.all_reduce(me, op=dist.ReduceOp.MAX)
        e2e = {"value": round(edge_feats / (float(me.item()) * 1e-3) / 1e9, 3), "unit": UNIT,
               "ms_per_step": round(float(me.item()), 3), "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "steps": ke,
               "note": "pinned host X -> device, step, device -> pinned host Y3 every step; copies of "
                       "step k+1 / k overlap compute on separate streams", "host_numa_node": numa}

    out = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": WORKLOAD, "graph": args.config, "n": n, "nnz": nnz, "rho": args.rho,
                   "reorder": args.reorder, "F": [F_in, F, HF], "heads": Hh, "scale": args.scale,
                   "group_size": info["group_size"], "tile_groups": info["tile_groups"],
                   "l2": "inputs larger than L2 (X 980 MB, activations 2.5 GB vs 126 MB); no flush",
                   "parallelism": f"row-partition x{world}" + ((" + NCCL ring exchange overlapped with layer-2 "
                                                                "source-block aggregation" if args.overlap else
                                                                " + GEMM-epilogue peer stores (CUDA IPC) + NCCL "
                                                                "barrier" if args.exchange == "peer" else
                                                                " + NCCL all-gather") if world > 1 else "")},
        "breakdown_ms": {k: round(float(v), 4) for k, v in zip(names, parts)},
        "plan": {"build_s": round(plan_s, 2), "gen_s": round(inp["gen_s"], 2), "n_groups": info["n_groups"],
                 "n_tiles": info["n_tiles"], "n_split_rows": info["n_split_rows"], "n_clusters": info["n_clusters"],
                 "ms_minhash": round(info["ms_minhash"], 1), "ms_lsh": round(info["ms_lsh"], 1),
                 "ms_merge": round(info["ms_merge"], 1)},
        "roofline": roofline,
        "clocks": clocks,
        "gpu_launches": int(launches),
        "e2e": e2e,
    }
    if world == 1 and not args.no_rho0 and args.rho != 0.0:
        del model
        torch.cuda.empty_cache()
        out["rho0"] = rho0_control(args, dev)
    if rank == 0 and world == 1 and not args.no_cpu:
        out["cpu_baseline"] = cpu_baseline(g, inp, args)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def bind_to_gpu_numa_node(dev):
    """Run this process on the CPUs of the GPU's NUMA node before the pinned
    host buffers of the e2e leg are allocated (first touch places them there),
    so the host<->device copies do not cross the socket link.  Plumbing only;
    returns the node, or None when the topology is not visible."""
    import torch
    try:
        pr = torch.cuda.get_device_properties(dev)
        bdf = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
        node = int(open(f"/sys/bus/pci/devices/{bdf}/numa_node").read().strip())
        if node < 0:
            return None
        cpus = set()
        for part in open(f"/sys/devices/system/node/node{node}/cpulist").read().strip().split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        if cpus:
            os.sched_setaffinity(0, cpus)
        return node
    except Exception:  # noqa: BLE001 (no sysfs, containers without the topology)
        return None


def measure_traffic(g, inp, model, kernel):
    """ncu DRAM bytes (read + write) of one launch of the dominant kernel on this
    run's graph and plan: the plan is saved (gnn_plan_save) and a probe process
    repeats the launch under `ncu --metrics dram__bytes_*` (cold cache, like the
    driver's launch list).  Returns (bytes or None, how)."""
    import shutil
    import tempfile
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not os.path.exists(ncu):
        return None, "ncu not found"
    d = tempfile.mkdtemp(prefix="gnn_traffic_")
    try:
        model.plan.save(os.path.join(d, "plan.gnnplan"))
        np.savez(os.path.join(d, "meta.npz"), n=g.n, F_in=inp["F_in"], F=inp["F"], H=inp["H"], Fh=inp["Fh"])
        # the probe launches the kernel twice (k_score_max for GAT is not matched):
        # profile the second launch
        cmd = [ncu, "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
               "--clock-control", "none", "-k", "regex:k_aggregate|k_stream_g4", "-s", "1", "-c", "1", "--csv",
               "--page", "raw",
               sys.executable, os.path.join(ROOT, "scripts", "traffic_probe.py"), d, kernel]
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=300)
        import csv
        import io
        rows = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
        rec = list(csv.reader(io.StringIO("\n".join(rows))))
        if len(rec) < 3:
            tail = (r.stdout[-300:] + r.stderr[-300:]).replace("\n", " ")
            return None, f"ncu produced no record (rc {r.returncode}): {tail}"
        h, units, vals = rec[0], rec[1], rec[2]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}

        def val(name):
            i = h.index(name)
            return float(vals[i].replace(",", "")) * scale.get(units[i], 1)
        tot = val("dram__bytes_read.sum") + val("dram__bytes_write.sum")
        it = h.index("gpu__time_duration.sum")
        t_ms = float(vals[it].replace(",", "")) * {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3,
                                                   "msecond": 1.0, "ms": 1.0, "second": 1e3,
                                                   "s": 1e3}.get(units[it].strip(), 1e-6)
        return int(tot), (f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum on one launch of "
                          f"{vals[h.index('Kernel Name')]} (this run's plan; cold cache; {t_ms:.3f} ms under ncu)")
    except Exception as e:  # noqa: BLE001
        return None, f"ncu capture failed: {e!r}"[:200]
    finally:
        shutil.rmtree(d, ignore_errors=True)


def rho0_control(args, dev):
    """The same step on the rho = 0 graph (no planted neighbour similarity, the
    control of SURVEY §8(d)): LAS has little to find there."""
    import torch
    from paper_conf_ppopp_huangzzys21_b200.model import RowPartitionedGCNGAT
    g, inp = make_inputs(args.config, 0.0, args.scale)
    t0 = time.time()
    m = RowPartitionedGCNGAT(g.rowptr, g.colidx, inp["W1"], inp["W2"], inp["W3"], inp["a_src"], inp["a_dst"],
                             inp["H"], inp["Fh"], reorder=args.reorder, device=dev)
    plan_s = time.time() - t0
    m.load_input(torch.from_numpy(inp["X"]), non_blocking=False)
    stream = torch.cuda.current_stream(dev)
    for _ in range(max(2, args.warmup)):
        m.step()
    k = max(3, min(args.steps, 5))
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(7)] for _ in range(k)]
    torch.cuda.synchronize(dev)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for i in range(k):
        m.step(events=evs[i])
    b.record(stream)
    torch.cuda.synchronize(dev)
    ms = a.elapsed_time(b) / k
    names = ["agg1_F100", "gemm1", "gemm2+allgather", "agg2_F256", "gemm3+allgather", "gat_agg_8x32"]
    parts = [sum(evs[i][j].elapsed_time(evs[i][j + 1]) for i in range(k)) / k for j in range(6)]
    info = m.plan.info
    del m
    torch.cuda.empty_cache()
    return {"rho": 0.0, "ms_per_step": round(ms, 4), "steps": k,
            "value": round(float(g.nnz) * (inp["F_in"] + inp["F"] + inp["H"] * inp["Fh"]) / (ms * 1e-3) / 1e9, 3),
            "breakdown_ms": {n: round(v, 4) for n, v in zip(names, parts)},
            "plan": {"build_s": round(plan_s, 2), "gen_s": round(inp["gen_s"], 2), "n_clusters": info["n_clusters"]},
            "note": "control graph without planted neighbour similarity (SURVEY §8(d) rho = 0); same step"}


# --------------------------------------------------------------------------- #
# oracle timing (cpu_baseline and --impl reference)
# --------------------------------------------------------------------------- #
def oracle_sample(g, inp, rows):
    """The step's three layers, oracle definitions, on a sample of destination rows."""
    import oracle
    X = inp["X"]
    F_in, F, Hh, Fh = inp["F_in"], inp["F"], inp["H"], inp["Fh"]
    rng = np.random.default_rng(5)
    Y1s = rng.random((g.n, F), dtype=np.float32)  # layer-2 input of the right shape (timing only)
    Zs = rng.random((g.n, Hh * Fh + Hh), dtype=np.float32)
    t = rng.random((g.n, Hh), dtype=np.float32)
    t0 = time.perf_counter()
    oracle.gcn_layer(g.rowptr, g.colidx, X, inp["W1"], relu=True, rows=rows)
    oracle.gcn_layer(g.rowptr, g.colidx, Y1s, inp["W2"], relu=False, rows=rows)
    oracle.gat_aggregate(g.rowptr, g.colidx, Zs, t, Hh, Fh, 0.2, rows=rows)
    dt = time.perf_counter() - t0
    deg = np.diff(g.rowptr)[rows].sum()
    return float(deg) * (F_in + F + Hh * Fh), dt


def cpu_baseline(g, inp, args, target_s=15.0):
    nrows = args.cpu_rows
    rng = np.random.default_rng(1)
    if nrows <= 0:
        rows = rng.choice(g.n, 2000, replace=False)
        units, dt = oracle_sample(g, inp, rows)
        nrows = int(min(g.n, max(2000, 2000 * target_s / max(dt, 1e-3))))
    rows = np.sort(rng.choice(g.n, nrows, replace=False))
    units, dt = oracle_sample(g, inp, rows)
    return {"value": round(units / dt / 1e9, 5), "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{nrows} random destination rows of the C5 step (3 layers, oracle fp64, single thread); "
                      f"{units / 1e9:.2f} G edge*feat in {dt:.1f} s",
            "cpu": _cpu_name(), "nproc": os.cpu_count()}


def _cpu_name():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if rank != 0:
        return
    import oracle
    oracle.build()
    g, inp = make_inputs(args.config, args.rho, args.scale)
    rng = np.random.default_rng(2)
    # size each step to ~6 s of oracle work
    rows = rng.choice(g.n, 1000, replace=False)
    u, dt = oracle_sample(g, inp, np.sort(rows))
    nrows = int(min(g.n, max(1000, 1000 * 6.0 / max(dt, 1e-3))))
    rows = np.sort(rng.choice(g.n, nrows, replace=False))
    for _ in range(args.warmup):
        oracle_sample(g, inp, rows[: max(1, nrows // 10)])
    tot_u, tot_t = 0.0, 0.0
    for _ in range(args.steps):
        u, dt = oracle_sample(g, inp, rows)
        tot_u += u
        tot_t += dt
    value = tot_u / tot_t / 1e9
    out = {"impl": "reference", "metric": METRIC, "value": round(value, 5), "unit": UNIT, "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(tot_t / args.steps * 1e3, 2),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": WORKLOAD, "graph": args.config, "n": g.n, "nnz": g.nnz, "rho": args.rho},
           "cpu_baseline": {"value": round(value, 5), "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": f"{nrows} random destination rows per step, 3 layers, oracle fp64",
                            "cpu": _cpu_name(), "nproc": os.cpu_count()},
           "e2e": {"value": round(value, 5), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def relaunch_under_torchrun(n):
    """`python bench.py --gpus N` without a launcher: re-exec this script under
    torch.distributed.run with N local ranks (127.0.0.1 rendezvous), NCCL's INFO
    lines on so the communicator's rank count is visible in the log."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, env=env)


def main():
    args = parse()
    world = os.environ.get("WORLD_SIZE")
    if world is None and args.gpus > 1:
        if args.impl == "ours":
            import torch
            have = torch.cuda.device_count()
            if have < args.gpus:
                sys.exit(f"bench.py --gpus {args.gpus}: only {have} CUDA device(s) visible")
        sys.exit(relaunch_under_torchrun(args.gpus))
    if world is not None and int(world) != args.gpus:
        sys.exit(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}; launch one rank per GPU")
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
