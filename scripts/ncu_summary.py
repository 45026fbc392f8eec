"""Summarise an ncu --set full report (run here, no GPU needed).

    python scripts/ncu_summary.py gpurun_out/prof.ncu-rep [--sass] [--json out.json]

Prints per kernel: duration, DRAM bytes, L1/L2 hit rates, occupancy, DRAM/L2
throughput, tensor-pipe activity, registers; with --sass the hottest SASS
instructions by warp-stall samples.  --json writes {kernel: dram_bytes} for
bench.py's roofline "traffic" field.
"""
import csv
import io
import json
import subprocess
import sys
from collections import Counter

KEYS = [
    ("gpu__time_duration.sum", "ms"),
    ("dram__bytes_read.sum", "rd"),
    ("dram__bytes_write.sum", "wr"),
    ("lts__t_sector_hit_rate.pct", "L2hit%"),
    ("l1tex__t_sector_hit_rate.pct", "L1hit%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps%"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram%"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2%"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor%"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__inst_executed.sum", "inst"),
]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-6, "us": 1e-3, "ms": 1.0,
        "s": 1e3}


def ncu(args):
    return subprocess.run(["ncu"] + args, capture_output=True, text=True).stdout


def raw(rep):
    rows = list(csv.reader(io.StringIO(ncu(["-i", rep, "--page", "raw", "--csv"]))))
    hdr, units, data = rows[0], rows[1], rows[2:]
    out = []
    for d in data:
        rec = {"kernel": d[hdr.index("Kernel Name")]}
        for k, short in KEYS:
            if k not in hdr:
                continue
            i = hdr.index(k)
            try:
                v = float(d[i])
            except ValueError:
                continue
            u = units[i]
            if short in ("rd", "wr"):
                v = v * UNIT.get(u, 1) / 1e9  # GB
            elif short == "ms":
                v = v * UNIT.get(u, 1)
            rec[short] = v
        out.append(rec)
    return out


def sass_hot(rep, top=12):
    rows = list(csv.reader(io.StringIO(ncu(["-i", rep, "--page", "source", "--csv", "--print-source", "sass"]))))
    kernels, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            kernels.append(cur)
        elif cur is not None:
            cur["rows"].append(r)
    for k in kernels:
        hdr = k["rows"][0]
        data = [r for r in k["rows"][1:] if len(r) == len(hdr)]
        i_src, i_s = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
        tot = sum(float(r[i_s] or 0) for r in data) or 1
        byop = Counter()
        for r in data:
            t = r[i_src].split()
            if not t:
                continue
            op = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
            byop[op.split(".")[0]] += float(r[i_s] or 0)
        print(f"\n{k['name'][:100]}")
        print("  stall share by opcode: " + ", ".join(f"{op} {v / tot * 100:.0f}%" for op, v in byop.most_common(8)))
        for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[:top]:
            print(f"   {float(r[i_s]) / tot * 100:5.1f}%  {r[i_src].strip()[:90]}")


def main():
    rep = sys.argv[1]
    recs = raw(rep)
    for r in recs:
        name = r["kernel"][:60]
        cols = " ".join(f"{s}={r[s]:.4g}" for _, s in KEYS if s in r)
        print(f"{name:60s} {cols}")
    if "--sass" in sys.argv:
        sass_hot(rep)
    if "--json" in sys.argv:
        out = {r["kernel"]: (r.get("rd", 0) + r.get("wr", 0)) * 1e9 for r in recs}
        json.dump(out, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)


if __name__ == "__main__":
    main()
