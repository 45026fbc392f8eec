"""Build libgnn.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension).

    python -m paper_conf_ppopp_huangzzys21_b200.build [--force] [--verbose]

Every .cu/.cpp under csrc/ is compiled with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` (no --use_fast_math:
IEEE div/sqrt are part of the bit-exact contract, R9) and linked
into ``paper_conf_ppopp_huangzzys21_b200/libgnn.so`` with the static CUDA runtime.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import hashlib
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
SO = os.path.join(PKG, "libgnn.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "-I", os.path.join(ROOT, "include"),
         "--expt-relaxed-constexpr"]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  [os.path.join(ROOT, "include", "gnn.h")])


def _digest(path, hdr_digest, extra=()):
    h = hashlib.sha1(open(path, "rb").read())
    h.update(hdr_digest)
    h.update(" ".join(ARCH + FLAGS + list(extra)).encode())
    return h.hexdigest()[:16]


def build(force: bool = False, verbose: bool = False, extra=(), out: str = None) -> str:
    """Build libgnn.so; `extra` nvcc flags (e.g. -DGNN_AGG_MINB=5) and `out`
    build an A/B variant library elsewhere (load it with GNN_LIB_PATH)."""
    extra = list(extra)
    so = out or SO
    build_dir = BUILD if not extra else os.path.join(BUILD, "v_" + hashlib.sha1(" ".join(extra).encode()).hexdigest()[:8])
    os.makedirs(build_dir, exist_ok=True)
    hd = hashlib.sha1()
    for hpath in _headers():
        hd.update(open(hpath, "rb").read())
    hdr = hd.digest()
    objs, jobs = [], []
    for src in _sources():
        obj = os.path.join(build_dir, os.path.basename(src) + "." + _digest(src, hdr, extra) + ".o")
        objs.append(obj)
        if force or not os.path.exists(obj):
            cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", src, "-o", obj + ".tmp"]
            if verbose and src.endswith(".cu"):
                cmd.insert(1, "-Xptxas=-v")
            jobs.append((cmd, obj))

    def run(job):
        cmd, obj = job
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {obj}:\n{r.stderr}")
        os.replace(obj + ".tmp", obj)
        return r.stderr

    if jobs:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(jobs))) as ex:
            for out in ex.map(run, jobs):
                if verbose and out:
                    sys.stderr.write(out)
    link_stamp = hashlib.sha1("".join(objs).encode()).hexdigest()[:16]
    stamp_file = so + ".stamp"
    if force or not os.path.exists(so) or not os.path.exists(stamp_file) or open(stamp_file).read() != link_stamp:
        os.makedirs(os.path.dirname(os.path.abspath(so)), exist_ok=True)
        tmp = so + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static", "-lpthread"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
        os.replace(tmp, so)
        with open(stamp_file, "w") as f:
            f.write(link_stamp)
    # drop stale objects
    keep = set(objs)
    for o in glob.glob(os.path.join(build_dir, "*.o")):
        if o not in keep:
            os.remove(o)
    return so


if __name__ == "__main__":
    args = sys.argv[1:]
    out = args[args.index("--out") + 1] if "--out" in args else None
    extra = [a for a in args if a.startswith("-D")]
    print(build(force="--force" in args, verbose="--verbose" in args, extra=extra, out=out))
