"""Build libmv.so in-tree: every CUDA source under csrc/ compiled for sm_100a with nvcc.

`python -m paper_conf_sigmod_wangygjxlwglxyy21_b200.build` (or __graft_entry__.build()).
The .so lands next to this file so that it travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import glob
import hashlib
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libmv.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-Xptxas", "-v"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _digest():
    h = hashlib.sha256()
    for p in sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [os.path.join(ROOT, "include", "mv.h"), __file__]:
        with open(p, "rb") as f:
            h.update(p.encode() + f.read())
    return h.hexdigest()


def build(force: bool = False, verbose: bool = False) -> str:
    stamp = LIB + ".sha256"
    dg = _digest()
    if not force and os.path.exists(LIB) and os.path.exists(stamp) and open(stamp).read().strip() == dg:
        return LIB
    # one nvcc per source in parallel (each .cu owns its kernels: no device linking), then link
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC]
    cflags = [f for f in FLAGS if f != "-shared"]

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        cmd = [NVCC, *ARCH, *cflags, *inc, "-c", "-o", obj, src]
        r = subprocess.run(cmd, capture_output=True, text=True)
        return obj, cmd, r

    with ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 4)) as ex:
        results = list(ex.map(compile_one, sources()))
    log = os.path.join(PKG, "build.log")
    text = ""
    failed = None
    for obj, cmd, r in results:
        text += " ".join(cmd) + "\n" + r.stdout + r.stderr
        if r.returncode != 0 and failed is None:
            failed = r
    if failed is None:
        lcmd = [NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", "-o", LIB, *[o for o, _, _ in results]]
        failed_link = subprocess.run(lcmd, capture_output=True, text=True)
        text += " ".join(lcmd) + "\n" + failed_link.stdout + failed_link.stderr
        if failed_link.returncode != 0:
            failed = failed_link
    with open(log, "w") as f:
        f.write(text)
    if failed is not None:
        sys.stderr.write(failed.stderr[-8000:])
        raise RuntimeError(f"nvcc failed (exit {failed.returncode}); see {log}")
    r = subprocess.CompletedProcess([], 0, "", text)
    if verbose:
        sys.stderr.write(r.stderr)
    with open(stamp, "w") as f:
        f.write(dg)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
