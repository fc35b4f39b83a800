"""Build libgstm.so in-tree with nvcc for sm_100a (no torch, no JIT cache).

    python -m paper_conf_cgo_xuwglgq14_b200.build [--force] [--verbose]

The shared library lands in paper_conf_cgo_xuwglgq14_b200/lib/libgstm.so,
which travels to the GPU box with the repo snapshot.
"""
from __future__ import annotations

import argparse
import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
SO = os.path.join(LIBDIR, "libgstm.so")
SOURCES = ["api.cu", "kernels.cu", "script.cu", "ubench.cu",
           "wl_ra.cu", "wl_bank.cu", "wl_ht.cu", "wl_eb.cu", "wl_km.cu", "km.cu"]     # one TU per workload: parallel build
HEADERS = ["kernels.cuh", "stm_kernels.cuh", "gstm/prim.cuh", "gstm/gen.cuh", "gstm/tx.cuh", "gstm/tx_pair.cuh",
           "gstm/tx_vbv.cuh", "gstm/workloads.cuh"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr"]


def nvcc() -> str:
    for c in [os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")]:
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "gstm.h"),
                                                                 os.path.abspath(__file__)]
    return max(os.path.getmtime(d) for d in deps) > os.path.getmtime(SO)


def build(force: bool = False, verbose: bool = False, ptxas_verbose: bool = False) -> str:
    if not force and not _stale():
        return SO
    os.makedirs(LIBDIR, exist_ok=True)
    objdir = os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    procs = []
    for src in SOURCES:
        obj = os.path.join(objdir, src.replace(".cu", ".o"))
        cmd = [nvcc()] + ARCH + FLAGS + ["-I", os.path.join(ROOT, "include"), "-I", CSRC, "-c",
                                         os.path.join(CSRC, src), "-o", obj]
        # e.g. GSTM_DEFINES="-DGSTM_STRICT_FENCES=1" (ablation builds; use --force)
        cmd += os.environ.get("GSTM_DEFINES", "").split()
        if ptxas_verbose:
            cmd += ["-Xptxas", "-v"]
        if verbose:
            print(" ".join(cmd), flush=True)
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
        objs.append(obj)
    failed = False
    for src, p in procs:
        out, _ = p.communicate()
        if p.returncode != 0 or (verbose and out):
            sys.stderr.write(f"--- {src} ---\n{out}")
        failed |= p.returncode != 0
    if failed:
        raise RuntimeError("nvcc failed")
    tmp = SO + f".tmp{os.getpid()}"
    cmd = [nvcc()] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs
    subprocess.check_call(cmd)
    os.replace(tmp, SO)
    return SO


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--ptxas", action="store_true")
    a = ap.parse_args()
    print(build(force=a.force, verbose=a.verbose, ptxas_verbose=a.ptxas))
