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
           "wl_ra.cu", "wl_bank.cu", "wl_ht.cu", "wl_eb.cu", "wl_eb16.cu", "wl_eb32.cu", "wl_km.cu", "km.cu"]     # one TU per workload: parallel build
HEADERS = ["kernels.cuh", "stm_kernels.cuh", "gstm/prim.cuh", "gstm/gen.cuh", "gstm/tx.cuh", "gstm/tx_pair.cuh",
           "gstm/tx_vbv.cuh", "gstm/tx_irr.cuh", "gstm/workloads.cuh"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr"]


def nvcc() -> str:
    for c in [os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")]:
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


# build flavours: lib/libgstm_<name>.so with extra defines (tests and tools
# load them by name, gstm.lib(flavour)); "" is the product library
FLAVOURS = {
    "": [],
    "strict": ["-DGSTM_STRICT_FENCES=1"],      # every fence the formal PTX model asks for
    "hlog": ["-DGSTM_HLOG=1"],                 # order-preserving hashed lock logs
    "phase": ["-DGSTM_PHASE_TIMING=1"],        # Figure 5 per-phase cycle counters
    "smem": ["-DGSTM_SMEM_LOGS=1"],            # bank / RA / KM logs in shared memory
}


def so_path(flavour: str = "") -> str:
    return os.path.join(LIBDIR, f"libgstm_{flavour}.so" if flavour else "libgstm.so")


def _stale(so: str = SO) -> bool:
    if not os.path.exists(so):
        return True
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "gstm.h"),
                                                                 os.path.abspath(__file__)]
    return max(os.path.getmtime(d) for d in deps) > os.path.getmtime(so)


def build(force: bool = False, verbose: bool = False, ptxas_verbose: bool = False, flavour: str = "") -> str:
    so = so_path(flavour)
    if not force and not _stale(so):
        return so
    os.makedirs(LIBDIR, exist_ok=True)
    objdir = os.path.join(HERE, "build", flavour or "default")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    procs = []
    for src in SOURCES:
        obj = os.path.join(objdir, src.replace(".cu", ".o"))
        cmd = [nvcc()] + ARCH + FLAGS + ["-I", os.path.join(ROOT, "include"), "-I", CSRC, "-c",
                                         os.path.join(CSRC, src), "-o", obj]
        cmd += FLAVOURS[flavour]
        # e.g. GSTM_DEFINES="-DGSTM_HT_MINB=3" (ablation builds of the product library; use --force)
        if not flavour:
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
    tmp = so + f".tmp{os.getpid()}"
    cmd = [nvcc()] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs
    subprocess.check_call(cmd)
    os.replace(tmp, so)
    return so


def build_all(force: bool = False) -> list:
    return [build(force=force, flavour=f) for f in FLAVOURS]


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--ptxas", action="store_true")
    ap.add_argument("--flavour", default="", choices=list(FLAVOURS) + ["all"])
    a = ap.parse_args()
    if a.flavour == "all":
        print("\n".join(build_all(force=a.force)))
    else:
        print(build(force=a.force, verbose=a.verbose, ptxas_verbose=a.ptxas, flavour=a.flavour))
