#!/usr/bin/env python
"""L2 round-trip latency of a random returning atomic vs load on the GPU.

    python tools/latency_probe.py [--table-bytes 8388608]

gstm_ubench kind 4 runs one dependent chain of random atom.or per thread, so
ops/s = threads / latency: latency_ns = threads / ops_per_s * 1e9.  Swept over
the number of resident threads to separate the unloaded round trip from
queueing under load.  Prints one JSON line per point.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--table-bytes", type=int, default=8 << 20)
    a = ap.parse_args()
    from paper_conf_cgo_xuwglgq14_b200 import build as B
    B.build()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G
    import torch
    torch.cuda.init()
    for threads in [256, 148 * 256, 148 * 1024, 148 * 2048]:
        n_ops = max(threads * 64, 1 << 20)
        ops, ms = G.gstm_ubench(4, a.table_bytes, n_ops, threads)
        print(json.dumps({"kind": "atom.or chain", "table_bytes": a.table_bytes, "threads": threads,
                          "ops_per_s": ops, "latency_ns": threads / ops * 1e9, "ms": ms}), flush=True)


if __name__ == "__main__":
    main()
