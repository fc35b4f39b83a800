#!/usr/bin/env python
"""Ablation runner: time one workload under several parameter variants.

    python tools/ablate.py --wl bank --variants 'mode=tbv' 'mode=hv' 'mode=tbv,snapshot_reuse=0'

Each variant: warm-up launches, then --steps launches timed with CUDA events
on a dedicated stream (L2 flushed between steps).  Prints one JSON line per
variant (tx/s, ms/launch, abort ratio, stats).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SHAPES = {
    "bank": dict(words=1 << 20, bits=20, T=1 << 20, K=16, params=dict(n_words=1 << 20)),
    "ra": dict(words=1 << 10, bits=10, T=256, K=4096, params=dict(n_reads=4, n_writes=4, n_words=1 << 10)),
    "ra_paper": dict(words=1 << 23, bits=20, T=65536, K=16, params=dict(n_reads=4, n_writes=4, n_words=1 << 23)),
    "ht": dict(words=(1 << 20) + 2 * (1 << 24), bits=22, T=1 << 22, K=4, params=dict()),
    "km": dict(words=1024 * 17, bits=20, T=1 << 24, K=1, params=dict()),
    # one version lock per 32-word-aligned k-means record
    "km_rec": dict(words=1024 * 32, bits=20, T=1 << 24, K=1, params=dict(km_stride=32, lock_shift=5)),
    "eb": dict(words=1 << 26, bits=22, T=1 << 18, K=16, params=dict(n_words=1 << 26, n_accesses=16)),
}
WL_OF = {"bank": "bank", "ra": "ra", "ra_paper": "ra", "ht": "ht", "km": "km", "km_rec": "km", "eb": "eb"}


def parse_variant(s: str) -> dict:
    out = {}
    for kv in filter(None, s.split(",")):
        k, v = kv.split("=")
        out[k] = v
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--wl", default="bank", choices=list(SHAPES))
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--T", type=int, default=None)
    ap.add_argument("--K", type=int, default=None)
    ap.add_argument("--bits", type=int, default=None)
    ap.add_argument("--variants", nargs="+", default=["mode=auto"])
    ap.add_argument("--torch-heap", action="store_true", help="attach a torch tensor as the heap")
    ap.add_argument("--sync", action="store_true", help="host sync after every step")
    ap.add_argument("--seed-base", type=int, default=0)
    ap.add_argument("--flush-first", action="store_true", help="allocate the L2-flush buffer before the handle")
    ap.add_argument("--pre-alloc-mb", type=int, default=0,
                    help="cudaMalloc this many MiB before the handle (moves the handle's physical pages)")
    ap.add_argument("--variant-timeout", type=int, default=240, help="seconds per variant process")
    ap.add_argument("--inproc", action="store_true",
                    help="run all variants in this process (default: one fresh process per variant, so "
                         "every variant sees the same allocation history)")
    a = ap.parse_args()

    if len(a.variants) > 1 and not a.inproc:
        import subprocess
        argv = [x for x in sys.argv[1:]]
        i = argv.index("--variants")
        j = i + 1
        while j < len(argv) and not argv[j].startswith("--"):
            j += 1
        base = argv[:i] + argv[j:]
        for v in a.variants:
            try:
                subprocess.run([sys.executable, os.path.abspath(__file__)] + base + ["--variants", v], check=False,
                               timeout=a.variant_timeout)
            except subprocess.TimeoutExpired:
                print(json.dumps({"wl": a.wl, "variant": v, "error": f"timeout {a.variant_timeout}s"}), flush=True)
        return

    import torch
    from paper_conf_cgo_xuwglgq14_b200 import build as B
    B.build()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G

    shp = dict(SHAPES[a.wl])
    T = a.T or shp["T"]
    K = a.K or shp["K"]
    bits = a.bits if a.bits is not None else shp["bits"]
    wl = WL_OF[a.wl]
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda") if a.flush_first else None
    pre = torch.empty(a.pre_alloc_mb << 18, dtype=torch.float32, device="cuda") if a.pre_alloc_mb else None
    for var in a.variants:
        kv = parse_variant(var)
        mode = kv.pop("mode", "auto")
        pad_mb = int(kv.pop("pad_mb", 0))       # shift where the handle's buffers land
        pad = torch.empty(pad_mb << 18, dtype=torch.float32, device="cuda") if pad_mb else None
        paired = bool(int(kv.pop("paired", 0)))
        words = int(kv.pop("words", 0)) or shp["words"]
        if wl == "km" and "km_stride" in kv:
            words = 1024 * int(kv["km_stride"])
        g = G.Gstm(words, bits, paired=paired)
        if flush is None:
            flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
        g.set_workload_defaults(wl, **dict(shp["params"], **{k: int(v) for k, v in kv.items()}))
        g.set_mode(mode)
        g.set_stream(stream)
        theap = None
        if a.torch_heap:
            theap = torch.empty(words, dtype=torch.int32, device="cuda")
            g.attach_heap(theap)
        g.init_heap(wl)
        for w in range(a.warmup):
            if wl == "ht":
                g.init_heap("ht")
            g.run(wl, T, K, 1000 + w)
        torch.cuda.synchronize()
        g.reset_stats_total()
        evs = []
        for s in range(a.steps):
            if wl == "ht":
                g.init_heap("ht")       # HT node ids are per launch: every step starts from an empty table
            flush.fill_(float(s))
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            g.launch(wl, T, K, a.seed_base + s)
            e1.record(stream)
            evs.append((e0, e1))
            if a.sync:
                stream.synchronize()
        torch.cuda.synchronize()
        tot_ms = sum(e0.elapsed_time(e1) for e0, e1 in evs)
        st, nl = g.stats_total(check=False)
        assert nl == a.steps
        done, ab = st.commits + st.commits_ro, st.aborts
        agg = {k: v for k, v in st.as_dict().items() if isinstance(v, int)}
        line = {"wl": a.wl, "variant": var, "T": T, "K": K, "bits": bits, "mode_used": G.MODE_NAMES[st.mode_used],
                "tx_per_s": done / (tot_ms * 1e-3), "ms_per_launch": tot_ms / a.steps,
                "abort_ratio": ab / max(1, ab + done), "stats": agg}
        ph = g.phase_cycles()
        if any(ph.values()):
            tot = sum(ph.values())
            line["phases_frac"] = {k: v / tot for k, v in ph.items()}
            line["phase_cycles"] = ph
        print(json.dumps(line), flush=True)
        g.close()


if __name__ == "__main__":
    main()
