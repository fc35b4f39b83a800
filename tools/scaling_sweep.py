#!/usr/bin/env python
"""Thread-scalability sweep of the STM variants (the paper's Figure 3 study,
P:300).

For each workload and concurrency-control mode, a FIXED batch of transactions
is run with T = 2^8 .. 2^20 STM threads (K = total / T transactions each);
one line per point: committed tx/s, abort ratio, ms.  CGL is not swept (the
paper: "it does not scale").  Points whose single launch would exceed the
time budget are skipped (STM-VBV serialises its writers).

    python tools/scaling_sweep.py --out profiles/r01_scaling.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# workload -> (heap words, lock bits, params, total transactions)
SHAPES = {
    # RA as the paper ran it (8M shared words, 1M locks)
    "ra": (1 << 23, 20, dict(n_reads=4, n_writes=4, n_words=1 << 23), 1 << 22),
    "bank": (1 << 20, 20, dict(n_words=1 << 20), 1 << 22),
    "ht": (None, 22, dict(), 1 << 22),
    "km": (1024 * 17, 20, dict(), 1 << 20),
    "eb": (1 << 24, 22, dict(n_words=1 << 24, n_accesses=16), 1 << 21),
}
MODES = ["auto", "hv", "tbv", "hv_backoff", "vbv", "fgl"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--wl", nargs="+", default=list(SHAPES))
    ap.add_argument("--modes", nargs="+", default=MODES)
    ap.add_argument("--tmin", type=int, default=8)
    ap.add_argument("--tmax", type=int, default=20)
    ap.add_argument("--budget-ms", type=float, default=4000.0, help="skip points predicted slower than this")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()

    import torch
    from paper_conf_cgo_xuwglgq14_b200 import build as B
    B.build()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G

    out = open(a.out, "a") if a.out else None
    for wl in a.wl:
        words, bits, params, total = SHAPES[wl]
        for mode in a.modes:
            last_rate = None
            for lt in range(a.tmin, a.tmax + 1, 2):
                T = 1 << lt
                K = max(1, total // T)
                if wl == "ht":
                    words = (1 << 20) + 2 * T * K
                if last_rate and (T * K) / last_rate * 1e3 > a.budget_ms * 4:
                    continue
                g = G.Gstm(words, bits)
                g.set_workload_defaults(wl, timeout_ms=int(a.budget_ms * 3), **params)
                g.set_mode(mode)
                g.init_heap(wl)
                # warm-up launch on a small slice, then the measured launch
                g.launch(wl, min(T, 1024), 1, 7)
                g.stats(check=False)
                if wl == "ht":
                    g.init_heap(wl)
                g.launch(wl, T, K, 11)
                st = g.stats(check=False)
                line = {"wl": wl, "mode": mode, "mode_used": G.MODE_NAMES[st.mode_used], "T": T, "K": K,
                        "tx": T * K, "tx_per_s": st.tx_per_s, "abort_ratio": st.abort_ratio,
                        "ms": st.elapsed_ms, "status": st.status}
                if st.status == 0:
                    last_rate = st.tx_per_s
                print(json.dumps(line), flush=True)
                if out:
                    out.write(json.dumps(line) + "\n")
                    out.flush()
                g.close()
                torch.cuda.synchronize()
    if out:
        out.close()


if __name__ == "__main__":
    main()
