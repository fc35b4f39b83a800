#!/usr/bin/env python
"""EigenBench-style contention sweep (BASELINE configs[3]; the Figure 4
study of P:319-325): hot-set size H x accesses per transaction A x
validation mode, plus the version-lock count sweep at large H.

    python tools/eb_sweep.py --out profiles/r01_eb_sweep.jsonl

Every point: fresh handle over a 2^26-word heap, one warm-up launch, then
`--steps` launches timed with CUDA events (L2 flushed in between).  A point
"completes" when every transaction committed before the watchdog; the sweep
is the livelock-freedom check of the north star.
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
    ap.add_argument("--out", default=None)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--heap-log2", type=int, default=26)
    ap.add_argument("--quick", action="store_true")
    a = ap.parse_args()

    import torch
    from paper_conf_cgo_xuwglgq14_b200 import build as B
    B.build()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G

    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    heap_words = 1 << a.heap_log2
    Hs = [10, 14, 18, 22, 26] if not a.quick else [10, 18, 26]
    As = [8, 16, 32, 64] if not a.quick else [8, 64]
    points = [(h, A, 22, m) for h in Hs for A in As for m in ("hv", "tbv")]
    points += [(26, 16, b, m) for b in (20, 24, 26) for m in ("hv", "tbv")]      # P:323 lock sweep
    points += [(h, 16, 22, "fgl") for h in (10, 18, 26)]
    points += [(h, 16, 22, "cgl") for h in (10, 18, 26)]
    out = open(a.out, "w") if a.out else None
    for (h, A, bits, mode) in points:
        H = 1 << h
        if mode == "cgl":
            T, K, cap = 1 << 12, 4, 0
        elif h <= 14:
            T, K, cap = 1 << 14, 4, 1 << 14 if h > 10 else 1 << 12    # concurrency cap for tiny hot sets
        else:
            T, K, cap = 1 << 18, 4, 0
        g = G.Gstm(heap_words, bits)
        g.set_workload_defaults("eb", n_words=H, n_accesses=A, max_threads=cap, timeout_ms=60000)
        g.set_mode(mode)
        g.set_stream(stream)
        g.init_heap("eb")
        g.run("eb", T, K, 7, check=False)
        torch.cuda.synchronize()
        g.reset_stats_total()
        evs = []
        for s in range(a.steps):
            flush.fill_(float(s))
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            g.launch("eb", T, K, 100 + s)
            e1.record(stream)
            evs.append((e0, e1))
        torch.cuda.synchronize()
        ms = sum(x.elapsed_time(y) for x, y in evs)
        st, n = g.stats_total(check=False)
        done = st.commits + st.commits_ro
        rec = {"H_log2": h, "A": A, "lock_bits": bits, "mode": mode, "threads": T, "tx_per_thread": K,
               "max_threads": cap, "tx_per_s": done / (ms * 1e-3), "ms_per_launch": ms / a.steps,
               "abort_ratio": st.aborts / max(1, st.aborts + done), "status": st.status,
               "completed": bool(st.status == 0 and done == T * K * a.steps),
               "postvalidations": st.postvalidations, "aborts_opacity": st.aborts_opacity,
               "aborts_prevbv": st.aborts_prevbv, "aborts_tbv": st.aborts_tbv,
               "aborts_commit_vbv": st.aborts_commit_vbv, "aborts_lock": st.aborts_lock}
        line = json.dumps(rec)
        print(line, flush=True)
        if out:
            out.write(line + "\n")
            out.flush()
        g.close()


if __name__ == "__main__":
    main()
