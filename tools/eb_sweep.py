#!/usr/bin/env python
"""EigenBench-style contention sweep (BASELINE configs[3]; the Figure 4
study of P:319-325): hot-set size H x accesses per transaction A, with the
STM, FGL and CGL measured at EVERY point, plus the version-lock count sweep
at large H.

    python tools/eb_sweep.py --out profiles/r02_eb_sweep_cm.jsonl

Every point runs over a 2^26-word heap (one fresh handle per measurement, one
warm-up launch, then a timed launch with CUDA events, L2 flushed before it).
Concurrency is a conflict knob where every pair of transactions conflicts, so
the STM's resident thread count (max_threads) is probed per point exactly as
CGL's thread count and backoff are probed (the fastest configuration of each
is reported).  A point "completes" when every transaction committed before
the watchdog: the sweep is the livelock-freedom check of the north star.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
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
    out = open(a.out, "w") if a.out else None

    def run(h, A, bits, mode, T, K, **kw):
        g = G.Gstm(heap_words, bits)
        g.set_workload_defaults("eb", n_words=1 << h, n_accesses=A, timeout_ms=60000, **kw)
        g.set_mode(mode)
        g.set_stream(stream)
        g.init_heap("eb")
        g.run("eb", min(T, 4096), 1, 7, check=False)          # warm-up
        flush.fill_(1.0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        g.launch("eb", T, K, 100)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        st = g.stats(check=False)
        g.close()
        done = st.commits + st.commits_ro
        return {"tx_per_s": done / (ms * 1e-3), "ms": ms, "abort_ratio": st.aborts / max(1, st.aborts + done),
                "status": st.status, "completed": bool(st.status == 0 and done == T * K), "threads": T,
                "tx_per_thread": K, "postvalidations": st.postvalidations, "aborts_opacity": st.aborts_opacity,
                "aborts_prevbv": st.aborts_prevbv, "aborts_tbv": st.aborts_tbv, "aborts_lock": st.aborts_lock,
                "serial_runs": st.serial_runs}

    def emit(rec):
        line = json.dumps(rec)
        print(line, flush=True)
        if out:
            out.write(line + "\n")
            out.flush()

    Hs = [10, 14, 18, 22, 26] if not a.quick else [10, 26]
    As = [8, 16, 32, 64] if not a.quick else [16, 64]
    for h in Hs:
        for A in As:
            t0 = time.perf_counter()
            bits = 22
            small = h <= 14
            T, K = (4096, 2) if small else (1 << 18, 4)
            # STM-HV: probe the concurrency (resident threads), keep the fastest
            caps = [128, 1024, 4096] if small else [1 << 14, 1 << 16, 0]
            probe = {}
            for cap in caps:
                r = run(h, A, bits, "hv", T if not small else 4096, 1, max_threads=cap)
                probe[cap] = r["tx_per_s"]
            cap = max(probe, key=probe.get)
            rec = {"H_log2": h, "A": A, "lock_bits": bits, "stm_concurrency_probe": {str(k): v for k, v in probe.items()},
                   "max_threads": cap}
            rec["hv"] = run(h, A, bits, "hv", T, K, max_threads=cap)
            rec["tbv"] = run(h, A, bits, "tbv", T, K, max_threads=cap)
            if A > 16:
                # the contention manager (serial tickets, irrevocable owner;
                # DESIGN.md §6.16), compiled into the A > 16 kernels
                rec["hv_cm"] = run(h, A, bits, "hv", T, K, max_threads=cap, serial_after=4)
            rec["fgl"] = run(h, A, bits, "fgl", T, K)
            # CGL: fastest of 1 warp per SM / 2^14 threads, Scheme #3 / TTAS + backoff, ~4K transactions
            cg = {}
            for Tc in (148 * 32, 1 << 14):
                for bo in (0, 256):
                    cg[(Tc, bo)] = run(h, A, bits, "cgl", Tc, 1, backoff_ns=bo)
            (Tc, bo) = max(cg, key=lambda k: cg[k]["tx_per_s"])
            rec["cgl"] = dict(cg[(Tc, bo)], backoff_ns=bo)
            best_stm = max(rec["hv"]["tx_per_s"], rec["tbv"]["tx_per_s"])
            rec["stm_over_cgl"] = best_stm / rec["cgl"]["tx_per_s"]
            if "hv_cm" in rec:
                rec["stm_cm_over_cgl"] = rec["hv_cm"]["tx_per_s"] / rec["cgl"]["tx_per_s"]
            rec["completed"] = all(rec[m]["completed"] for m in ("hv", "tbv", "fgl", "cgl", "hv_cm") if m in rec)
            rec["wall_s"] = round(time.perf_counter() - t0, 2)
            emit(rec)
    # version-lock count at the largest hot set
    for bits in (20, 22, 24, 26):
        rec = {"H_log2": 26, "A": 16, "lock_bits": bits, "lock_sweep": True}
        for mode in ("hv", "tbv"):
            rec[mode] = run(26, 16, bits, mode, 1 << 18, 4)
        emit(rec)


if __name__ == "__main__":
    main()
