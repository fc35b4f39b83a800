"""Figure 5 analogue: execution-time breakdown of a transactional
thread in Figure 5's seven categories -- native code, transaction
initialisation, buffering, consistency checking, acquiring/releasing locks,
committing, aborted transactions -- plus "other" (loop, refill, SIMT waiting
outside a transaction), for every BASELINE config, under STM-Optimized (the
paper's choice for Figure 5) and the other modes.  GPU only; uses the
"phase" build flavour (every lane times its own path, tx.cuh Tx::ph).

    python tools/fig5.py [--out profiles/r02_fig5.jsonl] [--configs km_c4,...] [--modes auto,hv,tbv]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_cgo_xuwglgq14_b200 import build as B  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--configs", default="km_c4,bank,ra_c0,ht_c2,eb_c3_h26_a16,eb_c3_h10_a64")
    ap.add_argument("--modes", default="auto,hv,tbv")
    a = ap.parse_args()
    B.build(flavour="phase")
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G
    rows = []
    for cfg in a.configs.split(","):
        for mode in a.modes.split(","):
            if cfg == "bank":
                g = G.Gstm(bench.ACCOUNTS, bench.BITS, paired=True, flavour="phase")
                g.set_workload_defaults("bank", n_words=bench.ACCOUNTS, prelock_vbv=0, k_lock=1, spin_cap=1)
                wl, T, K = "bank", bench.THREADS, bench.TX_PER_THREAD
            else:
                wl, words, bits, p, T, K, _, _ = bench.CONFIGS[cfg]
                g = G.Gstm(words, bits, flavour="phase")
                g.set_workload_defaults(wl, **p)
                if cfg == "eb_c3_h10_a64":
                    g.set_params(max_threads=4096)
            g.set_mode(mode)
            g.init_heap(wl)
            g.run(wl, T, K, 1)                          # warm-up
            g.init_heap(wl)
            g.reset_stats_total()
            st = g.run(wl, T, K, 2)
            ph = g.phase_cycles()
            in_tx = sum(v for k, v in ph.items() if k != "other")
            row = {"config": cfg, "mode": mode, "mode_used": G.MODE_NAMES[st.mode_used], "tx_per_s": st.tx_per_s,
                   "abort_ratio": st.abort_ratio, "cycles": ph,
                   "fraction_of_transactional_time": {k: v / in_tx for k, v in ph.items() if k != "other"},
                   "other_over_transactional": ph["other"] / max(1, in_tx),
                   "note": "phase flavour (instrumented: clock64 at every category switch; rates are slower "
                           "than the product build's)"}
            rows.append(row)
            f = row["fraction_of_transactional_time"]
            print(f"{cfg:15s} {mode:4s} ({row['mode_used']}) " +
                  " ".join(f"{k[:6]}={100 * v:5.1f}%" for k, v in f.items()) +
                  f" other/tx={row['other_over_transactional']:.2f}", flush=True)
            g.close()
    if a.out:
        with open(a.out, "w") as fo:
            for r in rows:
                fo.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
