"""One launch of a bench.py configuration, for ncu captures (GPU only).

    python tools/one_launch.py --config ht_c2 --mode hv [--launches 2] [--set k=v ...]

--config: a key of bench.CONFIGS, or "bank" (the headline: paired layout,
bench.py's headline variant).  The last launch is the one to profile
(`ncu --launch-skip <2*launches-1>` style filters, or -k stm_kernel -c 1
--launch-skip N).
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_cgo_xuwglgq14_b200 import build as B  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="bank")
    ap.add_argument("--mode", default="hv")
    ap.add_argument("--launches", type=int, default=2)
    ap.add_argument("--set", nargs="*", default=[], help="gstm_params_t overrides k=v")
    ap.add_argument("--paired", action="store_true", help="the paired layout (one lock per word)")
    a = ap.parse_args()
    B.build()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G
    kv = {k: int(v) for k, v in (s.split("=") for s in a.set)}
    if a.config == "bank":
        g = G.Gstm(bench.ACCOUNTS, bench.BITS, paired=True)
        g.set_workload_defaults("bank", n_words=bench.ACCOUNTS, prelock_vbv=0, k_lock=1, spin_cap=1, **kv)
        wl, T, K = "bank", bench.THREADS, bench.TX_PER_THREAD
    else:
        wl, words, bits, p, T, K, _, _ = bench.CONFIGS[a.config]
        if a.paired:
            bits = max(bits, (words - 1).bit_length())
        g = G.Gstm(words, bits, paired=a.paired)
        g.set_workload_defaults(wl, **dict(p, **kv))
    g.set_mode(a.mode)
    for k in range(a.launches):
        g.init_heap(wl)
        st = g.run(wl, T, K, 1 + k)
        n = max(1, st.commits + st.commits_ro)
        print(f"{a.config} {a.mode} launch {k}: {st.tx_per_s / 1e6:.1f} M tx/s, abort {st.abort_ratio:.3f}, "
              f"{st.elapsed_ms:.3f} ms; per tx: postval {st.postvalidations / n:.4f} vbv {st.vbv_runs / n:.4f} "
              f"spins {st.spins / n:.4f} lock_retries {st.lock_retries / n:.4f} ro {st.commits_ro / n:.3f} "
              f"serial {st.serial_runs}", flush=True)
    g.close()


if __name__ == "__main__":
    main()
