"""Tiny configurations of every kernel, for compute-sanitizer (memcheck,
racecheck, synccheck).  GPU only; run under the sanitizer:

    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_tiny.py

Every workload x mode x layout runs a few hundred transactions through the
C ABI and checks stamp-order replay against the oracle (so a sanitizer-clean
run is also a correct one).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import gpu_util as U  # noqa: E402

CASES = [
    ("ra", dict(n_reads=4, n_writes=4, n_words=64), 64, 2, 6),
    ("ra", dict(n_reads=3, n_words=16, ra_kind=1), 64, 2, 4),
    ("bank", dict(n_words=64), 96, 2, 6),
    ("ht", dict(ht_buckets=16, ht_key_range=64, ht_lookup_pct=50), 64, 2, 8),
    ("eb", dict(n_words=64, n_accesses=16), 64, 2, 6),
    ("km", dict(km_clusters=8, km_dims=4), 64, 2, 6),
]


def main():
    U.ensure_built()
    n = 0
    for wl, kw, T, K, bits in CASES:
        for mode in ("hv", "tbv", "hv_backoff", "vbv", "fgl", "cgl"):
            for paired in (False, True):
                if paired and wl in ("ht", "km"):
                    continue
                b = bits if not paired else max(bits, 7)
                g, gp, op, init = U.make(wl, T, K, b, mode=mode, paired=paired, **kw)
                U.run_verified(g, wl, op, init, T, K, 3)
                g.close()
                n += 1
    print(f"sanitize_tiny: {n} launches replayed", flush=True)


if __name__ == "__main__":
    main()
