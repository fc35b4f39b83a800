"""Helpers shared by the -m gpu tests: run the CUDA path through the C ABI and
check it against the CPU oracle (which it never imports itself)."""
from __future__ import annotations

import numpy as np

import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import build as B
from paper_conf_cgo_xuwglgq14_b200 import gstm as G

WL_FIELDS = ["n_reads", "n_writes", "ra_kind", "n_words", "n_accesses", "ht_buckets", "ht_lookup_pct",
             "ht_key_range", "km_clusters", "km_dims", "shard_bits", "shard", "km_stride", "km_assign", "ra_partition"]


def ensure_built():
    B.build()


def oracle_params(wl: str, gp: G.gstm_params_t) -> O.Params:
    return O.params(wl, **{f: getattr(gp, f) for f in WL_FIELDS})


def make(wl: str, T: int, K: int, bits: int, mode="auto", heap_words=None, paired=False, flavour="", **kw):
    """Create a handle sized for the workload, with verify on and the
    workload's device-side initial heap; returns (g, gp, op, init).
    paired=True uses the GSTM_CREATE_PAIRED layout; flavour selects a build
    flavour of the library (build.FLAVOURS)."""
    gp = G.gstm_default_params(wl)
    for k, v in kw.items():
        setattr(gp, k, int(v))
    gp.verify = 1
    op = oracle_params(wl, gp)
    words = O.footprint(op, T, K) if heap_words is None else heap_words
    if flavour:
        B.build(flavour=flavour)
    g = G.Gstm(words, bits, paired=paired, flavour=flavour)
    g.set_params(gp)
    g.set_mode(mode)
    g.init_heap(wl)
    init = O.init_heap(op, words)
    return g, gp, op, init


def run_verified(g: G.Gstm, wl: str, op: O.Params, init: np.ndarray, T: int, K: int, seed: int,
                 expect_status: int = 0):
    """Launch, then check: every tx committed exactly once, stamps dense,
    stamp-order replay reproduces the heap bit-exactly and every result."""
    g.launch(wl, T, K, seed)
    st = g.stats(check=False)
    assert st.status == expect_status, (st.status, G.last_error())
    n = T * K
    heap = g.read_heap(init.size)
    if n == 0:
        assert (heap == init).all()
        return st, heap, None, None
    stamps, results = g.read_tx_log(n)
    assert st.commits + st.commits_ro == n, st.as_dict()
    assert st.clock_end - st.clock_begin == st.commits
    upd = (stamps & O.RO_FLAG) == 0
    assert int(upd.sum()) == st.commits
    h = init.copy()
    rc, msg = O.replay(op, h, T, K, seed, stamps, results)
    assert rc == 0, msg
    assert (h == heap).all(), f"heap mismatch at {np.nonzero(h != heap)[0][:10]}"
    return st, heap, stamps, results
