"""GPU parity tests (-m gpu) of the library's build flavours (build.FLAVOURS):

* "strict": every fence a formal reading of the PTX memory model asks for
  (GSTM_STRICT_FENCES: a release fence after lock acquisition, A3.l79; an
  acq_rel clock increment and a release fence before the lock-release stores,
  DESIGN.md §6.2) -- the product build relies on L2 being the single
  coherence point instead; both must be serializable.
* "hlog": the order-preserving hashed lock log of P:115 in
  every local-memory-log kernel (RA, HT, EB, KM).
* "phase": the Figure 5 per-phase cycle counters:
  the instrumented kernel must stay serializable and account for its time.
* "smem": the bank, RA and KM logs in shared memory, [entry][lane] per warp
  (DESIGN.md §6.13).

Same checks as test_gpu_parity.py: stamp-order replay bit-exact, brute force
on tiny inputs, closed forms, livelock freedom on two words.
"""
import numpy as np
import pytest

import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import build as B
from paper_conf_cgo_xuwglgq14_b200 import gstm as G
import gpu_util as U

pytestmark = pytest.mark.gpu
FLAVOURS = ["strict", "hlog", "phase", "smem"]


@pytest.fixture(scope="module", autouse=True)
def _built():
    for f in [""] + FLAVOURS:
        B.build(flavour=f)


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("mode", ["hv", "tbv", "hv_backoff", "fgl", "cgl"])
def test_ra_config0_replay(flavour, mode):
    T, K = 256, 64
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, n_reads=4, n_writes=4, n_words=1024, flavour=flavour)
    for seed in (1, 2):
        st, heap, *_ = U.run_verified(g, "ra", op, init, T, K, seed)
        init = heap
    g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("paired", [False, True])
def test_bank_full_replay(flavour, paired):
    """BASELINE configs[1] at full size (2^20 accounts, 2^20 x 16), in the
    launch configuration bench.py times (HV, k_lock 1, spin_cap 1) on the
    paired layout, the paper's defaults on the split one."""
    T, K = 1 << 20, 16
    kw = dict(k_lock=1, spin_cap=1, prelock_vbv=0) if paired else {}
    g, gp, op, init = U.make("bank", T, K, 20, mode="hv", n_words=1 << 20, paired=paired, flavour=flavour, **kw)
    st, heap, *_ = U.run_verified(g, "bank", op, init, T, K, 7)
    assert int(heap.astype(np.int64).sum()) == 1000 << 20
    locks = g.read_locks()
    assert not (locks & 1).any()
    g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_ht_replay(flavour, mode):
    T, K = 1 << 18, 4
    g, gp, op, init = U.make("ht", T, K, 20, mode=mode, ht_buckets=1 << 16, ht_key_range=1 << 18, flavour=flavour)
    U.run_verified(g, "ht", op, init, T, K, 3)
    g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("H,A,bits,T", [(1 << 10, 16, 10, 1 << 10), (1 << 20, 32, 20, 1 << 15),
                                        (1 << 22, 64, 22, 1 << 14)])
def test_eb_points_replay(flavour, H, A, bits, T):
    g, gp, op, init = U.make("eb", T, 4, bits, mode="hv", n_words=H, n_accesses=A, heap_words=H, flavour=flavour)
    U.run_verified(g, "eb", op, init, T, 4, 11)
    g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_km_closed_form(flavour, mode):
    T, K = 1 << 16, 2
    g, gp, op, init = U.make("km", T, K, 16, mode=mode, flavour=flavour)
    st, heap, *_ = U.run_verified(g, "km", op, init, T, K, 5)
    d = g.dump_descr("km", T, K, 5).astype(np.int64)
    rec = heap.reshape(1024, 17).astype(np.int64)
    assert (rec[:, 0] == np.bincount(d[:, 0], minlength=1024)).all()
    sums = np.zeros((1024, 16), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:17])
    assert (rec[:, 1:] == sums).all()
    g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("mode", ["hv", "tbv"])
@pytest.mark.parametrize("wl,kw,T,K,words,bits", [
    ("bank", dict(n_words=4), 2, 4, 4, 1),
    ("ra", dict(n_reads=2, n_writes=2, n_words=6), 3, 2, 6, 1),
    ("eb", dict(n_accesses=6, n_words=5), 3, 2, 5, 1),
    ("km", dict(km_clusters=2, km_dims=2), 4, 2, 6, 2),
    ("ht", dict(ht_buckets=2, ht_lookup_pct=40, ht_key_range=3), 3, 2, 14, 2),
])
def test_brute_force_tiny(flavour, mode, wl, kw, T, K, words, bits):
    for seed in range(30):
        g, gp, op, init = U.make(wl, T, K, bits, mode=mode, heap_words=words, flavour=flavour, **kw)
        if wl == "bank":
            init = np.array([30, 200, 5, 90][:words], dtype=np.uint32)
            g.write_heap(init)
        st, heap, stamps, res = U.run_verified(g, wl, op, init, T, K, seed)
        n, match, nd = O.brute(op, init, T, K, seed, heap, res)
        assert match, (seed, n, nd)
        g.close()


@pytest.mark.parametrize("flavour", FLAVOURS)
@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("k_lock,pipeline", [(0, 1), (1, 4), (8, 0)])
def test_livelock_two_words(flavour, paired, k_lock, pipeline):
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 1 if paired else 10, mode="hv", paired=paired, n_reads=2, n_writes=2,
                             n_words=2, k_lock=k_lock, lock_pipeline=pipeline, flavour=flavour)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K
    reached = st.commits + st.aborts_prevbv + st.aborts_tbv + st.aborts_commit_vbv + st.aborts_lock
    assert st.pipelined_rounds <= reached
    g.close()


@pytest.mark.parametrize("variant,cap", [(4, 16), (5, 256)])
def test_hashed_lock_log_parity(variant, cap):
    """The hashed log's order is the sorted log's: sorted(set(ids))
    with the rd/wr bits OR-ed (Q4), capacity overflow reported."""
    rng = np.random.default_rng(100 + variant)
    for trial in range(200):
        n = int(rng.integers(0, cap + 8))
        ids = rng.integers(0, int(rng.choice([3, 40, 1 << 20])), n)
        e = (ids.astype(np.uint32) << 2) | rng.integers(1, 4, n).astype(np.uint32)
        want = O.lock_log(e)
        if want.size > cap:
            with pytest.raises(G.GstmError):
                G.gstm_lock_log(e, variant)
        else:
            assert G.gstm_lock_log(e, variant).tolist() == want.tolist()


@pytest.mark.parametrize("wl,kw,T,K,bits", [
    ("km", dict(), 1 << 16, 2, 16),
    ("bank", dict(n_words=1 << 16), 1 << 16, 4, 16),
    ("ht", dict(ht_buckets=1 << 16, ht_key_range=1 << 18), 1 << 16, 4, 18),
])
def test_phase_build_accounts_its_time(wl, kw, T, K, bits):
    """The instrumented build (Figure 5 categories) replays
    bit-exactly and its per-warp phase cycles are non-negative and cover the
    kernel: every category a committed transaction passes through is > 0."""
    g, gp, op, init = U.make(wl, T, K, bits, mode="hv", flavour="phase", **kw)
    g.reset_stats_total()
    U.run_verified(g, wl, op, init, T, K, 9)
    ph = g.phase_cycles()
    assert all(v >= 0 for v in ph.values())
    for k in ("native", "init", "buffering", "consistency", "locks", "commit", "other"):
        assert ph[k] > 0, (k, ph)
    g.close()
