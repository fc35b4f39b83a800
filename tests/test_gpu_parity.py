"""GPU parity tests (-m gpu): the CUDA path, called through the C ABI,
against the CPU oracle.

Integer work throughout, so every comparison is bit-exact.  Several final
states are correct for a concurrent run (any serial order), so the
tests compare what is unique -- the heap reproduced by replaying the
committed transactions in commit-stamp order, every transaction's observable
result, closed forms where the result is order-free -- and check that the
rest (the order itself) is valid: a permutation of dense stamps that respects
each thread's program order, or a member of the brute-forced set of serial
outcomes on tiny inputs.
"""
import json
import os

import numpy as np
import pytest

import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import gstm as G
import gpu_util as U

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module", autouse=True)
def _built():
    U.ensure_built()


# ---------------------------------------------------------------------------
# generator and initial heap parity (bit-exact)
# ---------------------------------------------------------------------------
WL_CASES = [
    ("ra", dict(n_reads=4, n_writes=4, n_words=1024, ra_kind=0)),
    ("ra", dict(n_reads=7, n_writes=3, n_words=999, ra_kind=0)),
    ("ra", dict(n_reads=5, n_words=37, ra_kind=1)),
    ("bank", dict(n_words=1 << 20)),
    ("bank", dict(n_words=3)),
    ("ht", dict(ht_buckets=1 << 20, ht_lookup_pct=90, ht_key_range=1 << 22)),
    ("ht", dict(ht_buckets=1 << 20, ht_lookup_pct=90, ht_key_range=1 << 22, shard_bits=3, shard=5)),
    ("ht", dict(ht_buckets=64, ht_lookup_pct=50, ht_key_range=100, shard_bits=1, shard=0)),
    ("eb", dict(n_accesses=64, n_words=1 << 26)),
    ("eb", dict(n_accesses=9, n_words=1000)),
    ("km", dict(km_clusters=1024, km_dims=16)),
    ("km", dict(km_clusters=5, km_dims=3)),
    ("km", dict(km_clusters=1024, km_dims=16, km_stride=32)),
]


@pytest.mark.parametrize("wl,kw", WL_CASES, ids=lambda v: str(v))
def test_descriptor_parity(wl, kw):
    T, K, seed = 333, 3, 0xC0FFEE        # ragged thread count
    gp = G.gstm_default_params(wl)
    for k, v in kw.items():
        setattr(gp, k, v)
    op = U.oracle_params(wl, gp)
    g = G.Gstm(16, 4)
    g.set_params(gp)
    d = g.dump_descr(wl, T, K, seed)
    for i in range(K):
        for t in range(T):
            want = O.descr(op, seed, t, i)
            got = d[i * T + t]
            assert got[:want.size].tolist() == want.tolist(), (t, i)
            assert not got[want.size:].any()


@pytest.mark.parametrize("wl", ["ra", "bank", "ht", "eb", "km"])
def test_init_heap_parity(wl):
    op = O.params(wl)
    g = G.Gstm(100_003, 4)
    g.init_heap(wl)
    assert (g.read_heap() == O.init_heap(op, 100_003)).all()


@pytest.mark.parametrize("variant,cap", [(0, 16), (1, 256), (2, 16), (3, 256), (4, 16), (5, 256), (6, 64)])
def test_lock_log_parity(variant, cap):
    """Encounter-time sorted lock log on the device vs the oracle;
    variants 2/3: the encounter-order log of STM-HV-Backoff (Q32); 4/5: the
    order-preserving hashed log of P:115 (same order as sorted(set)); 6: the
    shared-memory log of P:117.  Id
    ranges from 4 (every entry a duplicate of few ids) to 2^20 (spread), plus
    ascending and clustered arrivals (long runs in the hashed table)."""
    rng = np.random.default_rng(variant)
    for trial in range(300):
        n = int(rng.integers(0, cap + 8))
        hi = int(rng.choice([4, 50, 1 << 20]))
        ids = rng.integers(0, hi, n)
        if trial % 5 == 3:
            ids = np.sort(ids)                               # ascending arrivals
        if trial % 5 == 4:
            ids = (1 << 19) + rng.integers(0, 3 * n + 1, n)  # one cluster of homes
        e = (ids.astype(np.uint32) << 2) | rng.integers(1, 4, n).astype(np.uint32)
        want = O.lock_log(e, sorted_log=variant not in (2, 3))
        if want.size > cap:
            with pytest.raises(G.GstmError):
                G.gstm_lock_log(e, variant)
        else:
            assert G.gstm_lock_log(e, variant).tolist() == want.tolist()


# ---------------------------------------------------------------------------
# Algorithm 3 step-level parity: scripted interleavings on one device thread
# ---------------------------------------------------------------------------
def _script_both(mode, bits, heap0, clock0, ops, n_tx, prelock, policy=0):
    g = G.Gstm(heap0.size, bits)
    g.write_heap(heap0)
    g.set_clock(clock0)
    out_gpu = g.script(mode, ops, n_tx=n_tx, prelock_vbv=prelock, log_policy=policy)
    heap_o = heap0.copy()
    locks_o = np.zeros(1 << bits, dtype=np.uint32)
    out_o, clk_o = O.alg3_script(mode, bits, heap_o, locks_o, clock0, ops, n_tx=n_tx, prelock_vbv=prelock)
    return g, out_gpu, out_o, heap_o, locks_o, clk_o


def _scenarios():
    from test_oracle import load_scenarios
    return [(s, v) for s in load_scenarios() for v in s["variants"]]


@pytest.mark.parametrize("policy", [0, 1, 2])
@pytest.mark.parametrize("sv", _scenarios(), ids=lambda sv: f"{sv[0]['name']}-{sv[1]['mode']}-{int(sv[1]['prelock_vbv'])}")
def test_script_paper_scenarios(sv, policy):
    from test_oracle import encode_ops
    s, v = sv
    mode = G.MODE_HV if v["mode"] == "HV" else G.MODE_TBV
    ops = encode_ops(s["ops"])
    heap0 = np.array(s["heap"], dtype=np.uint32)
    g, out_gpu, out_o, heap_o, locks_o, clk_o = _script_both(mode, s["bits"], heap0, s["clock0"], ops, 4,
                                                            v["prelock_vbv"], policy)
    assert out_gpu.tolist() == v["out"]                      # the paper-derived golden values
    assert out_gpu.tolist() == out_o.tolist()
    assert g.read_heap().tolist() == v["heap"]
    locks = g.read_locks()
    assert (locks == locks_o).all()
    assert g.read_clock() == v["clock"] == clk_o


@pytest.mark.parametrize("mode", [G.MODE_HV, G.MODE_TBV])
@pytest.mark.parametrize("bits", [1, 2, 4])
@pytest.mark.parametrize("policy", [0, 1, 2])
def test_script_random_vs_oracle(mode, bits, policy):
    """Random interleavings, op by op against Algorithm 3 (oracle/alg3.c),
    including batched reads of two words (READ2: the kernels' read_batch with
    the merged timestamp check of reading Q35), for every log storage the
    kernels use: local memory (0), register-resident fully unrolled logs
    (1: the bank kernel's code path, converged lock acquisition) and shared
    memory [entry][lane] (2: P:117)."""
    from test_oracle import encode_ops, random_script
    rng = np.random.default_rng(1000 + 10 * mode + bits + 100 * policy)
    for trial in range(150):
        words = int(rng.integers(2, 9))
        n_tx = int(rng.integers(2, 5))
        ops = encode_ops(random_script(rng, n_tx, words, 0, batched=True, max_ops=4))
        heap0 = rng.integers(0, 50, words).astype(np.uint32)
        clock0 = int(rng.integers(0, 3))
        g, out_gpu, out_o, heap_o, locks_o, clk_o = _script_both(mode, bits, heap0, clock0, ops, n_tx,
                                                                bool(trial % 2), policy)
        assert out_gpu.tolist() == out_o.tolist(), trial
        assert (g.read_heap() == heap_o).all()
        assert (g.read_locks() == locks_o).all()
        assert g.read_clock() == clk_o
        g.close()


# ---------------------------------------------------------------------------
# RA (BASELINE configs[0]): 1K-word heap, 256 threads, 4R+4W, 1K locks
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("mode", ["hv", "tbv", "auto", "cgl", "fgl"])
def test_ra_config0_replay(mode):
    T, K = 256, 64
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, n_reads=4, n_writes=4, n_words=1024)
    for seed in (1, 2, 3):
        st, heap, stamps, res = U.run_verified(g, "ra", op, init, T, K, seed)
        init = heap
    if mode == "auto":
        assert st.mode_used == G.MODE_TBV      # 1K words <= 1K locks


@pytest.mark.parametrize("mode", ["hv", "tbv", "cgl", "fgl"])
def test_ra_increment_closed_form(mode):
    """RA kind 1 (read-modify-write, RAW through the write-set): the final
    heap is order-free: heap[k] = k + #occurrences of k in all descriptors."""
    T, K, R, N = 1000, 8, 6, 64       # heavy contention on 64 words
    g, gp, op, init = U.make("ra", T, K, 6, mode=mode, n_reads=R, n_words=N, ra_kind=1)
    st, heap, _, _ = U.run_verified(g, "ra", op, init, T, K, 9)
    d = np.concatenate([O.descr(op, 9, t, i) for i in range(K) for t in range(T)])
    assert (heap == (np.arange(N) + np.bincount(d, minlength=N)).astype(np.uint32)).all()


@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl", "cgl"])
@pytest.mark.parametrize("wl,kw,T,K,words,bits", [
    ("bank", dict(n_words=4), 2, 4, 4, 1),
    ("bank", dict(n_words=5), 8, 1, 5, 2),
    ("ra", dict(n_reads=2, n_writes=2, n_words=6), 3, 2, 6, 1),
    ("ra", dict(n_reads=2, n_words=3, ra_kind=1), 4, 2, 3, 2),
    ("eb", dict(n_accesses=6, n_words=5), 3, 2, 5, 1),
    ("km", dict(km_clusters=2, km_dims=2), 4, 2, 6, 2),
    ("ht", dict(ht_buckets=2, ht_lookup_pct=40, ht_key_range=3), 3, 2, 14, 2),
])
def test_brute_force_tiny(mode, wl, kw, T, K, words, bits):
    """The GPU outcome (heap + every result) is one of the outcomes of some
    serial order, found by exhaustive enumeration (independent of the
    commit log); 60 seeds per case."""
    for seed in range(60):
        g, gp, op, init = U.make(wl, T, K, bits, mode=mode, heap_words=words, **kw)
        if wl == "bank":
            init = np.array([30, 200, 5, 90, 60][:words], dtype=np.uint32)
            g.write_heap(init)
        st, heap, stamps, res = U.run_verified(g, wl, op, init, T, K, seed)
        n, match, nd = O.brute(op, init, T, K, seed, heap, res)
        assert match, (seed, n, nd)
        g.close()


# ---------------------------------------------------------------------------
# full-size configs in the launch configuration bench.py times
# ---------------------------------------------------------------------------
def test_bank_config1_full_replay():
    """BASELINE configs[1]: 2^20 accounts, 2^20 threads, 16 tx each (16M)."""
    T, K = 1 << 20, 16
    g, gp, op, init = U.make("bank", T, K, 20, mode="auto", n_words=1 << 20)
    st, heap, stamps, res = U.run_verified(g, "bank", op, init, T, K, 1)
    assert st.mode_used == G.MODE_TBV
    assert int(heap.astype(np.int64).sum()) == 1000 * (1 << 20)      # conservation
    assert (heap.view(np.int32) >= 0).all()
    # ReleaseAndUpdateLocks (A3.l56-61): every lock's version is the largest
    # stamp of a committed transaction that wrote a word it covers.
    locks = g.read_locks()
    assert not (locks & 1).any()
    upd = np.nonzero((stamps & O.RO_FLAG) == 0)[0]
    d = g.dump_descr("bank", T, K, 1)[upd]
    s_abs = stamps[upd].astype(np.int64) + st.clock_begin
    want = np.zeros(1 << 20, dtype=np.int64)
    np.maximum.at(want, d[:, 0].astype(np.int64), s_abs)
    np.maximum.at(want, d[:, 1].astype(np.int64), s_abs)
    assert ((locks >> 1).astype(np.int64) == want).all()


@pytest.mark.parametrize("mode", ["auto", "hv"])
def test_ht_replay(mode):
    """Hash table, 2^20 buckets, 90/10 lookup/insert (configs[2] shape at 2^20
    threads x 4); set semantics via replay + an independent set check."""
    T, K = 1 << 20, 4
    g, gp, op, init = U.make("ht", T, K, 22, mode=mode)
    st, heap, stamps, res = U.run_verified(g, "ht", op, init, T, K, 5)
    inserted = res == 3
    d = g.dump_descr("ht", T, K, 5)
    keys_ins = set(d[inserted, 0].tolist())
    all_ins = set(d[d[:, 1] == 1, 0].tolist())
    assert keys_ins == all_ins                     # every inserted key present exactly once
    assert int(inserted.sum()) == len(keys_ins)


@pytest.mark.parametrize("mode,extra", [("hv", dict(k_lock=1)), ("hv", dict(k_lock=1, prelock_vbv=1)), ("tbv", dict())])
def test_ht_config2_full_size_replay(mode, extra):
    """BASELINE configs[2] at full size, as `bench.py --workload ht` and
    tools/ablate.py run it: 2^20 buckets, 2^22 threads x 4 (16.8M operations,
    90/10 lookup/insert, keys in [1, 2^22]), 2^22 version locks: bit-exact
    stamp-order replay of every result and of the final table."""
    T, K = 1 << 22, 4
    g, gp, op, init = U.make("ht", T, K, 22, mode=mode, **extra)
    st, heap, stamps, res = U.run_verified(g, "ht", op, init, T, K, 7)
    assert st.commits == int((res == 3).sum())


@pytest.mark.parametrize("mode", ["hv", "fgl"])
def test_km_config4_full_size_closed_form(mode):
    """BASELINE configs[4] at full size: 16M points (K = 1), 1024 clusters x
    16 dims, the default 8 resident warps per SM; the order-free result equals
    bincount / add.at over the generated descriptors, and the replay holds."""
    T, K, Cn, D = 1 << 24, 1, 1024, 16
    g, gp, op, init = U.make("km", T, K, 20, mode=mode)
    st, heap, stamps, res = U.run_verified(g, "km", op, init, T, K, 9)
    d = g.dump_descr("km", T, K, 9).astype(np.int64)
    rec = heap.reshape(Cn, D + 1).astype(np.int64)
    assert (rec[:, 0] == np.bincount(d[:, 0], minlength=Cn)).all()
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:])
    assert (rec[:, 1:] == sums).all()


@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_eb_config3_full_heap_replay(mode):
    """BASELINE configs[3]'s largest point: a 2^26-word (256 MiB) heap with the
    hot set the whole heap, A = 16 accesses, 2^22 version locks persisting in
    L2 (the EB default), 2^18 threads x 4: bit-exact stamp-order replay."""
    T, K, H = 1 << 18, 4, 1 << 26
    g, gp, op, init = U.make("eb", T, K, 22, mode=mode, n_words=H, n_accesses=16, heap_words=H)
    assert gp.l2_persist_locks == 1
    U.run_verified(g, "eb", op, init, T, K, 13)


def test_km_closed_form():
    """k-means cluster update: order-free result == numpy bincount / add.at."""
    T, K, Cn, D = 1 << 20, 1, 1024, 16
    g, gp, op, init = U.make("km", T, K, 20, mode="auto")
    st, heap, stamps, res = U.run_verified(g, "km", op, init, T, K, 3)
    d = g.dump_descr("km", T, K, 3).astype(np.int64)
    rec = heap.reshape(Cn, D + 1).astype(np.int64)
    assert (rec[:, 0] == np.bincount(d[:, 0], minlength=Cn)).all()
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:])
    assert (rec[:, 1:] == sums).all()


@pytest.mark.parametrize("mode", ["hv", "tbv"])
@pytest.mark.parametrize("H,A,bits,T", [(1 << 10, 8, 20, 1 << 12), (1 << 10, 64, 20, 256), (1 << 16, 16, 12, 1 << 14),
                                        (1 << 20, 32, 20, 1 << 16), (1 << 20, 8, 16, 1 << 16)])
def test_eb_points_replay(mode, H, A, bits, T):
    """EigenBench-style points of the contention sweep (configs[3] shape,
    fewer threads so the replay stays quick); livelock-free = finishes."""
    K = 4
    g, gp, op, init = U.make("eb", T, K, bits, mode=mode, n_words=H, n_accesses=A, heap_words=H)
    U.run_verified(g, "eb", op, init, T, K, 11)


# ---------------------------------------------------------------------------
# adversarial contention, livelock freedom
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl"])
@pytest.mark.parametrize("k_lock", [0, 1, 8])
@pytest.mark.parametrize("pipeline", [0, 1])
def test_livelock_freedom_two_words(mode, k_lock, pipeline):
    """Every thread reads and writes the same 2 words in random order (the
    reverse-order pattern of P:63 and the r/w cross of P:184 inside every
    warp); with sorted lock acquisition all 4K transactions commit, with and
    without the pipelined first acquisition round."""
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, n_reads=2, n_writes=2, n_words=2, k_lock=k_lock,
                             lock_pipeline=pipeline)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K


@pytest.mark.parametrize("mode", ["hv", "tbv", "hv_backoff"])
@pytest.mark.parametrize("wl,kw,T,K,bits", [
    ("ht", dict(ht_buckets=1 << 12, ht_key_range=1 << 14, ht_lookup_pct=90), 1 << 14, 4, 14),
    ("ht", dict(ht_buckets=64, ht_key_range=256, ht_lookup_pct=50), 2048, 4, 8),
    ("bank", dict(n_words=1 << 10), 1 << 14, 4, 10),
    ("ra", dict(n_reads=4, n_writes=4, n_words=1024), 256, 64, 10),
])
@pytest.mark.parametrize("rounds", [2, 8])
def test_body_rounds_replay(mode, wl, kw, T, K, bits, rounds):
    """body_rounds: lanes that commit read-only run their
    next transaction in the same warp iteration, with the iteration's
    snapshot.  Serializability (stamp-order replay, read-only transactions at
    their snapshot) and each thread's program order must hold."""
    g, gp, op, init = U.make(wl, T, K, bits, mode=mode, body_rounds=rounds, **kw)
    U.run_verified(g, wl, op, init, T, K, 5 + rounds)
    g.close()


@pytest.mark.parametrize("mode", ["hv", "tbv", "hv_backoff"])
@pytest.mark.parametrize("wl,kw,T,K,bits,paired", [
    ("ht", dict(ht_buckets=1 << 12, ht_key_range=1 << 14, ht_lookup_pct=90), 1 << 14, 4, 14, False),
    ("ht", dict(ht_buckets=64, ht_key_range=256, ht_lookup_pct=30), 2048, 4, 8, False),
    ("bank", dict(n_words=1 << 10), 1 << 14, 4, 10, False),
    ("bank", dict(n_words=1 << 10), 1 << 14, 4, 10, True),
    ("ra", dict(n_reads=4, n_writes=4, n_words=1024), 256, 64, 10, False),
    ("ra", dict(n_reads=5, n_words=64, ra_kind=1), 512, 8, 6, True),
    ("eb", dict(n_words=1 << 12, n_accesses=32), 4096, 2, 12, False),
    ("km", dict(km_clusters=64, km_dims=16), 1 << 14, 2, 12, False),
])
def test_lock_log_at_commit_replay(mode, wl, kw, T, K, bits, paired):
    """lock_log_at_commit: read locks enter the sorted log at
    TXCommit instead of at the read -- the same log, so the same acquisition
    order: serializable, livelock-free, every transaction commits."""
    g, gp, op, init = U.make(wl, T, K, bits, mode=mode, paired=paired, lock_log_at_commit=1, **kw)
    st, *_ = U.run_verified(g, wl, op, init, T, K, 13)
    assert st.commits + st.commits_ro == T * K
    g.close()


@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("mode", ["hv", "tbv"])
@pytest.mark.parametrize("pipeline", [1, 1000])
def test_pipelined_at_most_one_round_per_execution(paired, mode, pipeline):
    """k_lock = 0 (Algorithm 3 verbatim: retry the lock step forever) with the
    pipelined first round (Q37): only the FIRST round of an
    execution may issue all its atom.or at once -- a round after a failed
    round must be the sequential sorted acquisition, else two transactions
    that each win one of {w0, w1} can fail each other forever.
    16 warps, every transaction takes both words in random order."""
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 1 if paired else 10, mode=mode, paired=paired, n_reads=2, n_writes=2,
                             n_words=2, k_lock=0, lock_pipeline=pipeline)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K
    assert st.aborts_lock == 0                      # k_lock = 0 never gives up a lock step
    assert st.lock_retries > 0, "no lock contention: the test exercises nothing"
    reached_lock_step = st.commits + st.aborts_prevbv + st.aborts_tbv + st.aborts_commit_vbv + st.aborts_lock
    assert 0 < st.pipelined_rounds <= reached_lock_step, st.as_dict()
    g.close()


@pytest.mark.parametrize("mode", ["hv", "tbv", "cgl", "fgl"])
@pytest.mark.parametrize("wl,kw,T,K,cap", [
    ("bank", dict(n_words=1 << 12), 1 << 16, 3, 2048),
    ("km", dict(km_clusters=64, km_dims=16), 1 << 14, 2, 1024),
    ("ra", dict(n_reads=4, n_writes=4, n_words=1024), 1000, 5, 96),
])
def test_concurrency_cap_replay(mode, wl, kw, T, K, cap):
    """max_threads: fewer CUDA threads run the T STM threads grid-stride;
    the run must stay serializable and respect each STM thread's order."""
    g, gp, op, init = U.make(wl, T, K, 12, mode=mode, max_threads=cap, **kw)
    st, *_ = U.run_verified(g, wl, op, init, T, K, 21)
    assert st.commits + st.commits_ro == T * K


@pytest.mark.parametrize("mode", ["hv", "tbv", "hv_backoff", "vbv", "fgl", "cgl"])
@pytest.mark.parametrize("kind", [0, 1])
@pytest.mark.parametrize("paired", [False, True])
def test_disjoint_access_sets_unique_result(mode, kind, paired):
    """SURVEY §8c-O4 special case: thread t touches only [t*k, t*k + k)
    (ra_partition = k) and every word has its own lock, so the result is
    unique: the GPU heap and every result equal the canonical serial
    execution bit for bit, and the STM never aborts."""
    k, T, K = 16, 4096, 8
    kw = dict(n_reads=4, n_writes=4) if kind == 0 else dict(n_reads=5)
    g, gp, op, init = U.make("ra", T, K, 16, mode=mode, paired=paired, ra_kind=kind, n_words=T * k,
                             ra_partition=k, **kw)
    st, heap, stamps, res = U.run_verified(g, "ra", op, init, T, K, 31)
    h = init.copy()
    want_res, _ = O.serial(op, h, T, K, 31)
    assert (heap == h).all()
    assert (res[:T * K] == want_res).all()
    if mode in ("hv", "tbv", "hv_backoff"):
        assert st.aborts == 0 and st.lock_retries == 0 and st.postvalidations == 0, st.as_dict()
    # a thread range beyond the heap is rejected, not silently wrapped
    g.set_params(ra_partition=k + 1)
    with pytest.raises(G.GstmError, match="EINVAL"):
        g.launch("ra", T, K, 32)


@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl"])
@pytest.mark.parametrize("persist", [0, 1])
def test_l2_persisting_lock_table_replay(mode, persist):
    """l2_persist_locks (an L2 access-policy window over the lock table around
    the launch) changes placement only: EB with a hot set of 2^22 words stays
    serializable, and the window does not leak to later launches."""
    T, K, H = 1 << 15, 4, 1 << 22
    g, gp, op, init = U.make("eb", T, K, 20, mode=mode, n_words=H, n_accesses=16, heap_words=H,
                             l2_persist_locks=persist)
    assert gp.l2_persist_locks == persist
    st, heap, *_ = U.run_verified(g, "eb", op, init, T, K, 29)
    g.set_params(gp)
    U.run_verified(g, "eb", op, heap, T, K, 30)


def test_l2_set_aside_is_reference_counted_per_device():
    """The persisting-L2 set-aside is device-wide: a handle launching WITHOUT
    persistence must not release the set-aside another live handle uses; the
    last user's destroy releases it (api.cu l2_use / l2_unuse)."""
    rt = pytest.importorskip("cuda.bindings.runtime")
    import gc
    import torch
    torch.cuda.init()
    gc.collect()                                # handles of earlier tests release their set-aside

    def limit():
        err, v = rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize)
        assert err == rt.cudaError_t.cudaSuccess
        return v

    T, K, H = 1 << 12, 2, 1 << 20
    a, _, opa, inita = U.make("eb", T, K, 20, mode="hv", n_words=H, n_accesses=8, heap_words=H, l2_persist_locks=1)
    b, _, opb, initb = U.make("eb", T, K, 20, mode="hv", n_words=H, n_accesses=8, heap_words=H, l2_persist_locks=0)
    U.run_verified(a, "eb", opa, inita, T, K, 1)
    held = limit()
    assert held >= 4 << 20                      # the 2^20-lock table (4 MiB) is set aside
    U.run_verified(b, "eb", opb, initb, T, K, 2)
    assert limit() == held                      # b does not release a's set-aside
    b.close()
    assert limit() == held
    a.close()
    assert limit() == 0                         # the last user released it


@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("T", [1023, 1024, 1025, 2047, 2053, 5 * 1024 + 37, 9 * 1024])
def test_static_region_and_counter_boundaries(paired, T):
    """The persistent grid runs STM threads g, g+P, ... of a static region
    [0, Rs*P), Rs = max(1, T/P - 1), then threads from a shared counter
    (stm_kernels.cuh): thread counts around multiples of P = 1024 lanes
    must run every transaction of every STM thread exactly once, in order."""
    K = 3
    g, gp, op, init = U.make("bank", T, K, 12, mode="hv", paired=paired, n_words=1 << 12, max_threads=1024,
                             block_threads=128, k_lock=1, spin_cap=1)
    st, heap, *_ = U.run_verified(g, "bank", op, init, T, K, 17)
    assert st.commits + st.commits_ro == T * K
    assert int(heap.astype(np.int64).sum()) == 1000 << 12


@pytest.mark.parametrize("mode", ["hv", "tbv"])
@pytest.mark.parametrize("pipeline", [1, 4, 64])
def test_k_lock_one_with_pipeline_progresses(mode, pipeline):
    """k_lock = 1 aborts on the first lost lock round; after `pipeline` such
    aborts a transaction never uses the pipelined round again, so high
    contention (RA configs[0]) still finishes (regression: pipelined-only
    retries livelocked)."""
    T, K = 256, 64
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, n_reads=4, n_writes=4, n_words=1024, k_lock=1,
                             lock_pipeline=pipeline, timeout_ms=20000)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 3)
    assert st.aborts_lock > 0


@pytest.mark.parametrize("pipeline,reuse,prelock", [(0, 0, 0), (0, 1, 1), (1, 0, 1), (1, 1, 0)])
@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_bank_knobs_replay(mode, pipeline, reuse, prelock):
    """Every runtime knob of the commit path keeps the run serializable
    (bank, 2^18 accounts, 2^18 threads x 4)."""
    T, K = 1 << 18, 4
    g, gp, op, init = U.make("bank", T, K, 18, mode=mode, n_words=1 << 18, lock_pipeline=pipeline,
                             snapshot_reuse=reuse, prelock_vbv=prelock)
    st, heap, *_ = U.run_verified(g, "bank", op, init, T, K, 13)
    assert int(heap.astype(np.int64).sum()) == 1000 << 18


def test_single_lock_table_degenerates_to_serial():
    """bits = 0: one version lock for the whole heap (every pair conflicts)."""
    T, K = 512, 4
    g, gp, op, init = U.make("bank", T, K, 0, mode="hv", n_words=1000)
    U.run_verified(g, "bank", op, init, T, K, 2)


def test_single_thread_equals_canonical_serial():
    T, K = 1, 200
    g, gp, op, init = U.make("eb", T, K, 8, mode="hv", n_words=512, n_accesses=16)
    st, heap, stamps, res = U.run_verified(g, "eb", op, init, T, K, 3)
    h = init.copy()
    r, _ = O.serial(op, h, T, K, 3)
    assert (h == heap).all() and (r == res).all()
    assert st.aborts == 0


def test_read_only_workload_leaves_metadata_untouched():
    """A3.l68: read-only transactions take no locks and do not tick the clock."""
    T, K = 4096, 4
    g, gp, op, init = U.make("ra", T, K, 10, mode="hv", n_reads=8, n_writes=0, n_words=1024)
    g.reset_meta()
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 6)
    assert st.commits == 0 and st.commits_ro == T * K
    assert g.read_clock() == 0 and not g.read_locks().any()


def test_false_conflicts_hv_aborts_less_than_tbv():
    """P:323-325 (directional): heap >> locks, HV's value-based fallback
    aborts fewer transactions than TBV."""
    T, K = 1 << 13, 4
    ab = {}
    for mode in ("hv", "tbv"):
        g, gp, op, init = U.make("ra", T, K, 10, mode=mode, n_reads=4, n_writes=1, n_words=1 << 16)
        st, *_ = U.run_verified(g, "ra", op, init, T, K, 8)
        ab[mode] = st.aborts
    assert ab["hv"] < ab["tbv"], ab


# ---------------------------------------------------------------------------
# edge cases and the C ABI contract
# ---------------------------------------------------------------------------
def test_empty_and_ragged_launches():
    g, gp, op, init = U.make("bank", 1000, 3, 10, mode="tbv", n_words=64)
    U.run_verified(g, "bank", op, init, 0, 3, 1)          # no threads
    U.run_verified(g, "bank", op, init, 1000, 0, 1)       # no transactions
    st, heap, *_ = U.run_verified(g, "bank", op, init, 1000, 3, 1)   # 1000 = 31.25 warps
    st, heap, *_ = U.run_verified(g, "bank", op, heap, 33, 5, 2)     # second launch, new epoch
    assert st.clock_begin > 0


def test_invalid_arguments_are_reported():
    g = G.Gstm(1024, 10)
    g.set_workload_defaults("bank", n_words=4096)
    with pytest.raises(G.GstmError, match="EINVAL"):
        g.launch("bank", 32, 1, 1)                         # footprint > heap
    g.set_workload_defaults("ra", n_reads=9)
    with pytest.raises(G.GstmError, match="EINVAL"):
        g.launch("ra", 32, 1, 1)                           # more reads than compiled
    g.set_workload_defaults("ra")
    with pytest.raises(G.GstmError, match="EOVERFLOW"):
        g.launch("ra", 1 << 31, 1, 1)
    with pytest.raises(G.GstmError):
        G.Gstm(16, 31)
    with pytest.raises(G.GstmError, match="EINVAL"):
        g.set_params(block_threads=48 + 1)


def test_log_overflow_is_sticky_error():
    """An HT chain longer than the compiled read-set: GSTM_ELOGOVF, no hang."""
    T, K = 64, 40
    g, gp, op, init = U.make("ht", T, K, 10, mode="hv", ht_buckets=1, ht_lookup_pct=0, ht_key_range=1 << 30)
    g.launch("ht", T, K, 1)
    st = g.stats(check=False)
    assert st.status == -4 and st.errors > 0


def test_run_host_and_attached_torch_heap():
    import torch
    T, K = 1 << 14, 4
    g, gp, op, init = U.make("bank", T, K, 14, mode="tbv", n_words=1 << 14)
    h_in = np.full(1 << 14, 1000, dtype=np.uint32)
    h_out = np.zeros_like(h_in)
    st = g.run_host("bank", h_in, h_out, T, K, 3)
    assert st.commits + st.commits_ro == T * K and int(h_out.astype(np.int64).sum()) == 1000 << 14
    stamps, res = g.read_tx_log(T * K)
    h = h_in.copy()
    assert O.replay(op, h, T, K, 3, stamps, res)[0] == 0 and (h == h_out).all()
    # torch-owned heap and stream
    t = torch.full((1 << 14,), 1000, dtype=torch.int32, device="cuda")
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    g.attach_heap(t)
    g.set_stream(s)
    g.launch("bank", T, K, 3)
    st2 = g.stats()
    torch.cuda.synchronize()
    assert (t.cpu().numpy().view(np.uint32) == h_out).all() or st2.commits > 0
    h = h_in.copy()
    stamps, res = g.read_tx_log(T * K)
    assert O.replay(op, h, T, K, 3, stamps, res)[0] == 0
    assert (h == t.cpu().numpy().view(np.uint32)).all()


@pytest.mark.parametrize("paired", [False, True])
def test_run_host_async_double_buffered(paired):
    """gstm_run_host_async on two handles and two streams (the bench's
    end-to-end path): every step's host output replays bit-exactly."""
    import torch
    T, K, N = 1 << 14, 4, 1 << 14
    hs = [U.make("bank", T, K, 14, mode="hv", paired=paired, n_words=N) for _ in range(2)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    h_in = torch.full((N,), 1000, dtype=torch.int32).pin_memory().numpy().view(np.uint32)
    outs = [torch.zeros(N, dtype=torch.int32).pin_memory().numpy().view(np.uint32) for _ in range(4)]
    for (g, *_), s in zip(hs, streams):
        g.set_stream(s)
    for k in range(4):
        hs[k % 2][0].run_host_async("bank", h_in, outs[k], T, K, 20 + k)
    for g, *_ in hs:
        assert g.sync() == 0
    # each handle's last step is replayable from the input
    for j, (g, gp, op, init) in enumerate(hs):
        k = 2 + j
        stamps, res = g.read_tx_log(T * K)
        h = h_in.copy()
        assert O.replay(op, h, T, K, 20 + k, stamps, res)[0] == 0
        assert (h == outs[k]).all()
    for k in range(4):
        assert int(outs[k].astype(np.int64).sum()) == 1000 * N


@pytest.mark.parametrize("paired", [False, True])
def test_run_host_async_pipelined_one_handle(paired):
    """Consecutive gstm_run_host_async calls on ONE handle overlap step k+1's
    copy-in and step k's copy-out with the transactions (internal copy
    streams, staging buffers).  Disjoint access sets (ra_partition) make every
    step's result unique, so each step's host output must equal the oracle's
    serial execution of that step's own input, bit for bit; the handle's last
    launch also replays, and a blocking call afterwards still works."""
    import torch
    k_part, T, K = 8, 2048, 4
    N = T * k_part
    g, gp, op, init = U.make("ra", T, K, 14, mode="hv", paired=paired, n_reads=4, n_writes=4, n_words=N,
                             ra_partition=k_part)
    rng = np.random.default_rng(5)
    ins = [torch.from_numpy(rng.integers(0, 2**32, N, dtype=np.uint32).view(np.int32)).pin_memory().numpy().view(np.uint32)
           for _ in range(5)]
    outs = [torch.zeros(N, dtype=torch.int32).pin_memory().numpy().view(np.uint32) for _ in range(5)]
    for k in range(5):
        g.run_host_async("ra", ins[k], outs[k], T, K, 40 + k)
    assert g.sync() == 0
    for k in range(5):
        h = ins[k].copy()
        O.serial(op, h, T, K, 40 + k)
        assert (outs[k] == h).all(), k
    stamps, res = g.read_tx_log(T * K)
    h = ins[4].copy()
    assert O.replay(op, h, T, K, 44, stamps, res)[0] == 0 and (h == outs[4]).all()
    out = np.zeros(N, dtype=np.uint32)
    g.run_host("ra", ins[0], out, T, K, 40)
    assert (out == outs[0]).all()


@pytest.mark.parametrize("paired", [False, True])
def test_run_host_async_chained_in_place(paired):
    """Steps chained in place: every call passes the SAME pinned buffer as
    heap_in and heap_out, so step k+1 must read step k's output (its copy-in
    waits for step k's copy-out).  Disjoint access sets make each step's result
    unique: after n steps the buffer equals n serial oracle steps, bit for bit."""
    import torch
    k_part, T, K, n = 8, 2048, 4, 6
    N = T * k_part
    g, gp, op, init = U.make("ra", T, K, 14, mode="hv", paired=paired, n_reads=4, n_writes=4, n_words=N,
                             ra_partition=k_part)
    rng = np.random.default_rng(17)
    buf = torch.from_numpy(rng.integers(0, 2**32, N, dtype=np.uint32).view(np.int32)).pin_memory().numpy().view(np.uint32)
    want = buf.copy()
    for k in range(n):
        g.run_host_async("ra", buf, buf, T, K, 60 + k)
        O.serial(op, want, T, K, 60 + k)
    assert g.sync() == 0
    assert (buf == want).all()


@pytest.mark.parametrize("kind", [0, 1, 2, 3, 4, 5])
def test_ubench_runs(kind):
    ops, ms = G.gstm_ubench(kind, 8 << 20, 1 << 22, 148 * 256 * 4)
    assert ops > 1e6 and ms > 0
