"""GPU parity tests of the PAIRED layout (-m gpu): every word stored next to
its version lock in one 8-byte slot (GSTM_CREATE_PAIRED).

Same oracle and same checks as test_gpu_parity.py: Algorithm 3 step parity
on scripts, bit-exact stamp-order replay, brute force on tiny inputs,
closed forms, lock-version invariant.  The paired layout needs one lock per
word (2^bits >= heap words), so the false-conflict cases stay with the split
layout.
"""
import numpy as np
import pytest

import gpu_util as U
import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import gstm as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _built():
    U.ensure_built()


def _script_both(mode, bits, heap0, clock0, ops, n_tx, prelock, policy=0):
    g = G.Gstm(heap0.size, bits, paired=True)
    g.write_heap(heap0)
    g.set_clock(clock0)
    out_gpu = g.script(mode, ops, n_tx=n_tx, prelock_vbv=prelock, log_policy=policy)
    heap_o = heap0.copy()
    locks_o = np.zeros(1 << bits, dtype=np.uint32)
    out_o, clk_o = O.alg3_script(mode, bits, heap_o, locks_o, clock0, ops, n_tx=n_tx, prelock_vbv=prelock)
    return g, out_gpu, out_o, heap_o, locks_o, clk_o


def _scenarios():
    from test_oracle import load_scenarios
    return [(s, v) for s in load_scenarios() for v in s["variants"] if (1 << s["bits"]) >= len(s["heap"])]


@pytest.mark.parametrize("sv", _scenarios(), ids=lambda sv: f"{sv[0]['name']}-{sv[1]['mode']}-{int(sv[1]['prelock_vbv'])}")
def test_paired_script_paper_scenarios(sv):
    from test_oracle import encode_ops
    s, v = sv
    mode = G.MODE_HV if v["mode"] == "HV" else G.MODE_TBV
    heap0 = np.array(s["heap"], dtype=np.uint32)
    g, out_gpu, out_o, heap_o, locks_o, clk_o = _script_both(mode, s["bits"], heap0, s["clock0"],
                                                            encode_ops(s["ops"]), 4, v["prelock_vbv"])
    assert out_gpu.tolist() == v["out"] == out_o.tolist()
    assert g.read_heap().tolist() == v["heap"]
    assert (g.read_locks() == locks_o).all()
    assert g.read_clock() == v["clock"] == clk_o


@pytest.mark.parametrize("mode", [G.MODE_HV, G.MODE_TBV])
@pytest.mark.parametrize("policy", [0, 1, 2])
def test_paired_script_random_vs_oracle(mode, policy):
    """As the split-layout test: local, register-resident and shared-memory
    logs, with batched reads (READ2, Q35)."""
    from test_oracle import encode_ops, random_script
    rng = np.random.default_rng(77 + mode + 10 * policy)
    for trial in range(200):
        bits = 4
        words = int(rng.integers(2, 17))
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


@pytest.mark.parametrize("mode", ["hv", "tbv", "auto", "cgl", "fgl"])
def test_paired_ra_config0_replay(mode):
    T, K = 256, 64
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, paired=True, n_reads=4, n_writes=4, n_words=1024)
    for seed in (1, 2):
        st, heap, *_ = U.run_verified(g, "ra", op, init, T, K, seed)
        init = heap


@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_paired_bank_config1_full_replay(mode):
    T, K = 1 << 20, 16
    g, gp, op, init = U.make("bank", T, K, 20, mode=mode, paired=True, n_words=1 << 20)
    st, heap, stamps, res = U.run_verified(g, "bank", op, init, T, K, 1)
    assert int(heap.astype(np.int64).sum()) == 1000 * (1 << 20)
    locks = g.read_locks()
    assert not (locks & 1).any()
    upd = np.nonzero((stamps & O.RO_FLAG) == 0)[0]
    d = g.dump_descr("bank", T, K, 1)[upd]
    s_abs = stamps[upd].astype(np.int64) + st.clock_begin
    want = np.zeros(1 << 20, dtype=np.int64)
    np.maximum.at(want, d[:, 0].astype(np.int64), s_abs)
    np.maximum.at(want, d[:, 1].astype(np.int64), s_abs)
    assert ((locks >> 1).astype(np.int64) == want).all()


def test_paired_bank_headline_variant_full_replay():
    """The exact configuration bench.py times (BASELINE configs[1] at full
    size): STM-HV, paired layout, no pre-lock VBV, k_lock = 1, spin_cap = 1,
    the bank defaults (first lock round pipelined for 4 executions, 16
    resident warps per SM); two launches on one handle (the second starts a
    new clock epoch on the first one's heap)."""
    T, K = 1 << 20, 16
    g, gp, op, init = U.make("bank", T, K, 20, mode="hv", paired=True, n_words=1 << 20, prelock_vbv=0, k_lock=1,
                             spin_cap=1)
    assert gp.lock_pipeline == 4 and gp.max_threads == 0
    for seed in (1, 2):
        st, heap, stamps, res = U.run_verified(g, "bank", op, init, T, K, seed)
        assert int(heap.astype(np.int64).sum()) == 1000 * (1 << 20)
        assert (heap.view(np.int32) >= 0).all()
        locks = g.read_locks()
        assert not (locks & 1).any()
        upd = np.nonzero((stamps & O.RO_FLAG) == 0)[0]
        d = g.dump_descr("bank", T, K, seed)[upd]
        s_abs = stamps[upd].astype(np.int64) + st.clock_begin
        want = np.zeros(1 << 20, dtype=np.int64)
        np.maximum.at(want, d[:, 0].astype(np.int64), s_abs)
        np.maximum.at(want, d[:, 1].astype(np.int64), s_abs)
        touched = want > 0
        assert ((locks >> 1).astype(np.int64)[touched] == want[touched]).all()
        init = heap


@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl", "cgl"])
@pytest.mark.parametrize("wl,kw,T,K,words,bits", [
    ("bank", dict(n_words=4), 2, 4, 4, 2),
    ("bank", dict(n_words=5), 8, 1, 5, 3),
    ("ra", dict(n_reads=2, n_writes=2, n_words=6), 3, 2, 6, 3),
    ("ra", dict(n_reads=2, n_words=3, ra_kind=1), 4, 2, 3, 2),
    ("eb", dict(n_accesses=6, n_words=5), 3, 2, 5, 3),
    ("km", dict(km_clusters=2, km_dims=2), 4, 2, 6, 3),
    ("ht", dict(ht_buckets=2, ht_lookup_pct=40, ht_key_range=3), 3, 2, 14, 4),
])
def test_paired_brute_force_tiny(mode, wl, kw, T, K, words, bits):
    for seed in range(40):
        g, gp, op, init = U.make(wl, T, K, bits, mode=mode, heap_words=words, paired=True, **kw)
        if wl == "bank":
            init = np.array([30, 200, 5, 90, 60][:words], dtype=np.uint32)
            g.write_heap(init)
        st, heap, stamps, res = U.run_verified(g, wl, op, init, T, K, seed)
        n, match, nd = O.brute(op, init, T, K, seed, heap, res)
        assert match, (seed, n, nd)
        g.close()


@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_paired_ht_km_eb(mode):
    T, K = 1 << 18, 4
    g, gp, op, init = U.make("ht", T, K, 22, mode=mode, paired=True)
    U.run_verified(g, "ht", op, init, T, K, 5)
    g, gp, op, init = U.make("km", 1 << 18, 1, 15, mode=mode, paired=True)
    st, heap, *_ = U.run_verified(g, "km", op, init, 1 << 18, 1, 3)
    d = g.dump_descr("km", 1 << 18, 1, 3).astype(np.int64)
    assert (heap.reshape(1024, 17)[:, 0] == np.bincount(d[:, 0], minlength=1024)).all()
    for H, A, Tt in [(1 << 10, 16, 1 << 10), (1 << 20, 32, 1 << 15)]:
        g, gp, op, init = U.make("eb", Tt, 4, max(10, H.bit_length() - 1), mode=mode, paired=True, n_words=H,
                                 n_accesses=A, heap_words=H)
        U.run_verified(g, "eb", op, init, Tt, 4, 11)


@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl"])
@pytest.mark.parametrize("pipeline,spin_cap", [(0, 0), (1, 0), (4, 1), (1000, 1)])
def test_paired_livelock_two_words(mode, pipeline, spin_cap):
    # lock_pipeline = N: a transaction pipelines the first lock round of its
    # first N executions; progress must hold for any finite N (stm_kernels.cuh)
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 1, mode=mode, paired=True, n_reads=2, n_writes=2, n_words=2,
                             lock_pipeline=pipeline, k_lock=1, spin_cap=spin_cap)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K


@pytest.mark.parametrize("pipeline,reuse,prelock", [(0, 0, 0), (1, 1, 1), (1, 0, 0)])
def test_paired_bank_knobs(pipeline, reuse, prelock):
    T, K = 1 << 18, 4
    g, gp, op, init = U.make("bank", T, K, 18, mode="hv", paired=True, n_words=1 << 18, lock_pipeline=pipeline,
                             snapshot_reuse=reuse, prelock_vbv=prelock, max_threads=1 << 16)
    st, heap, *_ = U.run_verified(g, "bank", op, init, T, K, 13)
    assert int(heap.astype(np.int64).sum()) == 1000 << 18


def test_paired_contract():
    with pytest.raises(G.GstmError, match="paired"):
        G.Gstm(1025, 10, paired=True)          # more words than locks
    g = G.Gstm(1024, 10, paired=True)
    import torch
    with pytest.raises(G.GstmError):
        g.attach_heap(torch.zeros(1024, dtype=torch.int32, device="cuda"))
    g.set_workload_defaults("ra", n_words=1024, lock_shift=2)
    with pytest.raises(G.GstmError, match="EINVAL"):
        g.launch("ra", 32, 1, 1)
    # host round trip and run_host through the packing kernels
    h = np.arange(1024, dtype=np.uint32) * 7
    g.write_heap(h)
    assert (g.read_heap() == h).all()
    assert (g.read_heap(10, offset=100) == h[100:110]).all()
    g.set_workload_defaults("ra", n_words=1024, verify=1)
    out = np.zeros_like(h)
    st = g.run_host("ra", h, out, 64, 8, 5)
    stamps, res = g.read_tx_log(64 * 8)
    hh = h.copy()
    op = O.params("ra", n_reads=4, n_writes=4, n_words=1024)
    assert O.replay(op, hh, 64, 8, 5, stamps, res)[0] == 0 and (hh == out).all()
