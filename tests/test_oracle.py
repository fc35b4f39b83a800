"""Pins for the CPU oracle (-m "not gpu").

Each test ties an oracle function to something other than itself: published
SplitMix64 vectors, exact integer identities, hand-derived fixtures
(tests/golden/), closed forms that hold in any serial order, library routines
(numpy bincount / add.at, Python sets and sorted()), multinomial counts, and
an independent formalisation of opacity applied to random scripts.
"""
import itertools
import json
import math
import os

import numpy as np
import pytest

import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# --------------------------------------------------------------------------
# generator (gen.c)
# --------------------------------------------------------------------------
def test_splitmix64_published_vectors():
    n = 0
    with open(os.path.join(GOLD, "splitmix64_vectors.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            x, k, out = line.split()
            assert O.draw(int(x, 0), int(k, 0)) == int(out, 0), line
            n += 1
    assert n == 8
    # splitmix64(x) is the first output of the stream with state x
    assert O.splitmix64(0) == 0xE220A8397B1DCDAF


def test_bounded_identities():
    M = (1 << 64) - 1
    for n in [1, 2, 3, 7, 100, 1 << 20, 12345678901, (1 << 63) + 5]:
        assert O.bounded(0, n) == 0
        assert O.bounded(M, n) == n - 1
        assert O.bounded(1 << 63, n) == n // 2
    for k in range(1, 64):
        for r in [1, 0xDEADBEEFCAFEBABE, M, 1 << 40]:
            assert O.bounded(r, 1 << k) == r >> (64 - k)     # multiply by 2^k = shift
    rng = np.random.default_rng(1)
    rs = sorted(int(v) for v in rng.integers(0, 1 << 63, 200, dtype=np.uint64) * 2)
    for n in [10, 1000, 99991]:
        vals = [O.bounded(r, n) for r in rs]
        assert vals == sorted(vals)                           # monotone in r
        assert all(0 <= v < n for v in vals)


def test_generator_uniformity_chi_square():
    # bucket 16: expected 4096 per cell; chi2 with 15 dof, p=1e-6 bound ~ 52
    counts = np.zeros(16)
    for t in range(256):
        for i in range(256):
            counts[O.bounded(O.draw(O.txkey(3, t, i), 0), 16)] += 1
    e = counts.sum() / 16
    chi2 = float(((counts - e) ** 2 / e).sum())
    assert chi2 < 52, chi2


def test_descriptor_ranges():
    pb = O.params("bank", n_words=1000)
    pk = O.params("km", km_clusters=1024, km_dims=16)
    ph = O.params("ht", ht_buckets=1 << 10, ht_lookup_pct=90, ht_key_range=1 << 22)
    ins = 0
    for t in range(64):
        for i in range(16):
            a, b, amt = O.descr(pb, 9, t, i)
            assert a != b and a < 1000 and b < 1000 and 1 <= amt <= 100
            d = O.descr(pk, 9, t, i)
            assert d[0] < 1024 and d.size == 17 and d[1:].max() <= 255
            key, is_ins, bucket = O.descr(ph, 9, t, i)
            assert 1 <= key <= 1 << 22 and bucket < 1 << 10
            ins += int(is_ins)
    assert 40 < ins < 170   # ~10% of 1024 inserts
    # re-execution of an aborted transaction regenerates it
    assert list(O.descr(pb, 9, 5, 3)) == list(O.descr(pb, 9, 5, 3))


# --------------------------------------------------------------------------
# serial executor (serial.c)
# --------------------------------------------------------------------------
def _load_fixtures():
    with open(os.path.join(GOLD, "serial_fixtures.json")) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _load_fixtures(), ids=lambda c: c["name"])
def test_serial_hand_fixtures(case):
    kw = dict(case["params"])
    wl = kw.pop("workload")
    p = O.params(wl, **kw)
    T, K, seed = case["T"], case["K"], case["seed"]
    for txid, d in case["descr"].items():
        txid = int(txid)
        assert list(map(int, O.descr(p, seed, txid % T, txid // T))) == d
    heap = np.array(case["init"], dtype=np.uint32)
    res, upd = O.serial(p, heap, T, K, seed)
    assert heap.tolist() == case["heap"]
    assert res.tolist() == case["results"]
    assert upd.astype(int).tolist() == case["is_update"]


@pytest.mark.parametrize("seed", [1, 2, 3, 77])
def test_bank_conservation_and_nonnegative(seed):
    p = O.params("bank", n_words=64)
    heap = np.full(64, 30, dtype=np.uint32)        # small balances: many skips
    res, upd = O.serial(p, heap, 32, 16, seed)
    assert int(heap.astype(np.int64).sum()) == 64 * 30
    assert (heap.view(np.int32) >= 0).all()
    assert 0 < int(upd.sum()) < 32 * 16
    assert (res == upd.astype(np.uint32)).all()


def test_bank_closed_form_without_skips():
    # with balances far above total possible outflow every transfer happens,
    # and the final balances are the same in every order: 10^6 - out + in.
    T, K, N = 16, 8, 32
    p = O.params("bank", n_words=N)
    heap = np.full(N, 1_000_000, dtype=np.uint32)
    res, upd = O.serial(p, heap, T, K, 5)
    assert upd.all()
    d = np.array([O.descr(p, 5, t, i) for i in range(K) for t in range(T)], dtype=np.int64)
    exp = np.full(N, 1_000_000, dtype=np.int64)
    np.add.at(exp, d[:, 0], -d[:, 2])
    np.add.at(exp, d[:, 1], d[:, 2])
    assert (heap.astype(np.int64) == exp).all()


def test_ra_increment_closed_form():
    # RA kind 1 increments every word it reads (read-after-write included):
    # final heap[k] = k + (number of times k occurs in all descriptors).
    T, K, R, N = 8, 16, 6, 16
    p = O.params("ra", n_reads=R, n_writes=R, n_words=N, ra_kind=1)
    heap = O.init_heap(p, N)
    res, upd = O.serial(p, heap, T, K, 3)
    d = np.concatenate([O.descr(p, 3, t, i) for i in range(K) for t in range(T)])
    exp = (np.arange(N) + np.bincount(d, minlength=N)).astype(np.uint32)
    assert (heap == exp).all()
    assert int(heap.astype(np.uint64).sum()) == N * (N - 1) // 2 + R * T * K


@pytest.mark.parametrize("stride", [0, 17, 32])
def test_km_closed_form(stride):
    T, K, Cn, D = 16, 8, 4, 16
    S = stride or D + 1
    p = O.params("km", km_clusters=Cn, km_dims=D, km_stride=stride)
    heap = np.zeros(Cn * S, dtype=np.uint32)
    assert O.footprint(p, T, K) == Cn * S
    res, upd = O.serial(p, heap, T, K, 8)
    d = np.array([O.descr(p, 8, t, i) for i in range(K) for t in range(T)], dtype=np.int64)
    cnt = np.bincount(d[:, 0], minlength=Cn)
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:])
    rec = heap.reshape(Cn, S)
    assert (rec[:, 0] == cnt).all() and (rec[:, 1:D + 1] == sums).all()
    assert (rec[:, D + 1:] == 0).all()          # record padding is never touched
    # result = count before: per cluster the results are 0..cnt-1 in order
    for c in range(Cn):
        assert sorted(res[d[:, 0] == c].tolist()) == list(range(cnt[c]))


def _ht_walk(heap, B, M, bucket):
    keys, h, seen = [], int(heap[bucket]), 0
    while h:
        keys.append(int(heap[B + h - 1]))
        h = int(heap[B + M + h - 1])
        seen += 1
        assert seen <= M
    return keys


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_ht_set_semantics(seed):
    T, K, B, KR = 32, 8, 16, 64
    M = T * K
    p = O.params("ht", ht_buckets=B, ht_lookup_pct=60, ht_key_range=KR)
    heap = np.zeros(B + 2 * M, dtype=np.uint32)
    res, upd = O.serial(p, heap, T, K, seed)
    present = set()
    for txid in range(T * K):
        key, ins, bucket = map(int, O.descr(p, seed, txid % T, txid // T))
        if not ins:
            assert res[txid] == (1 if key in present else 0)
        else:
            assert res[txid] == (2 if key in present else 3)
            present.add(key)
    allk = []
    for b in range(B):
        ks = _ht_walk(heap, B, M, b)
        allk += ks
        for k in ks:
            assert (O.lib().or_mix64(k) & (B - 1)) == b
    assert len(allk) == len(set(allk)) and set(allk) == present


def test_footprint_violation_is_an_error():
    p = O.params("bank", n_words=64)
    heap = np.zeros(8, dtype=np.uint32)   # smaller than the account range
    with pytest.raises(ValueError):
        O.serial(p, heap, 64, 4, 1)


# --------------------------------------------------------------------------
# replay (serial.c)
# --------------------------------------------------------------------------
def _canonical_log(p, init, T, K, seed):
    heap = init.copy()
    res, upd = O.serial(p, heap, T, K, seed)
    stamp = np.zeros(T * K, dtype=np.uint32)
    c = 0
    for x in range(T * K):
        if upd[x]:
            c += 1
            stamp[x] = c
        else:
            stamp[x] = O.RO_FLAG | c
    return heap, res, stamp


@pytest.mark.parametrize("wl,kw", [
    ("bank", dict(n_words=64)),
    ("ra", dict(n_reads=4, n_writes=4, n_words=64)),
    ("ht", dict(ht_buckets=8, ht_lookup_pct=50, ht_key_range=32)),
    ("km", dict(km_clusters=3, km_dims=4)),
    ("eb", dict(n_accesses=8, n_words=32)),
])
def test_replay_accepts_canonical_and_rejects_corruptions(wl, kw):
    T, K, seed = 16, 6, 4
    p = O.params(wl, **kw)
    words = O.footprint(p, T, K)
    init = O.init_heap(p, words)
    if wl == "bank":
        init[:] = 150
    final, res, stamp = _canonical_log(p, init, T, K, seed)
    h = init.copy()
    rc, msg = O.replay(p, h, T, K, seed, stamp, res)
    assert rc == 0, msg
    assert (h == final).all()
    upd_ids = [x for x in range(T * K) if not stamp[x] & O.RO_FLAG]
    ro_ids = [x for x in range(T * K) if stamp[x] & O.RO_FLAG]
    assert len(upd_ids) >= 2
    # duplicate stamp
    s = stamp.copy(); s[upd_ids[1]] = s[upd_ids[0]]
    assert O.replay(p, init.copy(), T, K, seed, s, res)[0] != 0
    # stamp out of range
    s = stamp.copy(); s[upd_ids[0]] = len(upd_ids) + 1
    assert O.replay(p, init.copy(), T, K, seed, s, res)[0] != 0
    # a wrong observable result
    r = res.copy(); r[upd_ids[-1]] ^= 1
    assert O.replay(p, init.copy(), T, K, seed, stamp, r)[0] != 0
    # an update tx reported as read-only
    s = stamp.copy(); s[upd_ids[-1]] = O.RO_FLAG | 0
    assert O.replay(p, init.copy(), T, K, seed, s, res)[0] != 0
    # thread order: swap the stamps of two txs of one thread
    t0 = upd_ids[0] % T
    mine = [x for x in upd_ids if x % T == t0]
    if len(mine) >= 2:
        s = stamp.copy(); s[mine[0]], s[mine[1]] = s[mine[1]], s[mine[0]]
        assert O.replay(p, init.copy(), T, K, seed, s, res)[0] != 0
    if ro_ids:
        s = stamp.copy(); s[ro_ids[0]] = O.RO_FLAG | (len(upd_ids) + 1)
        assert O.replay(p, init.copy(), T, K, seed, s, res)[0] != 0


def test_replay_detects_lost_update():
    # Two increments of the same word whose GPU results both claim to have
    # read the initial value (a lost update) cannot be replayed.
    p = O.params("ra", n_reads=1, n_writes=1, n_words=1, ra_kind=1)
    init = np.zeros(1, dtype=np.uint32)
    stamp = np.array([1, 2], dtype=np.uint32)
    assert O.replay(p, init.copy(), 2, 1, 1, stamp, np.array([0, 1], np.uint32))[0] == 0
    assert O.replay(p, init.copy(), 2, 1, 1, stamp, np.array([0, 0], np.uint32))[0] != 0


# --------------------------------------------------------------------------
# Algorithm 3 model (alg3.c)
# --------------------------------------------------------------------------
_OPS = {"BEGIN": O.OP_BEGIN, "READ": O.OP_READ, "WRITE": O.OP_WRITE, "COMMIT": O.OP_COMMIT, "READ2": O.OP_READ2}


def load_scenarios():
    with open(os.path.join(GOLD, "alg3_scenarios.json")) as f:
        return json.load(f)["scenarios"]


def encode_ops(ops):
    enc = []
    for op in ops:
        o = _OPS[op[0]]
        slot = op[1]
        word = op[2] if len(op) > 2 else 0
        val = op[3] if len(op) > 3 else 0
        enc.append([o, slot, word, val])
    return np.array(enc, dtype=np.uint32)


SCEN = [(s, v) for s in load_scenarios() for v in s["variants"]]


@pytest.mark.parametrize("sv", SCEN, ids=lambda sv: f"{sv[0]['name']}-{sv[1]['mode']}-{int(sv[1]['prelock_vbv'])}")
def test_alg3_paper_scenarios(sv):
    s, v = sv
    heap = np.array(s["heap"], dtype=np.uint32)
    locks = np.zeros(1 << s["bits"], dtype=np.uint32)
    mode = O.MODE_HV if v["mode"] == "HV" else O.MODE_TBV
    out, clock = O.alg3_script(mode, s["bits"], heap, locks, s["clock0"], encode_ops(s["ops"]),
                               prelock_vbv=v["prelock_vbv"])
    assert out.tolist() == v["out"]
    assert heap.tolist() == v["heap"]
    exp = np.zeros_like(locks)
    for k, val in v["locks"].items():
        exp[int(k)] = val
    assert locks.tolist() == exp.tolist()
    assert clock == v["clock"]


def test_lock_log_sorted_dedup():
    rng = np.random.default_rng(0)
    for _ in range(200):
        n = int(rng.integers(1, 40))
        ids = rng.integers(0, 50, n)
        bits = rng.integers(1, 3, n)
        entries = (ids << 2) | bits
        exp = {}
        for i, b in zip(ids.tolist(), bits.tolist()):
            exp[i] = exp.get(i, 0) | b
        want = [(i << 2) | exp[i] for i in sorted(exp)]
        assert O.lock_log(entries).tolist() == want
    # P:113-115 example order
    assert O.lock_log([(9 << 2) | 1, (3 << 2) | 2, (9 << 2) | 2, (1 << 2) | 1, (3 << 2) | 1]).tolist() == \
        [(1 << 2) | 1, (3 << 2) | 3, (9 << 2) | 3]


def test_lock_log_encounter_order():
    """Q32 (STM-HV-Backoff): first-occurrence order, bits merged; same
    set of entries as the sorted log."""
    assert O.lock_log([(9 << 2) | 1, (3 << 2) | 2, (9 << 2) | 2, (1 << 2) | 1, (3 << 2) | 1],
                      sorted_log=False).tolist() == [(9 << 2) | 3, (3 << 2) | 3, (1 << 2) | 1]
    rng = np.random.default_rng(1)
    for _ in range(200):
        n = int(rng.integers(1, 40))
        ids = rng.integers(0, 50, n)
        entries = (ids << 2) | rng.integers(1, 3, n)
        enc = O.lock_log(entries, sorted_log=False)
        # first occurrences, in order (numpy unique's return_index)
        _, first = np.unique(ids, return_index=True)
        assert (enc >> 2).tolist() == ids[np.sort(first)].tolist()
        assert sorted(enc.tolist()) == O.lock_log(entries).tolist()


def random_script(rng, n_tx, words, n_steps, batched=False, max_ops=5):
    """Random interleaving of n_tx transactions; each tx: BEGIN, 1..max_ops
    READ/WRITE (and, batched=True, READ2: a batched read of two words, Q35),
    COMMIT.  Returns the op list."""
    progs = []
    for s in range(n_tx):
        body = []
        for _ in range(int(rng.integers(1, max_ops + 1))):
            w = int(rng.integers(0, words))
            if batched and rng.random() < 0.3:
                body.append(["READ2", s, w, int(rng.integers(0, words))])
            elif rng.random() < 0.55:
                body.append(["READ", s, w])
            else:
                body.append(["WRITE", s, w, int(rng.integers(0, 1000))])
        progs.append([["BEGIN", s]] + body + [["COMMIT", s]])
    ops, pos = [], [0] * n_tx
    while any(pos[s] < len(progs[s]) for s in range(n_tx)):
        s = int(rng.choice([s for s in range(n_tx) if pos[s] < len(progs[s])]))
        ops.append(progs[s][pos[s]])
        pos[s] += 1
    return ops


def check_opacity(init, ops, out, final_heap, clock0, final_clock):
    """Independent formalisation of opacity: (1) committed update txs
    take effect atomically at their stamp, in stamp order; (2) aborted txs'
    writes are invisible; (3) every read a tx returns while it is opaque, and
    all of its earlier reads, equal the committed state at its current
    snapshot (own writes excepted).  Read-only committed txs read the state
    at their final snapshot."""
    history = {}     # stamp -> dict(word -> value)

    def state_at(S):
        st = list(init)
        for s in sorted(history):
            if s <= S:
                for w, v in history[s].items():
                    st[w] = v
        return st

    txs = {}
    for op, o in zip(ops, out.tolist()):
        kind, slot = op[0], op[1]
        if kind == "BEGIN":
            txs[slot] = {"reads": [], "writes": {}, "snap": o[0]}
            assert o[0] == clock0 + len(history)
        elif kind == "READ":
            tx = txs[slot]
            w = op[2]
            if w in tx["writes"]:
                assert o[0] == tx["writes"][w]
                continue
            tx["reads"].append((w, o[0]))
            tx["snap"] = o[2]
            if o[1]:
                st = state_at(o[2])
                for rw, rv in tx["reads"]:
                    assert st[rw] == rv, (op, o)
        elif kind == "READ2":
            tx = txs[slot]
            for w, v in ((op[2], o[0]), (op[3], o[1])):
                if w in tx["writes"]:
                    assert v == tx["writes"][w]
                else:
                    tx["reads"].append((w, v))
            tx["snap"] = o[2]
            if o[3] & 1:
                st = state_at(o[2])
                for rw, rv in tx["reads"]:
                    assert st[rw] == rv, (op, o)
        elif kind == "WRITE":
            txs[slot]["writes"][op[2]] = op[3]
        else:
            tx = txs[slot]
            ok, cause, stamp = o[0], o[1], o[2]
            if ok and cause == O.C_READONLY:
                st = state_at(tx["snap"])
                assert not tx["writes"]
                for rw, rv in tx["reads"]:
                    assert st[rw] == rv
            elif ok:
                assert stamp == clock0 + len(history) + 1
                st = state_at(stamp - 1)
                for rw, rv in tx["reads"]:
                    assert st[rw] == rv, ("stale read in committed tx", op)
                history[stamp] = dict(tx["writes"])
    assert final_clock == clock0 + len(history)
    assert list(final_heap) == state_at(final_clock)
    return len(history)


@pytest.mark.parametrize("mode", [O.MODE_HV, O.MODE_TBV])
@pytest.mark.parametrize("bits", [1, 2, 4])
def test_alg3_random_scripts_are_opaque(mode, bits):
    rng = np.random.default_rng(100 * mode + bits)
    commits = aborts = 0
    for trial in range(300):
        words = int(rng.integers(2, 9))
        n_tx = int(rng.integers(2, 5))
        ops = random_script(rng, n_tx, words, 0)
        init = rng.integers(0, 50, words).astype(np.uint32)
        heap = init.copy()
        locks = np.zeros(1 << bits, dtype=np.uint32)
        out, clk = O.alg3_script(mode, bits, heap, locks, 0, encode_ops(ops), n_tx=n_tx,
                                 prelock_vbv=bool(trial % 2))
        commits += check_opacity(init.tolist(), ops, out, heap.tolist(), 0, clk)
        aborts += sum(1 for op, o in zip(ops, out.tolist()) if op[0] == "COMMIT" and not o[0])
        assert not (locks & 1).any()          # no lock left held
        assert ((locks >> 1) <= clk).all()    # versions never exceed the clock
    assert commits > 100 and aborts > 10


@pytest.mark.parametrize("mode", [O.MODE_HV, O.MODE_TBV])
@pytest.mark.parametrize("bits", [1, 2, 4])
def test_alg3_batched_reads_are_opaque(mode, bits):
    """The batched TXRead of reading Q35 (OR_OP_READ2: value loads of both
    words, then ONE timestamp check with the newest version) keeps opacity
    under the independent checker, and a batch of two words that no
    other transaction touches returns what two sequential TXReads return."""
    rng = np.random.default_rng(500 + 100 * mode + bits)
    commits = batched = 0
    for trial in range(300):
        words = int(rng.integers(2, 9))
        n_tx = int(rng.integers(2, 5))
        ops = random_script(rng, n_tx, words, 0, batched=True)
        batched += sum(1 for op in ops if op[0] == "READ2")
        init = rng.integers(0, 50, words).astype(np.uint32)
        heap = init.copy()
        locks = np.zeros(1 << bits, dtype=np.uint32)
        out, clk = O.alg3_script(mode, bits, heap, locks, 0, encode_ops(ops), n_tx=n_tx,
                                 prelock_vbv=bool(trial % 2))
        commits += check_opacity(init.tolist(), ops, out, heap.tolist(), 0, clk)
        assert not (locks & 1).any()
    assert commits > 100 and batched > 200
    # a lone transaction: READ2(a, b) == READ a; READ b (values, snapshot, opacity)
    for trial in range(100):
        words = 6
        a, b = (int(x) for x in rng.integers(0, words, 2))
        init = rng.integers(0, 50, words).astype(np.uint32)
        w = int(rng.integers(0, words))
        one = [["BEGIN", 0], ["WRITE", 0, w, 7], ["READ2", 0, a, b], ["COMMIT", 0]]
        two = [["BEGIN", 0], ["WRITE", 0, w, 7], ["READ", 0, a], ["READ", 0, b], ["COMMIT", 0]]
        outs = []
        for script in (one, two):
            heap = init.copy()
            out, clk = O.alg3_script(mode, bits, heap, np.zeros(1 << bits, dtype=np.uint32), 3,
                                     encode_ops(script), n_tx=1)
            outs.append((out.tolist(), heap.tolist(), clk))
        (o1, h1, c1), (o2, h2, c2) = outs
        assert o1[2][:2] == [o2[2][0], o2[3][0]] and o1[2][2] == o2[3][2]
        assert (o1[2][3] & 1) == o2[3][1] and o1[3] == o2[4] and h1 == h2 and c1 == c2


def test_hv_aborts_no_more_than_tbv_on_false_conflicts():
    # Directional pin of P:323-325: with 2 locks for 16 words (mostly false
    # conflicts) HV's value-based fallback aborts fewer transactions than
    # TBV in aggregate.
    rng = np.random.default_rng(7)
    tot = {O.MODE_HV: 0, O.MODE_TBV: 0}
    for _ in range(400):
        words, n_tx = 16, 3
        ops = random_script(rng, n_tx, words, 0)
        init = rng.integers(0, 50, words).astype(np.uint32)
        for mode in tot:
            heap = init.copy()
            locks = np.zeros(2, dtype=np.uint32)
            out, _ = O.alg3_script(mode, 1, heap, locks, 0, encode_ops(ops), n_tx=n_tx)
            tot[mode] += sum(1 for op, o in zip(ops, out.tolist()) if op[0] == "COMMIT" and not o[0])
    assert tot[O.MODE_HV] < tot[O.MODE_TBV]


# --------------------------------------------------------------------------
# brute force (brute.c)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("T,K", [(2, 2), (3, 1), (2, 3), (3, 2), (4, 2), (8, 1)])
def test_brute_visits_multinomial_orders(T, K):
    p = O.params("ra", n_reads=1, n_writes=1, n_words=4, ra_kind=1)
    init = O.init_heap(p, 4)
    n, _, _ = O.brute(p, init, T, K, 1)
    assert n == math.factorial(T * K) // math.factorial(K) ** T


def test_brute_hand_enumerated_outcomes():
    # bank_skip fixture: the 6 serial orders were enumerated by hand and all
    # give heap [135,10,15,0], results [1,0,0,1].
    p = O.params("bank", n_words=4)
    init = np.array([50, 10, 100, 0], dtype=np.uint32)
    n, m, nd = O.brute(p, init, 2, 2, 11, np.array([135, 10, 15, 0]), np.array([1, 0, 0, 1]))
    assert (n, m, nd) == (6, True, 1)
    n, m, nd = O.brute(p, init, 2, 2, 11, np.array([135, 10, 15, 0]), np.array([1, 0, 1, 1]))
    assert (n, m) == (6, False)
    # km_records fixture: heap is order-free; the "count before" results of
    # the three cluster-1 txs (tx0 < tx2 in thread 0, tx3) give 3 outcomes:
    # (tx0,tx2,tx3) -> [0,0,1,2]; (tx0,tx3,tx2) -> [0,0,2,1]; (tx3,tx0,tx2) -> [1,0,2,0]
    p = O.params("km", km_clusters=2, km_dims=2)
    init = np.zeros(6, dtype=np.uint32)
    hq = np.array([1, 190, 215, 3, 107, 447])
    for rq, want in [([0, 0, 1, 2], True), ([0, 0, 2, 1], True), ([1, 0, 2, 0], True),
                     ([2, 0, 0, 1], False)]:
        n, m, nd = O.brute(p, init, 2, 2, 11, hq, np.array(rq))
        assert (n, m, nd) == (6, want, 3)


def test_brute_matches_python_permutations():
    # cross-check the enumerator against itertools on RA (kind 0) tiny inputs
    p = O.params("ra", n_reads=2, n_writes=1, n_words=3)
    T, K, seed = 3, 1, 21
    init = O.init_heap(p, 3)
    outs = set()
    for perm in itertools.permutations(range(T)):
        h = init.copy()
        res = [0] * T
        for t in perm:
            res[t], _ = O.exec_tx(p, h, T, K, seed, t, 0)
        outs.add((tuple(h.tolist()), tuple(res)))
    n, _, nd = O.brute(p, init, T, K, seed)
    assert n == 6 and nd == len(outs)
    for h, r in outs:
        assert O.brute(p, init, T, K, seed, np.array(h), np.array(r))[1]


# --------------------------------------------------------------------------
# key-partitioned HT: shard g of G = 2^bits owns the keys whose
# mix64 top bits are g; its transactions draw keys by rejection
# --------------------------------------------------------------------------
def test_key_partition_is_a_uniform_partition_independent_of_buckets():
    keys = np.arange(1, 1 << 15)
    for bits in (1, 2, 3):
        G = 1 << bits
        own = np.array([O.key_owner(int(k), bits) for k in keys])
        assert own.min() == 0 and own.max() == G - 1
        e = len(keys) / G
        counts = np.bincount(own, minlength=G)
        assert float(((counts - e) ** 2 / e).sum()) < 40, counts       # chi2, G-1 <= 7 dof
        if bits > 1:   # nested: the top bits-1 bits are the coarser partition
            coarse = np.array([O.key_owner(int(k), bits - 1) for k in keys])
            assert (own >> 1 == coarse).all()
    # the owner (top bits) is independent of the bucket (low bits): inside one
    # shard the keys still spread over all 16 buckets uniformly
    own = np.array([O.key_owner(int(k), 2) for k in keys])
    buckets = np.array([O.lib().or_mix64(int(k)) & 15 for k in keys[own == 1]])
    counts = np.bincount(buckets, minlength=16)
    e = counts.sum() / 16
    assert float(((counts - e) ** 2 / e).sum()) < 52, counts
    assert O.key_owner(12345, 0) == 0


@pytest.mark.parametrize("bits", [0, 1, 3])
def test_sharded_ht_key_is_first_owned_candidate(bits):
    KR, B = 1 << 22, 1 << 10
    for g in range(1 << bits):
        p = O.params("ht", ht_buckets=B, ht_lookup_pct=90, ht_key_range=KR, shard_bits=bits, shard=g)
        for t in range(40):
            for i in range(3):
                x = O.txkey(7, t, i)
                j, key = 0, None
                while key is None:
                    k = 1 + O.bounded(O.draw(x, j + 1 if j else 0), KR)
                    if O.key_owner(k, bits) == g:
                        key = k
                    j += 1
                d = O.descr(p, 7, t, i)
                assert int(d[0]) == key
                assert int(d[1]) == (1 if O.bounded(O.draw(x, 1), 100) >= 90 else 0)
                assert int(d[2]) == O.lib().or_mix64(key) & (B - 1)
                if bits == 0:   # no partition: the key is draw 0, as before
                    assert key == 1 + O.bounded(O.draw(x, 0), KR)


def test_sharded_ht_shards_are_disjoint_and_owned():
    T, K, B, KR, bits = 64, 4, 32, 512, 2
    M = T * K
    sets = []
    for g in range(1 << bits):
        p = O.params("ht", ht_buckets=B, ht_lookup_pct=50, ht_key_range=KR, shard_bits=bits, shard=g)
        heap = np.zeros(B + 2 * M, dtype=np.uint32)
        res, upd = O.serial(p, heap, T, K, 11)
        ks = [k for b in range(B) for k in _ht_walk(heap, B, M, b)]
        assert len(ks) == len(set(ks)) == int((res == 3).sum())
        assert all(O.key_owner(k, bits) == g for k in ks)
        sets.append(set(ks))
    for a in range(len(sets)):
        for b in range(a + 1, len(sets)):
            assert not (sets[a] & sets[b])


def test_sharded_ht_bad_shard_is_an_error():
    p = O.params("ht", ht_buckets=16, ht_lookup_pct=50, ht_key_range=64, shard_bits=1, shard=2)
    with pytest.raises(Exception):
        O.descr(p, 1, 0, 0)


# --------------------------------------------------------------------------
# k-means full iteration (km_assign = 1): assignment + update transactions +
# recenter = one Lloyd step of STAMP kmeans
# --------------------------------------------------------------------------
def _km_table(p, heap):
    c0 = O.km_centroids(p)
    return heap[c0:c0 + p.km_clusters * p.km_dims].reshape(p.km_clusters, p.km_dims).astype(np.int64)


@pytest.mark.parametrize("Cn,D", [(37, 5), (64, 16), (1, 3)])
def test_km_nearest_is_brute_force_argmin(Cn, D):
    rng = np.random.default_rng(Cn * 100 + D)
    p = O.params("km", km_clusters=Cn, km_dims=D, km_assign=1)
    heap = np.zeros(O.footprint(p, 1, 1), dtype=np.uint32)
    cent = rng.integers(0, 256, (Cn, D))
    if Cn > 2:
        cent[Cn - 1] = cent[1]                     # a duplicate row: the lower index must win
    heap[O.km_centroids(p):] = cent.reshape(-1)
    for _ in range(300):
        f = rng.integers(0, 256, D)
        d2 = ((f[None, :] - cent) ** 2).sum(1)
        assert O.km_nearest(p, heap, f) == int(np.argmin(d2))      # argmin: first minimum
    if Cn > 2:
        assert O.km_nearest(p, heap, cent[1]) == 1


def _wrapping_row(f, D):
    """A centroid row whose exact squared distance to f is ~2^64 but whose
    sum taken mod 2^64 is small: (2^32-1-f0)^2 = 2^64 - 2^33(1+f0) + (1+f0)^2,
    and dim 1 adds back just over 2^33(1+f0)."""
    import math
    row = [int(x) for x in f]
    row[0] = 0xFFFFFFFF
    need = (1 << 33) * (1 + int(f[0])) - (1 + int(f[0])) ** 2
    row[1] = int(f[1]) + math.isqrt(need) + 1
    return row


def test_km_nearest_exact_for_wide_uint32_centroids():
    """The assignment is the exact argmin of the integer squared distance
     for ANY uint32 centroid word: a row whose distance wraps
    modulo 2^64 to a small number must not win (Python big integers are the
    brute force)."""
    D, Cn = 16, 4
    p = O.params("km", km_clusters=Cn, km_dims=D, km_assign=1)
    rng = np.random.default_rng(9)
    for _ in range(50):
        f = rng.integers(0, 256, D)
        rows = [_wrapping_row(f, D), [int(x) + (3000 if d == 0 else 0) for d, x in enumerate(f)],
                [0xFFFFFFFF] * D, [int(x) for x in rng.integers(0, 1 << 32, D, dtype=np.uint64)]]
        exact = [sum((int(a) - int(b)) ** 2 for a, b in zip(f, r)) for r in rows]
        assert exact[0] % (1 << 64) < exact[1] < exact[0]   # a 64-bit sum would pick row 0
        heap = np.zeros(O.footprint(p, 1, 1), dtype=np.uint32)
        heap[O.km_centroids(p):] = np.array(rows, dtype=np.uint64).astype(np.uint32).reshape(-1)
        assert O.km_nearest(p, heap, f.astype(np.uint32)) == int(np.argmin(exact)) == 1


def test_km_init_centroids_and_footprint():
    p = O.params("km", km_clusters=8, km_dims=4, km_stride=8, km_assign=1)
    assert O.km_centroids(p) == 64 and O.footprint(p, 3, 3) == 64 + 32
    heap = O.init_heap(p, 96)
    assert not heap[:64].any()
    assert heap[64:].tolist() == [O.splitmix64(j) >> 56 for j in range(32)]


@pytest.mark.parametrize("stride", [0, 32])
def test_km_full_iteration_is_a_lloyd_step(stride):
    T, K, Cn, D = 64, 8, 16, 4
    p = O.params("km", km_clusters=Cn, km_dims=D, km_stride=stride, km_assign=1)
    S = stride or D + 1
    heap = O.init_heap(p, O.footprint(p, T, K))
    for it in range(3):
        cent = _km_table(p, heap).copy()
        res, upd = O.serial(p, heap, T, K, 40 + it)
        feats = np.array([O.descr(p, 40 + it, t, i)[1:] for i in range(K) for t in range(T)], dtype=np.int64)
        assign = np.argmin(((feats[:, None, :] - cent[None, :, :]) ** 2).sum(2), axis=1)
        rec = heap[:Cn * S].reshape(Cn, S).astype(np.int64)
        cnt = np.bincount(assign, minlength=Cn)
        sums = np.zeros((Cn, D), dtype=np.int64)
        np.add.at(sums, assign, feats)
        assert (rec[:, 0] == cnt).all() and (rec[:, 1:D + 1] == sums).all()
        assert (_km_table(p, heap) == cent).all()            # transactions never touch the centroids
        O.km_recenter(p, heap)
        want = np.where(cnt[:, None] > 0, sums // np.maximum(cnt, 1)[:, None], cent)
        assert (_km_table(p, heap) == want).all()
        assert not heap[:Cn * S].any()                       # accumulators restart from zero


# ---------------------------------------------------------------------------
# disjoint access sets: thread t touches only [t*k, t*k + k)
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("kind", [0, 1])
def test_ra_partition_descriptors_stay_in_the_thread_range(kind):
    """Every word of thread t's transactions lies in [t*k, t*k + k), and a
    thread range that does not fit the heap is rejected."""
    k, T, K = 16, 37, 5
    p = O.params("ra", n_reads=4, n_writes=3, ra_kind=kind, n_words=T * k, ra_partition=k)
    nw = 4 if kind == 1 else 7
    seen = set()
    for t in range(T):
        for i in range(K):
            d = O.descr(p, 9, t, i)
            words = d[:nw].astype(np.int64)
            assert ((words >= t * k) & (words < t * k + k)).all()
            seen.update(int(w) - t * k for w in words)
    assert seen == set(range(k))          # the draws cover the range (uniform bounded draws)
    small = O.params("ra", n_reads=4, n_writes=3, ra_kind=kind, n_words=T * k - 1, ra_partition=k)
    with pytest.raises(Exception):
        O.descr(small, 9, T - 1, 0)


@pytest.mark.parametrize("kind", [0, 1])
def test_ra_partition_result_is_order_independent(kind):
    """With disjoint access sets the final heap and every result do not depend
    on the serial order: canonical order (i-major) == thread-by-thread order ==
    reversed thread order, computed with the single-transaction executor."""
    k, T, K = 8, 24, 6
    p = O.params("ra", n_reads=3, n_writes=2, ra_kind=kind, n_words=T * k, ra_partition=k)
    init = O.init_heap(p, T * k)
    h0 = init.copy()
    res0, upd0 = O.serial(p, h0, T, K, 5)
    for order in (range(T), reversed(range(T))):
        h = init.copy()
        res = np.zeros(T * K, dtype=np.uint32)
        for t in order:
            for i in range(K):
                res[i * T + t], _ = O.exec_tx(p, h, T, K, 5, t, i)
        assert (h == h0).all()
        assert (res == res0).all()
    # and brute force over every interleaving of a tiny instance: one outcome
    q = O.params("ra", n_reads=2, n_writes=2, ra_kind=kind, n_words=6, ra_partition=2)
    n, match, nd = O.brute(q, O.init_heap(q, 6), 3, 2, 11)
    assert n > 1 and nd == 1
