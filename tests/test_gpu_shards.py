"""GPU tests (-m gpu) of the key-partitioned hash table (DESIGN.md
§8) and of the one-lock-per-record k-means layout, through the C
ABI, against the CPU oracle.

Sharded HT: shard g of G = 2^bits owns the keys whose mix64 top bits are g;
each shard is an independent GPU-STM instance (own heap, lock table, clock),
so every shard must replay bit-exactly on its own, and the shards together
must hold every inserted key exactly once, each in the shard that owns it.
On one GPU the G shards run one after the other on separate handles -- the
same per-rank code the multi-GPU bench runs, minus the final all-reduce
(covered by the gloo test in test_multiproc.py).
"""
import numpy as np
import pytest

import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import gstm as G
import gpu_util as U

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _built():
    U.ensure_built()


def _walk_keys(heap, B, M):
    heads = heap[:B].astype(np.int64)
    key, nxt = heap[B:B + M], heap[B + M:B + 2 * M]
    out = []
    cur = heads[heads != 0]
    steps = 0
    while cur.size:
        out.append(key[cur - 1])
        cur = nxt[cur - 1].astype(np.int64)
        cur = cur[cur != 0]
        steps += 1
        assert steps <= M
    return np.concatenate(out) if out else np.zeros(0, np.uint32)


@pytest.mark.parametrize("bits", [1, 2, 3])
@pytest.mark.parametrize("mode", ["hv", "tbv"])
def test_sharded_ht_replay_and_global_invariant(bits, mode):
    G_ = 1 << bits
    T, K, B, KR = 1 << 14, 4, 1 << 12, 1 << 16
    M = T * K
    seen = {}
    inserted_total = 0
    for g in range(G_):
        h, gp, op, init = U.make("ht", T, K, 16, mode=mode, ht_buckets=B, ht_key_range=KR, ht_lookup_pct=50,
                                 shard_bits=bits, shard=g)
        seed = 1000 + g          # each rank its own seed (bench.shard_seed)
        st, heap, stamps, res = U.run_verified(h, "ht", op, init, T, K, seed)
        d = h.dump_descr("ht", T, K, seed)
        assert all(O.key_owner(int(k), bits) == g for k in np.unique(d[:, 0]))
        keys = _walk_keys(heap, B, M)
        assert keys.size == np.unique(keys).size == int((res == 3).sum()) == st.commits
        assert set(keys.tolist()) == set(d[d[:, 1] == 1, 0].tolist())
        for k in keys.tolist():
            assert k not in seen
            seen[k] = g
        inserted_total += keys.size
        h.close()
    # global: the union of the shards is the set of distinct keys inserted anywhere
    assert len(seen) == inserted_total


def test_sharded_ht_bad_shard_rejected():
    with pytest.raises(G.GstmError):
        U.make("ht", 64, 1, 10, ht_buckets=16, ht_key_range=64, shard_bits=2, shard=4)[0].launch("ht", 64, 1, 1)


@pytest.mark.parametrize("mode", ["hv", "tbv", "fgl"])
def test_km_one_lock_per_record(mode):
    """k-means records padded to 32 words and 2^5-word lock stripes: every
    cluster record is guarded by ONE version lock (lock_shift 5).
    The result is order-free: it must equal bincount / add.at exactly."""
    T, K, Cn, D = 1 << 18, 1, 1024, 16
    h, gp, op, init = U.make("km", T, K, 20, mode=mode, km_stride=32, lock_shift=5)
    st, heap, stamps, res = U.run_verified(h, "km", op, init, T, K, 9)
    d = h.dump_descr("km", T, K, 9).astype(np.int64)
    rec = heap.reshape(Cn, 32).astype(np.int64)
    assert (rec[:, 0] == np.bincount(d[:, 0], minlength=Cn)).all()
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:])
    assert (rec[:, 1:D + 1] == sums).all()
    assert not rec[:, D + 1:].any()
    locks = h.read_locks(1 << 20)
    assert not (locks & 1).any()
    # every record's lock version is the stamp of its last committed update
    # (stamps are launch-relative: + clock_begin), all other locks untouched
    ver = locks >> 1
    last = np.zeros(Cn, dtype=np.int64)
    np.maximum.at(last, d[:, 0], stamps.astype(np.int64) + st.clock_begin)
    if mode != "fgl":
        assert (ver[np.arange(Cn)] == last).all()
        assert not ver[Cn:].any()
