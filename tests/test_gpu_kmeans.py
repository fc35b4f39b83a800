"""GPU tests (-m gpu): a full k-means iteration (STAMP kmeans,
P:244) through the C ABI -- the nearest-centroid assignment pass, the
transactional cluster updates, and gstm_km_recenter -- against the CPU
oracle and numpy.

k-means updates commute, so the heap after an iteration is unique: the
stamp-order replay must reproduce it bit-exactly, and it must equal the
closed form (bincount / add.at over the numpy argmin assignment).
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


def _closed_form(op, heap_before, feats):
    Cn, D = op.km_clusters, op.km_dims
    c0 = O.km_centroids(op)
    cent = heap_before[c0:c0 + Cn * D].reshape(Cn, D).astype(np.int64)
    # squared distances in uint64 (exact here: < 2^64; int64 would overflow
    # for centroid words near 2^32), 2048 points at a time
    assign = np.empty(len(feats), dtype=np.int64)
    for s in range(0, len(feats), 2048):
        diff = (feats[s:s + 2048, None, :] - cent[None, :, :]).astype(np.uint64)
        d2 = (diff * diff).sum(2, dtype=np.uint64)
        assign[s:s + 2048] = np.argmin(d2, axis=1)       # ties: first (lowest) index
    cnt = np.bincount(assign, minlength=Cn)
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, assign, feats)
    return cnt, sums


@pytest.mark.parametrize("mode,paired,stride,shift", [("hv", False, 0, 0), ("tbv", True, 0, 0), ("fgl", False, 0, 0),
                                                      ("hv", False, 32, 5)])
def test_km_full_iterations(mode, paired, stride, shift):
    T, K, Cn, D = 1 << 14, 2, 1024, 16
    bits = 20 if not paired else 16
    g, gp, op, init = U.make("km", T, K, bits, mode=mode, paired=paired, km_assign=1, km_stride=stride,
                             lock_shift=shift)
    S = stride or D + 1
    assert (g.read_heap() == init).all()                  # device centroid table == oracle's
    heap = init
    for it in range(3):
        seed = 77 + it
        st, after, stamps, res = U.run_verified(g, "km", op, heap, T, K, seed)
        feats = g.dump_descr("km", T, K, seed)[:, 1:D + 1].astype(np.int64)
        cnt, sums = _closed_form(op, heap, feats)
        rec = after[:Cn * S].reshape(Cn, S).astype(np.int64)
        assert (rec[:, 0] == cnt).all() and (rec[:, 1:D + 1] == sums).all()
        g.km_recenter()
        want = after.copy()
        O.km_recenter(op, want)
        heap = g.read_heap()
        assert (heap == want).all()
        assert not heap[:Cn * S].any()


def test_km_assign_ties_and_wide_centroids():
    """Duplicate centroid rows (the lower index wins) and centroid words >=
    4096 (the exact 64-bit distance path)."""
    T, K, Cn, D = 4096, 1, 64, 16
    g, gp, op, init = U.make("km", T, K, 16, mode="hv", km_clusters=Cn, km_dims=D, km_assign=1)
    rng = np.random.default_rng(5)
    for wide in (False, True):
        cent = rng.integers(0, 256, (Cn, D)).astype(np.uint32)
        cent[7] = cent[3]
        if wide:
            cent[10] = 1 << 20
            cent[11, 0] = 0xFFFFFFF0
        heap = init.copy()
        c0 = O.km_centroids(op)
        heap[c0:c0 + Cn * D] = cent.reshape(-1)
        g.write_heap(heap)
        st, after, *_ = U.run_verified(g, "km", op, heap, T, K, 3 + wide)
        feats = g.dump_descr("km", T, K, 3 + wide)[:, 1:D + 1].astype(np.int64)
        cnt, sums = _closed_form(op, heap, feats)
        assert (after[:Cn * (D + 1)].reshape(Cn, D + 1)[:, 0] == cnt).all()
        assert cnt[7] == 0                                   # never chosen over its twin, row 3


def test_km_assign_exact_when_64bit_sum_would_wrap():
    """The device assignment is the exact argmin for any uint32 centroid word
    (DESIGN.md §3.4): per point, a row whose squared distance (~2^64) wraps
    modulo 2^64 to a small number must lose to a row at distance 9e6."""
    import math
    T, K, Cn, D = 64, 1, 128, 16
    g, gp, op, init = U.make("km", T, K, 16, mode="hv", km_clusters=Cn, km_dims=D, km_assign=1)
    feats = g.dump_descr("km", T, K, 21)[:, 1:D + 1].astype(np.int64)
    cent = np.full((Cn, D), 0xFFFFFFFF, dtype=np.uint64)
    want = np.zeros(Cn, dtype=np.int64)
    for t in range(T):
        f = [int(x) for x in feats[t]]
        wrap = list(f)
        wrap[0] = 0xFFFFFFFF
        wrap[1] = f[1] + math.isqrt((1 << 33) * (1 + f[0]) - (1 + f[0]) ** 2) + 1
        near = list(f)
        near[0] += 3000
        cent[2 * t], cent[2 * t + 1] = wrap, near
        d_wrap = sum((a - b) ** 2 for a, b in zip(f, wrap))
        assert d_wrap % (1 << 64) < 3000 ** 2 < d_wrap
    rows = cent.tolist()
    for t in range(T):                              # exact argmin (first minimum), Python integers
        exact = [sum((int(a) - int(b)) ** 2 for a, b in zip(feats[t], row)) for row in rows]
        want[min(range(Cn), key=lambda c: (exact[c], c))] += 1
    assert want[1::2].sum() == T                    # every point's nearest is a "near" row
    heap = init.copy()
    c0 = O.km_centroids(op)
    heap[c0:c0 + Cn * D] = cent.astype(np.uint32).reshape(-1)
    g.write_heap(heap)
    st, after, *_ = U.run_verified(g, "km", op, heap, T, K, 21)
    assert (after[:Cn * (D + 1)].reshape(Cn, D + 1)[:, 0] == want).all()


def test_km_recenter_needs_assign():
    g, gp, op, init = U.make("km", 64, 1, 10)
    with pytest.raises(G.GstmError):
        g.km_recenter()
