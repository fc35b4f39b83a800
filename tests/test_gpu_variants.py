"""SURVEY §8f rows f1 and f2 on the GPU, through the C ABI:

* STM-HV-Backoff (GSTM_MODE_HV_BACKOFF): encounter-order locks, the
  first lock attempt in parallel across the warp, then the lanes that failed
  retry one at a time;
* STM-VBV (GSTM_MODE_VBV): NOrec-like value-based validation
  behind one global sequence lock;
* the unsorted-lock ablation (GSTM_MODE_HV_UNSORTED): encounter-order locks
  with the parallel retry of STM-HV-Sorting, which the paper says livelocks
  inside a warp.

Every run that completes is checked like the main modes: every transaction
committed once, stamps dense, stamp-order replay through the oracle
reproduces every result and the final heap bit for bit; tiny cases against
exhaustive enumeration of serial orders; order-free closed forms.
"""
import numpy as np
import pytest

import gpu_util as U
import oracle as O
from paper_conf_cgo_xuwglgq14_b200 import gstm as G

pytestmark = pytest.mark.gpu

ETIMEOUT = -6
LAYOUTS = [False, True]
LAYOUT_IDS = ["split", "paired"]


@pytest.fixture(scope="module", autouse=True)
def _built():
    U.ensure_built()


@pytest.mark.parametrize("paired", LAYOUTS, ids=LAYOUT_IDS)
@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
def test_ra_config0_replay(mode, paired):
    """BASELINE configs[0] (every transaction conflicts), 3 launches."""
    T, K = 256, 64
    g, gp, op, init = U.make("ra", T, K, 10, mode=mode, paired=paired, n_reads=4, n_writes=4, n_words=1024)
    for seed in (1, 2, 3):
        st, heap, stamps, res = U.run_verified(g, "ra", op, init, T, K, seed)
        assert st.mode_used == G.MODES[mode]
        init = heap


@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
def test_ra_increment_closed_form(mode):
    T, K, R, N = 1000, 8, 6, 64
    g, gp, op, init = U.make("ra", T, K, 6, mode=mode, n_reads=R, n_words=N, ra_kind=1)
    st, heap, _, _ = U.run_verified(g, "ra", op, init, T, K, 9)
    d = np.concatenate([O.descr(op, 9, t, i) for i in range(K) for t in range(T)])
    assert (heap == (np.arange(N) + np.bincount(d, minlength=N)).astype(np.uint32)).all()


@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
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
    for seed in range(40):
        g, gp, op, init = U.make(wl, T, K, bits, mode=mode, heap_words=words, **kw)
        if wl == "bank":
            init = np.array([30, 200, 5, 90, 60][:words], dtype=np.uint32)
            g.write_heap(init)
        st, heap, stamps, res = U.run_verified(g, wl, op, init, T, K, seed)
        n, match, nd = O.brute(op, init, T, K, seed, heap, res)
        assert match, (seed, n, nd)
        g.close()


@pytest.mark.parametrize("paired", LAYOUTS, ids=LAYOUT_IDS)
def test_backoff_bank_config1_full_replay(paired):
    """configs[1] at full size under STM-HV-Backoff, plus the lock-version
    invariant of ReleaseAndUpdateLocks (A3.l56-61)."""
    T, K = 1 << 20, 16
    g, gp, op, init = U.make("bank", T, K, 20, mode="hv_backoff", paired=paired, n_words=1 << 20)
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


@pytest.mark.parametrize("paired", LAYOUTS, ids=LAYOUT_IDS)
def test_vbv_bank_replay_lock_table_untouched(paired):
    """STM-VBV never reads or writes the version-lock table; commits are
    serialised by the sequence lock, the clock advances by the commits."""
    T, K = 1 << 16, 4
    g, gp, op, init = U.make("bank", T, K, 20, mode="vbv", paired=paired, n_words=1 << 20)
    st, heap, stamps, res = U.run_verified(g, "bank", op, init, T, K, 2)
    assert int(heap.astype(np.int64).sum()) == 1000 * (1 << 20)
    assert not g.read_locks().any()
    st2, heap2, *_ = U.run_verified(g, "bank", op, heap, T, K, 3)   # a second launch continues the clock
    assert st2.clock_begin == st.clock_end


@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
def test_ht_replay(mode):
    T, K = 1 << 18, 4
    g, gp, op, init = U.make("ht", T, K, 22, mode=mode)
    st, heap, stamps, res = U.run_verified(g, "ht", op, init, T, K, 5)
    d = g.dump_descr("ht", T, K, 5)
    assert set(d[res == 3, 0].tolist()) == set(d[d[:, 1] == 1, 0].tolist())


@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
def test_km_closed_form(mode):
    T, K, Cn, D = 1 << 16, 1, 1024, 16
    g, gp, op, init = U.make("km", T, K, 20, mode=mode)
    st, heap, stamps, res = U.run_verified(g, "km", op, init, T, K, 3)
    d = g.dump_descr("km", T, K, 3).astype(np.int64)
    rec = heap.reshape(Cn, D + 1).astype(np.int64)
    assert (rec[:, 0] == np.bincount(d[:, 0], minlength=Cn)).all()
    sums = np.zeros((Cn, D), dtype=np.int64)
    np.add.at(sums, d[:, 0], d[:, 1:])
    assert (rec[:, 1:] == sums).all()


@pytest.mark.parametrize("mode", ["hv_backoff", "vbv"])
@pytest.mark.parametrize("H,A,bits,T", [(1 << 10, 8, 20, 1 << 12), (1 << 10, 64, 20, 256), (1 << 20, 32, 20, 1 << 14)])
def test_eb_points_replay(mode, H, A, bits, T):
    K = 4
    g, gp, op, init = U.make("eb", T, K, bits, mode=mode, n_words=H, n_accesses=A, heap_words=H)
    U.run_verified(g, "eb", op, init, T, K, 11)


# ---------------------------------------------------------------------------
# the livelock of P:63 and the two cures the paper compares
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("k_lock", [0, 1, 8])
@pytest.mark.parametrize("paired", LAYOUTS, ids=LAYOUT_IDS)
def test_backoff_two_words_commits(k_lock, paired):
    """Every transaction reads and writes the same 2 words in random order,
    locks in encounter order: the sequential retry of STM-HV-Backoff lets
    every warp progress."""
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 10, mode="hv_backoff", paired=paired, n_reads=2, n_writes=2, n_words=2,
                             k_lock=k_lock, timeout_ms=20000)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K


def test_vbv_two_words_commits():
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 10, mode="vbv", n_reads=2, n_writes=2, n_words=2, timeout_ms=20000)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 4)
    assert st.commits == T * K


@pytest.mark.parametrize("pipeline", [0, 1])
def test_unsorted_parallel_retry_livelocks(pipeline):
    """The ablation: the same workload with encounter-order locks and the
    parallel retry -- two lanes of one warp that took the two locks in
    opposite orders fail together forever.  The kernel's watchdog
    ends the launch with GSTM_ETIMEOUT; not every transaction commits."""
    T, K = 512, 8
    g, gp, op, init = U.make("ra", T, K, 10, mode="hv_unsorted", n_reads=2, n_writes=2, n_words=2, k_lock=8,
                             lock_pipeline=pipeline, timeout_ms=300)
    g.launch("ra", T, K, 4)
    st = g.stats(check=False)
    assert st.status == ETIMEOUT, st.as_dict()
    assert st.commits + st.commits_ro < T * K
    assert st.lock_retries > 0
    g.reset_meta()


def test_unsorted_without_crossing_orders_is_fine():
    """Sanity of the ablation kernel itself: with one lock per transaction
    (RA increment of a single word) there is no order to get wrong."""
    T, K = 1024, 4
    g, gp, op, init = U.make("ra", T, K, 10, mode="hv_unsorted", n_reads=1, n_words=64, ra_kind=1)
    st, *_ = U.run_verified(g, "ra", op, init, T, K, 6)
    assert st.commits == T * K


# ---------------------------------------------------------------------------
# compute-sanitizer on tiny configurations of every kernel
# ---------------------------------------------------------------------------
@pytest.mark.slow
@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer_clean(tool):
    """memcheck (out-of-bounds / misaligned global, local and shared
    accesses), racecheck (shared-memory hazards: the per-thread counter slots)
    and synccheck (illegal __syncwarp / ballot masks: the lockstep and
    reconverge masks) report nothing on tiny runs of every workload, mode and
    layout, which also replay bit-exactly."""
    import os
    import shutil
    import subprocess
    import sys
    exe = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([exe, "--tool", tool, "--error-exitcode", "9", "--print-limit", "20",
                        sys.executable, os.path.join(root, "tools", "sanitize_tiny.py")],
                       capture_output=True, text=True, timeout=1500)
    if r.returncode != 0 and "closed on this pool" in r.stderr:
        pytest.skip("compute-sanitizer is disabled on this GPU pool (" + r.stderr.strip()[:80] + ")")
    assert r.returncode == 0, (r.stdout[-3000:], r.stderr[-3000:])
    assert "launches replayed" in r.stdout
    out = r.stdout + r.stderr
    assert "ERROR SUMMARY: 0 errors" in out or "(0 errors, 0 warnings)" in out, out[-2000:]
