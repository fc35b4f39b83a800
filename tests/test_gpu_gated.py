"""The gated pipelined lock round (`lock_pipeline_gated`):
a pipelined round whose lock log is longer than one 8-atomic chunk takes its
lowest lock alone, then every other lock at once.  It changes only how a
round acquires, so every launch must replay bit-exactly in stamp order
against the oracle (oracle/serial.c), and at most one round per
execution may be pipelined (Q37)."""
import pytest

import gpu_util as U

pytestmark = pytest.mark.gpu

GATED = dict(lock_pipeline=1000, lock_pipeline_gated=1)

# (workload, params, T, K, lock bits): lock logs of 9-32 entries
CASES = [
    ("km", dict(km_clusters=8, km_dims=16), 2048, 1, 10),       # 17 consecutive locks per record
    ("km", dict(km_clusters=64, km_dims=12), 4096, 1, 12),
    ("eb", dict(n_words=256, n_accesses=24), 1024, 4, 8),
    ("eb", dict(n_words=4096, n_accesses=32), 2048, 4, 12),
    ("ra", dict(n_reads=12, n_words=64, ra_kind=1), 512, 4, 6),   # increment: 12 read+write locks
]


@pytest.mark.parametrize("mode", ["hv", "tbv"])
@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_gated_round_replay(case, paired, mode):
    wl, kw, T, K, bits = CASES[case]
    if paired and wl == "km":
        pytest.skip("k-means runs on the split layout only")
    if paired:
        bits = max(bits, 12)
    g, gp, op, init = U.make(wl, T, K, bits, mode=mode, paired=paired, **GATED, **kw)
    try:
        st, _, _, _ = U.run_verified(g, wl, op, init, T, K, 17)
    finally:
        g.close()
    assert st.pipelined_rounds > 0, st.as_dict()
    # one pipelined (here: gated) round per execution at most, whatever k_lock
    assert st.pipelined_rounds <= st.attempts


@pytest.mark.parametrize("k_lock", [0, 1, 8])
def test_gated_round_progress_under_contention(k_lock):
    """Every contender of a k-means record (8 records, 4096 points) takes the
    gated round first; the launch completes for any k_lock and replays."""
    T = 4096
    g, gp, op, init = U.make("km", T, 1, 10, mode="hv", km_clusters=8, km_dims=16, k_lock=k_lock,
                             timeout_ms=30000, **GATED)
    try:
        st, _, _, _ = U.run_verified(g, "km", op, init, T, 1, 23)
    finally:
        g.close()
    assert st.pipelined_rounds > 0


@pytest.mark.parametrize("wl,kw,T,K,bits", [("eb", dict(n_words=256, n_accesses=16), 1024, 4, 8),
                                          ("ra", dict(n_reads=4, n_writes=4, n_words=64), 512, 8, 6),
                                          ("bank", dict(n_words=256), 2048, 4, 8)])
@pytest.mark.parametrize("k_lock", [0, 8])
def test_pipeline_abort_replay(wl, kw, T, K, bits, k_lock):
    """pipeline_abort: a failed pipelined round aborts the
    execution; the pipelined budget then counts every aborted execution.
    Replays bit-exactly and completes for k_lock 0 (infinite sequential
    rounds after the budget) and 8."""
    g, gp, op, init = U.make(wl, T, K, bits, mode="hv", lock_pipeline=4, pipeline_max_locks=16,
                             pipeline_abort=1, k_lock=k_lock, timeout_ms=30000, **kw)
    try:
        st, _, _, _ = U.run_verified(g, wl, op, init, T, K, 29)
    finally:
        g.close()
    assert st.pipelined_rounds > 0
    assert st.pipelined_rounds <= st.attempts
