"""The gated pipelined lock round (`lock_pipeline_gated`):
a pipelined round whose lock log is longer than one 8-atomic chunk takes its
lowest lock alone, then every other lock at once.  It changes only how a
round acquires, so every launch must replay bit-exactly in stamp order
against the oracle (oracle/serial.c), and at most one round per
execution may be pipelined (Q37)."""
import pytest

import gpu_util as U

pytestmark = pytest.mark.gpu

GATED = dict(lock_pipeline=1000, lock_pipeline_gated=1, pipeline_abort=0)

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


@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("k_lock", [0, 8])
def test_pipeline_abort_replay(paired, k_lock):
    """EB's adaptive pipelined round (pipeline_abort): a
    failed pipelined round aborts the execution, a warp pipelines only while
    its recent abort rate is low.  It applies where the footprint exceeds L2
    and there is a lock per <= 4 words: a 3 x 2^24-word hot set with 2^24
    locks (2^26 paired).  Replays bit-exactly and completes for k_lock 0 and 8."""
    T, K, words = 8192, 4, 3 << 24          # 192 MiB: clearly larger than the B200's L2
    bits = 26 if paired else 24
    g, gp, op, init = U.make("eb", T, K, bits, mode="hv", paired=paired, n_words=words, n_accesses=16,
                             k_lock=k_lock, timeout_ms=30000)
    assert gp.pipeline_abort and gp.lock_pipeline and gp.pipeline_max_locks >= 16   # EB's defaults
    try:
        st, _, _, _ = U.run_verified(g, "eb", op, init, T, K, 29)
    finally:
        g.close()
    assert st.pipelined_rounds > 0
    assert st.pipelined_rounds <= st.attempts


def test_pipeline_abort_stays_off_where_it_does_not_pay():
    """An L2-resident hot set keeps the sequential rounds (no pipelined
    round at all) although pipeline_abort is on."""
    T, K = 2048, 4
    g, gp, op, init = U.make("eb", T, K, 12, mode="hv", n_words=4096, n_accesses=16)
    try:
        st, _, _, _ = U.run_verified(g, "eb", op, init, T, K, 31)
    finally:
        g.close()
    assert st.pipelined_rounds == 0
