"""The contention manager (serial tickets; `serial_after`).

It only decides WHEN an execution starts -- every execution still runs
Algorithm 3 in full -- so every launch here must replay bit-exactly in stamp
order against the oracle (oracle/serial.c, the opacity definition of
P:234-236), whatever the ticket queue did.  The thresholds are forced low
(serial_after = 1, serial_commits huge) so that many executions run as the
ticket owner, with the queue taken and served under contention.
"""
import pytest

import gpu_util as U

pytestmark = pytest.mark.gpu

FORCE = dict(serial_after=1, serial_commits=1 << 16)

# (workload, params, T, K, lock bits)
CASES = [
    ("eb", dict(n_words=1024, n_accesses=64), 1024, 4, 10),    # the EB contention corner, scaled down
    ("eb", dict(n_words=64, n_accesses=20), 512, 4, 6),        # A <= 32 kernel, short transactions
    ("eb", dict(n_words=256, n_accesses=32), 512, 4, 8),       # A <= 32 kernel
    ("eb", dict(n_words=16, n_accesses=24), 512, 4, 4),        # duplicate lock ids inside every batch
    ("ra", dict(n_reads=4, n_writes=4, n_words=64), 512, 8, 6),
    ("ra", dict(n_reads=3, n_words=16, ra_kind=1), 256, 4, 4),
    ("km", dict(km_clusters=8, km_dims=4), 2048, 1, 10),
]


@pytest.mark.parametrize("mode", ["hv", "tbv", "hv_backoff"])
@pytest.mark.parametrize("paired", [False, True])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_serial_tickets_replay(case, paired, mode):
    wl, kw, T, K, bits = CASES[case]
    if paired and wl == "km":
        pytest.skip("k-means runs on the split layout only")
    if paired:
        bits = max(bits, 7)
    g, gp, op, init = U.make(wl, T, K, bits, mode=mode, paired=paired, **FORCE, **kw)
    try:
        st, _, _, _ = U.run_verified(g, wl, op, init, T, K, 11)
    finally:
        g.close()
    assert st.serial_runs > 0, st.as_dict()
    assert st.serial_runs <= st.attempts


@pytest.mark.parametrize("k_lock", [0, 1, 8])
def test_serial_corner_completes(k_lock):
    """The EB corner (every pair of transactions conflicts) with the library
    defaults for EB plus the contention manager: completes (no watchdog) and
    replays, for any k_lock -- 0 included (the owner pipelines only the first
    lock round of an execution, Q15/Q37)."""
    T, K = 2048, 2
    g, gp, op, init = U.make("eb", T, K, 10, mode="hv", n_words=1024, n_accesses=64, k_lock=k_lock,
                             serial_after=4, timeout_ms=30000)
    try:
        st, _, _, _ = U.run_verified(g, "eb", op, init, T, K, 5)
    finally:
        g.close()
    assert st.serial_runs > 0


@pytest.mark.parametrize("wl,kw,bits", [("bank", dict(n_words=64), 6),
                                        ("ht", dict(ht_buckets=16, ht_key_range=64, ht_lookup_pct=50), 8),
                                        ("eb", dict(n_words=64, n_accesses=16), 6)])
def test_serial_not_compiled_for_bank_ht(wl, kw, bits):
    """Bank, HT and the EB A <= 16 kernels leave the contention manager out
    (WL::kSerialGate, their register budget): serial_after is accepted and
    ignored."""
    T, K = 512, 4
    g, gp, op, init = U.make(wl, T, K, bits, mode="hv", **FORCE, **kw)
    try:
        st, _, _, _ = U.run_verified(g, wl, op, init, T, K, 2)
    finally:
        g.close()
    assert st.serial_runs == 0


def test_eb_default_manager_idle_at_low_contention():
    """EB enables the contention manager by default (serial_after 4); at low
    contention no transaction qualifies (the GPU commits far more than
    serial_commits per abort), so no ticket is ever taken."""
    T, K = 8192, 4
    g, gp, op, init = U.make("eb", T, K, 20, mode="hv", heap_words=1 << 20, n_words=1 << 20, n_accesses=32)
    assert gp.serial_after == 4
    try:
        st, _, _, _ = U.run_verified(g, "eb", op, init, T, K, 41)
    finally:
        g.close()
    assert st.serial_runs == 0, st.as_dict()


@pytest.mark.parametrize("flavour", ["strict", "phase", "hlog", "smem"])
def test_serial_tickets_in_build_flavours(flavour):
    """The serial owner path replays in every build flavour (strict PTX
    fences, Figure-5 phase timing, hashed and shared-memory lock logs)."""
    T, K = 1024, 4
    g, gp, op, init = U.make("eb", T, K, 10, mode="hv", flavour=flavour, n_words=1024, n_accesses=64, **FORCE)
    try:
        st, _, _, _ = U.run_verified(g, "eb", op, init, T, K, 43)
    finally:
        g.close()
    assert st.serial_runs > 0
