"""Op-mix roofline of the GPU-STM hot path.

The transaction kernels are bound by chains of dependent L2 round trips and by
L2 request throughput, not by streaming HBM bandwidth or tensor cores.  Their
roof is therefore MEASURED: ``gstm_ubench_mix`` runs, on a handle of the same
layout and size, conflict-free "transactions" made of exactly the memory
operations Algorithm 3 issues for one committed transaction of
the workload, phase by phase in its dependency order, with no STM logic around
them.  The per-transaction op counts come from the measured run itself (the
``reads_update / reads_ro / writes_update / locks_update`` statistics: log
sizes of the committed executions), so the roof is the best rate at which the
hardware can issue the committed transactions' own accesses.

This module only builds the phase programs (argument marshalling for the C
ABI's program format, include/gstm.h ``gstm_ubench_mix``); every operation
runs in the CUDA microkernel.  Measurement helper, not part of the STM path.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

# phase kinds (include/gstm.h gstm_ubench_mix)
LD_V, LD_L, ATOM_L, ST_V, ST_L, CLOCK, FENCE_REL, FENCE_ACQ = 1, 2, 3, 4, 5, 6, 7, 8
RECORDS = 0x100


def ph(kind: int, count: int = 1, slot0: int = 0) -> int:
    assert 0 <= count < 256 and 0 <= slot0 < 65536
    return kind | (count << 8) | (slot0 << 16)


@dataclass
class TxShape:
    """Memory shape of one committed transaction (Algorithm 3 on a workload
    body).  read_batches: sizes of the read batches in body order (each batch
    is one round trip of value loads, A3.l24, then -- split layout -- one of
    lock-word loads, l.28); the reads of batch k are word slots after those of
    batch k-1.  write_slots: the word slots written (A3.l37); locks: lock-log
    entries (A3.l34/l38), the first `locks` slots of reads + writes."""
    read_batches: list = field(default_factory=list)
    write_slots: list = field(default_factory=list)
    locks: int = 0

    @property
    def reads(self) -> int:
        return sum(self.read_batches)


def stm_program(shape: TxShape, paired: bool, hv_prelock: bool, pipelined) -> list:
    """Phases of one transaction under STM-HV/TBV (tx.cuh / tx_pair.cuh).
    pipelined: False (sorted, one lock at a time), True (one round trip) or
    "gated" (the lowest lock, then the rest in one round trip)."""
    p, slot = [], 0
    for n in shape.read_batches:                       # TXRead batches (A3.l21-35)
        if n <= 0:
            continue
        p.append(ph(LD_V, n, slot))                    # l.24 (paired: value and lock at once)
        if not paired:
            p.append(ph(FENCE_ACQ))                    # l.26
            p.append(ph(LD_L, n, slot))                # l.28
        slot += n
    if not shape.write_slots and not shape.locks:      # read-only: linearised at its snapshot (l.68)
        return p
    R = shape.reads
    if hv_prelock and R:
        p.append(ph(LD_V, R, 0))                       # l.71 pre-lock VBV, all reads at once
    n = shape.locks
    if pipelined == "gated" and n > 1:                 # the gated round (§6.4): the lowest lock, then the rest
        p.append(ph(ATOM_L, 1, 0))
        p.append(ph(ATOM_L, n - 1, 1))
    elif pipelined:
        p.append(ph(ATOM_L, n, 0))                     # l.45, one round trip
    else:
        p += [ph(ATOM_L, 1, k) for k in range(n)]      # l.44-48: sorted, one at a time (Q15)
    if not paired:
        p.append(ph(FENCE_ACQ))
        for s in shape.write_slots:                    # l.80-81 write-back
            p.append(ph(ST_V, 1, s))
        p.append(ph(FENCE_REL))                        # l.82
    p.append(ph(CLOCK))                                # l.83 (warp-aggregated)
    p.append(ph(ST_L, n, 0))                           # l.84 release (paired: value + version)
    return p


def mix(programs: list, records: tuple | None = None) -> list:
    """programs: [(weight, phases)]; weights are normalised to 65536."""
    programs = [(w, q) for w, q in programs if w > 0]
    tot = sum(w for w, _ in programs)
    ws = [int(round(65536 * w / tot)) for w, _ in programs]
    ws[-1] = 65536 - sum(ws[:-1])
    head = [len(programs) | (RECORDS if records else 0)]
    if records:
        head += [int(records[0]), int(records[1])]
    out = head
    for w, (_, q) in zip(ws, programs):
        out += [w, len(q)] + list(q)
    return out


def _split(x: float):
    """floor/ceil of a mean, with the weight of the ceil (the two programs
    that reproduce the mean exactly when the cost is linear in x)."""
    lo = math.floor(x)
    return lo, lo + 1, x - lo


def _shape(wl: str, reads: float, writes: float, locks: float, n_accesses: int = 0):
    """TxShape(s) with `reads` reads (may be fractional: two shapes, weights)."""
    lo, hi, f = _split(max(0.0, reads))
    out = []
    for r, w in ((lo, 1 - f), (hi, f)):
        if w <= 1e-9:
            continue
        if wl == "ht":          # bucket head, then (key, next) per chain node
            batches = [1] + [2] * max(0, (r - 1) // 2) + ([1] if r > 1 and (r - 1) % 2 else [])
        elif wl == "eb" or wl == "km" or wl == "bank":
            batches = [r]       # one read_batch / read_many of every non-RAW read
        else:                   # ra
            batches = [r]
        W = int(round(writes))
        ws = list(range(r, r + W)) if wl in ("ra", "eb", "ht") else list(range(min(W, r)))
        out.append((w, TxShape(batches, ws, int(round(locks)) if W or locks else 0)))
    return out


def programs_from_stats(wl: str, st, paired: bool, mode: str, prelock: bool, pipelined: bool,
                        records: tuple | None = None) -> list:
    """The op-mix program of the committed transactions of one measured run
    (st: gstm_stats_t or a dict with the same keys)."""
    g = (lambda k: getattr(st, k)) if not isinstance(st, dict) else st.__getitem__
    cu, cr = g("commits"), g("commits_ro")
    hv = mode in ("hv", "hv_backoff")
    progs = []
    if cu:
        for w, s in _shape(wl, g("reads_update") / cu, g("writes_update") / cu, g("locks_update") / cu):
            q = stm_program(s, paired, hv and prelock, pipelined)
            if records:
                # contention roof: what a record's commits cannot overlap is the
                # time its locks are held -- from the first lock atomic (A3.l45)
                # to the release (l.84); the next transaction's reads and
                # validation can run while the record is locked
                first = next(k for k, c in enumerate(q) if c & 0xff == ATOM_L)
                q = q[first:]
            progs.append((cu * w, q))
    if cr and not records:
        for w, s in _shape(wl, g("reads_ro") / cr, 0, 0):
            s.write_slots, s.locks = [], 0
            progs.append((cr * w, stm_program(s, paired, False, False)))
    assert 1 <= len(progs) <= 4, progs
    return mix(progs, records)


MAX_PHASES = 160


def validate(prog: list, words: int) -> None:
    """The checks gstm_ubench_mix applies, with a message (GSTM_EINVAL
    otherwise only says "bad program")."""
    n, pos = prog[0] & 0xff, 1
    if not 1 <= n <= 4:
        raise ValueError(f"{n} programs (1..4)")
    if prog[0] & RECORDS:
        pos = 3
        if prog[1] * prog[2] > words:
            raise ValueError(f"records {prog[1]} x stride {prog[2]} > {words} words")
    cum = 0
    for q in range(n):
        cum += prog[pos]
        k = prog[pos + 1]
        if k > MAX_PHASES:
            raise ValueError(f"program {q}: {k} phases > {MAX_PHASES}")
        for c in prog[pos + 2:pos + 2 + k]:
            if not 1 <= (c & 0xff) <= 8:
                raise ValueError(f"program {q}: bad phase kind {c & 0xff}")
        if sum(1 for c in prog[pos + 2:pos + 2 + k] if c & 0xff == CLOCK) > 1:
            raise ValueError(f"program {q}: more than one clock phase")
        pos += 2 + k
    if cum != 65536 or pos != len(prog):
        raise ValueError(f"weights sum {cum}, {pos} of {len(prog)} words parsed")


def op_counts(prog: list) -> dict:
    """Mean ops per transaction by class (the max-formula roof of SURVEY §8(d):
    roof = 1 / max_i(count_i / peak_i))."""
    n = prog[0] & 0xff
    pos = 3 if prog[0] & RECORDS else 1
    tot = {"ld": 0.0, "atom": 0.0, "st": 0.0, "clock": 0.0}
    for _ in range(n):
        w, k = prog[pos] / 65536.0, prog[pos + 1]
        for code in prog[pos + 2:pos + 2 + k]:
            kind, cnt = code & 0xff, (code >> 8) & 0xff
            if kind in (LD_V, LD_L):
                tot["ld"] += w * cnt
            elif kind == ATOM_L:
                tot["atom"] += w * cnt
            elif kind in (ST_V, ST_L):
                tot["st"] += w * cnt
            elif kind == CLOCK:
                tot["clock"] += w
        pos += 2 + k
    return tot


def round_trips(prog: list) -> float:
    """Mean dependent memory round trips per transaction: load, atomic and
    clock phases (stores are fire-and-forget; fences are not accesses)."""
    n = prog[0] & 0xff
    pos = 3 if prog[0] & RECORDS else 1
    rt = 0.0
    for _ in range(n):
        w, k = prog[pos] / 65536.0, prog[pos + 1]
        rt += w * sum(1 for c in prog[pos + 2:pos + 2 + k] if (c & 0xff) in (LD_V, LD_L, ATOM_L, CLOCK))
        pos += 2 + k
    return rt
