"""CPU oracle for the GPU-STM hot path (Xu et al., CGO 2014).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may import
this package.  The product path (``paper_conf_cgo_xuwglgq14_b200``) never
imports, links or executes it, and shares no code with it.

The C sources (gen.c, serial.c, alg3.c, brute.c; see oracle.h) are compiled
with plain ``gcc -O2`` into ``oracle/liboracle.so`` and called through ctypes.
Citations "P:n" are lines of the paper text; "A3.lk" lines of Algorithm 3.

Parity status per function (DESIGN.md §5 lists the pins):
  gen (splitmix64/draw/bounded/descr) -- pinned: published SplitMix64 vectors,
      exact multiply-shift identities, range/uniformity properties.
  serial executor (or_exec_tx/or_serial) -- pinned: hand-derived golden
      fixtures, bank conservation, RA-increment closed form, KM = numpy
      bincount/add.at, HT = Python set semantics.
  replay (or_replay) -- pinned: canonical order accepted, corrupted logs
      rejected (each corruption class).
  alg3 model (or_alg3_script) -- pinned: hand-derived paper scenarios
      (P:184 T1/T2, false conflict P:105/P:323, read-only l.68, release l.56-61)
      and serializability of random scripts checked by brute force.
  brute force (or_brute) -- pinned: multinomial count of serial orders,
      hand-enumerated outcome sets.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRCS = ["gen.c", "serial.c", "alg3.c", "brute.c"]

WL_RA, WL_BANK, WL_HT, WL_EB, WL_KM = 0, 1, 2, 3, 4
WORKLOADS = {"ra": WL_RA, "bank": WL_BANK, "ht": WL_HT, "eb": WL_EB, "km": WL_KM}
RO_FLAG = 0x80000000
MODE_HV, MODE_TBV = 1, 2
OP_BEGIN, OP_READ, OP_WRITE, OP_COMMIT, OP_READ2 = 0, 1, 2, 3, 4   # OP_READ2: batched read (Q35)
C_OK, C_OPACITY, C_PREVBV, C_TBV, C_COMMITVBV, C_READONLY = 0, 1, 2, 3, 4, 5


class Params(C.Structure):
    """Mirror of or_params_t (oracle.h).  Defined independently of the
    product's gstm_params_t."""
    _fields_ = [
        ("workload", C.c_int32),
        ("n_reads", C.c_uint32),
        ("n_writes", C.c_uint32),
        ("ra_kind", C.c_uint32),
        ("n_words", C.c_uint64),
        ("n_accesses", C.c_uint32),
        ("ht_buckets", C.c_uint32),
        ("ht_lookup_pct", C.c_uint32),
        ("ht_key_range", C.c_uint64),
        ("km_clusters", C.c_uint32),
        ("km_dims", C.c_uint32),
        ("shard_bits", C.c_uint32),
        ("shard", C.c_uint32),
        ("km_stride", C.c_uint32),
        ("km_assign", C.c_uint32),
        ("ra_partition", C.c_uint32),
    ]


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain gcc (no GPU code)."""
    srcs = [os.path.join(_HERE, s) for s in _SRCS]
    hdr = os.path.join(_HERE, "oracle.h")
    if not force and os.path.exists(_SO):
        newest = max(os.path.getmtime(p) for p in srcs + [hdr])
        if os.path.getmtime(_SO) >= newest:
            return _SO
    tmp = _SO + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-Wno-unused-parameter",
                           "-shared", "-fPIC", "-o", tmp] + srcs)
    os.replace(tmp, _SO)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        u64, u32, i32, i64 = C.c_uint64, C.c_uint32, C.c_int, C.c_int64
        P = C.POINTER
        L.or_mix64.restype = u64; L.or_mix64.argtypes = [u64]
        L.or_splitmix64.restype = u64; L.or_splitmix64.argtypes = [u64]
        L.or_draw.restype = u64; L.or_draw.argtypes = [u64, u64]
        L.or_bounded.restype = u64; L.or_bounded.argtypes = [u64, u64]
        L.or_txkey.restype = u64; L.or_txkey.argtypes = [u64, u64, u64]
        L.or_key_owner.restype = u32; L.or_key_owner.argtypes = [u64, u32]
        L.or_km_centroids.restype = u64; L.or_km_centroids.argtypes = [P(Params)]
        L.or_km_nearest.restype = u32; L.or_km_nearest.argtypes = [P(Params), P(u32), P(u32)]
        L.or_km_recenter.restype = None; L.or_km_recenter.argtypes = [P(Params), P(u32)]
        L.or_descr.restype = i32
        L.or_descr.argtypes = [P(Params), u64, u64, u64, P(u32), i32]
        L.or_footprint.restype = u64; L.or_footprint.argtypes = [P(Params), u64, u64]
        L.or_init_heap.restype = None; L.or_init_heap.argtypes = [P(Params), P(u32), u64]
        L.or_exec_tx.restype = i32
        L.or_exec_tx.argtypes = [P(Params), P(u32), u64, u64, u64, u64, u64, u64, P(u32), P(i32)]
        L.or_serial.restype = i32
        L.or_serial.argtypes = [P(Params), P(u32), u64, u64, u64, u64, P(u32), P(C.c_uint8)]
        L.or_replay.restype = i32
        L.or_replay.argtypes = [P(Params), P(u32), u64, u64, u64, u64, P(u32), P(u32), i32,
                                C.c_char_p, i32]
        L.or_alg3_script.restype = i32
        L.or_alg3_script.argtypes = [i32, i32, u32, P(u32), u64, P(u32), P(u64), P(u32), i32,
                                     P(u32), i32]
        L.or_lock_log.restype = i32
        L.or_lock_log.argtypes = [P(u32), i32, P(u32), i32]
        L.or_lock_log_encounter.restype = i32
        L.or_lock_log_encounter.argtypes = [P(u32), i32, P(u32), i32]
        L.or_brute.restype = i64
        L.or_brute.argtypes = [P(Params), P(u32), u64, u64, u64, u64, P(u32), P(u32), P(i32),
                               P(i64)]
        _lib = L
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


def params(workload, **kw) -> Params:
    """Build or_params_t.  workload: name or id; other fields by name."""
    p = Params()
    p.workload = WORKLOADS[workload] if isinstance(workload, str) else int(workload)
    for k, v in kw.items():
        if not hasattr(p, k):
            raise KeyError(k)
        setattr(p, k, int(v))
    return p


def splitmix64(x: int) -> int:
    return lib().or_splitmix64(x)


def draw(x: int, k: int) -> int:
    return lib().or_draw(x, k)


def bounded(r: int, n: int) -> int:
    return lib().or_bounded(r, n)


def km_centroids(p: Params) -> int:
    """Word offset of the k-means centroid table (after the records)."""
    return lib().or_km_centroids(C.byref(p))


def km_nearest(p: Params, heap: np.ndarray, f) -> int:
    f = np.ascontiguousarray(f, dtype=np.uint32)
    return lib().or_km_nearest(C.byref(p), _p(heap, C.c_uint32), _p(f, C.c_uint32))


def km_recenter(p: Params, heap: np.ndarray) -> None:
    """End of a Lloyd iteration (in place): centroids = floor means, records zeroed."""
    assert heap.dtype == np.uint32 and heap.flags.c_contiguous
    lib().or_km_recenter(C.byref(p), _p(heap, C.c_uint32))


def key_owner(key: int, bits: int) -> int:
    """Shard owning an HT key under a 2^bits-way partition."""
    return lib().or_key_owner(key, bits)


def txkey(seed: int, t: int, i: int) -> int:
    return lib().or_txkey(seed, t, i)


def descr(p: Params, seed: int, t: int, i: int, cap: int = 1024) -> np.ndarray:
    out = np.zeros(cap, dtype=np.uint32)
    n = lib().or_descr(C.byref(p), seed, t, i, _p(out, C.c_uint32), cap)
    if n < 0:
        raise ValueError("or_descr failed")
    return out[:n].copy()


def footprint(p: Params, T: int, K: int) -> int:
    return int(lib().or_footprint(C.byref(p), T, K))


def init_heap(p: Params, words: int) -> np.ndarray:
    h = np.zeros(words, dtype=np.uint32)
    lib().or_init_heap(C.byref(p), _p(h, C.c_uint32), words)
    return h


def exec_tx(p: Params, heap: np.ndarray, T: int, K: int, seed: int, t: int, i: int):
    """Execute tx (t, i) serially in place; returns (result, is_update)."""
    r = C.c_uint32(0)
    u = C.c_int(0)
    rc = lib().or_exec_tx(C.byref(p), _p(heap, C.c_uint32), heap.size, T, K, seed, t, i,
                          C.byref(r), C.byref(u))
    if rc:
        raise ValueError("footprint violation")
    return r.value, bool(u.value)


def serial(p: Params, heap: np.ndarray, T: int, K: int, seed: int):
    """Canonical serial execution (tx_id = i*T + t ascending), in place.
    Returns (results[tx_id], is_update[tx_id])."""
    n = T * K
    res = np.zeros(max(n, 1), dtype=np.uint32)
    upd = np.zeros(max(n, 1), dtype=np.uint8)
    rc = lib().or_serial(C.byref(p), _p(heap, C.c_uint32), heap.size, T, K, seed,
                         _p(res, C.c_uint32), _p(upd, C.c_uint8))
    if rc:
        raise ValueError("footprint violation")
    return res[:n], upd[:n].astype(bool)


def replay(p: Params, heap: np.ndarray, T: int, K: int, seed: int, tx_stamp: np.ndarray,
           tx_result: np.ndarray, check_thread_order: bool = True):
    """Stamp-order replay in place.  Returns (rc, message); rc == 0 is success."""
    tx_stamp = np.ascontiguousarray(tx_stamp, dtype=np.uint32)
    tx_result = np.ascontiguousarray(tx_result, dtype=np.uint32)
    assert tx_stamp.size >= T * K and tx_result.size >= T * K
    err = C.create_string_buffer(512)
    rc = lib().or_replay(C.byref(p), _p(heap, C.c_uint32), heap.size, T, K, seed,
                         _p(tx_stamp, C.c_uint32), _p(tx_result, C.c_uint32),
                         1 if check_thread_order else 0, err, 512)
    return rc, err.value.decode()


def alg3_script(mode: int, bits: int, heap: np.ndarray, lock_tab: np.ndarray, clock: int,
                ops, n_tx: int = 4, prelock_vbv: bool = True):
    """Run Algorithm 3 (sequential model) on a script.  ops: (n,4) uint32
    (op, slot, word, value).  heap and lock_tab are updated in place.
    Returns (out (n,4) uint32, clock)."""
    ops = np.ascontiguousarray(np.asarray(ops, dtype=np.uint32).reshape(-1, 4))
    out = np.zeros_like(ops)
    clk = C.c_uint64(clock)
    assert lock_tab.size == (1 << bits)
    rc = lib().or_alg3_script(mode, 1 if prelock_vbv else 0, bits, _p(heap, C.c_uint32), heap.size,
                              _p(lock_tab, C.c_uint32), C.byref(clk), _p(ops, C.c_uint32),
                              ops.shape[0], _p(out, C.c_uint32), n_tx)
    if rc:
        raise ValueError(f"or_alg3_script rc={rc}")
    return out, clk.value


def lock_log(entries, sorted_log: bool = True) -> np.ndarray:
    """Sorted lock log, or the encounter-order log (Q32)."""
    e = np.ascontiguousarray(np.asarray(entries, dtype=np.uint32))
    out = np.zeros(max(e.size, 1), dtype=np.uint32)
    fn = lib().or_lock_log if sorted_log else lib().or_lock_log_encounter
    n = fn(_p(e, C.c_uint32), e.size, _p(out, C.c_uint32), out.size)
    return out[:n].copy()


def brute(p: Params, init: np.ndarray, T: int, K: int, seed: int, heap_q=None, results_q=None):
    """Enumerate all serial orders.  Returns (n_orders, match, n_distinct)."""
    init = np.ascontiguousarray(init, dtype=np.uint32)
    m = C.c_int(0)
    nd = C.c_int64(0)
    hq = None if heap_q is None else np.ascontiguousarray(heap_q, dtype=np.uint32)
    rq = None if results_q is None else np.ascontiguousarray(results_q, dtype=np.uint32)
    n = lib().or_brute(C.byref(p), _p(init, C.c_uint32), init.size, T, K, seed,
                       None if hq is None else _p(hq, C.c_uint32),
                       None if rq is None else _p(rq, C.c_uint32), C.byref(m), C.byref(nd))
    if n < 0:
        raise ValueError(f"or_brute rc={n}")
    return int(n), bool(m.value), int(nd.value)
