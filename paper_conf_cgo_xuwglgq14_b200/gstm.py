"""Thin ctypes binding of the GPU-STM C ABI (include/gstm.h).

Argument marshalling only: every step of the transaction hot path runs in the
CUDA kernels of libgstm.so.  There is no CPU fallback: if the shared library
is missing or no CUDA device is present, calls raise GstmError.

Names follow the C ABI (gstm_create, gstm_launch, gstm_stats, ...).  The
``Gstm`` class is a convenience wrapper that owns a handle; PyTorch is used
only for device memory (``attach_heap``) and streams (``set_stream``).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libgstm.so")

WL_RA, WL_BANK, WL_HT, WL_EB, WL_KM = 0, 1, 2, 3, 4
WORKLOADS = {"ra": WL_RA, "bank": WL_BANK, "ht": WL_HT, "eb": WL_EB, "km": WL_KM}
MODE_AUTO, MODE_HV, MODE_TBV, MODE_CGL, MODE_FGL = 0, 1, 2, 3, 4
MODE_HV_BACKOFF, MODE_VBV, MODE_HV_UNSORTED = 5, 6, 7
MODES = {"auto": MODE_AUTO, "hv": MODE_HV, "tbv": MODE_TBV, "cgl": MODE_CGL, "fgl": MODE_FGL,
         "hv_backoff": MODE_HV_BACKOFF, "vbv": MODE_VBV, "hv_unsorted": MODE_HV_UNSORTED}
MODE_NAMES = {v: k for k, v in MODES.items()}
RO_FLAG = 0x80000000
API_VERSION = 2          # include/gstm.h GSTM_API_VERSION these structs mirror

STATUS = {0: "GSTM_OK", -1: "GSTM_EINVAL", -2: "GSTM_ENOMEM", -3: "GSTM_ECUDA", -4: "GSTM_ELOGOVF",
          -5: "GSTM_EOVERFLOW", -6: "GSTM_ETIMEOUT", -7: "GSTM_EBUSY", -8: "GSTM_ENODEV"}

# every symbol include/gstm.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "gstm_create", "gstm_create_ex", "gstm_flags", "gstm_destroy", "gstm_last_error", "gstm_api_version", "gstm_default_params",
    "gstm_set_params", "gstm_get_params", "gstm_set_mode", "gstm_set_stream", "gstm_attach_heap",
    "gstm_heap_words", "gstm_heap_ptr", "gstm_init_heap", "gstm_write_heap", "gstm_read_heap",
    "gstm_read_locks", "gstm_read_clock", "gstm_reset_meta", "gstm_set_clock", "gstm_launch", "gstm_stats",
    "gstm_stats_total", "gstm_reset_stats_total", "gstm_phase_cycles",
    "gstm_read_tx_log", "gstm_run_host", "gstm_descr_words", "gstm_dump_descr", "gstm_script",
    "gstm_lock_log", "gstm_ubench", "gstm_km_recenter", "gstm_run_host_async", "gstm_join", "gstm_sync",
    "gstm_ubench_mix", "gstm_script_ex",
]


class GstmError(RuntimeError):
    pass


class gstm_params_t(C.Structure):
    _fields_ = [
        ("n_reads", C.c_uint32), ("n_writes", C.c_uint32), ("ra_kind", C.c_uint32),
        ("n_words", C.c_uint64), ("n_accesses", C.c_uint32), ("ht_buckets", C.c_uint32),
        ("ht_lookup_pct", C.c_uint32), ("ht_key_range", C.c_uint64), ("km_clusters", C.c_uint32),
        ("km_dims", C.c_uint32), ("prelock_vbv", C.c_uint32), ("k_lock", C.c_uint32),
        ("backoff_ns", C.c_uint32), ("verify", C.c_uint32), ("block_threads", C.c_uint32),
        ("spin_cap", C.c_uint32), ("timeout_ms", C.c_uint32), ("snapshot_reuse", C.c_uint32),
        ("lock_pipeline", C.c_uint32), ("max_threads", C.c_uint32), ("lock_shift", C.c_uint32),
        ("shard_bits", C.c_uint32), ("shard", C.c_uint32), ("km_stride", C.c_uint32),
        ("km_assign", C.c_uint32), ("l2_persist_locks", C.c_uint32), ("ra_partition", C.c_uint32),
        ("body_rounds", C.c_uint32), ("pipeline_max_locks", C.c_uint32), ("lock_log_at_commit", C.c_uint32),
        ("serial_after", C.c_uint32), ("serial_commits", C.c_uint32), ("lock_pipeline_gated", C.c_uint32),
        ("pipeline_abort", C.c_uint32),
    ]


class gstm_stats_t(C.Structure):
    _fields_ = [
        ("commits", C.c_uint64), ("commits_ro", C.c_uint64), ("aborts", C.c_uint64),
        ("aborts_opacity", C.c_uint64), ("aborts_prevbv", C.c_uint64), ("aborts_tbv", C.c_uint64),
        ("aborts_commit_vbv", C.c_uint64), ("aborts_lock", C.c_uint64), ("lock_retries", C.c_uint64),
        ("postvalidations", C.c_uint64), ("vbv_runs", C.c_uint64), ("spins", C.c_uint64),
        ("attempts", C.c_uint64), ("errors", C.c_uint64), ("clock_begin", C.c_uint64),
        ("clock_end", C.c_uint64), ("elapsed_ms", C.c_double), ("tx_per_s", C.c_double),
        ("abort_ratio", C.c_double), ("status", C.c_int32), ("mode_used", C.c_int32),
        ("clock_slot", C.c_int32), ("pipelined_rounds", C.c_uint64),
        ("reads_update", C.c_uint64), ("reads_ro", C.c_uint64), ("writes_update", C.c_uint64),
        ("locks_update", C.c_uint64), ("serial_runs", C.c_uint64),
    ]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


_libs: dict = {}


def lib_path(flavour: str = "") -> str:
    """lib/libgstm.so, or lib/libgstm_<flavour>.so for a build flavour
    (build.FLAVOURS: "strict" PTX fences, "hlog" hashed lock logs, "phase"
    Figure-5 phase timing)."""
    return os.path.join(_HERE, "lib", f"libgstm_{flavour}.so" if flavour else "libgstm.so")


def lib(flavour: str = ""):
    """Load libgstm.so or a flavour of it (fails loudly if it was not built;
    there is no CPU fallback)."""
    if flavour not in _libs:
        path = lib_path(flavour)
        if not os.path.exists(path):
            raise GstmError(f"{path} missing: run `python -m paper_conf_cgo_xuwglgq14_b200.build"
                            f"{' --flavour ' + flavour if flavour else ''}` (there is no CPU fallback)")
        L = C.CDLL(path)
        P, V = C.POINTER, C.c_void_p
        u32, u64, i32 = C.c_uint32, C.c_uint64, C.c_int
        sig = {
            "gstm_create": (V, [u64, u32]),
            "gstm_create_ex": (V, [u64, u32, u32]),
            "gstm_flags": (u32, [V]),
            "gstm_destroy": (None, [V]),
            "gstm_last_error": (C.c_char_p, []),
            "gstm_api_version": (i32, []),
            "gstm_default_params": (i32, [i32, P(gstm_params_t)]),
            "gstm_set_params": (i32, [V, P(gstm_params_t)]),
            "gstm_get_params": (i32, [V, P(gstm_params_t)]),
            "gstm_set_mode": (i32, [V, i32]),
            "gstm_set_stream": (i32, [V, V]),
            "gstm_attach_heap": (i32, [V, V, u64]),
            "gstm_heap_words": (u64, [V]),
            "gstm_heap_ptr": (V, [V]),
            "gstm_init_heap": (i32, [V, i32]),
            "gstm_km_recenter": (i32, [V]),
            "gstm_run_host_async": (i32, [V, i32, V, V, u64, u64, u32, u64]),
            "gstm_sync": (i32, [V]),
            "gstm_join": (i32, [V]),
            "gstm_write_heap": (i32, [V, V, u64, u64]),
            "gstm_read_heap": (i32, [V, V, u64, u64]),
            "gstm_read_locks": (i32, [V, V, u64]),
            "gstm_read_clock": (i32, [V, P(u64)]),
            "gstm_reset_meta": (i32, [V]),
            "gstm_set_clock": (i32, [V, u64]),
            "gstm_launch": (i32, [V, i32, u64, u32, u64]),
            "gstm_stats": (i32, [V, P(gstm_stats_t)]),
            "gstm_stats_total": (i32, [V, P(gstm_stats_t), P(u64)]),
            "gstm_reset_stats_total": (i32, [V]),
            "gstm_phase_cycles": (i32, [V, V, i32]),
            "gstm_read_tx_log": (i32, [V, V, V, u64]),
            "gstm_run_host": (i32, [V, i32, V, V, u64, u64, u32, u64, P(gstm_stats_t)]),
            "gstm_descr_words": (i32, [V, i32]),
            "gstm_dump_descr": (i32, [V, i32, u64, u32, u64, V, u32]),
            "gstm_script": (i32, [V, i32, i32, V, i32, V, i32]),
            "gstm_script_ex": (i32, [V, i32, i32, V, i32, V, i32, i32]),
            "gstm_lock_log": (i32, [V, i32, V, i32]),
            "gstm_ubench": (i32, [i32, u64, u64, u32, P(C.c_double), P(C.c_double)]),
            "gstm_ubench_mix": (i32, [V, u64, V, u32, u64, u32, u32, P(C.c_double), P(C.c_double)]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        if L.gstm_api_version() != API_VERSION:
            # the ctypes structs below mirror include/gstm.h of this version
            raise GstmError(f"{path}: API version {L.gstm_api_version()}, binding expects {API_VERSION} "
                            "(rebuild: python -m paper_conf_cgo_xuwglgq14_b200.build --force)")
        _libs[flavour] = L
    return _libs[flavour]


def last_error(L=None) -> str:
    return (L or lib()).gstm_last_error().decode()


def _check(rc: int, what: str, L=None) -> int:
    if rc < 0:
        raise GstmError(f"{what}: {STATUS.get(rc, rc)}: {last_error(L)}")
    return rc


def _ptr(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(C.c_void_p)


# ---- function-style API with the C names --------------------------------
CREATE_PAIRED = 1


def gstm_create(heap_words: int, lock_table_bits: int, flags: int = 0, L=None):
    L = L or lib()
    h = L.gstm_create_ex(heap_words, lock_table_bits, flags) if flags else L.gstm_create(heap_words, lock_table_bits)
    if not h:
        raise GstmError(f"gstm_create: {last_error(L)}")
    return h


def gstm_destroy(h, L=None) -> None:
    (L or lib()).gstm_destroy(h)


def gstm_default_params(workload, L=None) -> gstm_params_t:
    p = gstm_params_t()
    _check((L or lib()).gstm_default_params(_wl(workload), C.byref(p)), "gstm_default_params", L)
    return p


def gstm_set_params(h, p: gstm_params_t, L=None) -> None:
    _check((L or lib()).gstm_set_params(h, C.byref(p)), "gstm_set_params", L)


def gstm_set_mode(h, mode, L=None) -> None:
    _check((L or lib()).gstm_set_mode(h, _mode(mode)), "gstm_set_mode", L)


def gstm_launch(h, workload, n_threads: int, tx_per_thread: int, seed: int, L=None) -> None:
    _check((L or lib()).gstm_launch(h, _wl(workload), n_threads, tx_per_thread, seed), "gstm_launch", L)


def gstm_stats(h, check: bool = True, L=None) -> gstm_stats_t:
    s = gstm_stats_t()
    rc = (L or lib()).gstm_stats(h, C.byref(s))
    if check:
        _check(rc, "gstm_stats", L)
    return s


def _wl(w) -> int:
    return WORKLOADS[w] if isinstance(w, str) else int(w)


def _mode(m) -> int:
    return MODES[m] if isinstance(m, str) else int(m)


class Gstm:
    """Owning wrapper of a gstm_t handle."""

    def __init__(self, heap_words: int, lock_table_bits: int, paired: bool = False, flavour: str = ""):
        """paired=True: GSTM_CREATE_PAIRED layout (each word next to its
        version lock; needs heap_words <= 2^lock_table_bits).  flavour: a
        build flavour of the library (lib_path)."""
        self.h = None
        self._L = lib(flavour)
        self.flavour = flavour
        self.h = gstm_create(heap_words, lock_table_bits, CREATE_PAIRED if paired else 0, L=self._L)
        self.bits = lock_table_bits
        self.paired = paired
        self._attached = None

    def close(self) -> None:
        if self.h:
            gstm_destroy(self.h, L=self._L)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # configuration
    def params(self) -> gstm_params_t:
        p = gstm_params_t()
        _check(self._L.gstm_get_params(self.h, C.byref(p)), "gstm_get_params", self._L)
        return p

    def set_params(self, p: gstm_params_t | None = None, **kw) -> gstm_params_t:
        if p is None:
            p = self.params()
        for k, v in kw.items():
            if not hasattr(p, k):
                raise KeyError(k)
            setattr(p, k, int(v))
        gstm_set_params(self.h, p, L=self._L)
        return p

    def set_workload_defaults(self, workload, **kw) -> gstm_params_t:
        p = gstm_default_params(workload, L=self._L)
        return self.set_params(p, **kw)

    def set_mode(self, mode) -> None:
        gstm_set_mode(self.h, mode, L=self._L)

    def set_stream(self, stream) -> None:
        """stream: a torch.cuda.Stream, an int handle, or None (the handle's
        private stream).  torch's legacy default stream has handle 0; it is
        passed as cudaStreamLegacy (1) so work really lands on it."""
        if stream is None:
            _check(self._L.gstm_set_stream(self.h, None), "gstm_set_stream", self._L)
            return
        ptr = int(getattr(stream, "cuda_stream", stream))
        _check(self._L.gstm_set_stream(self.h, C.c_void_p(ptr if ptr else 1)), "gstm_set_stream", self._L)

    def attach_heap(self, tensor) -> None:
        """Use a torch CUDA tensor (int32/uint32 storage) as the heap."""
        if tensor is None:
            _check(self._L.gstm_attach_heap(self.h, None, 0), "gstm_attach_heap", self._L)
            self._attached = None
            return
        assert tensor.is_cuda and tensor.is_contiguous() and tensor.element_size() == 4
        _check(self._L.gstm_attach_heap(self.h, C.c_void_p(tensor.data_ptr()), tensor.numel()), "gstm_attach_heap", self._L)
        self._attached = tensor

    @property
    def heap_words(self) -> int:
        return int(self._L.gstm_heap_words(self.h))

    # data
    def init_heap(self, workload) -> None:
        _check(self._L.gstm_init_heap(self.h, _wl(workload)), "gstm_init_heap", self._L)

    def km_recenter(self) -> None:
        """End of a k-means iteration (params.km_assign = 1): centroids =
        floor means of their records, records zeroed (asynchronous)."""
        _check(self._L.gstm_km_recenter(self.h), "gstm_km_recenter", self._L)

    def write_heap(self, a: np.ndarray, offset: int = 0) -> None:
        a = np.ascontiguousarray(a, dtype=np.uint32)
        _check(self._L.gstm_write_heap(self.h, _ptr(a), offset, a.size), "gstm_write_heap", self._L)

    def read_heap(self, words: int | None = None, offset: int = 0) -> np.ndarray:
        n = self.heap_words - offset if words is None else words
        out = np.empty(n, dtype=np.uint32)
        _check(self._L.gstm_read_heap(self.h, _ptr(out), offset, n), "gstm_read_heap", self._L)
        return out

    def read_locks(self, n: int | None = None) -> np.ndarray:
        n = (1 << self.bits) if n is None else n
        out = np.empty(n, dtype=np.uint32)
        _check(self._L.gstm_read_locks(self.h, _ptr(out), n), "gstm_read_locks", self._L)
        return out

    def read_clock(self) -> int:
        c = C.c_uint64(0)
        _check(self._L.gstm_read_clock(self.h, C.byref(c)), "gstm_read_clock", self._L)
        return c.value

    def reset_meta(self) -> None:
        _check(self._L.gstm_reset_meta(self.h), "gstm_reset_meta", self._L)

    def set_clock(self, value: int) -> None:
        _check(self._L.gstm_set_clock(self.h, value), "gstm_set_clock", self._L)

    # hot path
    def launch(self, workload, n_threads: int, tx_per_thread: int, seed: int) -> None:
        gstm_launch(self.h, workload, n_threads, tx_per_thread, seed, L=self._L)

    def stats(self, check: bool = True) -> gstm_stats_t:
        return gstm_stats(self.h, check, L=self._L)

    def stats_total(self, check: bool = True):
        """(stats summed since reset_stats_total, number of launches)"""
        s = gstm_stats_t()
        n = C.c_uint64(0)
        rc = self._L.gstm_stats_total(self.h, C.byref(s), C.byref(n))
        if check:
            _check(rc, "gstm_stats_total", self._L)
        return s, n.value

    # Figure 5's categories, in gstm_phase_cycles order
    PHASES = ["native", "init", "buffering", "consistency", "locks", "commit", "aborted", "other"]

    def phase_cycles(self) -> dict:
        """Figure 5 breakdown: SM cycles summed over lanes per category since
        reset_stats_total (needs the "phase" flavour: Gstm(..., flavour="phase"))."""
        out = np.zeros(8, dtype=np.uint64)
        _check(self._L.gstm_phase_cycles(self.h, _ptr(out), 8), "gstm_phase_cycles", self._L)
        return {k: int(out[i]) for i, k in enumerate(self.PHASES)}

    def reset_stats_total(self) -> None:
        _check(self._L.gstm_reset_stats_total(self.h), "gstm_reset_stats_total", self._L)

    def run(self, workload, n_threads: int, tx_per_thread: int, seed: int, check: bool = True) -> gstm_stats_t:
        self.launch(workload, n_threads, tx_per_thread, seed)
        return self.stats(check)

    def read_tx_log(self, n: int):
        st = np.empty(n, dtype=np.uint32)
        rs = np.empty(n, dtype=np.uint32)
        _check(self._L.gstm_read_tx_log(self.h, _ptr(st), _ptr(rs), n), "gstm_read_tx_log", self._L)
        return st, rs

    def run_host(self, workload, heap_in: np.ndarray, heap_out: np.ndarray, n_threads: int,
                 tx_per_thread: int, seed: int) -> gstm_stats_t:
        s = gstm_stats_t()
        assert heap_in.dtype == np.uint32 and heap_out.dtype == np.uint32 and heap_in.size == heap_out.size
        _check(self._L.gstm_run_host(self.h, _wl(workload), _ptr(heap_in), _ptr(heap_out), heap_in.size,
                                   n_threads, tx_per_thread, seed, C.byref(s)), "gstm_run_host", self._L)
        return s

    def run_host_async(self, workload, heap_in: np.ndarray, heap_out: np.ndarray, n_threads: int,
                       tx_per_thread: int, seed: int) -> None:
        """Enqueue copy-in, launch and copy-out; heap_out is valid after sync()."""
        assert heap_in.dtype == np.uint32 and heap_out.dtype == np.uint32 and heap_in.size == heap_out.size
        _check(self._L.gstm_run_host_async(self.h, _wl(workload), _ptr(heap_in), _ptr(heap_out), heap_in.size,
                                         n_threads, tx_per_thread, seed), "gstm_run_host_async", self._L)

    def join(self) -> int:
        """Make the handle's stream wait (device-side) for the last run_host_async copy-out."""
        return _check(self._L.gstm_join(self.h), "gstm_join", self._L)

    def sync(self) -> int:
        return _check(self._L.gstm_sync(self.h), "gstm_sync", self._L)

    # tests / measurement
    def descr_words(self, workload) -> int:
        return _check(self._L.gstm_descr_words(self.h, _wl(workload)), "gstm_descr_words", self._L)

    def dump_descr(self, workload, n_threads: int, tx_per_thread: int, seed: int, wpt: int | None = None):
        wpt = self.descr_words(workload) if wpt is None else wpt
        out = np.empty(n_threads * tx_per_thread * wpt, dtype=np.uint32)
        _check(self._L.gstm_dump_descr(self.h, _wl(workload), n_threads, tx_per_thread, seed, _ptr(out), wpt),
               "gstm_dump_descr", self._L)
        return out.reshape(n_threads * tx_per_thread, wpt)

    def script(self, mode, ops, n_tx: int = 4, prelock_vbv: bool = True, log_policy: int = 0) -> np.ndarray:
        """Scripted interleaving (gstm_script_ex); log_policy 0 local, 1
        register-resident, 2 shared-memory logs."""
        ops = np.ascontiguousarray(np.asarray(ops, dtype=np.uint32).reshape(-1, 4))
        out = np.zeros_like(ops)
        _check(self._L.gstm_script_ex(self.h, _mode(mode), 1 if prelock_vbv else 0, _ptr(ops), ops.shape[0],
                                    _ptr(out), n_tx, log_policy), "gstm_script_ex", self._L)
        return out


def gstm_lock_log(entries, variant: int = 0, flavour: str = "") -> np.ndarray:
    e = np.ascontiguousarray(np.asarray(entries, dtype=np.uint32))
    out = np.zeros(256, dtype=np.uint32)
    L = lib(flavour)
    n = _check(L.gstm_lock_log(_ptr(e), e.size, _ptr(out), variant), "gstm_lock_log", L)
    return out[:n].copy()


def gstm_ubench_mix(h, words: int, prog, n_tx: int, threads: int, block: int = 256, L=None):
    """Op-mix roof (include/gstm.h): returns (tx/s, ms).  Clobbers the
    handle's heap, lock table and clock."""
    pr = np.ascontiguousarray(np.asarray(prog, dtype=np.uint32))
    tps = C.c_double(0)
    ms = C.c_double(0)
    L = L or lib()
    _check(L.gstm_ubench_mix(h, words, _ptr(pr), pr.size, n_tx, threads, block, C.byref(tps), C.byref(ms)),
           "gstm_ubench_mix", L)
    return tps.value, ms.value


def gstm_ubench(kind: int, table_bytes: int, n_ops: int, threads: int):
    ops = C.c_double(0)
    ms = C.c_double(0)
    _check(lib().gstm_ubench(kind, table_bytes, n_ops, threads, C.byref(ops), C.byref(ms)), "gstm_ubench")
    return ops.value, ms.value
