/*
 * gstm.h -- C ABI of the B200-native GPU-STM hot path.
 *
 * Implements the per-thread transactional memory of Xu et al., "Software
 * Transactional Memory for GPU Architectures", CGO 2014 (the paper text is
 * cited as P:<line>; Algorithm 3 lines as A3.l<k>).  The host side mirrors the
 * paper's usage (Figure 1): STM_STARTUP / STM_SHUTDOWN allocate and
 * free the global metadata (gstm_create / gstm_destroy), a transactional
 * kernel runs every thread's transactions (gstm_launch), and the statistics
 * are read back (gstm_stats).
 *
 * Conventions (all functions):
 *   - extern "C", plain pointers and integers; no C++ types, no exceptions.
 *   - Functions returning int return GSTM_OK (0) or a negative gstm_status;
 *     the message for the last failure on the calling thread is in
 *     gstm_last_error().  The library never calls exit() or abort().
 *   - "device pointer" = CUDA global memory of the current device;
 *     "host pointer" = ordinary (optionally pinned) CPU memory.
 *   - Work is enqueued on the handle's stream (gstm_set_stream; default: a
 *     private non-blocking stream).  gstm_launch is asynchronous; gstm_stats
 *     and every gstm_read_* call synchronise that stream.
 *   - A handle is not thread-safe; use one handle per host thread.
 *   - Heap words are uint32.  Word w is protected by version lock
 *     w mod 2^lock_table_bits (reading Q2 in DESIGN.md §4).
 */
#ifndef GSTM_H
#define GSTM_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* 2: gstm_params_t gained serial_after, serial_commits, lock_pipeline_gated,
 *    pipeline_abort and
 *    gstm_stats_t gained serial_runs (appended; the structs are passed by
 *    pointer, so a client built against version 1 must be rebuilt) */
#define GSTM_API_VERSION 2

typedef struct gstm_handle gstm_t;   /* opaque; owns the lock table, clock, stats, logs, heap */

enum gstm_status {
    GSTM_OK = 0,
    GSTM_EINVAL = -1,     /* bad argument or workload parameters                  */
    GSTM_ENOMEM = -2,     /* device allocation failed                             */
    GSTM_ECUDA = -3,      /* CUDA runtime error (message in gstm_last_error)      */
    GSTM_ELOGOVF = -4,    /* a transaction needed more log entries than compiled  */
    GSTM_EOVERFLOW = -5,  /* stamp space: n_threads * tx_per_thread >= 2^31       */
    GSTM_ETIMEOUT = -6,   /* the device watchdog stopped the launch               */
    GSTM_EBUSY = -7,      /* no launch to report on                               */
    GSTM_ENODEV = -8      /* no CUDA device                                       */
};

/* Workloads.  RA = random array (Figure 1);
 * BANK = two-account transfer; HT = chained hash table, set semantics;
 * EB = EigenBench-style alternating read/write; KM = k-means
 * cluster-update transaction (STAMP kmeans). */
enum gstm_workload { GSTM_WL_RA = 0, GSTM_WL_BANK = 1, GSTM_WL_HT = 2, GSTM_WL_EB = 3, GSTM_WL_KM = 4 };

/* Concurrency control:
 *   AUTO = STM-Optimized: HV when the workload's shared words exceed the
 *          number of version locks, else TBV;
 *   HV   = STM-HV-Sorting (hierarchical validation);
 *   TBV  = STM-TBV-Sorting (timestamp validation only);
 *   CGL  = coarse-grain lock baseline, Scheme #3 of Algorithm 1;
 *   FGL  = fine-grain lock baseline (sorted per-stripe locks; P:288 notes the
 *          paper did not implement it);
 *   HV_BACKOFF = STM-HV-Backoff: HV with locks in encounter order;
 *          the first lock attempt is made by all lanes of a warp in parallel,
 *          lanes that failed retry one at a time while the others wait;
 *   VBV  = STM-VBV: NOrec-like value-based validation behind
 *          one global sequence lock, writers serialised (no lock table);
 *   HV_UNSORTED = ablation: HV with locks in encounter order and the parallel
 *          retry of HV -- exposed to the intra-warp livelock of P:63 (ends in
 *          GSTM_ETIMEOUT when it happens; for demonstrations only). */
enum gstm_mode {
    GSTM_MODE_AUTO = 0, GSTM_MODE_HV = 1, GSTM_MODE_TBV = 2, GSTM_MODE_CGL = 3, GSTM_MODE_FGL = 4,
    GSTM_MODE_HV_BACKOFF = 5, GSTM_MODE_VBV = 6, GSTM_MODE_HV_UNSORTED = 7
};

typedef struct {
    /* workload shape (which fields apply: DESIGN.md §3.3) */
    uint32_t n_reads;        /* RA: reads per tx (kind 0: <= 8; kind 1: <= 16)          */
    uint32_t n_writes;       /* RA kind 0: writes per tx (<= 8)                          */
    uint32_t ra_kind;        /* RA: 0 reads-then-writes, 1 increment each word read     */
    uint64_t n_words;        /* RA/BANK/EB: words addressed, [0, n_words) (EB: hot set) */
    uint32_t n_accesses;     /* EB: accesses per tx, alternating r/w (<= 64)            */
    uint32_t ht_buckets;     /* HT: bucket heads (power of two)                         */
    uint32_t ht_lookup_pct;  /* HT: percentage of lookups (rest inserts)                */
    uint64_t ht_key_range;   /* HT: keys uniform in [1, ht_key_range]                   */
    uint32_t km_clusters;    /* KM: cluster records                                     */
    uint32_t km_dims;        /* KM: features per point (<= 16)                          */
    /* runtime knobs */
    uint32_t prelock_vbv;    /* HV: value-validate before locking (A3.l71); 1, HT 0    */
    uint32_t k_lock;         /* lock-acquisition rounds before abort; 0 = inf   */
    uint32_t backoff_ns;     /* warp-uniform backoff after an abort; 0 = none           */
    uint32_t verify;         /* record per-tx stamp and result (gstm_read_tx_log)       */
    uint32_t block_threads;  /* CUDA block size (multiple of 32, <= 256), default 256   */
    uint32_t spin_cap;       /* bound on lock spins / PostValidation restarts; past it */
                             /*    the transaction re-executes (Q25, Q38).  0 = 65536; */
                             /*    default 65536 (bank, RA: 1)                         */
    uint32_t timeout_ms;     /* device watchdog per launch, default 60000               */
    uint32_t snapshot_reuse; /* 1: a warp that just committed starts its next txs at   */
                             /*    the clock value after its own commits instead of   */
                             /*    re-reading g_clock (A3.l4); default 1               */
    uint32_t lock_pipeline;  /* N > 0: the first lock-acquisition round of each of a   */
                             /*    transaction's first N executions issues all atom.or */
                             /*    at once; every other round is      */
                             /*    sequential in ascending id (every round after a     */
                             /*    failed one, for any k_lock; progress is kept for    */
                             /*    any N).  0: always sequential.  Local-memory        */
                             /*    logs pipeline only logs of <= 8 locks.              */
                             /*    Default 1 (RA: 0; EB: 16)                           */
    uint32_t max_threads;    /* concurrency cap: at most this many CUDA threads run the */
                             /*    n_threads STM threads; 0 = the workload's default:  */
                             /*    what fits on the chip, at most 16 resident warps   */
                             /*    per SM for bank and 8 for k-means */
    uint32_t lock_shift;     /* stripe size 2^lock_shift words per version lock      */
                             /*    (lock = (word >> shift) mod 2^bits); default 0     */
    uint32_t shard_bits;     /* HT key partition: G = 2^shard_bits     */
                             /*    shards (<= 8 bits); 0 = no partition               */
    uint32_t shard;          /* HT: this handle's shard g < G; it runs only keys     */
                             /*    whose mix64 top shard_bits bits equal g            */
    uint32_t km_stride;      /* KM: words per cluster record (>= km_dims + 1; 0 =    */
                             /*    km_dims + 1).  32 with lock_shift 5 = one version */
                             /*    lock per record                        */
    uint32_t km_assign;      /* KM: 1 = a full k-means iteration:   */
                             /*    each point joins its NEAREST centroid (exact int  */
                             /*    squared distance, ties -> lowest index) from the  */
                             /*    km_clusters x km_dims uint32 table stored after   */
                             /*    the records; gstm_launch runs the assignment pass */
                             /*    before the update transactions.  Table <= 64 KiB  */
    uint32_t l2_persist_locks; /* 1: the launch marks the version-lock table (split   */
                             /*    layout) as persisting in L2 (an access-policy      */
                             /*    window on the handle's stream, cleared after the   */
                             /*    launch; the device-wide L2 set-aside is reference- */
                             /*    counted per device and released when the last     */
                             /*    handle using it launches without it or is          */
                             /*    destroyed), so random heap lines streaming from    */
                             /*    HBM do not evict the locks (EB with a hot set      */
                             /*    larger than L2).  Default 0 (EB: 1)                */
    uint32_t ra_partition;   /* RA: k > 0 = STM thread t addresses only its own words */
                             /*    [t*k, t*k + k) (disjoint access sets: a unique,    */
                             /*    conflict-free result); needs        */
                             /*    n_threads * k <= n_words.  Default 0               */
    uint32_t body_rounds;    /* STM modes: a lane whose transaction committed read-  */
                             /*    only starts its next one in the same warp         */
                             /*    iteration, up to this many bodies per iteration   */
                             /*    (DESIGN.md §6.11); 0 or 1 = one body per          */
                             /*    iteration.  Default 1 (HT: see DESIGN.md)         */
    uint32_t pipeline_max_locks; /* local-memory lock logs: the pipelined first round */
                             /*    (lock_pipeline) is used only for logs of at most  */
                             /*    this many locks (issued 8 atom.or at a time);     */
                             /*    0 = 8.  Default 8 (EB: 16)                        */
    uint32_t lock_log_at_commit; /* 1: a read's lock enters the sorted lock log when   */
                             /*    the transaction reaches TXCommit with a write-set */
                             /*    instead of at the read (P:113's encounter time):  */
                             /*    the same sorted log and acquisition order, no     */
                             /*    sorting work for read-only transactions           */
                             /*    (DESIGN.md §6.15).  Default 0                     */
    uint32_t serial_after;   /* contention manager (the adaptive    */
                             /*    transaction scheduling P:313 and P:317 leave to   */
                             /*    future work): a transaction whose executions      */
                             /*    aborted >= serial_after times while g_clock       */
                             /*    advanced by < serial_commits per abort, and whose */
                             /*    attempts took longer per GPU-wide commit than a   */
                             /*    serial owner's execution takes (measured online;  */
                             /*    none yet: qualify), takes a ticket; while tickets */
                             /*    are outstanding no other transaction starts (one  */
                             /*    that aborted before and passes the same time test */
                             /*    joins the queue), and the holders run one at a    */
                             /*    time in ticket order (FIFO), each IRREVOCABLY: in */
                             /*    place, under encounter-time version locks,        */
                             /*    stamped while it holds them all -- serialised     */
                             /*    like an A3 commit (gstm/tx_irr.cuh).  Kernels of  */
                             /*    RA, KM and EB with A > 16 only (bank, HT and EB   */
                             /*    A <= 16 ignore it).  0 = off.  Default 0 (EB: 4)  */
    uint32_t serial_commits; /*    see serial_after; 0 = 4.  Default 4                */
    uint32_t lock_pipeline_gated; /* 1: a transaction's pipelined lock round (see    */
                             /*    lock_pipeline) whose local/shared-memory lock log */
                             /*    is longer than pipeline_max_locks takes its LOWEST */
                             /*    lock alone first (held: the round fails having    */
                             /*    touched nothing else) and then every other lock   */
                             /*    at once.  0: such logs take the  */
                             /*    sequential round.  Default 0 (KM: 1)              */
    uint32_t pipeline_abort; /* N > 0: a pipelined lock round that finds a lock     */
                             /*    held aborts the execution (re-executed with fresh */
                             /*    reads) instead of retrying sequential rounds, and */
                             /*    a warp pipelines only while its recent abort rate */
                             /*    (EMA x 256 over its lanes' executions) is below   */
                             /*    N; lock_pipeline still bounds a transaction's     */
                             /*    pipelined executions (progress).  */
                             /*    Applied only where it pays: a shared footprint   */
                             /*    larger than L2 and >= 1 lock per 4 words (else   */
                             /*    the launch runs sequential rounds); there the    */
                             /*    launch also skips the optional pre-lock VBV      */
                             /*    (A3.l71).  Default 0                             */
                             /*    (EB: 100, with lock_pipeline 16 and              */
                             /*    pipeline_max_locks 16)                            */
} gstm_params_t;

typedef struct {
    uint64_t commits;            /* committed update transactions (stamped, A3.l83)     */
    uint64_t commits_ro;         /* committed read-only transactions (A3.l68)           */
    uint64_t aborts;             /* sum of the abort causes below                       */
    uint64_t aborts_opacity;     /* isOpaque became false during execution (A3.l33)     */
    uint64_t aborts_prevbv;      /* pre-lock VBV failed (A3.l71-72)                     */
    uint64_t aborts_tbv;         /* TBV mode: version newer than snapshot at commit     */
    uint64_t aborts_commit_vbv;  /* VBV under locks failed (A3.l76-78)                  */
    uint64_t aborts_lock;        /* k_lock acquisition rounds exhausted         */
    uint64_t lock_retries;       /* failed lock-acquisition rounds (A3.l73-74)          */
    uint64_t postvalidations;    /* PostValidation calls (A3.l32)                       */
    uint64_t vbv_runs;           /* VBV passes (pre-lock, under locks, post-validation) */
    uint64_t spins;              /* lock-word re-reads while locked (A3.l27-29)         */
    uint64_t attempts;           /* transaction executions (commits + aborts)           */
    uint64_t errors;             /* transactions dropped on log overflow                */
    uint64_t clock_begin;        /* g_clock at launch start                             */
    uint64_t clock_end;          /* g_clock at launch end                               */
    double elapsed_ms;           /* device time of the launch (CUDA events)             */
    double tx_per_s;             /* (commits + commits_ro) / elapsed                    */
    double abort_ratio;          /* aborts / (aborts + commits + commits_ro)            */
    int32_t status;              /* GSTM_OK, GSTM_ELOGOVF, GSTM_ETIMEOUT                */
    int32_t mode_used;           /* gstm_mode actually run (AUTO resolved)              */
    int32_t clock_slot;          /* metadata line chosen for g_clock (-1: fixed word)   */
    uint64_t pipelined_rounds;   /* lock rounds that issued every atom.or at once       */
                                 /*    (lock_pipeline): only the first  */
                                 /*    round of an execution may be pipelined, so this  */
                                 /*    is <= the executions that reached TXCommit's     */
                                 /*    lock step (Q15, Q37)                             */
    /* log sizes summed over the COMMITTED executions of the STM modes (0 for
     * CGL/FGL/VBV): the per-transaction op counts of the op-mix roof
     * */
    uint64_t reads_update;       /* read-set entries (memory reads) of update commits  */
    uint64_t reads_ro;           /* read-set entries of read-only commits              */
    uint64_t writes_update;      /* write-set entries of update commits                */
    uint64_t locks_update;       /* lock-log entries (locks taken) of update commits   */
    uint64_t serial_runs;        /* executions run as the serial-ticket owner          */
                                 /*    (serial_after)                  */
} gstm_stats_t;

/* ---- lifecycle (STM_STARTUP / STM_SHUTDOWN) ------------------ */
/* Allocates a heap of heap_words uint32 (zeroed), a table of
 * 2^lock_table_bits version locks (0 <= bits <= 30, zeroed), the global clock
 * (0) and statistics.  For tables of >= 2^14 locks it places g_clock on the
 * fastest of 256 candidate L2 lines, measured with a short probe kernel
 * (~120 ms; GSTM_CLOCK_SLOT=k forces line k).  Synchronous.
 * Returns NULL on error (gstm_last_error). */
gstm_t* gstm_create(uint64_t heap_words, uint32_t lock_table_bits);
/* flags for gstm_create_ex */
#define GSTM_CREATE_PAIRED 1u
/* As gstm_create, with layout flags.  GSTM_CREATE_PAIRED stores word w and
 * its version lock w side by side in one 8-byte slot (value low half, lock
 * high half) so a read, a lock acquisition (which also
 * returns the value) and a write-back + unlock are one memory access each.
 * Requires 1 <= heap_words <= 2^lock_table_bits (one lock per word, stripe
 * 1).  The heap is still addressed by word index through every call below;
 * gstm_attach_heap is not available in this layout.  flags = 0 is
 * gstm_create (the paper's separate lock table). */
gstm_t* gstm_create_ex(uint64_t heap_words, uint32_t lock_table_bits, uint32_t flags);
uint32_t gstm_flags(const gstm_t* h);
/* Frees everything the handle owns (not an attached heap).  NULL is a no-op. */
void gstm_destroy(gstm_t* h);
/* Message of the last failure on this thread ("" if none).  Static storage. */
const char* gstm_last_error(void);
int gstm_api_version(void);

/* ---- configuration ----------------------------------------------------- */
/* Fills *out with the defaults for a workload (BASELINE-shaped sizes). */
int gstm_default_params(int workload, gstm_params_t* out);
int gstm_set_params(gstm_t* h, const gstm_params_t* p);
int gstm_get_params(const gstm_t* h, gstm_params_t* out);
int gstm_set_mode(gstm_t* h, int mode);
/* stream: a cudaStream_t (e.g. torch.cuda.current_stream().cuda_stream), or
 * cudaStreamLegacy ((void*)1) for the legacy default stream; NULL restores
 * the handle's private stream.  Borrowed, not destroyed. */
int gstm_set_stream(gstm_t* h, void* stream);
/* Use caller-owned device memory (>= words uint32, 4-byte aligned) as the
 * heap instead of the handle's own; borrowed: it must outlive the handle or
 * the next attach.  words == 0 or dev_ptr == NULL re-selects the own heap. */
int gstm_attach_heap(gstm_t* h, void* dev_ptr, uint64_t words);
uint64_t gstm_heap_words(const gstm_t* h);
/* device pointer of the current heap (for zero-copy views) */
void* gstm_heap_ptr(const gstm_t* h);

/* ---- data --------------------------------------------------------------- */
/* Device-side initial heap of a workload. */
int gstm_init_heap(gstm_t* h, int workload);
int gstm_write_heap(gstm_t* h, const uint32_t* host_src, uint64_t offset, uint64_t words);
int gstm_read_heap(gstm_t* h, uint32_t* host_dst, uint64_t offset, uint64_t words);
/* Version-lock table (2^bits uint32: LSB locked, bits 31..1 version). */
int gstm_read_locks(gstm_t* h, uint32_t* host_dst, uint64_t n);
int gstm_read_clock(gstm_t* h, uint64_t* out);
/* Zero the lock table and the clock (a new version epoch). */
int gstm_reset_meta(gstm_t* h);
/* Set the global clock (e.g. to start a scripted test at a given time);
 * value < 2^31 and >= every version in the lock table. */
int gstm_set_clock(gstm_t* h, uint64_t value);

/* ---- the hot path -------------------------------------------------------- */
/* Run n_threads STM threads, each executing tx_per_thread transactions of the
 * workload (tx_id = i*n_threads + t, generated from seed), under the
 * handle's mode, on the current heap.  Every transaction commits exactly once
 * (aborted attempts re-execute) unless the launch reports an error.  Stamps
 * of this launch are g_clock_begin+1 .. g_clock_end.  Asynchronous. */
int gstm_launch(gstm_t* h, int workload, uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed);
/* Synchronises, then reports the last launch.  Returns the launch status. */
int gstm_stats(gstm_t* h, gstm_stats_t* out);
/* Synchronises, then reports the counters summed over every launch since
 * gstm_reset_stats_total (or creation), so many launches can be enqueued
 * back to back without a host sync in between.  elapsed_ms / tx_per_s use
 * the device's %globaltimer between each launch's first and last kernel;
 * *launches (may be NULL) = number of launches summed.  Returns GSTM_OK or
 * the first error any of them reported. */
int gstm_stats_total(gstm_t* h, gstm_stats_t* out, uint64_t* launches);
int gstm_reset_stats_total(gstm_t* h);
/* Execution-time breakdown of the STM kernels since gstm_reset_stats_total
 * (the paper's Figure 5): SM cycles summed over every lane (each
 * lane times its own path) in Figure 5's categories: out[0] native code,
 * [1] transaction initialisation, [2] buffering (read/write/lock logging),
 * [3] consistency checking (lock-word checks, spins, PostValidation, VBV),
 * [4] acquiring/releasing locks, [5] committing (write-back, clock stamp),
 * [6] aborted transactions (every cycle of an execution that aborted), [7]
 * other (loop, refill, SIMT waiting outside a transaction).  Non-zero only in
 * the "phase" build flavour (lib/libgstm_phase.so, -DGSTM_PHASE_TIMING=1);
 * writes min(n, 16) entries. */
int gstm_phase_cycles(gstm_t* h, uint64_t* out, int n);
/* Verify mode (params.verify = 1): stamps[tx_id] = commit stamp - clock_begin
 * (1..C) for an update tx, or 0x80000000 | (snapshot - clock_begin) for a
 * read-only tx (linearised after that stamp); results[tx_id] = the
 * workload's observable result.  n = n_threads * tx_per_thread. */
int gstm_read_tx_log(gstm_t* h, uint32_t* stamps, uint32_t* results, uint64_t n);
/* End-to-end call with HOST buffers: copy heap_in (words) to the heap, launch,
 * copy the heap back to heap_out, synchronise and fill *stats (may be NULL).
 * heap_in/heap_out may alias; pinned memory gives full copy bandwidth. */
int gstm_run_host(gstm_t* h, int workload, const uint32_t* heap_in, uint32_t* heap_out, uint64_t words,
                  uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed, gstm_stats_t* stats);

/* End of a k-means iteration (params.km_assign = 1; STAMP kmeans):
 * for every cluster record with count > 0, centroid[c][d] = floor(sum_d /
 * count) (others keep their centroid), then every record is zeroed, ready
 * for the next iteration's gstm_launch.  Asynchronous on the handle's
 * stream.  GSTM_EINVAL without km_assign or if the heap cannot hold the
 * records and the centroid table.  gstm_init_heap(GSTM_WL_KM) with
 * km_assign fills the table with centroid word j = splitmix64(j) >> 56. */
int gstm_km_recenter(gstm_t* h);

/* As gstm_run_host without the final synchronisation, pipelined: the
 * host->device copy of heap_in goes on an internal copy-in stream into a
 * device staging buffer, the staging -> heap move (pack kernel on the paired
 * layout), the launch and the heap -> staging move go on the handle's stream,
 * and the device->host copy into heap_out on an internal copy-out stream,
 * ordered by events.  Consecutive calls on one handle therefore overlap step
 * k+1's copy-in and step k's copy-out with step k's / k+1's transactions
 * (DESIGN.md §7.1).  The first call after a gstm_join / gstm_sync starts
 * after all work already enqueued on the handle's stream.  Steps may be
 * chained in place (heap_in of a call overlapping heap_out of the previous
 * call): that call's copy-in then waits for the previous copy-out.  heap_in must stay
 * valid and heap_out must not be read until gstm_sync (or gstm_join followed
 * by a synchronisation of the handle's stream) returns; the stats of the
 * last launch are in gstm_stats after gstm_sync, the running totals in
 * gstm_stats_total.  words <= the heap size. */
int gstm_run_host_async(gstm_t* h, int workload, const uint32_t* heap_in, uint32_t* heap_out, uint64_t words,
                        uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed);
/* Make the handle's stream wait (on the device, without blocking the host)
 * for the last gstm_run_host_async copy-out, so an event recorded on that
 * stream afterwards follows every copy.  GSTM_OK; no-op without calls. */
int gstm_join(gstm_t* h);
/* gstm_join, then wait for everything enqueued on the handle's stream;
 * returns the status of the last launch (GSTM_OK if none). */
int gstm_sync(gstm_t* h);

/* ---- test and measurement entry points --------------------------------- */
/* Transaction descriptors as generated on the device:
 * host_out[(i*n_threads + t) * words_per_tx + k]; short descriptors are
 * zero-padded.  words_per_tx >= gstm_descr_words(h, workload). */
int gstm_descr_words(gstm_t* h, int workload);
int gstm_dump_descr(gstm_t* h, int workload, uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed,
                    uint32_t* host_out, uint32_t words_per_tx);
/* Scripted interleaving of up to 8 transactions on one device thread, on the
 * handle's heap, lock table and clock.  ops: n_ops x {op, slot, word, value}
 * with op 0 BEGIN, 1 READ, 2 WRITE, 3 COMMIT; out: n_ops x 4 words (format in
 * DESIGN.md §5.3).  mode: GSTM_MODE_HV or GSTM_MODE_TBV. */
int gstm_script(gstm_t* h, int mode, int prelock_vbv, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx);
/* As gstm_script, with op 4 READ2 {4, slot, word a, word b}: a batched read
 * of two words (the kernels' read_batch, reading Q35; out [value(a),
 * value(b), snapshot, isOpaque | PostValidation ran << 1]) and the log
 * storage of the transactions: log_policy 0 local memory (capacity 64 reads,
 * 64 writes, 128 locks; = gstm_script), 1 register-resident, fully unrolled
 * (8 / 8 / 16: the bank kernel's code), 2 shared memory [entry][lane] (16 /
 * 16 / 32).  A transaction that exceeds its capacity reports
 * isOpaque = 0 (log overflow). */
int gstm_script_ex(gstm_t* h, int mode, int prelock_vbv, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx,
                   int log_policy);
/* Insert entries (id<<2 | wr<<1 | rd, id < 2^20) into a device lock log
 * (variant 0: register-resident, capacity 16; 1: local memory, capacity 256;
 * both sorted by id.  Variants 2 and 3: the same capacities in
 * encounter order, the lock order of GSTM_MODE_HV_BACKOFF /
 * GSTM_MODE_HV_UNSORTED.  Variants 4 and 5: the order-preserving hashed log
 * of P:115 in local memory, capacity 16 / 256.  Variant 6: sorted, in shared
 * memory [entry][lane], capacity 64) and return the resulting log in
 * out; returns its length or a negative error. */
int gstm_lock_log(const uint32_t* entries, int n, uint32_t* out, int variant);
/* Roofline microbenchmark: kind 0 random atom.or, 1
 * same-address atom.add.u64, 2 random ld.relaxed, 3 random st.relaxed, 4
 * dependent atom.or chain, 5 warp-aggregated clock increments, 6/7/8 random
 * 8-byte atom.or / ld / st (the paired layout's accesses); over a table
 * of table_bytes (power of two) with `threads` threads (multiple of 256).
 * *ops_per_s = operations per second; *ms = kernel time. */
int gstm_ubench(int kind, uint64_t table_bytes, uint64_t n_ops, uint32_t threads, double* ops_per_s, double* ms);

/* Op-mix roofline microbenchmark: n_tx conflict-free
 * "transactions" on the handle's own memory (its layout, lock table and
 * g_clock line), each the exact memory operations Algorithm 3 issues for one
 * transaction of a workload, in its dependency order, without the STM logic.
 * prog (prog_words uint32): prog[0] = number of programs P (1..4), | 0x100
 * for record addressing (then prog[1] = records R, prog[2] = stride S: slot j
 * of thread t is word (t mod R)*S + j mod S -- with R threads, each record's
 * transactions form one serial chain, the contention roof of k-means), then per
 * program: weight (the P weights sum to 65536), n_phases (<= 160), and
 * n_phases phase words kind | count << 8 | slot0 << 16.  The ops of a phase
 * are independent; each phase's addresses depend on the previous phase's
 * results (one round trip per phase).  Op j of a phase touches word slot
 * slot0 + j of the transaction: a random word in [0, words), the same word in
 * every phase.  kind: 1 value load, 2 version-lock load, 3 lock atom.or, 4
 * value store, 5 lock store (on the paired layout 1-5 are 8-byte accesses to
 * the word's pair), 6 warp-aggregated atom.add on g_clock (count ignored),
 * 7 release fence, 8 acquire fence (at most one clock phase per program).
 * Warp-synchronous like the transaction kernel: the phases before the clock
 * run per lane, then one warp-collective clock increment for the lanes that
 * have one, then the phases after it.  threads (multiple of block, block a
 * multiple of 32 <= 256) sets the occupancy.  Synchronous; CLOBBERS the
 * heap, the lock table and the clock (which are reset: a new version epoch).
 * *tx_per_s = transactions per second; *ms (may be NULL) = kernel time. */
int gstm_ubench_mix(gstm_t* h, uint64_t words, const uint32_t* prog, uint32_t prog_words, uint64_t n_tx,
                    uint32_t threads, uint32_t block, double* tx_per_s, double* ms);

#ifdef __cplusplus
}
#endif
#endif
