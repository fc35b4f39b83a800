/*
 * oracle.h -- CPU oracle for the GPU-STM hot path (Xu et al., CGO 2014).
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library
 * under paper_conf_cgo_xuwglgq14_b200/csrc, its C ABI in include/gstm.h, or
 * the Python binding) may include, link, import or execute anything under
 * oracle/.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline
 * / --impl reference legs may.  The oracle shares no code, header, table or
 * constant generator with the CUDA path: the seeded input generator (gen.c)
 * is implemented independently on each side from the recipe in DESIGN.md §3.
 *
 * Citations: "P:n" = line n of the paper text;
 * "A3.lk" = line k of the paper's Algorithm 3.
 *
 * What the oracle computes:
 *   gen.c    the input recipe: counter-based SplitMix64 draws -> transaction
 *            descriptors for the five workloads (RA, bank, HT, EB, KM).
 *   serial.c the plain definition of the method's result.  GPU-STM guarantees
 *            opacity / strict serializability: committed
 *            transactions appear to execute one at a time, in the order of
 *            their commit stamps (A3.l83).  serial.c executes the
 *            same transactions one at a time (canonical order, or a given
 *            stamp order = "replay") directly on a uint32 heap.
 *   alg3.c   Algorithm 3 itself, line by line in the paper's notation, run
 *            as a sequential model on scripted interleavings of several
 *            transactions (for step-level parity of the device primitives).
 *   brute.c  brute-force enumeration of every serial order of a tiny
 *            transaction set ("some global total order").
 */
#ifndef GSTM_ORACLE_H
#define GSTM_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------- workloads ---------------- */
enum { OR_WL_RA = 0, OR_WL_BANK = 1, OR_WL_HT = 2, OR_WL_EB = 3, OR_WL_KM = 4 };

typedef struct {
    int32_t  workload;      /* OR_WL_*                                          */
    uint32_t n_reads;       /* RA: reads per tx                                 */
    uint32_t n_writes;      /* RA: writes per tx                                */
    uint32_t ra_kind;       /* RA: 0 = reads-then-writes, 1 = increment (r/w)   */
    uint64_t n_words;       /* RA/bank/EB: words addressed ([0,n_words)); EB: H */
    uint32_t n_accesses;    /* EB: accesses per tx (A, alternating r/w)         */
    uint32_t ht_buckets;    /* HT: number of bucket heads (power of two)        */
    uint32_t ht_lookup_pct; /* HT: percent of lookups                           */
    uint64_t ht_key_range;  /* HT: keys uniform in [1, ht_key_range]            */
    uint32_t km_clusters;   /* KM: clusters                                     */
    uint32_t km_dims;       /* KM: features per point                           */
    uint32_t shard_bits;    /* HT key partition: G = 2^shard_bits  */
    uint32_t shard;         /* HT: this shard g in [0, G); 0 bits = no partition */
    uint32_t km_stride;     /* KM: words per record, >= km_dims+1 (0: km_dims+1) */
    uint32_t km_assign;     /* KM: 1 = cluster = nearest centroid of the table   */
                            /*     after the records (a full Lloyd iteration)    */
    uint32_t ra_partition;  /* RA: k > 0 = thread t addresses only its own words */
                            /*     [t*k, t*k + k) (SURVEY §8c-O4 disjoint access */
                            /*     sets: a unique, conflict-free result); 0 = off */
} or_params_t;

/* ---------------- gen.c: the seeded input generator ---------------------- */
uint64_t or_mix64(uint64_t z);
uint64_t or_splitmix64(uint64_t x);
uint64_t or_draw(uint64_t x, uint64_t k);
uint64_t or_bounded(uint64_t r, uint64_t n);
uint64_t or_txkey(uint64_t seed, uint64_t t, uint64_t i);
/* Descriptor of transaction (t,i) as a flat list of uint32 words (layout in
 * DESIGN.md §3.3).  Returns the number of words written, or -1 if cap is too
 * small / params invalid. */
int or_descr(const or_params_t* p, uint64_t seed, uint64_t t, uint64_t i,
             uint32_t* out, int cap);
/* Owner shard of an HT key under a 2^bits-way key partition:
 * the top `bits` bits of mix64(key) (the bucket uses the low bits). */
uint32_t or_key_owner(uint64_t key, uint32_t bits);
/* Heap words the workload needs for T threads x K transactions. */
uint64_t or_footprint(const or_params_t* p, uint64_t T, uint64_t K);
/* Workload-defined initial heap. */
void or_init_heap(const or_params_t* p, uint32_t* heap, uint64_t words);

/* k-means, full iteration (km_assign = 1): the centroid
 * table (km_clusters x km_dims uint32) follows the records at word
 * or_km_centroids(p).  or_km_nearest = argmin_c sum_d (f_d - cent[c][d])^2,
 * exact integer arithmetic, ties to the lowest c.  or_km_recenter ends an
 * iteration: cent[c][d] = floor(sum_d / count) for every record with count >
 * 0 (others keep their centroid), then every record is zeroed. */
uint64_t or_km_centroids(const or_params_t* p);
uint32_t or_km_nearest(const or_params_t* p, const uint32_t* heap, const uint32_t* f);
void or_km_recenter(const or_params_t* p, uint32_t* heap);

/* ---------------- serial.c: serial executor and stamp-order replay ------- */
/* Execute transaction (t,i) serially on heap.  *result = observable result,
 * *is_update = 1 if the transaction wrote (update tx), 0 if read-only.
 * Returns 0, or -1 on a footprint violation. */
int or_exec_tx(const or_params_t* p, uint32_t* heap, uint64_t words,
               uint64_t T, uint64_t K, uint64_t seed, uint64_t t, uint64_t i,
               uint32_t* result, int* is_update);
/* Canonical serial order: tx_id = i*T + t ascending (i-major).  results[],
 * is_update[] indexed by tx_id (may be NULL). */
int or_serial(const or_params_t* p, uint32_t* heap, uint64_t words,
              uint64_t T, uint64_t K, uint64_t seed,
              uint32_t* results, uint8_t* is_update);
/* Stamp-order replay.
 * tx_stamp[tx_id]: commit stamp relative to the launch's starting clock for
 * an update tx (1..C, each exactly once), or OR_RO_FLAG | snapshot for a
 * read-only tx (linearised after stamp `snapshot`).  tx_result[tx_id] is the
 * GPU's observable result.  heap holds the initial heap and is advanced to
 * the replayed final heap.  Returns 0 on success or a negative code; a
 * message is written to err. */
#define OR_RO_FLAG 0x80000000u
int or_replay(const or_params_t* p, uint32_t* heap, uint64_t words,
              uint64_t T, uint64_t K, uint64_t seed,
              const uint32_t* tx_stamp, const uint32_t* tx_result,
              int check_thread_order, char* err, int errlen);

/* ---------------- alg3.c: Algorithm 3 sequential model ------------------- */
enum { OR_MODE_HV = 1, OR_MODE_TBV = 2 };
enum { OR_OP_BEGIN = 0, OR_OP_READ = 1, OR_OP_WRITE = 2, OR_OP_COMMIT = 3,
       OR_OP_READ2 = 4 /* batched TXRead of words (addr, value field), reading Q35 */ };
/* Abort causes reported by COMMIT. */
enum { OR_C_OK = 0, OR_C_OPACITY = 1, OR_C_PREVBV = 2, OR_C_TBV = 3,
       OR_C_COMMITVBV = 4, OR_C_READONLY = 5 };
/* Run a script of ops (4 uint32 each: op, tx slot, word, value) over up to
 * n_tx transaction slots on heap[words] with a 2^bits lock table and a global
 * clock that starts at clock0.  out gets 4 uint32 per op:
 *   BEGIN : snapshot, 0, 0, 0
 *   READ  : value, isOpaque, snapshot, postvalidation_ran
 *   WRITE : 0, 0, 0, 0
 *   COMMIT: ok, cause (OR_C_*), stamp (0 if none), vbv_runs
 * lock_tab (2^bits words) and *clock are inputs and outputs. */
int or_alg3_script(int mode, int prelock_vbv, uint32_t bits,
                   uint32_t* heap, uint64_t words, uint32_t* lock_tab,
                   uint64_t* clock, const uint32_t* ops, int n_ops,
                   uint32_t* out, int n_tx);
/* Encounter-time sorted lock log: insert the given entries
 * (lock_id<<2 | wr<<1 | rd) in order, return the resulting log. */
int or_lock_log(const uint32_t* entries, int n, uint32_t* out, int cap);
/* Encounter-order variant (STM-HV-Backoff; Q32): first
 * occurrence order, duplicates merged.  Returns the length or -1 (cap). */
int or_lock_log_encounter(const uint32_t* entries, int n, uint32_t* out, int cap);

/* ---------------- brute.c: every serial order of a tiny tx set ----------- */
/* Enumerate all interleavings of the T per-thread sequences of K txs
 * (program order kept, "some global total order") on the initial heap
 * init[words].  Returns the number of serial orders visited; *match is set to
 * 1 if some order yields exactly (heap_q, results_q) (results indexed by
 * tx_id), and *n_distinct to the number of distinct final (heap, results)
 * outcomes (capped at 1<<20). */
int64_t or_brute(const or_params_t* p, const uint32_t* init, uint64_t words,
                 uint64_t T, uint64_t K, uint64_t seed,
                 const uint32_t* heap_q, const uint32_t* results_q,
                 int* match, int64_t* n_distinct);

#ifdef __cplusplus
}
#endif
#endif
