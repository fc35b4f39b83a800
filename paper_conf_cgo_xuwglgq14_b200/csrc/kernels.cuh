// kernels.cuh -- launch parameters shared by the kernels and the C ABI layer.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "gstm/tx.cuh"
#include "gstm/tx_pair.cuh"
#include "gstm/tx_vbv.cuh"
#include "gstm/tx_irr.cuh"
#include "gstm/workloads.cuh"

namespace gstm {

// statistics counters (uint64 each), in the handle's metadata block
enum {
    S_COMMITS = 0, S_COMMITS_RO, S_AB_OPACITY, S_AB_PREVBV, S_AB_TBV, S_AB_COMMITVBV, S_AB_LOCK,
    S_LOCK_RETRIES, S_POSTVAL, S_VBV, S_SPINS, S_ATTEMPTS, S_ERRORS,
    S_PIPELINED,           // pipelined lock rounds: at most one per execution
    // log sizes of the COMMITTED executions (the algorithmic op counts of the
    // op-mix roof): reads appended to the read-set by update /
    // read-only commits, write-set entries and lock-log entries of update commits
    S_RD_UPD, S_RD_RO, S_WR_UPD, S_LK_UPD,
    S_SERIAL,              // executions run as the serial-ticket owner (contention manager)
    S_NSTATS
};

// metadata block layout (uint64 words; hot words on their own 128 B lines)
static_assert(S_NSTATS <= 29, "the running totals (M_TOTALS + S_NSTATS + 3) must end before M_PHASE");
enum {
    M_CLOCK = 0,           // g_clock
    M_CLOCK_BEGIN = 16,    // g_clock when the launch started (read-only in kernels)
    M_DEADLINE = 17,       // %globaltimer deadline for the watchdog
    M_CLOCK_END = 18,
    M_STATS = 32,          // S_NSTATS counters
    M_CGL_LOCK = 64,       // coarse-grain lock word (uint32)
    M_ERR = 80,            // error bits of the last launch (uint32)
    M_T_START = 81,        // %globaltimer at the start of the last launch
    M_TOTALS = 96,         // S_NSTATS counters summed over launches since reset
    M_T_LAUNCHES = 96 + S_NSTATS,      // launches since reset
    M_T_NS = 97 + S_NSTATS,            // device ns (globaltimer) since reset
    M_T_ERR = 98 + S_NSTATS,           // OR of the error bits since reset
    M_PHASE = 128,                     // 16 phase-cycle accumulators (GSTM_PHASE_TIMING builds)
    M_WORK = 144,                      // next unstarted STM thread (persistent grid), own line
    M_WORDS = 160,
    // after the 256 candidate g_clock lines (api.cu kClockCandidates x kClockStride)
    M_SEQ = M_WORDS + 256 * 288 + 16,  // STM-VBV global sequence lock, own line
    M_SERIAL = M_SEQ + 16,             // contention manager's ticket word {serving:32 | next:32}, own line
    M_SERIAL_EST = M_SERIAL + 1,       // ... and the owners' running mean execution time (ns), same line
};

constexpr int kPhaseWords = 16;    // M_PHASE .. M_PHASE + 15

enum { ERR_LOGOVF = 1, ERR_TIMEOUT = 2, ERR_INVALID = 4 };

enum { WL_RA = 0, WL_BANK = 1, WL_HT = 2, WL_EB = 3, WL_KM = 4 };
enum { KMODE_HV = 1, KMODE_TBV = 2, KMODE_CGL = 3, KMODE_FGL = 4, KMODE_HV_BACKOFF = 5, KMODE_VBV = 6, KMODE_HV_UNSORTED = 7 };
// lock order / retry policy of the STM kernel (kernels.cu)
enum { POL_SORTED = 0, POL_BACKOFF = 1, POL_UNSORTED = 2 };

struct KParams {
    Meta m;
    WlParams w;
    unsigned long long* meta;      // metadata block (M_*)
    uint32_t* tx_stamp;            // verify mode: per tx stamp / RO|snapshot (relative)
    uint32_t* tx_result;           // verify mode: per tx observable result
    uint64_t T;
    uint32_t K;
    uint64_t seed;
    uint32_t prelock_vbv, k_lock, backoff_ns, snapshot_reuse, lock_pipeline;
    uint64_t max_threads;          // 0: one CUDA thread per STM thread; else cap (grid-stride)
    uint32_t paired;               // paired layout (value | lock per u64, tx_pair.cuh)
    uint32_t body_rounds;          // >= 1: bodies per warp iteration for lanes that commit read-only
    uint32_t pipeline_max_locks;   // local-memory logs: pipeline the first round only up to this many locks
    uint32_t lock_log_at_commit;   // read locks enter the sorted lock log at TXCommit (Tx::insert_read_lock)
    uint32_t serial_after;         // contention manager: aborts before a transaction may take a serial ticket (0 = off)
    uint32_t serial_commits;       // ... only while the clock advanced by < serial_commits per abort
    uint32_t lock_pipeline_gated;  // pipelined rounds of longer local/shared logs: the lowest lock first, then the rest
    uint32_t pipeline_abort;       // a failed pipelined round aborts the execution (re-execute, fresh reads)
};

cudaError_t launch_prepare(unsigned long long* meta, const unsigned long long* clock, uint64_t timeout_ns, cudaStream_t s);
cudaError_t launch_finish(unsigned long long* meta, const unsigned long long* clock, cudaStream_t s);
cudaError_t launch_tx(int workload, int kmode, const KParams& kp, int block, cudaStream_t s);
cudaError_t launch_descr(int workload, const KParams& kp, uint32_t* out, int wpt, cudaStream_t s);
bool workload_check(int workload, const WlParams& w, uint64_t* footprint, int* descr_words);
cudaError_t launch_init_heap(int workload, uint32_t* heap, uint64_t words, int vshift, cudaStream_t s);
cudaError_t launch_pack(uint32_t* plain, uint32_t* pairs, uint64_t words, int to_pairs, cudaStream_t s);
cudaError_t launch_lock_halves(uint32_t* pairs, uint64_t words, uint32_t* out, cudaStream_t s);
cudaError_t launch_script(const Meta& m, int mode, int prelock, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx,
                          int policy, cudaStream_t s);
cudaError_t launch_lock_log(const uint32_t* entries, int n, uint32_t* out, int* out_n, int variant, cudaStream_t s);
cudaError_t launch_km_assign(const KParams& kp, uint32_t* cluster, cudaStream_t s);
cudaError_t launch_km_init_centroids(const Meta& m, uint64_t c0, uint64_t n, cudaStream_t s);
cudaError_t launch_km_recenter(const Meta& m, uint32_t C, uint32_t D, uint32_t stride, cudaStream_t s);
int ubench(int kind, uint64_t table_bytes, uint64_t n_ops, uint32_t threads, double* ops_per_s, double* ms);
int ubench_mix(const Meta& m, bool paired, uint64_t words, const uint32_t* prog, uint32_t prog_words, uint64_t n_tx,
               uint32_t threads, uint32_t block, cudaStream_t s, double* tx_per_s, double* ms);
int clock_calibrate_mix(unsigned long long* base, int n_candidates, int stride_words, uint32_t* locks, uint32_t lmask,
                        uint32_t* heap, uint32_t hmask, cudaStream_t s);

}  // namespace gstm
