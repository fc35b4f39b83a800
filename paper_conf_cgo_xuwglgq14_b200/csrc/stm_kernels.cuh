// stm_kernels.cuh -- the transaction kernels (STM-HV, STM-TBV, STM-HV-Backoff,
// STM-VBV, CGL, FGL), their helpers and their host launch templates.  Each
// workload's instantiations are compiled in their own translation unit
// (wl_*.cu) so the library builds in parallel.
//
// One CUDA thread = one STM thread t (Figure 1) that runs K
// transactions i = 0..K-1 (tx_id = i*T + t).  The loop is warp-uniform:
// every iteration the 32 lanes each attempt their current transaction
// together (lanes whose transaction committed move on to the next one, the
// others re-execute theirs), and commit is a warp-collective phase:
//   * lock acquisition rounds: lanes that fail to get a lock retry only
//     after the lanes of the same warp that got theirs finished committing
//     ("On locking failure, it retries after transactions within the same
//     warp finish committing"), for at most k_lock rounds;
//   * the committing lanes of a round take their commit stamps with ONE
//     atomic on the global clock (A3.l83 aggregated over the warp);
//   * the snapshot (A3.l4) is read once per warp and broadcast.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <mutex>
#include <set>
#include <tuple>
#include <type_traits>
#pragma once
#include "kernels.cuh"

namespace gstm {

using prim::FULL;

// WL::kLocalLogs (optional): keep the logs in local memory even when small
template <class WL, class = void>
struct LocalLogs { static constexpr bool value = false; };
template <class WL>
struct LocalLogs<WL, std::void_t<decltype(WL::kLocalLogs)>> { static constexpr bool value = WL::kLocalLogs; };

// WL::kConvergent (optional): every body calls read_batch exactly once, so
// the lanes that start bodies together may reconverge inside it (Tx::reconverge)
template <class WL, class = void>
struct Convergent { static constexpr bool value = false; };
template <class WL>
struct Convergent<WL, std::void_t<decltype(WL::kConvergent)>> { static constexpr bool value = WL::kConvergent; };

// WL::kLockstep (optional): the body runs warp-collective steps over the
// lanes that start bodies together (StmCtx::lockstep_mask, the HT chain walk)
template <class WL, class = void>
struct Lockstep { static constexpr bool value = false; };
template <class WL>
struct Lockstep<WL, std::void_t<decltype(WL::kLockstep)>> { static constexpr bool value = WL::kLockstep; };

// WL::kCompact (optional): rolled log loops, 4-wide validation (Tx COMPACT)
template <class WL, class = void>
struct Compact { static constexpr bool value = false; };
template <class WL>
struct Compact<WL, std::void_t<decltype(WL::kCompact)>> { static constexpr bool value = WL::kCompact; };

// WL::kHashedLog (optional; default GSTM_HLOG): local-memory lock logs are
// the order-preserving hash table of P:115 (Tx HLOG)
#ifndef GSTM_HLOG
#define GSTM_HLOG 0
#endif
template <class WL, class = void>
struct HashedLog { static constexpr bool value = GSTM_HLOG; };
template <class WL>
struct HashedLog<WL, std::void_t<decltype(WL::kHashedLog)>> { static constexpr bool value = WL::kHashedLog; };

// WL::kSmemLogs (optional; default GSTM_SMEM_LOGS for the workloads whose
// logs fit: bank, RA, KM): logs in shared memory, [entry][lane] per warp
// (Tx SMEM)
#ifndef GSTM_SMEM_LOGS
#define GSTM_SMEM_LOGS 0
#endif
template <class WL, class = void>
struct SmemLogs { static constexpr bool value = false; };
template <class WL>
struct SmemLogs<WL, std::void_t<decltype(WL::kSmemLogs)>> { static constexpr bool value = WL::kSmemLogs; };

// WL::kColdPostValidation (optional): PostValidation in its smallest form
// (Tx COLDPV) -- RA
template <class WL, class = void>
struct ColdPv { static constexpr bool value = false; };
template <class WL>
struct ColdPv<WL, std::void_t<decltype(WL::kColdPostValidation)>> { static constexpr bool value = WL::kColdPostValidation; };

// WL::kRunWriteback (optional): the write-set is runs of consecutive words
// (a record): write back with 16-byte vector stores (Tx::writeback_runs)
template <class WL, class = void>
struct RunWriteback { static constexpr bool value = false; };
template <class WL>
struct RunWriteback<WL, std::void_t<decltype(WL::kRunWriteback)>> { static constexpr bool value = WL::kRunWriteback; };

// WL::kSerialGate (optional): the contention manager (p.serial_after,
// DESIGN.md §6.16) is compiled into this workload's STM kernels.  Bank and
// HT (abort ratios 0.16 and 0.003) leave it out: it costs them 8-12
// registers
template <class WL, class = void>
struct SerialGate { static constexpr bool value = false; };
template <class WL>
struct SerialGate<WL, std::void_t<decltype(WL::kSerialGate)>> { static constexpr bool value = WL::kSerialGate; };

// WL::kWarpsPerSM (optional): resident STM warps per SM the persistent grid
// stops at (0 = as many as fit).  More concurrent transactions than that
// only add conflicts.
template <class WL, class = void>
struct WarpsPerSM { static constexpr int value = 0; };
template <class WL>
struct WarpsPerSM<WL, std::void_t<decltype(WL::kWarpsPerSM)>> { static constexpr int value = WL::kWarpsPerSM; };

__device__ __forceinline__ unsigned long long globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// A3.l4-5: snapshot <- g_clock; threadfence.  One acquire load per warp; the
// __syncwarp orders every lane's later accesses after it.
__device__ __forceinline__ uint32_t warp_snapshot(unsigned long long* clock)
{
    unsigned long long s = 0;
    if (prim::lane_id() == 0) s = prim::ld_acquire64(clock);
    s = __shfl_sync(FULL, s, 0);
    __syncwarp();
    return static_cast<uint32_t>(s);
}

// warp-aggregated commit stamp (A3.l83): lanes in `got` each receive a
// distinct stamp; one atom.add per warp round.  Every committing lane has
// drained its write-back with a release fence (l.82, in Tx::writeback); the
// __syncwarp orders those fences before the leader's atomic, and the one
// after orders the leader's acquire before every lane's lock release.  If
// any lane committed, *next_snap = base + n is the clock value right after
// the warp's own commits, a valid snapshot for its next transactions.
__device__ __forceinline__ uint32_t warp_stamp(unsigned long long* clock, bool got, unsigned& gm, uint32_t& next_snap)
{
    __syncwarp();
    gm = __ballot_sync(FULL, got);
    unsigned long long base = 0;
    if (gm) {
        const int leader = __ffs(gm) - 1;
#if GSTM_EXPERIMENT_NO_CLOCK   // measurement only: fake stamps, NOT serializable
        base = (static_cast<unsigned long long>(blockIdx.x) << 20) + threadIdx.x;
#else
        if (static_cast<int>(prim::lane_id()) == leader) base = clock_fetch_add(clock, __popc(gm));
#endif
        base = __shfl_sync(FULL, base, leader);
        __syncwarp();
        next_snap = static_cast<uint32_t>(base) + __popc(gm);
    }
    return static_cast<uint32_t>(base) + __popc(gm & prim::lanemask_lt()) + 1u;
}

// Statistics counters: one private 32-bit slot per thread and counter in
// block-shared memory (sh[k * kMaxBlock + threadIdx.x]: consecutive threads,
// consecutive banks), bumped with a plain shared load/add/store -- no atomics,
// so no same-address serialisation when every lane of a warp counts the same
// event (a 64-bit shared atomicAdd is a CAS loop on sm_100a: up to 32 rounds
// per warp and event).  Kept out of registers (they cost occupancy).  A slot
// cannot wrap: every event costs at least one L2 round trip (> 300 ns) and
// the watchdog ends a launch within timeout_ms (default 60 s), so one thread
// counts < 2^28 events per launch.  At exit, a warp shuffle reduction and
// one global atomic per counter per warp.
constexpr int kMaxBlock = 256;
struct Counters {
    uint32_t* sh;
    bool error = false;
    __device__ __forceinline__ void inc(int k, uint32_t v = 1u)
    {
        sh[k * kMaxBlock + threadIdx.x] += v;
        if (k == S_ERRORS) error = true;
    }
};

#define GSTM_COUNTERS(name)                                                 \
    __shared__ uint32_t name##_sh[S_NSTATS * kMaxBlock];                    \
    for (int k_ = 0; k_ < S_NSTATS; ++k_) name##_sh[k_ * kMaxBlock + threadIdx.x] = 0u; \
    Counters name{name##_sh}

// per-warp totals -> one global atomic per counter per warp
__device__ __forceinline__ void flush_counters(Counters& cnt, unsigned long long* stats)
{
    __syncwarp();
#pragma unroll 1
    for (int k = 0; k < S_NSTATS; ++k) {
        unsigned long long v = cnt.sh[k * kMaxBlock + threadIdx.x];
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(prim::FULL, v, o);
        if (prim::lane_id() == 0 && v) atomicAdd(stats + k, v);
    }
}

__device__ __forceinline__ void set_err(unsigned long long* meta, uint32_t bits)
{
    atomicOr(reinterpret_cast<unsigned int*>(meta + M_ERR), bits);
}

// warp-uniform watchdog check (every 16 iterations)
__device__ __forceinline__ bool warp_late(uint32_t iter, unsigned long long deadline)
{
    if (iter & 15u) return false;
    bool late = false;
    if (prim::lane_id() == 0) late = globaltimer() > deadline;
    return __shfl_sync(FULL, late, 0);
}

// ---------------------------------------------------------------------------
// Contention manager (p.serial_after != 0): the adaptive
// transaction scheduling the paper leaves to future work.
// One 64-bit word in the metadata block, M_SERIAL = {serving:32 | next:32},
// is a ticket queue.  A transaction that keeps aborting while the whole GPU
// commits little (g_clock advanced by < serial_commits per abort of its
// own), and for which one-at-a-time measures faster (serial_gate), takes a
// ticket; while any ticket is outstanding (next != serving) no other
// transaction STARTS an execution -- one that has aborted before and passes
// the same time test joins the queue instead -- and the holders run one at a time
// in ticket order: the owner (ticket == serving) runs its transaction
// irrevocably -- in place, under encounter-time locks, stamped while it holds
// them all (gstm/tx_irr.cuh) -- and then serves the next ticket.  The
// executions already in flight finish under Algorithm 3 beside it (they see
// the owner's words locked, as during any commit).  Every other execution
// runs Algorithm 3 in full; the owner is serialised at its stamp like any
// commit, so the replay checks hold for every schedule.
// ---------------------------------------------------------------------------
struct SerialState {
    uint32_t ticket = 0, serving = 0;
    uint32_t n_ab = 0;        // aborted executions of the current transaction
    uint32_t s_first = 0;     // snapshot of its first execution
    uint32_t t_first = 0;     // %globaltimer >> 10 (~us) at its first execution
    bool has_ticket = false;
    bool pending = false;     // the last poll saw tickets outstanding (warp-uniform)
    __device__ __forceinline__ bool owner() const { return has_ticket && ticket == serving; }
};

// Called once per warp iteration by every lane; `fresh`: this lane would
// start an execution of its current transaction (stage 0).  Returns whether
// it may.  The ticket word is read when this warp takes or holds a ticket,
// after a poll that saw tickets outstanding, and every 8th iteration
// otherwise (a stale "none outstanding" only lets an execution start beside
// the owner, where it meets the owner's words locked as during any commit).
__device__ __forceinline__ bool serial_gate(const KParams& p, SerialState& ss, bool fresh, uint32_t snap,
                                            uint32_t iter)
{
    unsigned long long* sw = p.meta + M_SERIAL;
    // candidates: aborted >= serial_after times while the clock advanced by
    // < serial_commits per abort; they qualify when, besides, the GPU's
    // commits during their attempts took longer each than a serial owner's
    // execution does (the owners' running mean, M_SERIAL_EST; none measured
    // yet: qualify) -- serialise only where one-at-a-time is faster
    const bool cand = fresh && !ss.has_ticket && ss.n_ab >= p.serial_after &&
                      snap - ss.s_first < p.serial_commits * ss.n_ab;
    // a transaction that aborted before joins a serial phase in progress --
    // once an owner was measured, and if one-at-a-time is faster for it too
    const bool joiner = fresh && !ss.has_ticket && ss.pending && ss.n_ab >= 1u;
    bool want = false;
    if (__any_sync(FULL, cand || joiner)) {
        unsigned long long est = 0, now = 0;
        if (prim::lane_id() == 0) {
            est = prim::ld_relaxed64(p.meta + M_SERIAL_EST);
            now = globaltimer() >> 10;
        }
        est = __shfl_sync(FULL, est, 0);
        now = __shfl_sync(FULL, now, 0);
        const unsigned long long elapsed_ns = static_cast<unsigned long long>(static_cast<uint32_t>(now) - ss.t_first) << 10;
        const bool slower = static_cast<unsigned long long>(snap - ss.s_first) * est < elapsed_ns;
        want = (cand && (est == 0 || slower)) || (joiner && est != 0 && slower);
    }
    const unsigned wm = __ballot_sync(FULL, want);
    const bool poll = wm || __any_sync(FULL, ss.has_ticket) || ss.pending || (iter & 7u) == 0u;
    if (poll) {
        unsigned long long w = 0;
        if (prim::lane_id() == 0)
            w = wm ? atomicAdd(sw, static_cast<unsigned long long>(__popc(wm))) : prim::ld_relaxed64(sw);
        w = __shfl_sync(FULL, w, 0);
        const uint32_t next = static_cast<uint32_t>(w) + __popc(wm);
        ss.serving = static_cast<uint32_t>(w >> 32);
        if (want) {
            ss.ticket = static_cast<uint32_t>(w) + __popc(wm & prim::lanemask_lt());
            ss.has_ticket = true;
        }
        ss.pending = next != ss.serving;
    }
    return ss.has_ticket ? ss.owner() : !ss.pending;
}

// the owner's transaction is done (committed or dropped): serve the next ticket
__device__ __forceinline__ void serial_release(const KParams& p, SerialState& ss)
{
    if (ss.owner()) {
        prim::fence_release();   // not needed for correctness (scheduling only); orders the owner's commit first
        atomicAdd(p.meta + M_SERIAL, 1ull << 32);
    }
    ss.has_ticket = false;
    ss.n_ab = 0;
}

// Per-category time breakdown (the Figure 5 study of P:329-333):
// the "phase" build flavour (-DGSTM_PHASE_TIMING=1) times every lane's own
// path in the paper's categories (tx.cuh PH_*, Tx::ph); at exit the per-lane
// totals are summed per warp and added to meta[M_PHASE + k].
template <class TX>
__device__ __forceinline__ void flush_phases(TX& tx, unsigned long long* dst)
{
#if GSTM_PHASE_TIMING
    tx.ph(PH_OTHER);
#pragma unroll 1
    for (int k = 0; k < PH_N; ++k) {
        unsigned long long v = tx.ph_tot[k];
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
        if (prim::lane_id() == 0) atomicAdd(dst + k, v);
    }
#endif
}

// ---------------------------------------------------------------------------
// STM kernel: GPU-STM with hierarchical validation (MODE_HV, "STM-HV-Sorting")
// or timestamp-only validation (MODE_TBV, "STM-TBV-Sorting").
// ---------------------------------------------------------------------------
//
// POL selects the lock order and retry policy:
//   POL_SORTED    the paper's GPU-STM: sorted lock log, every lane that lost
//                 a lock round retries in the warp's next round
//   POL_BACKOFF   STM-HV-Backoff: encounter-order lock log; the first attempt
//                 is made by all lanes in parallel, then the lanes that failed
//                 retry ONE AT A TIME while the others wait, after the winners
//                 committed
//   POL_UNSORTED  ablation: encounter-order lock log with the parallel retry
//                 of POL_SORTED -- exposed to the intra-warp livelock of P:63
// the transaction type of a workload's STM kernel
template <class WL, bool PAIR, int POL>
using StmTx = std::conditional_t<
    PAIR,
    TxPair<WL::RCAP, WL::WCAP, WL::LCAP, LocalLogs<WL>::value, POL == POL_SORTED, Compact<WL>::value,
           HashedLog<WL>::value, SmemLogs<WL>::value, ColdPv<WL>::value>,
    Tx<WL::RCAP, WL::WCAP, WL::LCAP, LocalLogs<WL>::value, POL == POL_SORTED, Compact<WL>::value, HashedLog<WL>::value,
       SmemLogs<WL>::value, ColdPv<WL>::value>>;

// dynamic shared memory of the STM kernel: the shared-memory logs, if any
template <class WL, bool PAIR, int POL>
constexpr size_t stm_smem_bytes(int block)
{
    using TX = StmTx<WL, PAIR, POL>;
    return TX::kSmem ? static_cast<size_t>(block) * TX::kSmemWords * sizeof(uint32_t) : 0;
}

template <class WL, int MODE, bool PAIR, int POL = POL_SORTED>
__global__ void __launch_bounds__(256, WL::kMinBlocks) stm_kernel(const KParams p)
{
    using TX = StmTx<WL, PAIR, POL>;
    // The grid is persistent (host sizes it to what fits on the chip, or to
    // p.max_threads): lane g runs STM threads g, g+P, ... g+(Rs-1)P of the
    // static region [0, S = Rs*P), Rs = max(1, T/P - 1) rounds, with no
    // shared counter; then a lane that has run all K transactions of its
    // thread takes the next unstarted thread of [S, T) from a global counter
    // (one warp-aggregated atomic), so no lane idles while work remains, the
    // tail stays balanced, and the program order of each STM thread is kept.
    // (A counter for every thread cost ~15% of the bank step: nearly every
    // warp iteration some lane finishes its thread, and every warp of the
    // chip hits the same word.)
    const uint64_t P = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    const uint64_t S = (p.T / P >= 2 ? p.T / P - 1 : 1) * P;
    uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (p.K == 0) t = p.T;
    const Meta m = p.m;
    const uint32_t clock_begin = static_cast<uint32_t>(p.meta[M_CLOCK_BEGIN]);
    const unsigned long long deadline = p.meta[M_DEADLINE];
    unsigned long long* work = p.meta + M_WORK;
    GSTM_COUNTERS(cnt);
    TX tx;
    if constexpr (TX::kSmem) {
        // this warp's [word][lane] region of the block's shared-memory logs
        extern __shared__ uint32_t gstm_smem_logs[];
        tx.bind_smem(gstm_smem_logs + (threadIdx.x >> 5) * 32 * TX::kSmemWords, static_cast<int>(prim::lane_id()));
    }
    tx.reset_stats();
    tx.set_id_bits(static_cast<uint32_t>(__popc(m.lock_mask)));   // lock ids < 2^bits (hashed log)
    tx.defer_rd = p.lock_log_at_commit != 0;
    uint32_t i = 0, iter = 0, backoff = 0, next_snap = 0, tries = 0, result = 0;
    uint32_t seq_fails = 0;   // POL_BACKOFF: consecutive failed sequential steps of this warp
    // stage 0: start (or re-execute) transaction (t, i); stage 1: its body
    // ran and it waits for its locks (a lost lock round is retried in the
    // warp's next iteration, after the winners committed)
    int stage = 0;
    bool timed_out = false, have_snap = false;
    uint32_t lock_aborts = 0;   // lock aborts of the current transaction
    int32_t ab_warp = 0;        // pipeline_abort: the warp's recent abort rate, EMA x 256 (warp-uniform)
    SerialState ss;             // contention manager (p.serial_after)
    const bool serial_on = SerialGate<WL>::value && p.serial_after != 0;
    // the serial owner's lock log: one slice per warp (one owner per warp at most)
    constexpr int kIrrWords = SerialGate<WL>::value ? 2 * IrrCtx<TX>::kCap : 1;
    __shared__ uint32_t irr_sh[(kMaxBlock / 32) * kIrrWords];
    uint32_t* const irr_log = irr_sh + (threadIdx.x >> 5) * kIrrWords;
    tx.ph_init();

    while (__any_sync(FULL, t < p.T)) {
        if (warp_late(iter++, deadline)) { timed_out = true; break; }
        const bool act = t < p.T;
        // (a lane the serial queue may hold back waits outside a transaction:
        // "other" until its execution starts, PH_INIT below)
        tx.ph(!act ? PH_OTHER : stage == 1 ? PH_LOCKS
              : (serial_on && (ss.pending || ss.has_ticket)) ? PH_OTHER : PH_INIT);
        // TXBegin l.4-5: a fresh clock read, or the clock value right after
        // this warp's own last commit (p.snapshot_reuse)
        const uint32_t snap = (have_snap && p.snapshot_reuse) ? next_snap : warp_snapshot(m.clock);
        have_snap = false;
        bool done = false, aborted = false, fin = false, ran = false;
        const bool may_start = serial_on ? serial_gate(p, ss, act && stage == 0 && i < p.K, snap, iter) : true;
        if (!may_start && act && stage == 0) tx.ph(PH_OTHER);   // held back by the serial queue: not in a transaction
        // Body rounds (p.body_rounds): a lane whose
        // transaction committed read-only (A3.l68: no locks, no stamp) starts
        // its next transaction in the same warp iteration, up to body_rounds
        // bodies, so lanes of a mostly read-only workload (HT: 90% lookups) do
        // not idle through the commit round of the warp's few update lanes.
        // Every round uses the iteration's snapshot (a valid, older one: more
        // validation at worst).  A lane that aborted, or holds an update to
        // commit, sits out the later rounds.
        bool cont = act && stage == 0 && may_start;
        // a lane's next transaction starts no earlier than where its last one
        // was linearised (PostValidation may have raised that snapshot above
        // the iteration's): per-thread real-time order
        uint32_t lane_snap = snap;
        for (uint32_t round = 0;; ++round) {
            const bool run = cont && i < p.K;
            if (round > 0 && (round >= p.body_rounds || !__any_sync(FULL, run))) break;
            cont = false;
            const unsigned body_mask =
                (Convergent<WL>::value || Lockstep<WL>::value) ? __ballot_sync(FULL, run) : 0u;
            if (run) {
                const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
                bool next = false;
                cnt.inc(S_ATTEMPTS);
                ran = true;
                if (serial_on) {
                    if (ss.n_ab == 0) {
                        ss.s_first = lane_snap;
                        ss.t_first = static_cast<uint32_t>(globaltimer() >> 10);
                    }
                    if (ss.has_ticket) cnt.inc(S_SERIAL);
                }
                result = 0;
                tx.ph(PH_INIT);
                const uint64_t x = gen::tx_key(p.seed, t, i);
                if (serial_on && ss.owner()) {
                    // the serial-ticket owner runs irrevocably: in place,
                    // under encounter-time locks, stamped while it holds
                    // them all (gstm/tx_irr.cuh)
                    IrrCtx<TX> ic{irr_log, irr_log + IrrCtx<TX>::kCap, m, deadline};
                    const unsigned long long t_own = globaltimer();
                    tx.ph(PH_NATIVE);
                    WL::body(ic, p.w, x, t, i, result);
                    tx.ph(PH_COMMIT);
                    const uint32_t s = ic.commit(m.clock);
                    {   // the owners' running mean execution time (one owner at a time)
                        unsigned long long* e = p.meta + M_SERIAL_EST;
                        const unsigned long long dt = globaltimer() - t_own, old = prim::ld_relaxed64(e);
                        prim::st_relaxed64(e, old ? (7 * old + dt) / 8 : dt);
                    }
                    tx.n_spin += ic.n_spin;
                    tx.ph_end(true);
                    if (ic.bad) {
                        cnt.inc(S_ERRORS);
                        if (globaltimer() > deadline) timed_out = true;
                    }
                    if (p.tx_stamp) {
                        p.tx_stamp[tx_id] = (s & 0x80000000u) ? 0x80000000u | ((s & 0x7fffffffu) - clock_begin)
                                                              : s - clock_begin;
                        p.tx_result[tx_id] = result;
                    }
                    if (s & 0x80000000u) {
                        cnt.inc(S_COMMITS_RO);
                        cnt.inc(S_RD_RO, static_cast<uint32_t>(ic.nr));
                    } else {
                        cnt.inc(S_COMMITS);
                        cnt.inc(S_RD_UPD, static_cast<uint32_t>(ic.nr));
                        cnt.inc(S_WR_UPD, static_cast<uint32_t>(ic.nw));
                        cnt.inc(S_LK_UPD, static_cast<uint32_t>(ic.nl_taken));
                    }
                    next = true;
                } else {
                    tx.begin(lane_snap);                                  // TXBegin l.2-3
                    tx.sync_mask = body_mask;
                    StmCtx<TX> ctx{tx, m, MODE};
                    tx.ph(PH_NATIVE);
                    WL::body(ctx, p.w, x, t, i, result);                 // TXRead / TXWrite
                    if (!tx.opaque) {
                        tx.ph_end(false);
                        if (tx.overflow) { cnt.inc(S_ERRORS); next = true; }  // sticky ELOGOVF, give up this tx
                        else { cnt.inc(S_AB_OPACITY); aborted = true; }  // Figure 1 / Q11
                    } else if (tx.read_only()) {                          // l.68: linearized at snapshot
                        tx.ph_end(true);
                        if (p.tx_stamp) {
                            p.tx_stamp[tx_id] = 0x80000000u | (tx.snapshot - clock_begin);
                            p.tx_result[tx_id] = result;
                        }
                        cnt.inc(S_COMMITS_RO);
                        cnt.inc(S_RD_RO, static_cast<uint32_t>(tx.nr));
                        next = true;
                        cont = true;
                        lane_snap = tx.snapshot;
                    } else {
                        tx.ph(PH_OTHER);                                  // waits for the warp's commit round
                        stage = 1;
                        // STM-HV-Backoff: an execution that follows a lock abort goes
                        // straight to the sequential step -- its parallel attempt
                        // already failed
                        tries = (POL == POL_BACKOFF && lock_aborts) ? 1u : 0u;
                    }
                }
                if (next) {                                           // the next transaction of thread t
                    fin = true;
                    ++i;
                    backoff = 0;
                    lock_aborts = 0;
                }
            }
        }
        // No lane may take a lock while another lane of its warp can still be
        // spinning on a lock in its read phase (A3.l27-29): under independent
        // thread scheduling the locker would then wait for the spinner at the
        // warp barrier in warp_stamp while the spinner waits for its lock.
        __syncwarp();
        // one warp-collective TXCommit round per iteration (l.67-85)
        bool got = false;
        // (POL_BACKOFF: only the first, parallel attempt happens here)
        if (act && stage == 1 && (POL != POL_BACKOFF || tries == 0)) {
            // the pipelined round (§6.4) only for the FIRST round of each of
            // the first p.lock_pipeline executions of a transaction: every
            // later round of an execution (tries > 0, counted for any k_lock,
            // 0 included) is the sequential sorted acquisition.  So at most
            // one round per execution is pipelined (S_PIPELINED checks it);
            // a round that follows a failed round is sequential, and among
            // sequential lanes the holder of the highest contended lock
            // always progresses (Q15, Q37).
            // (pipeline_abort: only while the WARP's recent executions rarely
            // aborted -- a warp-uniform choice, so its lanes do not split
            // between the two acquisition paths; under contention a pipelined
            // round holds every lock of a doomed commit, §6.4)
            const bool want_pipe = tries == 0 && lock_aborts < p.lock_pipeline &&
                                   (!p.pipeline_abort || ab_warp < static_cast<int32_t>(p.pipeline_abort));
            const int r = tx.commit_acquire(m, MODE, p.prelock_vbv != 0, want_pipe, p.pipeline_max_locks,
                                            p.lock_pipeline_gated != 0);
            if (tx.pipelined_round) cnt.inc(S_PIPELINED);
            if (r == C_OK) {
                got = true;
                // l.79-82
                if constexpr (RunWriteback<WL>::value) tx.writeback_runs(m);
                else tx.writeback(m);
            } else if (r == C_LOCK) {
                cnt.inc(S_LOCK_RETRIES);                              // l.73-74: retry next iteration
                // every failed round counts, whatever k_lock is: tries > 0
                // makes every later round of this execution sequential (Q15,
                // Q37; k_lock = 0 retries forever, but never pipelined again)
                tries += (tries != ~0u) ? 1u : 0u;
                if (POL == POL_BACKOFF) {
                    tries = 1;                                        // -> the sequential step below
                } else if ((p.k_lock && tries >= p.k_lock) || (p.pipeline_abort && tx.pipelined_round)) {
                    // (pipeline_abort: a lock another transaction holds in a
                    // failed pipelined round is being committed, so this
                    // execution's read of its word is stale -- re-execute now
                    // instead of retrying sequential rounds toward a failing
                    // VBV; after lock_pipeline such aborts the rounds are
                    // sequential again, §6.4)
                    stage = 0;
                    aborted = true;
                    ++lock_aborts;
                    cnt.inc(S_AB_LOCK);
                    tx.ph_end(false);
                }
                if (stage == 1) tx.ph(PH_OTHER);
            } else {
                stage = 0;
                aborted = true;
                cnt.inc(r == C_PREVBV ? S_AB_PREVBV : (r == C_TBV ? S_AB_TBV : S_AB_COMMITVBV));
                tx.ph_end(false);
            }
        }
        unsigned gm;
        const uint32_t stamp = warp_stamp(m.clock, got, gm, next_snap);   // l.83
        if (gm) have_snap = true;
        if (got) {
            tx.release_and_update(m, stamp);                          // l.84
            if (p.tx_stamp) {
                const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
                p.tx_stamp[tx_id] = stamp - clock_begin;
                p.tx_result[tx_id] = result;
            }
            cnt.inc(S_COMMITS);
            cnt.inc(S_RD_UPD, static_cast<uint32_t>(tx.nr));
            cnt.inc(S_WR_UPD, static_cast<uint32_t>(tx.nw));
            cnt.inc(S_LK_UPD, static_cast<uint32_t>(tx.nl));
            tx.ph_end(true);
            done = true;
        }
        if constexpr (POL == POL_BACKOFF) {
            // "Those who incur locking failures try to acquire locks
            // again sequentially, while the others are waiting (inactive)."
            // One lane at a time acquires, validates, writes back, stamps
            // (its own clock increment) and releases.  A lane that fails again
            // retries in the next iteration; more than k_lock failed
            // sequential attempts abort the transaction.
            unsigned seq = __ballot_sync(FULL, act && stage == 1 && tries > 0);
            // "a backoff mechanism specific to GPU": sequential
            // locking removes the livelock inside a warp; across warps two
            // sequential lanes can still take encounter-ordered locks
            // crosswise again and again, so a warp whose sequential step
            // failed waits a randomised, exponentially growing delay before
            // the next one -- warp-uniform, the only delay SIMT allows
            if (seq && seq_fails) {
                const uint32_t cap = 256u << min(seq_fails, 8u);
                const uint32_t r = static_cast<uint32_t>(gen::mix64((blockIdx.x * 8u + (threadIdx.x >> 5)) * 0x9E3779B97F4A7C15ull + iter));
                __nanosleep(__shfl_sync(FULL, r, 0) % cap);
            }
            bool seq_failed = false;
            while (seq) {
                const int L = __ffs(seq) - 1;
                seq &= seq - 1;
                uint32_t sl = 0;
                if (static_cast<int>(prim::lane_id()) == L) {
                    const int r = tx.commit_acquire(m, MODE, p.prelock_vbv != 0, false);
                    if (r == C_OK) {
                        // l.79-82
                        if constexpr (RunWriteback<WL>::value) tx.writeback_runs(m);
                        else tx.writeback(m);
                        sl = static_cast<uint32_t>(clock_fetch_add(m.clock, 1u)) + 1u;   // l.83
                        tx.release_and_update(m, sl);                 // l.84
                        if (p.tx_stamp) {
                            const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
                            p.tx_stamp[tx_id] = sl - clock_begin;
                            p.tx_result[tx_id] = result;
                        }
                        cnt.inc(S_COMMITS);
                        cnt.inc(S_RD_UPD, static_cast<uint32_t>(tx.nr));
                        cnt.inc(S_WR_UPD, static_cast<uint32_t>(tx.nw));
                        cnt.inc(S_LK_UPD, static_cast<uint32_t>(tx.nl));
                        tx.ph_end(true);
                        done = true;
                    } else if (r == C_LOCK) {
                        cnt.inc(S_LOCK_RETRIES);
                        seq_failed = true;
                        if (p.k_lock && ++tries > p.k_lock) {
                            stage = 0;
                            aborted = true;
                            ++lock_aborts;
                            cnt.inc(S_AB_LOCK);
                            tx.ph_end(false);
                        } else {
                            tx.ph(PH_OTHER);
                        }
                    } else {
                        stage = 0;
                        aborted = true;
                        tx.ph_end(false);
                        cnt.inc(r == C_PREVBV ? S_AB_PREVBV : (r == C_TBV ? S_AB_TBV : S_AB_COMMITVBV));
                    }
                }
                sl = __shfl_sync(FULL, sl, L);
                if (sl) { next_snap = sl; have_snap = true; }   // the latest own stamp: a valid snapshot
            }
            seq_failed = __any_sync(FULL, seq_failed);
            seq_fails = seq_failed ? seq_fails + 1u : 0u;
        }
        if (done) {
            fin = true;
            stage = 0;
            ++i;
            backoff = 0;
            lock_aborts = 0;
        }
        if (p.pipeline_abort) {
            const int na = __popc(__ballot_sync(FULL, aborted)), nc = __popc(__ballot_sync(FULL, done));
            if (na + nc) ab_warp += (na * 256 / (na + nc) - ab_warp) / 8;
        }
        if (!done && p.backoff_ns && aborted) {
            // exponential backoff after an abort (P:111 argues per-lane
            // delays cannot work under SIMT; lanes here sleep independently
            // under independent thread scheduling)
            backoff = backoff ? min(backoff * 2u, 64u * p.backoff_ns) : p.backoff_ns;
            __nanosleep(backoff);
        }
        if (serial_on) {
            if (fin) serial_release(p, ss);
            if (aborted) ++ss.n_ab;   // (an execution of the lane's NEXT transaction, if fin)
            // a warp whose lanes were all held back sleeps before polling
            // again (the warp holding the next ticket polls at once)
            if (!__any_sync(FULL, ran || stage == 1)) {
                const bool soon = ss.has_ticket && ss.ticket - ss.serving <= 1u;
                if (!__any_sync(FULL, soon)) __nanosleep(1000);
            }
        }
        // refill: lanes whose STM thread ran all K transactions take the next
        // one -- their next static thread, else one from the counter
        bool need = t < p.T && i >= p.K;
        if (need && t + P < S) {
            t += P;
            i = 0;
            need = false;
        }
        const unsigned nm = __ballot_sync(FULL, need);
        if (nm) {
            const int leader = __ffs(nm) - 1;
            unsigned long long base = 0;
            if (static_cast<int>(prim::lane_id()) == leader) base = atomicAdd(work, static_cast<unsigned long long>(__popc(nm)));
            base = __shfl_sync(FULL, base, leader);
            if (need) {
                t = S + base + __popc(nm & prim::lanemask_lt());
                i = 0;
            }
        }
    }
    flush_phases(tx, p.meta + M_PHASE);
    cnt.inc(S_POSTVAL, tx.n_postval);
    cnt.inc(S_VBV, tx.n_vbv);
    cnt.inc(S_SPINS, tx.n_spin);
    if (__any_sync(FULL, timed_out) && prim::lane_id() == 0) set_err(p.meta, ERR_TIMEOUT);
    if (__any_sync(FULL, cnt.error) && prim::lane_id() == 0) set_err(p.meta, ERR_LOGOVF);
    flush_counters(cnt, p.meta + M_STATS);
}

// ---------------------------------------------------------------------------
// CGL baseline: one global lock serialises every transaction, taken
// with Algorithm 1 Scheme #3 (diverge on failure) plus a test before
// the CAS.  The body runs in place; the stamp is taken under the lock.
// ---------------------------------------------------------------------------
template <class WL>
__global__ void __launch_bounds__(256, WL::kMinBlocks) cgl_kernel(const KParams p)
{
    const uint64_t P = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (p.K == 0) t = p.T;
    uint32_t* lock = reinterpret_cast<uint32_t*>(p.meta + M_CGL_LOCK);
    const uint32_t clock_begin = static_cast<uint32_t>(p.meta[M_CLOCK_BEGIN]);
    const unsigned long long deadline = p.meta[M_DEADLINE];
    GSTM_COUNTERS(cnt);
    uint32_t i = 0, iter = 0, backoff = 0;
    bool timed_out = false;
    while (__any_sync(FULL, t < p.T)) {
        if (warp_late(iter++, deadline)) { timed_out = true; break; }
        const bool act = t < p.T;
        if (act) {
            cnt.inc(S_ATTEMPTS);
            if (prim::ld_relaxed(lock) == 0 && prim::atom_cas_acquire(lock, 0u, 1u) == 0u) {
                backoff = 0;
                const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
                DirectCtx ctx{p.m, 0, false};
                uint32_t result = 0;
                WL::body(ctx, p.w, gen::tx_key(p.seed, t, i), t, i, result);   // critical section
                uint32_t s;
                if (ctx.nw) {
                    s = static_cast<uint32_t>(prim::atom_add_relaxed64(p.m.clock, 1ull)) + 1u - clock_begin;
                    cnt.inc(S_COMMITS);
                } else {
                    s = 0x80000000u | (static_cast<uint32_t>(prim::ld_relaxed64(p.m.clock)) - clock_begin);
                    cnt.inc(S_COMMITS_RO);
                }
                if (ctx.bad) cnt.inc(S_ERRORS);
                if (p.tx_stamp) { p.tx_stamp[tx_id] = s; p.tx_result[tx_id] = result; }
                prim::fence_release();
                prim::st_relaxed(lock, 0u);                           // Scheme #3 l.15
                if (++i >= p.K) { i = 0; t += P; }
            } else {
                cnt.inc(S_LOCK_RETRIES);
                // optional per-thread exponential backoff (test-and-test-and-set
                // with backoff; the paper's Scheme #3 has none: backoff_ns = 0)
                if (p.backoff_ns) {
                    backoff = backoff ? min(backoff * 2u, 256u * p.backoff_ns) : p.backoff_ns;
                    __nanosleep(backoff);
                }
            }
        }
    }
    if (__any_sync(FULL, timed_out) && prim::lane_id() == 0) set_err(p.meta, ERR_TIMEOUT);
    if (__any_sync(FULL, cnt.error) && prim::lane_id() == 0) set_err(p.meta, ERR_INVALID);
    flush_counters(cnt, p.meta + M_STATS);
}

// ---------------------------------------------------------------------------
// STM-VBV (NOrec-like; tx_vbv.cuh): one global sequence lock,
// value-based validation, writers serialised.  Each lane runs its
// transactions independently (no warp-collective step: a lane waiting for
// seq to become even never waits for its own warp).
// ---------------------------------------------------------------------------
template <class WL>
__global__ void __launch_bounds__(256, WL::kMinBlocks) vbv_kernel(const KParams p)
{
    using TX = TxVbv<WL::RCAP, WL::WCAP, LocalLogs<WL>::value>;
    const uint64_t P = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (p.K == 0) t = p.T;
    // STM-VBV waits on the global sequence lock, not on a word's version
    // lock: the short per-word spin bound of Q38 (spin_cap 1 for bank/RA)
    // does not apply -- it would turn every concurrent writer into an abort
    Meta m = p.m;
    m.spin_cap = max(m.spin_cap, 1u << 16);
    unsigned long long* seq = p.meta + M_SEQ;
    const uint32_t clock_begin = static_cast<uint32_t>(p.meta[M_CLOCK_BEGIN]);
    const unsigned long long deadline = p.meta[M_DEADLINE];
    GSTM_COUNTERS(cnt);
    TX tx;
    tx.reset_stats();
    uint32_t i = 0, iter = 0;
    bool timed_out = false;
    while (__any_sync(FULL, t < p.T)) {
        if (warp_late(iter++, deadline)) { timed_out = true; break; }
        if (t < p.T && !timed_out) {
            cnt.inc(S_ATTEMPTS);
            const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
            uint32_t result = 0;
            bool done = false, skip = false;
            tx.begin(m, seq);
            if (tx.opaque) {
                StmCtx<TX> ctx{tx, m, MODE_HV};
                WL::body(ctx, p.w, gen::tx_key(p.seed, t, i), t, i, result);
            }
            if (!tx.opaque) {
                if (tx.overflow) { cnt.inc(S_ERRORS); skip = true; }
                else cnt.inc(S_AB_OPACITY);
            } else if (tx.read_only()) {
                if (p.tx_stamp) {
                    p.tx_stamp[tx_id] = 0x80000000u | (static_cast<uint32_t>(tx.snapshot >> 1) - clock_begin);
                    p.tx_result[tx_id] = result;
                }
                cnt.inc(S_COMMITS_RO);
                done = true;
            } else {
                // NOrec retries the CAS until it wins or validation fails (some
                // writer wins every round, so this cannot livelock); k_lock
                // does not apply.  Bounded by the watchdog.
                int r = C_LOCK;
                for (uint32_t tries = 0; r == C_LOCK; ++tries) {
                    if ((tries & 15u) == 15u && globaltimer() > deadline) { timed_out = true; break; }
                    r = tx.try_lock(m);
                    if (r == C_LOCK) cnt.inc(S_LOCK_RETRIES);
                }
                if (r == C_OK) {
                    const uint32_t stamp = tx.writeback_and_release(m);
                    if (p.tx_stamp) {
                        p.tx_stamp[tx_id] = stamp - clock_begin;
                        p.tx_result[tx_id] = result;
                    }
                    cnt.inc(S_COMMITS);
                    done = true;
                } else if (r == C_COMMITVBV) {
                    cnt.inc(S_AB_COMMITVBV);
                }
            }
            if (done || skip) {
                if (++i >= p.K) { i = 0; t += P; }
            }
        }
    }
    cnt.inc(S_POSTVAL, tx.n_postval);
    cnt.inc(S_VBV, tx.n_vbv);
    cnt.inc(S_SPINS, tx.n_spin);
    if (__any_sync(FULL, timed_out) && prim::lane_id() == 0) set_err(p.meta, ERR_TIMEOUT);
    if (__any_sync(FULL, cnt.error) && prim::lane_id() == 0) set_err(p.meta, ERR_LOGOVF);
    flush_counters(cnt, p.meta + M_STATS);
}

// ---------------------------------------------------------------------------
// FGL baseline: the hand-locking a programmer would write -- one lock per
// stripe of the words the transaction will touch (per account, per bucket,
// per k-means record), acquired in ascending id with try-lock and
// release-all on failure, then the body in place.  No logs, no validation.
// (The paper did not implement FGL; north_star asks for it.)
// ---------------------------------------------------------------------------
template <class WL>
__global__ void __launch_bounds__(256, WL::kMinBlocks) fgl_kernel(const KParams p)
{
    using TX = Tx<1, 1, WL::FGL_LCAP>;      // only the sorted lock log is used
    const uint64_t P = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (p.K == 0) t = p.T;
    const Meta m = p.m;
    const uint32_t clock_begin = static_cast<uint32_t>(p.meta[M_CLOCK_BEGIN]);
    const unsigned long long deadline = p.meta[M_DEADLINE];
    GSTM_COUNTERS(cnt);
    TX lk;
    uint32_t i = 0, iter = 0;
    bool timed_out = false;
    while (__any_sync(FULL, t < p.T)) {
        if (warp_late(iter++, deadline)) { timed_out = true; break; }
        const bool act = t < p.T;
        const uint64_t tx_id = static_cast<uint64_t>(i) * p.T + t;
        bool got = false;
        int nw = 0;
        uint32_t result = 0;
        if (act) {
            cnt.inc(S_ATTEMPTS);
            const uint64_t x = gen::tx_key(p.seed, t, i);
            lk.begin(0);
            WL::fgl_words(p.w, x, t, i, [&](uint32_t w) { lk.insert_lock((m.lock_of(w) << 2) | 2u); });
            if (lk.overflow) {
                cnt.inc(S_ERRORS);
            } else if (lk.get_locks_and_tbv(m)) {
                got = true;
                DirectCtx ctx{m, 0, false};
                WL::body(ctx, p.w, x, t, i, result);
                nw = ctx.nw;
                if (ctx.bad) cnt.inc(S_ERRORS);
                prim::fence_release();          // in-place writes before stamp and unlock
            } else {
                cnt.inc(S_LOCK_RETRIES);
            }
        }
        unsigned gm;
        uint32_t unused_snap;
        const uint32_t stamp = warp_stamp(m.clock, got && nw > 0, gm, unused_snap);
        if (got) {
            uint32_t s;
            if (nw > 0) {
                s = stamp - clock_begin;
                cnt.inc(S_COMMITS);
            } else {
                s = 0x80000000u | (static_cast<uint32_t>(prim::ld_acquire64(m.clock)) - clock_begin);
                cnt.inc(S_COMMITS_RO);
            }
            if (p.tx_stamp) { p.tx_stamp[tx_id] = s; p.tx_result[tx_id] = result; }
            if (GSTM_STRICT_FENCES) prim::fence_release();
            lk.release_locks(m);
        }
        if (got || (act && lk.overflow)) {
            if (++i >= p.K) { i = 0; t += P; }
        } else if (act && p.backoff_ns) {
            __nanosleep(p.backoff_ns);
        }
    }
    if (__any_sync(FULL, timed_out) && prim::lane_id() == 0) set_err(p.meta, ERR_TIMEOUT);
    if (__any_sync(FULL, cnt.error) && prim::lane_id() == 0) set_err(p.meta, ERR_LOGOVF);
    flush_counters(cnt, p.meta + M_STATS);
}

// ---------------------------------------------------------------------------
// descriptor dump (generator parity test): out[(i*T + t) * wpt + k]
// ---------------------------------------------------------------------------
template <class WL>
__global__ void descr_kernel(const KParams p, uint32_t* out, int wpt)
{
    const uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (t >= p.T) return;
    for (uint32_t i = 0; i < p.K; ++i) {
        uint32_t d[WL::DESCR];
        const int n = WL::descr(p.w, gen::tx_key(p.seed, t, i), t, d);
        uint32_t* o = out + (static_cast<uint64_t>(i) * p.T + t) * wpt;
        for (int k = 0; k < wpt; ++k) o[k] = k < n ? d[k] : 0u;
    }
}

// ---------------------------------------------------------------------------
// host launch templates (instantiated per workload in wl_*.cu)
// ---------------------------------------------------------------------------
template <class K>
inline uint64_t resident_blocks(K kernel, int block, int warps_per_sm = 0, size_t smem = 0)
{
    // SM count of the CURRENT device (cached per device: one process may
    // drive handles on several GPUs; a racing first query stores the same value)
    static std::atomic<int> sms_of[64];
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64) {
        sms = sms_of[dev].load(std::memory_order_relaxed);
        if (!sms) {
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
            sms_of[dev].store(sms, std::memory_order_relaxed);
        }
    } else {
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, block, smem) != cudaSuccess || per_sm < 1) per_sm = 1;
    if (warps_per_sm > 0) per_sm = std::max(1, std::min(per_sm, warps_per_sm * 32 / block));
    return static_cast<uint64_t>(per_sm) * (sms > 0 ? sms : 148);
}

template <class K>
inline cudaError_t launch_stm(K kernel, const KParams& kp, int block, cudaStream_t s, int warps_per_sm = 0,
                              size_t smem = 0)
{
    if (smem > 0) {
        // opt in to the dynamic shared memory once per (kernel, device, size):
        // static + dynamic above 48 KB needs it (the counters take ~20 KB)
        static std::mutex mu;
        static std::set<std::tuple<const void*, int, size_t>> done;
        int dev = 0;
        cudaGetDevice(&dev);
        const auto key = std::make_tuple(reinterpret_cast<const void*>(kernel), dev, smem);
        std::lock_guard<std::mutex> g(mu);
        if (!done.count(key)) {
            const cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                       static_cast<int>(smem));
            if (e != cudaSuccess) return e;
            done.insert(key);
        }
    }
    uint64_t grid = (kp.T + block - 1) / block;
    grid = std::min<uint64_t>(grid, resident_blocks(kernel, block, kp.max_threads ? 0 : warps_per_sm, smem));
    if (kp.max_threads) grid = std::min<uint64_t>(grid, (kp.max_threads + block - 1) / block);   // concurrency cap
    if (grid == 0) return cudaSuccess;
    kernel<<<static_cast<unsigned>(grid), block, smem, s>>>(kp);
    return cudaGetLastError();
}

template <class WL>
cudaError_t launch_wl(int kmode, const KParams& kp, int block, cudaStream_t s)
{
    uint64_t grid = (kp.T + block - 1) / block;
    if (kp.max_threads) grid = std::min<uint64_t>(grid, (kp.max_threads + block - 1) / block);   // concurrency cap
    if (grid == 0) return cudaSuccess;
    const dim3 g(static_cast<unsigned>(grid)), b(block);
    constexpr int W = WarpsPerSM<WL>::value;
    switch (kmode) {
    case KMODE_HV:
        return kp.paired ? launch_stm(stm_kernel<WL, MODE_HV, true>, kp, block, s, W, stm_smem_bytes<WL, true, POL_SORTED>(block))
                         : launch_stm(stm_kernel<WL, MODE_HV, false>, kp, block, s, W, stm_smem_bytes<WL, false, POL_SORTED>(block));
    case KMODE_TBV:
        return kp.paired ? launch_stm(stm_kernel<WL, MODE_TBV, true>, kp, block, s, W, stm_smem_bytes<WL, true, POL_SORTED>(block))
                         : launch_stm(stm_kernel<WL, MODE_TBV, false>, kp, block, s, W, stm_smem_bytes<WL, false, POL_SORTED>(block));
    case KMODE_HV_BACKOFF:
        return kp.paired ? launch_stm(stm_kernel<WL, MODE_HV, true, POL_BACKOFF>, kp, block, s, W,
                                      stm_smem_bytes<WL, true, POL_BACKOFF>(block))
                         : launch_stm(stm_kernel<WL, MODE_HV, false, POL_BACKOFF>, kp, block, s, W,
                                      stm_smem_bytes<WL, false, POL_BACKOFF>(block));
    case KMODE_HV_UNSORTED:
        return kp.paired ? launch_stm(stm_kernel<WL, MODE_HV, true, POL_UNSORTED>, kp, block, s, W,
                                      stm_smem_bytes<WL, true, POL_UNSORTED>(block))
                         : launch_stm(stm_kernel<WL, MODE_HV, false, POL_UNSORTED>, kp, block, s, W,
                                      stm_smem_bytes<WL, false, POL_UNSORTED>(block));
    case KMODE_VBV: vbv_kernel<WL><<<g, b, 0, s>>>(kp); break;
    case KMODE_CGL: cgl_kernel<WL><<<g, b, 0, s>>>(kp); break;
    case KMODE_FGL: fgl_kernel<WL><<<g, b, 0, s>>>(kp); break;
    default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

template <class WL>
cudaError_t launch_descr_wl(const KParams& kp, uint32_t* out, int wpt, cudaStream_t s)
{
    const uint64_t grid = (kp.T + 255) / 256;
    if (grid) descr_kernel<WL><<<static_cast<unsigned>(grid), 256, 0, s>>>(kp, out, wpt);
    return cudaGetLastError();
}

template <class WL>
bool check_wl(const WlParams& w, uint64_t* fp, int* dw)
{
    if (!WL::check(w)) return false;
    *fp = WL::footprint(w);
    *dw = WL::DESCR;
    return true;
}

// one workload's entry points, explicitly instantiated
#define GSTM_INSTANTIATE_WL(WL)                                                                    \
    template cudaError_t launch_wl<WL>(int, const KParams&, int, cudaStream_t);                    \
    template cudaError_t launch_descr_wl<WL>(const KParams&, uint32_t*, int, cudaStream_t);        \
    template bool check_wl<WL>(const WlParams&, uint64_t*, int*);

}  // namespace gstm
