// tx.cuh -- GPU-STM per-thread transaction runtime (device side).
//
// Implements TXBegin / TXRead / TXWrite / TXCommit of Algorithm 3
// for one CUDA thread.  Logs live in per-thread arrays sized at compile time:
// with small capacities (RA, bank, KM) every loop is unrolled and the logs
// are registers; with large ones (EB, HT, scripts) they are per-thread local
// memory, which the hardware interleaves across the 32 lanes of a warp --
// exactly the "coalesced read-/write-set organization" of P:117 (entry i of
// the merged set belongs to lane i mod 32).
//
// Metadata: a global table of 32-bit version locks (LSB = locked,
// bits 31..1 = version), the global clock, and per transaction a read-set,
// a write-set with a 64-bit bloom filter and a local lock log kept
// sorted by lock id with rd/wr bits.
//
// The warp-collective parts of TXCommit (the warp-aware retry of P:147 and
// the aggregated clock increment of A3.l83) are in kernels.cu; this header
// holds the per-lane steps, which the scripted-interleaving kernel
// (script.cu) also calls one transaction at a time.
#pragma once
#include <cstdint>
#include "prim.cuh"

// ablation builds: -DGSTM_PV_ATTR=__noinline__
#ifndef GSTM_PV_ATTR
#define GSTM_PV_ATTR __forceinline__
#endif

// ablation switches: validation loads chunked 8-wide with
// local-memory logs (measured slower on EB: off); binary-search position in
// the sorted local lock log (EB A=64 +15%, KM +8%: on)
#ifndef GSTM_VBV_CHUNKED
#define GSTM_VBV_CHUNKED 0
#endif
#ifndef GSTM_LOG_BSEARCH
#define GSTM_LOG_BSEARCH 1
#endif

// a loop over a local-memory log: rolled in a compact Tx (kCompact), else
// left to the compiler
#define GSTM_LLOOP(...)                                        \
    do {                                                       \
        if constexpr (kCompact) {                              \
            _Pragma("unroll 1") __VA_ARGS__                    \
        } else {                                               \
            __VA_ARGS__                                        \
        }                                                      \
    } while (0)

// Figure 5 execution-time breakdown: build with
// -DGSTM_PHASE_TIMING=1 (the "phase" library flavour).  Every lane times its
// own path with clock64() and attributes the cycles to the paper's seven
// categories -- native code, transaction initialisation, buffering (read/write
// logging), consistency checking (lock-word checks, spins, PostValidation,
// VBV), acquiring/releasing locks, committing (write-back, clock stamp) and
// aborted transactions (every cycle of an execution that aborted) -- plus
// "other" (loop, refill, SIMT waiting outside a transaction).
#ifndef GSTM_PHASE_TIMING
#define GSTM_PHASE_TIMING 0
#endif

namespace gstm {

enum { PH_NATIVE = 0, PH_INIT, PH_BUFFER, PH_CONSIST, PH_LOCKS, PH_COMMIT, PH_TX_N, PH_ABORTED = PH_TX_N, PH_OTHER,
       PH_N };

enum { MODE_HV = 1, MODE_TBV = 2 };

// commit outcome / abort causes (same numbering as the C ABI stats)
enum { C_OK = 0, C_OPACITY = 1, C_PREVBV = 2, C_TBV = 3, C_COMMITVBV = 4, C_READONLY = 5, C_LOCK = 6 };

struct Meta {
    uint32_t* heap;                  // word w at heap[w << vshift]
    uint32_t* locks;                 // version lock i at locks[i << lshift]
    uint32_t lock_mask;              // 2^bits - 1
    uint32_t lock_shift;             // stripe = 2^shift words (0: one lock per word)
    uint32_t vshift, lshift;         // 0,0: the paper's separate lock table; 1,1: paired layout
    unsigned long long* clock;       // g_clock
    uint32_t spin_cap;               // bound on the l.27-29 spin and on PostValidation restarts

    // hash(addr) of P:113 (reading Q2): the version lock of a memory stripe
    // of 2^lock_shift consecutive words, modulo the table size
    __device__ __forceinline__ uint32_t lock_of(uint32_t w) const { return (w >> lock_shift) & lock_mask; }
    __device__ __forceinline__ uint32_t* val_ptr(uint32_t w) const { return heap + (static_cast<uint64_t>(w) << vshift); }
    __device__ __forceinline__ uint32_t* lock_ptr(uint32_t id) const { return locks + (static_cast<uint64_t>(id) << lshift); }
    // paired layout: word w and its version lock in one u64 (value low, lock high)
    __device__ __forceinline__ unsigned long long* pair_ptr(uint32_t w) const
    {
        return reinterpret_cast<unsigned long long*>(heap) + w;
    }
};

// A3.l83 version <- Atomic_inc(g_clock) + 1, for n commits at once (the
// lanes of a warp that commit together get base+1 .. base+n).  The acquire
// makes every earlier commit's write-back visible to the caller, so base+n is
// also a valid snapshot for the warp's next transactions.
__device__ __forceinline__ unsigned long long clock_fetch_add(unsigned long long* clock, unsigned n)
{
    if (GSTM_STRICT_FENCES) return prim::atom_add_acq_rel64(clock, n);
    return prim::atom_add_acquire64(clock, n);
}

// bloom-filter bit of a word (reading Q7): top 6 bits of a Fibonacci hash
__device__ __forceinline__ unsigned long long bloom_bit(uint32_t w)
{
    return 1ull << ((static_cast<unsigned long long>(w) * 0x9E3779B97F4A7C15ull) >> 58);
}

// SORTED = false: the lock log keeps encounter order (duplicates still
// merged) -- the lock order of STM-HV-Backoff and of the unsorted
// ablation; the paper's GPU-STM sorts.
// COMPACT = true: loops over local-memory logs stay rolled (one copy of each,
// `#pragma unroll 1`; validation loads 4 in flight) -- for kernels whose code
// outgrows the instruction cache (HT: DESIGN.md §6.9); else the compiler
// unrolls them (by 4) and validation keeps 8 loads in flight.
// A per-thread log array: registers / local memory (SMEM = false), or the
// literal organisation of P:117 in shared memory -- entry k of the 32 lanes of
// a warp in 32 consecutive words, [entry][lane], so the lanes' accesses to
// their k-th entries hit 32 different banks (SMEM = true; bind() sets the
// lane's column).
template <int CAP, bool SMEM>
struct LogArr {
    uint32_t a[CAP];
    __device__ __forceinline__ uint32_t& operator[](int k) { return a[k]; }
    __device__ __forceinline__ const uint32_t& operator[](int k) const { return a[k]; }
    __device__ __forceinline__ void bind(uint32_t*) {}
};
template <int CAP>
struct LogArr<CAP, true> {
    uint32_t* p;                          // shared memory: this lane's column
    __device__ __forceinline__ uint32_t& operator[](int k) { return p[k * 32]; }
    __device__ __forceinline__ const uint32_t& operator[](int k) const { return p[k * 32]; }
    __device__ __forceinline__ void bind(uint32_t* col) { p = col; }
};

// HLOG = true (local-memory logs, sorted): the lock log is the order-preserving
// hash table of P:115 instead of one sorted array.
// SMEM = true: the read-, write- and lock-logs live in shared memory, per warp
// [entry][lane]; the kernel binds them (bind_smem).
// COLDPV = true (local/shared-memory logs): PostValidation (A3.l6-20) in its
// smallest form -- rolled, one load at a time -- so the rare path does not
// crowd the instruction cache (RA paper-shaped: 0.94 -> 1.09 G tx/s)
template <int RCAP, int WCAP, int LCAP, bool LOCAL = false, bool SORTED = true, bool COMPACT = false, bool HLOG = false,
          bool SMEM = false, bool COLDPV = false>
struct Tx {
    // register-resident (unrolled) logs for small capacities unless the
    // workload asks for local memory (LOCAL: fewer registers, more warps) or
    // shared memory (SMEM)
    static constexpr bool kUnroll = !LOCAL && !SMEM && (RCAP <= 24 && WCAP <= 24 && LCAP <= 32);
    static constexpr bool kSmem = SMEM;
    static constexpr int kRcap = RCAP, kWcap = WCAP, kLcap = LCAP;
    static constexpr bool kCompact = COMPACT;
    // value / lock-word loads validation keeps in flight with local-memory logs
// compact (HT): validation is the cold path (PostValidation on 0.7% of the
// transactions), so its loops keep one load in flight and stay small in the
// instruction cache -- HT HV 6.87 -> 7.56 G tx/s with 1 vs 4
#ifndef GSTM_COMPACT_PV_WIDTH
#define GSTM_COMPACT_PV_WIDTH 1
#endif
    static constexpr int kPvWidth = COMPACT ? GSTM_COMPACT_PV_WIDTH : 8;
    static constexpr bool kColdPv = COLDPV && !kUnroll && !COMPACT;
    // order-preserving hashed lock log: kHs home slots (load factor
    // <= 1/2), then LCAP overflow slots (an entry never sits more than
    // LCAP - 1 slots past its home); occupancy bitmap in registers
    static constexpr bool kHlog = HLOG && SORTED && !kUnroll && !SMEM;
    static constexpr int kHs = 2 * LCAP;
    static constexpr int kTs = kHlog ? kHs + LCAP : LCAP;
    static constexpr int kBw = kHlog ? (kTs + 31) / 32 : 1;

    LogArr<RCAP, SMEM> r_addr, r_val;     // read-set  <addr,val>
    LogArr<WCAP, SMEM> w_addr, w_val;     // write-set <addr,val> (redo log)
    LogArr<kTs, SMEM> l_ent;              // sorted lock log (hashed: the table)
    LogArr<LCAP, SMEM> l_old;             // old lock words
    // shared-memory logs: words per thread, and the binding of every log to
    // this lane's column of its warp's [word][lane] region
    static constexpr int kSmemWords = 2 * RCAP + 2 * WCAP + kTs + LCAP;
    __device__ __forceinline__ void bind_smem(uint32_t* warp_region, int lane)
    {
        uint32_t* c = warp_region + lane;
        r_addr.bind(c);
        r_val.bind(c + 32 * RCAP);
        w_addr.bind(c + 32 * (2 * RCAP));
        w_val.bind(c + 32 * (2 * RCAP + WCAP));
        l_ent.bind(c + 32 * (2 * RCAP + 2 * WCAP));
        l_old.bind(c + 32 * (2 * RCAP + 2 * WCAP + kTs));
    }
    uint32_t occ[kBw];                    // hashed log: occupied slots
    uint32_t id_shift = 12;               // hashed log: 32 - lock-table bits (home = id's top bits)
    bool compacted;                       // hashed log: l_ent[0, nl) is the dense sorted log
    unsigned long long bloom;
#if GSTM_PHASE_TIMING
    uint32_t ph_acc[PH_TX_N];             // cycles of the current execution by category
    unsigned long long ph_tot[PH_N];      // totals (aborted executions summed into PH_ABORTED)
    int ph_cur = PH_OTHER;
    long long ph_t = 0;
    __device__ __forceinline__ void ph_init()
    {
        for (int k = 0; k < PH_TX_N; ++k) ph_acc[k] = 0u;
        for (int k = 0; k < PH_N; ++k) ph_tot[k] = 0ull;
        ph_cur = PH_OTHER;
        ph_t = clock64();
    }
    // the lane enters category k: the cycles since the last switch go to the
    // category it leaves
    __device__ __forceinline__ void ph(int k)
    {
        const long long now = clock64();
        if (ph_cur < PH_TX_N) ph_acc[ph_cur] += static_cast<uint32_t>(now - ph_t);
        else ph_tot[ph_cur] += static_cast<unsigned long long>(now - ph_t);
        ph_t = now;
        ph_cur = k;
    }
    // the execution ended: committed -> its cycles by category; aborted ->
    // all of them into PH_ABORTED
    __device__ __forceinline__ void ph_end(bool committed)
    {
        ph(PH_OTHER);
        for (int k = 0; k < PH_TX_N; ++k) {
            ph_tot[committed ? k : static_cast<int>(PH_ABORTED)] += ph_acc[k];
            ph_acc[k] = 0u;
        }
    }
#else
    __device__ __forceinline__ void ph_init() {}
    __device__ __forceinline__ void ph(int) {}
    __device__ __forceinline__ void ph_end(bool) {}
#endif
    int nr, nw, nl, n_acq;
    bool defer_rd = false;                // lock_log_at_commit: read locks inserted at TXCommit
    bool pipelined_round = false;         // the last commit_acquire issued a pipelined first round
    bool deferred_done;
    uint32_t snapshot;
    bool opaque, passTBV, overflow;
    uint32_t n_postval, n_vbv, n_spin;    // per-thread statistics
    // lanes of the warp that run this body together and call read_batch
    // exactly once (a convergent workload, stm_kernels.cuh); 0 = unknown
    unsigned sync_mask;

    __device__ __forceinline__ void reset_stats() { n_postval = n_vbv = n_spin = 0; }

    // ---- A3.l1-5 TXBegin (the clock load and fence are done by the caller,
    //      once per warp, see kernels.cu warp_snapshot) --------------------
    __device__ __forceinline__ void begin(uint32_t snap)
    {
        nr = nw = nl = n_acq = 0;                 // l.2
        deferred_done = false;
        bloom = 0ull;
        opaque = passTBV = true;                  // l.3
        overflow = false;
        snapshot = snap;                          // l.4
        sync_mask = 0u;
        if constexpr (kHlog) {
#pragma unroll
            for (int k = 0; k < kBw; ++k) occ[k] = 0u;
            compacted = false;
        }
    }

    // hashed log: ids are lock-table indices < 2^bits
    __device__ __forceinline__ void set_id_bits(uint32_t bits) { id_shift = 32u - bits; }

    // Reconverge the lanes that run their bodies together after a rare,
    // per-lane path (a lock spin, PostValidation): without it the warp stays
    // split and executes the rest of the body once per group of lanes.
    __device__ __forceinline__ void reconverge() const
    {
        if (sync_mask) __syncwarp(sync_mask);
    }

    __device__ __forceinline__ bool read_only() const { return nw == 0; }

    // ---- A3.l22-23: read-after-write through the bloom filter ------------
    __device__ __forceinline__ bool raw_lookup(uint32_t a, uint32_t& v) const
    {
        if (!(bloom & bloom_bit(a))) return false;
        bool hit = false;
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < WCAP; ++k)
                if (k < nw && w_addr[k] == a) { v = w_val[k]; hit = true; }
        } else {
            for (int k = 0; k < nw; ++k)
                if (w_addr[k] == a) { v = w_val[k]; hit = true; break; }
        }
        return hit;
    }

    // ---- A3.l25: append to the read-set (reading Q5: duplicates kept) ----
    __device__ __forceinline__ void append_read(uint32_t a, uint32_t v)
    {
        if (nr >= RCAP) { overflow = true; opaque = false; return; }
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
                if (k == nr) { r_addr[k] = a; r_val[k] = v; }
        } else {
            r_addr[nr] = a; r_val[nr] = v;
        }
        ++nr;
    }

    // ---- hashed log helpers: the occupancy bitmap stays in registers ------
    __device__ __forceinline__ uint32_t occ_word(int w) const
    {
        uint32_t v = 0u;
#pragma unroll
        for (int k = 0; k < kBw; ++k)
            if (k == w) v = occ[k];
        return v;
    }
    __device__ __forceinline__ bool occ_test(int sl) const { return (occ_word(sl >> 5) >> (sl & 31)) & 1u; }
    __device__ __forceinline__ void occ_set(int sl)
    {
#pragma unroll
        for (int k = 0; k < kBw; ++k)
            if (k == (sl >> 5)) occ[k] |= 1u << (sl & 31);
    }

    // ---- insert into the order-preserving hash table --------------
    // Home slot = the id's top bits scaled to kHs slots (monotone in id); the
    // occupied slots hold the entries in ascending id, each at or after its
    // home.  An entry with id' > id can only sit at or after home(id), so the
    // insert position is the first slot from home(id) that is empty or holds
    // an id' >= id; the run of occupied slots from there shifts right by one
    // (into the first empty slot).  Expected O(1) comparisons and moves
    // instead of O(n) ("the number of comparison steps is reduced").
    __device__ __forceinline__ void insert_lock_hashed(uint32_t e)
    {
        const uint32_t id = e >> 2;
        int sl = id_shift >= 32u ? 0 : static_cast<int>(__umulhi(id << id_shift, static_cast<uint32_t>(kHs)));
        bool occupied = occ_test(sl);
        while (occupied && (l_ent[sl] >> 2) < id) occupied = occ_test(++sl);
        if (occupied && (l_ent[sl] >> 2) == id) { l_ent[sl] |= (e & 3u); return; }   // Q4
        if (nl >= LCAP) { overflow = true; opaque = false; return; }
        int end = sl;                                        // first empty slot >= sl
        if (occupied) {
            int w = sl >> 5;
            uint32_t free = ~occ_word(w) & (~0u << (sl & 31));
            while (!free) free = ~occ_word(++w);
            end = (w << 5) + __ffs(free) - 1;
            GSTM_LLOOP(for (int k = end; k > sl; --k) l_ent[k] = l_ent[k - 1];);
        }
        occ_set(end);
        l_ent[sl] = e;
        ++nl;
    }

    // hashed log -> l_ent[0, nl) dense and ascending, for TXCommit (in place:
    // the k-th occupied slot is at index >= k)
    __device__ __forceinline__ void compact()
    {
        if constexpr (kHlog) {
            if (compacted) return;
            int j = 0;
#pragma unroll
            for (int w = 0; w < kBw; ++w) {
                uint32_t b = occ[w];
                while (b) {
                    const int sl = (w << 5) + __ffs(b) - 1;
                    b &= b - 1u;
                    l_ent[j++] = l_ent[sl];
                }
            }
            compacted = true;
        }
    }

    // A3.l34 for a read: insert its lock now (encounter time), or --
    // lock_log_at_commit (defer_rd) -- when the transaction reaches TXCommit
    // with a write-set (insert_deferred_reads).  The sorted log is a function
    // of the set of entries (insert order does not matter, Q4), so the
    // acquisition order and the livelock-freedom argument are the same; a
    // read-only transaction (HT lookups: 90%) skips the sorting it never uses.
    // (register-resident logs always insert at encounter time: a deferred
    // pass would index them dynamically and move them to local memory)
    __device__ __forceinline__ void insert_read_lock(uint32_t id)
    {
        if (kUnroll || !defer_rd) insert_lock((id << 2) | 1u);
    }
    __device__ __forceinline__ void insert_deferred_reads(const Meta& m)
    {
        if constexpr (!kUnroll) {
            if (!defer_rd || deferred_done) return;
            deferred_done = true;
#pragma unroll 1
            for (int k = 0; k < nr; ++k) insert_lock((m.lock_of(r_addr[k]) << 2) | 1u);
        }
    }

    // ---- P:113-115, A3.l34/l38: sorted insert into the local lock log ----
    // Entries are id<<2 | wr<<1 | rd, ascending by id; a duplicate id only
    // ORs its bits (no new entry).
    __device__ __forceinline__ void insert_lock(uint32_t e)
    {
        if constexpr (kHlog) {
            insert_lock_hashed(e);
            return;
        }
        const uint32_t id = e >> 2;
        if constexpr (kUnroll) {
            int pos = 0;
            bool dup = false;
#pragma unroll
            for (int k = 0; k < LCAP; ++k) {
                if (k < nl) {
                    const uint32_t ik = l_ent[k] >> 2;
                    pos += (ik < id) ? 1 : 0;
                    if (ik == id) { l_ent[k] |= (e & 3u); dup = true; }
                }
            }
            if (dup) return;
            if (nl >= LCAP) { overflow = true; opaque = false; return; }
            if constexpr (!SORTED) pos = nl;                         // encounter order: append
#pragma unroll
            for (int k = LCAP - 1; k > 0; --k)
                if (k <= nl && k > pos) l_ent[k] = l_ent[k - 1];
#pragma unroll
            for (int k = 0; k < LCAP; ++k)
                if (k == pos) l_ent[k] = e;
            ++nl;
        } else {
            int pos = 0;
            if constexpr (SORTED) {
                // ascending arrival (a record's words, a stripe) appends in O(1)
                if (nl > 0 && (l_ent[nl - 1] >> 2) < id) {
                    pos = nl;
                } else if constexpr (GSTM_LOG_BSEARCH) {
                    // binary search: log2(n) dependent log reads instead of
                    // up to n (EB's 16-64 random locks)
                    int hi = nl;
                    while (pos < hi) {
                        const int mid = (pos + hi) >> 1;
                        if ((l_ent[mid] >> 2) < id) pos = mid + 1;
                        else hi = mid;
                    }
                } else {
                    while (pos < nl && (l_ent[pos] >> 2) < id) ++pos;
                }
            } else {
                while (pos < nl && (l_ent[pos] >> 2) != id) ++pos;   // encounter order: find or append
            }
            if (pos < nl && (l_ent[pos] >> 2) == id) { l_ent[pos] |= (e & 3u); return; }
            if (nl >= LCAP) { overflow = true; opaque = false; return; }
            GSTM_LLOOP(for (int k = nl; k > pos; --k) l_ent[k] = l_ent[k - 1];);
            l_ent[pos] = e;
            ++nl;
        }
    }

    // ---- A3.l62-66 VBV: every logged value still in memory ---------------
    __device__ __forceinline__ bool vbv(const Meta& m)
    {
        ++n_vbv;
        bool ok = true;
        if constexpr (kUnroll) {
            uint32_t cur[RCAP];
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
                if (k < nr) cur[k] = prim::ld_relaxed(m.val_ptr(r_addr[k]));
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
                if (k < nr) ok &= (cur[k] == r_val[k]);
        } else if constexpr (!kCompact && !GSTM_VBV_CHUNKED) {
            for (int k = 0; k < nr; ++k)
                ok &= (prim::ld_relaxed(m.val_ptr(r_addr[k])) == r_val[k]);
        } else if constexpr (!kCompact) {
            // kPvWidth (8) loads in flight per chunk: a rolled loop would
            // wait for each load before issuing the next (HBM-latency chains
            // on EB's 2^26-word hot set)
            for (int k0 = 0; k0 < nr; k0 += kPvWidth) {
                uint32_t cur[kPvWidth];
#pragma unroll
                for (int j = 0; j < kPvWidth; ++j)
                    if (k0 + j < nr) cur[j] = prim::ld_relaxed(m.val_ptr(r_addr[k0 + j]));
#pragma unroll
                for (int j = 0; j < kPvWidth; ++j)
                    if (k0 + j < nr) ok &= (cur[j] == r_val[k0 + j]);
            }
        } else {
            // compact: kPvWidth loads in flight per chunk, one rolled copy per
            // call site (three sites in HV: A3.l71, l.76 and PostValidation's
            // l.9 -- code size is what the HT kernel's instruction fetch pays
            // for)
#pragma unroll 1
            for (int k0 = 0; k0 < nr; k0 += kPvWidth) {
                uint32_t cur[kPvWidth];
#pragma unroll
                for (int j = 0; j < kPvWidth; ++j)
                    if (k0 + j < nr) cur[j] = prim::ld_relaxed(m.val_ptr(r_addr[k0 + j]));
#pragma unroll
                for (int j = 0; j < kPvWidth; ++j)
                    if (k0 + j < nr) ok &= (cur[j] == r_val[k0 + j]);
            }
        }
        return ok;
    }

    // ---- A3.l6-20 PostValidation(version) --------------------------------
    // "snapshot <- version" (l.7) never lowers the snapshot (reading Q9);
    // restarts are bounded by spin_cap (the paper loops; bounded => abort).
    __device__ GSTM_PV_ATTR bool post_validation(const Meta& m, uint32_t version)
    {
        ++n_postval;
        if (version > snapshot) snapshot = version;                // l.7
        for (uint32_t restart = 0; restart <= m.spin_cap; ++restart) {   // l.8
            if constexpr (kColdPv) {
                // the cold-path form (COLDPV): rolled, one load at a time
                ++n_vbv;
                bool ok = true;
#pragma unroll 1
                for (int k = 0; k < nr; ++k) ok &= (prim::ld_relaxed(m.val_ptr(r_addr[k])) == r_val[k]);   // l.9-11
                if (!ok) return false;
            } else {
                if (!vbv(m)) return false;                           // l.9-11
            }
            prim::fence_acquire();                                   // l.12
            bool again = false;
            uint32_t newsnap = snapshot;
            if constexpr (kColdPv) {
#pragma unroll 1
                for (int k = 0; k < nr; ++k) {                       // l.13-19, one lock load at a time
                    const uint32_t vl = prim::ld_relaxed(m.lock_ptr(m.lock_of(r_addr[k])));
                    if ((vl & 1u) || (vl >> 1) > snapshot) {
                        newsnap = max(newsnap, vl >> 1);
                        again = true;
                    }
                }
            } else if constexpr (kUnroll) {
                uint32_t vl[RCAP];
#pragma unroll
                for (int k = 0; k < RCAP; ++k)                       // l.13
                    if (k < nr) vl[k] = prim::ld_relaxed(m.lock_ptr(m.lock_of(r_addr[k]))); // l.14
#pragma unroll
                for (int k = 0; k < RCAP; ++k)
                    if (k < nr && ((vl[k] & 1u) || (vl[k] >> 1) > snapshot)) {   // l.15-17
                        newsnap = max(newsnap, vl[k] >> 1);          // l.18 (Q9)
                        again = true;                                // l.19 goto loop
                    }
            } else {
                GSTM_LLOOP(for (int k0 = 0; k0 < nr; k0 += kPvWidth) {   // kPvWidth lock loads in flight
                    uint32_t vl[kPvWidth];
#pragma unroll
                    for (int j = 0; j < kPvWidth; ++j)
                        if (k0 + j < nr) vl[j] = prim::ld_relaxed(m.lock_ptr(m.lock_of(r_addr[k0 + j])));
#pragma unroll
                    for (int j = 0; j < kPvWidth; ++j)
                        if (k0 + j < nr && ((vl[j] & 1u) || (vl[j] >> 1) > snapshot)) {
                            newsnap = max(newsnap, vl[j] >> 1);
                            again = true;
                        }
                });
            }
            snapshot = newsnap;
            if (!again) return true;                                 // l.20
            if (restart) __nanosleep(64);
        }
        return false;
    }

    // ---- A3.l27-29: wait while locked; returns the unlocked lock word -----
    __device__ __forceinline__ uint32_t settle_lock(const Meta& m, uint32_t a, uint32_t vl)
    {
        uint32_t spins = 0;
        while (vl & 1u) {                                            // l.29
            if (++spins > m.spin_cap) { opaque = false; break; }
            if (GSTM_SPIN_NS) __nanosleep(GSTM_SPIN_NS);
            vl = prim::ld_relaxed(m.lock_ptr(m.lock_of(a)));      // l.28
        }
        n_spin += spins;
        return vl;
    }

    // ---- A3.l30-33: timestamp check, PostValidation (HV) or abort (TBV) ---
    __device__ __forceinline__ void check_version(const Meta& m, uint32_t version, int mode)
    {
        if (opaque && version > snapshot) {                          // l.31
            if (mode == MODE_HV) {
                if (!post_validation(m, version)) opaque = false;    // l.32-33
            } else {
                opaque = false;                                      // TBV-only (Q18)
            }
        }
    }

    // ---- A3.l27-33: wait while locked, then timestamp check --------------
    __device__ __forceinline__ void check_lock(const Meta& m, uint32_t a, uint32_t vl, int mode)
    {
        vl = settle_lock(m, a, vl);                                  // l.27-29
        check_version(m, vl >> 1, mode);                             // l.30-33
    }

    // ---- A3.l21-35 TXRead(addr) -------------------------------------------
    __device__ __forceinline__ uint32_t read(const Meta& m, uint32_t a, int mode)
    {
        uint32_t v;
        ph(PH_BUFFER);
        if (raw_lookup(a, v)) { ph(PH_NATIVE); return v; }          // l.22-23
        v = prim::ld_relaxed(m.val_ptr(a));                            // l.24
        append_read(a, v);                                           // l.25
        ph(PH_CONSIST);
        prim::fence_acquire();                                       // l.26
        const uint32_t vl = prim::ld_relaxed(m.lock_ptr(m.lock_of(a)));
        check_lock(m, a, vl, mode);                                  // l.27-33
        ph(PH_BUFFER);
        insert_read_lock(m.lock_of(a));                               // l.34
        ph(PH_NATIVE);
        return v;                                                    // l.35
    }

    // l.27-34 of a small batch (bank: 2; an HT chain step), fully unrolled:
    // ONE spin loop re-reads every still-locked lock word of the batch together
    // (l.27-29) and ONE timestamp check with the newest version (Q35): one copy
    // of each rare path, so the lanes of a warp that take it take it together
    // instead of one after the other
    template <int N>
    __device__ __forceinline__ void check_small(const Meta& m, const uint32_t (&a)[N], const bool (&need)[N],
                                                uint32_t (&vl)[N], int mode)
    {
        uint32_t spins = 0;
        bool locked = false;
#pragma unroll
        for (int k = 0; k < N; ++k) locked |= need[k] && (vl[k] & 1u);
        while (locked) {
            if (++spins > m.spin_cap) { opaque = false; break; }
            if (GSTM_SPIN_NS) __nanosleep(GSTM_SPIN_NS);
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k] && (vl[k] & 1u)) vl[k] = prim::ld_relaxed(m.lock_ptr(m.lock_of(a[k])));   // l.28
            locked = false;
#pragma unroll
            for (int k = 0; k < N; ++k) locked |= need[k] && (vl[k] & 1u);
        }
        n_spin += spins;
        reconverge();
        uint32_t newest = 0;
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) newest = max(newest, vl[k] >> 1);
        check_version(m, newest, mode);                          // l.30-33 (Q35)
        reconverge();
        ph(PH_BUFFER);
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k]) insert_read_lock(m.lock_of(a[k]));       // l.34
        } else {
            // local-memory logs: one inlined copy of the (looping) insert
#pragma unroll 1
            for (int k = 0; k < N; ++k) {
                uint32_t ak = 0;
                bool nk = false;
#pragma unroll
                for (int j = 0; j < N; ++j)
                    if (j == k) { ak = a[j]; nk = need[j]; }
                if (nk) insert_read_lock(m.lock_of(ak));         // l.34
            }
        }
    }

    // Batched TXRead of N words whose addresses are known together: the N
    // value loads (l.24) are issued back to back, one fence (l.26) orders all
    // of them before the N lock loads, then each read runs l.27-34 in order.
    // Equivalent to N sequential TXReads with the value loads hoisted: each
    // value is still checked against its lock after it was loaded (DESIGN.md
    // §6.3), but the transaction pays 2 dependent memory round trips instead
    // of 2N.  For batches of more than 4 words the timestamp checks are
    // merged: PostValidation
    // (l.32) runs at most once, with the newest version seen, after every
    // read of the batch is in the read-set -- the outcome sequential reads
    // reach (a read-set consistent at a snapshot >= every version read), and
    // one inlined copy of the rare path instead of N (code size: the
    // instruction cache).  The lock inserts go through one
    // rolled loop for the same reason.
    template <int N>
    __device__ __forceinline__ void read_batch(const Meta& m, const uint32_t (&a)[N], uint32_t (&v)[N], int n, int mode,
                                               uint32_t skip = 0u)
    {
        bool need[N];
        uint32_t vl[N];
        ph(PH_BUFFER);
#pragma unroll
        for (int k = 0; k < N; ++k) need[k] = (k < n) && !((skip >> k) & 1u) && !raw_lookup(a[k], v[k]);
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));    // l.24
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) append_read(a[k], v[k]);                    // l.25
        ph(PH_CONSIST);
        prim::fence_acquire();                                       // l.26
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) {
                // consecutive words of one stripe (a k-means record under one
                // lock) share one lock-word load: it is issued after every
                // value load of the batch, which is all l.26-28 asks
                if (N > 4 && k > 0 && need[k - 1] && m.lock_of(a[k]) == m.lock_of(a[k - 1])) vl[k] = vl[k - 1];
                else vl[k] = prim::ld_relaxed(m.lock_ptr(m.lock_of(a[k])));
            }
        if constexpr (N <= 4) {
            check_small<N>(m, a, need, vl, mode);
        } else {
            uint32_t newest = 0;
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k]) newest = max(newest, settle_lock(m, a[k], vl[k]) >> 1);   // l.27-30
            reconverge();
            check_version(m, newest, mode);                          // l.31-33
            reconverge();
            ph(PH_BUFFER);
#pragma unroll 1
            for (int k = 0; k < N; ++k) {
                uint32_t ak = 0;
                bool nk = false;
#pragma unroll
                for (int j = 0; j < N; ++j)
                    if (j == k) { ak = a[j]; nk = need[j]; }
                if (nk) insert_read_lock(m.lock_of(ak));
            }
        }
        ph(PH_NATIVE);
    }

    // Batched TXRead of n words (n only known at run time; arrays in local
    // memory): the value loads go out 8 at a time, one acquire fence orders
    // them before the lock-word loads, then l.27-34 per word.  skip[k] marks
    // reads the caller serves from its own write-set later.
    __device__ __forceinline__ void read_many(const Meta& m, const uint32_t* a, uint32_t* v, const bool* skip, int n,
                                              int mode)
    {
        uint32_t vl[kRcap];
        ph(PH_BUFFER);
#pragma unroll 8
        for (int k = 0; k < n; ++k)
            if (!skip[k]) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));   // l.24
        for (int k = 0; k < n; ++k)
            if (!skip[k]) append_read(a[k], v[k]);                    // l.25
        ph(PH_CONSIST);
        prim::fence_acquire();                                        // l.26
#pragma unroll 8
        for (int k = 0; k < n; ++k)
            if (!skip[k]) vl[k] = prim::ld_relaxed(m.lock_ptr(m.lock_of(a[k])));
        for (int k = 0; k < n; ++k)
            if (!skip[k]) {
                ph(PH_CONSIST);
                check_lock(m, a[k], vl[k], mode);                     // l.27-33
                ph(PH_BUFFER);
                insert_read_lock(m.lock_of(a[k]));                    // l.34
            }
        ph(PH_NATIVE);
    }

    // ---- A3.l36-38 TXWrite(addr, val): upsert, bloom, sorted lock insert --
    __device__ __forceinline__ void write(const Meta& m, uint32_t a, uint32_t v)
    {
        ph(PH_BUFFER);
        write_log(m, a, v);
        ph(PH_NATIVE);
    }
    __device__ __forceinline__ void write_log(const Meta& m, uint32_t a, uint32_t v)
    {
        bool found = false;
        if (bloom & bloom_bit(a)) {
            if constexpr (kUnroll) {
#pragma unroll
                for (int k = 0; k < WCAP; ++k)
                    if (k < nw && w_addr[k] == a) { w_val[k] = v; found = true; }
            } else {
                for (int k = 0; k < nw; ++k)
                    if (w_addr[k] == a) { w_val[k] = v; found = true; break; }
            }
        }
        if (!found) {                                                // l.37
            if (nw >= WCAP) { overflow = true; opaque = false; return; }
            if constexpr (kUnroll) {
#pragma unroll
                for (int k = 0; k < WCAP; ++k)
                    if (k == nw) { w_addr[k] = a; w_val[k] = v; }
            } else {
                w_addr[nw] = a; w_val[nw] = v;
            }
            ++nw;
            bloom |= bloom_bit(a);
        }
        insert_lock((m.lock_of(a) << 2) | 2u);                  // l.38
    }

    // ---- A3.l53-55 ReleaseLocks: restore the words this attempt acquired --
    __device__ __forceinline__ void release_locks(const Meta& m)
    {
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)
                if (k < n_acq) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), l_old[k]);
        } else {
            GSTM_LLOOP(for (int k = 0; k < n_acq; ++k) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), l_old[k]););
        }
        n_acq = 0;
    }

    // ---- A3.l43-52 GetLocksAndTBV -----------------------------------------
    // Locks are taken one at a time in ascending id and acquisition stops at
    // the first lock already held (reading Q15): this global order is what
    // makes lockstep retry livelock-free.
    __device__ __forceinline__ bool get_locks_and_tbv(const Meta& m)
    {
        compact();
        n_acq = 0;
        bool ok = true;
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k) {
                if (ok && k < nl) {
                    const uint32_t vl = prim::atom_or_acquire(m.lock_ptr(l_ent[k] >> 2), 1u);  // l.45
                    if (vl & 1u) {
                        ok = false;                                  // l.46-48
                    } else {
                        l_old[k] = vl;
                        n_acq = k + 1;
                        if ((l_ent[k] & 1u) && (vl >> 1) > snapshot) passTBV = false;  // l.49-51
                    }
                }
            }
        } else {
            for (int k = 0; k < nl; ++k) {
                const uint32_t vl = prim::atom_or_acquire(m.lock_ptr(l_ent[k] >> 2), 1u);
                if (vl & 1u) { ok = false; break; }
                l_old[k] = vl;
                n_acq = k + 1;
                if ((l_ent[k] & 1u) && (vl >> 1) > snapshot) passTBV = false;
            }
        }
        if (!ok) release_locks(m);                                   // l.47
        return ok;                                                   // l.52
    }

    // Register-resident logs: the pipelined first round and the sequential
    // sorted acquisition in ONE code path, so the lanes of a warp that make a
    // first attempt and those that retry after a lock abort share their memory
    // round trips instead of running one branch after the other: round 0
    // issues entry 0 for every lane and every entry for a pipelined lane;
    // sequential lanes then take entries 1.. one at a time in ascending id,
    // stopping at the first held lock (Q15), in lockstep with each other.
    __device__ __forceinline__ bool get_locks_and_tbv_converged(const Meta& m, bool pipelined)
    {
        static_assert(kUnroll, "converged acquisition needs register-resident logs");
        uint32_t vl[LCAP];
        bool ok = true;
        uint32_t set = 0;   // entries this attempt locked
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl && (k == 0 || pipelined)) vl[k] = prim::atom_or_relaxed(m.lock_ptr(l_ent[k] >> 2), 1u);   // l.45
        prim::fence_acquire();
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl && (k == 0 || pipelined)) {
                if (vl[k] & 1u) ok = false;                          // l.46
                else set |= 1u << k;
            }
#pragma unroll
        for (int k = 1; k < LCAP; ++k)
            if (!pipelined && ok && k < nl) {                        // next entry only after the last succeeded
                vl[k] = prim::atom_or_relaxed(m.lock_ptr(l_ent[k] >> 2), 1u);
                prim::fence_acquire();
                if (vl[k] & 1u) ok = false;
                else set |= 1u << k;
            }
        if (!ok) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)                           // l.47: undo what this attempt set
                if (set & (1u << k)) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), vl[k]);
            n_acq = 0;
            return false;
        }
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl) {
                l_old[k] = vl[k];
                if ((l_ent[k] & 1u) && (vl[k] >> 1) > snapshot) passTBV = false;   // l.49-51
            }
        n_acq = nl;
        return true;
    }

    // The same first round for local-memory logs (EB, HT, KM): the atom.or go
    // out kChunk at a time (their results land in registers, then in the
    // local log), so a transaction with n locks pays ceil(n / kChunk) memory
    // round trips instead of n.  On a conflict every lock this round set is
    // restored, as above.  The kernel uses it only for logs of at most
    // params.pipeline_max_locks entries (default kChunk, e.g. an HT insert):
    // with more locks, holding all of them while failing on one makes readers
    // spin (measured on EB A=16 and KM's 17 locks: -10% and -50%), and the
    // sequential order that stops at the first held lock is faster (DESIGN.md
    // §6.4) -- except where one round trip per lock dominates (§7.4).
    static constexpr int kChunk = 8;
    __device__ __forceinline__ bool get_locks_and_tbv_pipelined_local(const Meta& m)
    {
        bool ok = true;
        for (int k0 = 0; k0 < nl; k0 += kChunk) {
            uint32_t vl[kChunk];
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) vl[j] = prim::atom_or_relaxed(m.lock_ptr(l_ent[k0 + j] >> 2), 1u);   // l.45
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) {
                    l_old[k0 + j] = vl[j];
                    ok &= !(vl[j] & 1u);                             // l.46
                }
        }
        prim::fence_acquire();
        if (!ok) {
            GSTM_LLOOP(for (int k = 0; k < nl; ++k)                  // l.47: undo what we set
                if (!(l_old[k] & 1u)) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), l_old[k]););
            n_acq = 0;
            return false;
        }
        GSTM_LLOOP(for (int k = 0; k < nl; ++k)
            if ((l_ent[k] & 1u) && (l_old[k] >> 1) > snapshot) passTBV = false;);   // l.49-51
        n_acq = nl;
        return true;
    }

    // The gated pipelined round (local/shared-memory logs longer than one
    // pipelined chunk; `lock_pipeline_gated`): the lowest
    // lock alone first -- held by someone: the round fails having touched
    // nothing else, as the sequential round would -- then every other lock
    // at once (kChunk atomics in flight).  Where all contenders of a record
    // need the same lowest lock (k-means: 17 consecutive lock words), the
    // gate picks the winner and the lock-holding time drops from nl
    // dependent round trips to two.
    __device__ __forceinline__ bool get_locks_and_tbv_gated_local(const Meta& m)
    {
        n_acq = 0;
        const uint32_t v0 = prim::atom_or_acquire(m.lock_ptr(l_ent[0] >> 2), 1u);   // l.45, the gate
        if (v0 & 1u) return false;                                   // l.46-48: nothing held
        l_old[0] = v0;
        bool ok = true;
        for (int k0 = 1; k0 < nl; k0 += kChunk) {
            uint32_t vl[kChunk];
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) vl[j] = prim::atom_or_relaxed(m.lock_ptr(l_ent[k0 + j] >> 2), 1u);
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) {
                    l_old[k0 + j] = vl[j];
                    ok &= !(vl[j] & 1u);
                }
        }
        prim::fence_acquire();
        if (!ok) {
            GSTM_LLOOP(for (int k = 0; k < nl; ++k)                  // l.47: undo what this round set
                if (!(l_old[k] & 1u)) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), l_old[k]););
            return false;
        }
        GSTM_LLOOP(for (int k = 0; k < nl; ++k)
            if ((l_ent[k] & 1u) && (l_old[k] >> 1) > snapshot) passTBV = false;);   // l.49-51
        n_acq = nl;
        return true;
    }

    // Commit steps up to the write-back (A3.l67-78).  Returns C_OK when all
    // locks are held and the read-set is valid, C_LOCK on a lock conflict
    // (nothing held; retry, l.73-74), or an abort cause (nothing held).
    // want_pipe: this round may be the pipelined first round (§6.4); it is,
    // for local-memory logs, only if the (complete) log has at most
    // max_pipe_locks entries -- pipelined_round reports the decision
    __device__ __forceinline__ int commit_acquire(const Meta& m, int mode, bool prelock_vbv, bool want_pipe = false,
                                                  uint32_t max_pipe_locks = 8u, bool gated = false)
    {
        ph(PH_BUFFER);
        insert_deferred_reads(m);
        compact();
        const bool pipelined = want_pipe && (kUnroll || nl <= static_cast<int>(max_pipe_locks));
        const bool gate = want_pipe && gated && !pipelined && !kUnroll;   // (kUnroll: pipelined already)
        pipelined_round = pipelined || gate;
        ph(PH_CONSIST);
        if (mode == MODE_HV && prelock_vbv)
            if (!vbv(m)) return C_PREVBV;                            // l.71-72
        ph(PH_LOCKS);
        bool got;
        if constexpr (kUnroll) got = get_locks_and_tbv_converged(m, pipelined);
        else got = pipelined ? get_locks_and_tbv_pipelined_local(m)
                             : gate ? get_locks_and_tbv_gated_local(m) : get_locks_and_tbv(m);
        if (!got) return C_LOCK;                                     // l.73
        if (!passTBV) {                                              // l.75
            if (mode != MODE_HV) { release_locks(m); return C_TBV; } // Q18
            ph(PH_CONSIST);
            const bool ok = vbv(m);
            ph(PH_LOCKS);
            if (!ok) { release_locks(m); return C_COMMITVBV; }       // l.76-78
        }
        ph(PH_COMMIT);
        // l.79 threadfence: the acquiring atomics already returned (each
        // atom.acquire waits for its result), so no write-back below can be
        // performed before the locks are held; the strict build adds the
        // formal release fence.
        if (GSTM_STRICT_FENCES) prim::fence_release();
        return C_OK;
    }

    // ---- A3.l80-82 write-back (lazy update of the redo log) + fence ------
    // The release fence (MEMBAR.GPU) drains the write-back before the commit
    // stamp is taken and before any lock is released (l.82).
    __device__ __forceinline__ void writeback(const Meta& m)
    {
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < WCAP; ++k)
                if (k < nw) prim::st_relaxed(m.val_ptr(w_addr[k]), w_val[k]);
        } else {
            GSTM_LLOOP(for (int k = 0; k < nw; ++k) prim::st_relaxed(m.val_ptr(w_addr[k]), w_val[k]););
        }
        prim::fence_release();                                       // l.82
    }

    // The same write-back for a write-set made of runs of consecutive words
    // (a k-means record, WL::kRunWriteback): a run of 4 words starting on a
    // 16-byte boundary goes out as one vector store.  Split layout only.
    __device__ __forceinline__ void writeback_runs(const Meta& m)
    {
        for (int k = 0; k < nw;) {
            const uint32_t w = w_addr[k];
            uint32_t* ptr = m.val_ptr(w);
            if (m.vshift == 0 && k + 3 < nw && (reinterpret_cast<uintptr_t>(ptr) & 15u) == 0 &&
                w_addr[k + 1] == w + 1 && w_addr[k + 2] == w + 2 && w_addr[k + 3] == w + 3) {
                prim::st_relaxed_v4(ptr, w_val[k], w_val[k + 1], w_val[k + 2], w_val[k + 3]);
                k += 4;
            } else {
                prim::st_relaxed(ptr, w_val[k]);
                ++k;
            }
        }
        prim::fence_release();                                       // l.82
    }

    // ---- A3.l56-61 ReleaseAndUpdateLocks(version) -------------------------
    // Written locks get version<<1; read-only locks get back the exact word
    // the acquiring atomic returned (reading Q16: == lock - 1).
    __device__ __forceinline__ void release_and_update(const Meta& m, uint32_t version)
    {
        ph(PH_LOCKS);
        if (GSTM_STRICT_FENCES) prim::fence_release();
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)
                if (k < nl) prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), (l_ent[k] & 2u) ? (version << 1) : l_old[k]);
        } else {
            GSTM_LLOOP(for (int k = 0; k < nl; ++k)
                prim::st_relaxed(m.lock_ptr(l_ent[k] >> 2), (l_ent[k] & 2u) ? (version << 1) : l_old[k]););
        }
        n_acq = 0;
    }
};

}  // namespace gstm
