// workloads.cuh -- transaction bodies of the five synthetic workloads.
//
// The paper's workloads are random array (RA, Figure 1), hash table
// (HT), EigenBench (EB) and the STAMP ports; their values are not
// specified (Table 1 is lost).  The bodies here follow our recipe
// plus a bank transfer (BASELINE configs[1]).
// Each body is written once against a context type:
//   StmCtx    -- transactional TXRead / TXWrite (tx.cuh)
//   DirectCtx -- plain strong loads/stores, used by the CGL and FGL baselines
//                while they hold their locks.
// The addresses and constants come from the counter-based generator
// (gen.cuh), so an aborted transaction re-executes identically.
#pragma once
#include <cstdint>
#include <type_traits>
#include <utility>
#include "gen.cuh"
#include "prim.cuh"
#include "tx.cuh"

#ifndef GSTM_SMEM_LOGS
#define GSTM_SMEM_LOGS 0
#endif

namespace gstm {

struct WlParams {
    uint64_t n_words;        // RA / bank / EB: address range (EB: hot set H)
    uint32_t n_reads, n_writes, ra_kind, n_accesses;
    uint32_t ht_buckets, ht_lookup_pct;
    uint64_t ht_key_range;
    uint32_t km_clusters, km_dims, km_stride;   // KM record = km_stride words
    uint32_t km_assign;                         // KM: cluster = nearest centroid (full iteration)
    const uint32_t* km_cluster;                 // KM, km_assign: per-tx cluster from km_assign_kernel
    uint32_t shard_bits, shard;                 // HT key partition
    uint32_t ra_partition;                      // RA: k > 0 = thread t uses only [t*k, t*k + k)
    uint64_t T, K;           // launch shape (HT node layout needs M = T*K)
};

// ---- contexts --------------------------------------------------------------
// does the transaction type carry the warp-convergence mask (Tx, TxPair; not
// TxVbv, whose lanes run independently)?
template <class T, class = void>
struct HasSyncMask : std::false_type {};
template <class T>
struct HasSyncMask<T, std::void_t<decltype(std::declval<T&>().sync_mask)>> : std::true_type {};

template <class TX>
struct StmCtx {
    TX& tx;
    const Meta& m;
    int mode;
    __device__ __forceinline__ uint32_t read(uint32_t a) { return tx.read(m, a, mode); }
    template <int N>
    __device__ __forceinline__ void read_batch(const uint32_t (&a)[N], uint32_t (&v)[N], int n, uint32_t skip = 0u)
    {
        tx.template read_batch<N>(m, a, v, n, mode, skip);      // skip: words the caller reads later (RAW)
    }
    __device__ __forceinline__ void read_many(const uint32_t* a, uint32_t* v, const bool* skip, int n)
    {
        tx.read_many(m, a, v, skip, n, mode);
    }
    __device__ __forceinline__ void write(uint32_t a, uint32_t v) { tx.write(m, a, v); }
    // the body's write addresses, in write order (a hint for the irrevocable
    // owner, gstm/tx_irr.cuh; nothing to do here)
    __device__ __forceinline__ void will_write(const uint32_t*, int, int) {}
    __device__ __forceinline__ bool ok() const { return tx.opaque; }
    // the body found its own view inconsistent (e.g. a chain pointer out of
    // range): only possible for a transaction that is about to abort
    __device__ __forceinline__ void invalid() { tx.opaque = false; }
    // the transaction needs more log entries than compiled in: sticky error
    __device__ __forceinline__ void overflow() { tx.overflow = true; tx.opaque = false; }
    // lanes of the warp that run this body together (stm_kernels.cuh,
    // WL::kLockstep / kConvergent); 0 = unknown (then no warp-collective step)
    __device__ __forceinline__ unsigned lockstep_mask() const
    {
        if constexpr (HasSyncMask<TX>::value) return tx.sync_mask;
        else return 0u;
    }
    // the lanes that make the next read_batch call together (its reconverge)
    __device__ __forceinline__ void set_sync_mask(unsigned m)
    {
        if constexpr (HasSyncMask<TX>::value) tx.sync_mask = m;
    }
    static constexpr int kMaxChain = (TX::kRcap - 1) / 2;
};

struct DirectCtx {
    const Meta& m;
    int nw;
    bool bad;
    __device__ __forceinline__ uint32_t read(uint32_t a) { return prim::ld_relaxed(m.val_ptr(a)); }
    template <int N>
    __device__ __forceinline__ void read_batch(const uint32_t (&a)[N], uint32_t (&v)[N], int n, uint32_t skip = 0u)
    {
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (k < n && !((skip >> k) & 1u)) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));
    }
    __device__ __forceinline__ void read_many(const uint32_t* a, uint32_t* v, const bool* skip, int n)
    {
        for (int k = 0; k < n; ++k)
            if (!skip[k]) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));
    }
    __device__ __forceinline__ void write(uint32_t a, uint32_t v) { prim::st_relaxed(m.val_ptr(a), v); ++nw; }
    __device__ __forceinline__ void will_write(const uint32_t*, int, int) {}
    __device__ __forceinline__ bool ok() const { return !bad; }
    __device__ __forceinline__ void invalid() { bad = true; }
    __device__ __forceinline__ void overflow() { bad = true; }
    __device__ __forceinline__ unsigned lockstep_mask() const { return 0u; }
    __device__ __forceinline__ void set_sync_mask(unsigned) {}
    static constexpr int kMaxChain = 1 << 30;
};

__device__ __forceinline__ uint32_t lo32(uint64_t v) { return static_cast<uint32_t>(v); }

// RA word of draw r for STM thread t: uniform over [0, n_words), or over the
// thread's own range [t*k, t*k + k) with ra_partition = k (disjoint access
// sets)
__device__ __forceinline__ uint32_t ra_word(const WlParams& p, uint64_t r, uint64_t t)
{
    if (p.ra_partition) return static_cast<uint32_t>(t * p.ra_partition + gen::bounded(r, p.ra_partition));
    return static_cast<uint32_t>(gen::bounded(r, p.n_words));
}
__host__ __forceinline__ bool ra_partition_fits(const WlParams& p)
{
    return !p.ra_partition || p.T * p.ra_partition <= p.n_words;
}

// ---- RA kind 0: R reads then W writes (Figure 1 random array) -------------
// acc = sum of the words read; write w_j <- acc + c_j; result = acc.
struct RaWL {
    static constexpr int MAXR = 8, MAXW = 8;
    static constexpr int RCAP = MAXR, WCAP = MAXW, LCAP = MAXR + MAXW, FGL_LCAP = MAXR + MAXW;
    static constexpr bool kConvergent = true;   // one read_batch per body
#ifndef GSTM_RA_SMEM
#define GSTM_RA_SMEM 1
#endif
    // logs in shared memory, [entry][lane] (256 B per thread): RA
    // paper-shaped 835 -> 889 M tx/s, configs[0] +5%
    static constexpr bool kSmemLogs = GSTM_RA_SMEM || GSTM_SMEM_LOGS;
#ifndef GSTM_RA_LOCAL_LOGS
#define GSTM_RA_LOCAL_LOGS 1    // local-memory logs: 1.6x over the 128-register unrolled logs
#endif
    static constexpr bool kLocalLogs = GSTM_RA_LOCAL_LOGS;
    static constexpr bool kColdPostValidation = true;   // rare path kept small
    static constexpr bool kSerialGate = true;   // contention manager compiled in (stm_kernels.cuh §6.16)
#ifndef GSTM_RA_MINB
#define GSTM_RA_MINB 2
#endif
    static constexpr int kMinBlocks = GSTM_RA_MINB;
    static constexpr int DESCR = MAXR + 2 * MAXW;
    __host__ static bool check(const WlParams& p)
    {
        return p.ra_kind == 0 && p.n_reads <= MAXR && p.n_writes <= MAXW && p.n_words > 0 && ra_partition_fits(p);
    }
    __host__ static uint64_t footprint(const WlParams& p) { return p.n_words; }
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t t, uint64_t, uint32_t& result)
    {
        const int R = static_cast<int>(p.n_reads), W = static_cast<int>(p.n_writes);
        uint32_t a[MAXR], v[MAXR];
#pragma unroll
        for (int j = 0; j < MAXR; ++j)
            a[j] = j < R ? ra_word(p, gen::draw(x, j), t) : 0u;
        c.template read_batch<MAXR>(a, v, R);
        if (!c.ok()) return;
        uint32_t acc = 0;
#pragma unroll
        for (int j = 0; j < MAXR; ++j)
            if (j < R) acc += v[j];
        // rolled: one inlined copy of TXWrite (its sorted insert is unrolled
        // over the lock log) instead of MAXW -- keeps the kernel's code in
        // the instruction cache
#pragma unroll 1
        for (int j = 0; j < W; ++j) {
            const uint32_t w = ra_word(p, gen::draw(x, R + j), t);
            c.write(w, acc + lo32(gen::draw(x, R + W + j)));
        }
        result = acc;
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t t, uint64_t, F&& f)
    {
        const uint32_t R = p.n_reads, W = p.n_writes;
        for (uint32_t j = 0; j < R + W; ++j) f(ra_word(p, gen::draw(x, j), t));
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t t, uint32_t* out)
    {
        const uint32_t R = p.n_reads, W = p.n_writes;
        for (uint32_t j = 0; j < R + W; ++j) out[j] = ra_word(p, gen::draw(x, j), t);
        for (uint32_t j = 0; j < W; ++j) out[R + W + j] = lo32(gen::draw(x, R + W + j));
        return static_cast<int>(R + 2 * W);
    }
};

// ---- RA kind 1: increment form, read-modify-write of each r_j -------------
// (Figure 1 style: interleaved TXRead / TXWrite, with read-after-write
// through the write-set).  result = sum of the values read.
struct RaIncWL {
    static constexpr int MAXR = 16;
    static constexpr int RCAP = MAXR, WCAP = MAXR, LCAP = MAXR, FGL_LCAP = MAXR;
    static constexpr bool kLocalLogs = GSTM_RA_LOCAL_LOGS;
    static constexpr bool kColdPostValidation = true;   // rare path kept small
    static constexpr bool kSerialGate = true;   // contention manager compiled in (stm_kernels.cuh §6.16)
    static constexpr int kMinBlocks = 2;
    static constexpr int DESCR = MAXR;
    __host__ static bool check(const WlParams& p)
    {
        return p.ra_kind == 1 && p.n_reads <= MAXR && p.n_words > 0 && ra_partition_fits(p);
    }
    __host__ static uint64_t footprint(const WlParams& p) { return p.n_words; }
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t t, uint64_t, uint32_t& result)
    {
        uint32_t acc = 0;
        for (uint32_t j = 0; j < p.n_reads; ++j) {
            const uint32_t a = ra_word(p, gen::draw(x, j), t);
            const uint32_t v = c.read(a);
            if (!c.ok()) return;       // Figure 1: break when not opaque
            c.write(a, v + 1u);
            acc += v;
        }
        result = acc;
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t t, uint64_t, F&& f)
    {
        for (uint32_t j = 0; j < p.n_reads; ++j) f(ra_word(p, gen::draw(x, j), t));
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t t, uint32_t* out)
    {
        for (uint32_t j = 0; j < p.n_reads; ++j) out[j] = ra_word(p, gen::draw(x, j), t);
        return static_cast<int>(p.n_reads);
    }
};

// ---- bank transfer (BASELINE configs[1]) -----------------------------------
struct BankWL {
    static constexpr int RCAP = 2, WCAP = 2, LCAP = 2, FGL_LCAP = 2;   // a != b: at most 2 lock ids
    static constexpr bool kConvergent = true;   // one read_batch per body
    static constexpr bool kSmemLogs = GSTM_SMEM_LOGS;   // "smem" flavour: logs in shared memory
#ifndef GSTM_BANK_MINB
#define GSTM_BANK_MINB 2
#endif
    static constexpr int kMinBlocks = GSTM_BANK_MINB;   // 256-thread blocks per SM (register budget)
    // 16 resident warps per SM (2 x 256 threads): the measured optimum
    // between latency hiding and conflicts
    static constexpr int kWarpsPerSM = 16;
    static constexpr int DESCR = 3;
    __host__ static bool check(const WlParams& p) { return p.n_words >= 2 && p.n_words <= (1ull << 32); }
    __host__ static uint64_t footprint(const WlParams& p) { return p.n_words; }
    __device__ __forceinline__ static void accounts(const WlParams& p, uint64_t x, uint32_t& a, uint32_t& b, uint32_t& amt)
    {
        a = static_cast<uint32_t>(gen::bounded(gen::draw(x, 0), p.n_words));
        b = static_cast<uint32_t>(gen::bounded(gen::draw(x, 1), p.n_words - 1));
        b += (b >= a) ? 1u : 0u;
        amt = 1u + static_cast<uint32_t>(gen::bounded(gen::draw(x, 2), 100));
    }
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t, uint64_t, uint32_t& result)
    {
        uint32_t ad[2], v[2], amt;
        accounts(p, x, ad[0], ad[1], amt);
        c.template read_batch<2>(ad, v, 2);
        if (!c.ok()) return;
        if (static_cast<int32_t>(v[0]) >= static_cast<int32_t>(amt)) {
            c.write(ad[0], v[0] - amt);
            c.write(ad[1], v[1] + amt);
            result = 1;
        } else {
            result = 0;
        }
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t, uint64_t, F&& f)
    {
        uint32_t a, b, amt;
        accounts(p, x, a, b, amt);
        f(a);
        f(b);
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t, uint32_t* out)
    {
        accounts(p, x, out[0], out[1], out[2]);
        return 3;
    }
};

// ---- chained hash table, set semantics (BASELINE configs[2]) ---------------
// heap = [heads B | key[M] | next[M]], node n (1..M) of tx_id = n-1; 0 = null.
struct HtWL {
    static constexpr int MAXCHAIN = 24;
    static constexpr bool kLockstep = true;     // chain walks in warp lockstep (body uses lockstep_mask)
    static constexpr int RCAP = 1 + 2 * MAXCHAIN, WCAP = 3, LCAP = RCAP + WCAP, FGL_LCAP = 1;
    // code size is the HT kernel's limit (instruction fetch stalls, DESIGN.md
    // §6.9): rolled log loops; 64 registers for 4 blocks (32 warps) per SM
    static constexpr bool kCompact = true;
#ifndef GSTM_HT_MINB
#define GSTM_HT_MINB 4
#endif
    static constexpr int kMinBlocks = GSTM_HT_MINB;
    static constexpr int DESCR = 3;
    __host__ static bool check(const WlParams& p)
    {
        return p.ht_buckets && !(p.ht_buckets & (p.ht_buckets - 1)) && p.ht_key_range >= 1 &&
               p.ht_key_range < (1ull << 32) && p.ht_buckets + 2 * p.T * p.K < (1ull << 32) &&
               p.shard_bits <= 8 && (p.shard >> p.shard_bits) == 0;
    }
    __host__ static uint64_t footprint(const WlParams& p) { return p.ht_buckets + 2 * p.T * p.K; }
    // Key partition over G = 2^shard_bits GPUs: shard g owns
    // the keys whose mix64 top bits are g (the bucket uses the low bits) and
    // draws its keys by rejection on the transaction's own stream: candidate
    // 0 is draw 0 (the unpartitioned key), candidate j >= 1 is draw j+1
    // (draw 1 is the insert flag).  After 4096 candidates (probability
    // (1-1/G)^4096 < 1e-200) key = 0 reports an error.
    __device__ __forceinline__ static void key_of(const WlParams& p, uint64_t x, uint32_t& key, uint32_t& ins, uint32_t& bucket)
    {
        key = 1u + static_cast<uint32_t>(gen::bounded(gen::draw(x, 0), p.ht_key_range));
        if (p.shard_bits) {
            const int sh = 64 - static_cast<int>(p.shard_bits);
            for (uint32_t j = 2; (gen::mix64(key) >> sh) != p.shard; ++j) {
                if (j > 4096) { key = 0; break; }
                key = 1u + static_cast<uint32_t>(gen::bounded(gen::draw(x, j), p.ht_key_range));
            }
        }
        ins = gen::bounded(gen::draw(x, 1), 100) >= p.ht_lookup_pct ? 1u : 0u;
        bucket = static_cast<uint32_t>(gen::mix64(key) & (p.ht_buckets - 1));
    }
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t t, uint64_t i, uint32_t& result)
    {
        uint32_t key, ins, bucket;
        key_of(p, x, key, ins, bucket);
        // 32-bit word bases (check(): B + 2M < 2^32): one register each, so
        // the walk's addresses are not rematerialised from 64-bit products
        // under HV's 64-register budget
        const uint32_t M = static_cast<uint32_t>(p.T * p.K);
        const uint32_t kbase = p.ht_buckets - 1u;       // key[h] = heap[kbase + h]
        const uint32_t nbase = kbase + M;               // next[h] = heap[nbase + h]
        // lanes that run their bodies together walk their chains in lockstep:
        // one warp-collective step per chain node, so a step's loads, lock
        // checks and log inserts are executed once for every walking lane
        // instead of once per group of lanes that drifted apart (no lane
        // leaves the loop before the warp agrees every walk is over)
        const unsigned mask = c.lockstep_mask();
        bool live = key != 0;
        if (!live) c.overflow();                      // no owned key drawn (never in practice)
        // one TXRead call site for the whole walk (step 0: the bucket head;
        // step s > 0: key and next of the s-th node), so PostValidation and
        // the lock spin are inlined once
        uint32_t h0 = 0, h = 0, found = 0;
        uint32_t ka = bucket;   // the word a[0] reads: the bucket head, then key[h] (bucket is not
                                // used inside the walk, so it is not rematerialised at every step)
        bool walking = live;
        for (int steps = 0;; ++steps) {
            if (walking && steps > 0 && h > M) { c.invalid(); walking = live = false; }
            if (walking && steps > Ctx::kMaxChain) { c.overflow(); walking = live = false; }
            const unsigned wm = mask ? __ballot_sync(mask, walking) : (walking ? 1u : 0u);
            if (!wm) break;
            if (walking) {
                uint32_t a[2], v[2];
                a[0] = ka;                                                        // head / key[h]
                a[1] = nbase + h;                                                 // next[h]
                if (mask) c.set_sync_mask(wm);               // read_batch reconverges the walking lanes
                c.template read_batch<2>(a, v, steps ? 2 : 1);
                if (!c.ok()) {
                    walking = live = false;
                } else if (steps == 0) {
                    h0 = h = v[0];
                    walking = h != 0;
                } else if (v[0] == key) {
                    found = 1;
                    walking = false;
                } else {
                    h = v[1];
                    walking = h != 0;
                }
                ka = kbase + h;
            }
        }
        if (mask) c.set_sync_mask(0u);
        if (!live) return;
        if (!ins) { result = found; return; }
        if (found) { result = 2; return; }
        const uint32_t n = static_cast<uint32_t>(1 + i * p.T + t);
        c.write(kbase + n, key);
        c.write(nbase + n, h0);
        c.write(static_cast<uint32_t>(gen::mix64(key) & (p.ht_buckets - 1)), n);   // the bucket (key_of)
        result = 3;
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t, uint64_t, F&& f)
    {
        uint32_t key, ins, bucket;
        key_of(p, x, key, ins, bucket);
        f(bucket);      // one lock per bucket: node words are private until linked, then immutable
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t, uint32_t* out)
    {
        key_of(p, x, out[0], out[1], out[2]);
        return 3;
    }
};

// ---- EigenBench-style: A accesses alternating read / write over H words ----
// Compiled for A <= 16, <= 32 and <= 64 (the launch picks the smallest that
// fits): the logs and the body's address arrays are sized by MAXA, so an A=16
// transaction does not carry (and spill through L2) the frame of an A=64 one;
// A <= 16 keeps its logs in shared memory (256 B per thread, DESIGN.md
// §6.13) -- local-memory log traffic written through to L2 and evicted to HBM
// by the streaming heap was most of EB's excess DRAM traffic (§7.4).
#ifndef GSTM_EB16_SMEM
#define GSTM_EB16_SMEM 1
#endif
template <int MAXA_, bool SMEM_>
struct EbWLT {
    static constexpr int MAXA = MAXA_;
    static constexpr int RCAP = MAXA / 2, WCAP = MAXA / 2, LCAP = MAXA, FGL_LCAP = MAXA;
    static constexpr bool kSmemLogs = SMEM_ || (GSTM_SMEM_LOGS && MAXA <= 32);   // A=64: 256 KB per block
    static constexpr bool kLocalLogs = true;   // never register-resident (A=32 unrolled: 2.4x slower)
    // contention manager compiled in (stm_kernels.cuh) for A > 16 only: the A <= 16
    // kernel (hot set 2^26: 677 -> 650 M tx/s with it) never needs it (its worst sweep point, hot set
    // 2^10, runs 2.9x CGL)
    static constexpr bool kSerialGate = MAXA > 16;
#ifndef GSTM_EB16_MINB
#define GSTM_EB16_MINB 2
#endif
    static constexpr int kMinBlocks = MAXA <= 16 ? GSTM_EB16_MINB : 2;
    static constexpr int DESCR = 2 * MAXA;
    __host__ static bool check(const WlParams& p) { return p.n_accesses <= MAXA && p.n_words > 0; }
    __host__ static uint64_t footprint(const WlParams& p) { return p.n_words; }
    // All addresses are known up front, so the reads that are not
    // read-after-write are issued as one batch (Tx::read_many, DESIGN.md
    // §6.3); a read of a word this transaction wrote earlier is served from
    // the write-set in program order (A3.l22-23).
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t t, uint64_t i,
                                                uint32_t& result)
    {
        if constexpr (MAXA <= 16) body_regs(c, p, x, result);
        else body_local(c, p, x, result);
    }
    // A <= 16: the read and write addresses stay in registers (compile-time
    // indices); the non-RAW reads go out as ONE read_batch (the RAW ones
    // skipped, then served from the write-set in program order); no local
    // memory (the local arrays of body_local were written through to L2 on
    // every attempt)
    template <class Ctx>
    __device__ __forceinline__ static void body_regs(Ctx& c, const WlParams& p, uint64_t x, uint32_t& result)
    {
        constexpr int RM = MAXA / 2;
        const int A = static_cast<int>(p.n_accesses);
        uint32_t ra[RM], wa[RM], rv[RM];
#pragma unroll
        for (int r = 0; r < RM; ++r) {
            ra[r] = 2 * r < A ? static_cast<uint32_t>(gen::bounded(gen::draw(x, 2 * r), p.n_words)) : 0u;
            wa[r] = 2 * r + 1 < A ? static_cast<uint32_t>(gen::bounded(gen::draw(x, 2 * r + 1), p.n_words)) : 0u;
        }
        uint32_t rawm = 0;                            // read r follows a write of the same word
#pragma unroll
        for (int r = 0; r < RM; ++r)
#pragma unroll
            for (int w = 0; w < r; ++w)
                if (2 * w + 1 < A && wa[w] == ra[r]) rawm |= 1u << r;
        c.template read_batch<RM>(ra, rv, (A + 1) / 2, rawm);
        if (!c.ok()) return;
        uint32_t acc = 0;
#pragma unroll 1
        for (int j = 0; j < A; ++j) {
            const int r = j >> 1;
            uint32_t aj = 0, vj = 0;
#pragma unroll
            for (int k = 0; k < RM; ++k)
                if (k == r) { aj = (j & 1) ? wa[k] : ra[k]; vj = rv[k]; }
            if ((j & 1) == 0) {
                acc += ((rawm >> r) & 1u) ? c.read(aj) : vj;
                if (!c.ok()) return;
            } else {
                c.write(aj, acc + lo32(gen::draw(x, A + j)));
            }
        }
        result = acc;
    }
    template <class Ctx>
    __device__ __forceinline__ static void body_local(Ctx& c, const WlParams& p, uint64_t x, uint32_t& result)
    {
        const uint32_t A = p.n_accesses;
        uint32_t addr[MAXA], ra[MAXA / 2], rv[MAXA / 2];
        bool raw[MAXA / 2];
        for (uint32_t j = 0; j < A; ++j) addr[j] = static_cast<uint32_t>(gen::bounded(gen::draw(x, j), p.n_words));
        const uint32_t R = (A + 1) / 2;
        // read r is read-after-write if an earlier write has its address; a
        // 64-bit filter of the written addresses skips the scan for most reads
        unsigned long long wf = 0ull;
        for (uint32_t r = 0; r < R; ++r) {
            ra[r] = addr[2 * r];
            bool hit = false;
            if (wf & (1ull << (ra[r] & 63u)))
                for (uint32_t k = 1; k < 2 * r; k += 2) hit |= (addr[k] == ra[r]);
            raw[r] = hit;
            if (2 * r + 1 < A) wf |= 1ull << (addr[2 * r + 1] & 63u);
        }
        c.read_many(ra, rv, raw, static_cast<int>(R));
        if (!c.ok()) return;
        c.will_write(addr + 1, static_cast<int>(A / 2), 2);     // addr[1], addr[3], ...: the write order
        if (!c.ok()) return;
        uint32_t acc = 0;
        for (uint32_t j = 0; j < A; ++j) {
            if ((j & 1u) == 0) {
                acc += raw[j / 2] ? c.read(addr[j]) : rv[j / 2];
                if (!c.ok()) return;
            } else {
                c.write(addr[j], acc + lo32(gen::draw(x, A + j)));
            }
        }
        result = acc;
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t, uint64_t, F&& f)
    {
        for (uint32_t j = 0; j < p.n_accesses; ++j) f(static_cast<uint32_t>(gen::bounded(gen::draw(x, j), p.n_words)));
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t, uint32_t* out)
    {
        const uint32_t A = p.n_accesses;
        for (uint32_t j = 0; j < A; ++j) out[j] = static_cast<uint32_t>(gen::bounded(gen::draw(x, j), p.n_words));
        for (uint32_t j = 0; j < A; ++j) out[A + j] = lo32(gen::draw(x, A + j));
        return static_cast<int>(2 * A);
    }
};
using EbWL = EbWLT<64, false>;            // descriptors, checks; A in (32, 64]
using EbWL32 = EbWLT<32, false>;
using EbWL16 = EbWLT<16, GSTM_EB16_SMEM>;

// ---- k-means cluster update (STAMP kmeans' transactional step) -------------
// record of cluster c = [count, sum_0 .. sum_{D-1}] at word c*stride (stride >= D+1;
// the default D+1 packs the records, 32 aligns each to its own 128 B line).
struct KmWL {
    static constexpr int MAXD = 16;
    static constexpr int RCAP = MAXD + 1, WCAP = MAXD + 1, LCAP = MAXD + 1, FGL_LCAP = 1;
    static constexpr bool kConvergent = true;   // one read_batch per body
    static constexpr bool kRunWriteback = true;   // the record's words, in order
#ifndef GSTM_KM_SMEM
#define GSTM_KM_SMEM 1
#endif
    // logs in shared memory, [entry][lane] per warp: 19.3 -> 24.3 M
    // tx/s over local memory; 408 B per thread
    static constexpr bool kSmemLogs = GSTM_KM_SMEM || GSTM_SMEM_LOGS;
#ifndef GSTM_KM_LOCAL_LOGS
#define GSTM_KM_LOCAL_LOGS 1     // local-memory logs: 122 vs 254 registers, 2.5x faster
#endif
    static constexpr bool kLocalLogs = GSTM_KM_LOCAL_LOGS;
    // (PostValidation is hot here, 7-13 per commit: the cold form measured 26.4 -> 26.7 M tx/s,
    // one lock per record 43 -> 41; left off)
    static constexpr bool kSerialGate = true;   // contention manager compiled in (stm_kernels.cuh §6.16)
    static constexpr int kMinBlocks = GSTM_KM_LOCAL_LOGS ? 2 : 1;
    // 1024 records: 8 resident warps per SM is the measured optimum
    // (21.5 vs 17.9 M tx/s at 16)
    static constexpr int kWarpsPerSM = 8;
    static constexpr int DESCR = MAXD + 1;
    __host__ static bool check(const WlParams& p)
    {
        return p.km_clusters > 0 && p.km_dims <= MAXD && p.km_stride >= p.km_dims + 1 &&
               uint64_t(p.km_clusters) * p.km_stride < (1ull << 32);
    }
    // records, then (km_assign) the C x D centroid table
    __host__ static uint64_t footprint(const WlParams& p)
    {
        return uint64_t(p.km_clusters) * p.km_stride + (p.km_assign ? uint64_t(p.km_clusters) * p.km_dims : 0);
    }
    // the transaction's cluster: drawn by the generator, or (a full k-means
    // iteration) its point's nearest centroid, computed before the launch's
    // transactions by km_assign_kernel (km.cu)
    __device__ __forceinline__ static uint32_t cluster(const WlParams& p, uint64_t x, uint64_t t, uint64_t i)
    {
        if (p.km_cluster) return p.km_cluster[i * p.T + t];
        return static_cast<uint32_t>(gen::bounded(gen::draw(x, 0), p.km_clusters));
    }
    template <class Ctx>
    __device__ __forceinline__ static void body(Ctx& c, const WlParams& p, uint64_t x, uint64_t t, uint64_t i, uint32_t& result)
    {
        const int D = static_cast<int>(p.km_dims);
        const uint32_t base = cluster(p, x, t, i) * p.km_stride;
        uint32_t a[MAXD + 1], v[MAXD + 1];
#pragma unroll
        for (int k = 0; k <= MAXD; ++k) a[k] = base + k;
        c.template read_batch<MAXD + 1>(a, v, D + 1);
        if (!c.ok()) return;
        c.write(base, v[0] + 1u);
#pragma unroll 1
        for (int d = 0; d < D; ++d) c.write(base + 1 + d, v[1 + d] + static_cast<uint32_t>(gen::draw(x, 1 + d) >> 56));
        result = v[0];
    }
    template <class F>
    __device__ __forceinline__ static void fgl_words(const WlParams& p, uint64_t x, uint64_t t, uint64_t i, F&& f)
    {
        f(cluster(p, x, t, i) * p.km_stride);   // one lock per record
    }
    __device__ static int descr(const WlParams& p, uint64_t x, uint64_t, uint32_t* out)
    {
        out[0] = static_cast<uint32_t>(gen::bounded(gen::draw(x, 0), p.km_clusters));
        for (uint32_t d = 0; d < p.km_dims; ++d) out[1 + d] = static_cast<uint32_t>(gen::draw(x, 1 + d) >> 56);
        return static_cast<int>(1 + p.km_dims);
    }
};

}  // namespace gstm
