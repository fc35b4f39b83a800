// tx_irr.cuh -- irrevocable execution of the serial-ticket owner (the
// contention manager of stm_kernels.cuh).
//
// The paper leaves contention management to future work.
// Where every pair of transactions conflicts (the EB corner: 64 accesses
// over 1K words), at most one transaction commits at a time whatever the
// concurrency, and a transaction that runs alone still pays Algorithm 3's
// instrumentation: read-set appends, sorted lock-log inserts (O(n^2) for
// n = 64 locks), pre-lock VBV, lock acquisition, VBV under locks.  The
// ticket owner instead runs its body IN PLACE under encounter-time locks:
//   * every word is locked (atom.or on its version lock, A3.l45's lock word)
//     BEFORE it is read or written, and stays locked until the end; a lock
//     found held by another transaction is waited for -- its holder is a
//     committer of Algorithm 3 that releases within its commit round
//     (commits never wait while holding locks, A3.l46-48), so the wait ends;
//   * reads are plain loads of locked words, writes are plain stores;
//   * the end: fence (l.82), stamp = g_clock + 1 (l.83) while every lock is
//     held, then each lock is released -- with version stamp where the owner
//     wrote (l.84), with its old word where it only read.
// So the owner is serialised at its stamp exactly like an Algorithm 3 commit
// (a read-only owner at the clock value read while it still holds every
// lock, as A3.l68 places a read-only transaction at its snapshot), and the
// transactions running beside it see its words locked, as during any commit
// (A3.l27-29: they spin, then validate or abort).  It never aborts: the
// locks it holds only grow.  Its lock log (ent: id<<2 | wr<<1 | 1, old: the
// word before locking) is in encounter order; one atomic per distinct lock,
// batched 8 at a time where the body reads or declares (will_write) several
// words at once.
#pragma once
#include "tx.cuh"

namespace gstm {

__device__ __forceinline__ unsigned long long irr_globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// The owner's lock log lives in a per-warp slice of shared memory, ent[k]
// and old[k] contiguous: one lane of the warp is ever the owner, and per-lane
// local memory is interleaved across the 32 lanes (one 128 B line per entry),
// which a single lane running alone pays for in L1 misses.
template <class TX>
struct IrrCtx {
    static constexpr int kCap = TX::kLcap;
    uint32_t* ent;                // [kCap] id<<2 | wr<<1 | 1, encounter order
    uint32_t* old;                // [kCap] the lock word before we locked it
    const Meta& m;
    unsigned long long deadline;  // watchdog: a lock never released ends the wait (bad)
    int nl = 0;
    int nr = 0;                   // reads (the op-mix statistics, S_RD_*)
    int nl_taken = 0;             // locks held at the commit (S_LK_UPD)
    int nw = 0;
    bool bad = false;
    uint32_t n_spin = 0;

    // atom.or on version lock id: the lock word alone (the paper's table), or
    // -- paired layout, one lock per word -- the whole (value, lock) pair, the
    // same 64-bit operation the other transactions use on it (tx_pair.cuh)
    __device__ __forceinline__ uint32_t lock_atom(uint32_t id, bool acquire) const
    {
        if (m.lshift) {
            const unsigned long long old = acquire ? prim::atom_or_acquire_u64(m.pair_ptr(id), 1ull << 32)
                                                   : prim::atom_or_relaxed_u64(m.pair_ptr(id), 1ull << 32);
            return static_cast<uint32_t>(old >> 32);
        }
        return acquire ? prim::atom_or_acquire(m.lock_ptr(id), 1u) : prim::atom_or_relaxed(m.lock_ptr(id), 1u);
    }

    // the lock id is held by this execution already?  (asked only when the
    // atomic found the lock held)
    __device__ __forceinline__ int find(uint32_t id) const
    {
        for (int k = 0; k < nl; ++k)
            if ((ent[k] >> 2) == id) return k;
        return -1;
    }
    // the atomic on lock id returned v: record it, or it is ours, or wait
    __device__ __forceinline__ bool settle(uint32_t id, uint32_t v, bool wr)
    {
        if (v & 1u) {
            const int k = find(id);
            if (k >= 0) {
                if (wr) ent[k] |= 2u;
                return true;
            }
            // held by a committing transaction: wait for its release
            for (uint32_t s = 1;; ++s) {
                __nanosleep(64);
                ++n_spin;
                v = lock_atom(id, true);
                if (!(v & 1u)) break;
                if ((s & 255u) == 0u && irr_globaltimer() > deadline) { bad = true; return false; }
            }
        }
        if (nl >= kCap) {                  // more locks than compiled (cannot happen: LCAP >= accesses)
            prim::st_relaxed(m.lock_ptr(id), v);
            bad = true;
            return false;
        }
        ent[nl] = (id << 2) | (wr ? 2u : 0u) | 1u;
        old[nl] = v;
        ++nl;
        return true;
    }

    __device__ __forceinline__ uint32_t read(uint32_t a)
    {
        const uint32_t id = m.lock_of(a);
        if (!settle(id, lock_atom(id, true), false)) return 0u;
        ++nr;
        return prim::ld_relaxed(m.val_ptr(a));
    }
    // a batch: every lock atomic in flight at once, then the values
    template <int N>
    __device__ __forceinline__ void read_batch(const uint32_t (&a)[N], uint32_t (&v)[N], int n, uint32_t skip = 0u)
    {
        uint32_t lv[N];
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (k < n && !((skip >> k) & 1u)) lv[k] = lock_atom(m.lock_of(a[k]), false);
        prim::fence_acquire();
        // the locks this batch took first: a later atomic of the batch on
        // the same lock may have taken it after an earlier one found it held
        // by a committer, and that earlier one must then find it as ours
        bool ok = true;
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (k < n && !((skip >> k) & 1u) && !(lv[k] & 1u)) ok &= settle(m.lock_of(a[k]), lv[k], false);
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (k < n && !((skip >> k) & 1u) && (lv[k] & 1u)) ok &= settle(m.lock_of(a[k]), lv[k], false);
        if (!ok) return;
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (k < n && !((skip >> k) & 1u)) { v[k] = prim::ld_relaxed(m.val_ptr(a[k])); ++nr; }
    }
    __device__ __forceinline__ void read_many(const uint32_t* a, uint32_t* v, const bool* skip, int n)
    {
        constexpr int C = 8;
        for (int k0 = 0; k0 < n; k0 += C) {
            uint32_t lv[C];
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && !skip[k0 + j]) lv[j] = lock_atom(m.lock_of(a[k0 + j]), false);
            prim::fence_acquire();
            bool ok = true;                                          // (the locks taken first, as in read_batch)
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && !skip[k0 + j] && !(lv[j] & 1u)) ok &= settle(m.lock_of(a[k0 + j]), lv[j], false);
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && !skip[k0 + j] && (lv[j] & 1u)) ok &= settle(m.lock_of(a[k0 + j]), lv[j], false);
            if (!ok) return;
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && !skip[k0 + j]) { v[k0 + j] = prim::ld_relaxed(m.val_ptr(a[k0 + j])); ++nr; }
        }
    }
    // will_write hint: the body's write addresses a[0], a[stride], ... in the
    // order it will write them; their locks are taken now, 8 atomics in
    // flight at a time, and a write that follows the declared order needs
    // no atomic of its own
    const uint32_t* wa = nullptr;
    int wn = 0, wstride = 1, wcur = 0;
    __device__ __forceinline__ void will_write(const uint32_t* a, int n, int stride)
    {
        constexpr int C = 8;
        wa = a; wn = n; wstride = stride; wcur = 0;
        for (int k0 = 0; k0 < n; k0 += C) {
            uint32_t lv[C];
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n) lv[j] = lock_atom(m.lock_of(a[(k0 + j) * stride]), false);
            prim::fence_acquire();
            bool ok = true;                                          // (the locks taken first, as in read_batch)
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && !(lv[j] & 1u)) ok &= settle(m.lock_of(a[(k0 + j) * stride]), lv[j], true);
#pragma unroll
            for (int j = 0; j < C; ++j)
                if (k0 + j < n && (lv[j] & 1u)) ok &= settle(m.lock_of(a[(k0 + j) * stride]), lv[j], true);
            if (!ok) { wn = 0; return; }
        }
    }
    __device__ __forceinline__ void write(uint32_t a, uint32_t val)
    {
        if (wcur < wn && a == wa[wcur * wstride]) {                 // locked by will_write
            ++wcur;
            prim::st_relaxed(m.val_ptr(a), val);
            ++nw;
            return;
        }
        const uint32_t id = m.lock_of(a);
        if (!settle(id, lock_atom(id, true), true)) return;
        prim::st_relaxed(m.val_ptr(a), val);
        ++nw;
    }
    __device__ __forceinline__ bool ok() const { return !bad; }
    __device__ __forceinline__ void invalid() { bad = true; }
    __device__ __forceinline__ void overflow() { bad = true; }
    __device__ __forceinline__ unsigned lockstep_mask() const { return 0u; }
    __device__ __forceinline__ void set_sync_mask(unsigned) {}
    static constexpr int kMaxChain = (TX::kRcap - 1) / 2;

    // l.82-84 with every lock held: fence, stamp (update) or the clock value
    // (read-only), release.  Returns the stamp, or RO-flag | clock value.
    __device__ __forceinline__ uint32_t commit(unsigned long long* clock)
    {
        prim::fence_release();                                       // l.82: in-place writes first
        uint32_t s;
        if (nw) s = static_cast<uint32_t>(clock_fetch_add(clock, 1u)) + 1u;   // l.83
        else s = 0x80000000u | static_cast<uint32_t>(prim::ld_acquire64(clock));
        if (GSTM_STRICT_FENCES) prim::fence_release();
        const uint32_t version = s << 1;
        for (int k = 0; k < nl; ++k)                                 // l.84
            prim::st_relaxed(m.lock_ptr(ent[k] >> 2), (ent[k] & 2u) ? version : old[k]);
        nl_taken = nl;
        nl = 0;
        return s;
    }
};

}  // namespace gstm
