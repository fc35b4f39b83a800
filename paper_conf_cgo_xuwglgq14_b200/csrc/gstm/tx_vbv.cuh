// tx_vbv.cuh -- STM-VBV: value-based validation behind one global sequence
// lock, the NOrec-like variant the paper compares against (P:103, P:250,
// P:290).
//
// "A single global sequence lock (as used in NOrec [5]) can be used to filter
// out unnecessary validations ... during commit, memory updates of all
// transactions are serialized by the single lock".  The paper gives
// no pseudo-code; the steps below are NOrec's (Q33):
//   * seq (u64): even = no writer; a writer holds it (odd) while it writes
//     back.  seq = 2 * g_clock at the start of every launch, and a writer
//     committing from seq s stamps s/2 + 1 and stores it to g_clock, so the
//     commit stamps stay dense and the replay check applies unchanged.
//   * TXBegin: snapshot = seq once it is even.
//   * TXRead: value load (read-after-write through the write-set first),
//     append <addr,val> to the read-set; if seq moved since the snapshot,
//     revalidate: wait until seq is even, compare every logged value with
//     memory, and keep the result only if seq did not move meanwhile (the
//     read-set is then consistent at that new snapshot); a mismatch aborts.
//   * TXWrite: redo log (upsert), no locks.
//   * TXCommit: read-only -> commit at the snapshot.  Writer: CAS seq
//     snapshot -> snapshot+1; on failure revalidate and retry; then write
//     back, store the stamp to g_clock, release seq = snapshot+2.
// No version lock table is read or written.  Works on both heap layouts (only
// the value half of a paired word is touched).
#pragma once
#include <cstdint>
#include "prim.cuh"
#include "tx.cuh"

namespace gstm {

template <int RCAP, int WCAP, bool LOCAL = false>
struct TxVbv {
    static constexpr bool kUnroll = !LOCAL && (RCAP <= 24 && WCAP <= 24);
    static constexpr int kRcap = RCAP, kWcap = WCAP;

    uint32_t r_addr[RCAP], r_val[RCAP];
    uint32_t w_addr[WCAP], w_val[WCAP];
    unsigned long long bloom;
    unsigned long long* seq;              // the global sequence lock
    unsigned long long snapshot;          // an even seq value
    int nr, nw;
    bool opaque, overflow;
    uint32_t n_postval, n_vbv, n_spin;    // revalidations, value checks, spins

    __device__ __forceinline__ void reset_stats() { n_postval = n_vbv = n_spin = 0; }
    __device__ __forceinline__ bool read_only() const { return nw == 0; }

    // wait until no writer holds seq; false if the spin bound is hit
    __device__ __forceinline__ bool wait_even(const Meta& m, unsigned long long& s)
    {
        uint32_t spins = 0;
        s = prim::ld_acquire64(seq);
        while (s & 1ull) {
            if (++spins > m.spin_cap) { n_spin += spins; return false; }
            __nanosleep(32);
            s = prim::ld_acquire64(seq);
        }
        n_spin += spins;
        return true;
    }

    __device__ __forceinline__ void begin(const Meta& m, unsigned long long* seq_lock)
    {
        seq = seq_lock;
        nr = nw = 0;
        bloom = 0ull;
        overflow = false;
        opaque = wait_even(m, snapshot);
    }

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

    // every logged value still in memory
    __device__ __forceinline__ bool values_match(const Meta& m)
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
        } else {
            for (int k = 0; k < nr; ++k) ok &= (prim::ld_relaxed(m.val_ptr(r_addr[k])) == r_val[k]);
        }
        return ok;
    }

    // NOrec Validate: a seq value at which every logged value held
    __device__ __forceinline__ bool revalidate(const Meta& m)
    {
        ++n_postval;
        for (uint32_t round = 0; round <= m.spin_cap; ++round) {
            unsigned long long s;
            if (!wait_even(m, s)) return false;
            const bool ok = values_match(m);
            prim::fence_acquire();                      // value loads before the seq re-check
            if (prim::ld_relaxed64(seq) == s) {
                if (!ok) return false;
                snapshot = s;
                return true;
            }
        }
        return false;
    }

    // after new values were logged: still at the snapshot, or revalidate
    __device__ __forceinline__ void check_snapshot(const Meta& m)
    {
        prim::fence_acquire();                          // value loads before the seq load
        if (prim::ld_relaxed64(seq) != snapshot && !revalidate(m)) opaque = false;
    }

    __device__ __forceinline__ uint32_t read(const Meta& m, uint32_t a, int)
    {
        uint32_t v;
        if (!opaque) return 0;
        if (raw_lookup(a, v)) return v;
        v = prim::ld_relaxed(m.val_ptr(a));
        append_read(a, v);
        check_snapshot(m);
        return v;
    }

    template <int N>
    __device__ __forceinline__ void read_batch(const Meta& m, const uint32_t (&a)[N], uint32_t (&v)[N], int n, int,
                                               uint32_t skip = 0u)
    {
        if (!opaque) return;
        bool need[N];
#pragma unroll
        for (int k = 0; k < N; ++k) need[k] = (k < n) && !((skip >> k) & 1u) && !raw_lookup(a[k], v[k]);
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) append_read(a[k], v[k]);
        check_snapshot(m);
    }

    __device__ __forceinline__ void read_many(const Meta& m, const uint32_t* a, uint32_t* v, const bool* skip, int n, int)
    {
        if (!opaque) return;
#pragma unroll 8
        for (int k = 0; k < n; ++k)
            if (!skip[k]) v[k] = prim::ld_relaxed(m.val_ptr(a[k]));
        for (int k = 0; k < n; ++k)
            if (!skip[k]) append_read(a[k], v[k]);
        check_snapshot(m);
    }

    __device__ __forceinline__ void write(const Meta&, uint32_t a, uint32_t v)
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
        if (found) return;
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

    // Writer commit, one attempt: C_OK with seq held (odd), C_LOCK if another
    // writer got there first but the read-set is still valid at the new
    // snapshot (retry), C_COMMITVBV if it is not (abort).
    __device__ __forceinline__ int try_lock(const Meta& m)
    {
        if (prim::atom_cas_acquire64(seq, snapshot, snapshot + 1ull) == snapshot) return C_OK;
        return revalidate(m) ? C_LOCK : C_COMMITVBV;
    }

    // holding seq: write back, stamp, release.  Returns the stamp.
    __device__ __forceinline__ uint32_t writeback_and_release(const Meta& m)
    {
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < WCAP; ++k)
                if (k < nw) prim::st_relaxed(m.val_ptr(w_addr[k]), w_val[k]);
        } else {
            for (int k = 0; k < nw; ++k) prim::st_relaxed(m.val_ptr(w_addr[k]), w_val[k]);
        }
        const unsigned long long stamp = (snapshot >> 1) + 1ull;
        prim::st_relaxed64(m.clock, stamp);
        prim::fence_release();                          // write-back and stamp before the release
        prim::st_relaxed64(seq, snapshot + 2ull);
        return static_cast<uint32_t>(stamp);
    }
};

}  // namespace gstm
