// tx_pair.cuh -- GPU-STM on the PAIRED layout.
//
// The paper keeps a global table of version locks apart from the data and
// maps word w to lock hash(w).  When the table has one lock
// per word (2^bits >= heap words, stripe 1 -- the regime where P:252 picks
// TBV), the same logical structure can be laid out B200-first: word w and its
// version lock share one naturally aligned u64 (value in the low half, lock
// word in the high half).  Then
//   * TXRead is ONE 8-byte strong load: value and version lock read
//     atomically together (A3.l24 and l.28 at one instant, no fence l.26);
//   * PostValidation checks value and lock of each read word in one pass;
//   * lock acquisition `atom.or.b64` returns the word's current value with
//     the old lock, so the VBV under locks (A3.l76) needs no memory access;
//   * write-back and lock release of a written word are one 8-byte store
//     (value, stamp<<1), issued after the stamp: a reader that sees the word
//     still locked waits (A3.l27-29), so publishing the value with the
//     unlock is equivalent to l.80-84 and needs no release fence (l.82).
// Per bank transaction: 2 + 2 + 2 (+ clock) L2 requests instead of 14.
#pragma once
#include "tx.cuh"

namespace gstm {

template <int RCAP, int WCAP, int LCAP, bool LOCAL = false, bool SORTED = true, bool COMPACT = false,
          bool HLOG = false, bool SMEM = false, bool COLDPV = false>
struct TxPair : Tx<RCAP, WCAP, LCAP, LOCAL, SORTED, COMPACT, HLOG, SMEM, COLDPV> {
    using B = Tx<RCAP, WCAP, LCAP, LOCAL, SORTED, COMPACT, HLOG, SMEM, COLDPV>;
    using B::kUnroll;
    using B::r_addr;
    using B::r_val;
    using B::w_addr;
    using B::w_val;
    using B::l_ent;
    using B::l_old;
    using B::nr;
    using B::nw;
    using B::nl;
    using B::n_acq;
    using B::snapshot;
    using B::opaque;
    using B::passTBV;
    using B::n_postval;
    using B::n_vbv;
    using B::n_spin;
    using B::raw_lookup;
    using B::append_read;
    using B::reconverge;
    using B::insert_lock;
    using B::insert_read_lock;
    using B::kCompact;
    using B::ph;

    uint32_t l_val[LCAP];   // value each acquiring atom.or.b64 returned

    static __device__ __forceinline__ uint32_t lo(unsigned long long p) { return static_cast<uint32_t>(p); }
    static __device__ __forceinline__ uint32_t hi(unsigned long long p) { return static_cast<uint32_t>(p >> 32); }
    static __device__ __forceinline__ unsigned long long mk(uint32_t val, uint32_t lock)
    {
        return (static_cast<unsigned long long>(lock) << 32) | val;
    }

    // ---- A3.l6-20 PostValidation: value and lock of every read word from
    //      one atomic 8-byte load (l.9-11 and l.13-19 in one pass) --------
    __device__ __forceinline__ bool post_validation(const Meta& m, uint32_t version)
    {
        ++n_postval;
        ++n_vbv;
        if (version > snapshot) snapshot = version;                  // l.7 (Q9)
        for (uint32_t restart = 0; restart <= m.spin_cap; ++restart) {  // l.8
            bool again = false, ok = true;
            uint32_t newsnap = snapshot;
            if constexpr (kUnroll) {
                unsigned long long pv[RCAP];
#pragma unroll
                for (int k = 0; k < RCAP; ++k)
                    if (k < nr) pv[k] = prim::ld_relaxed_u64(m.pair_ptr(r_addr[k]));
#pragma unroll
                for (int k = 0; k < RCAP; ++k)
                    if (k < nr) {
                        ok &= (lo(pv[k]) == r_val[k]);                  // l.10
                        const uint32_t vl = hi(pv[k]);
                        if ((vl & 1u) || (vl >> 1) > snapshot) { newsnap = max(newsnap, vl >> 1); again = true; }
                    }
            } else {
                for (int k0 = 0; k0 < nr; k0 += 8) {                 // 8 pair loads in flight
                    unsigned long long pv[8];
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        if (k0 + j < nr) pv[j] = prim::ld_relaxed_u64(m.pair_ptr(r_addr[k0 + j]));
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        if (k0 + j < nr) {
                            ok &= (lo(pv[j]) == r_val[k0 + j]);
                            const uint32_t vl = hi(pv[j]);
                            if ((vl & 1u) || (vl >> 1) > snapshot) { newsnap = max(newsnap, vl >> 1); again = true; }
                        }
                }
            }
            if (!ok) return false;                                   // l.11
            snapshot = newsnap;                                      // l.18
            if (!again) return true;                                 // l.20
            if (restart) __nanosleep(64);
        }
        return false;
    }

    // A3.l27-29: while the word is locked re-read the pair (value and lock),
    // so the logged value is the one that goes with the version checked
    __device__ __forceinline__ unsigned long long settle(const Meta& m, uint32_t a, unsigned long long pv)
    {
        uint32_t spins = 0;
        while (hi(pv) & 1u) {
            if (++spins > m.spin_cap) { opaque = false; break; }
            if (GSTM_SPIN_NS) __nanosleep(GSTM_SPIN_NS);
            pv = prim::ld_relaxed_u64(m.pair_ptr(a));
        }
        n_spin += spins;
        return pv;
    }

    // A3.l30-33
    __device__ __forceinline__ void check_version(const Meta& m, uint32_t vl, int mode)
    {
        const uint32_t version = vl >> 1;
        if (opaque && version > snapshot) {
            if (mode == MODE_HV) {
                if (!post_validation(m, version)) opaque = false;
            } else {
                opaque = false;
            }
        }
    }

    __device__ __forceinline__ uint32_t read(const Meta& m, uint32_t a, int mode)
    {
        uint32_t v;
        ph(PH_BUFFER);
        if (raw_lookup(a, v)) { ph(PH_NATIVE); return v; }          // l.22-23
        unsigned long long pv = prim::ld_relaxed_u64(m.pair_ptr(a)); // l.24 (+ l.28)
        ph(PH_CONSIST);
        pv = settle(m, a, pv);                                       // l.27-29
        v = lo(pv);
        ph(PH_BUFFER);
        append_read(a, v);                                           // l.25
        ph(PH_CONSIST);
        check_version(m, hi(pv), mode);                              // l.30-33
        ph(PH_BUFFER);
        insert_read_lock(a);                                         // l.34 (lock id = word)
        ph(PH_NATIVE);
        return v;
    }

    template <int N>
    __device__ __forceinline__ void read_batch(const Meta& m, const uint32_t (&a)[N], uint32_t (&v)[N], int n, int mode,
                                               uint32_t skip = 0u)
    {
        bool need[N];
        unsigned long long pv[N];
        ph(PH_BUFFER);
#pragma unroll
        for (int k = 0; k < N; ++k) need[k] = (k < n) && !((skip >> k) & 1u) && !raw_lookup(a[k], v[k]);
#pragma unroll
        for (int k = 0; k < N; ++k)
            if (need[k]) pv[k] = prim::ld_relaxed_u64(m.pair_ptr(a[k]));
        ph(PH_CONSIST);
        if constexpr (N <= 4) {
            // small batches (bank: 2), fully unrolled: ONE spin loop re-reads
            // every still-locked pair of the batch together (l.27-29), and ONE
            // timestamp check with the newest version (Q35) -- a single copy
            // of each rare path, so lanes of a warp that take it take it
            // together instead of one after the other
            uint32_t spins = 0;
            bool locked = false;
#pragma unroll
            for (int k = 0; k < N; ++k) locked |= need[k] && (hi(pv[k]) & 1u);
            while (locked) {
                if (++spins > m.spin_cap) { opaque = false; break; }
                if (GSTM_SPIN_NS) __nanosleep(GSTM_SPIN_NS);
#pragma unroll
                for (int k = 0; k < N; ++k)
                    if (need[k] && (hi(pv[k]) & 1u)) pv[k] = prim::ld_relaxed_u64(m.pair_ptr(a[k]));
                locked = false;
#pragma unroll
                for (int k = 0; k < N; ++k) locked |= need[k] && (hi(pv[k]) & 1u);
            }
            n_spin += spins;
            reconverge();
            uint32_t newest = 0;
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k]) {
                    v[k] = lo(pv[k]);
                    append_read(a[k], v[k]);
                    newest = max(newest, hi(pv[k]) >> 1);
                }
            check_version(m, newest << 1, mode);                      // l.30-33 (Q35)
            reconverge();
            ph(PH_BUFFER);
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k]) insert_read_lock(a[k]);                 // l.34
        } else {
            uint32_t newest = 0;
#pragma unroll
            for (int k = 0; k < N; ++k)
                if (need[k]) {
                    pv[k] = settle(m, a[k], pv[k]);
                    v[k] = lo(pv[k]);
                    append_read(a[k], v[k]);
                    newest = max(newest, hi(pv[k]) >> 1);
                }
            reconverge();
            // one merged timestamp check per batch (tx.cuh read_batch)
            check_version(m, newest << 1, mode);
            reconverge();
            ph(PH_BUFFER);
#pragma unroll 1
            for (int k = 0; k < N; ++k) {
                uint32_t ak = 0;
                bool nk = false;
#pragma unroll
                for (int j = 0; j < N; ++j)
                    if (j == k) { ak = a[j]; nk = need[j]; }
                if (nk) insert_read_lock(ak);
            }
        }
        ph(PH_NATIVE);
    }

    __device__ __forceinline__ void read_many(const Meta& m, const uint32_t* a, uint32_t* v, const bool* skip, int n,
                                              int mode)
    {
        uint32_t vl[RCAP];
        ph(PH_BUFFER);
#pragma unroll 8
        for (int k = 0; k < n; ++k)
            if (!skip[k]) {
                const unsigned long long pv = prim::ld_relaxed_u64(m.pair_ptr(a[k]));
                v[k] = lo(pv);
                vl[k] = hi(pv);
            }
        for (int k = 0; k < n; ++k)
            if (!skip[k]) {
                if (vl[k] & 1u) {
                    ph(PH_CONSIST);
                    const unsigned long long pv = settle(m, a[k], mk(v[k], vl[k]));
                    v[k] = lo(pv);
                    vl[k] = hi(pv);
                    ph(PH_BUFFER);
                }
                append_read(a[k], v[k]);
            }
        for (int k = 0; k < n; ++k)
            if (!skip[k]) {
                ph(PH_CONSIST);
                check_version(m, vl[k], mode);
                ph(PH_BUFFER);
                insert_read_lock(a[k]);
            }
        ph(PH_NATIVE);
    }

    // ---- A3.l62-66 VBV from the values in memory --------------------------
    __device__ __forceinline__ bool vbv(const Meta& m)
    {
        ++n_vbv;
        bool ok = true;
        if constexpr (kUnroll) {
            unsigned long long pv[RCAP];
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
                if (k < nr) pv[k] = prim::ld_relaxed_u64(m.pair_ptr(r_addr[k]));
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
                if (k < nr) ok &= (lo(pv[k]) == r_val[k]);
        } else {
            for (int k0 = 0; k0 < nr; k0 += 8) {                     // 8 pair loads in flight
                uint32_t cur[8];
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    if (k0 + j < nr) cur[j] = lo(prim::ld_relaxed_u64(m.pair_ptr(r_addr[k0 + j])));
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    if (k0 + j < nr) ok &= (cur[j] == r_val[k0 + j]);
            }
        }
        return ok;
    }

    // ---- A3.l76 VBV under locks, from the values the atomics returned ----
    __device__ __forceinline__ bool vbv_locked()
    {
        ++n_vbv;
        bool ok = true;
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < RCAP; ++k)
#pragma unroll
                for (int j = 0; j < LCAP; ++j)
                    if (k < nr && j < nl && (l_ent[j] >> 2) == r_addr[k]) ok &= (l_val[j] == r_val[k]);
        } else {
            for (int k = 0; k < nr; ++k)
                for (int j = 0; j < nl; ++j)
                    if ((l_ent[j] >> 2) == r_addr[k]) { ok &= (l_val[j] == r_val[k]); break; }
        }
        return ok;
    }

    // ---- A3.l53-55 ReleaseLocks: put back the exact pairs we locked -------
    __device__ __forceinline__ void release_locks(const Meta& m)
    {
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)
                if (k < n_acq) prim::st_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), mk(l_val[k], l_old[k]));
        } else {
            for (int k = 0; k < n_acq; ++k) prim::st_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), mk(l_val[k], l_old[k]));
        }
        n_acq = 0;
    }

    // ---- A3.l43-52 GetLocksAndTBV, sequential in ascending id -------------
    __device__ __forceinline__ bool get_locks_and_tbv(const Meta& m)
    {
        B::compact();
        n_acq = 0;
        bool ok = true;
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k) {
                if (ok && k < nl) {
                    const unsigned long long old = prim::atom_or_acquire_u64(m.pair_ptr(l_ent[k] >> 2), 1ull << 32);  // l.45
                    if (hi(old) & 1u) {
                        ok = false;                                  // l.46-48
                    } else {
                        l_old[k] = hi(old);
                        l_val[k] = lo(old);
                        n_acq = k + 1;
                        if ((l_ent[k] & 1u) && (hi(old) >> 1) > snapshot) passTBV = false;  // l.49-51
                    }
                }
            }
        } else {
            for (int k = 0; k < nl; ++k) {
                const unsigned long long old = prim::atom_or_acquire_u64(m.pair_ptr(l_ent[k] >> 2), 1ull << 32);
                if (hi(old) & 1u) { ok = false; break; }
                l_old[k] = hi(old);
                l_val[k] = lo(old);
                n_acq = k + 1;
                if ((l_ent[k] & 1u) && (hi(old) >> 1) > snapshot) passTBV = false;
            }
        }
        if (!ok) release_locks(m);                                   // l.47
        return ok;
    }

    // Register-resident logs: the pipelined first round and the sequential
    // sorted acquisition in ONE code path (tx.cuh get_locks_and_tbv_converged):
    // round 0 issues entry 0 for every lane and every entry for a pipelined
    // lane; sequential lanes then take entries 1.. one at a time, stopping at
    // the first held lock (Q15), in lockstep with each other.
    __device__ __forceinline__ bool get_locks_and_tbv_converged(const Meta& m, bool pipelined)
    {
        static_assert(kUnroll, "converged acquisition needs register-resident logs");
        unsigned long long old[LCAP];
        bool ok = true;
        uint32_t set = 0;   // entries this attempt locked
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl && (k == 0 || pipelined)) old[k] = prim::atom_or_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), 1ull << 32);  // l.45
        prim::fence_acquire();
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl && (k == 0 || pipelined)) {
                if (hi(old[k]) & 1u) ok = false;                     // l.46
                else set |= 1u << k;
            }
#pragma unroll
        for (int k = 1; k < LCAP; ++k)
            if (!pipelined && ok && k < nl) {                        // sequential: next entry only after the last succeeded
                old[k] = prim::atom_or_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), 1ull << 32);
                prim::fence_acquire();
                if (hi(old[k]) & 1u) ok = false;
                else set |= 1u << k;
            }
        if (!ok) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)                           // l.47: undo what this attempt set
                if (set & (1u << k)) prim::st_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), old[k]);
            n_acq = 0;
            return false;
        }
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < nl) {
                l_old[k] = hi(old[k]);
                l_val[k] = lo(old[k]);
                if ((l_ent[k] & 1u) && (hi(old[k]) >> 1) > snapshot) passTBV = false;  // l.49-51
            }
        n_acq = nl;
        return true;
    }

    // local-memory logs: kChunk atom.or.b64 at a time (tx.cuh)
    static constexpr int kChunk = 8;
    __device__ __forceinline__ bool get_locks_and_tbv_pipelined_local(const Meta& m)
    {
        bool ok = true;
        for (int k0 = 0; k0 < nl; k0 += kChunk) {
            unsigned long long old[kChunk];
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) old[j] = prim::atom_or_relaxed_u64(m.pair_ptr(l_ent[k0 + j] >> 2), 1ull << 32);
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) {
                    l_old[k0 + j] = hi(old[j]);
                    l_val[k0 + j] = lo(old[j]);
                    ok &= !(hi(old[j]) & 1u);
                }
        }
        prim::fence_acquire();
        if (!ok) {
            for (int k = 0; k < nl; ++k)
                if (!(l_old[k] & 1u)) prim::st_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), mk(l_val[k], l_old[k]));
            n_acq = 0;
            return false;
        }
        for (int k = 0; k < nl; ++k)
            if ((l_ent[k] & 1u) && (l_old[k] >> 1) > snapshot) passTBV = false;
        n_acq = nl;
        return true;
    }

    // the gated pipelined round (tx.cuh get_locks_and_tbv_gated_local) on pairs
    __device__ __forceinline__ bool get_locks_and_tbv_gated_local(const Meta& m)
    {
        n_acq = 0;
        const unsigned long long o0 = prim::atom_or_acquire_u64(m.pair_ptr(l_ent[0] >> 2), 1ull << 32);   // the gate
        if (hi(o0) & 1u) return false;
        l_old[0] = hi(o0);
        l_val[0] = lo(o0);
        bool ok = true;
        for (int k0 = 1; k0 < nl; k0 += kChunk) {
            unsigned long long old[kChunk];
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) old[j] = prim::atom_or_relaxed_u64(m.pair_ptr(l_ent[k0 + j] >> 2), 1ull << 32);
#pragma unroll
            for (int j = 0; j < kChunk; ++j)
                if (k0 + j < nl) {
                    l_old[k0 + j] = hi(old[j]);
                    l_val[k0 + j] = lo(old[j]);
                    ok &= !(hi(old[j]) & 1u);
                }
        }
        prim::fence_acquire();
        if (!ok) {
            for (int k = 0; k < nl; ++k)
                if (!(l_old[k] & 1u)) prim::st_relaxed_u64(m.pair_ptr(l_ent[k] >> 2), mk(l_val[k], l_old[k]));
            return false;
        }
        for (int k = 0; k < nl; ++k)
            if ((l_ent[k] & 1u) && (l_old[k] >> 1) > snapshot) passTBV = false;
        n_acq = nl;
        return true;
    }

    // want_pipe: this round may be the pipelined first round (§6.4); it is,
    // for local-memory logs, only if the (complete) log has at most
    // max_pipe_locks entries -- pipelined_round reports the decision
    __device__ __forceinline__ int commit_acquire(const Meta& m, int mode, bool prelock_vbv, bool want_pipe = false,
                                                  uint32_t max_pipe_locks = 8u, bool gated = false)
    {
        ph(PH_BUFFER);
        B::insert_deferred_reads(m);
        B::compact();
        const bool pipelined = want_pipe && (kUnroll || nl <= static_cast<int>(max_pipe_locks));
        const bool gate = want_pipe && gated && !pipelined && !kUnroll;
        B::pipelined_round = pipelined || gate;
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
            if (mode != MODE_HV) { release_locks(m); return C_TBV; }
            ph(PH_CONSIST);
            const bool ok = vbv_locked();
            ph(PH_LOCKS);
            if (!ok) { release_locks(m); return C_COMMITVBV; }       // l.76-78
        }
        ph(PH_COMMIT);
        return C_OK;
    }

    // l.79-82: nothing to do here -- each written value is published
    // together with its unlock in release_and_update
    __device__ __forceinline__ void writeback(const Meta&) {}
    __device__ __forceinline__ void writeback_runs(const Meta&) {}

    // ---- A3.l80-84: written pairs get (new value, stamp<<1); read-only
    //      pairs get back exactly what the atomic returned --------------------
    __device__ __forceinline__ void release_and_update(const Meta& m, uint32_t version)
    {
        ph(PH_COMMIT);                   // the value write-back IS the release store here (l.80-84)
        if constexpr (kUnroll) {
#pragma unroll
            for (int k = 0; k < LCAP; ++k)
                if (k < nl) {
                    const uint32_t id = l_ent[k] >> 2;
                    uint32_t val = l_val[k], lock = l_old[k];
                    if (l_ent[k] & 2u) {
                        lock = version << 1;
#pragma unroll
                        for (int j = 0; j < WCAP; ++j)
                            if (j < nw && w_addr[j] == id) val = w_val[j];
                    }
                    prim::st_relaxed_u64(m.pair_ptr(id), mk(val, lock));
                }
        } else {
            for (int k = 0; k < nl; ++k) {
                const uint32_t id = l_ent[k] >> 2;
                uint32_t val = l_val[k], lock = l_old[k];
                if (l_ent[k] & 2u) {
                    lock = version << 1;
                    for (int j = 0; j < nw; ++j)
                        if (w_addr[j] == id) { val = w_val[j]; break; }
                }
                prim::st_relaxed_u64(m.pair_ptr(id), mk(val, lock));
            }
        }
        n_acq = 0;
    }
};

}  // namespace gstm
