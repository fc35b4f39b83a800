/*
 * alg3.c -- Algorithm 3 of the paper as a sequential model.
 * TEST INFRASTRUCTURE.
 *
 * Each function below follows one routine of Algorithm 3, in the paper's
 * order and notation; the comment on each step gives its Algorithm 3 line
 * ("l.k") and, where the extracted text is garbled or silent, the reading
 * taken (SURVEY §8c Q-numbers).  The model runs a script of
 * TXBegin / TXRead / TXWrite / TXCommit calls from several transactions,
 * interleaved one call at a time on one CPU thread, over a heap, a global
 * version-lock table and a global clock.  Because calls are atomic here, no
 * lock is ever held between calls, so the spin at l.27-29 and the lock
 * failure at l.46-48 never trigger; fences (l.5, 12, 26, 79, 82) have no
 * effect on one thread and are marked only.
 *
 * Metadata: global lock table of unsigned words, LSB = locked,
 * bits 31..1 = version; hash(addr) = addr mod 2^bits (reading Q2:
 * the "2nd-21th address bits" of a byte address = the low bits of the word
 * index).  Local lock log entries are lock_id<<2 | wr<<1 | rd, kept
 * sorted by lock id with duplicates merged (readings Q3/Q4).
 */
#include <string.h>
#include "oracle.h"

#define MAXLOG 512
#define MAXTX 16

typedef struct { uint64_t addr; uint32_t val; } entry_t;

typedef struct {
    entry_t  reads[MAXLOG];  int n_reads;   /* read-set  <addr,val>  */
    entry_t  writes[MAXLOG]; int n_writes;  /* write-set <addr,val> (redo)   */
    uint64_t bloom;                         /* write-set bloom filter*/
    uint32_t l_lockTab[MAXLOG]; int n_locks;/* sorted local lock table       */
    uint32_t acquired_old[MAXLOG]; int n_acquired;
    int      isOpaque, passTBV;
    uint64_t snapshot;
    int      postval_ran, vbv_runs;
} tx_t;

typedef struct {
    int mode, prelock_vbv;
    uint32_t mask;            /* 2^bits - 1 */
    uint32_t* heap; uint64_t words;
    uint32_t* g_lockTab;
    uint64_t g_clock;
} stm_t;

static uint32_t hash_addr(const stm_t* g, uint64_t addr) { return (uint32_t)(addr & g->mask); }

/* bloom bit (reading Q7): top 6 bits of a Fibonacci hash of the word index */
static uint64_t bloom_bit(uint64_t addr) { return 1ull << ((addr * 0x9E3779B97F4A7C15ull) >> 58); }

/* Sorted insert into the local lock table, merging a duplicate's rd/wr bits
 * ("a lock is inserted into a corresponding position in an
 * already-sorted lock-log"; "a lock is not inserted when the same lock
 * already exists").  The O(n^2) form of P:113; the bucketed form of P:115
 * produces the same ascending sequence. */
static int lock_log_insert(uint32_t* log, int* n, int cap, uint32_t entry)
{
    uint32_t id = entry >> 2;
    int pos = 0;
    while (pos < *n && (log[pos] >> 2) < id) ++pos;
    if (pos < *n && (log[pos] >> 2) == id) { log[pos] |= (entry & 3u); return 0; }
    if (*n >= cap) return -1;
    for (int k = *n; k > pos; --k) log[k] = log[k - 1];
    log[pos] = entry;
    ++*n;
    return 0;
}

int or_lock_log(const uint32_t* entries, int n, uint32_t* out, int cap)
{
    int m = 0;
    for (int k = 0; k < n; ++k)
        if (lock_log_insert(out, &m, cap, entries[k])) return -1;
    return m;
}

/* Encounter-order lock log (Q32): the lock order of STM-HV-Backoff
 * (P:250), which does not sort -- each lock id appears once, at the position
 * of its first access, carrying the OR of the rd/wr bits of all its accesses. */
int or_lock_log_encounter(const uint32_t* entries, int n, uint32_t* out, int cap)
{
    int m = 0;
    for (int k = 0; k < n; ++k) {
        const uint32_t id = entries[k] >> 2;
        int j = 0;
        while (j < m && (out[j] >> 2) != id) ++j;
        if (j < m) { out[j] |= entries[k] & 3u; continue; }
        if (m >= cap) return -1;
        out[m++] = entries[k];
    }
    return m;
}

/* 1: TXBegin */
static void TXBegin(stm_t* g, tx_t* tx)
{
    tx->n_reads = tx->n_writes = tx->n_locks = tx->n_acquired = 0;  /* l.2 */
    tx->bloom = 0;
    tx->isOpaque = tx->passTBV = 1;                                 /* l.3 */
    tx->snapshot = g->g_clock;                                      /* l.4 */
    /* l.5 threadfence() */
    tx->postval_ran = 0; tx->vbv_runs = 0;
}

/* 6: PostValidation(version) */
static int PostValidation(stm_t* g, tx_t* tx, uint64_t version)
{
    tx->postval_ran = 1;
    /* l.7 snapshot <- version; reading Q9: never lower it */
    if (version > tx->snapshot) tx->snapshot = version;
loop:                                                               /* l.8 */
    for (int k = 0; k < tx->n_reads; ++k)                           /* l.9 */
        if (g->heap[tx->reads[k].addr] != tx->reads[k].val)         /* l.10 */
            return 0;                                               /* l.11 */
    /* l.12 threadfence() */
    for (int k = 0; k < tx->n_reads; ++k) {                         /* l.13 */
        uint32_t versionLock = g->g_lockTab[hash_addr(g, tx->reads[k].addr)]; /* l.14 */
        uint32_t isLocked = versionLock & 1u;                       /* l.15 */
        uint64_t tmpVer = versionLock >> 1;                         /* l.16 */
        if (isLocked != 0 || tmpVer > tx->snapshot) {               /* l.17 */
            if (tmpVer > tx->snapshot) tx->snapshot = tmpVer;       /* l.18 (Q9) */
            goto loop;                                              /* l.19 */
        }
    }
    return 1;                                                       /* l.20 */
}

/* 21: TXRead(addr) */
static uint32_t TXRead(stm_t* g, tx_t* tx, uint64_t addr)
{
    if (tx->bloom & bloom_bit(addr))                                /* l.22, bloom P:135 */
        for (int k = 0; k < tx->n_writes; ++k)
            if (tx->writes[k].addr == addr) return tx->writes[k].val; /* l.23 */
    uint32_t val = g->heap[addr];                                   /* l.24 */
    if (tx->n_reads < MAXLOG) {                                     /* l.25 (Q5: append) */
        tx->reads[tx->n_reads].addr = addr; tx->reads[tx->n_reads].val = val; tx->n_reads++;
    }
    /* l.26 threadfence() */
    uint32_t versionLock;
    do versionLock = g->g_lockTab[hash_addr(g, addr)];              /* l.27-28 */
    while ((versionLock & 1u) != 0);                                /* l.29 (Q8) */
    uint64_t version = versionLock >> 1;                            /* l.30 */
    /* l.31; reading Q43: a transaction that is no longer opaque does not
     * re-validate (Figure 1 breaks out at the first !isOpaque) */
    if (tx->isOpaque && version > tx->snapshot) {
        if (g->mode == OR_MODE_HV) {
            if (!PostValidation(g, tx, version))                    /* l.32 */
                tx->isOpaque = 0;                                   /* l.33 */
        } else {
            tx->isOpaque = 0;   /* TBV-only variant (reading Q18) */
        }
    }
    lock_log_insert(tx->l_lockTab, &tx->n_locks, MAXLOG, (hash_addr(g, addr) << 2) | 1u); /* l.34 */
    return val;                                                     /* l.35 */
}

/* Reading Q35: a batched TXRead of two words whose
 * addresses are known together -- l.22-25 for each word (RAW from the
 * write-set, value load, append), one l.26 fence, l.27-30 for each word, then
 * ONE timestamp check l.31-33 with the newest version of the batch (the
 * outcome sequential TXReads reach: a read-set consistent at a snapshot >=
 * every version read), then l.34 for each word.  Output: vals[2]. */
static void TXRead2(stm_t* g, tx_t* tx, uint64_t a0, uint64_t a1, uint32_t* vals)
{
    uint64_t addr[2] = {a0, a1};
    int need[2];
    for (int i = 0; i < 2; ++i) {
        need[i] = 1;
        if (tx->bloom & bloom_bit(addr[i]))                         /* l.22 */
            for (int k = 0; k < tx->n_writes; ++k)
                if (tx->writes[k].addr == addr[i]) { vals[i] = tx->writes[k].val; need[i] = 0; break; } /* l.23 */
        if (need[i]) {
            vals[i] = g->heap[addr[i]];                             /* l.24 */
            if (tx->n_reads < MAXLOG) {                             /* l.25 */
                tx->reads[tx->n_reads].addr = addr[i]; tx->reads[tx->n_reads].val = vals[i]; tx->n_reads++;
            }
        }
    }
    /* l.26 threadfence() */
    uint64_t newest = 0;
    for (int i = 0; i < 2; ++i) {
        if (!need[i]) continue;
        uint32_t versionLock;
        do versionLock = g->g_lockTab[hash_addr(g, addr[i])];       /* l.27-28 */
        while ((versionLock & 1u) != 0);                            /* l.29 */
        if ((versionLock >> 1) > newest) newest = versionLock >> 1; /* l.30 */
    }
    if (tx->isOpaque && newest > tx->snapshot) {                    /* l.31, once (Q35; Q43) */
        if (g->mode == OR_MODE_HV) {
            if (!PostValidation(g, tx, newest))                     /* l.32 */
                tx->isOpaque = 0;                                   /* l.33 */
        } else {
            tx->isOpaque = 0;
        }
    }
    for (int i = 0; i < 2; ++i)
        if (need[i]) lock_log_insert(tx->l_lockTab, &tx->n_locks, MAXLOG, (hash_addr(g, addr[i]) << 2) | 1u); /* l.34 */
}

/* 36: TXWrite(addr, val) */
static void TXWrite(stm_t* g, tx_t* tx, uint64_t addr, uint32_t val)
{
    int k;
    for (k = 0; k < tx->n_writes; ++k)                              /* l.37 (Q6 upsert) */
        if (tx->writes[k].addr == addr) { tx->writes[k].val = val; break; }
    if (k == tx->n_writes && tx->n_writes < MAXLOG) {
        tx->writes[k].addr = addr; tx->writes[k].val = val; tx->n_writes++;
    }
    tx->bloom |= bloom_bit(addr);
    lock_log_insert(tx->l_lockTab, &tx->n_locks, MAXLOG, (hash_addr(g, addr) << 2) | 2u); /* l.38 */
}

/* 39-40: Atomic_or */
static uint32_t Atomic_or(uint32_t* a, uint32_t v) { uint32_t old = *a; *a = old | v; return old; }
/* 41-42: Atomic_inc */
static uint64_t Atomic_inc(uint64_t* a) { uint64_t old = *a; *a = old + 1; return old; }

/* 53: ReleaseLocks -- restore each acquired lock (l.55 "lock - 1"; Q16 stores
 * the exact old value, which equals lock - 1 because we set the LSB). */
static void ReleaseLocks(stm_t* g, tx_t* tx)
{
    for (int k = 0; k < tx->n_acquired; ++k)                        /* l.54 */
        g->g_lockTab[tx->l_lockTab[k] >> 2] = tx->acquired_old[k];  /* l.55 */
    tx->n_acquired = 0;
}

/* 43: GetLocksAndTBV */
static int GetLocksAndTBV(stm_t* g, tx_t* tx)
{
    tx->n_acquired = 0;
    for (int k = 0; k < tx->n_locks; ++k) {                         /* l.44 ascending id */
        uint32_t i = tx->l_lockTab[k] >> 2;
        uint32_t wr_rd = tx->l_lockTab[k] & 3u;
        uint32_t versionLock = Atomic_or(&g->g_lockTab[i], 1u);     /* l.45 */
        if ((versionLock & 1u) != 0) {                              /* l.46 */
            ReleaseLocks(g, tx);                                    /* l.47 */
            return 0;                                               /* l.48 */
        }
        tx->acquired_old[tx->n_acquired++] = versionLock;
        if (wr_rd & 1u)                                             /* l.49 rd = 1 */
            if ((uint64_t)(versionLock >> 1) > tx->snapshot)        /* l.50 */
                tx->passTBV = 0;                                    /* l.51 */
    }
    return 1;                                                       /* l.52 */
}

/* 56: ReleaseAndUpdateLocks(version) */
static void ReleaseAndUpdateLocks(stm_t* g, tx_t* tx, uint64_t version)
{
    for (int k = 0; k < tx->n_locks; ++k) {                         /* l.57 */
        uint32_t i = tx->l_lockTab[k] >> 2;
        if (tx->l_lockTab[k] & 2u)                                  /* l.58 wr = 1 */
            g->g_lockTab[i] = (uint32_t)(version << 1);             /* l.59 */
        else                                                        /* l.60 */
            g->g_lockTab[i] = tx->acquired_old[k];                  /* l.61 (Q16) */
    }
    tx->n_acquired = 0;
}

/* 62: VBV */
static int VBV(stm_t* g, tx_t* tx)
{
    tx->vbv_runs++;
    for (int k = 0; k < tx->n_reads; ++k)                           /* l.63 */
        if (g->heap[tx->reads[k].addr] != tx->reads[k].val)         /* l.64 */
            return 0;                                               /* l.65 */
    return 1;                                                       /* l.66 */
}

/* 67: TXCommit.  Returns ok; *cause gets OR_C_*, *stamp the version. */
static int TXCommit(stm_t* g, tx_t* tx, int* cause, uint64_t* stamp)
{
    *stamp = 0;
    if (!tx->isOpaque) { *cause = OR_C_OPACITY; return 0; }         /* Q11 */
    if (tx->n_writes == 0) { *cause = OR_C_READONLY; return 1; }    /* l.68-69 */
    int attempts = 0;
loop:                                                               /* l.70 */
    if (g->mode == OR_MODE_HV && g->prelock_vbv)                    /* l.71 "optional" (Q13) */
        if (!VBV(g, tx)) { *cause = OR_C_PREVBV; return 0; }        /* l.72 */
    if (!GetLocksAndTBV(g, tx)) {                                   /* l.73 */
        if (++attempts < 1000) goto loop;                           /* l.74 */
        *cause = OR_C_PREVBV; return 0;  /* unreachable in the sequential model */
    }
    if (tx->passTBV != 1) {                                         /* l.75 */
        if (g->mode == OR_MODE_TBV) {   /* TBV-only: no VBV, abort (Q18) */
            ReleaseLocks(g, tx); *cause = OR_C_TBV; return 0;
        }
        if (!VBV(g, tx)) {                                          /* l.76 */
            ReleaseLocks(g, tx);                                    /* l.77 */
            *cause = OR_C_COMMITVBV; return 0;                      /* l.78 */
        }
    }
    /* l.79 threadfence() */
    for (int k = 0; k < tx->n_writes; ++k)                          /* l.80 */
        g->heap[tx->writes[k].addr] = tx->writes[k].val;            /* l.81 */
    /* l.82 threadfence() */
    uint64_t version = Atomic_inc(&g->g_clock) + 1;                 /* l.83 */
    ReleaseAndUpdateLocks(g, tx, version);                          /* l.84 */
    *stamp = version; *cause = OR_C_OK;
    return 1;                                                       /* l.85 */
}

static tx_t g_txs[MAXTX];

int or_alg3_script(int mode, int prelock_vbv, uint32_t bits,
                   uint32_t* heap, uint64_t words, uint32_t* lock_tab,
                   uint64_t* clock, const uint32_t* ops, int n_ops,
                   uint32_t* out, int n_tx)
{
    if (n_tx > MAXTX || bits > 30 || (mode != OR_MODE_HV && mode != OR_MODE_TBV)) return -1;
    stm_t g;
    g.mode = mode; g.prelock_vbv = prelock_vbv;
    g.mask = (uint32_t)((1ull << bits) - 1);
    g.heap = heap; g.words = words; g.g_lockTab = lock_tab; g.g_clock = *clock;
    memset(g_txs, 0, sizeof(g_txs));
    for (int k = 0; k < n_ops; ++k) {
        uint32_t op = ops[4 * k], slot = ops[4 * k + 1], addr = ops[4 * k + 2], val = ops[4 * k + 3];
        uint32_t* o = &out[4 * k];
        o[0] = o[1] = o[2] = o[3] = 0;
        if (slot >= (uint32_t)n_tx || (op != OR_OP_BEGIN && op != OR_OP_COMMIT && addr >= words) ||
            (op == OR_OP_READ2 && val >= words)) return -2 - k;
        tx_t* tx = &g_txs[slot];
        switch (op) {
        case OR_OP_BEGIN:
            TXBegin(&g, tx);
            o[0] = (uint32_t)tx->snapshot;
            break;
        case OR_OP_READ:
            tx->postval_ran = 0;
            o[0] = TXRead(&g, tx, addr);
            o[1] = (uint32_t)tx->isOpaque; o[2] = (uint32_t)tx->snapshot; o[3] = (uint32_t)tx->postval_ran;
            break;
        case OR_OP_WRITE:
            TXWrite(&g, tx, addr, val);
            break;
        case OR_OP_READ2: {                 /* out: [val(addr), val(value field), snapshot, isOpaque | postval << 1] */
            uint32_t v2[2];
            tx->postval_ran = 0;
            TXRead2(&g, tx, addr, val, v2);
            o[0] = v2[0]; o[1] = v2[1]; o[2] = (uint32_t)tx->snapshot;
            o[3] = (uint32_t)tx->isOpaque | ((uint32_t)tx->postval_ran << 1);
            break;
        }
        case OR_OP_COMMIT: {
            int cause; uint64_t stamp;
            tx->vbv_runs = 0;
            o[0] = (uint32_t)TXCommit(&g, tx, &cause, &stamp);
            o[1] = (uint32_t)cause; o[2] = (uint32_t)stamp; o[3] = (uint32_t)tx->vbv_runs;
            break;
        }
        default:
            return -2 - k;
        }
    }
    *clock = g.g_clock;
    return 0;
}
