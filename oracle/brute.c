/*
 * brute.c -- every serial order of a tiny transaction set.  TEST
 * INFRASTRUCTURE.
 *
 * Serializability ("all transactions would appear to occur in some
 * global total order") admits several correct final states.  For tiny inputs
 * (<= ~10 transactions) we enumerate every total order that keeps each
 * thread's transactions in program order (i ascending), execute each order
 * serially (serial.c), and ask whether the queried (heap, results) outcome is
 * among them.  This check does not trust any commit log.
 */
#include <stdlib.h>
#include <string.h>
#include "oracle.h"

#define MAXT 16
#define HSET_BITS 20

typedef struct {
    const or_params_t* p;
    uint64_t words, T, K, seed, n;
    const uint32_t* heap_q; const uint32_t* results_q;
    uint32_t* results;     /* by tx_id, filled along the current path */
    uint64_t next[MAXT];
    int64_t visited;
    int match;
    uint64_t* hset; int64_t n_distinct; int err;
} bf_t;

static uint64_t fnv(uint64_t h, const uint32_t* w, uint64_t n)
{
    for (uint64_t k = 0; k < n; ++k) { h ^= w[k]; h *= 0x100000001b3ull; h ^= h >> 29; }
    return h;
}

static void hset_add(bf_t* b, uint64_t h)
{
    if (h == 0) h = 1;
    uint64_t m = (1ull << HSET_BITS) - 1, s = h & m;
    for (uint64_t probe = 0; probe <= m; ++probe, s = (s + 1) & m) {
        if (b->hset[s] == h) return;
        if (b->hset[s] == 0) { b->hset[s] = h; b->n_distinct++; return; }
    }
}

static void rec(bf_t* b, const uint32_t* heap, uint64_t depth)
{
    if (b->err) return;
    if (depth == b->n) {
        b->visited++;
        uint64_t h = fnv(fnv(0xcbf29ce484222325ull, heap, b->words), b->results, b->n);
        hset_add(b, h);
        if (!b->match && b->heap_q && b->results_q &&
            memcmp(heap, b->heap_q, b->words * 4) == 0 &&
            memcmp(b->results, b->results_q, b->n * 4) == 0)
            b->match = 1;
        return;
    }
    uint32_t* h2 = (uint32_t*)malloc(b->words * 4);
    if (!h2) { b->err = 1; return; }
    for (uint64_t t = 0; t < b->T; ++t) {
        if (b->next[t] >= b->K) continue;
        uint64_t i = b->next[t];
        memcpy(h2, heap, b->words * 4);
        uint32_t r; int u;
        if (or_exec_tx(b->p, h2, b->words, b->T, b->K, b->seed, t, i, &r, &u)) { b->err = 1; break; }
        b->results[i * b->T + t] = r;
        b->next[t]++;
        rec(b, h2, depth + 1);
        b->next[t]--;
    }
    free(h2);
}

int64_t or_brute(const or_params_t* p, const uint32_t* init, uint64_t words,
                 uint64_t T, uint64_t K, uint64_t seed,
                 const uint32_t* heap_q, const uint32_t* results_q,
                 int* match, int64_t* n_distinct)
{
    if (T == 0 || T > MAXT || T * K > 24) return -1;
    bf_t b;
    memset(&b, 0, sizeof(b));
    b.p = p; b.words = words; b.T = T; b.K = K; b.seed = seed; b.n = T * K;
    b.heap_q = heap_q; b.results_q = results_q;
    b.results = (uint32_t*)calloc(b.n + 1, 4);
    b.hset = (uint64_t*)calloc(1ull << HSET_BITS, 8);
    if (!b.results || !b.hset) { free(b.results); free(b.hset); return -2; }
    rec(&b, init, 0);
    free(b.results); free(b.hset);
    if (b.err) return -3;
    if (match) *match = b.match;
    if (n_distinct) *n_distinct = b.n_distinct;
    return b.visited;
}
