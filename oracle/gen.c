/*
 * gen.c -- the seeded input generator (oracle side).  TEST INFRASTRUCTURE.
 *
 * This module holds none of the method's arithmetic: it only turns
 * (seed, thread t, transaction index i) into the addresses and constants a
 * transaction uses (the "input recipe").  The CUDA side
 * implements the same recipe independently (no shared code or header); the
 * GPU-vs-oracle descriptor parity test checks that both agree bit for bit.
 *
 * Generator: SplitMix64 (Steele, Lea, Flood, "Fast splittable pseudorandom
 * number generators", OOPSLA 2014; Vigna's public-domain splitmix64.c).
 * Pinned in tests/test_oracle_gen.py against the published output vectors
 * (tests/golden/splitmix64_vectors.txt).
 *
 * The paper does not define its workloads' values (Table 1
 * lost at P:260); the recipes below are our readings (SURVEY
 * §8c-O2 / Q23), each chosen so that a lost update is observable.
 */
#include "oracle.h"

#define GOLDEN 0x9E3779B97F4A7C15ull  /* SplitMix64 increment (gamma)     */
#define TXMUL  0xC2B2AE3D27D4EB4Full  /* odd multiplier separating i      */

/* SplitMix64 output function ("mix64" / Stafford variant 13). */
uint64_t or_mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* First output of a SplitMix64 stream whose state is x. */
uint64_t or_splitmix64(uint64_t x) { return or_mix64(x + GOLDEN); }

/* k-th draw of the stream keyed by x: the (k+1)-th SplitMix64 output from
 * state x (draw(x,0), draw(x,1), ... are exactly the stream's outputs). */
uint64_t or_draw(uint64_t x, uint64_t k) { return or_splitmix64(x + k * GOLDEN); }

/* Uniform integer in [0, n): Lemire's multiply-shift, floor(r * n / 2^64). */
uint64_t or_bounded(uint64_t r, uint64_t n)
{
    return (uint64_t)(((unsigned __int128)r * (unsigned __int128)n) >> 64);
}

/* Per-transaction stream key.  A re-executed (aborted) transaction derives
 * the same key, so it regenerates the identical transaction. */
uint64_t or_txkey(uint64_t seed, uint64_t t, uint64_t i)
{
    return or_splitmix64(seed ^ (t * GOLDEN) ^ (i * TXMUL));
}

static uint32_t lo32(uint64_t v) { return (uint32_t)(v & 0xffffffffull); }

/* Descriptor layouts:
 *   RA kind 0 : r_0..r_{R-1}, w_0..w_{W-1}, c_0..c_{W-1}   (R + 2W words)
 *               r_j = bounded(draw(j), N); w_j = bounded(draw(R+j), N);
 *               c_j = lo32(draw(R+W+j))
 *   RA kind 1 : r_0..r_{R-1}                                (R words)
 *   BANK      : a, b, amt     a = bounded(draw0, N); b = bounded(draw1, N-1),
 *               b += (b >= a); amt = 1 + bounded(draw2, 100)
 *   HT        : key, is_insert, bucket
 *               key = 1 + bounded(draw0, KR); is_insert = bounded(draw1,100)
 *               >= lookup_pct; bucket = mix64(key) & (B-1)
 *   EB        : x_0..x_{A-1}, c_0..c_{A-1}   x_j = bounded(draw(j), H);
 *               c_j = lo32(draw(A+j))
 *   KM        : c, f_0..f_{D-1}   c = bounded(draw0, C); f_d = draw(1+d) >> 56
 */
uint32_t or_key_owner(uint64_t key, uint32_t bits)
{
    return bits ? (uint32_t)(or_mix64(key) >> (64 - bits)) : 0u;
}

int or_descr(const or_params_t* p, uint64_t seed, uint64_t t, uint64_t i,
             uint32_t* out, int cap)
{
    uint64_t x = or_txkey(seed, t, i);
    switch (p->workload) {
    case OR_WL_RA: {
        uint32_t R = p->n_reads, W = p->n_writes;
        uint64_t N = p->n_words, base = 0;
        if (N == 0) return -1;
        if (p->ra_partition) {
            /* disjoint access sets: thread t draws its words
             * from its own range [t*k, t*k + k) */
            base = t * (uint64_t)p->ra_partition;
            if (base + p->ra_partition > N) return -1;
            N = p->ra_partition;
        }
        if (p->ra_kind == 1) {
            if ((int)R > cap) return -1;
            for (uint32_t j = 0; j < R; ++j) out[j] = (uint32_t)(base + or_bounded(or_draw(x, j), N));
            return (int)R;
        }
        if ((int)(R + 2 * W) > cap) return -1;
        for (uint32_t j = 0; j < R; ++j) out[j] = (uint32_t)(base + or_bounded(or_draw(x, j), N));
        for (uint32_t j = 0; j < W; ++j) out[R + j] = (uint32_t)(base + or_bounded(or_draw(x, R + j), N));
        for (uint32_t j = 0; j < W; ++j) out[R + W + j] = lo32(or_draw(x, R + W + j));
        return (int)(R + 2 * W);
    }
    case OR_WL_BANK: {
        uint64_t N = p->n_words;
        if (N < 2 || cap < 3) return -1;
        uint64_t a = or_bounded(or_draw(x, 0), N);
        uint64_t b = or_bounded(or_draw(x, 1), N - 1);
        if (b >= a) b += 1;
        out[0] = (uint32_t)a; out[1] = (uint32_t)b;
        out[2] = 1u + (uint32_t)or_bounded(or_draw(x, 2), 100);
        return 3;
    }
    case OR_WL_HT: {
        if (cap < 3 || p->ht_buckets == 0 || (p->ht_buckets & (p->ht_buckets - 1))) return -1;
        if (p->shard_bits > 8 || (p->shard >> p->shard_bits) != 0) return -1;
        /* Key partition: the shard draws keys by rejection on
         * the transaction's stream -- candidate 0 is draw 0 (the unpartitioned
         * key), candidate j >= 1 is draw j+1 (draw 1 is the insert flag) --
         * and takes the first one it owns.  4096 candidates bound the loop;
         * running out (probability (1-2^-bits)^4096 < 1e-200) is an error. */
        uint64_t key = 0;
        for (uint64_t j = 0; j < 4096; ++j) {
            uint64_t k = 1 + or_bounded(or_draw(x, j ? j + 1 : 0), p->ht_key_range);
            if (or_key_owner(k, p->shard_bits) == p->shard) { key = k; break; }
        }
        if (key == 0) return -1;
        out[0] = (uint32_t)key;
        out[1] = or_bounded(or_draw(x, 1), 100) >= p->ht_lookup_pct ? 1u : 0u;
        out[2] = (uint32_t)(or_mix64(key) & (uint64_t)(p->ht_buckets - 1));
        return 3;
    }
    case OR_WL_EB: {
        uint32_t A = p->n_accesses;
        uint64_t H = p->n_words;
        if (H == 0 || (int)(2 * A) > cap) return -1;
        for (uint32_t j = 0; j < A; ++j) out[j] = (uint32_t)or_bounded(or_draw(x, j), H);
        for (uint32_t j = 0; j < A; ++j) out[A + j] = lo32(or_draw(x, A + j));
        return (int)(2 * A);
    }
    case OR_WL_KM: {
        uint32_t C = p->km_clusters, D = p->km_dims;
        if (C == 0 || (int)(1 + D) > cap) return -1;
        out[0] = (uint32_t)or_bounded(or_draw(x, 0), C);
        for (uint32_t d = 0; d < D; ++d) out[1 + d] = (uint32_t)(or_draw(x, 1 + d) >> 56);
        return (int)(1 + D);
    }
    }
    return -1;
}

uint64_t or_footprint(const or_params_t* p, uint64_t T, uint64_t K)
{
    switch (p->workload) {
    case OR_WL_RA: case OR_WL_BANK: case OR_WL_EB: return p->n_words;
    case OR_WL_HT: return (uint64_t)p->ht_buckets + 2ull * T * K;
    case OR_WL_KM: return or_km_centroids(p) + (p->km_assign ? (uint64_t)p->km_clusters * p->km_dims : 0);
    }
    return 0;
}

uint64_t or_km_centroids(const or_params_t* p)
{
    return (uint64_t)p->km_clusters * (p->km_stride ? p->km_stride : p->km_dims + 1ull);
}

/* Initial heaps: RA and EB heap[k] = k; bank 1000 per
 * account; HT empty (all heads null, node words 0); KM all records zero and,
 * with km_assign, centroid word j of the table = splitmix64(j) >> 56. */
void or_init_heap(const or_params_t* p, uint32_t* heap, uint64_t words)
{
    for (uint64_t k = 0; k < words; ++k) {
        switch (p->workload) {
        case OR_WL_RA: case OR_WL_EB: heap[k] = (uint32_t)k; break;
        case OR_WL_BANK: heap[k] = 1000u; break;
        default: heap[k] = 0u; break;
        }
    }
    if (p->workload == OR_WL_KM && p->km_assign) {
        uint64_t c0 = or_km_centroids(p), n = (uint64_t)p->km_clusters * p->km_dims;
        for (uint64_t j = 0; j < n && c0 + j < words; ++j) heap[c0 + j] = (uint32_t)(or_splitmix64(j) >> 56);
    }
}
