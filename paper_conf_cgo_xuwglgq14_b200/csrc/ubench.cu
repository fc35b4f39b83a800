// ubench.cu -- roofline microbenchmarks for the STM hot path (SURVEY §2.3
// K10, §8d).  The hot path is bound by L2 atomics / random L2 accesses, not
// by streaming HBM bandwidth or tensor cores, so its roofline denominators
// are measured here on the box with the same PTX operations the STM uses:
//   0  random atom.or.b32 (returning)  over a table of S bytes   (lock acquire)
//   1  same-address atom.add.u64 (returning), every thread        (global clock)
//   2  random ld.relaxed.gpu.u32 over S bytes                     (TXRead loads)
//   3  random st.relaxed.gpu.u32 over S bytes                     (write-back / release)
//   4  dependent chain of random atom.or (one per thread in flight): latency
//   5  same-address atom.add.u64 issued by one lane per warp      (aggregated clock)
//   6-8  random atom.or.b64 / ld.u64 / st.u64 over S bytes        (paired layout)
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cuda_runtime.h>
#include "kernels.cuh"

namespace gstm {

__device__ __forceinline__ uint32_t ub_hash(uint64_t a, uint64_t b)
{
    return static_cast<uint32_t>(gen::mix64(a * 0x9E3779B97F4A7C15ull + b) >> 32);
}

__global__ void ubench_kernel(int kind, uint32_t* table, uint32_t mask, unsigned long long* hot, uint32_t n_per_thread,
                              uint32_t* sink)
{
    const uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    switch (kind) {
    case 0:
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k) {
            uint32_t old;
            uint32_t* p = table + (ub_hash(t, k) & mask);
            asm volatile("atom.relaxed.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(0u) : "memory");
            acc += old;
        }
        break;
    case 1:
        for (uint32_t k = 0; k < n_per_thread; ++k) acc += static_cast<uint32_t>(prim::atom_add_relaxed64(hot, 1ull));
        break;
    case 2:
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k) acc += prim::ld_relaxed(table + (ub_hash(t, k) & mask));
        break;
    case 3:
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k) prim::st_relaxed(table + (ub_hash(t, k) & mask), k);
        break;
    case 4: {
        uint32_t idx = ub_hash(t, 0) & mask;
        for (uint32_t k = 0; k < n_per_thread; ++k) {
            uint32_t old;
            asm volatile("atom.relaxed.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(table + idx), "r"(0u) : "memory");
            idx = (idx + 1 + (old & 1u) + ub_hash(t, k + 1)) & mask;
            acc += old;
        }
        break;
    }
    case 5:
        if (prim::lane_id() == 0)
            for (uint32_t k = 0; k < n_per_thread; ++k) acc += static_cast<uint32_t>(prim::atom_add_relaxed64(hot, 32ull));
        break;
    // 8-byte versions (the paired layout's value|lock accesses)
    case 6: {
        unsigned long long* t64 = reinterpret_cast<unsigned long long*>(table);
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k)
            acc += static_cast<uint32_t>(prim::atom_or_relaxed_u64(t64 + ((ub_hash(t, k) & mask) >> 1), 0ull));
        break;
    }
    case 7: {
        unsigned long long* t64 = reinterpret_cast<unsigned long long*>(table);
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k)
            acc += static_cast<uint32_t>(prim::ld_relaxed_u64(t64 + ((ub_hash(t, k) & mask) >> 1)));
        break;
    }
    case 8: {
        unsigned long long* t64 = reinterpret_cast<unsigned long long*>(table);
#pragma unroll 4
        for (uint32_t k = 0; k < n_per_thread; ++k) prim::st_relaxed_u64(t64 + ((ub_hash(t, k) & mask) >> 1), k);
        break;
    }
    }
    if (acc == 0xdeadbeefu) sink[0] = acc;
}

// Probe with the commit path's traffic mix: per warp round, 2 random
// atom.or per lane on the lock table, 2 random loads per lane on the heap,
// then one warp-aggregated increment of the candidate clock word.
__global__ void clock_mix_probe_kernel(unsigned long long* word, uint32_t* locks, uint32_t lmask, uint32_t* heap,
                                       uint32_t hmask, uint32_t n, uint32_t* sink)
{
    const uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (uint32_t k = 0; k < n; ++k) {
        const uint32_t h1 = ub_hash(t, 2 * k), h2 = ub_hash(t, 2 * k + 1);
        acc += prim::ld_relaxed(heap + ((h1 + acc) & hmask)) + prim::ld_relaxed(heap + ((h2 + acc) & hmask));
        acc += prim::atom_or_relaxed(locks + ((h1 + acc) & lmask), 0u);
        acc += prim::atom_or_relaxed(locks + ((h2 + acc) & lmask), 0u);
        __syncwarp();
        unsigned long long b = 0;
        if (prim::lane_id() == 0) b = prim::atom_add_acquire64(word, 8ull + (acc & 0x40000000u));
        acc += static_cast<uint32_t>(__shfl_sync(0xffffffffu, b, 0)) & 1u;
    }
    if (acc == 0xdeadbeefu) sink[0] = 1;
}

// ---------------------------------------------------------------------------
// Op-mix roof: every thread runs conflict-free
// "transactions" made of exactly the memory operations Algorithm 3 issues for
// one transaction of a workload, in the same dependency order, with no STM
// logic around them (no logs, no validation branches, no retries).  A
// program is a list of phases; the ops of one phase are independent (issued
// back to back), and every phase's addresses depend on the previous phase's
// results, so each phase costs one memory round trip -- as in the kernel.
// Word slot j of a transaction is the same random word in every phase (the
// value load, the lock load, the lock atomic and the store of word j hit the
// same lines the kernel would).  Up to kMixProgs programs are mixed per
// transaction by weight (e.g. update vs read-only transactions in the
// proportions the measured run committed).
// ---------------------------------------------------------------------------
constexpr int kMixProgs = 4, kMixPhases = 160;
struct MixProg {
    uint32_t n_prog;
    uint32_t records, stride;            // records > 0: slot j of thread t = word (t mod records)*stride + j
    uint32_t cum[kMixProgs];             // cumulative weights out of 65536
    uint32_t n_ph[kMixProgs];
    uint32_t clk[kMixProgs];             // index of the program's CLOCK phase (n_ph: none; at most one)
    uint32_t ph[kMixProgs][kMixPhases];  // kind | count << 8 | slot0 << 16
};
enum { MIX_LD_V = 1, MIX_LD_L = 2, MIX_ATOM_L = 3, MIX_ST_V = 4, MIX_ST_L = 5, MIX_CLOCK = 6, MIX_FENCE_REL = 7,
       MIX_ACQ = 8, MIX_KINDS };

template <bool PAIR>
__device__ __forceinline__ uint32_t mix_phases(const MixProg& P, const Meta& m, uint64_t words, uint64_t t, uint64_t x,
                                               uint32_t prog, uint32_t from, uint32_t to, uint32_t dep)
{
    for (uint32_t ph = from; ph < to; ++ph) {
        const uint32_t code = P.ph[prog][ph];
        const uint32_t kind = code & 0xffu, cnt = (code >> 8) & 0xffu, s0 = code >> 16;
        uint32_t nd = 0;
        if (kind == MIX_FENCE_REL) {
            prim::fence_release();
        } else if (kind == MIX_ACQ) {
            prim::fence_acquire();
        } else {
#pragma unroll 8
            for (uint32_t j = 0; j < cnt; ++j) {
                const uint32_t w = P.records
                    ? static_cast<uint32_t>((t % P.records) * P.stride + ((s0 + j + dep) % P.stride))
                    : static_cast<uint32_t>(gen::bounded(gen::draw(x, s0 + j) ^ dep, words));
                if constexpr (PAIR) {
                    unsigned long long* pp = m.pair_ptr(w);
                    if (kind == MIX_LD_V || kind == MIX_LD_L) nd ^= static_cast<uint32_t>(prim::ld_relaxed_u64(pp));
                    else if (kind == MIX_ATOM_L) nd ^= static_cast<uint32_t>(prim::atom_or_relaxed_u64(pp, 0ull));
                    else prim::st_relaxed_u64(pp, dep);
                } else {
                    if (kind == MIX_LD_V) nd ^= prim::ld_relaxed(m.val_ptr(w));
                    else if (kind == MIX_LD_L) nd ^= prim::ld_relaxed(m.lock_ptr(m.lock_of(w)));
                    else if (kind == MIX_ATOM_L) nd ^= prim::atom_or_relaxed(m.lock_ptr(m.lock_of(w)), 0u);
                    else if (kind == MIX_ST_V) prim::st_relaxed(m.val_ptr(w), dep);
                    else prim::st_relaxed(m.lock_ptr(m.lock_of(w)), dep & ~1u);
                }
            }
        }
        // the next phase's addresses depend on this phase's results (one
        // round trip per phase); stores and fences leave dep unchanged
        dep ^= nd & 0x1u;
    }
    return dep;
}

// Warp-synchronous like the transaction kernel (stm_kernels.cuh): every
// transaction starts at a warp barrier; the phases before the clock (body,
// validation, locks, write-back) run per lane; then ONE warp-collective
// clock increment for the lanes whose program has one (warp_stamp, A3.l83);
// then the phases after it (release).  Without the barriers lanes that ran a
// shorter program drift into later transactions and split the warp into
// groups that each pay their own clock atomic.
template <bool PAIR>
__global__ void __launch_bounds__(256) ubench_mix_kernel(const MixProg P, const Meta m, uint64_t words, uint32_t n_per_thread,
                                                         uint32_t* sink)
{
    const uint64_t t = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    for (uint32_t k = 0; k < n_per_thread; ++k) {
        __syncwarp();
        const uint64_t x = gen::mix64(t * gen::kGamma + k);
        const uint32_t r = static_cast<uint32_t>(x >> 48);
        uint32_t prog = 0;
        while (prog + 1 < P.n_prog && r >= P.cum[prog]) ++prog;
        const uint32_t clk = P.clk[prog], n = P.n_ph[prog];
        uint32_t dep = mix_phases<PAIR>(P, m, words, t, x, prog, 0, clk, 0u);
        __syncwarp();
        const unsigned bm = __ballot_sync(prim::FULL, clk < n);
        if (bm) {
            const int leader = __ffs(bm) - 1;
            unsigned long long b = 0;
            if (static_cast<int>(prim::lane_id()) == leader) b = prim::atom_add_acquire64(m.clock, __popc(bm));
            b = __shfl_sync(prim::FULL, b, leader);
            dep ^= static_cast<uint32_t>(b) & 1u;
        }
        if (clk < n) dep = mix_phases<PAIR>(P, m, words, t, x, prog, clk + 1, n, dep);
        acc += dep;
    }
    if (acc == 0xdeadbeefu) sink[0] = acc;
}

int ubench_mix(const Meta& m, bool paired, uint64_t words, const uint32_t* prog, uint32_t prog_words, uint64_t n_tx,
               uint32_t threads, uint32_t block, cudaStream_t s, double* tx_per_s, double* ms_out)
{
    if (!prog || !tx_per_s || !words || words > (1ull << 32) || threads == 0 || block == 0 || block > 256 ||
        block % 32 || threads % block || prog_words < 1)
        return -1;
    MixProg P;
    memset(&P, 0, sizeof(P));
    P.n_prog = prog[0] & 0xffu;
    if (P.n_prog < 1 || P.n_prog > kMixProgs) return -1;
    uint32_t pos = 1, cum = 0;
    if (prog[0] & 0x100u) {              // record addressing: prog[1] = records, prog[2] = stride
        if (prog_words < 3 || !prog[1] || !prog[2] || uint64_t(prog[1]) * prog[2] > words) return -1;
        P.records = prog[1];
        P.stride = prog[2];
        pos = 3;
    }
    for (uint32_t q = 0; q < P.n_prog; ++q) {
        if (pos + 2 > prog_words) return -1;
        cum += prog[pos];
        P.cum[q] = cum;
        P.n_ph[q] = prog[pos + 1];
        pos += 2;
        if (P.n_ph[q] > kMixPhases || pos + P.n_ph[q] > prog_words) return -1;
        P.clk[q] = P.n_ph[q];
        for (uint32_t k = 0; k < P.n_ph[q]; ++k) {
            const uint32_t kind = prog[pos + k] & 0xffu;
            if (kind == 0 || kind >= MIX_KINDS) return -1;
            if (kind == MIX_CLOCK) {
                if (P.clk[q] != P.n_ph[q]) return -1;      // one clock increment per transaction
                P.clk[q] = k;
            }
            P.ph[q][k] = prog[pos + k];
        }
        pos += P.n_ph[q];
    }
    if (cum != 65536u) return -1;
    const uint32_t per = static_cast<uint32_t>((n_tx + threads - 1) / threads);
    uint32_t* sink = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    int rc = 0;
    if (cudaMalloc(&sink, 64) != cudaSuccess) return -2;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const unsigned grid = threads / block;
    auto run = [&]() {
        if (paired) ubench_mix_kernel<true><<<grid, block, 0, s>>>(P, m, words, per, sink);
        else ubench_mix_kernel<false><<<grid, block, 0, s>>>(P, m, words, per, sink);
    };
    run();                                            // warm-up
    cudaEventRecord(e0, s);
    run();
    cudaEventRecord(e1, s);
    if (cudaEventSynchronize(e1) != cudaSuccess || cudaGetLastError() != cudaSuccess) {
        rc = -3;
    } else {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        *tx_per_s = static_cast<double>(per) * threads / (ms * 1e-3);
        if (ms_out) *ms_out = ms;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    return rc;
}

// Returns the index of the candidate (word = base + k*stride_words) with
// the fastest probe, or -1 on error.  The L2 slice that owns g_clock is
// decided by its physical address, and on B200 the per-slice load of a
// 4 MiB table is uneven (ncu: max/avg lts requests 1.4), so the slice the
// hot clock lands on changes commit throughput by ~25%.
// The handle measures candidate lines once, with the commit path's mix of
// lock-table atomics, heap loads and clock increments, and keeps the fastest.
int clock_calibrate_mix(unsigned long long* base, int n_candidates, int stride_words, uint32_t* locks, uint32_t lmask,
                        uint32_t* heap, uint32_t hmask, cudaStream_t s)
{
    uint32_t* sink = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    int best = -1;
    float best_ms = 1e30f;
    if (cudaMalloc(&sink, 64) != cudaSuccess) return -1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    clock_mix_probe_kernel<<<148 * 8, 256, 0, s>>>(base, locks, lmask, heap, hmask, 16, sink);   // warm-up
    for (int k = 0; k < n_candidates; ++k) {
        unsigned long long* w = base + static_cast<size_t>(k) * stride_words;
        cudaEventRecord(e0, s);
        clock_mix_probe_kernel<<<148 * 8, 256, 0, s>>>(w, locks, lmask, heap, hmask, 16, sink);
        cudaEventRecord(e1, s);
        if (cudaEventSynchronize(e1) != cudaSuccess) { best = -1; goto out; }
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        if (getenv("GSTM_CALIB_VERBOSE")) fprintf(stderr, "clock candidate %d (mix): %.4f ms\n", k, ms);
        if (ms < best_ms) { best_ms = ms; best = k; }
    }
    cudaMemsetAsync(base, 0, static_cast<size_t>(n_candidates) * stride_words * 8, s);
    cudaStreamSynchronize(s);
out:
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    return best;
}

// Runs `kind` over a table of table_bytes (power of two) with `threads`
// threads doing n_ops in total.  Returns 0 and ops/s (for kind 5: clock
// increments per second, i.e. 32 per atomic), or a negative error.
int ubench(int kind, uint64_t table_bytes, uint64_t n_ops, uint32_t threads, double* ops_per_s, double* ms_out)
{
    if (kind < 0 || kind > 8 || threads == 0 || threads % 256 || table_bytes < 128 ||
        (table_bytes & (table_bytes - 1)))
        return -1;
    const uint32_t per = static_cast<uint32_t>((n_ops + threads - 1) / threads);
    uint32_t* table = nullptr;
    unsigned long long* hot = nullptr;
    uint32_t* sink = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    cudaStream_t s = nullptr;
    int rc = 0;
    if (cudaMalloc(&table, table_bytes) != cudaSuccess || cudaMalloc(&hot, 256) != cudaSuccess ||
        cudaMalloc(&sink, 256) != cudaSuccess) {
        rc = -2;
        goto out;
    }
    cudaMemset(table, 0, table_bytes);
    cudaMemset(hot, 0, 256);
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    {
        const uint32_t mask = static_cast<uint32_t>(table_bytes / 4 - 1);
        const unsigned grid = threads / 256;
        ubench_kernel<<<grid, 256, 0, s>>>(kind, table, mask, hot, per, sink);   // warm-up
        cudaEventRecord(e0, s);
        ubench_kernel<<<grid, 256, 0, s>>>(kind, table, mask, hot, per, sink);
        cudaEventRecord(e1, s);
        if (cudaEventSynchronize(e1) != cudaSuccess) { rc = -3; goto out; }
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        double total = static_cast<double>(per) * threads;
        if (kind == 5) total = static_cast<double>(per) * (threads / 32) * 32.0;
        *ops_per_s = total / (ms * 1e-3);
        if (ms_out) *ms_out = ms;
    }
out:
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    if (s) cudaStreamDestroy(s);
    cudaFree(table);
    cudaFree(hot);
    cudaFree(sink);
    return rc;
}

}  // namespace gstm
