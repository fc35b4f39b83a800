// gen.cuh -- device-side input generator.
//
// Counter-based SplitMix64 (Steele, Lea & Flood 2014): the draw for
// (seed, thread t, transaction index i, k) is a pure function, so a
// transaction that aborts regenerates exactly the same accesses when it is
// re-executed (nothing to checkpoint, cf. "register checkpoint").
// This is an independent implementation of the recipe; the CPU oracle has
// its own (oracle/gen.c) and tests/test_gpu_parity.py checks the two agree.
#pragma once
#include <cstdint>

namespace gstm {
namespace gen {

constexpr uint64_t kGamma = 0x9E3779B97F4A7C15ull;
constexpr uint64_t kTxMul = 0xC2B2AE3D27D4EB4Full;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// k-th output of the SplitMix64 stream whose state is x
__host__ __device__ __forceinline__ uint64_t draw(uint64_t x, uint64_t k)
{
    return mix64(x + (k + 1) * kGamma);
}

__host__ __device__ __forceinline__ uint64_t tx_key(uint64_t seed, uint64_t t, uint64_t i)
{
    return mix64((seed ^ (t * kGamma) ^ (i * kTxMul)) + kGamma);
}

// floor(r * n / 2^64)
__device__ __forceinline__ uint64_t bounded(uint64_t r, uint64_t n) { return __umul64hi(r, n); }

}  // namespace gen
}  // namespace gstm
