// kernels.cu -- the non-template kernels (launch prologue/epilogue, heap
// initialisation, paired-layout packing) and the per-workload dispatch; the
// transaction kernels are in stm_kernels.cuh, instantiated in wl_*.cu.
#include <algorithm>
#include <cstdint>
#include "kernels.cuh"

namespace gstm {

__device__ __forceinline__ unsigned long long globaltimer_ns()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

template <class WL> cudaError_t launch_wl(int kmode, const KParams& kp, int block, cudaStream_t s);
template <class WL> cudaError_t launch_descr_wl(const KParams& kp, uint32_t* out, int wpt, cudaStream_t s);
template <class WL> bool check_wl(const WlParams& w, uint64_t* fp, int* dw);

__global__ void prepare_kernel(unsigned long long* meta, const unsigned long long* clock, uint64_t timeout_ns)
{
    const unsigned long long now = globaltimer_ns();
    meta[M_CLOCK_BEGIN] = *clock;
    meta[M_DEADLINE] = now + timeout_ns;
    meta[M_T_START] = now;
    meta[M_WORK] = 0;
    meta[M_SEQ] = 2ull * *clock;                    // STM-VBV sequence lock (tx_vbv.cuh)
    meta[M_SERIAL] = 0;                             // contention manager: no ticket issued, none served
    meta[M_SERIAL_EST] = 0;                         // ... no owner time measured yet
    for (int k = 0; k < S_NSTATS; ++k) meta[M_STATS + k] = 0;
    *reinterpret_cast<uint32_t*>(meta + M_ERR) = 0;
    *reinterpret_cast<uint32_t*>(meta + M_CGL_LOCK) = 0;
}

// end of a launch: record the clock and fold this launch's counters into the
// running totals (so callers can enqueue many launches without syncing)
__global__ void finish_kernel(unsigned long long* meta, const unsigned long long* clock)
{
    meta[M_CLOCK_END] = *clock;
    for (int k = 0; k < S_NSTATS; ++k) meta[M_TOTALS + k] += meta[M_STATS + k];
    meta[M_T_LAUNCHES] += 1;
    meta[M_T_NS] += globaltimer_ns() - meta[M_T_START];
    meta[M_T_ERR] |= meta[M_ERR] & 0xffffffffull;
}

// workload-defined initial heaps
__global__ void init_heap_kernel(int workload, uint32_t* heap, uint64_t words, int vshift)
{
    for (uint64_t k = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k < words;
         k += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
        uint32_t v = 0;
        if (workload == WL_RA || workload == WL_EB) v = static_cast<uint32_t>(k);
        else if (workload == WL_BANK) v = 1000u;
        heap[k << vshift] = v;
    }
}

// paired layout <-> plain word array (values only; lock halves untouched)
__global__ void pack_kernel(uint32_t* plain, uint32_t* pairs, uint64_t words, int to_pairs)
{
    for (uint64_t k = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k < words;
         k += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
        if (to_pairs) pairs[2 * k] = plain[k];
        else plain[k] = pairs[2 * k];
    }
}

// lock halves of the paired layout: zero them, or copy them out
__global__ void lock_halves_kernel(uint32_t* pairs, uint64_t words, uint32_t* out)
{
    for (uint64_t k = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k < words;
         k += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
        if (out) out[k] = pairs[2 * k + 1];
        else pairs[2 * k + 1] = 0u;
    }
}

static unsigned grid_for(uint64_t n)
{
    uint64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 32) blocks = 148 * 32;
    return static_cast<unsigned>(blocks ? blocks : 1);
}

cudaError_t launch_pack(uint32_t* plain, uint32_t* pairs, uint64_t words, int to_pairs, cudaStream_t s)
{
    if (!words) return cudaSuccess;
    pack_kernel<<<grid_for(words), 256, 0, s>>>(plain, pairs, words, to_pairs);
    return cudaGetLastError();
}

cudaError_t launch_lock_halves(uint32_t* pairs, uint64_t words, uint32_t* out, cudaStream_t s)
{
    if (!words) return cudaSuccess;
    lock_halves_kernel<<<grid_for(words), 256, 0, s>>>(pairs, words, out);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// host launchers
// ---------------------------------------------------------------------------
cudaError_t launch_prepare(unsigned long long* meta, const unsigned long long* clock, uint64_t timeout_ns, cudaStream_t s)
{
    prepare_kernel<<<1, 1, 0, s>>>(meta, clock, timeout_ns);
    return cudaGetLastError();
}

cudaError_t launch_finish(unsigned long long* meta, const unsigned long long* clock, cudaStream_t s)
{
    finish_kernel<<<1, 1, 0, s>>>(meta, clock);
    return cudaGetLastError();
}

cudaError_t launch_init_heap(int workload, uint32_t* heap, uint64_t words, int vshift, cudaStream_t s)
{
    if (!words) return cudaSuccess;
    init_heap_kernel<<<grid_for(words), 256, 0, s>>>(workload, heap, words, vshift);
    return cudaGetLastError();
}


cudaError_t launch_tx(int workload, int kmode, const KParams& kp, int block, cudaStream_t s)
{
    switch (workload) {
    case WL_RA: return kp.w.ra_kind == 1 ? launch_wl<RaIncWL>(kmode, kp, block, s) : launch_wl<RaWL>(kmode, kp, block, s);
    case WL_BANK: return launch_wl<BankWL>(kmode, kp, block, s);
    case WL_HT: return launch_wl<HtWL>(kmode, kp, block, s);
    case WL_EB:   // the smallest compiled access count that fits (workloads.cuh EbWLT)
        return kp.w.n_accesses <= 16 ? launch_wl<EbWL16>(kmode, kp, block, s)
             : kp.w.n_accesses <= 32 ? launch_wl<EbWL32>(kmode, kp, block, s)
                                     : launch_wl<EbWL>(kmode, kp, block, s);
    case WL_KM: return launch_wl<KmWL>(kmode, kp, block, s);
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_descr(int workload, const KParams& kp, uint32_t* out, int wpt, cudaStream_t s)
{
    switch (workload) {
    case WL_RA: return kp.w.ra_kind == 1 ? launch_descr_wl<RaIncWL>(kp, out, wpt, s) : launch_descr_wl<RaWL>(kp, out, wpt, s);
    case WL_BANK: return launch_descr_wl<BankWL>(kp, out, wpt, s);
    case WL_HT: return launch_descr_wl<HtWL>(kp, out, wpt, s);
    case WL_EB: return launch_descr_wl<EbWL>(kp, out, wpt, s);
    case WL_KM: return launch_descr_wl<KmWL>(kp, out, wpt, s);
    }
    return cudaErrorInvalidValue;
}

bool workload_check(int workload, const WlParams& w, uint64_t* fp, int* dw)
{
    switch (workload) {
    case WL_RA: return w.ra_kind == 1 ? check_wl<RaIncWL>(w, fp, dw) : check_wl<RaWL>(w, fp, dw);
    case WL_BANK: return check_wl<BankWL>(w, fp, dw);
    case WL_HT: return check_wl<HtWL>(w, fp, dw);
    case WL_EB: return check_wl<EbWL>(w, fp, dw);
    case WL_KM: return check_wl<KmWL>(w, fp, dw);
    }
    return false;
}

}  // namespace gstm
