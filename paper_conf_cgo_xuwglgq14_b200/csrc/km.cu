// km.cu -- the non-transactional steps of a full k-means iteration (STAMP
// kmeans):
//   assignment  every point's nearest centroid (exact integer squared
//               Euclidean distance, ties to the lowest index), one CUDA-core
//               pass before the update transactions of the launch;
//   recenter    centroid = floor(mean) of its record, records zeroed
//               (gstm_km_recenter, the end of an iteration).
// The centroid table (C x D words) follows the records in the heap and is
// read-only while the update transactions run.
#include <cstdint>
#include "kernels.cuh"

namespace gstm {

// Centroid table staged once per block in shared memory (C*D <= 1024*16
// words = 64 KiB, dynamic); every lane of a warp reads the same centroid
// word (broadcast).  Point features come from the transaction's generator
// stream (f_d = draw(1+d) >> 56), exactly as the update transaction draws
// them.  Grid-stride over tx_id = i*T + t.
__global__ void __launch_bounds__(256) km_assign_kernel(const KParams p, uint32_t* cluster)
{
    extern __shared__ uint32_t cent[];
    const uint32_t C = p.w.km_clusters, D = p.w.km_dims;
    const uint64_t c0 = uint64_t(C) * p.w.km_stride;
    bool wide = false;
    for (uint32_t j = threadIdx.x; j < C * D; j += blockDim.x) {
        cent[j] = prim::ld_relaxed(p.m.val_ptr(c0 + j));
        wide |= cent[j] >= 4096u;
    }
    // features are < 256: with every centroid word < 4096 a squared distance
    // fits 32 bits (16 * 4096^2 = 2^28); otherwise the exact 128-bit loop
    wide = __syncthreads_or(wide);
    const uint64_t n = p.T * p.K;
    for (uint64_t id = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; id < n; id += uint64_t(gridDim.x) * blockDim.x) {
        const uint64_t t = id % p.T, i = id / p.T;
        const uint64_t x = gen::tx_key(p.seed, t, i);
        int32_t f[KmWL::MAXD];
#pragma unroll
        for (int d = 0; d < KmWL::MAXD; ++d) f[d] = d < static_cast<int>(D) ? static_cast<int32_t>(gen::draw(x, 1 + d) >> 56) : 0;
        uint32_t best = 0;
        if (!wide) {
            uint32_t best_d = 0xffffffffu;
            for (uint32_t c = 0; c < C; ++c) {
                const uint32_t* cc = cent + c * D;
                uint32_t dist = 0;
#pragma unroll
                for (int d = 0; d < KmWL::MAXD; ++d)
                    if (d < static_cast<int>(D)) {
                        const int32_t e = f[d] - static_cast<int32_t>(cc[d]);
                        dist += static_cast<uint32_t>(e * e);
                    }
                if (dist < best_d) { best_d = dist; best = c; }    // strict: ties keep the lowest c
            }
        } else {
            // any uint32 centroid word: |f - c| < 2^32, its square fits 64
            // bits unsigned, and 16 squares fit 128 bits -- exact, no wrap
            unsigned __int128 best_d = ~static_cast<unsigned __int128>(0);
            for (uint32_t c = 0; c < C; ++c) {
                const uint32_t* cc = cent + c * D;
                unsigned __int128 dist = 0;
                for (uint32_t d = 0; d < D; ++d) {
                    const uint32_t a = static_cast<uint32_t>(f[d]), b = cc[d];
                    const unsigned long long e = a > b ? static_cast<unsigned long long>(a - b) : static_cast<unsigned long long>(b - a);
                    dist += static_cast<unsigned __int128>(e * e);
                }
                if (dist < best_d) { best_d = dist; best = c; }
            }
        }
        cluster[id] = best;
    }
}

// centroid word j = splitmix64(j) >> 56
__global__ void km_init_centroids_kernel(Meta m, uint64_t c0, uint64_t n)
{
    for (uint64_t j = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; j < n; j += uint64_t(gridDim.x) * blockDim.x)
        *m.val_ptr(c0 + j) = static_cast<uint32_t>(gen::mix64(j + gen::kGamma) >> 56);
}

// one thread per cluster record
__global__ void km_recenter_kernel(Meta m, uint32_t C, uint32_t D, uint32_t stride)
{
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= C) return;
    const uint64_t rec = uint64_t(c) * stride, c0 = uint64_t(C) * stride + uint64_t(c) * D;
    const uint32_t cnt = *m.val_ptr(rec);
    for (uint32_t d = 0; d < D; ++d) {
        if (cnt) *m.val_ptr(c0 + d) = *m.val_ptr(rec + 1 + d) / cnt;
        *m.val_ptr(rec + 1 + d) = 0u;
    }
    *m.val_ptr(rec) = 0u;
}

cudaError_t launch_km_assign(const KParams& kp, uint32_t* cluster, cudaStream_t s)
{
    const size_t smem = size_t(kp.w.km_clusters) * kp.w.km_dims * 4;
    int sms = 148, dev = 0;
    cudaGetDevice(&dev);
    static bool attr[64];          // the attribute is set once per device
    if (dev < 0 || dev >= 64 || !attr[dev]) {
        cudaError_t e = cudaFuncSetAttribute(km_assign_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
        if (e != cudaSuccess) return e;
        if (dev >= 0 && dev < 64) attr[dev] = true;
    }
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t n = kp.T * kp.K;
    uint64_t grid = std::min<uint64_t>((n + 255) / 256, uint64_t(sms) * 3);   // 3 blocks of 64 KiB per SM
    if (grid == 0) return cudaSuccess;
    km_assign_kernel<<<static_cast<unsigned>(grid), 256, smem, s>>>(kp, cluster);
    return cudaGetLastError();
}

cudaError_t launch_km_init_centroids(const Meta& m, uint64_t c0, uint64_t n, cudaStream_t s)
{
    if (!n) return cudaSuccess;
    km_init_centroids_kernel<<<static_cast<unsigned>(std::min<uint64_t>((n + 255) / 256, 1024)), 256, 0, s>>>(m, c0, n);
    return cudaGetLastError();
}

cudaError_t launch_km_recenter(const Meta& m, uint32_t C, uint32_t D, uint32_t stride, cudaStream_t s)
{
    if (!C) return cudaSuccess;
    km_recenter_kernel<<<(C + 255) / 256, 256, 0, s>>>(m, C, D, stride);
    return cudaGetLastError();
}

}  // namespace gstm
