// wl_eb16.cu -- EbWL16 (A <= 16, shared-memory logs) instantiations of the
// transaction kernels (stm_kernels.cuh); one translation unit per workload
// variant keeps the build parallel.
#include "stm_kernels.cuh"

namespace gstm {
template cudaError_t launch_wl<EbWL16>(int, const KParams&, int, cudaStream_t);
}  // namespace gstm
