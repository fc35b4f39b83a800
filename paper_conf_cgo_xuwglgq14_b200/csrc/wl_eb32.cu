// wl_eb32.cu -- EbWL32 (16 < A <= 32) instantiations of the transaction
// kernels (stm_kernels.cuh); one translation unit per workload variant keeps
// the build parallel.
#include "stm_kernels.cuh"

namespace gstm {
template cudaError_t launch_wl<EbWL32>(int, const KParams&, int, cudaStream_t);
}  // namespace gstm
