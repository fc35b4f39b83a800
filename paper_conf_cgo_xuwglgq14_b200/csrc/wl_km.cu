// wl_km.cu -- KmWL instantiations of the transaction kernels
// (stm_kernels.cuh); one translation unit per workload keeps the build parallel.
#include "stm_kernels.cuh"

namespace gstm {
GSTM_INSTANTIATE_WL(KmWL)
}  // namespace gstm
