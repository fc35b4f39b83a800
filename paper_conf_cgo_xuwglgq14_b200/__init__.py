"""B200-native GPU-STM (Xu et al., CGO 2014): per-thread transactions with
hierarchical validation and encounter-time lock sorting, as sm_100a CUDA
behind the C ABI in include/gstm.h.  ``gstm`` is the ctypes binding."""
from .gstm import (Gstm, GstmError, gstm_create, gstm_default_params, gstm_destroy, gstm_launch,  # noqa: F401
                   gstm_lock_log, gstm_set_mode, gstm_set_params, gstm_stats, gstm_ubench, lib)
