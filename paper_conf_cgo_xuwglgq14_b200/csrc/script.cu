// script.cu -- scripted interleavings of several transactions on ONE device
// thread, through the same per-lane Tx code the workload kernels use.  Used
// for step-level parity of TXBegin / TXRead / TXWrite / TXCommit against the
// CPU model of Algorithm 3 (tests/test_gpu_parity.py).  Output format per op
// (4 words) matches DESIGN.md §5.3:
//   BEGIN  [snapshot, 0, 0, 0]
//   READ   [value, isOpaque, snapshot, postvalidation ran]
//   WRITE  [0, 0, 0, 0]
//   COMMIT [ok, cause, stamp, vbv runs]
//   READ2  [value(word), value(value field), snapshot, isOpaque | PostValidation ran << 1]
#include <cstdint>
#include "kernels.cuh"

namespace gstm {

constexpr int kMaxScriptTx = 8;

template <class ScriptTx>
__global__ void script_kernel(const Meta m, int mode, int prelock, const uint32_t* ops, int n_ops, uint32_t* out,
                              int n_tx)
{
    // shared-memory logs: transaction s takes column s of one [word][32] region
    __shared__ uint32_t region[ScriptTx::kSmem ? 32 * ScriptTx::kSmemWords : 1];
    if (threadIdx.x || blockIdx.x) return;
    ScriptTx tx[kMaxScriptTx];
    if constexpr (ScriptTx::kSmem)
        for (int s = 0; s < kMaxScriptTx; ++s) tx[s].bind_smem(region, s);
    for (int k = 0; k < n_ops; ++k) {
        const uint32_t op = ops[4 * k], s = ops[4 * k + 1], a = ops[4 * k + 2], v = ops[4 * k + 3];
        uint32_t o[4] = {0, 0, 0, 0};
        if (static_cast<int>(s) < n_tx) {
            ScriptTx& x = tx[s];
            switch (op) {
            case 0: {  // BEGIN
                const uint32_t snap = static_cast<uint32_t>(prim::ld_acquire64(m.clock));   // l.4-5
                x.reset_stats();
                x.begin(snap);
                o[0] = snap;
                break;
            }
            case 1: {  // READ
                x.n_postval = 0;
                o[0] = x.read(m, a, mode);
                o[1] = x.opaque ? 1u : 0u;
                o[2] = x.snapshot;
                o[3] = x.n_postval ? 1u : 0u;
                break;
            }
            case 2:  // WRITE
                x.write(m, a, v);
                break;
            case 4: {  // READ2: batched read of words a and v (read_batch, reading Q35)
                x.n_postval = 0;
                const uint32_t aa[2] = {a, v};
                uint32_t vv[2] = {0u, 0u};
                x.template read_batch<2>(m, aa, vv, 2, mode);
                o[0] = vv[0];
                o[1] = vv[1];
                o[2] = x.snapshot;
                o[3] = (x.opaque ? 1u : 0u) | (x.n_postval ? 2u : 0u);
                break;
            }
            case 3: {  // COMMIT
                x.n_vbv = 0;
                if (!x.opaque) { o[1] = C_OPACITY; break; }
                if (x.read_only()) { o[0] = 1; o[1] = C_READONLY; break; }
                int r = C_LOCK;
                for (int attempt = 0; attempt < 1000 && r == C_LOCK; ++attempt) r = x.commit_acquire(m, mode, prelock != 0);
                if (r == C_OK) {
                    x.writeback(m);                                                          // l.79-82
                    const uint32_t stamp = static_cast<uint32_t>(clock_fetch_add(m.clock, 1u)) + 1u;   // l.83
                    x.release_and_update(m, stamp);                                          // l.84
                    o[0] = 1; o[1] = C_OK; o[2] = stamp;
                } else {
                    o[1] = static_cast<uint32_t>(r);
                }
                o[3] = x.n_vbv;
                break;
            }
            default: o[0] = 0xffffffffu; break;
            }
        }
        for (int j = 0; j < 4; ++j) out[4 * k + j] = o[j];
    }
}

// lock-log parity kernel: insert entries into a register-resident (variant 0)
// or local-memory (variant 1) sorted lock log, their encounter-order
// counterparts (variants 2, 3: STM-HV-Backoff / unsorted ablation), or the
// order-preserving hashed log of P:115 (variants 4, 5: capacity 16 / 256),
// or the shared-memory log of P:117 (variant 6: capacity 64), and dump it.
template <int LCAP, bool SORTED, bool LOCAL = false, bool HLOG = false, bool SMEM = false>
__global__ void lock_log_kernel(const uint32_t* e, int n, uint32_t* out, int* out_n)
{
    using TX = Tx<1, 1, LCAP, LOCAL, SORTED, false, HLOG, SMEM>;
    __shared__ uint32_t region[SMEM ? 32 * TX::kSmemWords : 1];
    if (threadIdx.x || blockIdx.x) return;
    TX tx;
    if constexpr (SMEM) tx.bind_smem(region, 0);
    tx.begin(0);
    tx.set_id_bits(20);                   // the test's lock ids are < 2^20
    for (int k = 0; k < n; ++k) tx.insert_lock(e[k]);
    tx.compact();
    if constexpr (TX::kUnroll) {
#pragma unroll
        for (int k = 0; k < LCAP; ++k)
            if (k < tx.nl) out[k] = tx.l_ent[k];
    } else {
        for (int k = 0; k < tx.nl; ++k) out[k] = tx.l_ent[k];
    }
    *out_n = tx.overflow ? -1 : tx.nl;
}

// policy 0: local-memory logs (Tx<64,64,128>); 1: register-resident logs,
// the fully unrolled code the bank kernel runs (Tx<8,8,16>); 2: shared-memory
// logs, [entry][lane] (Tx<16,16,32, SMEM>)
cudaError_t launch_script(const Meta& m, int mode, int prelock, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx,
                          int policy, cudaStream_t s)
{
    if (n_tx > kMaxScriptTx || policy < 0 || policy > 2) return cudaErrorInvalidValue;
    if (m.vshift) {
        if (policy == 1) script_kernel<TxPair<8, 8, 16>><<<1, 32, 0, s>>>(m, mode, prelock, ops, n_ops, out, n_tx);
        else if (policy == 2)
            script_kernel<TxPair<16, 16, 32, false, true, false, false, true>><<<1, 32, 0, s>>>(m, mode, prelock, ops,
                                                                                              n_ops, out, n_tx);
        else script_kernel<TxPair<64, 64, 128>><<<1, 32, 0, s>>>(m, mode, prelock, ops, n_ops, out, n_tx);
    } else {
        if (policy == 1) script_kernel<Tx<8, 8, 16>><<<1, 32, 0, s>>>(m, mode, prelock, ops, n_ops, out, n_tx);
        else if (policy == 2)
            script_kernel<Tx<16, 16, 32, false, true, false, false, true>><<<1, 32, 0, s>>>(m, mode, prelock, ops, n_ops,
                                                                                          out, n_tx);
        else script_kernel<Tx<64, 64, 128>><<<1, 32, 0, s>>>(m, mode, prelock, ops, n_ops, out, n_tx);
    }
    return cudaGetLastError();
}

cudaError_t launch_lock_log(const uint32_t* entries, int n, uint32_t* out, int* out_n, int variant, cudaStream_t s)
{
    switch (variant) {
    case 0: lock_log_kernel<16, true><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    case 1: lock_log_kernel<256, true><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    case 2: lock_log_kernel<16, false><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    case 3: lock_log_kernel<256, false><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    // the order-preserving hashed log of P:115 (local memory)
    case 4: lock_log_kernel<16, true, true, true><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    case 5: lock_log_kernel<256, true, true, true><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    // shared-memory logs, [entry][lane]
    default: lock_log_kernel<64, true, false, false, true><<<1, 32, 0, s>>>(entries, n, out, out_n); break;
    }
    return cudaGetLastError();
}

}  // namespace gstm
