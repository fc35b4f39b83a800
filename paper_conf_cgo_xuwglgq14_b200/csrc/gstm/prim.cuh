// prim.cuh -- scoped memory operations and warp helpers for sm_100a.
//
// The paper's metadata lived in Fermi global memory accessed through
// `volatile` with __threadfence() fences.  On sm_70+ the L1 is
// not coherent for weak loads, so every access to shared STM data or metadata
// here is a *strong* gpu-scope operation (SASS LDG/STG/ATOMG .STRONG.GPU,
// which are served by the L2, the device's coherence point), and the paper's
// fences (A3.l5, l12, l26, l79, l82) become PTX acquire/release operations or
// `fence.acq_rel.gpu` (DESIGN.md §6.2 gives the ordering argument).
//
// SASS each helper compiles to (nvcc 12.9, sm_100a; checked with cuobjdump):
//   ld_relaxed        LDG.E.STRONG.GPU
//   ld_acquire        LDG.E.STRONG.GPU ; CCTL.IVALL
//   st_relaxed        STG.E.STRONG.GPU
//   fence_acq_rel     MEMBAR.ALL.GPU ; ERRBAR ; CGAERRBAR ; CCTL.IVALL
//   fence_acquire     CCTL.IVALL                (waits for the prior loads)
//   fence_release     MEMBAR.ALL.GPU ; ERRBAR ; CGAERRBAR
//   atom_or_acquire   ATOMG.E.OR.STRONG.GPU ; CCTL.IVALL
//   atom_add_acquire  ATOMG.E.ADD.64.STRONG.GPU ; CCTL.IVALL
//   atom_add_acq_rel  MEMBAR.ALL.GPU ; ATOMG.E.ADD.64.STRONG.GPU ; CCTL.IVALL
#pragma once
#include <cstdint>

// GSTM_STRICT_FENCES=1 adds the fences a purely formal reading of the PTX
// memory model asks for on top of the ones the hardware needs (DESIGN.md
// §6.2): a release fence after lock acquisition (A3.l79), an acq_rel clock
// increment and a release fence before the lock-release stores.  Default 0.
#ifndef GSTM_STRICT_FENCES
#define GSTM_STRICT_FENCES 0
#endif

// nanoseconds a reader sleeps between re-reads of a locked word (A3.l27-29)
#ifndef GSTM_SPIN_NS
#define GSTM_SPIN_NS 32
#endif
// measurement only (NOT a supported build): acquire operations become relaxed
// and fence.acquire disappears, to price the CCTL.IVALL they compile to
#ifndef GSTM_EXPERIMENT_NO_ACQ
#define GSTM_EXPERIMENT_NO_ACQ 0
#endif
#if GSTM_EXPERIMENT_NO_ACQ
#define GSTM_ACQ "relaxed"
#else
#define GSTM_ACQ "acquire"
#endif

namespace gstm {
namespace prim {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p)
{
    uint32_t v;
    asm volatile("ld." GSTM_ACQ ".gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ unsigned long long ld_acquire64(const unsigned long long* p)
{
    unsigned long long v;
    asm volatile("ld." GSTM_ACQ ".gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long* p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed(uint32_t* p, uint32_t v)
{
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// 16-byte vector store of 4 consecutive words (p 16-byte aligned): one L2
// request for a run of the write-set (the k-means record write-back)
__device__ __forceinline__ void st_relaxed_v4(uint32_t* p, uint32_t a, uint32_t b, uint32_t c, uint32_t d)
{
    asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(a), "r"(b), "r"(c), "r"(d)
                 : "memory");
}

__device__ __forceinline__ void st_relaxed64(unsigned long long* p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel()
{
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

// Acquire fence: with the strong reads before it, forms an acquire pattern
// (orders those reads before every later access).  SASS: CCTL.IVALL only --
// it waits for the prior loads, no MEMBAR.  This is what A3.l12/l26 need
// (value loads before lock-word loads).
__device__ __forceinline__ void fence_acquire()
{
#if GSTM_EXPERIMENT_NO_ACQ
    asm volatile("" ::: "memory");
#else
    asm volatile("fence.acquire.gpu;" ::: "memory");
#endif
}

// Release fence: orders every earlier access before the strong writes after
// it (SASS: MEMBAR.ALL.GPU).  A3.l82 (write-back before the clock / lock
// release).
__device__ __forceinline__ void fence_release()
{
    asm volatile("fence.release.gpu;" ::: "memory");
}

__device__ __forceinline__ unsigned long long atom_add_acquire64(unsigned long long* p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom." GSTM_ACQ ".gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t atom_or_acquire(uint32_t* p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom." GSTM_ACQ ".gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

// 8-byte accesses for the paired layout (value | version lock in one
// naturally aligned u64: single-copy atomic, one L2 request)
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long atom_or_acquire_u64(unsigned long long* p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom." GSTM_ACQ ".gpu.global.or.b64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ unsigned long long atom_or_relaxed_u64(unsigned long long* p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom.relaxed.gpu.global.or.b64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t atom_or_relaxed(uint32_t* p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom.relaxed.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t atom_cas_acquire(uint32_t* p, uint32_t cmp, uint32_t v)
{
    uint32_t old;
    asm volatile("atom." GSTM_ACQ ".gpu.global.cas.b32 %0, [%1], %2, %3;"
                 : "=r"(old) : "l"(p), "r"(cmp), "r"(v) : "memory");
    return old;
}

__device__ __forceinline__ unsigned long long atom_cas_acquire64(unsigned long long* p, unsigned long long cmp,
                                                                 unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom." GSTM_ACQ ".gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ unsigned long long atom_add_acq_rel64(unsigned long long* p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ unsigned long long atom_add_relaxed64(unsigned long long* p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t lane_id()
{
    uint32_t l;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}

__device__ __forceinline__ uint32_t lanemask_lt()
{
    uint32_t m;
    asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__device__ __forceinline__ void nanosleep(uint32_t ns)
{
    if (ns) __nanosleep(ns);
}

}  // namespace prim
}  // namespace gstm
