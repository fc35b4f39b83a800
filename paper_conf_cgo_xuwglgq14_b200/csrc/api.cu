// api.cu -- the C ABI (include/gstm.h) over the kernels in kernels.cu.
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <cuda_runtime.h>
#include "../../include/gstm.h"
#include "kernels.cuh"

using namespace gstm;

static thread_local char g_err[512] = "";

static void set_error(const char* fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

#define CUDA_TRY(expr)                                                                    \
    do {                                                                                  \
        cudaError_t e__ = (expr);                                                         \
        if (e__ != cudaSuccess) {                                                         \
            set_error("%s: %s (%s:%d)", #expr, cudaGetErrorString(e__), __FILE__, __LINE__); \
            return GSTM_ECUDA;                                                            \
        }                                                                                 \
    } while (0)

static constexpr size_t kMetaBytes = 1024 * 1024; // metadata block (M_WORDS used) + g_clock candidates
// candidate lines for g_clock after M_WORDS ... (only ~1 line in 32 is fast: on
// one B200, 2 of 64 probed lines ran the bank kernel at 9.6 G tx/s and the
// other 62 at 7.0-7.5; 256 candidates miss them all with
// probability ~0.03%)
static constexpr int kClockCandidates = 256;
static constexpr int kClockStride = 288;           // ... 2304 B apart (crosses 256 B and 2 KiB address bits)
static_assert(gstm::M_SEQ >= gstm::M_WORDS + kClockCandidates * kClockStride + 16 && gstm::M_SERIAL * 8 + 128 <= kMetaBytes,
              "STM-VBV sequence lock must sit on its own line after the clock candidates");

struct gstm_handle {
    char* block = nullptr;          // the single device allocation
    bool paired = false;            // GSTM_CREATE_PAIRED layout
    uint32_t* scratch = nullptr;    // paired layout: plain word buffer for copies
    uint64_t scratch_words = 0;
    unsigned long long* clock = nullptr;   // g_clock, on its own line inside the metadata block
    int clock_slot = -1;
    uint32_t* own_heap = nullptr;
    uint32_t* heap = nullptr;
    uint64_t heap_words = 0, own_words = 0;
    uint32_t* locks = nullptr;
    uint32_t bits = 0;
    unsigned long long* meta = nullptr;
    uint32_t* tx_stamp = nullptr;
    uint32_t* tx_result = nullptr;
    uint64_t log_cap = 0;
    uint32_t* km_cluster = nullptr;  // KM full iteration: per-tx nearest centroid (km.cu)
    uint64_t km_cap = 0;
    cudaStream_t own_stream = nullptr, stream = nullptr;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    // pipelined host-buffer steps (gstm_run_host_async): copy streams,
    // staging buffers and the events that order them
    cudaStream_t s_in = nullptr, s_out = nullptr;
    cudaEvent_t ev_call = nullptr, ev_in_ready = nullptr, ev_in_free = nullptr, ev_out_ready = nullptr,
                ev_out_free = nullptr;
    uint32_t* stage_in = nullptr;
    uint32_t* stage_out = nullptr;
    uint64_t stage_words = 0;
    bool pipe_open = false;          // a pipelined call is in flight since the last join
    const uint32_t* last_out = nullptr;   // heap_out of the last pipelined call (alias check)
    uint64_t last_out_words = 0;
    int dev = 0;                     // the device the handle was created on
    bool l2_user = false;            // counted in g_l2_users[dev] (l2_persist_locks)
    gstm_params_t params{};
    int mode = GSTM_MODE_AUTO;
    // last launch
    bool launched = false;
    int last_mode = 0;
    uint64_t last_n = 0;
    uint64_t clock_bound = 0;    // upper bound of g_clock (host-tracked)
};

// L2 persistence for the version-lock table (params.l2_persist_locks): an
// access-policy window on the handle's stream covering the lock table,
// hit property persisting, set around the transaction kernel's launch.
// The persisting set-aside (cudaLimitPersistingL2CacheSize) is device-wide and
// outlives the handle that set it, so it is reference-counted per device: a
// handle becomes a user at its first persisting launch and stops being one
// when it launches without persistence or is destroyed; the set-aside is
// released (limit 0, persisting lines demoted) when the last user stops --
// a leftover 64 MiB set-aside cut EB with a 256 MiB lock table from 411 to
// 170 M tx/s -- and never while another handle on the device still uses it.
static constexpr int kMaxDevices = 64;
static std::mutex g_l2_mu;
static int g_l2_users[kMaxDevices];
static size_t g_l2_limit[kMaxDevices];

static cudaError_t l2_limits(int dev, size_t* max_persist, size_t* max_window)
{
    static std::mutex mu;
    static size_t mp[kMaxDevices], mw[kMaxDevices];
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    std::lock_guard<std::mutex> g(mu);
    if (!mw[dev]) {
        cudaDeviceProp pr;
        cudaError_t e = cudaGetDeviceProperties(&pr, dev);
        if (e != cudaSuccess) return e;
        mp[dev] = pr.persistingL2CacheMaxSize;
        mw[dev] = pr.accessPolicyMaxWindowSize;
    }
    *max_persist = mp[dev];
    *max_window = mw[dev];
    return cudaSuccess;
}

// L2 size of a device (cached; the adaptive pipelined round's rule, launch)
static uint64_t l2_cache_bytes(int dev)
{
    static std::mutex mu;
    static uint64_t b[kMaxDevices];
    if (dev < 0 || dev >= kMaxDevices) return 0;
    std::lock_guard<std::mutex> g(mu);
    if (!b[dev]) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrL2CacheSize, dev) != cudaSuccess) return 0;
        b[dev] = static_cast<uint64_t>(v);
    }
    return b[dev];
}

// does the handle's lock table fit the persisting set-aside?  A larger table
// would only shrink the L2 left for everything else (measured: EB with 2^26
// locks, 256 MiB, 384 -> 146 M tx/s), so the knob then does nothing.
static bool l2_persist_fits(const gstm_t* h)
{
    size_t mp = 0, mw = 0;
    if (l2_limits(h->dev, &mp, &mw) != cudaSuccess || !mp || !mw) return false;
    return (sizeof(uint32_t) << h->bits) <= std::min(mp, mw);
}

// the handle stops using the set-aside; the last user on its device releases it
static cudaError_t l2_unuse(gstm_t* h)
{
    std::lock_guard<std::mutex> g(g_l2_mu);
    if (!h->l2_user) return cudaSuccess;
    h->l2_user = false;
    if (--g_l2_users[h->dev] > 0) return cudaSuccess;
    g_l2_users[h->dev] = 0;
    g_l2_limit[h->dev] = 0;
    int cur = 0;
    cudaGetDevice(&cur);
    if (cur != h->dev) cudaSetDevice(h->dev);
    cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
    if (e == cudaSuccess) e = cudaCtxResetPersistingL2Cache();
    if (cur != h->dev) cudaSetDevice(cur);
    return e;
}

// the handle uses the set-aside: grow the device's limit to what it needs
static cudaError_t l2_use(gstm_t* h, size_t lim)
{
    std::lock_guard<std::mutex> g(g_l2_mu);
    if (!h->l2_user) {
        h->l2_user = true;
        ++g_l2_users[h->dev];
    }
    if (lim <= g_l2_limit[h->dev]) return cudaSuccess;
    cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, lim);
    if (e == cudaSuccess) g_l2_limit[h->dev] = lim;
    return e;
}

static cudaError_t set_l2_lock_window(gstm_t* h, bool on)
{
    cudaStreamAttrValue a;
    memset(&a, 0, sizeof(a));
    if (on) {
        size_t mp = 0, mw = 0;
        cudaError_t e = l2_limits(h->dev, &mp, &mw);
        if (e != cudaSuccess) return e;
        const size_t bytes = std::min(sizeof(uint32_t) << h->bits, mw);
        const size_t lim = std::min(bytes, mp);
        e = l2_use(h, lim);
        if (e != cudaSuccess) return e;
        a.accessPolicyWindow.base_ptr = h->locks;
        a.accessPolicyWindow.num_bytes = bytes;
        a.accessPolicyWindow.hitRatio = bytes ? std::min(1.0f, static_cast<float>(lim) / static_cast<float>(bytes)) : 0.f;
        a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    }
    return cudaStreamSetAttribute(h->stream, cudaStreamAttributeAccessPolicyWindow, &a);
}

static gstm_params_t default_params(int workload)
{
    gstm_params_t p;
    memset(&p, 0, sizeof(p));
    p.n_reads = 4;
    p.n_writes = 4;
    p.ra_kind = 0;
    p.n_words = 1024;
    p.n_accesses = 16;
    p.ht_buckets = 1u << 20;
    p.ht_lookup_pct = 90;
    p.ht_key_range = 1ull << 22;
    p.km_clusters = 1024;
    p.km_dims = 16;
    p.prelock_vbv = 1;
    p.k_lock = 8;
    p.backoff_ns = 0;
    p.verify = 0;
    p.block_threads = 256;
    p.spin_cap = 1u << 16;
    p.timeout_ms = 60000;
    p.snapshot_reuse = 1;
    p.lock_pipeline = 1;
    p.body_rounds = 1;
    p.pipeline_max_locks = 8;
    p.serial_after = 0;
    p.serial_commits = 4;
    p.lock_pipeline_gated = 0;
    p.pipeline_abort = 0;
    // k-means: every contender of a record needs its lowest lock first; the
    // gated round holds the 17 locks for two round trips instead of 17
    // (26.5 -> 32.7 M tx/s; EB's random words lose with it)
    if (workload == GSTM_WL_KM) p.lock_pipeline_gated = 1;
    if (workload == GSTM_WL_BANK) {
        p.n_words = 1ull << 20;
        // a transaction pipelines the first lock round of its first 4
        // executions (9.21 vs 8.83 G tx/s with 1)
        p.lock_pipeline = 4;
    }
    // bank and RA: a word still locked after one re-read makes the transaction
    // re-execute in its warp's next iteration instead of holding the warp up
    // (Q38; RA 8M words: 776 -> 1007 M tx/s; EB is 7% slower with it, HT and
    // KM unchanged)
    if (workload == GSTM_WL_BANK || workload == GSTM_WL_RA) p.spin_cap = 1;
    // HT: the optional pre-lock VBV (A3.l71) ran on ~every update commit and
    // HT's inserts rarely contend (5.44 -> 5.86 G tx/s without it)
    if (workload == GSTM_WL_HT) p.prelock_vbv = 0;
    // HT: 90% of the transactions are read-only lookups that never use their
    // lock log; read locks enter it at TXCommit (write locks still at
    // encounter time): HV 6.81 -> 7.08, TBV 7.46 -> 7.89 G tx/s
    if (workload == GSTM_WL_HT) p.lock_log_at_commit = 1;
    if (workload == GSTM_WL_EB) {
        p.n_words = 1ull << 20;
        // the hot set may exceed L2: keep the lock table there (DESIGN.md §6.10:
        // hot set 2^26, A=16: 336 -> 369 M tx/s with 2^22 locks, 391 -> 453 with 2^24)
        p.l2_persist_locks = 1;
        // the adaptive contention manager (compiled into the
        // A > 16 kernels): serial tickets only where one-at-a-time measures
        // faster -- the corner (hot set 2^10, A = 64) 1.14 s -> 0.86 s per
        // launch, every other sweep point unchanged (no ticket taken)
        p.serial_after = 4;
    }
    // RA (random words, contended): the sequential first round is faster
    // even when the lock log fits one pipelined chunk (RA 8M words: 0.76 vs
    // 0.53 G tx/s)
    if (workload == GSTM_WL_RA) p.lock_pipeline = 0;
    // EB: logs of up to 16 locks take one pipelined round while the warp's
    // recent abort rate is below 100/256, and a failed pipelined round
    // re-executes at once (pipeline_abort): hot set 2^26 A=16 681 -> 761,
    // A=8 1535 -> 1729 M tx/s; the contended points run sequential rounds as
    // before (hot set 2^18-2^22 within 4%, the 2^10 corners unchanged)
    if (workload == GSTM_WL_EB) {
        p.lock_pipeline = 16;
        p.pipeline_max_locks = 16;
        p.pipeline_abort = 100;
    }
    return p;
}

static WlParams wl_params(const gstm_params_t& p, uint64_t T, uint64_t K)
{
    WlParams w;
    w.n_words = p.n_words;
    w.n_reads = p.n_reads;
    w.n_writes = p.n_writes;
    w.ra_kind = p.ra_kind;
    w.n_accesses = p.n_accesses;
    w.ht_buckets = p.ht_buckets;
    w.ht_lookup_pct = p.ht_lookup_pct;
    w.ht_key_range = p.ht_key_range;
    w.km_clusters = p.km_clusters;
    w.km_dims = p.km_dims;
    w.km_stride = p.km_stride ? p.km_stride : p.km_dims + 1;
    w.km_assign = p.km_assign;
    w.km_cluster = nullptr;
    w.shard_bits = p.shard_bits;
    w.shard = p.shard;
    w.ra_partition = p.ra_partition;
    w.T = T;
    w.K = K;
    return w;
}

static void fill_stats(gstm_stats_t* out, const unsigned long long* s, double ms, uint32_t err, int mode)
{
    memset(out, 0, sizeof(*out));
    out->commits = s[S_COMMITS];
    out->commits_ro = s[S_COMMITS_RO];
    out->aborts_opacity = s[S_AB_OPACITY];
    out->aborts_prevbv = s[S_AB_PREVBV];
    out->aborts_tbv = s[S_AB_TBV];
    out->aborts_commit_vbv = s[S_AB_COMMITVBV];
    out->aborts_lock = s[S_AB_LOCK];
    out->aborts = out->aborts_opacity + out->aborts_prevbv + out->aborts_tbv + out->aborts_commit_vbv + out->aborts_lock;
    out->lock_retries = s[S_LOCK_RETRIES];
    out->postvalidations = s[S_POSTVAL];
    out->vbv_runs = s[S_VBV];
    out->spins = s[S_SPINS];
    out->attempts = s[S_ATTEMPTS];
    out->errors = s[S_ERRORS];
    out->pipelined_rounds = s[S_PIPELINED];
    out->reads_update = s[S_RD_UPD];
    out->reads_ro = s[S_RD_RO];
    out->writes_update = s[S_WR_UPD];
    out->locks_update = s[S_LK_UPD];
    out->serial_runs = s[S_SERIAL];
    out->elapsed_ms = ms;
    const double done = static_cast<double>(out->commits + out->commits_ro);
    out->tx_per_s = ms > 0 ? done / (ms * 1e-3) : 0.0;
    out->abort_ratio = (done + out->aborts) > 0 ? out->aborts / (done + out->aborts) : 0.0;
    out->mode_used = mode;
    out->status = (err & ERR_TIMEOUT) ? GSTM_ETIMEOUT : (err & (ERR_LOGOVF | ERR_INVALID)) ? GSTM_ELOGOVF : GSTM_OK;
}

extern "C" {

const char* gstm_last_error(void) { return g_err; }
int gstm_api_version(void) { return GSTM_API_VERSION; }

int gstm_default_params(int workload, gstm_params_t* out)
{
    if (!out || workload < 0 || workload > 4) { set_error("gstm_default_params: bad argument"); return GSTM_EINVAL; }
    *out = default_params(workload);
    return GSTM_OK;
}

gstm_t* gstm_create(uint64_t heap_words, uint32_t lock_table_bits)
{
    return gstm_create_ex(heap_words, lock_table_bits, 0);
}

gstm_t* gstm_create_ex(uint64_t heap_words, uint32_t lock_table_bits, uint32_t flags)
{
    g_err[0] = 0;
    if (lock_table_bits > 30) { set_error("gstm_create: lock_table_bits %u > 30", lock_table_bits); return nullptr; }
    if (flags & ~uint32_t(GSTM_CREATE_PAIRED)) { set_error("gstm_create_ex: unknown flags 0x%x", flags); return nullptr; }
    const bool paired = (flags & GSTM_CREATE_PAIRED) != 0;
    if (paired && (heap_words == 0 || heap_words > (1ull << lock_table_bits))) {
        set_error("gstm_create_ex: the paired layout needs 1 <= heap_words <= 2^lock_table_bits (one lock per word)");
        return nullptr;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) { set_error("gstm_create: no CUDA device"); return nullptr; }
    gstm_t* h = new gstm_t();
    cudaGetDevice(&h->dev);
    if (h->dev < 0 || h->dev >= kMaxDevices) { set_error("gstm_create: device %d out of range", h->dev); delete h; return nullptr; }
    h->bits = lock_table_bits;
    h->paired = paired;
    h->params = default_params(GSTM_WL_RA);
    // one allocation, fixed layout: where the hot words land must not depend
    // on the caller's other allocations.  Split (the paper's): [metadata |
    // lock table | heap].  Paired: [metadata | heap_words x (value, lock)].
    const size_t lock_bytes = paired ? 0 : (sizeof(uint32_t) << lock_table_bits);
    const size_t heap_bytes = ((paired ? heap_words * 8 : heap_words * 4) + 255) & ~size_t(255);
    if (cudaMalloc(&h->block, kMetaBytes + lock_bytes + heap_bytes) != cudaSuccess) goto oom;
    h->meta = reinterpret_cast<unsigned long long*>(h->block);
    if (paired) {
        h->own_heap = reinterpret_cast<uint32_t*>(h->block + kMetaBytes);
        h->locks = h->own_heap + 1;
    } else {
        h->locks = reinterpret_cast<uint32_t*>(h->block + kMetaBytes);
        h->own_heap = heap_words ? reinterpret_cast<uint32_t*>(h->block + kMetaBytes + lock_bytes) : nullptr;
    }
    h->clock = h->meta + M_CLOCK;
    if (cudaStreamCreateWithFlags(&h->own_stream, cudaStreamNonBlocking) != cudaSuccess) goto cuerr;
    if (cudaEventCreate(&h->ev0) != cudaSuccess || cudaEventCreate(&h->ev1) != cudaSuccess) goto cuerr;
    h->stream = h->own_stream;
    h->heap = h->own_heap;
    h->heap_words = h->own_words = heap_words;
    if (cudaMemsetAsync(h->block, 0, kMetaBytes + lock_bytes + heap_bytes, h->stream) != cudaSuccess) goto cuerr;
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) goto cuerr;
    {
        // place g_clock on the candidate line with the fastest probe
        // (DESIGN.md §6.5); GSTM_CLOCK_SLOT=k forces candidate k,
        // GSTM_CLOCK_SLOT=-1 the fixed word M_CLOCK
        const char* cs = getenv("GSTM_CLOCK_SLOT");
        int slot;
        if (cs) {
            slot = atoi(cs);
        } else if (lock_table_bits < 14) {
            slot = -1;          // small tables: the hot-slice effect is negligible, skip the probe
        } else {
            // the probe's random lock-table and heap traffic goes over the
            // handle's own tables (for the paired layout: the pair array)
            uint32_t* tbl = paired ? h->own_heap : h->locks;
            const uint64_t tbl_words = paired ? 2 * heap_words : (1ull << lock_table_bits);
            uint32_t* hp = paired ? h->own_heap : (heap_words ? h->own_heap : h->locks);
            const uint64_t hp_words = paired ? 2 * heap_words : (heap_words ? heap_words : tbl_words);
            uint64_t t2 = 1, h2 = 1;
            while (t2 * 2 <= tbl_words) t2 *= 2;
            while (h2 * 2 <= hp_words) h2 *= 2;
            slot = clock_calibrate_mix(h->meta + M_WORDS, kClockCandidates, kClockStride, tbl,
                                       static_cast<uint32_t>(t2 - 1), hp, static_cast<uint32_t>(h2 - 1), h->stream);
        }
        if (slot >= kClockCandidates) slot = kClockCandidates - 1;
        h->clock_slot = slot;
        h->clock = slot < 0 ? h->meta + M_CLOCK : h->meta + M_WORDS + static_cast<size_t>(slot) * kClockStride;
    }
    return h;
oom:
    set_error("gstm_create: out of device memory (heap %llu words, 2^%u locks)", (unsigned long long)heap_words,
              lock_table_bits);
    gstm_destroy(h);
    return nullptr;
cuerr:
    set_error("gstm_create: %s", cudaGetErrorString(cudaGetLastError()));
    gstm_destroy(h);
    return nullptr;
}

uint32_t gstm_flags(const gstm_t* h) { return h && h->paired ? GSTM_CREATE_PAIRED : 0u; }

void gstm_destroy(gstm_t* h)
{
    if (!h) return;
    if (h->stream) cudaStreamSynchronize(h->stream);
    l2_unuse(h);
    cudaFree(h->block);
    cudaFree(h->scratch);
    cudaFree(h->tx_stamp);
    cudaFree(h->tx_result);
    cudaFree(h->km_cluster);
    if (h->s_in) cudaStreamSynchronize(h->s_in);
    if (h->s_out) cudaStreamSynchronize(h->s_out);
    cudaFree(h->stage_in);
    cudaFree(h->stage_out);
    for (cudaEvent_t e : {h->ev0, h->ev1, h->ev_call, h->ev_in_ready, h->ev_in_free, h->ev_out_ready, h->ev_out_free})
        if (e) cudaEventDestroy(e);
    if (h->s_in) cudaStreamDestroy(h->s_in);
    if (h->s_out) cudaStreamDestroy(h->s_out);
    if (h->own_stream) cudaStreamDestroy(h->own_stream);
    delete h;
}

int gstm_set_params(gstm_t* h, const gstm_params_t* p)
{
    if (!h || !p) { set_error("gstm_set_params: NULL"); return GSTM_EINVAL; }
    if (p->block_threads == 0 || p->block_threads > 256 || p->block_threads % 32) {
        set_error("gstm_set_params: block_threads must be a multiple of 32 in [32, 256]");
        return GSTM_EINVAL;
    }
    h->params = *p;
    return GSTM_OK;
}

int gstm_get_params(const gstm_t* h, gstm_params_t* out)
{
    if (!h || !out) { set_error("gstm_get_params: NULL"); return GSTM_EINVAL; }
    *out = h->params;
    return GSTM_OK;
}

int gstm_set_mode(gstm_t* h, int mode)
{
    if (!h || mode < GSTM_MODE_AUTO || mode > GSTM_MODE_HV_UNSORTED) { set_error("gstm_set_mode: bad mode %d", mode); return GSTM_EINVAL; }
    h->mode = mode;
    return GSTM_OK;
}

int gstm_set_stream(gstm_t* h, void* stream)
{
    if (!h) { set_error("gstm_set_stream: NULL"); return GSTM_EINVAL; }
    h->stream = stream ? static_cast<cudaStream_t>(stream) : h->own_stream;
    return GSTM_OK;
}

int gstm_attach_heap(gstm_t* h, void* dev_ptr, uint64_t words)
{
    if (!h) { set_error("gstm_attach_heap: NULL"); return GSTM_EINVAL; }
    if (!dev_ptr || !words) {
        h->heap = h->own_heap;
        h->heap_words = h->own_words;
        return GSTM_OK;
    }
    if (h->paired) { set_error("gstm_attach_heap: not available with the paired layout"); return GSTM_EINVAL; }
    if (reinterpret_cast<uintptr_t>(dev_ptr) & 3) { set_error("gstm_attach_heap: unaligned pointer"); return GSTM_EINVAL; }
    h->heap = static_cast<uint32_t*>(dev_ptr);
    h->heap_words = words;
    return GSTM_OK;
}

uint64_t gstm_heap_words(const gstm_t* h) { return h ? h->heap_words : 0; }
void* gstm_heap_ptr(const gstm_t* h) { return h ? h->heap : nullptr; }

// paired layout: a plain device buffer of `words` words for packing
static int ensure_scratch(gstm_t* h, uint64_t words)
{
    if (h->scratch_words >= words) return GSTM_OK;
    cudaFree(h->scratch);
    h->scratch = nullptr;
    h->scratch_words = 0;
    if (cudaMalloc(&h->scratch, words * 4) != cudaSuccess) { set_error("out of device memory (scratch)"); return GSTM_ENOMEM; }
    h->scratch_words = words;
    return GSTM_OK;
}

// the device view of the handle's heap and lock table (tx.cuh Meta)
static Meta meta_of(const gstm_t* h)
{
    Meta m;
    memset(&m, 0, sizeof(m));
    m.heap = h->heap;
    m.locks = h->locks;
    m.lock_mask = static_cast<uint32_t>((1ull << h->bits) - 1);
    m.clock = h->clock;
    m.spin_cap = h->params.spin_cap ? h->params.spin_cap : (1u << 16);
    m.lock_shift = h->params.lock_shift;
    m.vshift = m.lshift = h->paired ? 1u : 0u;
    return m;
}

int gstm_init_heap(gstm_t* h, int workload)
{
    if (!h || workload < 0 || workload > 4) { set_error("gstm_init_heap: bad argument"); return GSTM_EINVAL; }
    CUDA_TRY(launch_init_heap(workload, h->heap, h->heap_words, h->paired ? 1 : 0, h->stream));
    const gstm_params_t& P = h->params;
    if (workload == GSTM_WL_KM && P.km_assign) {
        // the centroid table after the records
        const uint64_t stride = P.km_stride ? P.km_stride : P.km_dims + 1ull;
        const uint64_t c0 = uint64_t(P.km_clusters) * stride, n = uint64_t(P.km_clusters) * P.km_dims;
        if (c0 + n > h->heap_words) { set_error("gstm_init_heap: k-means centroid table beyond the heap"); return GSTM_EINVAL; }
        CUDA_TRY(launch_km_init_centroids(meta_of(h), c0, n, h->stream));
    }
    return GSTM_OK;
}

int gstm_km_recenter(gstm_t* h)
{
    if (!h) { set_error("gstm_km_recenter: NULL handle"); return GSTM_EINVAL; }
    const gstm_params_t& P = h->params;
    const uint64_t stride = P.km_stride ? P.km_stride : P.km_dims + 1ull;
    if (!P.km_assign || P.km_clusters == 0 || P.km_dims > 16 || stride < P.km_dims + 1ull ||
        uint64_t(P.km_clusters) * (stride + P.km_dims) > h->heap_words) {
        set_error("gstm_km_recenter: needs km_assign = 1 and a heap holding the records and the centroid table");
        return GSTM_EINVAL;
    }
    CUDA_TRY(launch_km_recenter(meta_of(h), P.km_clusters, P.km_dims, static_cast<uint32_t>(stride), h->stream));
    return GSTM_OK;
}

// host -> heap words [offset, offset+words), asynchronous on the handle's stream
static int copy_in(gstm_t* h, const uint32_t* src, uint64_t offset, uint64_t words)
{
    if (!words) return GSTM_OK;
    if (!h->paired) {
        CUDA_TRY(cudaMemcpyAsync(h->heap + offset, src, words * 4, cudaMemcpyHostToDevice, h->stream));
        return GSTM_OK;
    }
    int rc = ensure_scratch(h, words);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(h->scratch, src, words * 4, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(launch_pack(h->scratch, h->heap + 2 * offset, words, 1, h->stream));
    return GSTM_OK;
}

static int copy_out(gstm_t* h, uint32_t* dst, uint64_t offset, uint64_t words)
{
    if (!words) return GSTM_OK;
    if (!h->paired) {
        CUDA_TRY(cudaMemcpyAsync(dst, h->heap + offset, words * 4, cudaMemcpyDeviceToHost, h->stream));
        return GSTM_OK;
    }
    int rc = ensure_scratch(h, words);
    if (rc) return rc;
    CUDA_TRY(launch_pack(h->scratch, h->heap + 2 * offset, words, 0, h->stream));
    CUDA_TRY(cudaMemcpyAsync(dst, h->scratch, words * 4, cudaMemcpyDeviceToHost, h->stream));
    return GSTM_OK;
}

int gstm_write_heap(gstm_t* h, const uint32_t* src, uint64_t offset, uint64_t words)
{
    if (!h || (!src && words) || offset + words > h->heap_words) { set_error("gstm_write_heap: bad range"); return GSTM_EINVAL; }
    int rc = copy_in(h, src, offset, words);
    if (rc) return rc;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return GSTM_OK;
}

int gstm_read_heap(gstm_t* h, uint32_t* dst, uint64_t offset, uint64_t words)
{
    if (!h || (!dst && words) || offset + words > h->heap_words) { set_error("gstm_read_heap: bad range"); return GSTM_EINVAL; }
    int rc = copy_out(h, dst, offset, words);
    if (rc) return rc;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return GSTM_OK;
}

int gstm_read_locks(gstm_t* h, uint32_t* dst, uint64_t n)
{
    if (!h || !dst || n > (1ull << h->bits)) { set_error("gstm_read_locks: bad range"); return GSTM_EINVAL; }
    if (!h->paired) {
        CUDA_TRY(cudaMemcpyAsync(dst, h->locks, n * 4, cudaMemcpyDeviceToHost, h->stream));
    } else {
        // lock i lives next to word i; locks of ids >= heap_words are never used
        const uint64_t m = n < h->own_words ? n : h->own_words;
        int rc = ensure_scratch(h, m ? m : 1);
        if (rc) return rc;
        CUDA_TRY(launch_lock_halves(h->own_heap, m, h->scratch, h->stream));
        if (m) CUDA_TRY(cudaMemcpyAsync(dst, h->scratch, m * 4, cudaMemcpyDeviceToHost, h->stream));
        for (uint64_t k = m; k < n; ++k) dst[k] = 0;
    }
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return GSTM_OK;
}

int gstm_read_clock(gstm_t* h, uint64_t* out)
{
    if (!h || !out) { set_error("gstm_read_clock: NULL"); return GSTM_EINVAL; }
    unsigned long long c = 0;
    CUDA_TRY(cudaMemcpyAsync(&c, h->clock, 8, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    *out = c;
    return GSTM_OK;
}

int gstm_reset_meta(gstm_t* h)
{
    if (!h) { set_error("gstm_reset_meta: NULL"); return GSTM_EINVAL; }
    if (h->paired) CUDA_TRY(launch_lock_halves(h->own_heap, h->own_words, nullptr, h->stream));
    else CUDA_TRY(cudaMemsetAsync(h->locks, 0, sizeof(uint32_t) << h->bits, h->stream));
    CUDA_TRY(cudaMemsetAsync(h->clock, 0, 8, h->stream));
    h->clock_bound = 0;
    return GSTM_OK;
}

int gstm_set_clock(gstm_t* h, uint64_t value)
{
    if (!h || value >= (1ull << 31)) { set_error("gstm_set_clock: bad argument"); return GSTM_EINVAL; }
    unsigned long long v = value;
    CUDA_TRY(cudaMemcpyAsync(h->clock, &v, 8, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    if (value > h->clock_bound) h->clock_bound = value;
    return GSTM_OK;
}

static int resolve_mode(const gstm_t* h, uint64_t footprint)
{
    if (h->mode != GSTM_MODE_AUTO) return h->mode;
    // STM-Optimized: HV when shared data exceeds the version locks
    return footprint > (1ull << h->bits) ? GSTM_MODE_HV : GSTM_MODE_TBV;
}

int gstm_launch(gstm_t* h, int workload, uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed)
{
    if (!h) { set_error("gstm_launch: NULL handle"); return GSTM_EINVAL; }
    const gstm_params_t& P = h->params;
    WlParams w = wl_params(P, n_threads, tx_per_thread);
    uint64_t fp = 0;
    int dw = 0;
    if (workload < 0 || workload > 4 || !workload_check(workload, w, &fp, &dw)) {
        set_error("gstm_launch: invalid parameters for workload %d", workload);
        return GSTM_EINVAL;
    }
    if (fp > h->heap_words) {
        set_error("gstm_launch: workload footprint %llu words > heap %llu words", (unsigned long long)fp,
                  (unsigned long long)h->heap_words);
        return GSTM_EINVAL;
    }
    if (n_threads > (1ull << 32)) { set_error("gstm_launch: n_threads > 2^32"); return GSTM_EINVAL; }
    if (h->paired && P.lock_shift) { set_error("gstm_launch: the paired layout has one lock per word (lock_shift 0)"); return GSTM_EINVAL; }
    if (P.lock_shift > 31) { set_error("gstm_launch: lock_shift > 31"); return GSTM_EINVAL; }
    const uint64_t n_tx = n_threads * tx_per_thread;
    if (n_tx >= (1ull << 31) - 2) { set_error("gstm_launch: %llu transactions >= 2^31", (unsigned long long)n_tx); return GSTM_EOVERFLOW; }
    // 31-bit versions: start a new version epoch before they can wrap
    if (h->clock_bound + n_tx >= (1ull << 31) - 2) {
        int rc = gstm_reset_meta(h);
        if (rc) return rc;
    }
    if (P.verify && n_tx > h->log_cap) {
        cudaFree(h->tx_stamp);
        cudaFree(h->tx_result);
        h->tx_stamp = h->tx_result = nullptr;
        h->log_cap = 0;
        if (cudaMalloc(&h->tx_stamp, n_tx * 4) != cudaSuccess || cudaMalloc(&h->tx_result, n_tx * 4) != cudaSuccess) {
            cudaFree(h->tx_stamp);
            h->tx_stamp = nullptr;
            set_error("gstm_launch: cannot allocate the verify log (%llu tx)", (unsigned long long)n_tx);
            return GSTM_ENOMEM;
        }
        h->log_cap = n_tx;
    }
    const bool km_assign = workload == GSTM_WL_KM && P.km_assign;
    if (km_assign && n_tx > h->km_cap) {
        cudaFree(h->km_cluster);
        h->km_cluster = nullptr;
        h->km_cap = 0;
        if (cudaMalloc(&h->km_cluster, n_tx * 4) != cudaSuccess) {
            h->km_cluster = nullptr;
            set_error("gstm_launch: cannot allocate the k-means assignment (%llu points)", (unsigned long long)n_tx);
            return GSTM_ENOMEM;
        }
        h->km_cap = n_tx;
    }
    if (km_assign && uint64_t(P.km_clusters) * P.km_dims > 16384) {
        set_error("gstm_launch: k-means centroid table > 64 KiB (km_clusters * km_dims > 16384)");
        return GSTM_EINVAL;
    }
    const int mode = resolve_mode(h, fp);
    KParams kp;
    memset(&kp, 0, sizeof(kp));
    kp.m = meta_of(h);
    kp.paired = h->paired ? 1u : 0u;
    kp.w = w;
    kp.meta = h->meta;
    kp.tx_stamp = P.verify ? h->tx_stamp : nullptr;
    kp.tx_result = P.verify ? h->tx_result : nullptr;
    kp.T = n_threads;
    kp.K = tx_per_thread;
    kp.seed = seed;
    kp.prelock_vbv = P.prelock_vbv;
    kp.k_lock = P.k_lock;
    kp.backoff_ns = P.backoff_ns;
    kp.snapshot_reuse = P.snapshot_reuse;
    kp.lock_pipeline = P.lock_pipeline;
    kp.max_threads = P.max_threads;
    kp.body_rounds = P.body_rounds ? P.body_rounds : 1u;
    kp.pipeline_max_locks = P.pipeline_max_locks ? P.pipeline_max_locks : 8u;
    kp.lock_log_at_commit = P.lock_log_at_commit;
    kp.serial_after = P.serial_after;
    kp.serial_commits = P.serial_commits ? P.serial_commits : 4u;
    kp.lock_pipeline_gated = P.lock_pipeline_gated;
    kp.pipeline_abort = P.pipeline_abort;
    if (P.pipeline_abort) {
        // the adaptive pipelined round pays where sequential rounds are slow
        // and false conflicts rare: a shared footprint larger than L2 (every
        // commit's VBV and write-back go to HBM) and at least one version lock
        // per 4 words; elsewhere (L2-resident hot sets, few locks) the rounds
        // stay sequential (EB hot set 2^26 with 2^24 locks
        // +11%, with 2^20-2^22 locks -6..-32% if it were on)
        const uint64_t l2 = l2_cache_bytes(h->dev);
        const bool pays = l2 && fp * 4 > l2 && (1ull << h->bits) * 4 >= fp;
        if (!pays) {
            kp.lock_pipeline = 0;
            kp.pipeline_abort = 0;
        } else {
            // ... and there the optional pre-lock VBV (A3.l71, "to reduce lock
            // contention") only adds an HBM round trip before the atomics: a
            // failed pipelined round re-executes anyway (767 -> 804 M tx/s)
            kp.prelock_vbv = 0;
        }
    }
    const uint64_t timeout_ns = static_cast<uint64_t>(P.timeout_ms ? P.timeout_ms : 60000) * 1000000ull;
    CUDA_TRY(cudaEventRecord(h->ev0, h->stream));
    CUDA_TRY(launch_prepare(h->meta, h->clock, timeout_ns, h->stream));
    if (km_assign && n_tx) {
        // a full k-means iteration: every point's nearest centroid first
        CUDA_TRY(launch_km_assign(kp, h->km_cluster, h->stream));
        kp.w.km_cluster = h->km_cluster;
    }
    const bool persist = P.l2_persist_locks && !h->paired && h->locks && l2_persist_fits(h);
    if (persist) CUDA_TRY(set_l2_lock_window(h, true));
    else CUDA_TRY(l2_unuse(h));
    CUDA_TRY(launch_tx(workload, mode, kp, P.block_threads ? P.block_threads : 256, h->stream));
    if (persist) CUDA_TRY(set_l2_lock_window(h, false));
    CUDA_TRY(launch_finish(h->meta, h->clock, h->stream));
    CUDA_TRY(cudaEventRecord(h->ev1, h->stream));
    h->clock_bound += n_tx;
    h->launched = true;
    h->last_mode = mode;
    h->last_n = n_tx;
    return GSTM_OK;
}

int gstm_stats(gstm_t* h, gstm_stats_t* out)
{
    if (!h || !out) { set_error("gstm_stats: NULL"); return GSTM_EINVAL; }
    if (!h->launched) { set_error("gstm_stats: no launch"); return GSTM_EBUSY; }
    CUDA_TRY(cudaEventSynchronize(h->ev1));
    unsigned long long m[M_WORDS];
    CUDA_TRY(cudaMemcpyAsync(m, h->meta, sizeof(m), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    float ms = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&ms, h->ev0, h->ev1));
    fill_stats(out, m + M_STATS, ms, static_cast<uint32_t>(m[M_ERR]), h->last_mode);
    out->clock_slot = h->clock_slot;
    out->clock_begin = m[M_CLOCK_BEGIN];
    out->clock_end = m[M_CLOCK_END];
    if (out->status) set_error("gstm_stats: launch reported %s", out->status == GSTM_ETIMEOUT ? "watchdog timeout" : "log overflow");
    return out->status;
}

int gstm_stats_total(gstm_t* h, gstm_stats_t* out, uint64_t* launches)
{
    if (!h || !out) { set_error("gstm_stats_total: NULL"); return GSTM_EINVAL; }
    unsigned long long m[M_WORDS];
    CUDA_TRY(cudaMemcpyAsync(m, h->meta, sizeof(m), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    fill_stats(out, m + M_TOTALS, m[M_T_NS] * 1e-6, static_cast<uint32_t>(m[M_T_ERR]), h->last_mode);
    out->clock_slot = h->clock_slot;
    out->clock_end = m[M_CLOCK_END];
    if (launches) *launches = m[M_T_LAUNCHES];
    if (out->status) set_error("gstm_stats_total: a launch reported %s", out->status == GSTM_ETIMEOUT ? "watchdog timeout" : "log overflow");
    return out->status;
}

int gstm_reset_stats_total(gstm_t* h)
{
    if (!h) { set_error("gstm_reset_stats_total: NULL"); return GSTM_EINVAL; }
    CUDA_TRY(cudaMemsetAsync(h->meta + M_TOTALS, 0, (M_PHASE + kPhaseWords - M_TOTALS) * 8, h->stream));
    return GSTM_OK;
}

int gstm_phase_cycles(gstm_t* h, uint64_t* out, int n)
{
    if (!h || !out || n < 0) { set_error("gstm_phase_cycles: bad argument"); return GSTM_EINVAL; }
    unsigned long long ph[kPhaseWords];
    CUDA_TRY(cudaMemcpyAsync(ph, h->meta + M_PHASE, sizeof(ph), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    for (int k = 0; k < n && k < kPhaseWords; ++k) out[k] = ph[k];
    return GSTM_OK;
}

int gstm_read_tx_log(gstm_t* h, uint32_t* stamps, uint32_t* results, uint64_t n)
{
    if (!h) { set_error("gstm_read_tx_log: NULL"); return GSTM_EINVAL; }
    if (!h->launched || !h->tx_stamp || n > h->log_cap) { set_error("gstm_read_tx_log: no verify log of %llu entries", (unsigned long long)n); return GSTM_EBUSY; }
    if (stamps) CUDA_TRY(cudaMemcpyAsync(stamps, h->tx_stamp, n * 4, cudaMemcpyDeviceToHost, h->stream));
    if (results) CUDA_TRY(cudaMemcpyAsync(results, h->tx_result, n * 4, cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return GSTM_OK;
}

int gstm_run_host(gstm_t* h, int workload, const uint32_t* heap_in, uint32_t* heap_out, uint64_t words,
                  uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed, gstm_stats_t* stats)
{
    if (!h || words > h->heap_words || (words && (!heap_in || !heap_out))) { set_error("gstm_run_host: bad buffers"); return GSTM_EINVAL; }
    int rc = copy_in(h, heap_in, 0, words);
    if (rc) return rc;
    rc = gstm_launch(h, workload, n_threads, tx_per_thread, seed);
    if (rc) return rc;
    rc = copy_out(h, heap_out, 0, words);
    if (rc) return rc;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    gstm_stats_t local;
    return gstm_stats(h, stats ? stats : &local);
}

static int ensure_pipe(gstm_t* h, uint64_t words)
{
    if (!h->s_in) {
        CUDA_TRY(cudaStreamCreateWithFlags(&h->s_in, cudaStreamNonBlocking));
        CUDA_TRY(cudaStreamCreateWithFlags(&h->s_out, cudaStreamNonBlocking));
        for (cudaEvent_t* e : {&h->ev_call, &h->ev_in_ready, &h->ev_in_free, &h->ev_out_ready, &h->ev_out_free})
            CUDA_TRY(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    }
    if (h->stage_words < words) {
        // the staging buffers may still be in use by calls in flight
        CUDA_TRY(cudaStreamSynchronize(h->s_in));
        CUDA_TRY(cudaStreamSynchronize(h->stream));
        CUDA_TRY(cudaStreamSynchronize(h->s_out));
        cudaFree(h->stage_in);
        cudaFree(h->stage_out);
        h->stage_in = h->stage_out = nullptr;
        h->stage_words = 0;
        if (cudaMalloc(&h->stage_in, words * 4) != cudaSuccess || cudaMalloc(&h->stage_out, words * 4) != cudaSuccess) {
            set_error("out of device memory (staging)");
            return GSTM_ENOMEM;
        }
        h->stage_words = words;
    }
    return GSTM_OK;
}

int gstm_run_host_async(gstm_t* h, int workload, const uint32_t* heap_in, uint32_t* heap_out, uint64_t words,
                        uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed)
{
    if (!h || words > h->heap_words || (words && (!heap_in || !heap_out))) { set_error("gstm_run_host_async: bad buffers"); return GSTM_EINVAL; }
    if (!words) return gstm_launch(h, workload, n_threads, tx_per_thread, seed);
    int rc = ensure_pipe(h, words);
    if (rc) return rc;
    if (!h->pipe_open) {
        // the first call of a pipeline follows everything already enqueued
        // on the handle's stream (e.g. the caller's start event)
        CUDA_TRY(cudaEventRecord(h->ev_call, h->stream));
        CUDA_TRY(cudaStreamWaitEvent(h->s_in, h->ev_call, 0));
        CUDA_TRY(cudaStreamWaitEvent(h->s_out, h->ev_call, 0));
        h->pipe_open = true;
    }
    // copy-in: into the staging buffer once the previous step moved it out;
    // if heap_in overlaps the previous call's heap_out (steps chained in
    // place), also after that call's copy-out wrote it
    CUDA_TRY(cudaStreamWaitEvent(h->s_in, h->ev_in_free, 0));
    if (h->last_out && heap_in < h->last_out + h->last_out_words && h->last_out < heap_in + words)
        CUDA_TRY(cudaStreamWaitEvent(h->s_in, h->ev_out_free, 0));
    CUDA_TRY(cudaMemcpyAsync(h->stage_in, heap_in, words * 4, cudaMemcpyHostToDevice, h->s_in));
    CUDA_TRY(cudaEventRecord(h->ev_in_ready, h->s_in));
    // the step on the handle's stream: staging -> heap, transactions, heap -> staging
    CUDA_TRY(cudaStreamWaitEvent(h->stream, h->ev_in_ready, 0));
    if (h->paired) CUDA_TRY(launch_pack(h->stage_in, h->heap, words, 1, h->stream));
    else CUDA_TRY(cudaMemcpyAsync(h->heap, h->stage_in, words * 4, cudaMemcpyDeviceToDevice, h->stream));
    CUDA_TRY(cudaEventRecord(h->ev_in_free, h->stream));
    rc = gstm_launch(h, workload, n_threads, tx_per_thread, seed);
    if (rc) return rc;
    CUDA_TRY(cudaStreamWaitEvent(h->stream, h->ev_out_free, 0));
    if (h->paired) CUDA_TRY(launch_pack(h->stage_out, h->heap, words, 0, h->stream));
    else CUDA_TRY(cudaMemcpyAsync(h->stage_out, h->heap, words * 4, cudaMemcpyDeviceToDevice, h->stream));
    CUDA_TRY(cudaEventRecord(h->ev_out_ready, h->stream));
    // copy-out on its own stream, overlapping the next step's transactions
    CUDA_TRY(cudaStreamWaitEvent(h->s_out, h->ev_out_ready, 0));
    CUDA_TRY(cudaMemcpyAsync(heap_out, h->stage_out, words * 4, cudaMemcpyDeviceToHost, h->s_out));
    CUDA_TRY(cudaEventRecord(h->ev_out_free, h->s_out));
    h->last_out = heap_out;
    h->last_out_words = words;
    return GSTM_OK;
}

int gstm_join(gstm_t* h)
{
    if (!h) { set_error("gstm_join: NULL handle"); return GSTM_EINVAL; }
    if (h->pipe_open) {
        CUDA_TRY(cudaStreamWaitEvent(h->stream, h->ev_out_free, 0));
        h->pipe_open = false;
        h->last_out = nullptr;     // the next call's copy-in follows this join
        h->last_out_words = 0;
    }
    return GSTM_OK;
}

int gstm_sync(gstm_t* h)
{
    if (!h) { set_error("gstm_sync: NULL handle"); return GSTM_EINVAL; }
    int rc = gstm_join(h);
    if (rc) return rc;
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    if (!h->launched) return GSTM_OK;
    gstm_stats_t s;
    return gstm_stats(h, &s);
}

int gstm_descr_words(gstm_t* h, int workload)
{
    if (!h) { set_error("gstm_descr_words: NULL"); return GSTM_EINVAL; }
    WlParams w = wl_params(h->params, 1, 1);
    uint64_t fp;
    int dw = 0;
    if (!workload_check(workload, w, &fp, &dw)) { set_error("gstm_descr_words: invalid workload params"); return GSTM_EINVAL; }
    return dw;
}

int gstm_dump_descr(gstm_t* h, int workload, uint64_t n_threads, uint32_t tx_per_thread, uint64_t seed,
                    uint32_t* host_out, uint32_t words_per_tx)
{
    if (!h || !host_out) { set_error("gstm_dump_descr: NULL"); return GSTM_EINVAL; }
    WlParams w = wl_params(h->params, n_threads, tx_per_thread);
    uint64_t fp;
    int dw = 0;
    if (!workload_check(workload, w, &fp, &dw) || static_cast<int>(words_per_tx) < dw) {
        set_error("gstm_dump_descr: invalid workload params or words_per_tx < %d", dw);
        return GSTM_EINVAL;
    }
    const uint64_t n = n_threads * tx_per_thread * words_per_tx;
    if (!n) return GSTM_OK;
    uint32_t* d = nullptr;
    CUDA_TRY(cudaMalloc(&d, n * 4));
    KParams kp;
    memset(&kp, 0, sizeof(kp));
    kp.w = w;
    kp.T = n_threads;
    kp.K = tx_per_thread;
    kp.seed = seed;
    cudaError_t e = launch_descr(workload, kp, d, static_cast<int>(words_per_tx), h->stream);
    if (e == cudaSuccess) e = cudaMemcpyAsync(host_out, d, n * 4, cudaMemcpyDeviceToHost, h->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
    cudaFree(d);
    if (e != cudaSuccess) { set_error("gstm_dump_descr: %s", cudaGetErrorString(e)); return GSTM_ECUDA; }
    return GSTM_OK;
}

int gstm_script(gstm_t* h, int mode, int prelock_vbv, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx)
{
    return gstm_script_ex(h, mode, prelock_vbv, ops, n_ops, out, n_tx, 0);
}

int gstm_script_ex(gstm_t* h, int mode, int prelock_vbv, const uint32_t* ops, int n_ops, uint32_t* out, int n_tx,
                   int log_policy)
{
    if (!h || !ops || !out || n_ops < 0 || n_tx < 1 || n_tx > 8 || (mode != GSTM_MODE_HV && mode != GSTM_MODE_TBV) ||
        log_policy < 0 || log_policy > 2) {
        set_error("gstm_script: bad argument");
        return GSTM_EINVAL;
    }
    for (int k = 0; k < n_ops; ++k) {
        const uint32_t op = ops[4 * k], slot = ops[4 * k + 1], word = ops[4 * k + 2], val = ops[4 * k + 3];
        if (op > 4 || slot >= static_cast<uint32_t>(n_tx) || ((op == 1 || op == 2 || op == 4) && word >= h->heap_words) ||
            (op == 4 && val >= h->heap_words)) {
            set_error("gstm_script: bad op %d", k);
            return GSTM_EINVAL;
        }
    }
    if (!n_ops) return GSTM_OK;
    uint32_t *dops = nullptr, *dout = nullptr;
    CUDA_TRY(cudaMalloc(&dops, n_ops * 16));
    cudaError_t e = cudaMalloc(&dout, n_ops * 16);
    Meta m;
    m.heap = h->heap;
    m.locks = h->locks;
    m.lock_mask = static_cast<uint32_t>((1ull << h->bits) - 1);
    m.clock = h->clock;
    m.spin_cap = 64;
    m.lock_shift = 0;
    m.vshift = m.lshift = h->paired ? 1u : 0u;
    if (e == cudaSuccess) e = cudaMemcpyAsync(dops, ops, n_ops * 16, cudaMemcpyHostToDevice, h->stream);
    if (e == cudaSuccess) e = launch_script(m, mode, prelock_vbv, dops, n_ops, dout, n_tx, log_policy, h->stream);
    if (e == cudaSuccess) e = cudaMemcpyAsync(out, dout, n_ops * 16, cudaMemcpyDeviceToHost, h->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
    cudaFree(dops);
    cudaFree(dout);
    if (e != cudaSuccess) { set_error("gstm_script: %s", cudaGetErrorString(e)); return GSTM_ECUDA; }
    return GSTM_OK;
}

int gstm_lock_log(const uint32_t* entries, int n, uint32_t* out, int variant)
{
    if (!entries || !out || n < 0 || n > 4096 || variant < 0 || variant > 6) { set_error("gstm_lock_log: bad argument"); return GSTM_EINVAL; }
    uint32_t *de = nullptr, *dout = nullptr;
    int* dn = nullptr;
    CUDA_TRY(cudaMalloc(&de, (n + 1) * 4));
    CUDA_TRY(cudaMalloc(&dout, 256 * 4));
    CUDA_TRY(cudaMalloc(&dn, 4));
    int cnt = 0;
    cudaError_t e = cudaMemcpy(de, entries, n * 4, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = launch_lock_log(de, n, dout, dn, variant, 0);
    if (e == cudaSuccess) e = cudaMemcpy(&cnt, dn, 4, cudaMemcpyDeviceToHost);
    if (e == cudaSuccess && cnt > 0) e = cudaMemcpy(out, dout, cnt * 4, cudaMemcpyDeviceToHost);
    cudaFree(de);
    cudaFree(dout);
    cudaFree(dn);
    if (e != cudaSuccess) { set_error("gstm_lock_log: %s", cudaGetErrorString(e)); return GSTM_ECUDA; }
    if (cnt < 0) { set_error("gstm_lock_log: capacity exceeded"); return GSTM_ELOGOVF; }
    return cnt;
}

int gstm_ubench(int kind, uint64_t table_bytes, uint64_t n_ops, uint32_t threads, double* ops_per_s, double* ms)
{
    if (!ops_per_s) { set_error("gstm_ubench: NULL"); return GSTM_EINVAL; }
    const int rc = ubench(kind, table_bytes, n_ops, threads, ops_per_s, ms);
    if (rc == -1) { set_error("gstm_ubench: bad argument"); return GSTM_EINVAL; }
    if (rc) { set_error("gstm_ubench: CUDA failure %d", rc); return GSTM_ECUDA; }
    return GSTM_OK;
}

int gstm_ubench_mix(gstm_t* h, uint64_t words, const uint32_t* prog, uint32_t prog_words, uint64_t n_tx,
                    uint32_t threads, uint32_t block, double* tx_per_s, double* ms)
{
    if (!h || !tx_per_s || words > h->heap_words) { set_error("gstm_ubench_mix: bad argument"); return GSTM_EINVAL; }
    const int rc = ubench_mix(meta_of(h), h->paired, words, prog, prog_words, n_tx, threads, block, h->stream,
                              tx_per_s, ms);
    if (rc == -1) { set_error("gstm_ubench_mix: bad program or launch shape"); return GSTM_EINVAL; }
    if (rc) { set_error("gstm_ubench_mix: CUDA failure %d", rc); return GSTM_ECUDA; }
    // the clobbered lock table and clock start a new version epoch
    return gstm_reset_meta(h);
}

}  // extern "C"
