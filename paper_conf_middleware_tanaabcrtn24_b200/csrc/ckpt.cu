// ckpt.cu -- host side of libckpt.so: the C ABI declared in include/ckpt.h.
//
// Validation, tree layout (level-major flattened array, R13),
// device allocation (stream-ordered pool), metadata staging and kernel
// launches for K1 (leaf.cuh), K2 (levels.cuh), K3/K4 (compare.cuh).  Every
// step of the path runs in those kernels; there is no host or CPU fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cfloat>
#include <cmath>
#include <cstdio>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <functional>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/ckpt.h"
#include "compare.cuh"
#include "hash.cuh"
#include "leaf.cuh"
#include "levels.cuh"

using namespace ckpt;

// ---------------------------------------------------------------------------
// errors
// ---------------------------------------------------------------------------
static thread_local std::string g_last_error;
static std::atomic<uint64_t> g_launches{0};

static ckpt_status fail(ckpt_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

#define CK_CUDA(expr)                                                                       \
    do {                                                                                    \
        cudaError_t e_ = (expr);                                                            \
        if (e_ != cudaSuccess) {                                                            \
            return fail(e_ == cudaErrorMemoryAllocation ? CKPT_ENOMEM : CKPT_ECUDA,         \
                        std::string(#expr) + ": " + cudaGetErrorString(e_));                \
        }                                                                                   \
    } while (0)

#define CK_LAUNCH()                                                                         \
    do {                                                                                    \
        g_launches.fetch_add(1, std::memory_order_relaxed);                                 \
        cudaError_t e_ = cudaGetLastError();                                                \
        if (e_ != cudaSuccess)                                                              \
            return fail(CKPT_ECUDA, std::string("kernel launch: ") + cudaGetErrorString(e_)); \
    } while (0)

// Kernel launch with programmatic stream serialisation (see pdl_enter in
// hash.cuh); CKPT_PDL=0 in the environment turns the attribute off.
static bool pdl_on() {
    static const bool on = [] {
        const char *e = std::getenv("CKPT_PDL");
        return !(e && e[0] == '0');
    }();
    return on;
}

template <typename... KArgs, typename... Args>
static cudaError_t launch_k(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                            cudaStream_t s, Args &&...args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl_on() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// ---------------------------------------------------------------------------
// optional per-kernel-family event timing (ckpt_profile_*)
// ---------------------------------------------------------------------------
struct ProfRec { int k; cudaEvent_t a, b; };
static std::atomic<int> g_prof_on{0};
static std::mutex g_prof_mu;
static std::vector<ProfRec> g_prof;

struct ProfScope {
    int k;
    cudaStream_t s;
    cudaEvent_t a = nullptr, b = nullptr;
    ProfScope(int k_, cudaStream_t s_) : k(k_), s(s_) {
        if (g_prof_on.load(std::memory_order_relaxed) & (1 << k_)) {
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            cudaEventRecord(a, s);
        }
    }
    ~ProfScope() {
        if (a) {
            cudaEventRecord(b, s);
            std::lock_guard<std::mutex> lk(g_prof_mu);
            g_prof.push_back({k, a, b});
        }
    }
};

#define CK_TRY(expr)                         \
    do {                                     \
        ckpt_status s_ = (expr);             \
        if (s_ != CKPT_OK) return s_;        \
    } while (0)

// ---------------------------------------------------------------------------
// device properties
// ---------------------------------------------------------------------------
struct DevInfo {
    int sms = 0;
    int max_threads_sm = 0;
    bool pool_set = false;
};
static std::mutex g_dev_mu;
static DevInfo g_dev[64];

static cudaStream_t g_side[64];

// Per-device non-blocking side stream for K2.
static ckpt_status side_stream(int dev, cudaStream_t *out) {
    std::lock_guard<std::mutex> lk(g_dev_mu);
    if (!g_side[dev & 63]) {
        // lowest priority: K2's CTAs only take SM slots the diff/verify kernels leave free
        int lo = 0, hi = 0;
        CK_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        CK_CUDA(cudaStreamCreateWithPriority(&g_side[dev & 63], cudaStreamNonBlocking, lo));
    }
    *out = g_side[dev & 63];
    return CKPT_OK;
}

static ckpt_status dev_info(int *dev_out, DevInfo *info) {
    int dev = 0;
    CK_CUDA(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_dev_mu);
    DevInfo &d = g_dev[dev & 63];
    if (d.sms == 0) {
        CK_CUDA(cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev));
        CK_CUDA(cudaDeviceGetAttribute(&d.max_threads_sm, cudaDevAttrMaxThreadsPerMultiProcessor, dev));
        int major = 0, minor = 0;
        CK_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
        CK_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
        if (major != 10 || minor != 0) {
            d.sms = 0;
            return fail(CKPT_ECUDA, "libckpt is built for sm_100a (B200); device has sm_" +
                                        std::to_string(major) + std::to_string(minor));
        }
    }
    if (!d.pool_set) {
        cudaMemPool_t pool;
        CK_CUDA(cudaDeviceGetDefaultMemPool(&pool, dev));
        // keep freed blocks mapped in the pool (re-mapping tens of GB per call costs more
        // than the copies); ckpt_trim_device_memory() returns them to the driver
        uint64_t thr = UINT64_MAX;
        CK_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
        d.pool_set = true;
    }
    if (dev_out) *dev_out = dev;
    if (info) *info = d;
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// pinned staging ring for small host->device metadata copies
// ---------------------------------------------------------------------------
struct PinnedRing {
    std::mutex mu;
    uint8_t *base = nullptr;
    size_t cap = 0, head = 0;
    struct Span { size_t lo, hi; cudaEvent_t ev; };
    std::deque<Span> live;

    ckpt_status copy(void *dst_dev, const void *src, size_t bytes, cudaStream_t s) {
        std::lock_guard<std::mutex> lk(mu);
        const size_t n_copy = bytes;
        bytes = (bytes + 255) & ~size_t(255);
        if (base == nullptr) {
            cap = std::max<size_t>(64ull << 20, bytes);
            CK_CUDA(cudaHostAlloc((void **)&base, cap, cudaHostAllocPortable));
        }
        if (bytes > cap) return fail(CKPT_ENOMEM, "metadata larger than the staging ring");
        if (head + bytes > cap) head = 0;
        const size_t lo = head, hi = head + bytes;
        // wait for in-flight copies that still read [lo, hi)
        for (auto it = live.begin(); it != live.end();) {
            if (it->lo < hi && lo < it->hi) {
                CK_CUDA(cudaEventSynchronize(it->ev));
                cudaEventDestroy(it->ev);
                it = live.erase(it);
            } else if (cudaEventQuery(it->ev) == cudaSuccess) {
                cudaEventDestroy(it->ev);
                it = live.erase(it);
            } else {
                ++it;
            }
        }
        std::memcpy(base + lo, src, n_copy);
        CK_CUDA(cudaMemcpyAsync(dst_dev, base + lo, n_copy, cudaMemcpyHostToDevice, s));
        cudaEvent_t ev;
        CK_CUDA(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        CK_CUDA(cudaEventRecord(ev, s));
        live.push_back({lo, hi, ev});
        head = hi;
        return CKPT_OK;
    }
};
static PinnedRing g_ring;

// ---------------------------------------------------------------------------
// tree
// ---------------------------------------------------------------------------
struct ckpt_tree {
    int device = 0;
    cudaStream_t stream = nullptr;
    ckpt_dtype dtype = CKPT_F32;
    uint32_t chunk_bytes = 0;
    double eps = 0.0;
    uint32_t hash_block = 16;              // bytes per chained Murmur3F call, <= chunk_bytes (R23)
    bool from_digests = false;
    uint32_t n_arrays = 0;
    uint32_t n_levels = 0;                 // max height
    std::vector<uint64_t> n_elems;         // per array
    std::vector<uint64_t> n_leaves;        // per array
    std::vector<uint32_t> height;          // per array
    std::vector<uint64_t> off, cnt;        // [l * n_arrays + a]
    std::vector<uint64_t> level_base, level_total;
    std::vector<uint64_t> chunk_base;      // per array
    uint64_t total_leaves = 0;
    uint64_t array_nodes = 0;              // nodes of all array levels
    uint64_t top_off = 0, top_nodes = 0;
    uint4 *nodes = nullptr;                // device
    uint8_t *meta = nullptr;               // device metadata blob
    // device views into meta
    const uint64_t *d_off = nullptr, *d_cnt = nullptr, *d_level_base = nullptr,
                   *d_level_total = nullptr, *d_chunk_base = nullptr;
    const uint32_t *d_height = nullptr;
    const uint64_t *d_gbegin = nullptr;
    uint64_t n_groups = 0;
    cudaEvent_t levels_done = nullptr;     // recorded after K2 (on the side stream)
    std::vector<uint64_t> meta_host;       // the device blob's contents (8-byte words)
    uint32_t o_off = 0, o_cnt = 0, o_lb = 0, o_lt = 0, o_cb = 0, o_h = 0, o_g = 0;
};

// Work that reads a tree's interior levels or roots waits for K2 first (K2
// runs on a side stream so it overlaps the leaf-only diff and the verify).
static ckpt_status wait_levels(const ckpt_tree *t, cudaStream_t s) {
    if (t && t->levels_done) CK_CUDA(cudaStreamWaitEvent(s, t->levels_done, 0));
    return CKPT_OK;
}

static uint32_t tree_height(uint64_t L) {
    uint32_t h = 1;
    while (L > 1) { L = (L + 1) / 2; ++h; }
    return h;
}

// Lay out an array-level tree over per-array leaf counts.
static void layout(ckpt_tree *t, const std::vector<uint64_t> &leaves) {
    const uint32_t na = (uint32_t)leaves.size();
    t->n_arrays = na;
    t->n_leaves = leaves;
    t->height.resize(na);
    t->n_levels = 1;
    for (uint32_t a = 0; a < na; ++a) {
        t->height[a] = tree_height(leaves[a]);
        t->n_levels = std::max(t->n_levels, t->height[a]);
    }
    const uint32_t nl = t->n_levels;
    t->off.assign((size_t)nl * na, 0);
    t->cnt.assign((size_t)nl * na, 0);
    t->level_base.assign(nl + 1, 0);
    t->level_total.assign(nl + 1, 0);
    uint64_t pos = 0;
    for (uint32_t l = 0; l < nl; ++l) {
        t->level_base[l] = pos;
        for (uint32_t a = 0; a < na; ++a) {
            uint64_t c = 0;
            if (l < t->height[a]) {
                c = leaves[a];
                for (uint32_t k = 0; k < l; ++k) c = (c + 1) / 2;
            }
            t->off[(size_t)l * na + a] = pos;
            t->cnt[(size_t)l * na + a] = c;
            pos += c;
        }
        t->level_total[l] = pos - t->level_base[l];
    }
    t->array_nodes = pos;
    t->level_base[nl] = pos;
    t->chunk_base.resize(na);
    uint64_t cb = 0;
    for (uint32_t a = 0; a < na; ++a) { t->chunk_base[a] = cb; cb += leaves[a]; }
    t->total_leaves = cb;
    t->top_off = pos;
    uint64_t tn = 0, n = na;
    for (;;) { tn += n; if (n == 1) break; n = (n + 1) / 2; }
    t->top_nodes = tn;
}

static size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

static bool quant_params(double eps, QuantParams *q) {
    if (!(eps >= 0.0) || std::isinf(eps)) return false;
    std::memset(q, 0, sizeof(*q));
    q->m1 = 0x52dce729ull;
    q->m2 = 0x38495ab5ull;
    if (eps == 0.0) return true;
    const double inv = 1.0 / eps;
    if (!std::isfinite(inv)) return false;
    q->inv = inv;
    int ex;
    const double fr = std::frexp(inv, &ex);            // inv = fr * 2^ex, fr in [0.5,1)
    q->inv_m = (uint64_t)std::ldexp(fr, 53);           // exact 53-bit integer
    q->inv_e = ex - 53;
    q->r64 = std::ldexp(1.0, 50) / inv;                // |x| < r64 => |x*inv| < 2^51
    float r32;
    if (q->r64 >= (double)FLT_MAX) {
        r32 = INFINITY;
    } else {
        r32 = (float)q->r64;
        if ((double)r32 > q->r64) r32 = std::nextafterf(r32, 0.0f);
    }
    q->r32 = r32;
    return true;
}

static ckpt_status check_common(ckpt_dtype dtype, uint32_t chunk_bytes, double eps) {
    if (dtype != CKPT_F32 && dtype != CKPT_F64) return fail(CKPT_EINVAL, "unknown dtype");
    if (chunk_bytes == 0 || chunk_bytes % 16 != 0)
        return fail(CKPT_EINVAL, "chunk_bytes must be a positive multiple of 16");
    QuantParams q;
    if (!quant_params(eps, &q)) return fail(CKPT_EINVAL, "eps must be finite, >= 0, with 1/eps finite");
    return CKPT_OK;
}

// Hash block size (R23): a positive multiple of 16, or 0 = the whole chunk;
// sizes >= chunk_bytes are the whole chunk.  Returns the effective size.
static ckpt_status norm_block(uint32_t hb, uint32_t C, uint32_t *out) {
    if (hb % 16 != 0) return fail(CKPT_EINVAL, "hash_block must be a multiple of 16 (0 = whole chunk)");
    *out = (hb == 0 || hb > C) ? C : hb;
    return CKPT_OK;
}

template <int DT, bool RAW, int CB, bool PAIR, bool WIDE = false>
static ckpt_status launch_leaf_t(const LeafParams &P, cudaStream_t s, int sms) {
    const uint64_t tasks = P.n_tasks;
    // f32 pair mode below 32 KB chunks: the 72-register kernel (leaf.cuh, leaf_pair_kernel)
    bool capped = false;
    auto k = leaf_kernel<DT, RAW, CB, PAIR, WIDE>;
    if constexpr (PAIR && DT == 0 && CB < (int)kLeafPairMaxChunk) {
        if (P.chunk < kLeafPairMaxChunk) {
            capped = true;
            k = leaf_pair_kernel<DT, RAW, CB, WIDE>;
        }
    }
    static std::atomic<int> cached_per_sm[2] = {{0}, {0}};
    std::atomic<int> &cached = cached_per_sm[capped ? 1 : 0];
    int per_sm = cached.load(std::memory_order_relaxed);
    if (per_sm == 0) {
        CK_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kLeafSmem));
        CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kLeafWarps * 32, kLeafSmem));
        per_sm = std::max(per_sm, 1);
        cached.store(per_sm, std::memory_order_relaxed);
    } else {
        CK_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kLeafSmem));
    }
    // Few tasks (fewer 32-chunk tasks than resident warps, e.g. large chunks): one-warp CTAs, one
    // per task, so the block scheduler spreads the chains evenly over the SMs (8-warp CTAs
    // would put 16 warps on some SMs and 8 on others, and the loaded SMs set the time).
    const uint64_t resident = (uint64_t)sms * per_sm * kLeafWarps;
    const bool few = tasks < resident;
    const unsigned cta_warps = few ? 1u : (unsigned)kLeafWarps;
    const size_t smem = (size_t)cta_warps * kWarpSmem + 16;
    uint64_t want = (tasks + cta_warps - 1) / cta_warps;
    uint64_t grid = few ? want : std::min<uint64_t>(want, (uint64_t)sms * per_sm);
    ProfScope prof(0, s);
    CK_CUDA(launch_k(k, dim3((unsigned)grid), dim3(cta_warps * 32), smem, s, P));
    CK_LAUNCH();
    return CKPT_OK;
}

template <int DT, bool RAW>
static ckpt_status launch_leaf_dt(const LeafParams &P, cudaStream_t s, int sms, bool pair) {
    const uint32_t C = P.chunk;
    if (P.hb16 != 1) {   // wide hash blocks (R23): the bench chunk size specialised, others generic
        if (pair) {
            if (C == 4096) return launch_leaf_t<DT, RAW, 4096, true, true>(P, s, sms);
            return launch_leaf_t<DT, RAW, 0, true, true>(P, s, sms);
        }
        if (C == 4096) return launch_leaf_t<DT, RAW, 4096, false, true>(P, s, sms);
        return launch_leaf_t<DT, RAW, 0, false, true>(P, s, sms);
    }
    if (pair) {   // fused pair mode: the configs[2] sweep's chunk sizes specialised, others generic
        if constexpr (!RAW) {
            switch (C) {
                case 512: return launch_leaf_t<DT, RAW, 512, true>(P, s, sms);
                case 1024: return launch_leaf_t<DT, RAW, 1024, true>(P, s, sms);
                case 2048: return launch_leaf_t<DT, RAW, 2048, true>(P, s, sms);
                case 4096: return launch_leaf_t<DT, RAW, 4096, true>(P, s, sms);
                case 8192: return launch_leaf_t<DT, RAW, 8192, true>(P, s, sms);
                case 16384: return launch_leaf_t<DT, RAW, 16384, true>(P, s, sms);
                case 32768: return launch_leaf_t<DT, RAW, 32768, true>(P, s, sms);
                case 65536: return launch_leaf_t<DT, RAW, 65536, true>(P, s, sms);
                default: break;
            }
        }
        return launch_leaf_t<DT, RAW, 0, true>(P, s, sms);
    }
    if (!RAW) {
        switch (C) {
            case 512: return launch_leaf_t<DT, RAW, 512, false>(P, s, sms);
            case 1024: return launch_leaf_t<DT, RAW, 1024, false>(P, s, sms);
            case 2048: return launch_leaf_t<DT, RAW, 2048, false>(P, s, sms);
            case 4096: return launch_leaf_t<DT, RAW, 4096, false>(P, s, sms);
            case 8192: return launch_leaf_t<DT, RAW, 8192, false>(P, s, sms);
            case 16384: return launch_leaf_t<DT, RAW, 16384, false>(P, s, sms);
            case 32768: return launch_leaf_t<DT, RAW, 32768, false>(P, s, sms);
            case 65536: return launch_leaf_t<DT, RAW, 65536, false>(P, s, sms);
            default: break;
        }
    }
    return launch_leaf_t<DT, RAW, 0, false>(P, s, sms);
}

// K2 for up to kMaxLevelTrees trees in one launch.
static ckpt_status get_scratch(int dev, cudaStream_t s, size_t n_states, uint64_t **states,
                               unsigned long long **ticket, uint32_t *epoch);

static ckpt_status launch_levels(ckpt_tree *const *trees, int n, cudaStream_t s) {
    static std::atomic<int> attr_done{0};
    if (!attr_done.load()) {
        CK_CUDA(cudaFuncSetAttribute(levels_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kLevelSmem));
        attr_done.store(1);
    }
    int dev = 0;
    CK_CUDA(cudaGetDevice(&dev));
    uint64_t *unused_states;
    unsigned long long *tickets;
    uint32_t unused_epoch;
    CK_TRY(get_scratch(dev, s, 0, &unused_states, &tickets, &unused_epoch));
    static LevelBatch b;                      // large (kernel parameters); filled per launch
    static std::mutex b_mu;
    std::lock_guard<std::mutex> lk(b_mu);
    for (int k0 = 0; k0 < n; k0 += kMaxLevelTrees) {
        std::memset(&b, 0, offsetof(LevelBatch, blob));
        b.n = std::min(kMaxLevelTrees, n - k0);
        unsigned ctas = 0;
        uint32_t words = 0;
        for (int i = 0; i < b.n; ++i) {
            ckpt_tree *t = trees[k0 + i];
            LevelParams &p = b.t[i];
            p.nodes = t->nodes;
            p.meta = t->meta;
            p.meta_words = (uint32_t)t->meta_host.size();
            if (words + p.meta_words <= (uint32_t)kLevelInlineWords) {
                std::memcpy(b.blob + words, t->meta_host.data(), (size_t)p.meta_words * 8);
                p.inl = (int)words;
                words += p.meta_words;
            } else {
                p.inl = -1;
                CK_TRY(g_ring.copy(t->meta, t->meta_host.data(), t->meta_host.size() * 8, s));
            }
            p.o_off = t->o_off;
            p.o_cnt = t->o_cnt;
            p.o_lb = t->o_lb;
            p.o_lt = t->o_lt;
            p.o_h = t->o_h;
            p.o_g = t->o_g;
            p.top_off = t->top_off;
            p.ticket = reinterpret_cast<unsigned int *>(tickets + 1 + i);   // slot 0: compactions
            p.n_arrays = (int)t->n_arrays;
            p.n_levels = (int)t->n_levels;
            p.ls = 0;
            p.n_groups = (unsigned)t->n_groups;
            b.cta_begin[i] = ctas;
            ctas += (unsigned)t->n_groups;
        }
        b.cta_begin[b.n] = ctas;
        ProfScope prof(1, s);
        CK_CUDA(launch_k(levels_kernel, dim3(ctas), dim3(kLevelThreads), kLevelSmem, s, b));
        CK_LAUNCH();
    }
    return CKPT_OK;
}

// Allocate a laid-out tree's node storage and device metadata blob:
// [off][cnt][level_base][level_total][chunk_base][height][gbegin][ticket]
static ckpt_status prepare_tree(ckpt_tree *t, cudaStream_t s) {
    const uint32_t na = t->n_arrays;
    std::vector<uint64_t> gbegin(na);
    uint64_t groups = 0;
    for (uint32_t a = 0; a < na; ++a) {
        gbegin[a] = groups;
        groups += (t->cnt[a] + kGroup - 1) / kGroup;   // level 0 counts
    }
    t->n_groups = groups;
    auto al8 = [](size_t x) { return (x + 7) & ~size_t(7); };
    size_t o = 0;
    t->o_off = (uint32_t)o; o = al8(o + t->off.size() * 8);
    t->o_cnt = (uint32_t)o; o = al8(o + t->cnt.size() * 8);
    t->o_lb = (uint32_t)o;  o = al8(o + t->level_base.size() * 8);
    t->o_lt = (uint32_t)o;  o = al8(o + t->level_total.size() * 8);
    t->o_cb = (uint32_t)o;  o = al8(o + (size_t)na * 8);
    t->o_h = (uint32_t)o;   o = al8(o + (size_t)na * 4);
    t->o_g = (uint32_t)o;   o = al8(o + (size_t)na * 8);
    const size_t total = o;
    t->meta_host.assign(total / 8, 0);
    uint8_t *blob = reinterpret_cast<uint8_t *>(t->meta_host.data());
    std::memcpy(blob + t->o_off, t->off.data(), t->off.size() * 8);
    std::memcpy(blob + t->o_cnt, t->cnt.data(), t->cnt.size() * 8);
    std::memcpy(blob + t->o_lb, t->level_base.data(), t->level_base.size() * 8);
    std::memcpy(blob + t->o_lt, t->level_total.data(), t->level_total.size() * 8);
    std::memcpy(blob + t->o_cb, t->chunk_base.data(), (size_t)na * 8);
    std::memcpy(blob + t->o_h, t->height.data(), (size_t)na * 4);
    std::memcpy(blob + t->o_g, gbegin.data(), (size_t)na * 8);
    CK_CUDA(cudaMallocAsync((void **)&t->nodes, (t->array_nodes + t->top_nodes) * 16, s));
    CK_CUDA(cudaMallocAsync((void **)&t->meta, total, s));
    // the blob reaches `meta` through K2 (inline parameters) or a staging copy there
    t->d_off = (const uint64_t *)(t->meta + t->o_off);
    t->d_cnt = (const uint64_t *)(t->meta + t->o_cnt);
    t->d_level_base = (const uint64_t *)(t->meta + t->o_lb);
    t->d_level_total = (const uint64_t *)(t->meta + t->o_lt);
    t->d_chunk_base = (const uint64_t *)(t->meta + t->o_cb);
    t->d_height = (const uint32_t *)(t->meta + t->o_h);
    t->d_gbegin = (const uint64_t *)(t->meta + t->o_g);
    return CKPT_OK;
}

// One leaf-kernel launch over every array of every tree in `table`.
static ckpt_status launch_leaves(const std::vector<LeafArray> &table, uint64_t tasks,
                                 ckpt_dtype dtype, double eps, uint32_t C, uint32_t hash_block,
                                 cudaStream_t s, int sms, const PairParams *pair,
                                 unsigned long long *ticket) {
    if (!ticket) return fail(CKPT_EINVAL, "leaf launch without a task ticket");
    LeafParams P;
    std::memset(&P, 0, sizeof(P));
    quant_params(eps, &P.q);
    P.hb16 = hash_block / 16;
    if (pair) P.pr = *pair;
    P.ticket = ticket;
    P.n_arrays = (int)table.size();
    P.n_tasks = tasks;
    P.chunk = C;
    LeafArray *d_tab = nullptr;
    if (table.size() <= (size_t)kLeafInline) {
        for (size_t a = 0; a < table.size(); ++a) P.inl[a] = table[a];
    } else {
        const size_t bytes = table.size() * sizeof(LeafArray);
        CK_CUDA(cudaMallocAsync((void **)&d_tab, bytes, s));
        CK_TRY(g_ring.copy(d_tab, table.data(), bytes, s));
        P.arrays = d_tab;
    }
    const bool pm = pair != nullptr;
    if (eps == 0.0) {
        if (dtype == CKPT_F32) CK_TRY((launch_leaf_dt<0, true>(P, s, sms, pm)));
        else CK_TRY((launch_leaf_dt<1, true>(P, s, sms, pm)));
    } else {
        if (dtype == CKPT_F32) CK_TRY((launch_leaf_dt<0, false>(P, s, sms, pm)));
        else CK_TRY((launch_leaf_dt<1, false>(P, s, sms, pm)));
    }
    if (d_tab) CK_CUDA(cudaFreeAsync(d_tab, s));
    return CKPT_OK;
}

struct Scratch {
    uint64_t *states = nullptr;
    size_t cap = 0;
    unsigned long long *ticket = nullptr;
    uint32_t epoch = 0;
    uint8_t *work = nullptr;       // K4 per-chunk counts + hit bitmasks
    size_t work_cap = 0;
    unsigned int *pair_ctr = nullptr;   // fused pair mode: one self-resetting counter per pair-task
    size_t pair_cap = 0;
    uint8_t *pair_flags = nullptr;      // fused pair mode: one flag byte per chunk
    size_t flags_cap = 0;
    uint8_t *tile = nullptr;            // fused pair mode: K1 tile compaction buffers
    size_t tile_pairs = 0;              // pair-tasks the buffers hold
};
static std::mutex g_scr_mu;
static std::map<std::pair<int, cudaStream_t>, Scratch> g_scr;

static ckpt_status get_pair_flags(int dev, cudaStream_t s, size_t n, uint8_t **flags) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    Scratch &sc = g_scr[std::make_pair(dev, s)];
    n = std::max<size_t>(n, 256);
    if (sc.flags_cap < n) {
        if (sc.pair_flags) CK_CUDA(cudaFreeAsync(sc.pair_flags, s));
        sc.flags_cap = std::max<size_t>(n, 2 * sc.flags_cap);
        CK_CUDA(cudaMallocAsync((void **)&sc.pair_flags, sc.flags_cap, s));
    }
    *flags = sc.pair_flags;
    return CKPT_OK;
}

constexpr int kLeafTicketSlot = 16;   // 8-byte slot of the per-stream ticket block used by K1

// CKPT_TILE_GATHER=1: always place the fused path's chunk list with tile_gather_kernel
// (A/B and tests of that path; by default K4a reads the tiles itself).
static bool tile_gather_forced() {
    static const bool on = [] {
        const char *e = std::getenv("CKPT_TILE_GATHER");
        return e && e[0] == '1';
    }();
    return on;
}

// K1 tile-compaction buffers for n_pair pair-tasks (leaf.cuh PairParams):
// [tctr: n_tiles u32, zeroed once; self-resetting] [tagg: n_tiles u32]
// [tmask: n_pair u32] [tbase: n_pair u64] [tids: n_tiles * kTileTasks * 32 u64]
static ckpt_status get_tile_scratch(int dev, cudaStream_t s, uint64_t n_pair, PairParams *pp) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    Scratch &sc = g_scr[std::make_pair(dev, s)];
    n_pair = std::max<uint64_t>(n_pair, 1);
    auto layout_of = [](uint64_t np, size_t o[5]) {
        const uint64_t nt = (np + kTileTasks - 1) / kTileTasks;
        o[0] = 0;
        o[1] = align256(nt * 4);
        o[2] = o[1] + align256(nt * 4);
        o[3] = o[2] + align256(np * 4);
        o[4] = o[3] + align256(np * 8);
        return o[4] + nt * kTileTasks * 32 * 8;
    };
    size_t o[5];
    if (sc.tile_pairs < n_pair) {
        if (sc.tile) CK_CUDA(cudaFreeAsync(sc.tile, s));
        sc.tile_pairs = std::max<uint64_t>(n_pair, 2 * sc.tile_pairs);
        const size_t bytes = layout_of(sc.tile_pairs, o);
        CK_CUDA(cudaMallocAsync((void **)&sc.tile, bytes, s));
        CK_CUDA(cudaMemsetAsync(sc.tile, 0, o[1], s));      // tile counters
    }
    layout_of(sc.tile_pairs, o);
    pp->tctr = (unsigned int *)(sc.tile + o[0]);
    pp->tagg = (uint32_t *)(sc.tile + o[1]);
    pp->tmask = (uint32_t *)(sc.tile + o[2]);
    pp->tbase = (uint64_t *)(sc.tile + o[3]);
    pp->tids = (uint64_t *)(sc.tile + o[4]);
    return CKPT_OK;
}

// Zero-initialised pair-task counters (they return to 0 after every launch).
static ckpt_status get_pair_ctr(int dev, cudaStream_t s, size_t n, unsigned int **ctr) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    Scratch &sc = g_scr[std::make_pair(dev, s)];
    n = std::max<size_t>(n, 1);
    if (sc.pair_cap < n) {
        if (sc.pair_ctr) CK_CUDA(cudaFreeAsync(sc.pair_ctr, s));
        sc.pair_cap = std::max<size_t>(n, 2 * sc.pair_cap);
        CK_CUDA(cudaMallocAsync((void **)&sc.pair_ctr, sc.pair_cap * 4, s));
        CK_CUDA(cudaMemsetAsync(sc.pair_ctr, 0, sc.pair_cap * 4, s));
    }
    *ctr = sc.pair_ctr;
    return CKPT_OK;
}

// Trees of several checkpoints with one leaf-kernel launch.  `pair` != NULL:
// fused pair mode (two checkpoints of identical shape; see PairParams).
static ckpt_status build_batch_impl(const void *const *data, const uint64_t *n,
                                    const uint32_t *arrays_per_tree, uint32_t n_trees,
                                    ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                    uint32_t hash_block, void *stream, ckpt_tree **out,
                                    const PairParams *pair) {
    if (!out || n_trees == 0 || !arrays_per_tree) return fail(CKPT_EINVAL, "no trees / NULL out");
    for (uint32_t k = 0; k < n_trees; ++k) out[k] = nullptr;
    if (!data || !n) return fail(CKPT_EINVAL, "no arrays");
    CK_TRY(check_common(dtype, chunk_bytes, eps));
    CK_TRY(norm_block(hash_block, chunk_bytes, &hash_block));
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    uint64_t total_arrays = 0;
    for (uint32_t k = 0; k < n_trees; ++k) {
        if (arrays_per_tree[k] == 0 || arrays_per_tree[k] >= (1u << 20))
            return fail(CKPT_EINVAL, "every tree needs 1 .. 2^20-1 arrays");
        total_arrays += arrays_per_tree[k];
    }
    for (uint64_t a = 0; a < total_arrays; ++a) {
        if (!data[a]) return fail(CKPT_EINVAL, "NULL data pointer");
        if (n[a] == 0) return fail(CKPT_EINVAL, "empty array (n == 0)");
        if ((uintptr_t)data[a] % 16 != 0) return fail(CKPT_EINVAL, "data must be 16-byte aligned");
        if (n[a] > (1ull << 50)) return fail(CKPT_EINVAL, "array too large");
    }
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<LeafArray> table;
    table.reserve(total_arrays);
    uint64_t task = 0, a0 = 0;
    ckpt_status st = CKPT_OK;
    for (uint32_t k = 0; k < n_trees && st == CKPT_OK; ++k) {
        const uint32_t na = arrays_per_tree[k];
        ckpt_tree *t = new ckpt_tree();
        out[k] = t;
        t->device = dev;
        t->stream = s;
        t->dtype = dtype;
        t->chunk_bytes = chunk_bytes;
        t->eps = eps;
        t->hash_block = hash_block;
        t->n_elems.assign(n + a0, n + a0 + na);
        std::vector<uint64_t> leaves(na);
        for (uint32_t a = 0; a < na; ++a) leaves[a] = (n[a0 + a] * esz + chunk_bytes - 1) / chunk_bytes;
        layout(t, leaves);
        st = prepare_tree(t, s);
        for (uint32_t a = 0; a < na && st == CKPT_OK; ++a) {
            LeafArray e;
            e.data = (const uint8_t *)data[a0 + a];
            e.nbytes = n[a0 + a] * esz;
            e.n_leaves = leaves[a];
            e.n_full = e.nbytes / chunk_bytes;
            e.task_begin = task;
            e.out = t->nodes + t->off[a];      // level 0 of array a
            e.chunk_base = t->chunk_base[a];
            table.push_back(e);
            task += (leaves[a] + kRows - 1) / kRows;
        }
        a0 += na;
    }
    PairParams pp;
    unsigned long long *ticket = nullptr;
    if (pair) {
        pp = *pair;
        pp.n_pair = task / 2;                  // A's tasks; B's are the same count
        st = get_pair_ctr(dev, s, pp.n_pair, &pp.ctr);
    }
    if (st == CKPT_OK) {   // in-order dynamic tasks (no tail imbalance)
        uint64_t *unused_states;
        uint32_t unused_epoch;
        st = get_scratch(dev, s, 0, &unused_states, &ticket, &unused_epoch);
        ticket += kLeafTicketSlot;
    }
    if (st == CKPT_OK)
        st = launch_leaves(table, task, dtype, eps, chunk_bytes, hash_block, s, di.sms,
                           pair ? &pp : nullptr, ticket);
    if (st == CKPT_OK) {
        // K2 on the side stream, after the leaves; each tree records its own event
        cudaStream_t ss = nullptr;
        cudaEvent_t leaves_done = nullptr;
        st = side_stream(dev, &ss);
        if (st == CKPT_OK && (cudaEventCreateWithFlags(&leaves_done, cudaEventDisableTiming) != cudaSuccess ||
                              cudaEventRecord(leaves_done, s) != cudaSuccess ||
                              cudaStreamWaitEvent(ss, leaves_done, 0) != cudaSuccess))
            st = fail(CKPT_ECUDA, "side-stream fork");
        if (leaves_done) cudaEventDestroy(leaves_done);
        if (st == CKPT_OK) st = launch_levels(out, (int)n_trees, ss);
        for (uint32_t k = 0; k < n_trees && st == CKPT_OK; ++k) {
            if (cudaEventCreateWithFlags(&out[k]->levels_done, cudaEventDisableTiming) != cudaSuccess ||
                cudaEventRecord(out[k]->levels_done, ss) != cudaSuccess)
                st = fail(CKPT_ECUDA, "side-stream join event");
        }
    }
    if (st != CKPT_OK) {
        for (uint32_t k = 0; k < n_trees; ++k) { ckpt_tree_free_on(out[k], stream); out[k] = nullptr; }
        return st;
    }
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_build_batch(const void *const *data, const uint64_t *n,
                                             const uint32_t *arrays_per_tree, uint32_t n_trees,
                                             ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                             void *stream, ckpt_tree **out) {
    return build_batch_impl(data, n, arrays_per_tree, n_trees, dtype, chunk_bytes, eps, 16, stream,
                            out, nullptr);
}

extern "C" ckpt_status ckpt_tree_build_batch_ex(const void *const *data, const uint64_t *n,
                                                const uint32_t *arrays_per_tree, uint32_t n_trees,
                                                ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                                uint32_t hash_block, void *stream, ckpt_tree **out) {
    return build_batch_impl(data, n, arrays_per_tree, n_trees, dtype, chunk_bytes, eps, hash_block,
                            stream, out, nullptr);
}

extern "C" ckpt_status ckpt_tree_build_arrays(const void *const *data, const uint64_t *n,
                                              uint32_t n_arrays, ckpt_dtype dtype,
                                              uint32_t chunk_bytes, double eps, void *stream,
                                              ckpt_tree **out) {
    if (!out) return fail(CKPT_EINVAL, "out is NULL");
    *out = nullptr;
    if (n_arrays == 0) return fail(CKPT_EINVAL, "no arrays");
    return ckpt_tree_build_batch(data, n, &n_arrays, 1, dtype, chunk_bytes, eps, stream, out);
}

extern "C" ckpt_status ckpt_tree_build(const void *data, uint64_t n, ckpt_dtype dtype,
                                       uint32_t chunk_bytes, double eps, void *stream,
                                       ckpt_tree **out) {
    const void *d[1] = {data};
    uint64_t nn[1] = {n};
    return ckpt_tree_build_arrays(d, nn, 1, dtype, chunk_bytes, eps, stream, out);
}

extern "C" ckpt_status ckpt_tree_from_digests(const void *digests16, uint64_t count, void *stream,
                                              ckpt_tree **out) {
    if (!out) return fail(CKPT_EINVAL, "out is NULL");
    *out = nullptr;
    if (!digests16 || count == 0) return fail(CKPT_EINVAL, "no digests");
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    ckpt_tree *t = new ckpt_tree();
    t->device = dev;
    t->stream = s;
    t->from_digests = true;
    t->chunk_bytes = 16;
    t->n_elems.assign(1, count);
    layout(t, std::vector<uint64_t>{count});
    ckpt_status st = prepare_tree(t, s);
    if (st == CKPT_OK && cudaMemcpyAsync(t->nodes, digests16, count * 16, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        st = fail(CKPT_ECUDA, "digest copy");
    if (st == CKPT_OK) st = launch_levels(&t, 1, s);
    if (st != CKPT_OK) { ckpt_tree_free_on(t, stream); return st; }
    *out = t;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_from_digests_batch(const void *digests16, const uint64_t *counts,
                                                    uint32_t n_trees, void *stream, ckpt_tree **out) {
    if (!out) return fail(CKPT_EINVAL, "out is NULL");
    for (uint32_t k = 0; k < n_trees; ++k) out[k] = nullptr;
    if (!digests16 || !counts || n_trees == 0) return fail(CKPT_EINVAL, "no digests");
    for (uint32_t k = 0; k < n_trees; ++k)
        if (counts[k] == 0) return fail(CKPT_EINVAL, "empty digest list");
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    ckpt_status st = CKPT_OK;
    const uint8_t *src = (const uint8_t *)digests16;
    for (uint32_t k = 0; k < n_trees && st == CKPT_OK; ++k) {
        ckpt_tree *t = new ckpt_tree();
        out[k] = t;
        t->device = dev;
        t->stream = s;
        t->from_digests = true;
        t->chunk_bytes = 16;
        t->n_elems.assign(1, counts[k]);
        layout(t, std::vector<uint64_t>{counts[k]});
        st = prepare_tree(t, s);
        if (st == CKPT_OK && cudaMemcpyAsync(t->nodes, src, counts[k] * 16, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
            st = fail(CKPT_ECUDA, "digest copy");
        src += counts[k] * 16;
    }
    if (st == CKPT_OK) st = launch_levels(out, (int)n_trees, s);
    if (st != CKPT_OK) {
        for (uint32_t k = 0; k < n_trees; ++k) { ckpt_tree_free_on(out[k], stream); out[k] = nullptr; }
        return st;
    }
    return CKPT_OK;
}

extern "C" void ckpt_tree_free_on(ckpt_tree *t, void *stream) {
    if (!t) return;
    cudaStream_t s = (cudaStream_t)stream;
    int cur = 0;
    cudaGetDevice(&cur);
    if (cur != t->device) cudaSetDevice(t->device);
    if (t->levels_done) {
        cudaStreamWaitEvent(s, t->levels_done, 0);
        cudaEventDestroy(t->levels_done);
    }
    if (t->nodes) cudaFreeAsync(t->nodes, s);
    if (t->meta) cudaFreeAsync(t->meta, s);
    if (cur != t->device) cudaSetDevice(cur);
    delete t;
}

extern "C" void ckpt_tree_free(ckpt_tree *t) {
    if (!t) return;
    ckpt_tree_free_on(t, t->stream);
}

// ---------------------------------------------------------------------------
// stage 1: diff (K3)
// ---------------------------------------------------------------------------
static ckpt_status check_pair(const ckpt_tree *a, const ckpt_tree *b) {
    if (!a || !b) return fail(CKPT_EINVAL, "NULL tree");
    if (a->from_digests || b->from_digests)
        return fail(CKPT_EINVAL, "trees built from digests cannot be diffed");
    if (a->dtype != b->dtype || a->chunk_bytes != b->chunk_bytes ||
        std::memcmp(&a->eps, &b->eps, sizeof(double)) != 0 || a->n_arrays != b->n_arrays ||
        a->n_elems != b->n_elems || a->hash_block != b->hash_block)
        return fail(CKPT_EMISMATCH,
                    "trees differ in dtype, chunk_bytes, eps, hash_block or array shapes");
    if (a->device != b->device) return fail(CKPT_EMISMATCH, "trees live on different devices");
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// per-(device, stream) scratch for the ordered compactions: look-back states
// tagged with a launch epoch (never cleared) and a self-resetting ticket.
// ---------------------------------------------------------------------------

static ckpt_status get_scratch(int dev, cudaStream_t s, size_t n_states, uint64_t **states,
                               unsigned long long **ticket, uint32_t *epoch) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    Scratch &sc = g_scr[std::make_pair(dev, s)];
    if (!sc.ticket) {
        CK_CUDA(cudaMallocAsync((void **)&sc.ticket, 256, s));
        CK_CUDA(cudaMemsetAsync(sc.ticket, 0, 256, s));
    }
    n_states = std::max<size_t>(n_states, 1);
    bool cleared = false;
    if (sc.cap < n_states) {
        if (sc.states) CK_CUDA(cudaFreeAsync(sc.states, s));
        sc.cap = std::max<size_t>(n_states, std::max<size_t>(2 * sc.cap, 4096));
        CK_CUDA(cudaMallocAsync((void **)&sc.states, sc.cap * 8, s));
        CK_CUDA(cudaMemsetAsync(sc.states, 0, sc.cap * 8, s));
        cleared = true;
    }
    if (++sc.epoch >= (1u << 24)) {                  // epoch wrap: clear once, restart at 1
        if (!cleared) CK_CUDA(cudaMemsetAsync(sc.states, 0, sc.cap * 8, s));
        sc.epoch = 1;
    }
    *states = sc.states;
    *ticket = sc.ticket;
    *epoch = sc.epoch;
    return CKPT_OK;
}

// Free every scratch buffer of (dev, s) on s and forget the entry: called before a
// stream the library created for one call (compare_host / compare_stream) is
// destroyed, so per-call streams do not leave scratch allocations behind.
static void release_scratch(int dev, cudaStream_t s) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    auto it = g_scr.find(std::make_pair(dev, s));
    if (it == g_scr.end()) return;
    Scratch &sc = it->second;
    void *bufs[] = {sc.states, sc.ticket, sc.work, sc.pair_ctr, sc.pair_flags, sc.tile};
    for (void *b : bufs)
        if (b) cudaFreeAsync(b, s);
    g_scr.erase(it);
}

// Stream-ordered work buffer of at least `bytes` (grows, never shrinks).
static ckpt_status get_work(int dev, cudaStream_t s, size_t bytes, uint8_t **work) {
    std::lock_guard<std::mutex> lk(g_scr_mu);
    Scratch &sc = g_scr[std::make_pair(dev, s)];
    bytes = std::max<size_t>(bytes, 256);
    if (sc.work_cap < bytes) {
        if (sc.work) CK_CUDA(cudaFreeAsync(sc.work, s));
        sc.work_cap = std::max<size_t>(bytes, std::min<size_t>(2 * sc.work_cap, bytes + (64u << 20)));
        CK_CUDA(cudaMallocAsync((void **)&sc.work, sc.work_cap, s));
    }
    *work = sc.work;
    return CKPT_OK;
}

static ckpt_status launch_compact(int mode, const uint4 *la, const uint4 *lb, const uint8_t *flags,
                                  uint64_t n, uint64_t *out, uint64_t cap, uint64_t *count,
                                  cudaStream_t s, int sms, uint64_t base = 0) {
    const uint64_t tile = mode == 0 ? compact_tile<0>() : compact_tile<1>();
    const uint64_t n_tiles = (n + tile - 1) / tile;
    int dev = 0;
    CK_CUDA(cudaGetDevice(&dev));
    CompactParams p;
    CK_TRY(get_scratch(dev, s, n_tiles, &p.states, &p.ticket, &p.epoch));
    p.leaf_a = la;
    p.leaf_b = lb;
    p.flags = flags;
    p.n = n;
    p.out = out;
    p.cap = cap;
    p.count = count;
    p.base = base;
    // co-resident grid (the look-back relies on it); static tile striding
    static std::atomic<int> occ0{0}, occ1{0};
    std::atomic<int> &occ = mode == 0 ? occ0 : occ1;
    int per_sm = occ.load();
    if (per_sm == 0) {
        if (mode == 0) CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, compact_kernel<0>, kCompactThreads, 0));
        else CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, compact_kernel<1>, kCompactThreads, 0));
        per_sm = std::max(per_sm, 1);
        occ.store(per_sm);
    }
    const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(n_tiles, (uint64_t)sms * per_sm));
    ProfScope prof(2, s);
    CK_CUDA(launch_k(mode == 0 ? compact_kernel<0> : compact_kernel<1>, dim3(grid), dim3(kCompactThreads), 0, s, p));
    CK_LAUNCH();
    return CKPT_OK;
}

// BFS start level (R16): the level closest to the root whose node count over
// all arrays is >= T (0 = the leaves).
static uint32_t start_level(const ckpt_tree *a, uint64_t T) {
    const uint32_t na = a->n_arrays;
    for (int l = (int)a->n_levels - 1; l >= 0; --l) {
        uint64_t tot = 0;
        for (uint32_t k = 0; k < na; ++k) {
            const uint32_t ll = std::min<uint32_t>((uint32_t)l, a->height[k] - 1);
            tot += a->cnt[(size_t)ll * na + k];
        }
        if (tot >= T) return (uint32_t)l;
    }
    return 0;
}

extern "C" ckpt_status ckpt_tree_diff_async(const ckpt_tree *a, const ckpt_tree *b, uint64_t T,
                                            uint64_t *chunks, uint64_t cap, uint64_t *n_chunks_dev,
                                            void *stream) {
    CK_TRY(check_pair(a, b));
    if (!n_chunks_dev || (!chunks && cap)) return fail(CKPT_EINVAL, "NULL output");
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    if (T == 0) T = (uint64_t)di.sms * (uint64_t)di.max_threads_sm;
    const uint32_t na = a->n_arrays;
    const uint32_t l0 = start_level(a, T);
    if (l0 > 0) {
        CK_TRY(wait_levels(a, s));
        CK_TRY(wait_levels(b, s));
    }
    if (l0 == 0) {
        return launch_compact(0, a->nodes, b->nodes, nullptr, a->total_leaves, chunks, cap,
                              n_chunks_dev, s, di.sms);
    }
    // BFS from l0: frontier of (array, level, node) entries
    std::vector<uint64_t> sbegin(na);
    std::vector<uint32_t> slevel(na);
    uint64_t n_start = 0;
    for (uint32_t k = 0; k < na; ++k) {
        slevel[k] = std::min<uint32_t>(l0, a->height[k] - 1);
        sbegin[k] = n_start;
        n_start += a->cnt[(size_t)slevel[k] * na + k];
    }
    const uint64_t L = a->total_leaves;
    const size_t o_sb = 0;
    const size_t o_sl = align256(o_sb + (size_t)na * 8);
    const size_t o_cnt = align256(o_sl + (size_t)na * 4);
    const size_t o_flags = align256(o_cnt + (size_t)(l0 + 2) * 8);
    const size_t o_f0 = align256(o_flags + L);
    const size_t o_f1 = align256(o_f0 + L * 8);
    const size_t total = align256(o_f1 + L * 8);
    uint8_t *scr = nullptr;
    CK_CUDA(cudaMallocAsync((void **)&scr, total, s));
    std::vector<uint8_t> tbl(o_cnt, 0);
    std::memcpy(tbl.data() + o_sb, sbegin.data(), (size_t)na * 8);
    std::memcpy(tbl.data() + o_sl, slevel.data(), (size_t)na * 4);
    CK_TRY(g_ring.copy(scr, tbl.data(), tbl.size(), s));
    CK_CUDA(cudaMemsetAsync(scr + o_cnt, 0, o_f0 - o_cnt, s));   // counters + flags
    BfsParams p;
    p.na = a->nodes;
    p.nb = b->nodes;
    p.off = a->d_off;
    p.cnt = a->d_cnt;
    p.chunk_base = a->d_chunk_base;
    p.sbegin = (const uint64_t *)(scr + o_sb);
    p.slevel = (const uint32_t *)(scr + o_sl);
    p.n_start = n_start;
    p.n_arrays = (int)na;
    p.flags = scr + o_flags;
    unsigned long long *cnts = (unsigned long long *)(scr + o_cnt);
    uint64_t *fr[2] = {(uint64_t *)(scr + o_f0), (uint64_t *)(scr + o_f1)};
    const unsigned grid_first = (unsigned)std::min<uint64_t>((n_start + 255) / 256, (uint64_t)di.sms * 8);
    {
        ProfScope prof(2, s);
        CK_CUDA(launch_k(bfs_first_kernel, dim3(grid_first), dim3(256), 0, s, p, fr[0], cnts));
    }
    CK_LAUNCH();
    for (uint32_t step = 1; step <= l0; ++step) {
        ProfScope prof(2, s);
        CK_CUDA(launch_k(bfs_step_kernel, dim3((unsigned)di.sms * 8), dim3(256), 0, s, p,
                         (const uint64_t *)fr[(step - 1) & 1], (const unsigned long long *)(cnts + step - 1),
                         fr[step & 1], cnts + step));
        CK_LAUNCH();
    }
    CK_TRY(launch_compact(1, nullptr, nullptr, scr + o_flags, L, chunks, cap, n_chunks_dev, s, di.sms));
    CK_CUDA(cudaFreeAsync(scr, s));
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_diff(const ckpt_tree *a, const ckpt_tree *b, uint64_t *chunks,
                                      uint64_t cap, uint64_t *n_chunks, void *stream) {
    if (!n_chunks) return fail(CKPT_EINVAL, "n_chunks is NULL");
    cudaStream_t s = (cudaStream_t)stream;
    uint64_t *dcount = nullptr;
    CK_TRY(check_pair(a, b));
    CK_CUDA(cudaMallocAsync((void **)&dcount, 8, s));
    ckpt_status st = ckpt_tree_diff_async(a, b, 0, chunks, cap, dcount, stream);
    if (st == CKPT_OK) {
        CK_CUDA(cudaMemcpyAsync(n_chunks, dcount, 8, cudaMemcpyDeviceToHost, s));
        CK_CUDA(cudaFreeAsync(dcount, s));
        CK_CUDA(cudaStreamSynchronize(s));
        if (*n_chunks > cap) return fail(CKPT_ETRUNC, "chunk list longer than cap");
        return CKPT_OK;
    }
    cudaFreeAsync(dcount, s);
    return st;
}

// ---------------------------------------------------------------------------
// stage 2: verify (K4)
// ---------------------------------------------------------------------------
// before_emit (optional): called after the scan kernel (the full count is in
// *n_diff_dev once the stream reaches that point) and before the emit kernel;
// it may replace the output buffer and its capacity (exact-size outputs).
using EmitHook = std::function<ckpt_status(uint64_t **idx, uint64_t *cap)>;

static ckpt_status verify_impl(const void *const *a, const void *const *b, const uint64_t *n,
                               uint32_t na, ckpt_dtype dtype, uint32_t chunk_bytes,
                               const uint64_t *chunks, const uint64_t *n_chunks_dev,
                               uint64_t n_chunks_host, uint64_t chunks_cap, double eps,
                               uint64_t *idx, uint64_t cap, uint64_t *n_diff_dev, cudaStream_t s,
                               const EmitHook &before_emit = nullptr, uint64_t chunk_base0 = 0,
                               uint64_t elem_base0 = 0, const PairParams *tiles = nullptr) {
    if (!a || !b || !n || na == 0) return fail(CKPT_EINVAL, "no arrays");
    if (!n_diff_dev || (!idx && cap && !before_emit)) return fail(CKPT_EINVAL, "NULL output");
    CK_TRY(check_common(dtype, chunk_bytes, eps));
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    std::vector<VerifyArray> va(na);
    std::vector<uint64_t> cb(na);
    uint64_t c = chunk_base0, e = elem_base0;   // global ids of the first array's chunk / element 0
    for (uint32_t k = 0; k < na; ++k) {
        if (!a[k] || !b[k]) return fail(CKPT_EINVAL, "NULL data pointer");
        if ((uintptr_t)a[k] % 16 || (uintptr_t)b[k] % 16)
            return fail(CKPT_EINVAL, "data must be 16-byte aligned");
        if (n[k] == 0) return fail(CKPT_EINVAL, "empty array (n == 0)");
        va[k].a = (const uint8_t *)a[k];
        va[k].b = (const uint8_t *)b[k];
        va[k].n = n[k];
        va[k].chunk_base = c;
        va[k].elem_base = e;
        cb[k] = c;
        c += (n[k] * esz + chunk_bytes - 1) / chunk_bytes;
        e += n[k];
    }
    if (chunks_cap && !chunks) return fail(CKPT_EINVAL, "NULL chunk list");
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    const uint64_t max_chunks = std::min<uint64_t>(chunks_cap, c - chunk_base0);
    VerifyParams p;
    std::memset(&p, 0, sizeof(p));
    uint8_t *tab = nullptr;
    if (na <= (uint32_t)kVerifyInline) {
        // small array tables ride in the kernel parameters: no copy, no allocation
        for (uint32_t k = 0; k < na; ++k) { p.inl[k] = va[k]; p.inl_base[k] = cb[k]; }
    } else {
        const size_t o_cb = align256((size_t)na * sizeof(VerifyArray));
        std::vector<uint8_t> tbl(o_cb + (size_t)na * 8, 0);
        std::memcpy(tbl.data(), va.data(), (size_t)na * sizeof(VerifyArray));
        std::memcpy(tbl.data() + o_cb, cb.data(), (size_t)na * 8);
        CK_CUDA(cudaMallocAsync((void **)&tab, tbl.size(), s));
        CK_TRY(g_ring.copy(tab, tbl.data(), tbl.size(), s));
        p.arrays = (const VerifyArray *)tab;
        p.chunk_base = (const uint64_t *)(tab + o_cb);
    }
    p.n_arrays = (int)na;
    p.chunks = chunks;
    p.n_chunks_dev = n_chunks_dev;
    p.n_chunks_host = n_chunks_host;
    p.chunks_cap = chunks_cap;
    p.per = chunk_bytes / (uint32_t)esz;
    p.groups = (uint32_t)((p.per + 1023) / 1024);   // 32 words of 32 bits per 1024 elements
    p.eps = eps;
    p.out = idx;
    p.cap = cap;
    p.count = n_diff_dev;
    if (tiles) {
        // fused pair path: K4a reads K1's tile compaction and writes the chunk list + its count
        p.tagg = tiles->tagg;
        p.tids = tiles->tids;
        p.n_tiles = (uint32_t)((tiles->n_pair + kTileTasks - 1) / kTileTasks);
        p.tile_ids = (uint32_t)kTileTasks * 32;
        p.list_out = const_cast<uint64_t *>(chunks);
        p.n_chunks_out = const_cast<uint64_t *>(n_chunks_dev);
    }
    static std::atomic<int> occ[5] = {{0}, {0}, {0}, {0}, {0}};
    const int d = dtype == CKPT_F32 ? 0 : 1;
    if (occ[d].load() == 0) {
        int m = 0, e = 0, sc = 0;
        if (d == 0) {
            CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&m, verify_mark_kernel<0>, kVerifyThreads, 0));
            CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&e, verify_emit_kernel<0>, kVerifyThreads, 0));
        } else {
            CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&m, verify_mark_kernel<1>, kVerifyThreads, 0));
            CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&e, verify_emit_kernel<1>, kVerifyThreads, 0));
        }
        CK_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&sc, verify_scan_kernel, kVerifyThreads, 0));
        occ[4].store(std::max(sc, 1));
        occ[2 + d].store(std::max(e, 1));
        occ[d].store(std::max(m, 1));
    }
    const uint64_t warp_ctas = (max_chunks + kVerifyWarps - 1) / kVerifyWarps;
    const unsigned g_mark = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(warp_ctas, (uint64_t)di.sms * occ[d].load()));
    const unsigned g_emit = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(warp_ctas, (uint64_t)di.sms * occ[2 + d].load()));
    // co-resident grid (the look-back relies on it); tiles are strided statically
    const uint64_t max_tiles = (max_chunks + kVerifyScanTile - 1) / kVerifyScanTile;
    const unsigned g_scan = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(max_tiles, (uint64_t)di.sms * occ[4].load()));
    unsigned long long *ticket_unused = nullptr;
    CK_TRY(get_scratch(dev, s, max_tiles, &p.states, &ticket_unused, &p.epoch));
    const size_t o_off = align256((size_t)max_chunks * 4);
    const size_t o_mask = o_off + align256((size_t)max_chunks * 8);
    uint8_t *work = nullptr;
    CK_TRY(get_work(dev, s, o_mask + (size_t)max_chunks * p.groups * 128, &work));
    p.cnt = (uint32_t *)work;
    p.off = (uint64_t *)(work + o_off);
    p.mask = (uint32_t *)(work + o_mask);
    {
        ProfScope prof(3, s);
        CK_CUDA(launch_k(d == 0 ? verify_mark_kernel<0> : verify_mark_kernel<1>, dim3(g_mark),
                         dim3(kVerifyThreads), 0, s, p));
        CK_LAUNCH();
        CK_CUDA(launch_k(verify_scan_kernel, dim3(g_scan), dim3(kVerifyThreads), 0, s, p));
        CK_LAUNCH();
        if (before_emit) CK_TRY(before_emit(&p.out, &p.cap));
        CK_CUDA(launch_k(d == 0 ? verify_emit_kernel<0> : verify_emit_kernel<1>, dim3(g_emit),
                         dim3(kVerifyThreads), 0, s, p));
    }
    CK_LAUNCH();
    if (tab) CK_CUDA(cudaFreeAsync(tab, s));
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// stages 1+2 in one call (diff kernel(s) then the verify kernel, no host sync)
// ---------------------------------------------------------------------------
extern "C" ckpt_status ckpt_diff_verify_async(const ckpt_tree *ta, const ckpt_tree *tb,
                                              const void *const *a, const void *const *b,
                                              uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                                              uint64_t idx_cap, uint64_t *counts_dev, void *stream) {
    CK_TRY(check_pair(ta, tb));
    if (!a || !b || !counts_dev || (!chunks && chunks_cap) || (!idx && idx_cap))
        return fail(CKPT_EINVAL, "NULL argument");
    CK_TRY(ckpt_tree_diff_async(ta, tb, 0, chunks, chunks_cap, counts_dev, stream));
    return verify_impl(a, b, ta->n_elems.data(), ta->n_arrays, ta->dtype, ta->chunk_bytes, chunks,
                       counts_dev, 0, chunks_cap, ta->eps, idx, idx_cap, counts_dev + 1,
                       (cudaStream_t)stream);
}

// ---------------------------------------------------------------------------
// fused pair compare: K1 in pair mode (digest compare and
// element marking in-kernel), then the ordered chunk list and the element ids
// ---------------------------------------------------------------------------
static ckpt_status compare_pair_impl(const void *const *a, const void *const *b, const uint64_t *n,
                                     uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                     double eps, uint32_t hash_block, uint64_t *chunks,
                                     uint64_t chunks_cap, uint64_t *idx, uint64_t idx_cap,
                                     uint64_t *counts_dev, void *stream, ckpt_tree **out_a,
                                     ckpt_tree **out_b, const EmitHook &before_emit) {
    if (out_a) *out_a = nullptr;
    if (out_b) *out_b = nullptr;
    if (!a || !b || !n || n_arrays == 0) return fail(CKPT_EINVAL, "no arrays");
    if (!out_a || !out_b) return fail(CKPT_EINVAL, "NULL tree outputs");
    if (!counts_dev || (!chunks && chunks_cap) || (!idx && idx_cap))
        return fail(CKPT_EINVAL, "NULL argument");
    if (n_arrays >= (1u << 20)) return fail(CKPT_EINVAL, "too many arrays");
    CK_TRY(check_common(dtype, chunk_bytes, eps));
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    uint64_t L = 0;
    for (uint32_t k = 0; k < n_arrays; ++k) L += (n[k] * esz + chunk_bytes - 1) / chunk_bytes;
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    PairParams pp;
    std::memset(&pp, 0, sizeof(pp));
    pp.m = (int)n_arrays;
    // flag bytes live in their own per-stream buffer (verify's work buffer may regrow)
    CK_TRY(get_pair_flags(dev, s, L, &pp.flags));
    uint64_t n_pair = 0;                          // pair-tasks: kRows chunks of one array each
    for (uint32_t k = 0; k < n_arrays; ++k) n_pair += ((n[k] * esz + chunk_bytes - 1) / chunk_bytes + kRows - 1) / kRows;
    CK_TRY(get_tile_scratch(dev, s, n_pair, &pp));
    std::vector<const void *> data(2 * (size_t)n_arrays);
    std::vector<uint64_t> nn(2 * (size_t)n_arrays);
    for (uint32_t k = 0; k < n_arrays; ++k) {
        data[k] = a[k];
        data[n_arrays + k] = b[k];
        nn[k] = nn[n_arrays + k] = n[k];
    }
    const uint32_t apt[2] = {n_arrays, n_arrays};
    ckpt_tree *trees[2] = {nullptr, nullptr};
    CK_TRY(build_batch_impl(data.data(), nn.data(), apt, 2, dtype, chunk_bytes, eps, hash_block, stream,
                            trees, &pp));
    // the ordered chunk list from K1's per-tile compaction: read by K4a directly (up to
    // kVerifyMaxTiles tiles), else placed by one gather pass
    ckpt_status st = CKPT_OK;
    const uint64_t n_tiles = (n_pair + kTileTasks - 1) / kTileTasks;
    const bool tiles_in_mark = n_tiles <= (uint64_t)kVerifyMaxTiles && chunks_cap > 0 && !tile_gather_forced();
    pp.n_pair = n_pair;
    if (!tiles_in_mark) {
        TileGatherParams g;
        g.tagg = pp.tagg;
        g.tids = pp.tids;
        g.n_tiles = (n_pair + kTileTasks - 1) / kTileTasks;
        g.tile_ids = (uint64_t)kTileTasks * 32;
        g.out = chunks;
        g.cap = chunks_cap;
        g.count = counts_dev;
        const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(g.n_tiles, (uint64_t)di.sms * 8));
        ProfScope prof(2, s);
        if (launch_k(tile_gather_kernel, dim3(grid), dim3(kGatherThreads), 0, s, g) != cudaSuccess)
            st = fail(CKPT_ECUDA, "tile gather launch");
    }
    if (st == CKPT_OK)
        st = verify_impl(a, b, n, n_arrays, dtype, chunk_bytes, chunks, counts_dev, 0, chunks_cap, eps,
                         idx, idx_cap, counts_dev + 1, s, before_emit, 0, 0, tiles_in_mark ? &pp : nullptr);
    if (st != CKPT_OK) {
        ckpt_tree_free_on(trees[0], stream);
        ckpt_tree_free_on(trees[1], stream);
        return st;
    }
    *out_a = trees[0];
    *out_b = trees[1];
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_compare_pair_ex(const void *const *a, const void *const *b,
                                            const uint64_t *n, uint32_t n_arrays, ckpt_dtype dtype,
                                            uint32_t chunk_bytes, double eps, uint32_t hash_block,
                                            uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                                            uint64_t idx_cap, uint64_t *counts_dev, void *stream,
                                            ckpt_tree **out_a, ckpt_tree **out_b) {
    return compare_pair_impl(a, b, n, n_arrays, dtype, chunk_bytes, eps, hash_block, chunks,
                             chunks_cap, idx, idx_cap, counts_dev, stream, out_a, out_b, nullptr);
}

extern "C" ckpt_status ckpt_compare_pair_async(const void *const *a, const void *const *b,
                                               const uint64_t *n, uint32_t n_arrays,
                                               ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                               uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                                               uint64_t idx_cap, uint64_t *counts_dev, void *stream,
                                               ckpt_tree **out_a, ckpt_tree **out_b) {
    return ckpt_compare_pair_ex(a, b, n, n_arrays, dtype, chunk_bytes, eps, 16, chunks, chunks_cap,
                                idx, idx_cap, counts_dev, stream, out_a, out_b);
}

extern "C" ckpt_status ckpt_verify_arrays_async(const void *const *a, const void *const *b,
                                                const uint64_t *n, uint32_t n_arrays,
                                                ckpt_dtype dtype, uint32_t chunk_bytes,
                                                const uint64_t *chunks, const uint64_t *n_chunks_dev,
                                                uint64_t chunks_cap, double eps, uint64_t *idx,
                                                uint64_t cap, uint64_t *n_diff_dev, void *stream) {
    if (!n_chunks_dev) return fail(CKPT_EINVAL, "n_chunks_dev is NULL");
    return verify_impl(a, b, n, n_arrays, dtype, chunk_bytes, chunks, n_chunks_dev, 0, chunks_cap,
                       eps, idx, cap, n_diff_dev, (cudaStream_t)stream);
}

extern "C" ckpt_status ckpt_verify(const void *a, const void *b, uint64_t n, ckpt_dtype dtype,
                                   uint32_t chunk_bytes, const uint64_t *chunks, uint64_t n_chunks,
                                   double eps, uint64_t *idx, uint64_t cap, uint64_t *n_diff,
                                   void *stream) {
    if (!n_diff) return fail(CKPT_EINVAL, "n_diff is NULL");
    cudaStream_t s = (cudaStream_t)stream;
    const void *pa[1] = {a}, *pb[1] = {b};
    uint64_t nn[1] = {n};
    uint64_t *dcount = nullptr;
    CK_CUDA(cudaMallocAsync((void **)&dcount, 8, s));
    ckpt_status st = verify_impl(pa, pb, nn, 1, dtype, chunk_bytes, chunks, nullptr, n_chunks,
                                 n_chunks, eps, idx, cap, dcount, s);
    if (st != CKPT_OK) { cudaFreeAsync(dcount, s); return st; }
    CK_CUDA(cudaMemcpyAsync(n_diff, dcount, 8, cudaMemcpyDeviceToHost, s));
    CK_CUDA(cudaFreeAsync(dcount, s));
    CK_CUDA(cudaStreamSynchronize(s));
    if (*n_diff > cap) return fail(CKPT_ETRUNC, "difference list longer than cap");
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// whole pipeline
// ---------------------------------------------------------------------------
extern "C" ckpt_status ckpt_tree_root(const ckpt_tree *t, uint8_t out16[16], void *stream) {
    if (!t || !out16) return fail(CKPT_EINVAL, "NULL argument");
    cudaStream_t s = (cudaStream_t)stream;
    CK_TRY(wait_levels(t, s));
    CK_CUDA(cudaMemcpyAsync(out16, t->nodes + t->top_off + t->top_nodes - 1, 16,
                            cudaMemcpyDeviceToHost, s));
    CK_CUDA(cudaStreamSynchronize(s));
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_compare(const void *const *a, const void *const *b, const uint64_t *n,
                                    uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                    double eps, uint64_t *chunks, uint64_t chunks_cap,
                                    uint64_t *idx, uint64_t idx_cap, uint64_t *n_chunks,
                                    uint64_t *n_diff, uint8_t *root_a16, uint8_t *root_b16,
                                    void *stream) {
    if (!n_chunks || !n_diff) return fail(CKPT_EINVAL, "NULL count output");
    if (!a || !b || !n || n_arrays == 0) return fail(CKPT_EINVAL, "no arrays");
    cudaStream_t s = (cudaStream_t)stream;
    ckpt_tree *ta = nullptr, *tb = nullptr;
    uint64_t *dc = nullptr;
    // both runs' leaves in one leaf-kernel launch (fuller last wave)
    std::vector<const void *> ab(a, a + n_arrays);
    ab.insert(ab.end(), b, b + n_arrays);
    std::vector<uint64_t> nn(n, n + n_arrays);
    nn.insert(nn.end(), n, n + n_arrays);
    const uint32_t per[2] = {n_arrays, n_arrays};
    ckpt_tree *tt[2] = {nullptr, nullptr};
    ckpt_status st = ckpt_tree_build_batch(ab.data(), nn.data(), per, 2, dtype, chunk_bytes, eps, stream, tt);
    ta = tt[0];
    tb = tt[1];
    if (st == CKPT_OK && cudaMallocAsync((void **)&dc, 16, s) != cudaSuccess)
        st = fail(CKPT_ENOMEM, "count scratch");
    if (st == CKPT_OK) st = ckpt_tree_diff_async(ta, tb, 0, chunks, chunks_cap, dc, stream);
    if (st == CKPT_OK)
        st = verify_impl(a, b, n, n_arrays, dtype, chunk_bytes, chunks, dc, 0, chunks_cap, eps, idx,
                         idx_cap, dc + 1, s);
    uint64_t hc[2] = {0, 0};
    if (st == CKPT_OK && cudaMemcpyAsync(hc, dc, 16, cudaMemcpyDeviceToHost, s) != cudaSuccess)
        st = fail(CKPT_ECUDA, "count copy");
    if (st == CKPT_OK && root_a16) st = ckpt_tree_root(ta, root_a16, stream);
    if (st == CKPT_OK && root_b16) st = ckpt_tree_root(tb, root_b16, stream);
    if (st == CKPT_OK && cudaStreamSynchronize(s) != cudaSuccess) st = fail(CKPT_ECUDA, "sync");
    if (dc) cudaFreeAsync(dc, s);
    ckpt_tree_free_on(ta, stream);
    ckpt_tree_free_on(tb, stream);
    if (st != CKPT_OK) return st;
    *n_chunks = hc[0];
    *n_diff = hc[1];
    if (hc[0] > chunks_cap || hc[1] > idx_cap) return fail(CKPT_ETRUNC, "output longer than cap");
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_compare_host(const void *const *a, const void *const *b,
                                         const uint64_t *n, uint32_t n_arrays, ckpt_dtype dtype,
                                         uint32_t chunk_bytes, double eps, uint64_t *idx,
                                         uint64_t idx_cap, uint64_t *n_chunks, uint64_t *n_diff,
                                         uint8_t *root_a16, uint8_t *root_b16) {
    if (!a || !b || !n || n_arrays == 0) return fail(CKPT_EINVAL, "no arrays");
    if (!n_chunks || !n_diff || (!idx && idx_cap)) return fail(CKPT_EINVAL, "NULL output");
    CK_TRY(check_common(dtype, chunk_bytes, eps));
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    uint64_t L = 0, bytes = 0;
    for (uint32_t k = 0; k < n_arrays; ++k) {
        if (!a[k] || !b[k] || n[k] == 0) return fail(CKPT_EINVAL, "NULL or empty array");
        L += (n[k] * esz + chunk_bytes - 1) / chunk_bytes;
        bytes += align256(n[k] * esz);
    }
    cudaStream_t sk = nullptr;
    CK_CUDA(cudaStreamCreateWithFlags(&sk, cudaStreamNonBlocking));
    // one staging allocation for both runs (the pool keeps it mapped between calls)
    uint8_t *stage = nullptr;
    uint64_t *dchunks = nullptr, *didx = nullptr, *dc = nullptr;
    std::vector<const void *> da(n_arrays), db(n_arrays);
    ckpt_tree *ta = nullptr, *tb = nullptr;
    uint64_t hc[2] = {0, 0};
    ckpt_status st = CKPT_OK;
    auto cu = [&](cudaError_t e, const char *what) {
        if (st == CKPT_OK && e != cudaSuccess)
            st = fail(e == cudaErrorMemoryAllocation ? CKPT_ENOMEM : CKPT_ECUDA,
                      std::string(what) + ": " + cudaGetErrorString(e));
    };
    cu(cudaMallocAsync((void **)&stage, 2 * bytes, sk), "alloc staging");
    cu(cudaMallocAsync((void **)&dchunks, L * 8, sk), "alloc chunks");
    cu(cudaMallocAsync((void **)&dc, 16, sk), "alloc counts");
    uint64_t off = 0;
    for (uint32_t k = 0; k < n_arrays && st == CKPT_OK; ++k) {
        da[k] = stage + off;
        db[k] = stage + bytes + off;
        off += align256(n[k] * esz);
    }
    for (uint32_t k = 0; k < n_arrays && st == CKPT_OK; ++k)
        cu(cudaMemcpyAsync((void *)da[k], a[k], n[k] * esz, cudaMemcpyHostToDevice, sk), "H2D A");
    for (uint32_t k = 0; k < n_arrays && st == CKPT_OK; ++k)
        cu(cudaMemcpyAsync((void *)db[k], b[k], n[k] * esz, cudaMemcpyHostToDevice, sk), "H2D B");
    // the element-id buffer is sized to the count (read back after the verify scan)
    const EmitHook hook = [&](uint64_t **out, uint64_t *cap) -> ckpt_status {
        CK_CUDA(cudaMemcpyAsync(hc, dc, 16, cudaMemcpyDeviceToHost, sk));
        CK_CUDA(cudaStreamSynchronize(sk));
        const uint64_t want = std::min(hc[1], idx_cap);
        CK_CUDA(cudaMallocAsync((void **)&didx, std::max<uint64_t>(want, 1) * 8, sk));
        *out = didx;
        *cap = want;
        return CKPT_OK;
    };
    if (st == CKPT_OK)
        st = compare_pair_impl(da.data(), db.data(), n, n_arrays, dtype, chunk_bytes, eps, 16, dchunks,
                               L, nullptr, 0, dc, sk, &ta, &tb, hook);
    if (st == CKPT_OK && idx_cap && hc[1])
        cu(cudaMemcpyAsync(idx, didx, std::min(hc[1], idx_cap) * 8, cudaMemcpyDeviceToHost, sk), "D2H idx");
    if (st == CKPT_OK && root_a16) st = ckpt_tree_root(ta, root_a16, sk);
    if (st == CKPT_OK && root_b16) st = ckpt_tree_root(tb, root_b16, sk);
    cu(cudaStreamSynchronize(sk), "sync");
    ckpt_tree_free_on(ta, sk);
    ckpt_tree_free_on(tb, sk);
    if (stage) cudaFreeAsync(stage, sk);
    if (dchunks) cudaFreeAsync(dchunks, sk);
    if (didx) cudaFreeAsync(didx, sk);
    if (dc) cudaFreeAsync(dc, sk);
    release_scratch(dev, sk);
    cudaStreamSynchronize(sk);
    cudaStreamDestroy(sk);
    if (st != CKPT_OK) return st;
    *n_chunks = hc[0];
    *n_diff = hc[1];
    if (hc[1] > idx_cap) return fail(CKPT_ETRUNC, "difference list longer than cap");
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// out-of-core streaming compare: host-resident runs are
// streamed through a two-slot device ring of chunk-aligned segments; the H2D
// copy of segment k+1 (copy stream) overlaps the leaf hashing, the in-kernel
// digest compare, the compaction and the verify of segment k (compute
// stream).  Leaves land at their global position in full-size trees, so the
// trees (and roots) equal the in-HBM build; device memory is bounded by the
// ring, the trees, one flag byte per chunk and the per-segment outputs.
// The paper's pipeline overlaps I/O and hashing the same way (Fig. 3
// P:476-495), there from Lustre through io_uring.
// ---------------------------------------------------------------------------
static ckpt_status alloc_tree(const uint64_t *n, uint32_t na, ckpt_dtype dtype, uint32_t C, double eps,
                              uint32_t hb, int dev, cudaStream_t s, ckpt_tree **out) {
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    ckpt_tree *t = new ckpt_tree();
    t->device = dev;
    t->stream = s;
    t->dtype = dtype;
    t->chunk_bytes = C;
    t->eps = eps;
    t->hash_block = hb;
    t->n_elems.assign(n, n + na);
    std::vector<uint64_t> leaves(na);
    for (uint32_t a = 0; a < na; ++a) leaves[a] = (n[a] * esz + C - 1) / C;
    layout(t, leaves);
    ckpt_status st = prepare_tree(t, s);
    if (st != CKPT_OK) { ckpt_tree_free_on(t, s); return st; }
    *out = t;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_compare_stream(const void *const *a, const void *const *b,
                                           const uint64_t *n, uint32_t n_arrays, ckpt_dtype dtype,
                                           uint32_t chunk_bytes, double eps, uint32_t hash_block,
                                           uint64_t segment_bytes, uint64_t *chunks,
                                           uint64_t chunks_cap, uint64_t *idx, uint64_t idx_cap,
                                           uint64_t *n_chunks, uint64_t *n_diff, uint8_t *root_a16,
                                           uint8_t *root_b16) {
    if (!a || !b || !n || n_arrays == 0) return fail(CKPT_EINVAL, "no arrays");
    if (!n_chunks || !n_diff || (!idx && idx_cap) || (!chunks && chunks_cap))
        return fail(CKPT_EINVAL, "NULL output");
    CK_TRY(check_common(dtype, chunk_bytes, eps));
    CK_TRY(norm_block(hash_block, chunk_bytes, &hash_block));
    const uint64_t esz = dtype == CKPT_F32 ? 4 : 8;
    for (uint32_t k = 0; k < n_arrays; ++k)
        if (!a[k] || !b[k] || n[k] == 0) return fail(CKPT_EINVAL, "NULL or empty array");
    const uint64_t seg = std::max<uint64_t>(1, segment_bytes / chunk_bytes) * chunk_bytes;
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    // segments: (array, byte offset, bytes, global chunk id, global element id)
    struct Seg { uint32_t a; uint64_t off, bytes, chunk0, elem0; };
    std::vector<Seg> segs;
    uint64_t L = 0, E = 0;
    for (uint32_t k = 0; k < n_arrays; ++k) {
        const uint64_t nb = n[k] * esz;
        for (uint64_t o = 0; o < nb; o += seg)
            segs.push_back({k, o, std::min(seg, nb - o), L + o / chunk_bytes, E + o / esz});
        L += (nb + chunk_bytes - 1) / chunk_bytes;
        E += n[k];
    }
    cudaStream_t sc = nullptr, sk = nullptr;
    CK_CUDA(cudaStreamCreateWithFlags(&sc, cudaStreamNonBlocking));
    CK_CUDA(cudaStreamCreateWithFlags(&sk, cudaStreamNonBlocking));
    cudaEvent_t copied[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr};
    uint8_t *ring = nullptr, *flags = nullptr;
    uint64_t *dchunks = nullptr, *didx = nullptr, *dc = nullptr;
    uint64_t didx_cap = 0;
    ckpt_tree *ta = nullptr, *tb = nullptr;
    uint64_t tot_c = 0, tot_e = 0;
    ckpt_status st = CKPT_OK;
    auto cu = [&](cudaError_t e, const char *what) {
        if (st == CKPT_OK && e != cudaSuccess)
            st = fail(e == cudaErrorMemoryAllocation ? CKPT_ENOMEM : CKPT_ECUDA,
                      std::string(what) + ": " + cudaGetErrorString(e));
    };
    for (int i = 0; i < 2; ++i) {
        cu(cudaEventCreateWithFlags(&copied[i], cudaEventDisableTiming), "event");
        cu(cudaEventCreateWithFlags(&freed[i], cudaEventDisableTiming), "event");
    }
    cu(cudaMallocAsync((void **)&ring, 4 * seg, sk), "alloc ring");          // 2 slots x (A, B)
    cu(cudaMallocAsync((void **)&flags, std::max<uint64_t>(L, 1), sk), "alloc flags");
    cu(cudaMallocAsync((void **)&dchunks, std::max<uint64_t>(seg / chunk_bytes, 1) * 8, sk), "alloc chunks");
    cu(cudaMallocAsync((void **)&dc, 16, sk), "alloc counts");
    if (st == CKPT_OK) st = alloc_tree(n, n_arrays, dtype, chunk_bytes, eps, hash_block, dev, sk, &ta);
    if (st == CKPT_OK) st = alloc_tree(n, n_arrays, dtype, chunk_bytes, eps, hash_block, dev, sk, &tb);
    // the ring exists before the copy stream uses it
    cu(cudaEventRecord(freed[0], sk), "event");
    cu(cudaEventRecord(freed[1], sk), "event");
    uint64_t hc[2] = {0, 0};
    unsigned int *ctr = nullptr;
    unsigned long long *ticket = nullptr;
    auto enqueue_copy = [&](size_t k) {
        const Seg &g = segs[k];
        const int sl = (int)(k & 1);
        uint8_t *da = ring + (size_t)sl * 2 * seg, *db = da + seg;
        cu(cudaStreamWaitEvent(sc, freed[sl], 0), "wait slot");
        cu(cudaMemcpyAsync(da, (const uint8_t *)a[g.a] + g.off, g.bytes, cudaMemcpyHostToDevice, sc), "H2D A");
        cu(cudaMemcpyAsync(db, (const uint8_t *)b[g.a] + g.off, g.bytes, cudaMemcpyHostToDevice, sc), "H2D B");
        cu(cudaEventRecord(copied[sl], sc), "event");
    };
    if (st == CKPT_OK && !segs.empty()) enqueue_copy(0);
    for (size_t k = 0; k < segs.size() && st == CKPT_OK; ++k) {
        const Seg &g = segs[k];
        const int sl = (int)(k & 1);
        uint8_t *da = ring + (size_t)sl * 2 * seg, *db = da + seg;
        if (k + 1 < segs.size()) enqueue_copy(k + 1);        // overlaps everything below
        cu(cudaStreamWaitEvent(sk, copied[sl], 0), "wait copy");
        // leaves of both runs' segment in one pair-mode launch, written at their global slots
        const uint64_t nl = (g.bytes + chunk_bytes - 1) / chunk_bytes;
        const uint64_t local0 = g.off / chunk_bytes;                  // chunk index inside the array
        const uint64_t tasks_per = (nl + kRows - 1) / kRows;
        std::vector<LeafArray> table(2);
        ckpt_tree *tt[2] = {ta, tb};
        uint8_t *src[2] = {da, db};
        for (int r = 0; r < 2; ++r) {
            LeafArray &e = table[r];
            e.data = src[r];
            e.nbytes = g.bytes;
            e.n_leaves = nl;
            e.n_full = g.bytes / chunk_bytes;
            e.task_begin = (uint64_t)r * tasks_per;
            e.out = tt[r]->nodes + tt[r]->off[g.a] + local0;
            e.chunk_base = g.chunk0;
        }
        PairParams pp;
        std::memset(&pp, 0, sizeof(pp));
        pp.flags = flags;
        pp.n_pair = tasks_per;
        pp.m = 1;
        if (st == CKPT_OK) st = get_pair_ctr(dev, sk, tasks_per, &ctr);
        pp.ctr = ctr;
        if (st == CKPT_OK && !ticket) {
            uint64_t *unused_states;
            uint32_t unused_epoch;
            st = get_scratch(dev, sk, 0, &unused_states, &ticket, &unused_epoch);
            ticket += kLeafTicketSlot;
        }
        if (st == CKPT_OK)
            st = launch_leaves(table, 2 * tasks_per, dtype, eps, chunk_bytes, hash_block, sk, di.sms, &pp,
                               ticket);
        // this segment's flagged chunks (global ids), then its verify
        if (st == CKPT_OK)
            st = launch_compact(1, nullptr, nullptr, flags + g.chunk0, nl, dchunks, nl, dc, sk, di.sms,
                                g.chunk0);
        uint64_t seg_c = 0, seg_e = 0;
        const EmitHook hook = [&](uint64_t **out, uint64_t *cap) -> ckpt_status {
            CK_CUDA(cudaMemcpyAsync(hc, dc, 16, cudaMemcpyDeviceToHost, sk));
            CK_CUDA(cudaStreamSynchronize(sk));
            seg_c = hc[0];
            seg_e = hc[1];
            if (seg_e > didx_cap) {
                if (didx) CK_CUDA(cudaFreeAsync(didx, sk));
                didx_cap = std::max<uint64_t>(seg_e, 2 * didx_cap);
                CK_CUDA(cudaMallocAsync((void **)&didx, didx_cap * 8, sk));
            }
            *out = didx;
            *cap = didx_cap;
            return CKPT_OK;
        };
        const void *va[1] = {da}, *vb[1] = {db};
        const uint64_t vn[1] = {g.bytes / esz};
        if (st == CKPT_OK)
            st = verify_impl(va, vb, vn, 1, dtype, chunk_bytes, dchunks, dc, 0, nl, eps, nullptr, 0, dc + 1,
                             sk, hook, g.chunk0, g.elem0);
        cu(cudaEventRecord(freed[sl], sk), "event");          // slot reusable after the verify
        // append this segment's ids to the caller's host buffers (ascending across segments)
        if (st == CKPT_OK && seg_c && tot_c < chunks_cap)
            cu(cudaMemcpyAsync(chunks + tot_c, dchunks, std::min(seg_c, chunks_cap - tot_c) * 8,
                               cudaMemcpyDeviceToHost, sk), "D2H chunks");
        if (st == CKPT_OK && seg_e && tot_e < idx_cap)
            cu(cudaMemcpyAsync(idx + tot_e, didx, std::min(seg_e, idx_cap - tot_e) * 8,
                               cudaMemcpyDeviceToHost, sk), "D2H idx");
        tot_c += seg_c;
        tot_e += seg_e;
    }
    if (st == CKPT_OK) {
        ckpt_tree *both[2] = {ta, tb};
        st = launch_levels(both, 2, sk);
    }
    if (st == CKPT_OK && root_a16) st = ckpt_tree_root(ta, root_a16, sk);
    if (st == CKPT_OK && root_b16) st = ckpt_tree_root(tb, root_b16, sk);
    cu(cudaStreamSynchronize(sk), "sync");
    cudaStreamSynchronize(sc);
    ckpt_tree_free_on(ta, sk);
    ckpt_tree_free_on(tb, sk);
    if (ring) cudaFreeAsync(ring, sk);
    if (flags) cudaFreeAsync(flags, sk);
    if (dchunks) cudaFreeAsync(dchunks, sk);
    if (didx) cudaFreeAsync(didx, sk);
    if (dc) cudaFreeAsync(dc, sk);
    release_scratch(dev, sk);
    cudaStreamSynchronize(sk);
    for (int i = 0; i < 2; ++i) {
        if (copied[i]) cudaEventDestroy(copied[i]);
        if (freed[i]) cudaEventDestroy(freed[i]);
    }
    cudaStreamDestroy(sc);
    cudaStreamDestroy(sk);
    if (st != CKPT_OK) return st;
    *n_chunks = tot_c;
    *n_diff = tot_e;
    if (tot_c > chunks_cap || tot_e > idx_cap) return fail(CKPT_ETRUNC, "output longer than cap");
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// tree persistence: the tree is created at capture time
// and stored with the checkpoint; a later comparison loads it
// instead of re-hashing that run
// ---------------------------------------------------------------------------
static const char kTreeMagic[8] = {'C', 'K', 'P', 'T', 'T', 'R', 'E', '1'};
constexpr uint32_t kTreeFormat = 1;
constexpr size_t kTreeHdr = 40;   // fixed part before n_elems[]

static size_t ser_prefix(uint32_t na) { return kTreeHdr + (size_t)na * 8 + 8 + 16; }

extern "C" ckpt_status ckpt_tree_serialized_size(const ckpt_tree *t, uint64_t *bytes) {
    if (!t || !bytes) return fail(CKPT_EINVAL, "NULL argument");
    if (t->from_digests) return fail(CKPT_EINVAL, "trees built from digests are not serialisable");
    *bytes = ser_prefix(t->n_arrays) + (t->array_nodes + t->top_nodes) * 16;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_serialize(const ckpt_tree *t, void *dst, uint64_t cap,
                                           uint64_t *written, void *stream) {
    uint64_t need = 0;
    CK_TRY(ckpt_tree_serialized_size(t, &need));
    if (!dst || !written) return fail(CKPT_EINVAL, "NULL argument");
    *written = need;
    if (cap < need) return fail(CKPT_EINVAL, "destination smaller than ckpt_tree_serialized_size");
    uint8_t *o = (uint8_t *)dst;
    std::memset(o, 0, ser_prefix(t->n_arrays));
    std::memcpy(o, kTreeMagic, 8);
    const uint32_t hdr32[5] = {kTreeFormat, (uint32_t)t->dtype, t->chunk_bytes, t->hash_block, 0};
    std::memcpy(o + 8, hdr32, 16);
    std::memcpy(o + 24, &t->eps, 8);
    std::memcpy(o + 32, &t->n_arrays, 4);
    std::memcpy(o + kTreeHdr, t->n_elems.data(), (size_t)t->n_arrays * 8);
    const uint64_t nodes = t->array_nodes + t->top_nodes;
    std::memcpy(o + kTreeHdr + (size_t)t->n_arrays * 8, &nodes, 8);
    cudaStream_t s = (cudaStream_t)stream;
    CK_TRY(wait_levels(t, s));
    uint8_t *body = o + ser_prefix(t->n_arrays);
    CK_CUDA(cudaMemcpyAsync(body, t->nodes, nodes * 16, cudaMemcpyDeviceToHost, s));
    CK_CUDA(cudaStreamSynchronize(s));
    std::memcpy(o + ser_prefix(t->n_arrays) - 16, body + (nodes - 1) * 16, 16);   // the root
    return CKPT_OK;
}

// Host-only parse of a serialised tree (no device work): header checks and
// the layout the body must have.
static ckpt_status parse_tree(const uint8_t *in, uint64_t bytes, ckpt_tree *t) {
    if (bytes < kTreeHdr || std::memcmp(in, kTreeMagic, 8) != 0)
        return fail(CKPT_EINVAL, "not a serialised ckpt tree (bad magic)");
    uint32_t hdr32[5];
    std::memcpy(hdr32, in + 8, 16);
    if (hdr32[0] != kTreeFormat) return fail(CKPT_EINVAL, "unsupported tree format version");
    if (hdr32[1] != CKPT_F32 && hdr32[1] != CKPT_F64) return fail(CKPT_EINVAL, "bad dtype in tree header");
    t->dtype = (ckpt_dtype)hdr32[1];
    t->chunk_bytes = hdr32[2];
    t->hash_block = hdr32[3];
    std::memcpy(&t->eps, in + 24, 8);
    CK_TRY(check_common(t->dtype, t->chunk_bytes, t->eps));
    if (t->hash_block == 0 || t->hash_block % 16 || t->hash_block > t->chunk_bytes)
        return fail(CKPT_EINVAL, "bad hash_block in tree header");
    uint32_t na = 0;
    std::memcpy(&na, in + 32, 4);
    if (na == 0 || na >= (1u << 20)) return fail(CKPT_EINVAL, "bad array count in tree header");
    if (bytes < ser_prefix(na)) return fail(CKPT_EINVAL, "truncated tree header");
    t->n_elems.resize(na);
    std::memcpy(t->n_elems.data(), in + kTreeHdr, (size_t)na * 8);
    const uint64_t esz = t->dtype == CKPT_F32 ? 4 : 8;
    std::vector<uint64_t> leaves(na);
    for (uint32_t a = 0; a < na; ++a) {
        if (t->n_elems[a] == 0 || t->n_elems[a] > (1ull << 50)) return fail(CKPT_EINVAL, "bad array length");
        leaves[a] = (t->n_elems[a] * esz + t->chunk_bytes - 1) / t->chunk_bytes;
    }
    layout(t, leaves);
    uint64_t nodes = 0;
    std::memcpy(&nodes, in + kTreeHdr + (size_t)na * 8, 8);
    if (nodes != t->array_nodes + t->top_nodes) return fail(CKPT_EINVAL, "node count does not match the header");
    if (bytes != ser_prefix(na) + nodes * 16) return fail(CKPT_EINVAL, "serialised tree has the wrong size");
    if (std::memcmp(in + ser_prefix(na) - 16, in + ser_prefix(na) + (nodes - 1) * 16, 16) != 0)
        return fail(CKPT_EINVAL, "stored root does not match the last node");
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_deserialize(const void *src, uint64_t bytes, void *stream,
                                             ckpt_tree **out) {
    if (!out) return fail(CKPT_EINVAL, "out is NULL");
    *out = nullptr;
    if (!src) return fail(CKPT_EINVAL, "src is NULL");
    ckpt_tree tmp;
    CK_TRY(parse_tree((const uint8_t *)src, bytes, &tmp));      // no device work before this
    int dev;
    DevInfo di;
    CK_TRY(dev_info(&dev, &di));
    cudaStream_t s = (cudaStream_t)stream;
    ckpt_tree *t = new ckpt_tree(tmp);
    t->device = dev;
    t->stream = s;
    t->levels_done = nullptr;
    ckpt_status st = prepare_tree(t, s);
    const uint64_t nodes = t->array_nodes + t->top_nodes;
    if (st == CKPT_OK)
        st = g_ring.copy(t->meta, t->meta_host.data(), t->meta_host.size() * 8, s);
    if (st == CKPT_OK &&
        cudaMemcpyAsync(t->nodes, (const uint8_t *)src + ser_prefix(t->n_arrays), nodes * 16,
                        cudaMemcpyHostToDevice, s) != cudaSuccess)
        st = fail(CKPT_ECUDA, "tree upload");
    // the caller's buffer may be pageable and reused at once: finish the upload
    if (st == CKPT_OK && cudaStreamSynchronize(s) != cudaSuccess) st = fail(CKPT_ECUDA, "sync");
    if (st != CKPT_OK) { ckpt_tree_free_on(t, stream); return st; }
    *out = t;
    return CKPT_OK;
}

// Compare a live checkpoint (run B, device) with a stored run A: A's tree is
// loaded from its serialised form instead of re-hashing A, B's tree is built
// with A's parameters, the trees are diffed and only the flagged chunks of A
// are read (a_data may be host memory the device can address: pinned /
// registered host memory through UVA, so the verify kernel reads just those
// chunks over the host link, the two-stage I/O of P:568-578).
extern "C" ckpt_status ckpt_compare_saved(const void *saved_a, uint64_t saved_bytes,
                                          const void *const *a_data, const void *const *b,
                                          const uint64_t *n, uint32_t n_arrays, uint64_t *chunks,
                                          uint64_t chunks_cap, uint64_t *idx, uint64_t idx_cap,
                                          uint64_t *counts_dev, void *stream, ckpt_tree **out_a,
                                          ckpt_tree **out_b) {
    if (out_a) *out_a = nullptr;
    if (out_b) *out_b = nullptr;
    if (!out_a || !out_b || !a_data || !b || !n || !counts_dev || (!chunks && chunks_cap) ||
        (!idx && idx_cap))
        return fail(CKPT_EINVAL, "NULL argument");
    ckpt_tree hdr;
    CK_TRY(parse_tree((const uint8_t *)saved_a, saved_bytes, &hdr));
    if (hdr.n_arrays != n_arrays || !std::equal(hdr.n_elems.begin(), hdr.n_elems.end(), n))
        return fail(CKPT_EMISMATCH, "live checkpoint shape differs from the stored tree");
    ckpt_tree *ta = nullptr, *tb = nullptr;
    CK_TRY(ckpt_tree_deserialize(saved_a, saved_bytes, stream, &ta));
    ckpt_status st = build_batch_impl(b, n, &n_arrays, 1, ta->dtype, ta->chunk_bytes, ta->eps,
                                      ta->hash_block, stream, &tb, nullptr);
    if (st == CKPT_OK)
        st = ckpt_diff_verify_async(ta, tb, a_data, b, chunks, chunks_cap, idx, idx_cap, counts_dev,
                                    stream);
    if (st != CKPT_OK) {
        ckpt_tree_free_on(ta, stream);
        ckpt_tree_free_on(tb, stream);
        return st;
    }
    *out_a = ta;
    *out_b = tb;
    return CKPT_OK;
}

// ---------------------------------------------------------------------------
// accessors
// ---------------------------------------------------------------------------
extern "C" ckpt_status ckpt_tree_wait(const ckpt_tree *t, void *stream) {
    if (!t) return fail(CKPT_EINVAL, "NULL tree");
    return wait_levels(t, (cudaStream_t)stream);
}

extern "C" ckpt_status ckpt_tree_info(const ckpt_tree *t, uint32_t *n_arrays, uint64_t *n_leaves,
                                      uint32_t *n_levels, uint64_t *n_nodes) {
    if (!t) return fail(CKPT_EINVAL, "NULL tree");
    if (n_arrays) *n_arrays = t->n_arrays;
    if (n_leaves) *n_leaves = t->total_leaves;
    if (n_levels) *n_levels = t->n_levels;
    if (n_nodes) *n_nodes = t->array_nodes;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_params(const ckpt_tree *t, ckpt_dtype *dtype, uint32_t *chunk_bytes,
                                        double *eps, uint32_t *hash_block) {
    if (!t) return fail(CKPT_EINVAL, "NULL tree");
    if (t->from_digests) return fail(CKPT_EINVAL, "tree built from digests has no hashing parameters");
    if (dtype) *dtype = t->dtype;
    if (chunk_bytes) *chunk_bytes = t->chunk_bytes;
    if (eps) *eps = t->eps;
    if (hash_block) *hash_block = t->hash_block;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_array_roots(const ckpt_tree *t, void *dst, void *stream) {
    if (!t || !dst) return fail(CKPT_EINVAL, "NULL argument");
    CK_TRY(wait_levels(t, (cudaStream_t)stream));
    CK_CUDA(cudaMemcpyAsync(dst, t->nodes + t->top_off, (size_t)t->n_arrays * 16,
                            cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_array_info(const ckpt_tree *t, uint32_t array, uint64_t *n_leaves,
                                            uint64_t *n_nodes) {
    if (!t || array >= t->n_arrays) return fail(CKPT_EINVAL, "bad tree or array index");
    uint64_t tot = 0;
    for (uint32_t l = 0; l < t->height[array]; ++l) tot += t->cnt[(size_t)l * t->n_arrays + array];
    if (n_leaves) *n_leaves = t->n_leaves[array];
    if (n_nodes) *n_nodes = tot;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_tree_nodes(const ckpt_tree *t, uint32_t array, void *dst,
                                       uint64_t cap_bytes, void *stream) {
    uint64_t nn = 0;
    CK_TRY(ckpt_tree_array_info(t, array, nullptr, &nn));
    if (!dst || cap_bytes < nn * 16) return fail(CKPT_EINVAL, "destination too small");
    CK_TRY(wait_levels(t, (cudaStream_t)stream));
    uint8_t *d = (uint8_t *)dst;
    for (uint32_t l = 0; l < t->height[array]; ++l) {
        const size_t i = (size_t)l * t->n_arrays + array;
        CK_CUDA(cudaMemcpyAsync(d, t->nodes + t->off[i], t->cnt[i] * 16, cudaMemcpyDeviceToDevice,
                                (cudaStream_t)stream));
        d += t->cnt[i] * 16;
    }
    return CKPT_OK;
}

extern "C" uint64_t ckpt_default_bfs_threshold(void) {
    int dev;
    DevInfo di;
    if (dev_info(&dev, &di) != CKPT_OK) return 0;
    return (uint64_t)di.sms * (uint64_t)di.max_threads_sm;
}

extern "C" uint64_t ckpt_launch_count(void) { return g_launches.load(); }

extern "C" ckpt_status ckpt_trim_device_memory(void) {
    int dev = 0;
    CK_CUDA(cudaGetDevice(&dev));
    CK_CUDA(cudaDeviceSynchronize());
    cudaMemPool_t pool;
    CK_CUDA(cudaDeviceGetDefaultMemPool(&pool, dev));
    CK_CUDA(cudaMemPoolTrimTo(pool, 0));
    return CKPT_OK;
}

extern "C" const char *ckpt_strerror(ckpt_status s) {
    switch (s) {
        case CKPT_OK: return "ok";
        case CKPT_EINVAL: return "invalid argument";
        case CKPT_EMISMATCH: return "trees do not match in shape or parameters";
        case CKPT_ENOMEM: return "out of device memory";
        case CKPT_ECUDA: return "CUDA error";
        case CKPT_ETRUNC: return "output truncated to capacity";
    }
    return "unknown status";
}

extern "C" const char *ckpt_last_error(void) { return g_last_error.c_str(); }

extern "C" uint32_t ckpt_version(void) { return (1u << 16) | 0u; }

extern "C" void ckpt_profile_enable(int mask) { g_prof_on.store(mask & 0xF); }

extern "C" void ckpt_profile_reset(void) {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    for (auto &r : g_prof) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    g_prof.clear();
}

extern "C" ckpt_status ckpt_profile_read(int k, double *ms, uint64_t *launches) {
    if (!ms || !launches) return fail(CKPT_EINVAL, "NULL output");
    std::lock_guard<std::mutex> lk(g_prof_mu);
    double tot = 0.0;
    uint64_t n = 0;
    for (auto &r : g_prof) {
        if (r.k != k) continue;
        CK_CUDA(cudaEventSynchronize(r.b));
        float e = 0.f;
        CK_CUDA(cudaEventElapsedTime(&e, r.a, r.b));
        tot += e;
        ++n;
    }
    *ms = tot;
    *launches = n;
    return CKPT_OK;
}

extern "C" ckpt_status ckpt_profile_timeline(double *out, uint64_t cap, uint64_t *n_records) {
    if (!n_records || (!out && cap)) return fail(CKPT_EINVAL, "NULL output");
    std::lock_guard<std::mutex> lk(g_prof_mu);
    *n_records = g_prof.size();
    if (g_prof.empty()) return CKPT_OK;
    for (auto &r : g_prof) CK_CUDA(cudaEventSynchronize(r.b));
    cudaEvent_t base = g_prof[0].a;
    for (size_t i = 0; i < g_prof.size() && i < cap; ++i) {
        float s0 = 0.f, s1 = 0.f;
        CK_CUDA(cudaEventElapsedTime(&s0, base, g_prof[i].a));
        CK_CUDA(cudaEventElapsedTime(&s1, base, g_prof[i].b));
        out[3 * i] = g_prof[i].k;
        out[3 * i + 1] = s0;
        out[3 * i + 2] = s1;
    }
    return CKPT_OK;
}
