// tt_api.cu -- the C ABI of libtt.so (declared and documented in include/tt.h).
// Argument checking, tree upload / adoption, and kernel dispatch.  No compute
// happens here: every step of the traversal runs in the kernels of kern_*.cu.
#include <cuda_runtime.h>

#include <atomic>
#include <limits>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <unordered_map>
#include <vector>

#include "tt_internal.h"
#include "blob_cache.h"

// kern_bh_group.cu: return a tree's child-group array for reuse (device
// idle), or free it for good
void tt_bh_groups_release(void *grp);
void tt_bh_groups_discard(void *grp);

// build_nn_gpu.cu (declared here rather than in tt_internal.h)
int tt_build_nn_gpu_impl(const float *pts, long long n, int dim, int ld, void *stream, tt_blob_header *hdr,
                         void **blob);

namespace {

std::atomic<int> g_last_cuda_error{0};

tt_status cuda_fail(cudaError_t e) {
    g_last_cuda_error.store((int)e);
    if (e == cudaErrorMemoryAllocation) return TT_ERR_OOM;
    return TT_ERR_CUDA;
}

tt_status have_device() {
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n <= 0) {
        g_last_cuda_error.store((int)(e != cudaSuccess ? e : cudaErrorNoDevice));
        return TT_ERR_CUDA;
    }
    return TT_OK;
}

bool aligned(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

bool dim_supported(int d) { return (d >= 1 && d <= 8) || d == 16; }

// Default AUTO thresholds (levels of common tree path for lockstep), see
// tt_traverse_opts.auto_min_depth and DESIGN.md §4.5.
constexpr int kAutoBH = 3, kAutoPC = 255, kAutoKNN = 4, kAutoVP = 4, kAutoNN = 4;

// Shared-memory budgets for the staged top levels, per kernel (bytes/node):
// the budget trades staged levels against occupancy.
constexpr int kTopBH = 32 * 1024, kTopPC = 32 * 1024, kTopKNN = 16 * 1024, kTopVP = 4 * 1024, kTopNN = 8 * 1024;

// Canonical preorder id of every device node (for the stats hashes): the
// blob numbers the top levels level by level, so the map is rebuilt on the
// host from the records' child links (first child first, the Fig.2 order)
// once per tree and kept on the device.  Stats-only; synchronous.
tt_status ensure_preorder(tt_tree *t) {
    std::lock_guard<std::mutex> lk(t->grp_mu);
    if (t->d_pre) return TT_OK;
    const int64_t N = t->hdr.n_nodes;
    const size_t rb = (size_t)t->hdr.rec_bytes;
    std::vector<int32_t> rec;
    std::vector<int32_t> pre;
    try {
        rec.resize((size_t)N * rb / 4);
        pre.assign((size_t)N, -1);
    } catch (const std::bad_alloc &) {
        return TT_ERR_OOM;
    }
    cudaError_t e = cudaMemcpy(rec.data(), t->dev.rec, (size_t)N * rb, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_fail(e);
    const size_t w = rb / 4;  // int32 words per record
    auto at = [&](int64_t v, int f) { return rec[(size_t)v * w + (size_t)f]; };
    std::vector<int32_t> stk;
    stk.push_back(0);
    int32_t next = 0;
    std::vector<int32_t> kids;
    while (!stk.empty()) {
        const int32_t v = stk.back();
        stk.pop_back();
        if (v < 0 || v >= N || pre[(size_t)v] >= 0) return TT_ERR_INVALID_ARG;  // not a tree
        pre[(size_t)v] = next++;
        kids.clear();
        if (t->hdr.kind == TT_KIND_OCT) {  // first_child (word 4), then the skip chain (word 5)
            const int32_t end = at(v, 5);
            for (int32_t c = at(v, 4); c >= 0 && c != end; c = at(c, 5)) kids.push_back(c);
        } else {  // KD {left, right, ...}, VP {in, out, ...}, NN {left, right, ...}
            for (int f = 0; f < 2; ++f)
                if (at(v, f) >= 0) kids.push_back(at(v, f));
        }
        for (size_t i = kids.size(); i-- > 0;) stk.push_back(kids[i]);
    }
    if (next != N) return TT_ERR_INVALID_ARG;
    int32_t *d = nullptr;
    e = cudaMalloc((void **)&d, sizeof(int32_t) * (size_t)N);
    if (e == cudaSuccess) e = cudaMemcpy(d, pre.data(), sizeof(int32_t) * (size_t)N, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        if (d) cudaFree(d);
        return cuda_fail(e);
    }
    t->d_pre = d;
    return TT_OK;
}

tt_status setup_common(const tt_tree *t, int kind, int64_t n, const tt_traverse_opts *o, int default_amd,
                       int stage_bytes_per_node, int stage_budget, tt_common_params &c, tt_launch_cfg &cfg,
                       tt_stream s, bool allow_switch = false) {
    if (!t) return TT_ERR_INVALID_ARG;
    if (t->hdr.kind != kind) return TT_ERR_KIND_MISMATCH;
    if (n < 0 || n > (int64_t)0xffffffffu * 32) return TT_ERR_INVALID_ARG;
    std::memset(&c, 0, sizeof(c));
    c.tree = t->dev;
    if (const char *ev = std::getenv("TT_STAGE_BYTES")) stage_budget = std::atoi(ev);  // tuning sweeps only
    c.top_count = tt_stage_count(t->hdr, stage_bytes_per_node, stage_budget);
    c.height = t->hdr.height;
    c.n = n;
    c.mode = TT_MODE_AUTO;
    c.auto_min_depth = default_amd;
    for (int i = 0; i < 3; ++i) c.root_center[i] = t->hdr.root_center[i];
    c.root_side = t->hdr.root_side;
    cfg.block_threads = 256;
    cfg.ctas_per_sm = 0;
    if (const char *ev = std::getenv("TT_CTAS_PER_SM")) cfg.ctas_per_sm = std::atoi(ev);  // tuning sweeps only
    cfg.stream = s;
    cfg.variant = TT_VARIANT_AUTOROPES;
    if (o) {
        if (o->mode < TT_MODE_AUTO || o->mode > TT_MODE_INDEPENDENT) return TT_ERR_INVALID_ARG;
        c.mode = o->mode;
        if (o->auto_min_depth >= 0) c.auto_min_depth = o->auto_min_depth;
        c.order = o->order;
        if (o->stats) {
            c.st_visits = o->stats->visits;
            c.st_warp_fetches = o->stats->warp_fetches;
            c.st_warp_steps = o->stats->warp_steps;
            c.st_warp_mode = o->stats->warp_mode;
            c.st_hash = o->stats->visit_hash;
            c.st_set = o->stats->visit_set;
            c.st_point_tests = o->stats->point_tests;
            if (c.st_hash || c.st_set) {
                tt_status ps = ensure_preorder(const_cast<tt_tree *>(t));
                if (ps != TT_OK) return ps;
                c.pre = t->d_pre;
            }
        }
        if (o->block_threads != 0 && o->block_threads != 256) return TT_ERR_UNSUPPORTED;
        if (o->ctas_per_sm < 0) return TT_ERR_INVALID_ARG;
        if (o->ctas_per_sm > 0) cfg.ctas_per_sm = o->ctas_per_sm;
        if (o->variant != TT_VARIANT_AUTOROPES && o->variant != TT_VARIANT_RECURSIVE &&
            o->variant != TT_VARIANT_STACK && o->variant != TT_VARIANT_SPLIT && o->variant != TT_VARIANT_GROUPS &&
            o->variant != TT_VARIANT_ROPES)
            return TT_ERR_INVALID_ARG;
        if (o->variant == TT_VARIANT_RECURSIVE && o->mode == TT_MODE_LOCKSTEP) return TT_ERR_UNSUPPORTED;
        cfg.variant = o->variant;
        if (o->switch_below < 0 || o->switch_below > 33) return TT_ERR_INVALID_ARG;
        if (o->switch_below != 0 && (!allow_switch || o->variant != TT_VARIANT_AUTOROPES))
            return TT_ERR_UNSUPPORTED;  // kNN autoropes only
        c.switch_below = o->switch_below;
    }
    unsigned slot = __atomic_fetch_add(&const_cast<tt_tree *>(t)->slot_next, 1u, __ATOMIC_RELAXED) % TT_COUNTER_SLOTS;
    c.counter = t->d_counters + 2 * slot;
    return TT_OK;
}

// Tile-counter arrays of tree handles, recycled: a tree per time step would
// otherwise cudaMalloc / cudaFree 256 B per step (each cudaFree synchronises).
// (kept per device: a process that switches devices never gets another GPU's)
std::mutex g_ctr_mu;
std::vector<std::pair<uint32_t *, int>> g_ctr_free;

cudaError_t counters_take(uint32_t **out) {
    int dev = -1;
    cudaGetDevice(&dev);
    {
        std::lock_guard<std::mutex> lk(g_ctr_mu);
        for (size_t i = g_ctr_free.size(); i-- > 0;) {
            if (g_ctr_free[i].second != dev) continue;
            *out = g_ctr_free[i].first;
            g_ctr_free.erase(g_ctr_free.begin() + (long)i);
            return cudaSuccess;
        }
    }
    return cudaMalloc((void **)out, sizeof(uint32_t) * 2 * TT_COUNTER_SLOTS);
}

// caller guarantees the device is idle and current
void counters_release(uint32_t *c) {
    if (!c) return;
    int dev = -1;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(g_ctr_mu);
    if (g_ctr_free.size() >= 8) {
        cudaFree(c);
        return;
    }
    g_ctr_free.emplace_back(c, dev);
}

// Wrap a device blob (already in device memory, owned) into a tree handle.
tt_status adopt_blob(const tt_blob_header &h, void *d_blob, cudaStream_t cs, tt_tree **out) {
    tt_tree *t = new (std::nothrow) tt_tree();
    if (!t) return TT_ERR_OOM;
    t->hdr = h;
    t->bytes = (size_t)h.total;
    t->d_blob = d_blob;
    cudaError_t e = counters_take(&t->d_counters);
    if (e == cudaSuccess) e = cudaMemsetAsync(t->d_counters, 0, sizeof(uint32_t) * 2 * TT_COUNTER_SLOTS, cs);
    if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) {
        if (t->d_counters) counters_release(t->d_counters);
        delete t;
        return cuda_fail(e);
    }
    auto *base = static_cast<unsigned char *>(t->d_blob);
    t->dev.hdr_dev = reinterpret_cast<const tt_blob_header *>(base);
    t->dev.rec = base + h.off_rec;
    t->dev.box = h.off_box ? reinterpret_cast<const float *>(base + h.off_box) : nullptr;
    t->dev.pts = h.off_pts ? reinterpret_cast<const float *>(base + h.off_pts) : nullptr;
    t->dev.pid = h.off_pid ? reinterpret_cast<const int32_t *>(base + h.off_pid) : nullptr;
    t->dev.vpt = h.off_vpt ? reinterpret_cast<const float *>(base + h.off_vpt) : nullptr;
    t->dev.cbox = h.off_cbox ? reinterpret_cast<const float *>(base + h.off_cbox) : nullptr;
    t->slot_next = 0;
    *out = t;
    return TT_OK;
}

tt_status finish_launch(int err) {
    if (err == -1) return TT_ERR_UNSUPPORTED;
    if (err != 0) return cuda_fail((cudaError_t)err);
    return TT_OK;
}

// L2 persisting access-policy window over the start of a tree's hot records
// (the top levels come first in the blob and in the BH group array), for
// trees larger than L2 (configs[4]: BH-16M 0.8 GB, kNN-16M 0.6 GB; SURVEY
// §3(3)).  Opt-in, TT_L2_PERSIST_MB=<MiB of persisting L2>: the set-aside is
// device-wide and the window a stream attribute, so the library only touches
// them when asked.  Set for one launch, cleared after it is queued (kernels
// take the stream's policy at launch).  Measured on configs[4]:
// neutral (BH-16M 53.90 vs 53.89 ms, kNN-16M 918 vs 918 ms with the 79 MiB
// maximum set aside): both walks are issue-bound, not L2-miss-bound.
struct L2Window {
    cudaStream_t s = nullptr;
    bool on = false;
    L2Window(cudaStream_t st, const void *base, size_t bytes) : s(st) {
        static const long long mb = [] {
            const char *e = std::getenv("TT_L2_PERSIST_MB");
            return e ? std::atoll(e) : 0LL;
        }();
        if (mb <= 0 || !base || bytes == 0) return;
        cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
        if (cudaStreamIsCapturing(s, &cap) != cudaSuccess || cap != cudaStreamCaptureStatusNone) {
            cudaGetLastError();
            return;  // (attributes cannot change inside a CUDA-graph capture)
        }
        int dev = 0, max_persist = 0, max_win = 0;
        if (cudaGetDevice(&dev) != cudaSuccess) return;
        cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, dev);
        cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, dev);
        const size_t limit = std::min((size_t)mb << 20, (size_t)max_persist);
        if (limit == 0 || max_win <= 0) return;
        size_t cur = 0;
        cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
        if (cur != limit && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, limit) != cudaSuccess) {
            cudaGetLastError();
            return;
        }
        cudaStreamAttrValue v{};
        v.accessPolicyWindow.base_ptr = const_cast<void *>(base);
        v.accessPolicyWindow.num_bytes = std::min(bytes, (size_t)max_win);
        v.accessPolicyWindow.hitRatio = std::min(1.0f, (float)limit / (float)v.accessPolicyWindow.num_bytes);
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        const cudaError_t e = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
        on = e == cudaSuccess;
        static std::atomic<bool> told{false};
        if (!told.exchange(true)) {  // asked for explicitly: say (once) what was set
            std::fprintf(stderr, "tt: L2 persisting window %s: %zu MiB of %zu MiB, hit ratio %.2f\n",
                         on ? "set" : cudaGetErrorString(e), limit >> 20,
                         (size_t)v.accessPolicyWindow.num_bytes >> 20, v.accessPolicyWindow.hitRatio);
        }
        if (!on) cudaGetLastError();
    }
    ~L2Window() {
        if (!on) return;
        cudaStreamAttrValue v{};
        v.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
    }
};

}  // namespace

// Blob cache of the GPU builders.  A fresh cudaMalloc / cudaFree of a
// tens-of-MB blob per time step cost 1-10 ms each (and varied run to run);
// freed blobs are kept (at most kBlobCacheKeep) and reused by a later build
// whose blob fits in [bytes, 2 * bytes].
namespace {
struct BlobInfo {
    size_t bytes;
    int device;
};
std::mutex g_blob_mu;
std::unordered_map<void *, BlobInfo> g_blob_info;  // every cached-kind blob alive or free
std::vector<void *> g_blob_free;
constexpr size_t kBlobCacheKeep = 2;
int current_device() {
    int d = -1;
    cudaGetDevice(&d);
    return d;
}
}  // namespace

int tt_blob_take(size_t bytes, void **out) {
    const int dev = current_device();
    {
        std::lock_guard<std::mutex> lk(g_blob_mu);
        for (size_t i = 0; i < g_blob_free.size(); ++i) {
            void *p = g_blob_free[i];
            const BlobInfo &bi = g_blob_info[p];
            if (bi.device == dev && bi.bytes >= bytes && bi.bytes <= 2 * bytes) {
                g_blob_free.erase(g_blob_free.begin() + (long)i);
                *out = p;
                return cudaSuccess;
            }
        }
    }
    // slack (1/8, in 2-MiB steps) so the next time step's tree fits too
    const size_t alloc = ((bytes + bytes / 8) + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
    void *p = nullptr;
    cudaError_t e = cudaMalloc(&p, alloc);
    if (e) return e;
    std::lock_guard<std::mutex> lk(g_blob_mu);
    g_blob_info[p] = BlobInfo{alloc, dev};
    *out = p;
    return cudaSuccess;
}

bool tt_blob_is_cached_kind(void *blob) {
    std::lock_guard<std::mutex> lk(g_blob_mu);
    return g_blob_info.count(blob) != 0;
}

void tt_blob_release(void *blob) {
    if (!blob) return;
    std::lock_guard<std::mutex> lk(g_blob_mu);
    if (g_blob_free.size() >= kBlobCacheKeep) {
        // evict the oldest free blob, keep the newest
        void *old = g_blob_free.front();
        g_blob_free.erase(g_blob_free.begin());
        g_blob_info.erase(old);
        cudaFree(old);
    }
    g_blob_free.push_back(blob);
}

void tt_blob_discard(void *blob) {
    if (!blob) return;
    {
        std::lock_guard<std::mutex> lk(g_blob_mu);
        g_blob_info.erase(blob);  // a later cudaMalloc may return this address
    }
    cudaFree(blob);
}

extern "C" {

const char *tt_status_string(tt_status s) {
    switch (s) {
    case TT_OK: return "TT_OK";
    case TT_ERR_INVALID_ARG: return "TT_ERR_INVALID_ARG";
    case TT_ERR_CUDA: return "TT_ERR_CUDA";
    case TT_ERR_OOM: return "TT_ERR_OOM";
    case TT_ERR_TREE_TOO_DEEP: return "TT_ERR_TREE_TOO_DEEP";
    case TT_ERR_KIND_MISMATCH: return "TT_ERR_KIND_MISMATCH";
    case TT_ERR_UNSUPPORTED: return "TT_ERR_UNSUPPORTED";
    }
    return "TT_ERR_UNKNOWN";
}

int32_t tt_last_cuda_error(void) { return g_last_cuda_error.load(); }

const char *tt_build_info(void) {
    return "libtt sm_100a (-gencode arch=compute_100a,code=sm_100a); blob v1; top budget 32 KiB; block 256";
}

tt_status tt_tree_pack_size(const tt_tree_desc *d, size_t *bytes) {
    if (!bytes) return TT_ERR_INVALID_ARG;
    int st = TT_OK;
    size_t b = tt_pack_size_impl(d, &st);
    if (st != TT_OK) return (tt_status)st;
    *bytes = b;
    return TT_OK;
}

tt_status tt_tree_pack(const tt_tree_desc *d, void *host_blob, size_t bytes) {
    return (tt_status)tt_pack_impl(d, host_blob, bytes);
}

tt_status tt_tree_from_blob(const void *blob, size_t bytes, int32_t mem, tt_stream s, tt_tree **out) {
    if (!blob || !out || bytes < sizeof(tt_blob_header)) return TT_ERR_INVALID_ARG;
    if (mem != TT_MEM_HOST && mem != TT_MEM_DEVICE) return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    cudaStream_t cs = (cudaStream_t)s;
    tt_blob_header h;
    cudaError_t e;
    if (mem == TT_MEM_HOST) {
        std::memcpy(&h, blob, sizeof(h));
    } else {
        e = cudaMemcpyAsync(&h, blob, sizeof(h), cudaMemcpyDeviceToHost, cs);
        if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
        if (e != cudaSuccess) return cuda_fail(e);
    }
    if (h.magic != TT_BLOB_MAGIC || h.version != TT_BLOB_VERSION || h.total > bytes || h.n_nodes <= 0 ||
        h.top_count < 1 || h.top_count > h.n_nodes)
        return TT_ERR_INVALID_ARG;
    void *d_blob = nullptr;
    e = cudaMalloc(&d_blob, (size_t)h.total);
    if (e != cudaSuccess) return cuda_fail(e);
    e = cudaMemcpyAsync(d_blob, blob, (size_t)h.total,
                        mem == TT_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice, cs);
    if (e != cudaSuccess) {
        cudaFree(d_blob);
        return cuda_fail(e);
    }
    st = adopt_blob(h, d_blob, cs, out);
    if (st != TT_OK) cudaFree(d_blob);
    return st;
}

tt_status tt_build_oct_device(const float *bodies, int64_t n, tt_stream s, tt_tree **out) {
    return tt_build_oct_device_order(bodies, n, nullptr, s, out);
}

tt_status tt_build_oct_device_order(const float *bodies, int64_t n, uint32_t *order_out, tt_stream s, tt_tree **out) {
    if (!bodies || !out || n <= 0 || n > INT32_MAX / 3 || !aligned(bodies, 16)) return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    tt_blob_header h;
    void *d_blob = nullptr;
    const int e = tt_build_oct_gpu_impl(bodies, n, s, &h, &d_blob, order_out);
    if (e) return cuda_fail((cudaError_t)e);
    if (h.height > TT_MAX_HEIGHT) {
        tt_blob_discard(d_blob);
        return TT_ERR_TREE_TOO_DEEP;
    }
    st = adopt_blob(h, d_blob, (cudaStream_t)s, out);
    if (st != TT_OK) tt_blob_discard(d_blob);
    return st;
}

tt_status tt_build_kd_device(const float *pts, int64_t n, int32_t dim, int32_t ld, int32_t leaf_size, tt_stream s,
                             tt_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim || leaf_size <= 0)
        return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    tt_blob_header h;
    void *d_blob = nullptr;
    const int e = tt_build_kd_gpu_impl(pts, n, dim, ld, leaf_size, s, &h, &d_blob);
    if (e) return cuda_fail((cudaError_t)e);
    st = adopt_blob(h, d_blob, (cudaStream_t)s, out);
    if (st != TT_OK) tt_blob_discard(d_blob);
    return st;
}

tt_status tt_build_vp_device(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_stream s, tt_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim)
        return TT_ERR_INVALID_ARG;
    if (!dim_supported(dim)) return TT_ERR_UNSUPPORTED;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    tt_blob_header h;
    void *d_blob = nullptr;
    const int e = tt_build_vp_gpu_impl(pts, n, dim, ld, s, &h, &d_blob);
    if (e) return cuda_fail((cudaError_t)e);
    if (h.height > TT_MAX_HEIGHT) {
        tt_blob_discard(d_blob);
        return TT_ERR_TREE_TOO_DEEP;
    }
    st = adopt_blob(h, d_blob, (cudaStream_t)s, out);
    if (st != TT_OK) tt_blob_discard(d_blob);
    return st;
}

tt_status tt_build_nn_device(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_stream s, tt_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim)
        return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    tt_blob_header h;
    void *d_blob = nullptr;
    const int e = tt_build_nn_gpu_impl(pts, n, dim, ld, s, &h, &d_blob);
    if (e) return cuda_fail((cudaError_t)e);
    if (h.height > TT_MAX_HEIGHT) {
        tt_blob_discard(d_blob);
        return TT_ERR_TREE_TOO_DEEP;
    }
    st = adopt_blob(h, d_blob, (cudaStream_t)s, out);
    if (st != TT_OK) tt_blob_discard(d_blob);
    return st;
}

tt_status tt_tree_download(const tt_tree *t, void *host_blob, size_t bytes) {
    if (!t || !host_blob || bytes < t->bytes) return TT_ERR_INVALID_ARG;
    const cudaError_t e = cudaMemcpy(host_blob, t->d_blob, t->bytes, cudaMemcpyDeviceToHost);
    return e == cudaSuccess ? TT_OK : cuda_fail(e);
}

tt_status tt_tree_copy_blob(const tt_tree *t, void *dst, size_t bytes, int32_t mem, tt_stream s) {
    if (!t || !dst || bytes < t->bytes || (mem != TT_MEM_HOST && mem != TT_MEM_DEVICE)) return TT_ERR_INVALID_ARG;
    cudaError_t e;
    if (mem == TT_MEM_HOST) {
        e = cudaMemcpyAsync(dst, t->d_blob, t->bytes, cudaMemcpyDeviceToHost, (cudaStream_t)s);
        if (e == cudaSuccess) e = cudaStreamSynchronize((cudaStream_t)s);
    } else {
        e = cudaMemcpyAsync(dst, t->d_blob, t->bytes, cudaMemcpyDeviceToDevice, (cudaStream_t)s);
    }
    return e == cudaSuccess ? TT_OK : cuda_fail(e);
}

tt_status tt_tree_upload(const tt_tree_desc *d, tt_stream s, tt_tree **out) {
    if (!out) return TT_ERR_INVALID_ARG;
    size_t bytes = 0;
    tt_status st = tt_tree_pack_size(d, &bytes);
    if (st != TT_OK) return st;
    st = have_device();
    if (st != TT_OK) return st;
    void *host = nullptr;
    cudaError_t e = cudaMallocHost(&host, bytes);
    if (e != cudaSuccess) return cuda_fail(e);
    st = tt_tree_pack(d, host, bytes);
    if (st == TT_OK) st = tt_tree_from_blob(host, bytes, TT_MEM_HOST, s, out);
    cudaFreeHost(host);
    return st;
}

tt_status tt_tree_free(tt_tree *t) {
    if (!t) return TT_OK;
    // Buffers are recycled (blob of a GPU-built tree, tile counters, child
    // groups) only once the device is known idle; if the synchronisation
    // fails they are freed instead, never handed to a later tree.
    const cudaError_t e1 = cudaDeviceSynchronize();
    const bool idle = e1 == cudaSuccess;
    if (tt_blob_is_cached_kind(t->d_blob)) {
        if (idle) tt_blob_release(t->d_blob);
        else tt_blob_discard(t->d_blob);
    } else {
        cudaFree(t->d_blob);
    }
    if (idle) counters_release(t->d_counters);
    else cudaFree(t->d_counters);
    if (idle) tt_bh_groups_release(t->d_grp);
    else tt_bh_groups_discard(t->d_grp);
    if (t->grp_ready) cudaEventDestroy(t->grp_ready);
    if (t->d_pre) cudaFree(t->d_pre);
    delete t;
    return idle ? TT_OK : cuda_fail(e1);
}

tt_status tt_tree_get_info(const tt_tree *t, tt_tree_info *o) {
    if (!t || !o) return TT_ERR_INVALID_ARG;
    o->kind = t->hdr.kind;
    o->dim = t->hdr.dim;
    o->dim_padded = t->hdr.dp;
    o->height = t->hdr.height;
    o->n_nodes = t->hdr.n_nodes;
    o->n_points = t->hdr.n_points;
    o->top_levels = t->hdr.top_levels;
    o->top_count = t->hdr.top_count;
    o->device_bytes = (int64_t)t->bytes;
    o->device_blob = t->d_blob;
    return TT_OK;
}

tt_status tt_sort_points(const tt_tree *t, const float *pts, int64_t n, int32_t ld, uint32_t *perm_out,
                         uint64_t *keys_out, tt_stream s) {
    if (!t || n < 0 || n > INT32_MAX) return TT_ERR_INVALID_ARG;
    if (n == 0) return TT_OK;
    if (!pts || !perm_out) return TT_ERR_INVALID_ARG;
    if (ld < (t->hdr.kind == TT_KIND_OCT ? 3 : t->hdr.dim)) return TT_ERR_INVALID_ARG;
    if (t->hdr.kind != TT_KIND_OCT && !dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    int e = tt_launch_sort(t, pts, n, ld, perm_out, keys_out, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

tt_status tt_schedule_tiles(const tt_tree *t, const float *pts, int64_t n, int32_t ld, const uint32_t *perm_in,
                            uint32_t *perm_out, tt_stream s) {
    if (!t || n < 0 || n > INT32_MAX) return TT_ERR_INVALID_ARG;
    if (n == 0) return TT_OK;
    if (!pts || !perm_in || !perm_out) return TT_ERR_INVALID_ARG;
    if (ld < (t->hdr.kind == TT_KIND_OCT ? 3 : t->hdr.dim)) return TT_ERR_INVALID_ARG;
    if (t->hdr.kind != TT_KIND_OCT && !dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    const int tile = t->hdr.kind == TT_KIND_OCT ? 32 * TT_BH_POINTS_PER_LANE : 32;
    int e = tt_launch_schedule(t, pts, n, ld, perm_in, perm_out, tile, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

tt_status tt_traverse_bh(const tt_tree *t, const float *bodies, const int32_t *self_ids, int64_t n, float theta,
                         float eps, float *acc_out, const tt_traverse_opts *opts, tt_stream s) {
    tt_bh_params p;
    tt_launch_cfg cfg;
    tt_status st = setup_common(t, TT_KIND_OCT, n, opts, kAutoBH, 32, kTopBH, p.c, cfg, s);
    if (st != TT_OK) return st;
    if (!(theta >= 0.0f) || !(eps >= 0.0f)) return TT_ERR_INVALID_ARG;
    if (n == 0) return TT_OK;
    if (!bodies || !acc_out || !aligned(bodies, 16) || !aligned(acc_out, 16)) return TT_ERR_INVALID_ARG;
    st = have_device();
    if (st != TT_OK) return st;
    if (cfg.variant == TT_VARIANT_SPLIT) return TT_ERR_UNSUPPORTED;  // PC only
    // BH default: lockstep warps walk by child groups (kern_bh_group.cu);
    // TT_VARIANT_ROPES keeps the per-node lockstep walk over ropes (kern_bh.cu)
    // (the child-group stack holds 8 entries per level: deeper custom trees,
    // or trees with more than 8 cell children per node -- tt_blob_header
    // oct_flags -- take the stackless per-node walk, or fail if groups were
    // requested; more than 8 children in all (depth-32 buckets) are staged 8
    // at a time by the WIDE kernel)
    const bool groups_shape = 8 * (t->hdr.height + 2) <= 320 &&  // kStackPerWarp of kern_bh_group.cu
                              (t->hdr.oct_flags & TT_OCT_FEW_CELL_KIDS);
    const bool groups_size = t->hdr.n_nodes < (1LL << 27);  // 32-bit byte offsets into the group array
    const bool groups_fit = groups_shape && groups_size;
    const bool wide = !(t->hdr.oct_flags & TT_OCT_NARROW);
    if (cfg.variant == TT_VARIANT_AUTOROPES) cfg.variant = groups_fit ? TT_VARIANT_GROUPS : TT_VARIANT_ROPES;
    if (cfg.variant == TT_VARIANT_GROUPS && !groups_shape) return TT_ERR_TREE_TOO_DEEP;
    if (cfg.variant == TT_VARIANT_GROUPS && !groups_size) return TT_ERR_UNSUPPORTED;
    if (cfg.variant == TT_VARIANT_GROUPS) {
        tt_tree *mt = const_cast<tt_tree *>(t);
        std::lock_guard<std::mutex> lk(mt->grp_mu);
        if (!mt->d_grp) {
            void *g = nullptr;
            int e = tt_bh_groups_build(t->dev.rec, t->hdr.n_nodes, t->hdr.n_points, s, &g);
            if (e) return cuda_fail((cudaError_t)e);
            // launches on other streams wait for the build (queued on s)
            if (!mt->grp_ready) e = cudaEventCreateWithFlags(&mt->grp_ready, cudaEventDisableTiming);
            if (!e) e = cudaEventRecord(mt->grp_ready, (cudaStream_t)s);
            if (e) {
                cudaStreamSynchronize((cudaStream_t)s);
                tt_bh_groups_release(g);
                return cuda_fail((cudaError_t)e);
            }
            mt->d_grp = g;
            mt->grp_stream = s;
            mt->grp_done = false;
        }
        // a launch on another stream waits for the build until it is known
        // complete (then no further calls: nothing to wait for, and no event
        // wait inside a later CUDA-graph capture)
        if (!mt->grp_done) {
            const cudaError_t q = cudaEventQuery(mt->grp_ready);
            if (q == cudaSuccess) {
                mt->grp_done = true;
            } else if (q == cudaErrorNotReady) {
                if (s != mt->grp_stream) {
                    const cudaError_t e = cudaStreamWaitEvent((cudaStream_t)s, mt->grp_ready, 0);
                    if (e) return cuda_fail(e);
                }
            } else {
                return cuda_fail(q);
            }
        }
    }
    p.bodies = reinterpret_cast<const float4 *>(bodies);
    p.self_ids = self_ids;
    // dsq_root = fl32(side^2 / theta^2) in fp64 (reading R8); theta = 0 -> +inf
    if (theta == 0.0f) {
        p.dsq_root = std::numeric_limits<float>::infinity();
    } else {
        const double th = (double)theta;
        p.dsq_root = (float)((t->hdr.root_side * t->hdr.root_side) / (th * th));
    }
    p.eps2 = eps * eps;
    p.acc = reinterpret_cast<float4 *>(acc_out);
    const L2Window l2w((cudaStream_t)s, cfg.variant == TT_VARIANT_GROUPS ? t->d_grp : t->dev.rec,
                       (size_t)t->hdr.n_nodes * sizeof(tt_oct_rec));
    return finish_launch(cfg.variant == TT_VARIANT_RECURSIVE ? tt_launch_bh_recursive(p, cfg)
                         : cfg.variant == TT_VARIANT_STACK   ? tt_launch_bh_stack(p, cfg)
                         : cfg.variant == TT_VARIANT_GROUPS  ? tt_launch_bh_group(p, t->d_grp, t->hdr.n_nodes, t->hdr.n_points, wide, cfg)
                                                             : tt_launch_bh(p, cfg));  // ROPES
}

tt_status tt_traverse_pc(const tt_tree *t, const float *q, int64_t n, int32_t ld, float radius, uint32_t *count_out,
                         const tt_traverse_opts *opts, tt_stream s) {
    if (!t) return TT_ERR_INVALID_ARG;  // (the staging size below reads t->hdr)
    tt_pc_params p;
    tt_launch_cfg cfg;
    tt_status st = setup_common(t, TT_KIND_KD, n, opts, kAutoPC, 32 + 8 * t->hdr.dp, kTopPC, p.c, cfg, s);
    if (st != TT_OK) return st;
    if (!(radius >= 0.0f)) return TT_ERR_INVALID_ARG;
    if (ld < t->hdr.dim) return TT_ERR_INVALID_ARG;
    if (!dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    if (n == 0) return TT_OK;
    if (!q || !count_out) return TT_ERR_INVALID_ARG;
    st = have_device();
    if (st != TT_OK) return st;
    p.q = q;
    p.ld = ld;
    p.r2 = radius * radius;  // rn(r*r), reading R1
    p.count = count_out;
    if (cfg.variant == TT_VARIANT_GROUPS || cfg.variant == TT_VARIANT_ROPES) return TT_ERR_UNSUPPORTED;  // BH only
    // AUTO with the default threshold: a launch with fewer 32-point tiles than
    // resident warps (148 SMs x 32) cannot fill the GPU one lane per point --
    // it is the latency of its longest walks -- so each point's walk is split
    // over 16 lanes (TT_VARIANT_SPLIT; configs[0]: 0.10 vs
    // 0.18 ms)
    const bool default_amd = !opts || opts->auto_min_depth < 0;
    if (cfg.variant == TT_VARIANT_AUTOROPES && p.c.mode == TT_MODE_AUTO && default_amd) {
        int dev = 0, nsm = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);  // the current device's
        if ((n + 31) / 32 < (int64_t)nsm * 32) cfg.variant = TT_VARIANT_SPLIT;
    }
    return finish_launch(cfg.variant == TT_VARIANT_RECURSIVE ? tt_launch_pc_recursive(p, t->hdr.dim, cfg)
                         : cfg.variant == TT_VARIANT_STACK   ? tt_launch_pc_stack(p, t->hdr.dim, cfg)
                         : cfg.variant == TT_VARIANT_SPLIT   ? tt_launch_pc_split(p, t->hdr.dim, cfg)
                                                             : tt_launch_pc(p, t->hdr.dim, cfg));
}

tt_status tt_traverse_knn(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t k, int32_t *idx_out,
                          float *d2_out, const tt_traverse_opts *opts, tt_stream s) {
    if (!t) return TT_ERR_INVALID_ARG;  // (the staging size below reads t->hdr)
    tt_knn_params p;
    tt_launch_cfg cfg;
    tt_status st = setup_common(t, TT_KIND_KD, n, opts, kAutoKNN, 32 + 16 * t->hdr.dp, kTopKNN, p.c, cfg, s, true);
    if (st != TT_OK) return st;
    if (k < 1) return TT_ERR_INVALID_ARG;
    if (k > TT_MAX_K) return TT_ERR_UNSUPPORTED;
    if (ld < t->hdr.dim) return TT_ERR_INVALID_ARG;
    if (!dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    if (n == 0) return TT_OK;
    if (!q || !idx_out || !d2_out) return TT_ERR_INVALID_ARG;
    st = have_device();
    if (st != TT_OK) return st;
    p.q = q;
    p.ld = ld;
    p.k = k;
    p.idx = idx_out;
    p.d2 = d2_out;
    if (cfg.variant == TT_VARIANT_STACK || cfg.variant == TT_VARIANT_SPLIT || cfg.variant == TT_VARIANT_GROUPS ||
        cfg.variant == TT_VARIANT_ROPES)
        return TT_ERR_UNSUPPORTED;  // guided kernels already keep rope stacks; SPLIT is PC, GROUPS / ROPES BH only
    const L2Window l2w((cudaStream_t)s, t->dev.rec, (size_t)t->hdr.n_nodes * sizeof(tt_kd_rec));
    return finish_launch(cfg.variant == TT_VARIANT_RECURSIVE ? tt_launch_knn_recursive(p, t->hdr.dim, cfg)
                                                            : tt_launch_knn(p, t->hdr.dim, cfg));
}

tt_status tt_traverse_vp(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t *idx_out, float *d2_out,
                         const tt_traverse_opts *opts, tt_stream s) {
    if (!t) return TT_ERR_INVALID_ARG;  // (the staging size below reads t->hdr)
    tt_vp_params p;
    tt_launch_cfg cfg;
    tt_status st = setup_common(t, TT_KIND_VP, n, opts, kAutoVP, 16 + 4 * t->hdr.dp, kTopVP, p.c, cfg, s);
    if (st != TT_OK) return st;
    if (ld < t->hdr.dim) return TT_ERR_INVALID_ARG;
    if (!dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    if (n == 0) return TT_OK;
    if (!q || !idx_out || !d2_out) return TT_ERR_INVALID_ARG;
    st = have_device();
    if (st != TT_OK) return st;
    p.q = q;
    p.ld = ld;
    p.idx = idx_out;
    p.d2 = d2_out;
    if (cfg.variant == TT_VARIANT_STACK || cfg.variant == TT_VARIANT_SPLIT || cfg.variant == TT_VARIANT_GROUPS ||
        cfg.variant == TT_VARIANT_ROPES)
        return TT_ERR_UNSUPPORTED;  // guided kernels already keep rope stacks; SPLIT is PC, GROUPS / ROPES BH only
    return finish_launch(cfg.variant == TT_VARIANT_RECURSIVE ? tt_launch_vp_recursive(p, t->hdr.dim, cfg)
                                                            : tt_launch_vp(p, t->hdr.dim, cfg));
}

tt_status tt_traverse_nn(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t *idx_out, float *d2_out,
                         const tt_traverse_opts *opts, tt_stream s) {
    if (!t) return TT_ERR_INVALID_ARG;  // (the staging size below reads t->hdr)
    tt_nn_params p;
    tt_launch_cfg cfg;
    tt_status st = setup_common(t, TT_KIND_NN, n, opts, kAutoNN, 16 + 12 * t->hdr.dp, kTopNN, p.c, cfg, s);
    if (st != TT_OK) return st;
    if (ld < t->hdr.dim) return TT_ERR_INVALID_ARG;
    if (!dim_supported(t->hdr.dim)) return TT_ERR_UNSUPPORTED;
    if (cfg.variant != TT_VARIANT_AUTOROPES) return TT_ERR_UNSUPPORTED;  // no recursive / stack variant for NN
    if (n == 0) return TT_OK;
    if (!q || !idx_out || !d2_out) return TT_ERR_INVALID_ARG;
    st = have_device();
    if (st != TT_OK) return st;
    p.q = q;
    p.ld = ld;
    p.idx = idx_out;
    p.d2 = d2_out;
    return finish_launch(tt_launch_nn(p, t->hdr.dim, cfg));
}

tt_status tt_diag_chase(const void *records, int64_t nrec, int32_t per_lane, int64_t steps, int32_t ctas_per_sm,
                        uint32_t *sink, tt_stream s) {
    if (!records || !sink || nrec <= 0 || nrec > INT32_MAX || steps < 0 || ctas_per_sm < 0 ||
        (per_lane != 0 && per_lane != 1) || !aligned(records, 32))
        return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    const int e = tt_launch_chase(records, nrec, steps, per_lane, ctas_per_sm, sink, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

tt_status tt_diag_l2read(const void *buf, int64_t bytes, int32_t reps, uint32_t *sink, tt_stream s) {
    if (!buf || !sink || bytes < 32 || reps < 1 || !aligned(buf, 32)) return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    const int e = tt_launch_l2read(buf, bytes, reps, sink, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

tt_status tt_kick_drift(float *bodies, float *vel, const float *acc, int64_t n, float dt_kick, float dt_drift,
                        tt_stream s) {
    if (n < 0) return TT_ERR_INVALID_ARG;
    if (n == 0) return TT_OK;
    if (!bodies || !vel || !acc || !aligned(bodies, 16) || !aligned(vel, 16) || !aligned(acc, 16))
        return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    const int e = tt_launch_kick_drift(bodies, vel, acc, n, dt_kick, dt_drift, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

tt_status tt_kick_drift_permuted(const float *bodies, const float *vel, const float *acc, const int32_t *perm,
                                 const int32_t *ids, int64_t n, float dt_kick, float dt_drift, float *bodies_out,
                                 float *vel_out, int32_t *ids_out, tt_stream s) {
    if (n < 0) return TT_ERR_INVALID_ARG;
    if (n == 0) return TT_OK;
    if (!bodies || !vel || !acc || !perm || !bodies_out || !vel_out || (ids && !ids_out) || !aligned(bodies, 16) ||
        !aligned(vel, 16) || !aligned(acc, 16) || !aligned(bodies_out, 16) || !aligned(vel_out, 16))
        return TT_ERR_INVALID_ARG;
    tt_status st = have_device();
    if (st != TT_OK) return st;
    const int e = tt_launch_kick_drift_permuted(bodies, vel, acc, perm, ids, n, dt_kick, dt_drift, bodies_out, vel_out,
                                                ids ? ids_out : nullptr, s);
    return e ? cuda_fail((cudaError_t)e) : TT_OK;
}

}  // extern "C"
