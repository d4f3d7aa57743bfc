// tt_internal.h -- device layout of a packed tree and the launch parameter
// blocks shared between the C-ABI layer (tt_api.cu) and the kernels.
// Product code only; nothing here is shared with oracle/.
#pragma once

#include <cstddef>
#include <cstdint>
#include <mutex>

#include <cuda_runtime_api.h>
#include <vector_types.h>

#include "../../include/tt.h"

#define TT_BLOB_MAGIC 0x31425454u /* "TTB1" */
#define TT_BLOB_VERSION 2u
#define TT_END (-1)               /* rope past the last node = end of traversal */
#define TT_TOP_BYTES (32 * 1024)  /* shared-memory budget for the staged top levels */
#define TT_COUNTER_SLOTS 256      /* tile-scheduler counter slots per tree */
#define TT_TOP_LEVELS_MAX 32      /* levels tracked in the header's level_prefix */
// tt_blob_header.oct_flags (what the child-group BH walk may assume):
#define TT_OCT_NARROW 1           /* height <= 32 and every node has <= 8 children */
#define TT_OCT_FEW_CELL_KIDS 2    /* every node has <= 8 children that are cells    */

// ---------------------------------------------------------------------------
// Packed node records: one 32-byte sector per node, two 128-bit field groups
// split by use (Fig.9b lines 9/11).
//
// OCT: g = {com.x, com.y, com.z, mass}   -- read at every visit
//      t = {first_child | -1, skip | END, body | -1, level}
// KD:  t = {left | -1, right | -1, skip | END, level}
//      u = {split (float bits), split_dim | -1, pbegin, pcount}
//      + box[2*dp] floats (lo[dp], hi[dp]) in a separate array
// VP:  t = {in | -1, out | -1, r_in_max (float bits), r_out_min (float bits)}
//      + vpt[dp] vantage coordinates and pid (vantage point's original id)
// NN:  t = {left | -1, right | -1, split (float bits), split_dim | -1}
//      + box[2*dp] tight subtree box, vpt[dp] the node's point, pid (its id)
// ---------------------------------------------------------------------------
struct alignas(16) tt_oct_rec {
    float gx, gy, gz, gm;
    int32_t first_child, skip, body, level;
};
struct alignas(16) tt_kd_rec {
    int32_t left, right, skip, level;
    float split;
    int32_t dim, pbegin, pcount;
};
struct alignas(16) tt_vp_rec {
    int32_t in, out;
    float r_in_max, r_out_min;
};
static_assert(sizeof(tt_oct_rec) == 32, "oct record = one 32-B sector");
static_assert(sizeof(tt_kd_rec) == 32, "kd record = one 32-B sector");
struct alignas(16) tt_nn_rec {
    int32_t left, right;
    float split;
    int32_t dim;
};
static_assert(sizeof(tt_vp_rec) == 16, "vp header = one 128-bit group");
static_assert(sizeof(tt_nn_rec) == 16, "nn header = one 128-bit group");

// Blob = header + sections, every section 256-byte aligned, offsets relative to
// the blob start (position independent: the blob can be broadcast as bytes).
struct tt_blob_header {
    uint32_t magic, version;
    int32_t kind, dim, dp, height, leaf_size, top_levels, top_count;
    int32_t oct_flags;  // OCT: TT_OCT_* bits below (0 for other kinds / unknown)
    // level_prefix[L] = number of nodes with level < L, for L <= top_levels; the
    // top region is numbered level by level, so its first level_prefix[L]
    // records are exactly the top L levels (each kernel stages what fits).
    int32_t level_prefix[TT_TOP_LEVELS_MAX + 1], pad1;
    int64_t n_nodes, n_points;
    double root_center[3], root_side;
    uint64_t off_rec, off_box, off_pts, off_pid, off_vpt, total;
    uint64_t rec_bytes; // bytes per record in the rec section (32 or 16)
    uint64_t off_cbox;  // KD: children's boxes per node [n][2 children][lo dp, hi dp] (0 = leaf)
};

// Device-side view of an uploaded tree.
struct tt_dev_tree {
    const tt_blob_header *hdr_dev;
    const void *rec;      // records, top nodes first
    const float *box;     // KD, NN: [n_nodes][2*dp]
    const float *pts;     // KD: [n_points][dp] tree order
    const int32_t *pid;   // KD: [n_points]; VP, NN: [n_nodes]
    const float *vpt;     // VP, NN: [n_nodes][dp] the node's point
    const float *cbox;    // KD: [n_nodes][2][2*dp] boxes of the two children
};

// ---------------------------------------------------------------------------
// Launch parameter blocks (passed by value to the kernels).
struct tt_common_params {
    tt_dev_tree tree;
    int32_t top_count;     // nodes staged in shared memory
    int32_t height;
    int64_t n;             // points in this launch
    const uint32_t *order; // nullable
    int32_t mode;          // tt_mode
    int32_t auto_min_depth;
    int32_t switch_below;  // dynamic L->N switching threshold (kNN), 0 = never
    uint32_t *counter;     // [2] tile scheduler: next tile, finished CTAs
    // stats (nullable)
    uint32_t *st_visits, *st_warp_fetches, *st_warp_steps;
    uint8_t *st_warp_mode;
    // per-point visit hashes (nullable; `pre` = canonical preorder id of every
    // device node, set whenever a hash is requested) and leaf-point tests
    uint64_t *st_hash, *st_set;
    const int32_t *pre;
    uint32_t *st_point_tests;
    // root cube (OCT AUTO mode)
    double root_center[3], root_side;
};

struct tt_bh_params {
    tt_common_params c;
    const float4 *bodies;
    const int32_t *self_ids;
    float dsq_root, eps2;
    float4 *acc;
};

struct tt_pc_params {
    tt_common_params c;
    const float *q;
    int32_t ld;
    float r2;
    uint32_t *count;
};

struct tt_knn_params {
    tt_common_params c;
    const float *q;
    int32_t ld, k;
    int32_t *idx;
    float *d2;
};

struct tt_vp_params {
    tt_common_params c;
    const float *q;
    int32_t ld;
    int32_t *idx;
    float *d2;
};

// NN: same argument block as VP
typedef tt_vp_params tt_nn_params;

// Host-side handle.
struct tt_tree {
    tt_blob_header hdr;
    void *d_blob;
    size_t bytes;
    tt_dev_tree dev;
    uint32_t *d_counters;  // [TT_COUNTER_SLOTS][2]
    unsigned slot_next;
    int32_t *d_pre = nullptr;  // canonical preorder id of every device node (stats hashes), built on first use
    void *d_grp = nullptr;  // OCT: child-group records (kern_bh_group.cu), built on first use
    cudaEvent_t grp_ready = nullptr;  // recorded on the stream of that build
    tt_stream grp_stream = nullptr;   // the stream of that build
    bool grp_done = false;            // the build is known complete
    std::mutex grp_mu;
};

// Launchers (kernels/*.cu).  Return a cudaError_t as int.
struct tt_launch_cfg {
    int block_threads;
    int ctas_per_sm;
    void *stream;
    int variant;  // tt_variant
};
int tt_launch_bh(const tt_bh_params &p, const tt_launch_cfg &cfg);
int tt_launch_pc(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_knn(const tt_knn_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_vp(const tt_vp_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_nn(const tt_nn_params &p, int dim, const tt_launch_cfg &cfg);
// naive recursive baseline (kern_recursive.cu)
int tt_launch_bh_recursive(const tt_bh_params &p, const tt_launch_cfg &cfg);
int tt_launch_pc_recursive(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_knn_recursive(const tt_knn_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_vp_recursive(const tt_vp_params &p, int dim, const tt_launch_cfg &cfg);
// explicit rope-stack variant, unguided kernels (kern_stack.cu)
int tt_launch_bh_stack(const tt_bh_params &p, const tt_launch_cfg &cfg);
// lockstep walk by child groups (kern_bh_group.cu)
int tt_bh_groups_build(const void *rec, long long nn, long long np, void *stream, void **grp_out);
int tt_launch_bh_group(const tt_bh_params &p, const void *grp, long long nn, long long np, bool wide,
                       const tt_launch_cfg &cfg);
int tt_launch_pc_stack(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg);
// one point's traversal split over a 16-lane group (kern_pc_split.cu)
int tt_launch_pc_split(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg);
int tt_launch_sort(const tt_tree *t, const float *pts, int64_t n, int32_t ld, uint32_t *perm,
                   uint64_t *keys_out, void *stream);
int tt_launch_schedule(const tt_tree *t, const float *pts, int64_t n, int32_t ld, const uint32_t *perm_in,
                       uint32_t *perm_out, int tile, void *stream);

// Nodes of the largest level-complete top prefix whose staged bytes fit `budget`.
inline int tt_stage_count(const tt_blob_header &h, int bytes_per_node, int budget) {
    int best = 1;  // the root always fits
    for (int L = 1; L <= h.top_levels; ++L) {
        const long long c = h.level_prefix[L];
        if (c * bytes_per_node <= budget) best = (int)c;
        else break;
    }
    return best;
}

// GPU oct-tree build (build_oct_gpu.cu): fills the host header copy and a
// cudaMalloc'd device blob; returns a cudaError_t.
int tt_build_oct_gpu_impl(const float *bodies, long long n, void *stream, tt_blob_header *hdr, void **blob,
                          unsigned *order_out = nullptr);

int tt_launch_kick_drift(float *x, float *v, const float *a, long long n, float dtk, float dtd, void *stream);
int tt_launch_kick_drift_permuted(const float *x, const float *v, const float *a, const int *perm, const int *ids,
                                  long long n, float dtk, float dtd, float *xo, float *vo, int *ido, void *stream);

int tt_build_kd_gpu_impl(const float *pts, long long n, int dim, int ld, int leaf, void *stream, tt_blob_header *hdr,
                         void **blob);

int tt_build_vp_gpu_impl(const float *pts, long long n, int dim, int ld, void *stream, tt_blob_header *hdr,
                         void **blob);

// Diagnostics (kern_diag.cu): dependent 32-B record chase.
int tt_launch_l2read(const void *buf, long long bytes, int reps, unsigned *sink, void *stream);
int tt_launch_chase(const void *rec, long long nrec, long long steps, int per_lane, int ctas_per_sm, unsigned *sink,
                    void *stream);

// Default mempool keeps freed stream-ordered scratch across syncs (kern_sort.cu).
void tt_keep_pool_memory();

// Host helpers (host_build.cpp / pack.cpp)
size_t tt_pack_size_impl(const tt_tree_desc *d, int *status);
int tt_pack_impl(const tt_tree_desc *d, void *blob, size_t bytes);
