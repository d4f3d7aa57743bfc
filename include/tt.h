/*
 * tt.h -- C ABI of the B200-native batched point-by-tree traversal library
 * (libtt.so), after Goldfarb, Jo & Kulkarni, "General Transformations for GPU
 * Execution of Tree Traversals", SC'13.  "P:Lx-y" cites /root/reference/PAPER.md.
 *
 * The method (Fig.1): many independent points each walk one shared
 * tree; at every node a truncation test either stops the walk below that node
 * or the point is updated and recurses into the children.  The library
 * implements the paper's GPU form of it:
 *   - autoropes (§3): the recursion becomes an iterative preorder
 *     walk -- stackless via per-node ropes ("skip") for unguided traversals,
 *     or an explicit rope stack (children pushed in reverse call order,
 *     non-invariant arguments pushed with the node) for guided ones;
 *   - lockstep traversal (§4.2, Fig.8): a warp walks the union of
 *     its 32 points' traversals under an active mask (ballot), one node fetch
 *     per warp; guided traversals reduce their call sets per warp by majority
 *     vote (§4.3);
 *   - point sorting (§4.4) and the choice between lockstep and
 *     independent traversal, made here per warp.
 *
 * Conventions (all entry points):
 *   - Every call returns tt_status; TT_OK == 0, errors are negative.  Calls
 *     never abort or throw.  Argument errors are detected before any work.
 *   - Traversal / sort calls are asynchronous on the caller's stream
 *     (tt_stream = cudaStream_t; 0 = legacy default stream).  Device faults
 *     surface at the caller's next synchronisation (and via tt_last_cuda_error).
 *   - Point, order and result buffers are caller-owned DEVICE memory; the
 *     library never frees them.  There is no CPU fallback: without a CUDA
 *     device every traversal returns TT_ERR_CUDA.
 *   - Results are written in the caller's original point order: result i
 *     belongs to point i, whether or not an `order` permutation is used.
 *   - n == 0 is valid and launches nothing.
 *   - Inputs must be finite; NaN/Inf coordinates give unspecified results.
 */
#ifndef TT_H
#define TT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum tt_status {
    TT_OK = 0,
    TT_ERR_INVALID_ARG = -1,   /* null/misaligned pointer, bad size or parameter   */
    TT_ERR_CUDA = -2,          /* CUDA runtime error (see tt_last_cuda_error)      */
    TT_ERR_OOM = -3,           /* host or device allocation failed                 */
    TT_ERR_TREE_TOO_DEEP = -4, /* tree height exceeds the compiled stack capacity  */
    TT_ERR_KIND_MISMATCH = -5, /* e.g. tt_traverse_bh on a kd-tree                 */
    TT_ERR_UNSUPPORTED = -6    /* parameter outside what the kernels implement     */
} tt_status;

typedef enum tt_kind {
    TT_KIND_OCT = 1, /* Barnes-Hut oct-tree of bodies     */
    TT_KIND_KD = 2,  /* kd-tree              */
    TT_KIND_VP = 3,  /* vantage-point tree [27]                    */
    TT_KIND_NN = 4   /* point-per-node kd-tree of the NN benchmark */
} tt_kind;

typedef enum tt_mode {
    TT_MODE_AUTO = 0,        /* per-warp choice, see tt_traverse_opts.auto_min_depth */
    TT_MODE_LOCKSTEP = 1,    /* "L" in Table 1                         */
    TT_MODE_INDEPENDENT = 2  /* "N" in Table 1: non-lockstep autoropes                */
} tt_mode;

typedef enum tt_mem { TT_MEM_HOST = 0, TT_MEM_DEVICE = 1 } tt_mem;

typedef void *tt_stream; /* cudaStream_t */

#define TT_MAX_HEIGHT 48      /* rope-stack capacity bound (levels)            */
#define TT_MAX_DIM 16         /* point dimensionality supported by the kernels */
#define TT_MAX_K 32           /* kNN k supported by the kernels                */
#ifndef TT_BH_POINTS_PER_LANE
#define TT_BH_POINTS_PER_LANE 2 /* a BH warp tile holds 32*2 = 64 bodies (2 per
                                   lane); its tt_stats warp_* entry covers 64
                                   points (other kernels: 32 points, 1 per lane) */
#endif

/* ------------------------------------------------------------------------ */
/* Host-side tree construction (build rules: DESIGN.md R3, R8a, R9, R12).   */
/* The paper takes the tree as given by the application; these
 * builders produce the canonical left-biased linearisation (preorder, first
 * child first, rope = preorder index after the subtree, Fig.2).
 * Points are read from host memory (row-major, leading dimension `ld` floats)
 * and copied; the host tree owns its arrays until tt_host_tree_free.        */
typedef struct tt_host_tree tt_host_tree;

tt_status tt_build_kd(const float *pts, int64_t n, int32_t dim, int32_t ld, int32_t leaf_size,
                      tt_host_tree **out);
/* bodies: n rows of (x, y, z, mass). */
tt_status tt_build_oct(const float *bodies, int64_t n, tt_host_tree **out);
tt_status tt_build_vp(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_host_tree **out);
/* NEXT-3 (R21): point-per-node kd-tree -- each node holds the median of its
 * set on (x[dim], id) along the largest-extent dimension (lowest on ties)
 * and the tight box of its subtree; left = the points before it, right =
 * the points after it.                                                    */
tt_status tt_build_nn(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_host_tree **out);
void tt_host_tree_free(tt_host_tree *t);

/* Canonical tree description, all arrays in preorder (host memory).  Node
 * indices are preorder indices; -1 = absent.  Produced by tt_host_tree_desc,
 * or filled by the caller with its own tree.                              */
typedef struct tt_tree_desc {
    int32_t kind;            /* tt_kind                                          */
    int32_t dim;             /* point dimension (3 for OCT)                      */
    int32_t height;          /* max node level (root = 0)                        */
    int32_t leaf_size;       /* kd bucket size (informative)                     */
    int64_t n_nodes;
    int64_t n_points;
    const int32_t *first_child; /* [n_nodes] first child (OCT/KD), -1 for a leaf  */
    const int32_t *skip;        /* [n_nodes] rope: preorder index after subtree   */
    const int32_t *level;       /* [n_nodes]                                      */
    const int32_t *pbegin;      /* [n_nodes] first tree-order point of subtree    */
    const int32_t *pcount;      /* [n_nodes] points in subtree                    */
    /* KD (and NN: the split of the node's own point)                        */
    const int32_t *split_dim;   /* [n_nodes] -1 for a leaf                        */
    const float *split;         /* [n_nodes]                                      */
    const float *lo, *hi;       /* [n_nodes * dim] tight bounding boxes (KD, NN)  */
    /* OCT */
    const float *com;           /* [n_nodes * 4] centre of mass x,y,z and mass    */
    const int32_t *body;        /* [n_nodes] OCT: body id of a leaf, -1 for a cell;
                                   VP: id of the node's vantage point;
                                   NN: id of the node's own point                */
    double root_center[3];
    double root_side;
    /* VP (NN: in_child = left, out_child = right)                          */
    const int32_t *in_child;    /* [n_nodes] inside child or -1                   */
    const int32_t *out_child;   /* [n_nodes] outside child or -1                  */
    const float *r_in_max;      /* [n_nodes] max distance vp -> inside points     */
    const float *r_out_min;     /* [n_nodes] min distance vp -> outside points    */
    /* points */
    const int32_t *tree_order;  /* [n_points] original id of j-th tree-order point*/
    const float *points;        /* [n_points * dim] by ORIGINAL id (OCT: 4 floats)*/
} tt_tree_desc;

tt_status tt_host_tree_desc(const tt_host_tree *t, tt_tree_desc *out);

/* ------------------------------------------------------------------------ */
/* a0: tree upload ("an identical linearized copy of the tree is
 * constructed using a left-biased linearization, with the nodes structured
 * according to [the field-split] layout ... and copied to the GPU's global
 * memory").  Layout: one 32-byte record per node (two 128-bit
 * field groups split by use), int32 node indices, the nodes of
 * the top `top_levels` levels renumbered first so one bulk copy stages them
 * in shared memory.  The packed blob is position-independent, so it can be
 * NCCL-broadcast as bytes and adopted on another GPU.
 * Errors: TT_ERR_INVALID_ARG (inconsistent desc), TT_ERR_TREE_TOO_DEEP
 * (height > TT_MAX_HEIGHT), TT_ERR_UNSUPPORTED (dim > TT_MAX_DIM),
 * TT_ERR_OOM, TT_ERR_CUDA.  The returned tree owns its device memory until
 * tt_tree_free; it is read-only, so concurrent traversals are safe (each
 * launch takes one of 256 per-tree tile-scheduler slots round-robin and
 * frees it when its last CTA finishes: at most 256 launches of one tree may
 * be in flight at once).                                                  */
typedef struct tt_tree tt_tree;

tt_status tt_tree_pack_size(const tt_tree_desc *d, size_t *bytes);
tt_status tt_tree_pack(const tt_tree_desc *d, void *host_blob, size_t bytes);
/* mem = TT_MEM_HOST: blob in host memory (copied H2D on `s`);
 * mem = TT_MEM_DEVICE: blob already in device memory (e.g. after an NCCL
 * broadcast); it is copied device-to-device, the caller keeps ownership.
 * The call synchronises `s` before returning.                             */
tt_status tt_tree_from_blob(const void *blob, size_t bytes, int32_t mem, tt_stream s, tt_tree **out);
tt_status tt_tree_upload(const tt_tree_desc *d, tt_stream s, tt_tree **out);
/* NEXT-1: build a Barnes-Hut oct-tree on the GPU from device bodies (n rows
 * of x, y, z, mass; 16-B aligned) straight into the packed device layout --
 * the same bytes tt_tree_pack produces for tt_build_oct of the same bodies
 * (build rules R8a/R9).  Synchronises `s`.  Errors: TT_ERR_INVALID_ARG,
 * TT_ERR_TREE_TOO_DEEP (never for R9 trees: height <= 33), TT_ERR_CUDA/OOM. */
tt_status tt_build_oct_device(const float *bodies, int64_t n, tt_stream s, tt_tree **out);
/* The same build, also writing the bodies' tree order: order_out (device,
 * n uint32, nullable) = body indices in leaf preorder (Fig.2 order of the
 * leaves; the bodies of a depth-32 bucket by index, R9) -- the order the
 * build has already sorted them into, so a time step can traverse in it
 * without a separate tt_sort_points (§4.4: any order that makes
 * neighbouring traversals similar; this one refines the 63-bit key of
 * tt_sort_points to all 32 levels).  Synchronises `s` twice.               */
tt_status tt_build_oct_device_order(const float *bodies, int64_t n, uint32_t *order_out, tt_stream s, tt_tree **out);
/* NEXT-1: build a kd-tree (median splits, reading R3) on the GPU from device
 * points (n rows of `ld` floats, dim <= TT_MAX_DIM) straight into the packed
 * device layout -- the bytes tt_tree_pack produces for tt_build_kd.
 * Synchronises `s` once per tree level.                                    */
tt_status tt_build_kd_device(const float *pts, int64_t n, int32_t dim, int32_t ld, int32_t leaf_size, tt_stream s,
                             tt_tree **out);
/* NEXT-1: build a vantage-point tree (reading R12) on the GPU, same contract
 * as tt_build_kd_device (bytes identical to tt_tree_pack of tt_build_vp). */
tt_status tt_build_vp_device(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_stream s, tt_tree **out);
/* NEXT-1 for the NEXT-3 NN tree: build the point-per-node kd-tree (reading
 * R21) on the GPU, same contract as tt_build_kd_device (bytes identical to
 * tt_tree_pack of tt_build_nn).                                            */
tt_status tt_build_nn_device(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_stream s, tt_tree **out);
/* Copy the packed device blob back to host memory (bytes >= device_bytes of
 * tt_tree_get_info); synchronous.  E.g. to checkpoint a tree.              */
tt_status tt_tree_download(const tt_tree *t, void *host_blob, size_t bytes);
/* Copy the packed blob to caller-owned memory: mem = TT_MEM_HOST (host, like
 * tt_tree_download; synchronous) or TT_MEM_DEVICE (device, asynchronous on
 * `s`) -- e.g. the send buffer of the NCCL broadcast of a GPU-built tree
 * (§8(e)), adopted on the other ranks with tt_tree_from_blob(DEVICE).
 * Errors: TT_ERR_INVALID_ARG (null, bytes < device_bytes, bad mem), TT_ERR_CUDA. */
tt_status tt_tree_copy_blob(const tt_tree *t, void *dst, size_t bytes, int32_t mem, tt_stream s);
tt_status tt_tree_free(tt_tree *t);

typedef struct tt_tree_info {
    int32_t kind, dim, dim_padded, height;
    int64_t n_nodes, n_points;
    int32_t top_levels;      /* levels staged in shared memory                   */
    int32_t top_count;       /* nodes in those levels                           */
    int64_t device_bytes;    /* bytes of the packed device layout               */
    const void *device_blob; /* device pointer of the packed layout             */
} tt_tree_info;
tt_status tt_tree_get_info(const tt_tree *t, tt_tree_info *out);

/* ------------------------------------------------------------------------ */
/* a1: point sort (§4.4).  Key = where the point's descent of the
 * tree by the build's split rule ends: kd -> the leaf's first tree-order
 * point (tree order); oct -> the index, along the 3-D Hilbert curve of the
 * root cube, of the point's 16-level cell of the cube hierarchy (octant bits
 * from the build's fp64 comparisons; reading R18b: more compact warp tiles
 * than the Morton / leaf-preorder order); vp -> 2-bit-per-level path code;
 * nn -> the same code of the left-iff-x[dim]<split descent.  A
 * stable radix sort of (key, index) gives perm: perm[j] = original index of
 * the j-th point in key order (ties by index).  pts: device, n rows of `ld`
 * floats (OCT: ld >= 4 or 3).  keys_out (nullable): the keys, in input order.
 * Temporary device memory is taken stream-ordered (cudaMallocAsync).      */
tt_status tt_sort_points(const tt_tree *t, const float *pts, int64_t n, int32_t ld,
                         uint32_t *perm_out, uint64_t *keys_out, tt_stream s);

/* a1b: longest-first tile schedule (Graham's LPT rule over
 * the persistent kernels' warp tiles).  Reorders whole tiles of perm_in --
 * T consecutive entries, T = 32 for kd/vp trees (the kNN, PC and VP kernels'
 * tile) -- so that tiles with the largest estimated traversal cost come
 * first; the entries inside a tile and the ragged last tile (n mod T) keep
 * their places, and equal estimates keep their order.  Estimate per point,
 * from one greedy descent: kd -> largest pinned d2 to the points of the leaf
 * the split rule reaches; vp -> smallest distance to a vantage point on the
 * inside-iff-d<=r_in path; tile = the largest over its points.  Oct trees:
 * and NN trees: a plain copy (BH tiles are near-uniform, §4.6).  Traversal results never
 * depend on the order, only the schedule does.  pts: device, n rows of `ld`
 * floats (the points perm_in indexes); perm_in/perm_out: device [n], may be
 * the same buffer.  Temporary device memory is stream-ordered.            */
tt_status tt_schedule_tiles(const tt_tree *t, const float *pts, int64_t n, int32_t ld,
                            const uint32_t *perm_in, uint32_t *perm_out, tt_stream s);

/* ------------------------------------------------------------------------ */
/* a2-a6: traversal launch options (all optional; pass NULL for defaults).  */
typedef struct tt_stats {
    uint32_t *visits;        /* [n] per point: truncation tests it performed (the
                                paper's per-point node count)      */
    uint32_t *warp_fetches;  /* [ceil(n/T)] node records fetched by the warp tile
                                (lockstep: one per step; independent: per lane);
                                T = 32 points per tile (BH: 32*TT_BH_POINTS_PER_LANE) */
    uint32_t *warp_steps;    /* [ceil(n/T)] loop iterations of the warp          */
    uint8_t *warp_mode;      /* [ceil(n/T)] 1 = lockstep, 2 = independent,
                                3 = lockstep switched to independent          */
    /* Per-point hashes of the nodes the point tested (nullable; requesting
     * either builds, once per tree, a map from device node to canonical
     * preorder id pre -- the numbering of tt_tree_desc):
     *   visit_hash: h = h*31 + pre + 1 over the tested nodes in the order the
     *     point tested them (the recursive order, §3.3, is kept by
     *     every independent walk, the per-node lockstep BH / PC walks and the
     *     explicit-stack variants; kNN / VP / NN lockstep lanes follow the
     *     warp's majority-vote order, §4.3).  Written 0 for points of walks
     *     that do not keep a per-point order: BH child-group lockstep tiles
     *     and TT_VARIANT_SPLIT (reading R23);
     *   visit_set: sum over the tested nodes of mix64(pre + 1) mod 2^64
     *     (mix64 = the splitmix64 finaliser): order-insensitive, written by
     *     every walk.                                                        */
    uint64_t *visit_hash;    /* [n]                                              */
    uint64_t *visit_set;     /* [n]                                              */
    uint32_t *point_tests;   /* [n] kNN / PC: bucket points whose distance the
                                point computed (SURVEY §8(d) kNN bytes: 16 B per
                                inner node + 32 B per leaf point); nullable     */
} tt_stats;

typedef struct tt_traverse_opts {
    int32_t mode;            /* tt_mode                                          */
    int32_t auto_min_depth;  /* AUTO: T, the tree level of the per-warp coherence
                                test -- lockstep iff the warp's points, in launch
                                order, change their level-T cell (oct: 2^T grid
                                cell of the root cube; kd / vp: T-level descent
                                path) fewer than 8 times (0 = always lockstep,
                                >= 64 = never); -1 = kernel default, measured on
                                B200: BH 3, kNN 4, VP 4, PC never
                                (10k-point PC is latency-bound: independent wins);
                                PC AUTO with the default threshold and fewer
                                32-point tiles than resident warps (SMs x 32)
                                splits each point's walk over 16 lanes
                                (TT_VARIANT_SPLIT; warp_* stats left untouched) */
    const uint32_t *order;   /* [n] device, nullable: lane j of the launch processes
                                point order[j] (e.g. perm from tt_sort_points);
                                results still go to the point's own slot        */
    const tt_stats *stats;   /* host struct of device pointers, nullable         */
    int32_t block_threads;   /* 0 = default (256)                               */
    int32_t ctas_per_sm;     /* 0 = occupancy maximum                            */
    int32_t variant;         /* tt_variant: 0 = autoropes (the method; for BH
                                the child-group lockstep walk, 4);
                                1 = naive recursive baseline (P:L1084-1090,
                                independent mode only -- LOCKSTEP is
                                TT_ERR_UNSUPPORTED; it fills stats->visits only,
                                the warp_* arrays are left untouched);
                                2 = explicit rope stack, the paper's Fig.9b
                                form (BH and PC only, else TT_ERR_UNSUPPORTED):
                                independent = per-thread stacks interleaved in
                                global memory, lockstep = one (node, mask)
                                stack per warp in shared memory;
                                AUTO = BH lockstep, PC independent; 32-point
                                warp tiles;
                                3 = split (PC only, else TT_ERR_UNSUPPORTED):
                                each point's walk is split by subtree over a
                                16-lane group (for point sets too small to fill
                                the GPU one lane per point, e.g. configs[0]);
                                mode is ignored, stats->visits only;
                                4 = groups (BH only; BH's default, 0 selects
                                it): lockstep warps expand a whole cell per
                                step -- its children, stored contiguously in a
                                group array built on the first such call and
                                kept with the tree, are loaded together and
                                tested by every body that opened the cell;
                                independent warps take the stackless rope walk;
                                5 = ropes (BH only): the per-node Fig.8
                                lockstep walk over stored ropes             */
    int32_t switch_below;    /* NEXT-3 dynamic L->N switching (kNN only, else
                                must be 0): a lockstep warp whose active lanes at
                                a node number fewer than this converts its warp
                                rope stack into per-lane stacks (each lane keeps
                                the entries whose mask holds it, in order) and
                                finishes the tile independently; tt_stats
                                warp_mode = 3 for such tiles.  0 = never (default);
                                33 = at the root (= independent).  Results never
                                depend on it.                                   */
} tt_traverse_opts;

typedef enum tt_variant {
    TT_VARIANT_AUTOROPES = 0,
    TT_VARIANT_RECURSIVE = 1,
    TT_VARIANT_STACK = 2,
    TT_VARIANT_SPLIT = 3,
    TT_VARIANT_GROUPS = 4,
    TT_VARIANT_ROPES = 5
} tt_variant;

/* Barnes-Hut force pass (Fig.9): bodies float4 (x,y,z,m) rows;
 * self_ids[i] (nullable; default i) is the leaf body id whose interaction
 * point i skips (R9); a negative id skips nothing.  A cell is opened iff it is a cell and
 * |com - x|^2 < dsq_L, dsq_L = dsq_root * 0.25^L, dsq_root = (side/theta)^2
 * (theta == 0 -> +inf: every cell opened).  acc_out: float4 (ax,ay,az,0),
 * G = 1, softening eps.  Opening decisions use pinned fp32 arithmetic:
 * |com - x|^2 = fma(dz, dz, fma(dy, dy, dx*dx)) (reading R8).
 * Variants: AUTOROPES (default) walks lockstep warps by child groups
 * (TT_VARIANT_GROUPS) when the tree allows it -- height <= 38, <= 8 cell
 * children per cell, < 2^27 nodes -- else by per-node ropes (ROPES);
 * requesting GROUPS for a tree that does not allow it returns
 * TT_ERR_TREE_TOO_DEEP (height / children) or TT_ERR_UNSUPPORTED (size).
 * Opt-in, environment TT_L2_PERSIST_MB=<MiB>: an L2 persisting access-policy
 * window over the top of the tree for each launch (device-wide set-aside;
 * the stream's window is cleared after the launch; not inside a graph
 * capture).  Results never depend on it. */
tt_status tt_traverse_bh(const tt_tree *t, const float *bodies, const int32_t *self_ids, int64_t n,
                         float theta, float eps, float *acc_out, const tt_traverse_opts *opts,
                         tt_stream s);

/* 2-point correlation (Fig.4/6/8):
 * count_out[i] = #{data points p : d2(q_i, p) <= rn(radius^2)}.  q: n rows of
 * `ld` floats, dim = tree dim.                                             */
tt_status tt_traverse_pc(const tt_tree *t, const float *q, int64_t n, int32_t ld, float radius,
                         uint32_t *count_out, const tt_traverse_opts *opts, tt_stream s);

/* k-nearest neighbours (Fig.5/7): the k
 * data points with the smallest (d2, id), ascending; idx_out/d2_out are n*k
 * row-major; padded with (-1, +inf) when the tree holds fewer than k points.
 * 1 <= k <= TT_MAX_K.                                                     */
tt_status tt_traverse_knn(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t k,
                          int32_t *idx_out, float *d2_out, const tt_traverse_opts *opts,
                          tt_stream s);

/* Vantage-point-tree nearest neighbour ([27]): argmin (d2, id). */
tt_status tt_traverse_vp(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t *idx_out,
                         float *d2_out, const tt_traverse_opts *opts, tt_stream s);

/* NEXT-3: nearest neighbour over the point-per-node kd-tree of the paper's NN
 * benchmark (tt_build_nn, reading R21): argmin (d2, id), the
 * same answer as tt_traverse_knn with k = 1 and tt_traverse_vp.  Fig.5
 * pattern: truncate iff the pinned distance to the node's tight box > best
 * d2; update with the node's point; near = q[dim] < split ? left : right,
 * visited first.  AUTO default threshold 4.                              */
tt_status tt_traverse_nn(const tt_tree *t, const float *q, int64_t n, int32_t ld, int32_t *idx_out,
                         float *d2_out, const tt_traverse_opts *opts, tt_stream s);

/* NEXT-4: one kick-drift update of a Barnes-Hut time step (leapfrog KDK is
 * kick(dt/2)+drift(dt), rebuild + force pass, kick(dt/2)):
 * v += acc * dt_kick; x += v * dt_drift.  bodies (x,y,z,m), vel (vx,vy,vz,-)
 * and acc (ax,ay,az,-) are n float4 rows in device memory (16-B aligned);
 * fp32 with one rounding per operation; asynchronous on `s`.              */
tt_status tt_kick_drift(float *bodies, float *vel, const float *acc, int64_t n, float dt_kick, float dt_drift,
                        tt_stream s);

/* NEXT-4, sharded time step: the same update, gathered
 * through a permutation: for j < n, with i = perm[j],
 *   vel_out[j]    = vel[i] + acc[i] * dt_kick      (x, y, z; w copied)
 *   bodies_out[j] = bodies[i] + vel_out[j] * dt_drift (x, y, z; mass copied)
 *   ids_out[j]    = ids[i]                           (if ids != NULL)
 * perm is typically a contiguous slice of tt_sort_points' permutation, so a
 * rank's shard of the sorted order is written contiguously and the bodies
 * travel in sorted order.  Inputs and outputs are device float4 rows (16-B
 * aligned) and must not overlap; perm entries index the input rows and are
 * not range-checked (caller's contract).  Asynchronous on `s`.            */
tt_status tt_kick_drift_permuted(const float *bodies, const float *vel, const float *acc, const int32_t *perm,
                                 const int32_t *ids, int64_t n, float dt_kick, float dt_drift, float *bodies_out,
                                 float *vel_out, int32_t *ids_out, tt_stream s);

/* ------------------------------------------------------------------------ */
/* Diagnostics (not part of the method; SURVEY §8(d) "diagnostic ceilings").
 * The dependent-load ceiling of a tree walk: every warp (per_lane = 0, the
 * lockstep access: one warp-uniform 32-B record per step) or every lane
 * (per_lane = 1, independent walks) follows its own chain through `nrec`
 * 32-byte records for `steps` steps, with the traversal kernels' launch shape
 * (256-thread CTAs, <= 4 per SM or ctas_per_sm).  records: device, 32-B
 * aligned; the int32 at byte offset 16 of record i is the index of the next
 * record (0 <= next < nrec).  sink: device uint32 (written only to keep the
 * loads).  Asynchronous on `s`; the caller times it.  Errors:
 * TT_ERR_INVALID_ARG, TT_ERR_CUDA.                                        */
tt_status tt_diag_chase(const void *records, int64_t nrec, int32_t per_lane, int64_t steps, int32_t ctas_per_sm,
                        uint32_t *sink, tt_stream s);
/* The L2 read-bandwidth ceiling: 8 x 256-thread CTAs per SM read `bytes`
 * (a multiple of 32, smaller than L2 to be L2-resident) of `buf` `reps`
 * times with ld.global.cg (L2 only, not L1), 32 B per thread per
 * iteration; bytes * reps / time = L2 read GB/s.  buf: device, 32-B
 * aligned; sink as above.  Asynchronous; the caller times it.
 * Errors: TT_ERR_INVALID_ARG, TT_ERR_CUDA.                                 */
tt_status tt_diag_l2read(const void *buf, int64_t bytes, int32_t reps, uint32_t *sink, tt_stream s);

/* ------------------------------------------------------------------------ */
const char *tt_status_string(tt_status s);
/* Last CUDA error code seen by the library (cudaError_t as int), 0 if none. */
int32_t tt_last_cuda_error(void);
/* Version / build identification string (compiled arch, flags). */
const char *tt_build_info(void);

#ifdef __cplusplus
}
#endif
#endif /* TT_H */
