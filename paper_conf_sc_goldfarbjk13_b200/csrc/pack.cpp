// pack.cpp -- canonical tree description -> position-independent device blob.
//
// The paper copies "an identical linearized copy of the tree ... using a
// left-biased linearization, with the nodes structured according to the
// layout strategy" to global memory, splitting node fields by
// use.  B200 form:
//   * one 32-byte record per node = one DRAM/L2 sector, read as two 128-bit
//     loads (the use-split groups of Fig.9b lines 9 and 11);
//   * int32 node indices, rope (skip) stored on every node (Fig.2 ropes);
//   * the nodes of the top `top_levels` levels are renumbered first, level by
//     level (preorder within a level), the rest follow in preorder, so one
//     bulk copy of a prefix stages the top L levels in shared memory (each
//     kernel picks the L that fits its budget).  The walk only follows
//     explicit child / rope indices and node levels, so it is independent of
//     the numbering.
#include <cstring>
#include <new>
#include <vector>

#include "tt_internal.h"

namespace {

inline uint64_t align256(uint64_t x) { return (x + 255) & ~uint64_t(255); }

int dim_padded(int dim) { return (dim + 3) & ~3; }

int stage_bytes_per_node(int kind, int dp) {
    if (kind == TT_KIND_OCT) return 32;
    if (kind == TT_KIND_KD) return 32 + 8 * dp;
    if (kind == TT_KIND_NN) return 16 + 12 * dp;  // record + box + point
    return 16 + 4 * dp;                            // VP
}

int validate(const tt_tree_desc *d) {
    if (!d) return TT_ERR_INVALID_ARG;
    if (d->kind != TT_KIND_OCT && d->kind != TT_KIND_KD && d->kind != TT_KIND_VP && d->kind != TT_KIND_NN)
        return TT_ERR_INVALID_ARG;
    if (d->n_nodes <= 0 || d->n_nodes > INT32_MAX - 1 || d->n_points <= 0 || d->n_points > INT32_MAX - 1)
        return TT_ERR_INVALID_ARG;
    if (d->dim <= 0) return TT_ERR_INVALID_ARG;
    if (d->dim > TT_MAX_DIM) return TT_ERR_UNSUPPORTED;
    if (d->kind == TT_KIND_OCT && d->dim != 3) return TT_ERR_INVALID_ARG;
    if (d->height < 0) return TT_ERR_INVALID_ARG;
    if (d->height > TT_MAX_HEIGHT) return TT_ERR_TREE_TOO_DEEP;
    if (!d->first_child || !d->skip || !d->level || !d->pbegin || !d->pcount) return TT_ERR_INVALID_ARG;
    if (d->kind == TT_KIND_KD && (!d->split_dim || !d->split || !d->lo || !d->hi || !d->tree_order || !d->points))
        return TT_ERR_INVALID_ARG;
    if (d->kind == TT_KIND_OCT && (!d->com || !d->body)) return TT_ERR_INVALID_ARG;
    if (d->kind == TT_KIND_VP &&
        (!d->body || !d->in_child || !d->out_child || !d->r_in_max || !d->r_out_min || !d->points))
        return TT_ERR_INVALID_ARG;
    if (d->kind == TT_KIND_NN &&
        (!d->body || !d->in_child || !d->out_child || !d->split || !d->split_dim || !d->points || !d->lo ||
         !d->hi))
        return TT_ERR_INVALID_ARG;
    const int64_t N = d->n_nodes;
    for (int64_t v = 0; v < N; ++v) {
        if (d->skip[v] <= v || d->skip[v] > N) return TT_ERR_INVALID_ARG;
        if (d->first_child[v] != -1 && (d->first_child[v] != v + 1 || d->first_child[v] >= N))
            return TT_ERR_INVALID_ARG;
        if (d->level[v] < 0 || d->level[v] > d->height) return TT_ERR_INVALID_ARG;
        if (d->kind == TT_KIND_KD) {
            if ((d->split_dim[v] < 0) != (d->first_child[v] < 0)) return TT_ERR_INVALID_ARG;
            if (d->split_dim[v] >= d->dim) return TT_ERR_INVALID_ARG;
            if (d->first_child[v] >= 0 && d->skip[d->first_child[v]] >= d->skip[v]) return TT_ERR_INVALID_ARG;
        }
        if (d->kind == TT_KIND_VP || d->kind == TT_KIND_NN) {
            if (d->body[v] < 0 || d->body[v] >= d->n_points) return TT_ERR_INVALID_ARG;
            if (d->in_child[v] >= N || d->out_child[v] >= N) return TT_ERR_INVALID_ARG;
        }
        if (d->kind == TT_KIND_NN) {
            const bool inner = d->in_child[v] >= 0 || d->out_child[v] >= 0;
            if (inner != (d->split_dim[v] >= 0) || d->split_dim[v] >= d->dim) return TT_ERR_INVALID_ARG;
        }
        if (d->kind == TT_KIND_OCT && d->body[v] >= d->n_points) return TT_ERR_INVALID_ARG;
        if (d->pbegin[v] < 0 || d->pcount[v] < 0 || (int64_t)d->pbegin[v] + d->pcount[v] > d->n_points)
            return TT_ERR_INVALID_ARG;
    }
    if (d->kind == TT_KIND_KD)
        for (int64_t i = 0; i < d->n_points; ++i)
            if (d->tree_order[i] < 0 || d->tree_order[i] >= d->n_points) return TT_ERR_INVALID_ARG;
    return TT_OK;
}

void plan(const tt_tree_desc *d, tt_blob_header &h, std::vector<int32_t> *newidx) {
    std::memset(&h, 0, sizeof(h));
    h.magic = TT_BLOB_MAGIC;
    h.version = TT_BLOB_VERSION;
    h.kind = d->kind;
    h.dim = d->dim;
    h.dp = dim_padded(d->dim);
    h.height = d->height;
    h.leaf_size = d->leaf_size;
    h.n_nodes = d->n_nodes;
    h.n_points = d->n_points;
    for (int i = 0; i < 3; ++i) h.root_center[i] = d->root_center[i];
    h.root_side = d->root_side;
    // top levels that fit the shared-memory budget
    std::vector<int64_t> per_level((size_t)d->height + 2, 0);
    for (int64_t v = 0; v < d->n_nodes; ++v) per_level[(size_t)d->level[v]]++;
    const int sb = stage_bytes_per_node(d->kind, h.dp);
    int64_t acc = 0;
    int L = 0;
    h.level_prefix[0] = 0;
    while (L <= d->height && L < TT_TOP_LEVELS_MAX && (acc + per_level[(size_t)L]) * sb <= TT_TOP_BYTES) {
        acc += per_level[(size_t)L];
        ++L;
        h.level_prefix[L] = (int32_t)acc;
    }
    h.top_levels = L;
    h.top_count = (int32_t)acc;
    if (d->kind == TT_KIND_OCT) {
        // what the child-group BH walk may assume (kern_bh_group.cu): at most 8
        // children staged per group and at most 8 cell children pushed per level.
        // R9 trees: only depth-32 buckets exceed 8 children, and those are
        // leaves -- the GPU builder writes the same bits from the height alone.
        int64_t max_kids = 0, max_cell_kids = 0;
        for (int64_t v = 0; v < d->n_nodes; ++v) {
            int64_t k = 0, kc = 0;
            for (int32_t c = d->first_child[v]; c >= 0 && c < d->skip[v]; c = d->skip[c]) {
                ++k;
                kc += d->first_child[c] >= 0;
            }
            if (k > max_kids) max_kids = k;
            if (kc > max_cell_kids) max_cell_kids = kc;
        }
        h.oct_flags = ((d->height <= 32 && max_kids <= 8) ? TT_OCT_NARROW : 0) |
                      (max_cell_kids <= 8 ? TT_OCT_FEW_CELL_KIDS : 0);
    }
    h.rec_bytes = (d->kind == TT_KIND_VP || d->kind == TT_KIND_NN) ? 16 : 32;
    uint64_t off = align256(sizeof(tt_blob_header));
    h.off_rec = off;
    off = align256(off + (uint64_t)d->n_nodes * h.rec_bytes);
    if (d->kind == TT_KIND_KD) {
        h.off_box = off;
        off = align256(off + (uint64_t)d->n_nodes * 2 * h.dp * sizeof(float));
        h.off_pts = off;
        off = align256(off + (uint64_t)d->n_points * h.dp * sizeof(float));
        h.off_pid = off;
        off = align256(off + (uint64_t)d->n_points * sizeof(int32_t));
        h.off_cbox = off;
        off = align256(off + (uint64_t)d->n_nodes * 4 * h.dp * sizeof(float));
    } else if (d->kind == TT_KIND_VP || d->kind == TT_KIND_NN) {
        if (d->kind == TT_KIND_NN) {
            h.off_box = off;
            off = align256(off + (uint64_t)d->n_nodes * 2 * h.dp * sizeof(float));
        }
        h.off_vpt = off;
        off = align256(off + (uint64_t)d->n_nodes * h.dp * sizeof(float));
        h.off_pid = off;
        off = align256(off + (uint64_t)d->n_nodes * sizeof(int32_t));
    }
    h.total = off;
    if (newidx) {
        // top region level by level (preorder within a level), then the rest
        // of the tree in preorder
        newidx->assign((size_t)d->n_nodes, -1);
        std::vector<int32_t> next(h.level_prefix, h.level_prefix + h.top_levels + 1);
        int32_t b = h.top_count;
        for (int64_t v = 0; v < d->n_nodes; ++v) {
            const int l = d->level[v];
            (*newidx)[(size_t)v] = l < h.top_levels ? next[(size_t)l]++ : b++;
        }
    }
}

}  // namespace

size_t tt_pack_size_impl(const tt_tree_desc *d, int *status) {
    int st = validate(d);
    if (status) *status = st;
    if (st != TT_OK) return 0;
    tt_blob_header h;
    plan(d, h, nullptr);
    return (size_t)h.total;
}

int tt_pack_impl(const tt_tree_desc *d, void *blob, size_t bytes) {
    int st = validate(d);
    if (st != TT_OK) return st;
    if (!blob) return TT_ERR_INVALID_ARG;
    tt_blob_header h;
    std::vector<int32_t> nx;
    try {
        plan(d, h, &nx);
    } catch (const std::bad_alloc &) {
        return TT_ERR_OOM;
    }
    if (bytes < h.total) return TT_ERR_INVALID_ARG;
    auto *base = static_cast<unsigned char *>(blob);
    std::memset(base, 0, (size_t)h.total);
    std::memcpy(base, &h, sizeof(h));
    const int64_t N = d->n_nodes;
    auto map = [&](int32_t c) -> int32_t { return (c < 0 || c >= N) ? TT_END : nx[(size_t)c]; };
    if (d->kind == TT_KIND_OCT) {
        auto *rec = reinterpret_cast<tt_oct_rec *>(base + h.off_rec);
        for (int64_t v = 0; v < N; ++v) {
            tt_oct_rec &r = rec[nx[(size_t)v]];
            r.gx = d->com[v * 4 + 0];
            r.gy = d->com[v * 4 + 1];
            r.gz = d->com[v * 4 + 2];
            r.gm = d->com[v * 4 + 3];
            r.first_child = map(d->first_child[v]);
            r.skip = map(d->skip[v]);
            r.body = d->body[v];
            r.level = d->level[v];
        }
    } else if (d->kind == TT_KIND_KD) {
        auto *rec = reinterpret_cast<tt_kd_rec *>(base + h.off_rec);
        auto *box = reinterpret_cast<float *>(base + h.off_box);
        for (int64_t v = 0; v < N; ++v) {
            const int32_t nv = nx[(size_t)v];
            tt_kd_rec &r = rec[nv];
            const int32_t l = d->first_child[v];
            r.left = map(l);
            r.right = l >= 0 ? map(d->skip[l]) : TT_END;
            r.skip = map(d->skip[v]);
            r.level = d->level[v];
            r.split = d->split[v];
            r.dim = d->split_dim[v];
            r.pbegin = d->pbegin[v];
            r.pcount = d->pcount[v];
            float *b = box + (size_t)nv * 2 * h.dp;
            for (int k = 0; k < d->dim; ++k) {
                b[k] = d->lo[v * d->dim + k];
                b[h.dp + k] = d->hi[v * d->dim + k];
            }
        }
        // children's boxes stored with the parent: the kNN walk tests a child's
        // box while expanding the parent (one load group per visited node)
        auto *cbox = reinterpret_cast<float *>(base + h.off_cbox);
        for (int64_t v = 0; v < N; ++v) {
            const int32_t l = d->first_child[v];
            if (l < 0) continue;
            const int32_t kids[2] = {l, d->skip[l]};
            float *dst = cbox + (size_t)nx[(size_t)v] * 4 * h.dp;
            for (int c = 0; c < 2; ++c)
                for (int k = 0; k < d->dim; ++k) {
                    dst[c * 2 * h.dp + k] = d->lo[(int64_t)kids[c] * d->dim + k];
                    dst[c * 2 * h.dp + h.dp + k] = d->hi[(int64_t)kids[c] * d->dim + k];
                }
        }
        auto *pts = reinterpret_cast<float *>(base + h.off_pts);
        auto *pid = reinterpret_cast<int32_t *>(base + h.off_pid);
        for (int64_t j = 0; j < d->n_points; ++j) {
            const int32_t id = d->tree_order[j];
            pid[j] = id;
            std::memcpy(pts + (size_t)j * h.dp, d->points + (size_t)id * d->dim, sizeof(float) * d->dim);
        }
    } else if (d->kind == TT_KIND_NN) {
        auto *rec = reinterpret_cast<tt_nn_rec *>(base + h.off_rec);
        auto *box = reinterpret_cast<float *>(base + h.off_box);
        auto *vpt = reinterpret_cast<float *>(base + h.off_vpt);
        auto *pid = reinterpret_cast<int32_t *>(base + h.off_pid);
        for (int64_t v = 0; v < N; ++v) {
            const int32_t nv = nx[(size_t)v];
            tt_nn_rec &r = rec[nv];
            r.left = map(d->in_child[v]);
            r.right = map(d->out_child[v]);
            r.split = d->split[v];
            r.dim = d->split_dim[v];
            float *bx = box + (size_t)nv * 2 * h.dp;
            for (int k = 0; k < d->dim; ++k) {
                bx[k] = d->lo[v * d->dim + k];
                bx[h.dp + k] = d->hi[v * d->dim + k];
            }
            pid[nv] = d->body[v];
            std::memcpy(vpt + (size_t)nv * h.dp, d->points + (size_t)d->body[v] * d->dim, sizeof(float) * d->dim);
        }
    } else {
        auto *rec = reinterpret_cast<tt_vp_rec *>(base + h.off_rec);
        auto *vpt = reinterpret_cast<float *>(base + h.off_vpt);
        auto *pid = reinterpret_cast<int32_t *>(base + h.off_pid);
        for (int64_t v = 0; v < N; ++v) {
            const int32_t nv = nx[(size_t)v];
            tt_vp_rec &r = rec[nv];
            r.in = map(d->in_child[v]);
            r.out = map(d->out_child[v]);
            r.r_in_max = d->r_in_max[v];
            r.r_out_min = d->r_out_min[v];
            pid[nv] = d->body[v];
            std::memcpy(vpt + (size_t)nv * h.dp, d->points + (size_t)d->body[v] * d->dim, sizeof(float) * d->dim);
        }
    }
    return TT_OK;
}
