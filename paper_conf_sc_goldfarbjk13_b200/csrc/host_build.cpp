// host_build.cpp -- host tree builders producing the canonical left-biased
// linearisation (preorder, first child first, rope = index after the subtree;
// P:L1063-1067, Fig.2).  Build rules are the DESIGN.md readings
// R3 (kd), R8a/R9 (oct), R12 (vp), R21 (nn).  Compiled with -ffp-contract=off so the
// fp32 distance used by the vp build is the pinned R0 sequence.
//
// Each builder partitions one index array in place: a node owns a contiguous
// range [b, e) of it, children own consecutive sub-ranges in visit order, so
// the final array IS the tree order of the points.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <limits>
#include <new>
#include <vector>

#include "tt_internal.h"

struct tt_host_tree {
    int32_t kind = 0, dim = 0, height = 0, leaf_size = 1;
    int64_t n_points = 0;
    std::vector<float> points;  // by original id, row stride = dim (OCT: 4)
    std::vector<int32_t> first_child, skip, level, pbegin, pcount;
    std::vector<int32_t> split_dim, body, in_child, out_child;
    std::vector<float> split, lo, hi, com, r_in_max, r_out_min;
    std::vector<int32_t> ids;   // tree order
    double root_center[3] = {0, 0, 0}, root_side = 0;
};

namespace {

constexpr int kOctMaxDepth = 32;  // R9

int32_t new_node(tt_host_tree &t, int lvl, int32_t b, int32_t e) {
    int32_t v = (int32_t)t.level.size();
    t.first_child.push_back(-1);
    t.skip.push_back(-1);
    t.level.push_back(lvl);
    t.pbegin.push_back(b);
    t.pcount.push_back(e - b);
    t.split_dim.push_back(-1);
    t.split.push_back(0.0f);
    t.body.push_back(-1);
    t.in_child.push_back(-1);
    t.out_child.push_back(-1);
    t.r_in_max.push_back(0.0f);
    t.r_out_min.push_back(0.0f);
    if (lvl > t.height) t.height = lvl;
    return v;
}

// pinned fp32 squared distance (R0): sequential, one rounding per op
inline float d2_pinned(const float *a, const float *b, int dim) {
    float t0 = a[0] - b[0];
    float s = t0 * t0;
    for (int d = 1; d < dim; ++d) {
        float t = a[d] - b[d];
        float tt = t * t;
        s = s + tt;
    }
    return s;
}

// ----------------------------------------------------------------- kd (R3)
void kd_rec(tt_host_tree &t, int32_t b, int32_t e, int lvl) {
    const int D = t.dim;
    int32_t v = new_node(t, lvl, b, e);
    std::vector<float> lo(D, std::numeric_limits<float>::infinity());
    std::vector<float> hi(D, -std::numeric_limits<float>::infinity());
    for (int32_t i = b; i < e; ++i) {
        const float *p = &t.points[(size_t)t.ids[i] * D];
        for (int d = 0; d < D; ++d) {
            lo[d] = std::min(lo[d], p[d]);
            hi[d] = std::max(hi[d], p[d]);
        }
    }
    t.lo.insert(t.lo.end(), lo.begin(), lo.end());
    t.hi.insert(t.hi.end(), hi.begin(), hi.end());
    const int32_t n = e - b;
    if (n <= t.leaf_size) {
        std::sort(t.ids.begin() + b, t.ids.begin() + e);
        t.skip[v] = (int32_t)t.level.size();
        return;
    }
    int sd = 0;
    float ext = hi[0] - lo[0];
    for (int d = 1; d < D; ++d) {
        float x = hi[d] - lo[d];
        if (x > ext) { ext = x; sd = d; }
    }
    const float *P = t.points.data();
    auto less = [P, D, sd](int32_t a, int32_t c) {
        float xa = P[(size_t)a * D + sd], xc = P[(size_t)c * D + sd];
        return xa < xc || (xa == xc && a < c);
    };
    const int32_t m = b + n / 2;
    std::nth_element(t.ids.begin() + b, t.ids.begin() + m, t.ids.begin() + e, less);
    t.split_dim[v] = sd;
    t.split[v] = P[(size_t)t.ids[m] * D + sd];
    t.first_child[v] = (int32_t)t.level.size();
    kd_rec(t, b, m, lvl + 1);
    kd_rec(t, m, e, lvl + 1);
    t.skip[v] = (int32_t)t.level.size();
}

// ---------------------------------------------------------- oct (R8a, R9)
struct Moments { double m0, m1[3]; };

Moments oct_rec(tt_host_tree &t, int32_t b, int32_t e, const double c[3], double side, int lvl) {
    int32_t v = new_node(t, lvl, b, e);
    Moments M{0.0, {0.0, 0.0, 0.0}};
    const float *P = t.points.data();
    auto leaf = [&](int32_t node, int32_t id) {
        const float *p = P + (size_t)id * 4;
        t.body[node] = id;
        for (int d = 0; d < 3; ++d) t.com[(size_t)node * 4 + d] = p[d];
        t.com[(size_t)node * 4 + 3] = p[3];
        Moments m{(double)p[3], {(double)p[3] * (double)p[0], (double)p[3] * (double)p[1],
                                 (double)p[3] * (double)p[2]}};
        return m;
    };
    auto grow_com = [&t](int32_t node) {
        t.com.resize(((size_t)node + 1) * 4, 0.0f);
    };
    grow_com(v);
    if (e - b == 1) {
        M = leaf(v, t.ids[b]);
        t.skip[v] = (int32_t)t.level.size();
        return M;
    }
    if (lvl >= kOctMaxDepth) {
        // bucket cell: bodies as single-body leaf children, ids ascending
        std::sort(t.ids.begin() + b, t.ids.begin() + e);
        t.first_child[v] = (int32_t)t.level.size();
        for (int32_t i = b; i < e; ++i) {
            int32_t lf = new_node(t, lvl + 1, i, i + 1);
            grow_com(lf);
            Moments m = leaf(lf, t.ids[i]);
            t.skip[lf] = (int32_t)t.level.size();
            M.m0 += m.m0;
            for (int d = 0; d < 3; ++d) M.m1[d] += m.m1[d];
        }
    } else {
        // stable counting partition by octant (fp64 comparisons)
        int32_t cnt[8] = {0};
        std::vector<uint8_t> oct((size_t)(e - b));
        for (int32_t i = b; i < e; ++i) {
            const float *p = P + (size_t)t.ids[i] * 4;
            int o = ((double)p[0] >= c[0]) | (((double)p[1] >= c[1]) << 1) | (((double)p[2] >= c[2]) << 2);
            oct[i - b] = (uint8_t)o;
            cnt[o]++;
        }
        int32_t start[9];
        start[0] = b;
        for (int o = 0; o < 8; ++o) start[o + 1] = start[o] + cnt[o];
        std::vector<int32_t> tmp((size_t)(e - b));
        int32_t pos[8];
        for (int o = 0; o < 8; ++o) pos[o] = start[o] - b;
        for (int32_t i = b; i < e; ++i) tmp[pos[oct[i - b]]++] = t.ids[i];
        std::copy(tmp.begin(), tmp.end(), t.ids.begin() + b);
        const double h = side * 0.25;
        t.first_child[v] = (int32_t)t.level.size();
        for (int o = 0; o < 8; ++o) {
            if (!cnt[o]) continue;
            double cc[3] = {c[0] + ((o & 1) ? h : -h), c[1] + ((o & 2) ? h : -h), c[2] + ((o & 4) ? h : -h)};
            Moments m = oct_rec(t, start[o], start[o + 1], cc, side * 0.5, lvl + 1);
            M.m0 += m.m0;
            for (int d = 0; d < 3; ++d) M.m1[d] += m.m1[d];
        }
    }
    for (int d = 0; d < 3; ++d) t.com[(size_t)v * 4 + d] = (float)(M.m0 != 0.0 ? M.m1[d] / M.m0 : 0.0);
    t.com[(size_t)v * 4 + 3] = (float)M.m0;
    t.skip[v] = (int32_t)t.level.size();
    return M;
}

// ------------------------------------------------------------------ vp (R12)
void vp_rec(tt_host_tree &t, int32_t b, int32_t e, int lvl, std::vector<float> &key) {
    int32_t v = new_node(t, lvl, b, e);
    const int D = t.dim;
    auto mn = std::min_element(t.ids.begin() + b, t.ids.begin() + e);
    std::iter_swap(t.ids.begin() + b, mn);
    const int32_t vp = t.ids[b];
    t.body[v] = vp;
    const int32_t r = e - b - 1;
    if (r == 0) {
        t.skip[v] = (int32_t)t.level.size();
        return;
    }
    const float *P = t.points.data();
    const float *pv = P + (size_t)vp * D;
    for (int32_t i = b + 1; i < e; ++i) key[t.ids[i]] = d2_pinned(pv, P + (size_t)t.ids[i] * D, D);
    const float *K = key.data();
    auto less = [K](int32_t a, int32_t c) { return K[a] < K[c] || (K[a] == K[c] && a < c); };
    const int32_t nin = r / 2;
    const int32_t mid = b + 1 + nin;  // first outside element after partition
    std::nth_element(t.ids.begin() + b + 1, t.ids.begin() + mid, t.ids.begin() + e, less);
    float rin2 = 0.0f;
    for (int32_t i = b + 1; i < mid; ++i) rin2 = std::max(rin2, K[t.ids[i]]);
    t.r_in_max[v] = nin > 0 ? std::sqrt(rin2) : 0.0f;
    t.r_out_min[v] = std::sqrt(K[t.ids[mid]]);
    if (nin > 0) {
        t.in_child[v] = (int32_t)t.level.size();
        vp_rec(t, b + 1, mid, lvl + 1, key);
    }
    t.out_child[v] = (int32_t)t.level.size();
    vp_rec(t, mid, e, lvl + 1, key);
    t.first_child[v] = t.in_child[v] >= 0 ? t.in_child[v] : t.out_child[v];
    t.skip[v] = (int32_t)t.level.size();
}

// ------------------------------------------------------------------ nn (R21)
// Point-per-node kd-tree (the paper's NN benchmark): the node
// holds the median of its set on (x[dim], id) along the largest-extent
// dimension; left = the elements before it, right = those after it.  The
// node's point goes first in its range so subtrees stay contiguous.  Every
// node keeps the tight box of its subtree (the truncation test, R21).
void nn_rec(tt_host_tree &t, int32_t b, int32_t e, int lvl) {
    const int D = t.dim;
    int32_t v = new_node(t, lvl, b, e);
    const int32_t n = e - b;
    float lo[TT_MAX_DIM], hi[TT_MAX_DIM];
    for (int d = 0; d < D; ++d) {
        lo[d] = std::numeric_limits<float>::infinity();
        hi[d] = -std::numeric_limits<float>::infinity();
    }
    for (int32_t i = b; i < e; ++i) {
        const float *p = &t.points[(size_t)t.ids[i] * D];
        for (int d = 0; d < D; ++d) {
            lo[d] = std::min(lo[d], p[d]);
            hi[d] = std::max(hi[d], p[d]);
        }
    }
    t.lo.insert(t.lo.end(), lo, lo + D);  // tight box of the subtree (can_correlate)
    t.hi.insert(t.hi.end(), hi, hi + D);
    if (n == 1) {
        t.body[v] = t.ids[b];
        t.skip[v] = (int32_t)t.level.size();
        return;
    }
    int sd = 0;
    float ext = hi[0] - lo[0];
    for (int d = 1; d < D; ++d) {
        float x = hi[d] - lo[d];
        if (x > ext) { ext = x; sd = d; }
    }
    const float *P = t.points.data();
    auto less = [P, D, sd](int32_t a, int32_t c) {
        float xa = P[(size_t)a * D + sd], xc = P[(size_t)c * D + sd];
        return xa < xc || (xa == xc && a < c);
    };
    const int32_t m = n / 2;
    std::nth_element(t.ids.begin() + b, t.ids.begin() + b + m, t.ids.begin() + e, less);
    // the left elements are those before position b+m; move the median to b
    std::rotate(t.ids.begin() + b, t.ids.begin() + b + m, t.ids.begin() + b + m + 1);
    const int32_t me = t.ids[b];
    t.body[v] = me;
    t.split_dim[v] = sd;
    t.split[v] = P[(size_t)me * D + sd];
    if (m > 0) {
        t.in_child[v] = (int32_t)t.level.size();
        nn_rec(t, b + 1, b + 1 + m, lvl + 1);
    }
    if (n - m - 1 > 0) {
        t.out_child[v] = (int32_t)t.level.size();
        nn_rec(t, b + 1 + m, e, lvl + 1);
    }
    t.first_child[v] = t.in_child[v] >= 0 ? t.in_child[v] : t.out_child[v];
    t.skip[v] = (int32_t)t.level.size();
}

template <class F>
tt_status guarded(F &&f) {
    try {
        return f();
    } catch (const std::bad_alloc &) {
        return TT_ERR_OOM;
    } catch (...) {
        return TT_ERR_INVALID_ARG;
    }
}

}  // namespace

extern "C" {

tt_status tt_build_kd(const float *pts, int64_t n, int32_t dim, int32_t ld, int32_t leaf_size,
                      tt_host_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim ||
        leaf_size <= 0)
        return TT_ERR_INVALID_ARG;
    return guarded([&] {
        auto *t = new tt_host_tree();
        t->kind = TT_KIND_KD;
        t->dim = dim;
        t->leaf_size = leaf_size;
        t->n_points = n;
        t->points.resize((size_t)n * dim);
        for (int64_t i = 0; i < n; ++i)
            std::memcpy(&t->points[(size_t)i * dim], pts + (size_t)i * ld, sizeof(float) * dim);
        t->ids.resize((size_t)n);
        for (int64_t i = 0; i < n; ++i) t->ids[i] = (int32_t)i;
        kd_rec(*t, 0, (int32_t)n, 0);
        *out = t;
        return TT_OK;
    });
}

tt_status tt_build_oct(const float *bodies, int64_t n, tt_host_tree **out) {
    if (!bodies || !out || n <= 0 || n > INT32_MAX / 3) return TT_ERR_INVALID_ARG;
    return guarded([&] {
        auto *t = new tt_host_tree();
        t->kind = TT_KIND_OCT;
        t->dim = 3;
        t->n_points = n;
        t->points.assign(bodies, bodies + (size_t)n * 4);
        float lo[3], hi[3];
        for (int d = 0; d < 3; ++d) {
            lo[d] = std::numeric_limits<float>::infinity();
            hi[d] = -std::numeric_limits<float>::infinity();
        }
        for (int64_t i = 0; i < n; ++i)
            for (int d = 0; d < 3; ++d) {
                lo[d] = std::min(lo[d], bodies[i * 4 + d]);
                hi[d] = std::max(hi[d], bodies[i * 4 + d]);
            }
        double side = 0.0;
        for (int d = 0; d < 3; ++d) {
            t->root_center[d] = ((double)lo[d] + (double)hi[d]) * 0.5;
            side = std::max(side, (double)hi[d] - (double)lo[d]);
        }
        if (side == 0.0) side = 1.0;
        t->root_side = side;
        t->ids.resize((size_t)n);
        for (int64_t i = 0; i < n; ++i) t->ids[i] = (int32_t)i;
        t->com.reserve((size_t)n * 8);
        oct_rec(*t, 0, (int32_t)n, t->root_center, side, 0);
        *out = t;
        return TT_OK;
    });
}

tt_status tt_build_vp(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_host_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim)
        return TT_ERR_INVALID_ARG;
    return guarded([&] {
        auto *t = new tt_host_tree();
        t->kind = TT_KIND_VP;
        t->dim = dim;
        t->n_points = n;
        t->points.resize((size_t)n * dim);
        for (int64_t i = 0; i < n; ++i)
            std::memcpy(&t->points[(size_t)i * dim], pts + (size_t)i * ld, sizeof(float) * dim);
        t->ids.resize((size_t)n);
        for (int64_t i = 0; i < n; ++i) t->ids[i] = (int32_t)i;
        std::vector<float> key((size_t)n);
        vp_rec(*t, 0, (int32_t)n, 0, key);
        *out = t;
        return TT_OK;
    });
}

tt_status tt_build_nn(const float *pts, int64_t n, int32_t dim, int32_t ld, tt_host_tree **out) {
    if (!pts || !out || n <= 0 || n > INT32_MAX / 2 || dim <= 0 || dim > TT_MAX_DIM || ld < dim)
        return TT_ERR_INVALID_ARG;
    return guarded([&] {
        auto *t = new tt_host_tree();
        t->kind = TT_KIND_NN;
        t->dim = dim;
        t->n_points = n;
        t->points.resize((size_t)n * dim);
        for (int64_t i = 0; i < n; ++i)
            std::memcpy(&t->points[(size_t)i * dim], pts + (size_t)i * ld, sizeof(float) * dim);
        t->ids.resize((size_t)n);
        for (int64_t i = 0; i < n; ++i) t->ids[i] = (int32_t)i;
        nn_rec(*t, 0, (int32_t)n, 0);
        *out = t;
        return TT_OK;
    });
}

void tt_host_tree_free(tt_host_tree *t) { delete t; }

tt_status tt_host_tree_desc(const tt_host_tree *t, tt_tree_desc *d) {
    if (!t || !d) return TT_ERR_INVALID_ARG;
    std::memset(d, 0, sizeof(*d));
    d->kind = t->kind;
    d->dim = t->dim;
    d->height = t->height;
    d->leaf_size = t->leaf_size;
    d->n_nodes = (int64_t)t->level.size();
    d->n_points = t->n_points;
    d->first_child = t->first_child.data();
    d->skip = t->skip.data();
    d->level = t->level.data();
    d->pbegin = t->pbegin.data();
    d->pcount = t->pcount.data();
    d->tree_order = t->ids.data();
    d->points = t->points.data();
    if (t->kind == TT_KIND_KD) {
        d->split_dim = t->split_dim.data();
        d->split = t->split.data();
        d->lo = t->lo.data();
        d->hi = t->hi.data();
    } else if (t->kind == TT_KIND_OCT) {
        d->com = t->com.data();
        d->body = t->body.data();
        for (int i = 0; i < 3; ++i) d->root_center[i] = t->root_center[i];
        d->root_side = t->root_side;
    } else if (t->kind == TT_KIND_NN) {
        d->body = t->body.data();  // the node's point id
        d->split_dim = t->split_dim.data();
        d->split = t->split.data();
        d->in_child = t->in_child.data();    // left
        d->out_child = t->out_child.data();  // right
        d->lo = t->lo.data();                // tight subtree boxes
        d->hi = t->hi.data();
    } else {
        d->body = t->body.data();  // vantage point id per node
        d->in_child = t->in_child.data();
        d->out_child = t->out_child.data();
        d->r_in_max = t->r_in_max.data();
        d->r_out_min = t->r_out_min.data();
    }
    return TT_OK;
}

}  // extern "C"
