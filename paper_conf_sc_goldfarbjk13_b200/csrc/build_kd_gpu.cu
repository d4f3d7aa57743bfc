// build_kd_gpu.cu -- kd-tree construction on the GPU (kd part),
// straight into the packed device blob (same bytes as tt_tree_pack of the host
// builder, R3 build rule).
//
// Level-synchronous median splits over one permutation array `ids`: every node
// owns a contiguous range [b, b+c) of it, so children keep their parent's
// range and a level is processed with whole-array passes:
//   * every element knows its range start b (rstart[i]); per-range data
//     (count, preorder index, split dim) live at index b of position arrays;
//   * tight boxes of all ranges created at this level: warp-segmented min/max
//     with one atomic per range run (float order via int/uint atomics);
//   * split dim = largest fp32 extent (lowest dim on ties);
//   * order inside the ranges: two stable global radix sorts keyed by
//     (b, id) then (b, x[dim]) -- ranges never move, so this sorts every range
//     by (x[dim], id) (internal nodes) or by id (leaves) in one go;
//   * children: left [b, b + c/2), right [b + c/2, b + c); preorder indices
//     follow from subtree sizes, which for median splits depend only on c.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <cstring>
#include <vector>

#include "build_common.cuh"

namespace {

// nodes of a subtree holding c points (median splits, leaf iff c <= L):
// a full binary tree, 2 * leaves - 1; at depth j the counts are
// ceil(c/2^j) (c mod 2^j of them) and floor(c/2^j) (the rest).
__host__ __device__ inline long long kd_nodes(long long c, int L) {
    if (c <= L) return 1;
    int j = 0;
    while (((c + (1ll << j) - 1) >> j) > L) ++j;  // smallest j: ceil(c/2^j) <= L
    const long long pj = 1ll << (j - 1);
    const long long hi = (c + pj - 1) / pj, lo = c / pj;
    const long long n_hi = (hi == lo) ? pj : c % pj, n_lo = pj - n_hi;
    long long leaves;
    if (lo > L || hi == lo) leaves = 2 * pj;  // every depth-(j-1) node splits
    else leaves = 2 * n_hi + n_lo;
    return 2 * leaves - 1;
}

__device__ __forceinline__ unsigned ordered(float x) {  // float -> order-preserving uint
    const unsigned u = __float_as_uint(x);
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

struct Level {
    int *rstart;       // [n] range start of element position i
    int *cnt, *cnt2;   // [n] count of the range starting at b (double buffered)
    int *pre, *pre2;   // [n] preorder index of the range starting at b
    int *sdim;         // [n] split dim of the internal range at b (-1 leaf)
    unsigned char *fresh, *fresh2;  // [n] range at b created at this level
    float *blo, *bhi;  // [n * D] box of the range at b (atomics)
};

__global__ void init_kernel(long long n, int *ids, int *rstart, int *cnt, int *pre, unsigned char *fresh) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        ids[i] = (int)i;
        rstart[i] = 0;
        cnt[i] = i == 0 ? (int)n : 0;
        pre[i] = 0;
        fresh[i] = i == 0;
    }
}

__global__ void box_init_kernel(long long n, int D, const int *rstart, const unsigned char *fresh, float *blo,
                                float *bhi) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (rstart[i] != i || !fresh[i]) continue;
        for (int d = 0; d < D; ++d) {
            blo[i * D + d] = INFINITY;
            bhi[i * D + d] = -INFINITY;
        }
    }
}

__device__ __forceinline__ void atomic_min_f(float *a, float v) {
    if (__float_as_int(v) >= 0) atomicMin(reinterpret_cast<int *>(a), __float_as_int(v));
    else atomicMax(reinterpret_cast<unsigned *>(a), __float_as_uint(v));
}
__device__ __forceinline__ void atomic_max_f(float *a, float v) {
    if (__float_as_int(v) >= 0) atomicMax(reinterpret_cast<int *>(a), __float_as_int(v));
    else atomicMin(reinterpret_cast<unsigned *>(a), __float_as_uint(v));
}

// tight boxes of the fresh ranges: a warp reduces each run of equal range
// starts among its 32 consecutive positions, one atomic per run and dim
__global__ void box_kernel(long long n, int D, const float *pts, int ld, const int *ids, const int *rstart,
                           const unsigned char *fresh, float *blo, float *bhi) {
    const int lane = threadIdx.x & 31;
    const long long nw = (n + 31) / 32;
    for (long long w = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / 32; w < nw;
         w += ((long long)gridDim.x * blockDim.x) / 32) {
        const long long i = w * 32 + lane;
        const bool in = i < n;
        const int b = in ? rstart[i] : -1;
        const bool act = in && fresh[b];
        const int prev = __shfl_up_sync(TT_FULL, b, 1);
        const bool head = act && (lane == 0 || prev != b);
        const unsigned heads = __ballot_sync(TT_FULL, head);
        for (int d = 0; d < D; ++d) {
            float mn = act ? pts[(long long)ids[i] * ld + d] : INFINITY;
            float mx = act ? mn : -INFINITY;
            // segmented (by equal b) reduction towards each run's head
            for (int o = 1; o < 32; o <<= 1) {
                const float omn = __shfl_down_sync(TT_FULL, mn, o);
                const float omx = __shfl_down_sync(TT_FULL, mx, o);
                const int ob = __shfl_down_sync(TT_FULL, b, o);
                if (lane + o < 32 && ob == b) {
                    mn = fminf(mn, omn);
                    mx = fmaxf(mx, omx);
                }
            }
            // the shuffle-down tree leaves each run's value at its head only if
            // the run is contiguous, which it is (ranges are contiguous)
            if ((heads >> lane) & 1u) {
                atomic_min_f(blo + (long long)b * D + d, mn);
                atomic_max_f(bhi + (long long)b * D + d, mx);
            }
        }
    }
}

// per fresh range: split dim (or -1 for a leaf)
__global__ void split_dim_kernel(long long n, int D, int L, const int *rstart, const int *cnt,
                                 const unsigned char *fresh, const float *blo, const float *bhi, int *sdim) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (rstart[i] != i) continue;
        if (!fresh[i] || cnt[i] <= L) {
            sdim[i] = -1;
            continue;
        }
        int sd = 0;
        float ext = bhi[i * D] - blo[i * D];
        for (int d = 1; d < D; ++d) {
            const float e = bhi[i * D + d] - blo[i * D + d];
            if (e > ext) {
                ext = e;
                sd = d;
            }
        }
        sdim[i] = sd;
    }
}

// pass 1 key: (b, id); pass 2 key: (b, x[dim]) for internal ranges, (b, 0) otherwise
__global__ void key_kernel(long long n, int pass, const float *pts, int ld, const int *ids, const int *rstart,
                           const int *sdim, const unsigned char *fresh, unsigned long long *key) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        unsigned lowbits;
        if (pass == 1) lowbits = (unsigned)ids[i];
        else lowbits = (fresh[b] && sdim[b] >= 0) ? ordered(pts[(long long)ids[i] * ld + sdim[b]]) : 0u;
        key[i] = ((unsigned long long)(unsigned)b << 32) | lowbits;
    }
}

struct NodeOut {
    int *level, *skip, *first_child, *split_dim, *pbegin, *pcount;
    float *split, *lo, *hi;  // canonical preorder, lo/hi [nodes * D]
};

// record the fresh ranges as nodes and create the next level's ranges
__global__ void emit_kernel(long long n, int D, int L, int level, const float *pts, int ld, const int *ids,
                            Level lv, NodeOut out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = lv.rstart[i];
        const int c = lv.cnt[b];
        const bool fresh = lv.fresh[b];
        if (i == b) {  // the range head writes the node and the children's heads
            if (fresh) {
                const int v = lv.pre[b];
                out.level[v] = level;
                out.skip[v] = v + (int)kd_nodes(c, L);
                out.pbegin[v] = b;
                out.pcount[v] = c;
                for (int d = 0; d < D; ++d) {
                    out.lo[(long long)v * D + d] = lv.blo[(long long)b * D + d];
                    out.hi[(long long)v * D + d] = lv.bhi[(long long)b * D + d];
                }
                const int sd = lv.sdim[b];
                out.split_dim[v] = sd;
                if (sd >= 0) {
                    const int m = b + c / 2;
                    out.split[v] = pts[(long long)ids[m] * ld + sd];
                    out.first_child[v] = v + 1;
                    lv.cnt2[b] = c / 2;
                    lv.pre2[b] = v + 1;
                    lv.fresh2[b] = 1;
                    lv.cnt2[m] = c - c / 2;
                    lv.pre2[m] = v + 1 + (int)kd_nodes(c / 2, L);
                    lv.fresh2[m] = 1;
                } else {
                    out.split[v] = 0.0f;
                    out.first_child[v] = -1;
                    lv.cnt2[b] = c;
                    lv.pre2[b] = v;
                    lv.fresh2[b] = 0;
                }
            } else {
                lv.cnt2[b] = c;
                lv.pre2[b] = lv.pre[b];
                lv.fresh2[b] = 0;
            }
        }
    }
}

__global__ void restart_kernel(long long n, int L, const int *cnt, const unsigned char *fresh, const int *sdim,
                               int *rstart) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        if (fresh[b] && sdim[b] >= 0) {
            const int m = b + cnt[b] / 2;
            rstart[i] = i >= m ? m : b;
        }
    }
}

__global__ void count_fresh_kernel(long long n, const int *rstart, const unsigned char *fresh2, int *flag) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        if (rstart[i] == i && fresh2[i]) atomicAdd(flag, 1);
}

__global__ void kd_records_kernel(long long nn, int D, int dp, NodeOut o, const int *newidx, tt_kd_rec *rec,
                                  float *box, float *cbox) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x) {
        const int nv = newidx[v];
        tt_kd_rec r;
        const int l = o.first_child[v];
        auto map = [&](int c) { return (c < 0 || c >= nn) ? TT_END : newidx[c]; };
        r.left = map(l);
        r.right = l >= 0 ? map(o.skip[l]) : TT_END;
        r.skip = map(o.skip[v]);
        r.level = o.level[v];
        r.split = o.split[v];
        r.dim = o.split_dim[v];
        r.pbegin = o.pbegin[v];
        r.pcount = o.pcount[v];
        rec[nv] = r;
        for (int k = 0; k < D; ++k) {
            box[(long long)nv * 2 * dp + k] = o.lo[(long long)v * D + k];
            box[(long long)nv * 2 * dp + dp + k] = o.hi[(long long)v * D + k];
        }
        if (l >= 0) {
            const int kids[2] = {l, o.skip[l]};
            for (int c = 0; c < 2; ++c)
                for (int k = 0; k < D; ++k) {
                    cbox[(long long)nv * 4 * dp + c * 2 * dp + k] = o.lo[(long long)kids[c] * D + k];
                    cbox[(long long)nv * 4 * dp + c * 2 * dp + dp + k] = o.hi[(long long)kids[c] * D + k];
                }
        }
    }
}

__global__ void kd_points_kernel(long long n, int D, int dp, const float *pts, int ld, const int *ids, float *opts,
                                 int *pid) {
    for (long long j = blockIdx.x * (long long)blockDim.x + threadIdx.x; j < n; j += (long long)gridDim.x * blockDim.x) {
        const int id = ids[j];
        pid[j] = id;
        for (int k = 0; k < D; ++k) opts[j * dp + k] = pts[(long long)id * ld + k];
    }
}

}  // namespace

int tt_build_kd_gpu_impl(const float *pts, long long n, int D, int ld, int L, void *stream, tt_blob_header *hdr_out,
                         void **blob_out) {
    cudaStream_t s = (cudaStream_t)stream;
    tt_keep_pool_memory();
    Scratch W{s};
    const unsigned G = build_grid(n);
    int *ids = W.get<int>(n), *ids2 = W.get<int>(n);
    Level lv;
    lv.rstart = W.get<int>(n);
    lv.cnt = W.get<int>(n);
    lv.cnt2 = W.get<int>(n);
    lv.pre = W.get<int>(n);
    lv.pre2 = W.get<int>(n);
    lv.sdim = W.get<int>(n);
    lv.fresh = W.get<unsigned char>(n);
    lv.fresh2 = W.get<unsigned char>(n);
    lv.blo = W.get<float>(n * D);
    lv.bhi = W.get<float>(n * D);
    auto *key = W.get<unsigned long long>(n), *key2 = W.get<unsigned long long>(n);
    int *flag = W.get<int>(1);
    const long long nn = kd_nodes(n, L);
    NodeOut o;
    o.level = W.get<int>(nn);
    o.skip = W.get<int>(nn);
    o.first_child = W.get<int>(nn);
    o.split_dim = W.get<int>(nn);
    o.pbegin = W.get<int>(nn);
    o.pcount = W.get<int>(nn);
    o.split = W.get<float>(nn);
    o.lo = W.get<float>(nn * D);
    o.hi = W.get<float>(nn * D);
    size_t sb = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, sb, key, key2, ids, ids2, (int)n, 0, 64, s);
    void *st = W.get<unsigned char>(sb);
    if (W.e) return W.e;
    cudaError_t e;
    init_kernel<<<G, 256, 0, s>>>(n, ids, lv.rstart, lv.cnt, lv.pre, lv.fresh);
    for (int level = 0;; ++level) {
        box_init_kernel<<<G, 256, 0, s>>>(n, D, lv.rstart, lv.fresh, lv.blo, lv.bhi);
        box_kernel<<<G, 256, 0, s>>>(n, D, pts, ld, ids, lv.rstart, lv.fresh, lv.blo, lv.bhi);
        split_dim_kernel<<<G, 256, 0, s>>>(n, D, L, lv.rstart, lv.cnt, lv.fresh, lv.blo, lv.bhi, lv.sdim);
        for (int pass = 1; pass <= 2; ++pass) {
            key_kernel<<<G, 256, 0, s>>>(n, pass, pts, ld, ids, lv.rstart, lv.sdim, lv.fresh, key);
            size_t q = sb;
            if ((e = cub::DeviceRadixSort::SortPairs(st, q, key, key2, ids, ids2, (int)n, 0, 64, s))) return e;
            std::swap(ids, ids2);
        }
        emit_kernel<<<G, 256, 0, s>>>(n, D, L, level, pts, ld, ids, lv, o);
        restart_kernel<<<G, 256, 0, s>>>(n, L, lv.cnt, lv.fresh, lv.sdim, lv.rstart);
        std::swap(lv.cnt, lv.cnt2);
        std::swap(lv.pre, lv.pre2);
        std::swap(lv.fresh, lv.fresh2);
        // another level iff some range was created by this one
        if ((e = cudaMemsetAsync(flag, 0, sizeof(int), s))) return e;
        count_fresh_kernel<<<G, 256, 0, s>>>(n, lv.rstart, lv.fresh, flag);
        int hf = 0;
        if ((e = cudaMemcpyAsync(&hf, flag, sizeof(int), cudaMemcpyDeviceToHost, s))) return e;
        if ((e = cudaStreamSynchronize(s))) return e;
        if (!hf) break;
        if (level > TT_MAX_HEIGHT) return cudaErrorInvalidValue;
    }

    // header + top-first renumbering (pack.cpp plan)
    const int dp = (D + 3) & ~3;
    tt_blob_header h;
    header_base(h, TT_KIND_KD, D, L, nn, n);
    h.rec_bytes = 32;
    int *newidx = W.get<int>(nn);
    if (W.e) return W.e;
    if ((e = renumber_top_first(o.level, nn, 32 + 8 * dp, h, newidx, W))) return e;
    const unsigned GN = build_grid(nn);
    uint64_t off = align256(sizeof(tt_blob_header));
    h.off_rec = off;
    off = align256(off + (uint64_t)nn * 32);
    h.off_box = off;
    off = align256(off + (uint64_t)nn * 2 * dp * 4);
    h.off_pts = off;
    off = align256(off + (uint64_t)n * dp * 4);
    h.off_pid = off;
    off = align256(off + (uint64_t)n * 4);
    h.off_cbox = off;
    off = align256(off + (uint64_t)nn * 4 * dp * 4);
    h.total = off;
    void *blob = nullptr;
    if ((e = alloc_blob(h, s, &blob))) return e;
    auto *base = static_cast<unsigned char *>(blob);
    kd_records_kernel<<<GN, 256, 0, s>>>(nn, D, dp, o, newidx, reinterpret_cast<tt_kd_rec *>(base + h.off_rec),
                                         reinterpret_cast<float *>(base + h.off_box),
                                         reinterpret_cast<float *>(base + h.off_cbox));
    kd_points_kernel<<<G, 256, 0, s>>>(n, D, dp, pts, ld, ids, reinterpret_cast<float *>(base + h.off_pts),
                                      reinterpret_cast<int *>(base + h.off_pid));
    if ((e = cudaGetLastError()) || (e = cudaStreamSynchronize(s))) {
        tt_blob_discard(blob);
        return e;
    }
    *hdr_out = h;
    *blob_out = blob;
    return 0;
}
