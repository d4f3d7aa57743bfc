// build_nn_gpu.cu -- point-per-node kd-tree (the NN benchmark's tree, reading
// R21) built on the GPU straight into the packed device blob: the same bytes
// as tt_tree_pack of tt_build_nn.
//
// The level-synchronous scheme of build_kd_gpu.cu / build_vp_gpu.cu: every
// node owns a range [b, b+c) of one permutation array; per level
//   * tight boxes of the ranges created at this level (warp-segmented min/max,
//     one atomic per range run and dim);
//   * split dim = largest fp32 extent (lowest dim on ties);
//   * two stable global radix sorts keyed (b, id) then (b, x[dim]) sort every
//     fresh range by (x[dim], id);
//   * the node takes the element at b + c/2 (its point and split value); the
//     elements before it form the left range, those after it the right one,
//     and the median's own position becomes a finished one-point range.
// A node's subtree holds exactly its c points, so the preorder index of the
// left child is pre+1, of the right child pre+1+c/2, and the rope pre+c.
#include <cub/device/device_radix_sort.cuh>

#include "build_common.cuh"

namespace {

__device__ __forceinline__ unsigned ordered_f(float x) {  // float -> order-preserving uint
    const unsigned u = __float_as_uint(x);
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

__device__ __forceinline__ void atomic_min_f(float *a, float v) {
    if (__float_as_int(v) >= 0) atomicMin(reinterpret_cast<int *>(a), __float_as_int(v));
    else atomicMax(reinterpret_cast<unsigned *>(a), __float_as_uint(v));
}
__device__ __forceinline__ void atomic_max_f(float *a, float v) {
    if (__float_as_int(v) >= 0) atomicMax(reinterpret_cast<int *>(a), __float_as_int(v));
    else atomicMin(reinterpret_cast<unsigned *>(a), __float_as_uint(v));
}

__global__ void ninit_kernel(long long n, int D, int *ids, int *rstart, int *cnt, int *pre, unsigned char *fresh) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        ids[i] = (int)i;
        rstart[i] = 0;
        cnt[i] = i == 0 ? (int)n : 0;
        pre[i] = 0;
        fresh[i] = i == 0;
    }
}

__global__ void nbox_init_kernel(long long n, int D, const int *rstart, const unsigned char *fresh, float *blo,
                                 float *bhi) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (rstart[i] != i || !fresh[i]) continue;
        for (int d = 0; d < D; ++d) {
            blo[i * D + d] = INFINITY;
            bhi[i * D + d] = -INFINITY;
        }
    }
}

// tight boxes of the fresh ranges (ranges are contiguous runs of equal b)
__global__ void nbox_kernel(long long n, int D, const float *pts, int ld, const int *ids, const int *rstart,
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
            for (int o = 1; o < 32; o <<= 1) {
                const float omn = __shfl_down_sync(TT_FULL, mn, o);
                const float omx = __shfl_down_sync(TT_FULL, mx, o);
                const int ob = __shfl_down_sync(TT_FULL, b, o);
                if (lane + o < 32 && ob == b) {
                    mn = fminf(mn, omn);
                    mx = fmaxf(mx, omx);
                }
            }
            if ((heads >> lane) & 1u) {
                atomic_min_f(blo + (long long)b * D + d, mn);
                atomic_max_f(bhi + (long long)b * D + d, mx);
            }
        }
    }
}

// split dim of every fresh range of >= 2 points (-1: a one-point leaf)
__global__ void nsplit_dim_kernel(long long n, int D, const int *rstart, const int *cnt, const unsigned char *fresh,
                                  const float *blo, const float *bhi, int *sdim) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (rstart[i] != i) continue;
        if (!fresh[i] || cnt[i] < 2) {
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

// pass 1 key (b, id); pass 2 key (b, x[dim]) for fresh internal ranges
__global__ void nkey_kernel(long long n, int pass, const float *pts, int ld, const int *ids, const int *rstart,
                            const int *sdim, const unsigned char *fresh, unsigned long long *key) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        unsigned low;
        if (pass == 1) low = (unsigned)ids[i];
        else low = (fresh[b] && sdim[b] >= 0) ? ordered_f(pts[(long long)ids[i] * ld + sdim[b]]) : 0u;
        key[i] = ((unsigned long long)(unsigned)b << 32) | low;
    }
}

struct NnOut {
    int *level, *left, *right, *sdim, *pt;
    float *split, *lo, *hi;  // canonical preorder; lo/hi [nodes * D]
};

__global__ void nemit_kernel(long long n, int D, int level, const float *pts, int ld, const int *ids,
                             const int *rstart, const int *cnt, const int *pre, const unsigned char *fresh,
                             const int *sdim, const float *blo, const float *bhi, int *cnt2, int *pre2,
                             unsigned char *fresh2, NnOut o) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        if (i != b) continue;
        const int c = cnt[b];
        if (!fresh[b]) {
            cnt2[b] = c;
            pre2[b] = pre[b];
            fresh2[b] = 0;
            continue;
        }
        const int v = pre[b];
        o.level[v] = level;
        for (int d = 0; d < D; ++d) {
            o.lo[(long long)v * D + d] = blo[(long long)b * D + d];
            o.hi[(long long)v * D + d] = bhi[(long long)b * D + d];
        }
        const int sd = sdim[b];
        o.sdim[v] = sd;
        if (sd < 0) {  // one point: a leaf
            o.pt[v] = ids[b];
            o.split[v] = 0.0f;
            o.left[v] = o.right[v] = -1;
            cnt2[b] = 1;
            pre2[b] = v;
            fresh2[b] = 0;
            continue;
        }
        const int m = c / 2, nr = c - m - 1;
        const int me = ids[b + m];
        o.pt[v] = me;
        o.split[v] = pts[(long long)me * ld + sd];
        o.left[v] = v + 1;  // m >= 1
        o.right[v] = nr > 0 ? v + 1 + m : -1;
        cnt2[b] = m;
        pre2[b] = v + 1;
        fresh2[b] = 1;
        cnt2[b + m] = 1;  // the node's own point: a finished one-point range
        pre2[b + m] = v;
        fresh2[b + m] = 0;
        if (nr > 0) {
            cnt2[b + m + 1] = nr;
            pre2[b + m + 1] = v + 1 + m;
            fresh2[b + m + 1] = 1;
        }
    }
}

__global__ void nrestart_kernel(long long n, const int *cnt, const unsigned char *fresh, const int *sdim,
                                int *rstart) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        if (!fresh[b] || sdim[b] < 0) continue;
        const int m = b + cnt[b] / 2;
        rstart[i] = i < m ? b : (i == m ? m : m + 1);
    }
}

__global__ void ncount_fresh_kernel(long long n, const int *rstart, const unsigned char *fresh, int *flag) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        if (rstart[i] == i && fresh[i]) atomicAdd(flag, 1);
}

__global__ void nn_records_kernel(long long nn, int D, int dp, const float *pts, int ld, NnOut o, const int *newidx,
                                  tt_nn_rec *rec, float *box, float *vpt, int *pid) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x) {
        const int nv = newidx[v];
        tt_nn_rec r;
        r.left = o.left[v] >= 0 ? newidx[o.left[v]] : TT_END;
        r.right = o.right[v] >= 0 ? newidx[o.right[v]] : TT_END;
        r.split = o.split[v];
        r.dim = o.sdim[v];
        rec[nv] = r;
        pid[nv] = o.pt[v];
        for (int k = 0; k < D; ++k) {
            box[(long long)nv * 2 * dp + k] = o.lo[(long long)v * D + k];
            box[(long long)nv * 2 * dp + dp + k] = o.hi[(long long)v * D + k];
            vpt[(long long)nv * dp + k] = pts[(long long)o.pt[v] * ld + k];
        }
    }
}

}  // namespace

int tt_build_nn_gpu_impl(const float *pts, long long n, int D, int ld, void *stream, tt_blob_header *hdr_out,
                         void **blob_out) {
    cudaStream_t s = (cudaStream_t)stream;
    tt_keep_pool_memory();
    Scratch W{s};
    const unsigned G = build_grid(n);
    int *ids = W.get<int>(n), *ids2 = W.get<int>(n);
    int *rstart = W.get<int>(n), *cnt = W.get<int>(n), *cnt2 = W.get<int>(n), *pre = W.get<int>(n),
        *pre2 = W.get<int>(n), *sdim = W.get<int>(n);
    unsigned char *fresh = W.get<unsigned char>(n), *fresh2 = W.get<unsigned char>(n);
    float *blo = W.get<float>(n * D), *bhi = W.get<float>(n * D);
    auto *key = W.get<unsigned long long>(n), *key2 = W.get<unsigned long long>(n);
    int *flag = W.get<int>(1);
    const long long nn = n;
    NnOut o;
    o.level = W.get<int>(nn);
    o.left = W.get<int>(nn);
    o.right = W.get<int>(nn);
    o.sdim = W.get<int>(nn);
    o.pt = W.get<int>(nn);
    o.split = W.get<float>(nn);
    o.lo = W.get<float>(nn * D);
    o.hi = W.get<float>(nn * D);
    size_t sb = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, sb, key, key2, ids, ids2, (int)n, 0, 64, s);
    void *st = W.get<unsigned char>(sb);
    if (W.e) return W.e;
    cudaError_t e;
    ninit_kernel<<<G, 256, 0, s>>>(n, D, ids, rstart, cnt, pre, fresh);
    for (int level = 0;; ++level) {
        nbox_init_kernel<<<G, 256, 0, s>>>(n, D, rstart, fresh, blo, bhi);
        nbox_kernel<<<G, 256, 0, s>>>(n, D, pts, ld, ids, rstart, fresh, blo, bhi);
        nsplit_dim_kernel<<<G, 256, 0, s>>>(n, D, rstart, cnt, fresh, blo, bhi, sdim);
        for (int pass = 1; pass <= 2; ++pass) {
            nkey_kernel<<<G, 256, 0, s>>>(n, pass, pts, ld, ids, rstart, sdim, fresh, key);
            size_t q = sb;
            if ((e = cub::DeviceRadixSort::SortPairs(st, q, key, key2, ids, ids2, (int)n, 0, 64, s))) return e;
            std::swap(ids, ids2);
        }
        nemit_kernel<<<G, 256, 0, s>>>(n, D, level, pts, ld, ids, rstart, cnt, pre, fresh, sdim, blo, bhi, cnt2, pre2,
                                       fresh2, o);
        nrestart_kernel<<<G, 256, 0, s>>>(n, cnt, fresh, sdim, rstart);
        std::swap(cnt, cnt2);
        std::swap(pre, pre2);
        std::swap(fresh, fresh2);
        if ((e = cudaMemsetAsync(flag, 0, sizeof(int), s))) return e;
        ncount_fresh_kernel<<<G, 256, 0, s>>>(n, rstart, fresh, flag);
        int hf = 0;
        if ((e = cudaMemcpyAsync(&hf, flag, sizeof(int), cudaMemcpyDeviceToHost, s))) return e;
        if ((e = cudaStreamSynchronize(s))) return e;
        if (!hf) break;
        if (level > TT_MAX_HEIGHT) return cudaErrorInvalidValue;
    }
    const int dp = (D + 3) & ~3;
    tt_blob_header h;
    header_base(h, TT_KIND_NN, D, 1, nn, n);
    h.rec_bytes = 16;
    int *newidx = W.get<int>(nn);
    if (W.e) return W.e;
    if ((e = renumber_top_first(o.level, nn, 16 + 12 * dp, h, newidx, W))) return e;
    uint64_t off = align256(sizeof(tt_blob_header));
    h.off_rec = off;
    off = align256(off + (uint64_t)nn * 16);
    h.off_box = off;
    off = align256(off + (uint64_t)nn * 2 * dp * 4);
    h.off_vpt = off;
    off = align256(off + (uint64_t)nn * dp * 4);
    h.off_pid = off;
    off = align256(off + (uint64_t)nn * 4);
    h.total = off;
    void *blob = nullptr;
    if ((e = alloc_blob(h, s, &blob))) return e;
    auto *base = static_cast<unsigned char *>(blob);
    nn_records_kernel<<<build_grid(nn), 256, 0, s>>>(nn, D, dp, pts, ld, o, newidx,
                                                     reinterpret_cast<tt_nn_rec *>(base + h.off_rec),
                                                     reinterpret_cast<float *>(base + h.off_box),
                                                     reinterpret_cast<float *>(base + h.off_vpt),
                                                     reinterpret_cast<int *>(base + h.off_pid));
    if ((e = cudaGetLastError()) || (e = cudaStreamSynchronize(s))) {
        tt_blob_discard(blob);
        return e;
    }
    *hdr_out = h;
    *blob_out = blob;
    return 0;
}
