// build_vp_gpu.cu -- vantage-point tree construction on the GPU (SURVEY NEXT-1,
// vp part), straight into the packed device blob (same bytes as tt_tree_pack
// of the host builder, R12 build rule).
//
// Same level-synchronous scheme as build_kd_gpu.cu: every node owns a range
// [b, b+c) of one permutation array; per level two stable global radix sorts
// order every fresh range by (b, id) -- which puts the vantage point (the
// smallest id) at b -- and then by (b, pinned d2 to that vantage point), the
// vantage point itself keyed 0 so it stays first.  Inside = the next
// floor((c-1)/2) positions, outside = the rest; a node's subtree holds exactly
// its c points, so preorder indices are b-independent offsets: inside child
// pre+1, outside child pre+1+nin, rope pre+c.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <cstring>
#include <vector>

#include "build_common.cuh"

namespace {

__device__ __forceinline__ unsigned ordered_nonneg(float x) { return __float_as_uint(x) | 0x80000000u; }

template <int DIM>
__device__ __forceinline__ float d2_to(const float *pts, int ld, int a, int b) {
    float q[DIM];
#pragma unroll
    for (int d = 0; d < DIM; ++d) q[d] = pts[(long long)a * ld + d];
    float p[DIM];
#pragma unroll
    for (int d = 0; d < DIM; ++d) p[d] = pts[(long long)b * ld + d];
    return tt::pinned_d2<DIM>(q, p);
}

__global__ void vinit_kernel(long long n, int *ids, int *rstart, int *cnt, int *pre, unsigned char *fresh) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        ids[i] = (int)i;
        rstart[i] = 0;
        cnt[i] = i == 0 ? (int)n : 0;
        pre[i] = 0;
        fresh[i] = i == 0;
    }
}

template <int DIM>
__global__ void vkey_kernel(long long n, int pass, const float *pts, int ld, const int *ids, const int *rstart,
                            const unsigned char *fresh, unsigned long long *key) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        unsigned low;
        if (pass == 1) low = (unsigned)ids[i];
        else if (!fresh[b] || i == b) low = 0u;  // the vantage point (smallest id) stays first
        else low = ordered_nonneg(d2_to<DIM>(pts, ld, ids[b], ids[i]));
        key[i] = ((unsigned long long)(unsigned)b << 32) | low;
    }
}

struct VpOut {
    int *level, *skip, *first_child, *in_child, *out_child, *vp, *pbegin, *pcount;
    float *rin, *rout;
};

template <int DIM>
__global__ void vemit_kernel(long long n, int level, const float *pts, int ld, const int *ids, const int *rstart,
                             const int *cnt, const int *pre, const unsigned char *fresh, int *cnt2, int *pre2,
                             unsigned char *fresh2, VpOut o) {
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
        const int r = c - 1, nin = r / 2;
        o.level[v] = level;
        o.skip[v] = v + c;
        o.vp[v] = ids[b];
        o.pbegin[v] = b;
        o.pcount[v] = c;
        o.in_child[v] = nin > 0 ? v + 1 : -1;
        o.out_child[v] = r - nin > 0 ? v + 1 + nin : -1;
        o.first_child[v] = r == 0 ? -1 : (nin > 0 ? v + 1 : v + 1 + nin);
        o.rin[v] = nin > 0 ? __fsqrt_rn(d2_to<DIM>(pts, ld, ids[b], ids[b + nin])) : 0.0f;
        o.rout[v] = r > 0 ? __fsqrt_rn(d2_to<DIM>(pts, ld, ids[b], ids[b + 1 + nin])) : 0.0f;
        // the vantage point's position becomes a finished one-point range
        cnt2[b] = 1;
        pre2[b] = v;
        fresh2[b] = 0;
        if (nin > 0) {
            cnt2[b + 1] = nin;
            pre2[b + 1] = v + 1;
            fresh2[b + 1] = 1;
        }
        if (r - nin > 0) {
            cnt2[b + 1 + nin] = r - nin;
            pre2[b + 1 + nin] = v + 1 + nin;
            fresh2[b + 1 + nin] = 1;
        }
    }
}

__global__ void vrestart_kernel(long long n, const int *cnt, const unsigned char *fresh, int *rstart) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int b = rstart[i];
        if (!fresh[b] || i == b) continue;
        const int nin = (cnt[b] - 1) / 2;
        rstart[i] = i < b + 1 + nin ? b + 1 : b + 1 + nin;
    }
}

__global__ void vcount_fresh_kernel(long long n, const int *rstart, const unsigned char *fresh, int *flag) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        if (rstart[i] == i && fresh[i]) atomicAdd(flag, 1);
}

__global__ void vp_records_kernel(long long nn, int D, int dp, const float *pts, int ld, VpOut o, const int *newidx,
                                  tt_vp_rec *rec, float *vpt, int *pid) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x) {
        const int nv = newidx[v];
        tt_vp_rec r;
        r.in = o.in_child[v] >= 0 ? newidx[o.in_child[v]] : TT_END;
        r.out = o.out_child[v] >= 0 ? newidx[o.out_child[v]] : TT_END;
        r.r_in_max = o.rin[v];
        r.r_out_min = o.rout[v];
        rec[nv] = r;
        pid[nv] = o.vp[v];
        for (int k = 0; k < D; ++k) vpt[(long long)nv * dp + k] = pts[(long long)o.vp[v] * ld + k];
    }
}

template <int DIM>
int build_vp(const float *pts, long long n, int ld, cudaStream_t s, tt_blob_header *hdr_out, void **blob_out) {
    constexpr int D = DIM;
    tt_keep_pool_memory();
    Scratch W{s};
    const unsigned G = build_grid(n);
    int *ids = W.get<int>(n), *ids2 = W.get<int>(n);
    int *rstart = W.get<int>(n), *cnt = W.get<int>(n), *cnt2 = W.get<int>(n), *pre = W.get<int>(n),
        *pre2 = W.get<int>(n);
    unsigned char *fresh = W.get<unsigned char>(n), *fresh2 = W.get<unsigned char>(n);
    auto *key = W.get<unsigned long long>(n), *key2 = W.get<unsigned long long>(n);
    int *flag = W.get<int>(1);
    const long long nn = n;
    VpOut o;
    o.level = W.get<int>(nn);
    o.skip = W.get<int>(nn);
    o.first_child = W.get<int>(nn);
    o.in_child = W.get<int>(nn);
    o.out_child = W.get<int>(nn);
    o.vp = W.get<int>(nn);
    o.pbegin = W.get<int>(nn);
    o.pcount = W.get<int>(nn);
    o.rin = W.get<float>(nn);
    o.rout = W.get<float>(nn);
    size_t sb = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, sb, key, key2, ids, ids2, (int)n, 0, 64, s);
    void *st = W.get<unsigned char>(sb);
    if (W.e) return W.e;
    cudaError_t e;
    vinit_kernel<<<G, 256, 0, s>>>(n, ids, rstart, cnt, pre, fresh);
    for (int level = 0;; ++level) {
        for (int pass = 1; pass <= 2; ++pass) {
            vkey_kernel<DIM><<<G, 256, 0, s>>>(n, pass, pts, ld, ids, rstart, fresh, key);
            size_t q = sb;
            if ((e = cub::DeviceRadixSort::SortPairs(st, q, key, key2, ids, ids2, (int)n, 0, 64, s))) return e;
            std::swap(ids, ids2);
        }
        vemit_kernel<DIM><<<G, 256, 0, s>>>(n, level, pts, ld, ids, rstart, cnt, pre, fresh, cnt2, pre2, fresh2, o);
        vrestart_kernel<<<G, 256, 0, s>>>(n, cnt, fresh, rstart);
        std::swap(cnt, cnt2);
        std::swap(pre, pre2);
        std::swap(fresh, fresh2);
        if ((e = cudaMemsetAsync(flag, 0, sizeof(int), s))) return e;
        vcount_fresh_kernel<<<G, 256, 0, s>>>(n, rstart, fresh, flag);
        int hf = 0;
        if ((e = cudaMemcpyAsync(&hf, flag, sizeof(int), cudaMemcpyDeviceToHost, s))) return e;
        if ((e = cudaStreamSynchronize(s))) return e;
        if (!hf) break;
        if (level > TT_MAX_HEIGHT) return cudaErrorInvalidValue;
    }
    const int dp = (D + 3) & ~3;
    tt_blob_header h;
    header_base(h, TT_KIND_VP, D, 1, nn, n);
    h.rec_bytes = 16;
    int *newidx = W.get<int>(nn);
    if (W.e) return W.e;
    if ((e = renumber_top_first(o.level, nn, 16 + 4 * dp, h, newidx, W))) return e;
    uint64_t off = align256(sizeof(tt_blob_header));
    h.off_rec = off;
    off = align256(off + (uint64_t)nn * 16);
    h.off_vpt = off;
    off = align256(off + (uint64_t)nn * dp * 4);
    h.off_pid = off;
    off = align256(off + (uint64_t)nn * 4);
    h.total = off;
    void *blob = nullptr;
    if ((e = alloc_blob(h, s, &blob))) return e;
    auto *base = static_cast<unsigned char *>(blob);
    vp_records_kernel<<<G, 256, 0, s>>>(nn, D, dp, pts, ld, o, newidx, reinterpret_cast<tt_vp_rec *>(base + h.off_rec),
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

}  // namespace

int tt_build_vp_gpu_impl(const float *pts, long long n, int dim, int ld, void *stream, tt_blob_header *hdr,
                         void **blob) {
    cudaStream_t s = (cudaStream_t)stream;
    switch (dim) {
    case 1: return build_vp<1>(pts, n, ld, s, hdr, blob);
    case 2: return build_vp<2>(pts, n, ld, s, hdr, blob);
    case 3: return build_vp<3>(pts, n, ld, s, hdr, blob);
    case 4: return build_vp<4>(pts, n, ld, s, hdr, blob);
    case 5: return build_vp<5>(pts, n, ld, s, hdr, blob);
    case 6: return build_vp<6>(pts, n, ld, s, hdr, blob);
    case 7: return build_vp<7>(pts, n, ld, s, hdr, blob);
    case 8: return build_vp<8>(pts, n, ld, s, hdr, blob);
    case 16: return build_vp<16>(pts, n, ld, s, hdr, blob);
    default: return (int)cudaErrorInvalidValue;
    }
}
