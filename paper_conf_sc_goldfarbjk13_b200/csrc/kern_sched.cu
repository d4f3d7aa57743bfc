// kern_sched.cu -- longest-first tile schedule (a1b).
//
// The traversal kernels are persistent: each warp takes the next 32-point
// tile (64 for the oct-tree kernel) of the launch order from a global atomic
// counter.  Tile costs vary (cv ~0.55 for kNN/VP), and with ~6 tiles per
// resident warp the tiles handed out last set a long tail.  Dispatching the
// expensive tiles first (Graham's longest-processing-time rule) removes most
// of it.  The cost of a tile is estimated from one greedy descent per point,
// the same descent the point sort makes:
//   kd : the leaf reached by the split rule; the largest pinned d2 from the
//        point to that leaf's points (an upper bound on the point's k-NN
//        radius when the leaf holds >= k points: the ball the search must
//        cover);
//   vp : the smallest distance to a vantage point on the inside-iff-d<=r_in
//        path (the tau the search starts pruning with);
//   nn : the smallest pinned d2 to a node point on the left-iff-x<split
//        path (likewise).
// tile key = the largest estimate of its points (a lockstep warp runs as long
// as its most expensive lane).  Whole tiles move; the points inside a tile
// and the ragged last tile stay where they are, so the similarity of the
// point sort is kept and results are unchanged (they never depend on order).
// The radix sort of the tile keys is CUB's (a library sort primitive).
#include <cub/device/device_radix_sort.cuh>

#include "kern_common.cuh"

namespace {

using namespace tt;

int grid_for(long long n) {
    long long g = (n + 255) / 256;
    if (g > 148 * 16) g = 148 * 16;
    return (int)(g < 1 ? 1 : g);
}

template <int DIM>
__device__ __forceinline__ float kd_cost(const tt_kd_rec *rec, const float *tpts, int dp, const float (&q)[DIM]) {
    int cur = 0;
    for (;;) {
        const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
        const int4 u = __ldg(reinterpret_cast<const int4 *>(rec + cur) + 1);
        if (t.x < 0) {
            float c = 0.f;
            for (int j = u.z; j < u.z + u.w; ++j) {
                float p[DIM];
                load_row_nc<DIM>(p, tpts + (size_t)j * dp);
                c = fmaxf(c, pinned_d2<DIM>(q, p));
            }
            return c;
        }
        cur = select_dim<DIM>(q, u.y) < __int_as_float(u.x) ? t.x : t.y;
    }
}

template <int DIM>
__device__ __forceinline__ float vp_cost(const tt_vp_rec *rec, const float *vpt, int dp, const float (&q)[DIM]) {
    int cur = 0;
    float best = __int_as_float(0x7f800000);
    for (int l = 0; l < TT_MAX_HEIGHT + 2 && cur >= 0; ++l) {
        const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
        float v[DIM];
        load_row_nc<DIM>(v, vpt + (size_t)cur * dp);
        const float d = __fsqrt_rn(pinned_d2<DIM>(q, v));
        best = fminf(best, d);
        cur = d <= __int_as_float(t.z) ? t.x : t.y;
    }
    return best;
}

template <int DIM>
__device__ __forceinline__ float nn_cost(const tt_nn_rec *rec, const float *vpt, int dp, const float (&q)[DIM]) {
    int cur = 0;
    float best = __int_as_float(0x7f800000);
    for (int l = 0; l < TT_MAX_HEIGHT + 2 && cur >= 0; ++l) {
        const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
        float v[DIM];
        load_row_nc<DIM>(v, vpt + (size_t)cur * dp);
        best = fminf(best, pinned_d2<DIM>(q, v));
        if (t.w < 0) break;
        cur = select_dim<DIM>(q, t.w) < __int_as_float(t.z) ? t.x : t.y;
    }
    return best;
}

// one warp per tile: key = bits of the largest (non-negative) estimate
template <int DIM>
__global__ void tile_cost_kernel(int kind, const void *rec, const float *tpts, const float *vpt, int dp,
                                 const float *pts, int ld, const uint32_t *perm, long long n, int T,
                                 long long ntiles, unsigned *key, unsigned *tile_id) {
    const int lane = threadIdx.x & 31;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long w = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5; w < ntiles; w += nw) {
        float c = 0.f;
        for (int j = lane; j < T; j += 32) {
            const long long pos = w * T + j;
            if (pos >= n) break;
            float q[DIM];
            load_query<DIM>(q, pts, perm[pos], ld);
            const float e = kind == TT_KIND_KD   ? kd_cost<DIM>(static_cast<const tt_kd_rec *>(rec), tpts, dp, q)
                            : kind == TT_KIND_NN ? nn_cost<DIM>(static_cast<const tt_nn_rec *>(rec), vpt, dp, q)
                                                 : vp_cost<DIM>(static_cast<const tt_vp_rec *>(rec), vpt, dp, q);
            c = fmaxf(c, e);
        }
        // non-negative floats order like their bit patterns (+inf included)
        const unsigned m = __reduce_max_sync(TT_FULL, __float_as_uint(c));
        if (lane == 0) {
            key[w] = m;
            tile_id[w] = (unsigned)w;
        }
    }
}

__global__ void gather_tiles_kernel(const uint32_t *in, uint32_t *out, const unsigned *order, long long nfull,
                                    int T, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const long long t = i / T;
        out[i] = t < nfull ? in[(long long)order[t] * T + (i - t * T)] : in[i];
    }
}

template <int DIM>
void launch_cost(const tt_tree *t, const float *pts, int ld, const uint32_t *perm, long long n, int T,
                 long long nfull, unsigned *key, unsigned *ids, cudaStream_t s) {
    const long long g = (nfull * 32 + 255) / 256;
    const int grid = (int)(g < 1 ? 1 : (g > 148 * 16 ? 148 * 16 : g));
    tile_cost_kernel<DIM><<<grid, 256, 0, s>>>(t->hdr.kind, t->dev.rec, t->dev.pts, t->dev.vpt, t->hdr.dp, pts, ld,
                                               perm, n, T, nfull, key, ids);
}

}  // namespace

int tt_launch_schedule(const tt_tree *t, const float *pts, int64_t n, int32_t ld, const uint32_t *perm_in,
                       uint32_t *perm_out, int tile, void *stream) {
    cudaStream_t s = (cudaStream_t)stream;
    tt_keep_pool_memory();
    const long long nfull = n / tile;  // the ragged last tile stays last
    unsigned *key = nullptr, *key_alt = nullptr, *ids = nullptr, *ids_alt = nullptr;
    uint32_t *src = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    cudaError_t e = cudaSuccess;
#define TT_CK(x)                         \
    do {                                 \
        e = (x);                         \
        if (e != cudaSuccess) goto done; \
    } while (0)
    if (nfull < 2 || t->hdr.kind == TT_KIND_OCT) {  // nothing to reorder / no estimate
        if (perm_out != perm_in)
            TT_CK(cudaMemcpyAsync(perm_out, perm_in, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s));
        goto done;
    }
    TT_CK(cudaMallocAsync((void **)&key, sizeof(unsigned) * nfull, s));
    TT_CK(cudaMallocAsync((void **)&key_alt, sizeof(unsigned) * nfull, s));
    TT_CK(cudaMallocAsync((void **)&ids, sizeof(unsigned) * nfull, s));
    TT_CK(cudaMallocAsync((void **)&ids_alt, sizeof(unsigned) * nfull, s));
    switch (t->hdr.dim) {
    case 1: launch_cost<1>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 2: launch_cost<2>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 3: launch_cost<3>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 4: launch_cost<4>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 5: launch_cost<5>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 6: launch_cost<6>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 7: launch_cost<7>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 8: launch_cost<8>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    case 16: launch_cost<16>(t, pts, ld, perm_in, n, tile, nfull, key, ids, s); break;
    default: e = cudaErrorInvalidValue; goto done;
    }
    TT_CK(cudaGetLastError());
    // stable descending sort: equal estimates keep the point-sort order
    TT_CK(cub::DeviceRadixSort::SortPairsDescending(nullptr, tmp_bytes, key, key_alt, ids, ids_alt, (int)nfull, 0, 32,
                                                    s));
    TT_CK(cudaMallocAsync(&tmp, tmp_bytes, s));
    TT_CK(cub::DeviceRadixSort::SortPairsDescending(tmp, tmp_bytes, key, key_alt, ids, ids_alt, (int)nfull, 0, 32, s));
    if (perm_out == perm_in) {
        TT_CK(cudaMallocAsync((void **)&src, sizeof(uint32_t) * n, s));
        TT_CK(cudaMemcpyAsync(src, perm_in, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s));
    }
    gather_tiles_kernel<<<grid_for(n), 256, 0, s>>>(src ? src : perm_in, perm_out, ids_alt, nfull, tile, n);
    TT_CK(cudaGetLastError());
done:
    if (src) cudaFreeAsync(src, s);
    if (tmp) cudaFreeAsync(tmp, s);
    if (ids_alt) cudaFreeAsync(ids_alt, s);
    if (ids) cudaFreeAsync(ids, s);
    if (key_alt) cudaFreeAsync(key_alt, s);
    if (key) cudaFreeAsync(key, s);
#undef TT_CK
    return (int)e;
}
