// kern_sort.cu -- point sorting for traversal similarity (§4.4).
//
// Key = where the point's descent of the tree by the build's split rule ends,
// in tree (preorder) order, so that points whose traversals start alike sit in
// the same warp:
//   kd : leaf reached by "left iff x[dim] < split" -> its first tree-order
//        point index (leaves are numbered in preorder);
//   oct: the point's 16-level cell of the cube hierarchy (octant bits from
//        fp64 comparisons exactly as the build partitions bodies), ordered
//        along the 3-D Hilbert curve (48-bit key, reading R18b);
//   vp : 2-bit-per-level code (inside = 01, outside = 10, end = 00) of the
//        inside-iff-d<=r_in_max descent; a node sorts before its subtree;
//   nn : the same code (left = 01, right = 10) of the left-iff-x[dim]<split
//        descent of the point-per-node kd-tree.
// A stable LSD radix sort of (key, index) then yields perm (ties by index).
// The key kernel is ours; the radix sort is CUB's DeviceRadixSort (a library
// sort primitive, like a library GEMM).
#include <cub/device/device_radix_sort.cuh>

#include "kern_common.cuh"

namespace {

using namespace tt;

__global__ void iota_kernel(uint32_t *v, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        v[i] = (uint32_t)i;
}

// Levels of the oct sort key (reading R18b): cells of side root/2^16 -- for
// the 1M / 16M Plummer configs fewer than 0.01 bodies per cell even in the
// core, so the ties left to the index order are immaterial -- and a 48-bit
// key: 6 radix passes instead of 8.
constexpr int kOctKeyLevels = 16;

// spread the low 16 bits of v to every third bit (bit b -> bit 3b)
__device__ __forceinline__ unsigned long long spread3(unsigned v) {
    unsigned long long x = v & 0xffffull;
    x = (x | (x << 16)) & 0x0000ff0000ffull;
    x = (x | (x << 8)) & 0x00f00f00f00full;
    x = (x | (x << 4)) & 0x0c30c30c30c3ull;
    x = (x | (x << 2)) & 0x249249249249ull;
    return x;
}

// Hilbert index (Skilling's transpose algorithm) of the kOctKeyLevels-level
// cell whose coordinate bits are (ix, iy, iz), bits interleaved x, y, z from
// the top.  Branch-free and unrolled (the per-bit exchange as selects: lanes
// of a warp take different branches), the interleave by bit spreading.
__device__ __forceinline__ unsigned long long hilbert_key(unsigned ix, unsigned iy, unsigned iz) {
    unsigned X[3] = {ix, iy, iz};
#pragma unroll
    for (unsigned Q = 1u << (kOctKeyLevels - 1); Q > 1; Q >>= 1) {
        const unsigned P = Q - 1;
#pragma unroll
        for (int i = 0; i < 3; ++i) {
            // X[i] & Q: invert the low bits of X[0]; else exchange them with X[i]'s
            const bool inv = (X[i] & Q) != 0;
            const unsigned t = (X[0] ^ X[i]) & P;
            if (i == 0) {
                X[0] ^= inv ? P : 0u;  // (t == 0 for i == 0)
            } else {
                X[0] ^= inv ? P : t;
                X[i] ^= inv ? 0u : t;
            }
        }
    }
    X[1] ^= X[0];
    X[2] ^= X[1];
    unsigned t = 0;
#pragma unroll
    for (unsigned Q = 1u << (kOctKeyLevels - 1); Q > 1; Q >>= 1) t ^= (X[2] & Q) ? Q - 1 : 0u;
    X[0] ^= t;
    X[1] ^= t;
    X[2] ^= t;
    return (spread3(X[0]) << 2) | (spread3(X[1]) << 1) | spread3(X[2]);
}

// Oct sort key (reading R18b): the kOctKeyLevels-level cell of the point's descent
// through the cube hierarchy (octant bits from fp64 comparisons, as the
// build), ordered along the Hilbert curve of the root cube.
__global__ void oct_keys(const float *pts, long long n, int ld, double cx, double cy, double cz, double side,
                         unsigned long long *keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const float *p = pts + i * ld;
        const double x = p[0], y = p[1], z = p[2];
        double c0 = cx, c1 = cy, c2 = cz, s = side;
        unsigned ix = 0, iy = 0, iz = 0;
#pragma unroll 1
        for (int l = 0; l < kOctKeyLevels; ++l) {
            const double h = s * 0.25;
            const int o = (x >= c0) | ((y >= c1) << 1) | ((z >= c2) << 2);
            ix = (ix << 1) | (unsigned)(o & 1);
            iy = (iy << 1) | (unsigned)((o >> 1) & 1);
            iz = (iz << 1) | (unsigned)(o >> 2);
            c0 += (o & 1) ? h : -h;
            c1 += (o & 2) ? h : -h;
            c2 += (o & 4) ? h : -h;
            s *= 0.5;
        }
        keys[i] = hilbert_key(ix, iy, iz);
    }
}

template <int DIM>
__global__ void kd_keys(const tt_kd_rec *rec, const float *pts, long long n, int ld, unsigned long long *keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        float q[DIM];
        load_query<DIM>(q, pts, i, ld);
        int cur = 0;
        for (;;) {
            const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
            const int4 u = __ldg(reinterpret_cast<const int4 *>(rec + cur) + 1);
            if (t.x < 0) {
                keys[i] = (unsigned long long)u.z;
                break;
            }
            cur = select_dim<DIM>(q, u.y) < __int_as_float(u.x) ? t.x : t.y;
        }
    }
}

template <int DIM>
__global__ void vp_keys(const tt_vp_rec *rec, const float *vpt, int dp, const float *pts, long long n, int ld,
                        unsigned long long *keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        float q[DIM];
        load_query<DIM>(q, pts, i, ld);
        int cur = 0;
        unsigned long long code = 0;
        for (int l = 0; l < 31; ++l) {
            const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
            float v[DIM];
            load_row_nc<DIM>(v, vpt + (size_t)cur * dp);
            const float d = __fsqrt_rn(pinned_d2<DIM>(q, v));
            const bool inside = d <= __int_as_float(t.z);
            const int nx = inside ? t.x : t.y;
            if (nx < 0) break;
            code |= (unsigned long long)(inside ? 1 : 2) << (62 - 2 * l);
            cur = nx;
        }
        keys[i] = code;
    }
}

template <int DIM>
__global__ void nn_keys(const tt_nn_rec *rec, const float *pts, long long n, int ld, unsigned long long *keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        float q[DIM];
        load_query<DIM>(q, pts, i, ld);
        int cur = 0;
        unsigned long long code = 0;
        for (int l = 0; l < 31; ++l) {
            const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + cur));
            if (t.w < 0) break;
            const bool left = select_dim<DIM>(q, t.w) < __int_as_float(t.z);
            const int nx = left ? t.x : t.y;
            if (nx < 0) break;
            code |= (unsigned long long)(left ? 1 : 2) << (62 - 2 * l);
            cur = nx;
        }
        keys[i] = code;
    }
}

int grid_for(long long n) {
    long long g = (n + 255) / 256;
    if (g > 148 * 16) g = 148 * 16;
    return (int)(g < 1 ? 1 : g);
}

template <int DIM>
void launch_keys(const tt_tree *t, const float *pts, long long n, int ld, unsigned long long *keys,
                 cudaStream_t s) {
    if (t->hdr.kind == TT_KIND_KD)
        kd_keys<DIM><<<grid_for(n), 256, 0, s>>>(static_cast<const tt_kd_rec *>(t->dev.rec), pts, n, ld, keys);
    else if (t->hdr.kind == TT_KIND_NN)
        nn_keys<DIM><<<grid_for(n), 256, 0, s>>>(static_cast<const tt_nn_rec *>(t->dev.rec), pts, n, ld, keys);
    else
        vp_keys<DIM><<<grid_for(n), 256, 0, s>>>(static_cast<const tt_vp_rec *>(t->dev.rec), t->dev.vpt, t->hdr.dp,
                                                pts, n, ld, keys);
}

}  // namespace

// Keep freed stream-ordered scratch in the device's default pool across
// synchronisations (the default release threshold of 0 returns it to the OS
// at every sync, and the next cudaMallocAsync maps fresh memory: ~ms).
void tt_keep_pool_memory() {
    static int done_dev = -1;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev == done_dev) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    done_dev = dev;
}

int tt_launch_sort(const tt_tree *t, const float *pts, int64_t n, int32_t ld, uint32_t *perm, uint64_t *keys_out,
                   void *stream) {
    cudaStream_t s = (cudaStream_t)stream;
    tt_keep_pool_memory();
    unsigned long long *keys = nullptr, *keys_alt = nullptr;
    uint32_t *vals = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    cudaError_t e;
    int end_bit = 64;
    if (t->hdr.kind == TT_KIND_KD) {
        end_bit = 1;
        while (end_bit < 63 && (1ull << end_bit) <= (unsigned long long)t->hdr.n_points) ++end_bit;
    } else if (t->hdr.kind == TT_KIND_OCT) {
        end_bit = 3 * kOctKeyLevels;
    }
#define TT_CK(x)                         \
    do {                                 \
        e = (x);                         \
        if (e != cudaSuccess) goto done; \
    } while (0)
    TT_CK(cudaMallocAsync((void **)&keys, sizeof(unsigned long long) * n, s));
    TT_CK(cudaMallocAsync((void **)&keys_alt, sizeof(unsigned long long) * n, s));
    TT_CK(cudaMallocAsync((void **)&vals, sizeof(uint32_t) * n, s));
    if (t->hdr.kind == TT_KIND_OCT) {
        oct_keys<<<grid_for(n), 256, 0, s>>>(pts, n, ld, t->hdr.root_center[0], t->hdr.root_center[1],
                                             t->hdr.root_center[2], t->hdr.root_side, keys);
    } else {
        switch (t->hdr.dim) {
        case 1: launch_keys<1>(t, pts, n, ld, keys, s); break;
        case 2: launch_keys<2>(t, pts, n, ld, keys, s); break;
        case 3: launch_keys<3>(t, pts, n, ld, keys, s); break;
        case 4: launch_keys<4>(t, pts, n, ld, keys, s); break;
        case 5: launch_keys<5>(t, pts, n, ld, keys, s); break;
        case 6: launch_keys<6>(t, pts, n, ld, keys, s); break;
        case 7: launch_keys<7>(t, pts, n, ld, keys, s); break;
        case 8: launch_keys<8>(t, pts, n, ld, keys, s); break;
        case 16: launch_keys<16>(t, pts, n, ld, keys, s); break;
        default: e = cudaErrorInvalidValue; goto done;
        }
    }
    TT_CK(cudaGetLastError());
    if (keys_out) TT_CK(cudaMemcpyAsync(keys_out, keys, sizeof(uint64_t) * n, cudaMemcpyDeviceToDevice, s));
    iota_kernel<<<grid_for(n), 256, 0, s>>>(vals, n);
    TT_CK(cudaGetLastError());
    TT_CK(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, keys, keys_alt, vals, perm, (int)n, 0, end_bit, s));
    TT_CK(cudaMallocAsync(&tmp, tmp_bytes, s));
    TT_CK(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, keys, keys_alt, vals, perm, (int)n, 0, end_bit, s));
done:
    if (tmp) cudaFreeAsync(tmp, s);
    if (vals) cudaFreeAsync(vals, s);
    if (keys_alt) cudaFreeAsync(keys_alt, s);
    if (keys) cudaFreeAsync(keys, s);
#undef TT_CK
    return (int)e;
}
