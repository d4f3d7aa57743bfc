// build_common.cuh -- helpers shared by the GPU tree builders
// (build_{oct,kd,vp}_gpu.cu): stream-ordered scratch, grid sizing, and the
// top-levels-first renumbering of pack.cpp (nodes of the top levels first,
// level by level in preorder, then the rest in preorder).
#pragma once

#include <cub/device/device_scan.cuh>

#include <cstring>
#include <vector>

#include "kern_common.cuh"
#include "blob_cache.h"

namespace {

inline unsigned build_grid(long long n) {
    long long g = (n + 255) / 256;
    if (g > 148 * 8) g = 148 * 8;
    return (unsigned)(g < 1 ? 1 : g);
}

inline uint64_t align256(uint64_t x) { return (x + 255) & ~uint64_t(255); }

// Stream-ordered scratch allocations, released (stream-ordered) at scope exit.
struct Scratch {
    cudaStream_t s;
    cudaError_t e = cudaSuccess;
    std::vector<void *> ptrs;
    template <class T>
    T *get(size_t count) {
        void *p = nullptr;
        if (e == cudaSuccess) e = cudaMallocAsync(&p, count * sizeof(T) + 16, s);
        if (e == cudaSuccess) ptrs.push_back(p);
        return static_cast<T *>(p);
    }
    ~Scratch() {
        for (void *p : ptrs) cudaFreeAsync(p, s);
    }
};

__global__ void level_hist_kernel(const int *level, long long nn, unsigned *hist) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x)
        atomicAdd(hist + level[v], 1u);
}
// flag[v] = node v on level l (l >= 0) / outside the top region (l < 0)
__global__ void level_flag_kernel(const int *level, long long nn, int top_levels, int l, int *flag) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x)
        flag[v] = l < 0 ? (level[v] >= top_levels) : (level[v] == l);
}
__global__ void level_assign_kernel(const int *level, const int *rank, long long nn, int top_levels, int l, int offset,
                                    int *newidx) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x)
        if (l < 0 ? level[v] >= top_levels : level[v] == l) newidx[v] = offset + rank[v];
}

// Fill h.height / top_levels / top_count / level_prefix from the node levels
// (same plan as pack.cpp for `stage_bytes` per staged node) and compute the
// device index newidx[v] of every canonical (preorder) node v.
// known_hist (nullable): the level histogram, already on the host (no sync).
inline cudaError_t renumber_top_first(const int *level, long long nn, int stage_bytes, tt_blob_header &h,
                                      int *newidx, Scratch &W, const unsigned *known_hist = nullptr) {
    cudaStream_t s = W.s;
    const unsigned GN = build_grid(nn);
    int *flag = W.get<int>(nn + 1), *rank = W.get<int>(nn + 1);
    size_t sb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, sb, flag, rank, (int)nn, s);
    void *st = W.get<unsigned char>(sb);
    if (W.e) return W.e;
    cudaError_t e;
    unsigned hh[64];
    if (known_hist) {
        std::memcpy(hh, known_hist, sizeof(hh));
    } else {
        unsigned *hist = W.get<unsigned>(64);
        if (W.e) return W.e;
        if ((e = cudaMemsetAsync(hist, 0, 64 * sizeof(unsigned), s))) return e;
        level_hist_kernel<<<GN, 256, 0, s>>>(level, nn, hist);
        if ((e = cudaMemcpyAsync(hh, hist, sizeof(hh), cudaMemcpyDeviceToHost, s))) return e;
        if ((e = cudaStreamSynchronize(s))) return e;
    }
    int height = 0;
    for (int l = 0; l < 64; ++l)
        if (hh[l]) height = l;
    h.height = height;
    long long acc = 0;
    int L = 0;
    h.level_prefix[0] = 0;
    while (L <= height && L < TT_TOP_LEVELS_MAX && (acc + (long long)hh[L]) * stage_bytes <= TT_TOP_BYTES) {
        acc += hh[L];
        ++L;
        h.level_prefix[L] = (int32_t)acc;
    }
    h.top_levels = L;
    h.top_count = (int32_t)acc;
    for (int l = -1; l < h.top_levels; ++l) {
        level_flag_kernel<<<GN, 256, 0, s>>>(level, nn, h.top_levels, l, flag);
        size_t q = sb;
        if ((e = cub::DeviceScan::ExclusiveSum(st, q, flag, rank, (int)nn, s))) return e;
        level_assign_kernel<<<GN, 256, 0, s>>>(level, rank, nn, h.top_levels, l,
                                               l < 0 ? h.top_count : h.level_prefix[l], newidx);
    }
    return cudaGetLastError();
}

inline void header_base(tt_blob_header &h, int kind, int dim, int leaf, long long n_nodes, long long n_points) {
    std::memset(&h, 0, sizeof(h));
    h.magic = TT_BLOB_MAGIC;
    h.version = TT_BLOB_VERSION;
    h.kind = kind;
    h.dim = dim;
    h.dp = (dim + 3) & ~3;
    h.leaf_size = leaf;
    h.n_nodes = n_nodes;
    h.n_points = n_points;
}

// cudaMalloc the blob, zero it, write the header
inline cudaError_t alloc_blob(const tt_blob_header &h, cudaStream_t s, void **blob) {
    // recycled from freed device-built trees when one fits (tt_api.cu):
    // time stepping builds a tree every step
    cudaError_t e = (cudaError_t)tt_blob_take((size_t)h.total, blob);
    if (e) return e;
    if ((e = cudaMemsetAsync(*blob, 0, h.total, s)) ||
        (e = cudaMemcpyAsync(*blob, &h, sizeof(h), cudaMemcpyHostToDevice, s))) {
        tt_blob_discard(*blob);
        *blob = nullptr;
    }
    return e;
}

}  // namespace
