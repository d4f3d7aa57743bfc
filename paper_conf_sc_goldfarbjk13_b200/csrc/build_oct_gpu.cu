// build_oct_gpu.cu -- Barnes-Hut oct-tree construction on the GPU (SURVEY
// NEXT-1): bodies in device memory -> the packed device blob of a0, without a
// host round trip.  It applies exactly the build rules of the host builder
// (R8a/R9) and emits the same bytes as tt_tree_pack of the host
// tree (tested), so the traversal kernels and the oracle parity carry over.
//
//   1. bounding box (fp32 min/max) -> root cube in fp64;
//   2. per body the 32 octant digits of its descent through the cube
//      hierarchy (fp64 comparisons, as the host partition), packed in two
//      words; stable radix sort by (digits, id) = tree order of the leaves;
//   3. d_i = shared leading digits of sorted neighbours.  Body i starts the
//      cells at levels d_{i-1}+1 .. min(d_i, 32) and its leaf at level
//      max(d_{i-1}, d_i) + 1 (level 33 = child of a depth-32 bucket, R9);
//      numbering the nodes by (first body, level) IS the preorder of Fig.2;
//   4. a cell's rope = first node of the first body past its run (binary
//      search over the sorted digits);
//   5. mass / first moment bottom-up level by level, children in octant
//      order, fp64, rounded once (R8a);
//   6. top-levels-first renumbering and 32-byte records (pack.cpp layout).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <cfloat>
#include <cmath>
#include <cstring>
#include <vector>

#include "build_common.cuh"

namespace {

constexpr int kMaxDepth = 32;  // R9
constexpr int kDigits = 32;    // digits 0..31 decide levels 1..32

__global__ void bbox_kernel(const float4 *b, long long n, float *out /*[6]: lo xyz, hi xyz*/) {
    float lo[3] = {INFINITY, INFINITY, INFINITY}, hi[3] = {-INFINITY, -INFINITY, -INFINITY};
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const float4 p = b[i];
        lo[0] = fminf(lo[0], p.x); lo[1] = fminf(lo[1], p.y); lo[2] = fminf(lo[2], p.z);
        hi[0] = fmaxf(hi[0], p.x); hi[1] = fmaxf(hi[1], p.y); hi[2] = fmaxf(hi[2], p.z);
    }
    for (int d = 0; d < 3; ++d) {
        for (int o = 16; o; o >>= 1) {
            lo[d] = fminf(lo[d], __shfl_xor_sync(TT_FULL, lo[d], o));
            hi[d] = fmaxf(hi[d], __shfl_xor_sync(TT_FULL, hi[d], o));
        }
    }
    if ((threadIdx.x & 31) == 0) {
        // float min/max via ordered-int atomics (values are finite)
        for (int d = 0; d < 3; ++d) {
            int l = __float_as_int(lo[d]), h = __float_as_int(hi[d]);
            int *ol = reinterpret_cast<int *>(out) + d, *oh = reinterpret_cast<int *>(out) + 3 + d;
            if (l >= 0) atomicMin(ol, l);
            else atomicMax(reinterpret_cast<unsigned *>(ol), (unsigned)l);
            if (h >= 0) atomicMax(oh, h);
            else atomicMin(reinterpret_cast<unsigned *>(oh), (unsigned)h);
        }
    }
}

struct Cube {
    double c[3], side;
};

// What the host needs from the device, read back with ONE synchronisation:
// the root cube (header), the node count (allocation sizes) and the level
// histogram (top-levels-first plan).
struct BuildInfo {
    Cube cube;
    int n_nodes, pad;
    unsigned hist[64];
};

__global__ void box_init_kernel(float *box) {
    if (threadIdx.x < 6) box[threadIdx.x] = threadIdx.x < 3 ? INFINITY : -INFINITY;
}

// root cube from the fp32 bounding box, in fp64 (R8a): centre = midpoint,
// side = max extent (1 for a single point)
__global__ void cube_kernel(const float *box, BuildInfo *info) {
    if (threadIdx.x == 0) {
        double side = 0.0;
        for (int d = 0; d < 3; ++d) {
            info->cube.c[d] = ((double)box[d] + (double)box[3 + d]) * 0.5;
            side = fmax(side, (double)box[3 + d] - (double)box[d]);
        }
        info->cube.side = side == 0.0 ? 1.0 : side;
    }
}

__global__ void digits_kernel(const float4 *b, long long n, const BuildInfo *info, unsigned long long *k0,
                              unsigned long long *k1, unsigned *ids) {
    const Cube cube = info->cube;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const float4 p = b[i];
        const double x = p.x, y = p.y, z = p.z;
        double c0 = cube.c[0], c1 = cube.c[1], c2 = cube.c[2], s = cube.side;
        unsigned long long a = 0, bb = 0;
#pragma unroll 1
        for (int l = 0; l < kDigits; ++l) {
            const double h = s * 0.25;
            const int o = (x >= c0) | ((y >= c1) << 1) | ((z >= c2) << 2);
            if (l < 21) a = (a << 3) | (unsigned)o;
            else bb = (bb << 3) | (unsigned)o;
            c0 += (o & 1) ? h : -h;
            c1 += (o & 2) ? h : -h;
            c2 += (o & 4) ? h : -h;
            s *= 0.5;
        }
        k0[i] = a;   // digits 0..20 in bits 62..0
        k1[i] = bb;  // digits 21..31 in bits 32..0
        ids[i] = (unsigned)i;
    }
}

// shared leading digits of two digit strings (0..32)
__device__ __forceinline__ int common_digits(unsigned long long a0, unsigned long long a1, unsigned long long b0,
                                             unsigned long long b1) {
    const unsigned long long x = a0 ^ b0;
    if (x) return (__clzll((long long)x) - 1) / 3;
    const unsigned long long y = a1 ^ b1;
    if (y) return 21 + (__clzll((long long)y) - 31) / 3;
    return kDigits;
}

// d[i] = common digits of sorted bodies i and i+1 (-1 for the last); cnt[i] =
// nodes started by body i.
// ... and the level histogram of the nodes emit_kernel will write (cells at
// levels dprev+1 .. min(dnext, 32), the leaf at max(dprev, dnext) + 1)
__global__ void count_kernel(const unsigned long long *k0, const unsigned long long *k1, long long n, int *dn,
                             int *cnt, unsigned *hist) {
    __shared__ unsigned sh[64];
    if (threadIdx.x < 64) sh[threadIdx.x] = 0;
    __syncthreads();
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int dprev = i > 0 ? common_digits(k0[i - 1], k1[i - 1], k0[i], k1[i]) : -1;
        const int dnext = i + 1 < n ? common_digits(k0[i], k1[i], k0[i + 1], k1[i + 1]) : -1;
        dn[i] = dnext;
        const int top = min(dnext, kMaxDepth);
        const int cells = max(0, top - dprev);
        cnt[i] = cells + 1;
        for (int L = dprev + 1; L <= top; ++L) atomicAdd(sh + L, 1u);
        atomicAdd(sh + min(max(dprev, dnext) + 1, kMaxDepth + 1), 1u);
    }
    __syncthreads();
    if (threadIdx.x < 64 && sh[threadIdx.x]) atomicAdd(hist + threadIdx.x, sh[threadIdx.x]);
}

__global__ void info_count_kernel(const int *base, long long n, BuildInfo *info) {
    if (threadIdx.x == 0) info->n_nodes = base[n];
}

struct NodeArrays {
    int *level, *first_body, *skip, *body;  // canonical preorder
    double *m0, *m1;                          // [n_nodes], [n_nodes*3]
};

// emit the nodes of body i: cells (i, L) for L = dprev+1 .. min(dnext, 32), leaf last
__global__ void emit_kernel(const unsigned long long *k0, const unsigned long long *k1, const unsigned *ids,
                            const int *dn, const int *base, long long n, long long n_nodes, NodeArrays A) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int dprev = i > 0 ? dn[i - 1] : -1;
        const int dnext = dn[i];
        const int b = base[i];
        const int cells = max(0, min(dnext, kMaxDepth) - dprev);
        for (int c = 0; c < cells; ++c) {
            const int L = dprev + 1 + c;
            // run end: first j > i whose shared digits with i are < L
            long long lo = i + 1, hi = n;
            while (lo < hi) {
                const long long mid = (lo + hi) >> 1;
                const int cd = common_digits(k0[i], k1[i], k0[mid], k1[mid]);
                if (cd >= L) lo = mid + 1;
                else hi = mid;
            }
            const int v = b + c;
            A.level[v] = L;
            A.first_body[v] = (int)i;
            A.skip[v] = lo < n ? base[lo] : (int)n_nodes;
            A.body[v] = -1;
        }
        const int v = b + cells;
        A.level[v] = max(dprev, dnext) + 1;
        A.first_body[v] = (int)i;
        A.skip[v] = i + 1 < n ? base[i + 1] : (int)n_nodes;
        A.body[v] = (int)ids[i];
    }
}

// moments of the nodes at `lvl`: leaves from their body, cells from their
// children (first child = v + 1, siblings along the ropes), in octant order
__global__ void moments_kernel(const float4 *bodies, long long n_nodes, int lvl, NodeArrays A) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n_nodes;
         v += (long long)gridDim.x * blockDim.x) {
        if (A.level[v] != lvl) continue;
        if (A.body[v] >= 0) {
            const float4 p = bodies[A.body[v]];
            A.m0[v] = (double)p.w;
            A.m1[3 * v + 0] = (double)p.w * (double)p.x;
            A.m1[3 * v + 1] = (double)p.w * (double)p.y;
            A.m1[3 * v + 2] = (double)p.w * (double)p.z;
            continue;
        }
        double m0 = 0.0, x = 0.0, y = 0.0, z = 0.0;
        for (long long c = v + 1; c != A.skip[v]; c = A.skip[c]) {
            m0 += A.m0[c];
            x += A.m1[3 * c + 0];
            y += A.m1[3 * c + 1];
            z += A.m1[3 * c + 2];
        }
        A.m0[v] = m0;
        A.m1[3 * v + 0] = x;
        A.m1[3 * v + 1] = y;
        A.m1[3 * v + 2] = z;
    }
}

__global__ void records_kernel(long long n_nodes, NodeArrays A, const int *newidx, tt_oct_rec *rec) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n_nodes;
         v += (long long)gridDim.x * blockDim.x) {
        tt_oct_rec r;
        const double m0 = A.m0[v];
        r.gx = (float)(m0 != 0.0 ? A.m1[3 * v + 0] / m0 : 0.0);
        r.gy = (float)(m0 != 0.0 ? A.m1[3 * v + 1] / m0 : 0.0);
        r.gz = (float)(m0 != 0.0 ? A.m1[3 * v + 2] / m0 : 0.0);
        r.gm = (float)m0;
        r.first_child = A.body[v] >= 0 ? TT_END : newidx[v + 1];
        r.skip = A.skip[v] < n_nodes ? newidx[A.skip[v]] : TT_END;
        r.body = A.body[v];
        r.level = A.level[v];
        rec[newidx[v]] = r;
    }
}

// leaves copy the body's fp32 position and mass verbatim (as the host does)
__global__ void leaf_fix_kernel(const float4 *bodies, long long n_nodes, NodeArrays A, const int *newidx,
                                tt_oct_rec *rec) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n_nodes;
         v += (long long)gridDim.x * blockDim.x) {
        if (A.body[v] < 0) continue;
        const float4 p = bodies[A.body[v]];
        tt_oct_rec &r = rec[newidx[v]];
        r.gx = p.x;
        r.gy = p.y;
        r.gz = p.z;
        r.gm = p.w;
    }
}

__global__ void gather_u64(const unsigned long long *src, const unsigned *perm, long long n, unsigned long long *dst) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        dst[i] = src[perm[i]];
}

}  // namespace

// Build on `stream`: writes the host copy of the blob header and a cudaMalloc'd
// device blob (caller owns it).  Synchronises the stream twice: once to read
// the root cube, node count and level histogram (one struct), once at the
// end.  order_out (nullable, device [n]): the bodies' tree order (leaf
// preorder), i.e. the sorted ids of step 2.
int tt_build_oct_gpu_impl(const float *bodies_f, long long n, void *stream, tt_blob_header *hdr_out,
                          void **blob_out, unsigned *order_out) {
    cudaStream_t s = (cudaStream_t)stream;
    const float4 *bodies = reinterpret_cast<const float4 *>(bodies_f);
    tt_keep_pool_memory();
    Scratch W{s};
    const unsigned G = build_grid(n);

    // 1. root cube (on the device)
    float *d_box = W.get<float>(6);
    BuildInfo *d_info = W.get<BuildInfo>(1);
    if (W.e) return W.e;
    cudaError_t e = cudaMemsetAsync(d_info, 0, sizeof(BuildInfo), s);
    if (e) return e;
    box_init_kernel<<<1, 32, 0, s>>>(d_box);
    bbox_kernel<<<G, 256, 0, s>>>(bodies, n, d_box);
    cube_kernel<<<1, 32, 0, s>>>(d_box, d_info);

    // 2. digits + stable sort by (digits, id)
    auto *k0 = W.get<unsigned long long>(n), *k1 = W.get<unsigned long long>(n);
    auto *kt = W.get<unsigned long long>(n), *kt2 = W.get<unsigned long long>(n);
    auto *ids = W.get<unsigned>(n), *ids_t = W.get<unsigned>(n), *ids_s = W.get<unsigned>(n);
    if (W.e) return W.e;
    digits_kernel<<<G, 256, 0, s>>>(bodies, n, d_info, k0, k1, ids);
    size_t b1 = 0, b2 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, b1, k1, kt, ids, ids_t, (int)n, 0, 33, s);
    cub::DeviceRadixSort::SortPairs(nullptr, b2, kt, kt2, ids_t, ids_s, (int)n, 0, 63, s);
    void *ct = W.get<unsigned char>(std::max(b1, b2));
    if (W.e) return W.e;
    size_t cb = std::max(b1, b2);
    if ((e = cub::DeviceRadixSort::SortPairs(ct, cb, k1, kt, ids, ids_t, (int)n, 0, 33, s))) return e;
    gather_u64<<<G, 256, 0, s>>>(k0, ids_t, n, kt);  // k0 in k1-sorted order
    cb = std::max(b1, b2);
    if ((e = cub::DeviceRadixSort::SortPairs(ct, cb, kt, kt2, ids_t, ids_s, (int)n, 0, 63, s))) return e;
    auto *k0s = W.get<unsigned long long>(n), *k1s = W.get<unsigned long long>(n);
    if (W.e) return W.e;
    gather_u64<<<G, 256, 0, s>>>(k0, ids_s, n, k0s);
    gather_u64<<<G, 256, 0, s>>>(k1, ids_s, n, k1s);
    if (order_out && (e = cudaMemcpyAsync(order_out, ids_s, sizeof(unsigned) * (size_t)n, cudaMemcpyDeviceToDevice, s)))
        return e;

    // 3. node counts per body (and the level histogram), preorder bases
    int *dn = W.get<int>(n), *cnt = W.get<int>(n + 1), *base = W.get<int>(n + 1);
    if (W.e) return W.e;
    count_kernel<<<G, 256, 0, s>>>(k0s, k1s, n, dn, cnt, d_info->hist);
    if ((e = cudaMemsetAsync(cnt + n, 0, sizeof(int), s))) return e;
    size_t sb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, sb, cnt, base, (int)(n + 1), s);
    void *st = W.get<unsigned char>(sb);
    if (W.e) return W.e;
    if ((e = cub::DeviceScan::ExclusiveSum(st, sb, cnt, base, (int)(n + 1), s))) return e;
    info_count_kernel<<<1, 32, 0, s>>>(base, n, d_info);
    BuildInfo info;
    if ((e = cudaMemcpyAsync(&info, d_info, sizeof(info), cudaMemcpyDeviceToHost, s))) return e;
    if ((e = cudaStreamSynchronize(s))) return e;
    const long long n_nodes = info.n_nodes;
    const Cube cube = info.cube;
    int height = 0;
    for (int l = 0; l < 64; ++l)
        if (info.hist[l]) height = l;

    // 4. nodes in preorder
    NodeArrays A;
    A.level = W.get<int>(n_nodes);
    A.first_body = W.get<int>(n_nodes);
    A.skip = W.get<int>(n_nodes);
    A.body = W.get<int>(n_nodes);
    A.m0 = W.get<double>(n_nodes);
    A.m1 = W.get<double>(3 * n_nodes);
    if (W.e) return W.e;
    const unsigned GN = build_grid(n_nodes);
    emit_kernel<<<G, 256, 0, s>>>(k0s, k1s, ids_s, dn, base, n, n_nodes, A);

    // 5. moments bottom-up
    for (int l = height; l >= 0; --l) moments_kernel<<<GN, 256, 0, s>>>(bodies, n_nodes, l, A);

    // 6. header (same plan as pack.cpp), renumbering, records
    tt_blob_header h;
    header_base(h, TT_KIND_OCT, 3, 1, n_nodes, n);
    for (int d = 0; d < 3; ++d) h.root_center[d] = cube.c[d];
    h.root_side = cube.side;
    h.rec_bytes = 32;
    // R9 trees: more than 8 children only in depth-32 buckets (height 33),
    // whose children are leaves (same bits as pack.cpp computes)
    h.oct_flags = (height <= 32 ? TT_OCT_NARROW : 0) | TT_OCT_FEW_CELL_KIDS;
    int *newidx = W.get<int>(n_nodes);
    if (W.e) return W.e;
    if ((e = renumber_top_first(A.level, n_nodes, 32, h, newidx, W, info.hist))) return e;
    h.off_rec = align256(sizeof(tt_blob_header));
    h.total = align256(h.off_rec + (uint64_t)n_nodes * 32);
    void *blob = nullptr;
    if ((e = alloc_blob(h, s, &blob))) return e;
    auto *base_b = static_cast<unsigned char *>(blob);
    auto *rec = reinterpret_cast<tt_oct_rec *>(base_b + h.off_rec);
    records_kernel<<<GN, 256, 0, s>>>(n_nodes, A, newidx, rec);
    leaf_fix_kernel<<<GN, 256, 0, s>>>(bodies, n_nodes, A, newidx, rec);
    if ((e = cudaGetLastError()) || (e = cudaStreamSynchronize(s))) {
        tt_blob_discard(blob);
        return e;
    }
    *hdr_out = h;
    *blob_out = blob;
    return 0;
}
