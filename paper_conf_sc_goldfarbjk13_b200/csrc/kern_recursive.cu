// kern_recursive.cu -- the naive recursive GPU baseline.
//
// The paper compares its autoroped kernels against "a naive GPU
// implementation that uses CUDA compute capability 2.0's support for
// recursion to directly map the recursive algorithm to the GPU ... the only
// difference between the naive implementations and ours is the use of
// autoropes" (Table 1's "Improv. vs Recurse" column).  These
// kernels are that baseline on sm_100a: the point loop is strip-mined over the
// grid (Fig.9b lines 2-3) and every thread calls a literally recursive
// __device__ function over the same packed tree, with the same pinned
// arithmetic -- so results and per-point visit counts are identical to the
// autoroped independent (N) kernels.  Only the non-lockstep variant is built.
// Selected with tt_traverse_opts.variant = TT_VARIANT_RECURSIVE.
#include "kern_common.cuh"

// a negative self id means "no self leaf": -2 matches no record's body field
// (cells carry -1 there)
static __device__ __forceinline__ int tt_self_id(int s) { return s < 0 ? -2 : s; }

namespace {

using namespace tt;

constexpr int kBlock = 128;
#define TT_VP_EPS_R 0x1p-12f

// ------------------------------------------------------------------ BH
struct BhCtx {
    const tt_oct_rec *rec;
    float4 b;
    int self;
    float eps2;
    double ax, ay, az;
    unsigned visits;
    const int32_t *pre;  // stats hashes (nullable)
    VHash vh;
};

__device__ void bh_rec(BhCtx &c, int node, float dsq) {
    ++c.visits;
    if (c.pre) c.vh.add(c.pre, node);
    const float4 g = __ldg(reinterpret_cast<const float4 *>(&c.rec[node].gx));
    const int4 t = __ldg(reinterpret_cast<const int4 *>(&c.rec[node].first_child));
    const float dx = __fsub_rn(g.x, c.b.x), dy = __fsub_rn(g.y, c.b.y), dz = __fsub_rn(g.z, c.b.z);
    const float drsq = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));  // R8
    if (t.x >= 0 && drsq < dsq) {  // !far_enough && type != LEAF (Fig.9a line 2)
        const float cd = __fmul_rn(dsq, 0.25f);
        // children of a cell: first_child, then the rope chain of siblings
        for (int ch = t.x; ch != t.y; ch = __ldg(&c.rec[ch].skip)) bh_rec(c, ch, cd);
        return;
    }
    if (t.z == c.self) return;
    const float inv = rsqrt_ftz(__fadd_rn(drsq, c.eps2));
    const float f = g.w * (inv * inv) * inv;
    c.ax += (double)(f * dx);
    c.ay += (double)(f * dy);
    c.az += (double)(f * dz);
}

__global__ void __launch_bounds__(kBlock) bh_rec_kernel(const tt_bh_params P) {
    const tt_oct_rec *rec = static_cast<const tt_oct_rec *>(P.c.tree.rec);
    for (long long pos = blockIdx.x * (long long)blockDim.x + threadIdx.x; pos < P.c.n;
         pos += (long long)gridDim.x * blockDim.x) {
        const long long pid = P.c.order ? (long long)P.c.order[pos] : pos;
        BhCtx c{rec, __ldg(P.bodies + pid), P.self_ids ? tt_self_id(__ldg(P.self_ids + pid)) : (int)pid, P.eps2, 0, 0, 0, 0,
                P.c.pre, VHash{}};
        bh_rec(c, 0, P.dsq_root);
        P.acc[pid] = make_float4((float)c.ax, (float)c.ay, (float)c.az, 0.f);
        if (P.c.st_visits) P.c.st_visits[pid] = c.visits;
        if (c.pre) c.vh.store(P.c, pid);
    }
}

// ------------------------------------------------------------------ PC
template <int DIM>
struct PcCtx {
    const tt_kd_rec *rec;
    const float *box, *pts;
    int dp;
    float q[DIM];
    float r2;
    unsigned count, visits, ptests;
    const int32_t *pre;
    VHash vh;
};

template <int DIM>
__device__ void pc_rec(PcCtx<DIM> &c, int node) {
    ++c.visits;
    if (c.pre) c.vh.add(c.pre, node);
    float lo[DIM], hi[DIM];
    load_row_nc<DIM>(lo, c.box + (size_t)node * 2 * c.dp);
    load_row_nc<DIM>(hi, c.box + (size_t)node * 2 * c.dp + c.dp);
    if (pinned_boxd2<DIM>(c.q, lo, hi) > c.r2) return;  // !can_correlate (Fig.4 line 2)
    const int4 t = __ldg(reinterpret_cast<const int4 *>(c.rec + node));
    if (t.x < 0) {  // update_correlation
        const int4 u = __ldg(reinterpret_cast<const int4 *>(c.rec + node) + 1);
        c.ptests += (unsigned)u.w;
        if (u.w == 1) {
            ++c.count;
        } else {
            for (int j = u.z; j < u.z + u.w; ++j) {
                float p[DIM];
                load_row_nc<DIM>(p, c.pts + (size_t)j * c.dp);
                c.count += pinned_d2<DIM>(c.q, p) <= c.r2;
            }
        }
        return;
    }
    pc_rec<DIM>(c, t.x);
    pc_rec<DIM>(c, t.y);
}

template <int DIM>
__global__ void __launch_bounds__(kBlock) pc_rec_kernel(const tt_pc_params P) {
    for (long long pos = blockIdx.x * (long long)blockDim.x + threadIdx.x; pos < P.c.n;
         pos += (long long)gridDim.x * blockDim.x) {
        const long long pid = P.c.order ? (long long)P.c.order[pos] : pos;
        PcCtx<DIM> c;
        c.rec = static_cast<const tt_kd_rec *>(P.c.tree.rec);
        c.box = P.c.tree.box;
        c.pts = P.c.tree.pts;
        c.dp = (DIM + 3) & ~3;
        load_query<DIM>(c.q, P.q, pid, P.ld);
        c.r2 = P.r2;
        c.count = c.visits = c.ptests = 0;
        c.pre = P.c.pre;
        c.vh = VHash{};
        pc_rec<DIM>(c, 0);
        P.count[pid] = c.count;
        if (P.c.st_visits) P.c.st_visits[pid] = c.visits;
        if (P.c.st_point_tests) P.c.st_point_tests[pid] = c.ptests;
        if (c.pre) c.vh.store(P.c, pid);
    }
}

// ------------------------------------------------------------------ kNN
template <int DIM, int KT>
struct KnnCtx {
    const tt_kd_rec *rec;
    const float *box, *pts;
    const int32_t *pid;
    int dp;
    float q[DIM];
    float d[KT];
    unsigned i[KT];
    unsigned visits, ptests;
    const int32_t *pre;
    VHash vh;
    __device__ void insert(float dd, unsigned ii) {
        d[KT - 1] = dd;
        i[KT - 1] = ii;
#pragma unroll
        for (int j = KT - 1; j > 0; --j) {
            const bool sw = d[j] < d[j - 1] || (d[j] == d[j - 1] && i[j] < i[j - 1]);
            if (sw) {
                const float td = d[j - 1];
                const unsigned ti = i[j - 1];
                d[j - 1] = d[j];
                i[j - 1] = i[j];
                d[j] = td;
                i[j] = ti;
            }
        }
    }
};

template <int DIM, int KT>
__device__ void knn_rec(KnnCtx<DIM, KT> &c, int node) {
    ++c.visits;
    if (c.pre) c.vh.add(c.pre, node);
    if (c.d[KT - 1] < __int_as_float(0x7f800000)) {  // list full: can_correlate (R5a)
        float lo[DIM], hi[DIM];
        load_row_nc<DIM>(lo, c.box + (size_t)node * 2 * c.dp);
        load_row_nc<DIM>(hi, c.box + (size_t)node * 2 * c.dp + c.dp);
        if (pinned_boxd2<DIM>(c.q, lo, hi) > c.d[KT - 1]) return;
    }
    const int4 t = __ldg(reinterpret_cast<const int4 *>(c.rec + node));
    const int4 u = __ldg(reinterpret_cast<const int4 *>(c.rec + node) + 1);
    if (t.x < 0) {  // update_closest
        c.ptests += (unsigned)u.w;
        for (int j = u.z; j < u.z + u.w; ++j) {
            float p[DIM];
            load_row_nc<DIM>(p, c.pts + (size_t)j * c.dp);
            const float d2 = pinned_d2<DIM>(c.q, p);
            const unsigned id = (unsigned)__ldg(c.pid + j);
            if (d2 < c.d[KT - 1] || (d2 == c.d[KT - 1] && id < c.i[KT - 1])) c.insert(d2, id);
        }
        return;
    }
    if (select_dim<DIM>(c.q, u.y) < __int_as_float(u.x)) {  // closer_to_left (R5)
        knn_rec<DIM, KT>(c, t.x);
        knn_rec<DIM, KT>(c, t.y);
    } else {
        knn_rec<DIM, KT>(c, t.y);
        knn_rec<DIM, KT>(c, t.x);
    }
}

template <int DIM, int KT>
__global__ void __launch_bounds__(kBlock) knn_rec_kernel(const tt_knn_params P) {
    for (long long pos = blockIdx.x * (long long)blockDim.x + threadIdx.x; pos < P.c.n;
         pos += (long long)gridDim.x * blockDim.x) {
        const long long pid = P.c.order ? (long long)P.c.order[pos] : pos;
        KnnCtx<DIM, KT> c;
        c.rec = static_cast<const tt_kd_rec *>(P.c.tree.rec);
        c.box = P.c.tree.box;
        c.pts = P.c.tree.pts;
        c.pid = P.c.tree.pid;
        c.dp = (DIM + 3) & ~3;
        load_query<DIM>(c.q, P.q, pid, P.ld);
#pragma unroll
        for (int j = 0; j < KT; ++j) {
            c.d[j] = j >= KT - P.k ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
            c.i[j] = 0xffffffffu;
        }
        c.visits = c.ptests = 0;
        c.pre = P.c.pre;
        c.vh = VHash{};
        knn_rec<DIM, KT>(c, 0);
        for (int j = KT - P.k; j < KT; ++j) {
            const int slot = j - (KT - P.k);
            P.idx[pid * P.k + slot] = c.i[j] == 0xffffffffu ? -1 : (int)c.i[j];
            P.d2[pid * P.k + slot] = c.d[j];
        }
        if (P.c.st_visits) P.c.st_visits[pid] = c.visits;
        if (P.c.st_point_tests) P.c.st_point_tests[pid] = c.ptests;
        if (c.pre) c.vh.store(P.c, pid);
    }
}

// ------------------------------------------------------------------- VP
template <int DIM>
struct VpCtx {
    const tt_vp_rec *rec;
    const float *vpt;
    const int32_t *pid;
    float q[DIM];
    float best, tau;
    unsigned best_i, visits;
    const int32_t *pre;
    VHash vh;
};

template <int DIM>
__device__ void vp_rec(VpCtx<DIM> &c, int node, float lb, float sc) {
    ++c.visits;
    if (c.pre) c.vh.add(c.pre, node);
    if (__fsub_rn(lb, c.tau) > __fmul_rn(TT_VP_EPS_R, __fadd_rn(sc, c.tau))) return;
    const int4 t = __ldg(reinterpret_cast<const int4 *>(c.rec + node));
    float v[DIM];
    load_row_nc<DIM>(v, c.vpt + (size_t)node * ((DIM + 3) & ~3));
    const float d2 = pinned_d2<DIM>(c.q, v);  // update
    const unsigned id = (unsigned)__ldg(c.pid + node);
    if (d2 < c.best || (d2 == c.best && id < c.best_i)) {
        c.best = d2;
        c.best_i = id;
        c.tau = __fsqrt_rn(d2);
    }
    const float d = __fsqrt_rn(d2);
    const float rin = __int_as_float(t.z), rout = __int_as_float(t.w);
    if (d <= rin) {
        if (t.x >= 0) vp_rec<DIM>(c, t.x, __fsub_rn(d, rin), __fadd_rn(d, rin));
        if (t.y >= 0) vp_rec<DIM>(c, t.y, __fsub_rn(rout, d), __fadd_rn(d, rout));
    } else {
        if (t.y >= 0) vp_rec<DIM>(c, t.y, __fsub_rn(rout, d), __fadd_rn(d, rout));
        if (t.x >= 0) vp_rec<DIM>(c, t.x, __fsub_rn(d, rin), __fadd_rn(d, rin));
    }
}

template <int DIM>
__global__ void __launch_bounds__(kBlock) vp_rec_kernel(const tt_vp_params P) {
    for (long long pos = blockIdx.x * (long long)blockDim.x + threadIdx.x; pos < P.c.n;
         pos += (long long)gridDim.x * blockDim.x) {
        const long long pid = P.c.order ? (long long)P.c.order[pos] : pos;
        VpCtx<DIM> c;
        c.rec = static_cast<const tt_vp_rec *>(P.c.tree.rec);
        c.vpt = P.c.tree.vpt;
        c.pid = P.c.tree.pid;
        load_query<DIM>(c.q, P.q, pid, P.ld);
        c.best = c.tau = __int_as_float(0x7f800000);
        c.best_i = 0xffffffffu;
        c.visits = 0;
        c.pre = P.c.pre;
        c.vh = VHash{};
        vp_rec<DIM>(c, 0, __int_as_float(0xff800000), 0.f);
        P.idx[pid] = c.best_i == 0xffffffffu ? -1 : (int)c.best_i;
        P.d2[pid] = c.best;
        if (P.c.st_visits) P.c.st_visits[pid] = c.visits;
        if (c.pre) c.vh.store(P.c, pid);
    }
}

// --------------------------------------------------------------- launch
int prepare_stack(int height) {
    // every recursion level keeps one frame per thread; size the per-thread
    // stack for the tree height (device-wide limit, raised only)
    size_t cur = 0;
    cudaDeviceGetLimit(&cur, cudaLimitStackSize);
    const size_t want = (size_t)(height + 4) * 512 + 2048;
    if (cur < want) return (int)cudaDeviceSetLimit(cudaLimitStackSize, want);
    return 0;
}

template <class K>
unsigned grid_of(K kern, long long n) {
    int dev = 0, nsm = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, 0);
    long long g = (long long)nsm * (occ > 0 ? occ : 1);
    const long long need = (n + kBlock - 1) / kBlock;
    if (g > need) g = need;
    return (unsigned)(g < 1 ? 1 : g);
}

}  // namespace

int tt_launch_bh_recursive(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    int e = prepare_stack(p.c.height);
    if (e) return e;
    bh_rec_kernel<<<grid_of(bh_rec_kernel, p.c.n), kBlock, 0, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}

template <int DIM>
static int pc_rec_dim(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    pc_rec_kernel<DIM><<<grid_of(pc_rec_kernel<DIM>, p.c.n), kBlock, 0, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}
int tt_launch_pc_recursive(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg) {
    int e = prepare_stack(p.c.height);
    if (e) return e;
    switch (dim) {
    case 2: return pc_rec_dim<2>(p, cfg);
    case 3: return pc_rec_dim<3>(p, cfg);
    case 7: return pc_rec_dim<7>(p, cfg);
    case 16: return pc_rec_dim<16>(p, cfg);
    default: return -1;
    }
}

template <int DIM, int KT>
static int knn_rec_dk(const tt_knn_params &p, const tt_launch_cfg &cfg) {
    knn_rec_kernel<DIM, KT><<<grid_of(knn_rec_kernel<DIM, KT>, p.c.n), kBlock, 0, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}
template <int DIM>
static int knn_rec_dim(const tt_knn_params &p, const tt_launch_cfg &cfg) {
    if (p.k <= 1) return knn_rec_dk<DIM, 1>(p, cfg);
    if (p.k <= 8) return knn_rec_dk<DIM, 8>(p, cfg);
    if (p.k <= 16) return knn_rec_dk<DIM, 16>(p, cfg);
    return knn_rec_dk<DIM, 32>(p, cfg);
}
int tt_launch_knn_recursive(const tt_knn_params &p, int dim, const tt_launch_cfg &cfg) {
    int e = prepare_stack(p.c.height);
    if (e) return e;
    switch (dim) {
    case 2: return knn_rec_dim<2>(p, cfg);
    case 3: return knn_rec_dim<3>(p, cfg);
    case 7: return knn_rec_dim<7>(p, cfg);
    case 16: return knn_rec_dim<16>(p, cfg);
    default: return -1;
    }
}

template <int DIM>
static int vp_rec_dim(const tt_vp_params &p, const tt_launch_cfg &cfg) {
    vp_rec_kernel<DIM><<<grid_of(vp_rec_kernel<DIM>, p.c.n), kBlock, 0, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}
int tt_launch_vp_recursive(const tt_vp_params &p, int dim, const tt_launch_cfg &cfg) {
    int e = prepare_stack(p.c.height);
    if (e) return e;
    switch (dim) {
    case 2: return vp_rec_dim<2>(p, cfg);
    case 3: return vp_rec_dim<3>(p, cfg);
    case 7: return vp_rec_dim<7>(p, cfg);
    case 16: return vp_rec_dim<16>(p, cfg);
    default: return -1;
    }
}
