// kern_stack.cu -- explicit rope-stack variant of the unguided kernels
// (TT_VARIANT_STACK): the paper's own GPU form of BH and PC.
//
// Fig.9b turns the recursion into a loop over an explicit rope
// stack: pop a node, test it, push its children in reverse order so they pop
// in the recursive order.  §5.2 lays the stacks out two ways:
//   * independent: one stack per thread in global memory, interleaved so that
//     adjacent threads at the same depth touch adjacent words ("the threads'
//     stacks are interleaved in memory");
//   * lockstep: one stack per warp in shared memory holding (node, mask) --
//     "use shared memory to maintain the rope stack once per warp"
//     (P:L1015-1023), the Fig.8 form.
// Our packed record has no child array (children are reached by first_child
// and the sibling rope), so an opened cell pushes its first child as
// (child, end = the cell's rope), and popping (c, end) first re-pushes the
// pending sibling (rope(c), end) when rope(c) != end.  That is the same stack
// discipline and visit order as pushing all children in reverse, with stack
// depth <= height + 1 and no extra record loads.
// The method's kernels (kern_bh.cu / kern_pc.cu) need no stack at all for
// unguided walks (skip ropes + per-lane wait levels); this variant exists to
// measure that choice.  Same pinned arithmetic and update rules, so counts
// and per-point visit counts equal the oracle's; BH sums are flushed fp32 ->
// fp64 every 16 pops (as the method's kernel does every 16 steps).
// One point per lane, 32-point warp tiles.  AUTO: BH lockstep, PC independent
// (the defaults measured for the method's kernels).
#include <type_traits>

#include "kern_common.cuh"

// a negative self id means "no self leaf": -2 matches no record's body field
// (cells carry -1 there)
static __device__ __forceinline__ int tt_self_id(int s) { return s < 0 ? -2 : s; }

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kWarps = kBlock / 32;
constexpr int kFlush = 16;

struct WarpEntry {
    int node, end;
    unsigned mask;
};

__device__ __forceinline__ int2 gpop(const int2 *st, int sp, long long stride, long long gtid) {
    return st[(long long)sp * stride + gtid];
}
__device__ __forceinline__ void gpush(int2 *st, int sp, long long stride, long long gtid, int node, int end) {
    st[(long long)sp * stride + gtid] = make_int2(node, end);
}

// ---------------------------------------------------------------------- BH
struct BhLane {
    float4 b;
    int self;
    float ax, ay, az;
    double AX, AY, AZ;
    __device__ __forceinline__ void flush() {
        AX += (double)ax;
        AY += (double)ay;
        AZ += (double)az;
        ax = ay = az = 0.f;
    }
};

// Fig.9a/b: returns true iff the lane opens the cell; otherwise updates.
// s_dsq[L] = dsq_root * 0.25^L ("dsq*0.25" per level, Fig.9a line 4).
__device__ __forceinline__ bool bh_visit(BhLane &L, float4 g, int4 t, const float *s_dsq, float eps2) {
    const float dx = __fsub_rn(g.x, L.b.x), dy = __fsub_rn(g.y, L.b.y), dz = __fsub_rn(g.z, L.b.z);
    const float drsq = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));  // R8
    if (t.x >= 0 && drsq < s_dsq[t.w]) return true;
    if (t.z != L.self) {
        const float inv = rsqrt_ftz(__fadd_rn(drsq, eps2));
        const float f = g.w * (inv * inv) * inv;
        L.ax = fmaf(f, dx, L.ax);
        L.ay = fmaf(f, dy, L.ay);
        L.az = fmaf(f, dz, L.az);
    }
    return false;
}

template <bool STATS>
__global__ void __launch_bounds__(kBlock) bh_stack_kernel(const tt_bh_params P, int2 *gstack, int cap) {
    __shared__ WarpEntry s_stack[kWarps][TT_MAX_HEIGHT + 2];
    __shared__ float s_dsq[64];
    if (threadIdx.x == 0) {
        float d = P.dsq_root;
        for (int l = 0; l < 64; ++l) {
            s_dsq[l] = d;
            d = __fmul_rn(d, 0.25f);
        }
    }
    __syncthreads();
    const tt_oct_rec *rec = static_cast<const tt_oct_rec *>(P.c.tree.rec);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const long long gtid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long n = P.c.n, ntiles = (n + 31) >> 5;
    const bool lock = P.c.mode != TT_MODE_INDEPENDENT;
    WarpEntry *ws = s_stack[warp];
    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        const long long pos = tile * 32 + lane;
        const bool valid = pos < n;
        const long long pid = valid ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
        BhLane L;
        L.b = valid ? __ldg(P.bodies + pid) : make_float4(0.f, 0.f, 0.f, 0.f);
        L.self = valid ? (P.self_ids ? tt_self_id(__ldg(P.self_ids + pid)) : (int)pid) : -2;
        L.ax = L.ay = L.az = 0.f;
        L.AX = L.AY = L.AZ = 0.0;
        unsigned visits = 0, fetches = 0, steps = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        if (lock) {
            // Fig.8 with the stack in shared memory, once per warp; lane 0 owns
            // the stack, the popped entry is broadcast with __shfl_sync
            const unsigned vmask = __ballot_sync(TT_FULL, valid);
            int sp = 0;
            if (lane == 0) ws[0] = WarpEntry{0, TT_END, vmask};
            sp = 1;
            int k = 0;
            while (sp > 0) {
                WarpEntry e;
                if (lane == 0) e = ws[sp - 1];
                e.node = __shfl_sync(TT_FULL, e.node, 0);
                e.end = __shfl_sync(TT_FULL, e.end, 0);
                e.mask = __shfl_sync(TT_FULL, e.mask, 0);
                --sp;
                const float4 g = __ldg(reinterpret_cast<const float4 *>(&rec[e.node].gx));
                const int4 t = __ldg(reinterpret_cast<const int4 *>(&rec[e.node].first_child));
                if (STATS) ++steps;
                // pending sibling first (popped after this node's subtree)
                if (t.y != e.end) {
                    if (lane == 0) ws[sp] = WarpEntry{t.y, e.end, e.mask};
                    ++sp;
                }
                const bool active = (e.mask >> lane) & 1u;
                bool open = false;
                if (active) {
                    if (STATS) {
                        ++visits;
                        if (hashing) vh.add(P.c.pre, e.node);
                    }
                    open = bh_visit(L, g, t, s_dsq, P.eps2);
                    if (++k == kFlush) {  // per lane, after each kFlush own visits (as N)
                        L.flush();
                        k = 0;
                    }
                }
                const unsigned cmask = __ballot_sync(TT_FULL, open);
                if (cmask) {
                    if (lane == 0) ws[sp] = WarpEntry{t.x, t.y, cmask};
                    ++sp;
                }
                __syncwarp();
            }
            fetches = steps;
        } else {
            // one stack per thread, interleaved in global memory
            int sp = 0, k = 0;
            if (valid) {
                gpush(gstack, 0, stride, gtid, 0, TT_END);
                sp = 1;
            }
            while (sp > 0) {
                const int2 e = gpop(gstack, --sp, stride, gtid);
                const float4 g = __ldg(reinterpret_cast<const float4 *>(&rec[e.x].gx));
                const int4 t = __ldg(reinterpret_cast<const int4 *>(&rec[e.x].first_child));
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, e.x);
                }
                if (t.y != e.y) gpush(gstack, sp++, stride, gtid, t.y, e.y);
                if (bh_visit(L, g, t, s_dsq, P.eps2)) gpush(gstack, sp++, stride, gtid, t.x, t.y);
                if (++k == kFlush) {
                    L.flush();
                    k = 0;
                }
            }
            if (STATS) {
                fetches = warp_sum(visits);
                steps = __reduce_max_sync(TT_FULL, visits);
            }
        }
        L.flush();
        if (valid) {
            P.acc[pid] = make_float4((float)L.AX, (float)L.AY, (float)L.AZ, 0.f);
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
            if (hashing) vh.store(P.c, pid);
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
    }
    (void)cap;
    cta_finish(P.c.counter);
}

// ---------------------------------------------------------------------- PC
// Fig.4: truncate iff the node's tight box is farther than r; a leaf updates.
// Returns true iff the lane descends into the node's children.
template <int DIM>
__device__ __forceinline__ bool pc_visit(const tt_pc_params &P, const tt_kd_rec *rec, int node, int4 t, int dp,
                                         const float (&q)[DIM], unsigned &count, unsigned &ptests) {
    float lo[DIM], hi[DIM];
    load_row_nc<DIM>(lo, P.c.tree.box + (size_t)node * 2 * dp);
    load_row_nc<DIM>(hi, P.c.tree.box + (size_t)node * 2 * dp + dp);
    if (pinned_boxd2<DIM>(q, lo, hi) > P.r2) return false;  // !can_correlate
    if (t.x >= 0) return true;
    const int4 u = __ldg(reinterpret_cast<const int4 *>(rec + node) + 1);
    ptests += (unsigned)u.w;
    for (int j = u.z; j < u.z + u.w; ++j) {  // update_correlation over the bucket
        float p[DIM];
        load_row_nc<DIM>(p, P.c.tree.pts + (size_t)j * dp);
        count += pinned_d2<DIM>(q, p) <= P.r2;
    }
    return false;
}

template <int DIM, bool STATS>
__global__ void __launch_bounds__(kBlock) pc_stack_kernel(const tt_pc_params P, int2 *gstack, int cap) {
    constexpr int DP = (DIM + 3) & ~3;
    __shared__ WarpEntry s_stack[kWarps][TT_MAX_HEIGHT + 2];
    const tt_kd_rec *rec = static_cast<const tt_kd_rec *>(P.c.tree.rec);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const long long gtid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long n = P.c.n, ntiles = (n + 31) >> 5;
    const bool lock = P.c.mode == TT_MODE_LOCKSTEP;
    WarpEntry *ws = s_stack[warp];
    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        const long long pos = tile * 32 + lane;
        const bool valid = pos < n;
        const long long pid = valid ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
        float q[DIM];
        if (valid) load_query<DIM>(q, P.q, pid, P.ld);
        else
#pragma unroll
            for (int d = 0; d < DIM; ++d) q[d] = 0.f;
        unsigned count = 0, visits = 0, fetches = 0, steps = 0, ptests = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        if (lock) {
            const unsigned vmask = __ballot_sync(TT_FULL, valid);
            if (lane == 0) ws[0] = WarpEntry{0, TT_END, vmask};
            int sp = 1;
            while (sp > 0) {
                WarpEntry e;
                if (lane == 0) e = ws[sp - 1];
                e.node = __shfl_sync(TT_FULL, e.node, 0);
                e.end = __shfl_sync(TT_FULL, e.end, 0);
                e.mask = __shfl_sync(TT_FULL, e.mask, 0);
                --sp;
                const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + e.node));
                if (STATS) ++steps;
                if (t.z != e.end) {
                    if (lane == 0) ws[sp] = WarpEntry{t.z, e.end, e.mask};
                    ++sp;
                }
                bool down = false;
                if ((e.mask >> lane) & 1u) {
                    if (STATS) {
                        ++visits;
                        if (hashing) vh.add(P.c.pre, e.node);
                    }
                    down = pc_visit<DIM>(P, rec, e.node, t, DP, q, count, ptests);
                }
                const unsigned cmask = __ballot_sync(TT_FULL, down);
                if (cmask) {
                    if (lane == 0) ws[sp] = WarpEntry{t.x, t.z, cmask};
                    ++sp;
                }
                __syncwarp();
            }
            fetches = steps;
        } else {
            int sp = 0;
            if (valid) {
                gpush(gstack, 0, stride, gtid, 0, TT_END);
                sp = 1;
            }
            while (sp > 0) {
                const int2 e = gpop(gstack, --sp, stride, gtid);
                const int4 t = __ldg(reinterpret_cast<const int4 *>(rec + e.x));
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, e.x);
                }
                if (t.z != e.y) gpush(gstack, sp++, stride, gtid, t.z, e.y);
                if (pc_visit<DIM>(P, rec, e.x, t, DP, q, count, ptests)) gpush(gstack, sp++, stride, gtid, t.x, t.z);
            }
            if (STATS) {
                fetches = warp_sum(visits);
                steps = __reduce_max_sync(TT_FULL, visits);
            }
        }
        if (valid) {
            P.count[pid] = count;
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
            if (STATS && P.c.st_point_tests) P.c.st_point_tests[pid] = ptests;
            if (hashing) vh.store(P.c, pid);
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
    }
    (void)cap;
    cta_finish(P.c.counter);
}

// ------------------------------------------------------------------ launch
// Persistent grid (occupancy x SMs); the interleaved global stacks hold
// (height + 2) int2 entries per resident thread, stream-ordered scratch.
template <typename Kern, typename Params>
int launch_with_stack(Kern kern, const Params &p, const tt_launch_cfg &cfg) {
    int dev = 0, nsm = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, 0);
    if (e != cudaSuccess) return (int)e;
    if (cfg.ctas_per_sm > 0 && cfg.ctas_per_sm < occ) occ = cfg.ctas_per_sm;
    if (occ < 1) occ = 1;
    const long long ntiles = (p.c.n + 31) / 32;
    long long grid = (long long)nsm * occ;
    const long long need = (ntiles + kWarps - 1) / kWarps;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    const int cap = p.c.height + 2;
    int2 *gstack = nullptr;
    const cudaStream_t s = (cudaStream_t)cfg.stream;
    if (p.c.mode == TT_MODE_INDEPENDENT || (p.c.mode == TT_MODE_AUTO && std::is_same<Params, tt_pc_params>::value)) {
        tt_keep_pool_memory();
        e = cudaMallocAsync((void **)&gstack, sizeof(int2) * (size_t)cap * (size_t)grid * kBlock, s);
        if (e != cudaSuccess) return (int)e;
    }
    kern<<<(unsigned)grid, kBlock, 0, s>>>(p, gstack, cap);
    e = cudaGetLastError();
    if (gstack) cudaFreeAsync(gstack, s);
    return (int)e;
}

template <int DIM>
int launch_pc_dim(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    return stats ? launch_with_stack(pc_stack_kernel<DIM, true>, p, cfg)
                 : launch_with_stack(pc_stack_kernel<DIM, false>, p, cfg);
}

}  // namespace

int tt_launch_bh_stack(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    if (p.c.height + 2 > TT_MAX_HEIGHT + 2) return -1;
    const bool stats = stats_on(p.c);
    return stats ? launch_with_stack(bh_stack_kernel<true>, p, cfg) : launch_with_stack(bh_stack_kernel<false>, p, cfg);
}

int tt_launch_pc_stack(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg) {
    if (p.c.height + 2 > TT_MAX_HEIGHT + 2) return -1;
    switch (dim) {
    case 1: return launch_pc_dim<1>(p, cfg);
    case 2: return launch_pc_dim<2>(p, cfg);
    case 3: return launch_pc_dim<3>(p, cfg);
    case 4: return launch_pc_dim<4>(p, cfg);
    case 5: return launch_pc_dim<5>(p, cfg);
    case 6: return launch_pc_dim<6>(p, cfg);
    case 7: return launch_pc_dim<7>(p, cfg);
    case 8: return launch_pc_dim<8>(p, cfg);
    case 16: return launch_pc_dim<16>(p, cfg);
    default: return -1;
    }
}
