// kern_bh.cu -- Barnes-Hut force traversal (Fig.9), sm_100a.
//
// Unguided traversal (one call set): every body visits children in
// octant order, so the autoroped walk needs no stack at all -- the packed tree
// stores the rope (skip) of every node (Fig.2), and the walk is
//     next = descend ? first_child : skip.
// Lockstep (Fig.8) without a mask stack: the warp holds one
// uniform `cur`; lane i is active at `cur` iff level[cur] <= wait_i.  A lane
// that truncates (or interacts) at node m waits with wait_i = level[m]: every
// node inside subtree(m) is deeper than m and the first node after it (the
// rope target skip[m]) is not, so the lane re-activates exactly at the node
// its own traversal visits next.  The warp descends iff any
// active lane opens the cell (__any_sync = Fig.8's warp_and of masks).
// Each lane therefore tests exactly its own recursive visit sequence: results
// and per-point visit counts are bit-identical to the independent walk.
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kSmemHdr = 384;  // [0,16) mbarrier, [16,272) dsq table (64 floats)

__device__ __forceinline__ void ld_rec(const tt_oct_rec *s_top, const tt_oct_rec *g, int top, int cur,
                                       float4 &gg, int4 &tt) {
    if (cur < top) {
        gg = *reinterpret_cast<const float4 *>(&s_top[cur].gx);
        tt = *reinterpret_cast<const int4 *>(&s_top[cur].first_child);
    } else {
        gg = __ldg(reinterpret_cast<const float4 *>(&g[cur].gx));
        tt = __ldg(reinterpret_cast<const int4 *>(&g[cur].first_child));
    }
}

// 63-bit octant path of a body through the root cube (fp64 comparisons, R8a).
__device__ __forceinline__ unsigned long long oct_path(float4 b, const double c0[3], double side, int levels) {
    double c[3] = {c0[0], c0[1], c0[2]};
    unsigned long long code = 0;
    for (int l = 0; l < levels; ++l) {
        double h = side * 0.25;
        int o = ((double)b.x >= c[0]) | (((double)b.y >= c[1]) << 1) | (((double)b.z >= c[2]) << 2);
        code = (code << 3) | (unsigned)o;
        c[0] += (o & 1) ? h : -h;
        c[1] += (o & 2) ? h : -h;
        c[2] += (o & 4) ? h : -h;
        side *= 0.5;
    }
    return code;
}

template <bool STATS>
__global__ void __launch_bounds__(kBlock) bh_kernel(const tt_bh_params P) {
    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    float *s_dsq = reinterpret_cast<float *>(smem + 16);
    tt_oct_rec *s_top = reinterpret_cast<tt_oct_rec *>(smem + kSmemHdr);
    const tt_oct_rec *g_rec = static_cast<const tt_oct_rec *>(P.c.tree.rec);
    const int top = P.c.top_count;

    // dsq_L = dsq_root * 0.25^L (Fig.9a line 4: "dsq*0.25" per level), exact.
    if (threadIdx.x == 0) {
        float d = P.dsq_root;
        for (int l = 0; l < 64; ++l) {
            s_dsq[l] = d;
            d = __fmul_rn(d, 0.25f);
        }
    }
    StageChunk ch[1] = {{s_top, g_rec, (unsigned)top * 32u}};
    stage_top(bar, ch);
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const long long n = P.c.n;
    const long long ntiles = (n + 31) >> 5;
    const float eps2 = P.eps2;

    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        const long long pos = tile * 32 + lane;
        const bool valid = pos < n;
        const long long pid = valid ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
        const float4 b = valid ? __ldg(P.bodies + pid) : make_float4(0.f, 0.f, 0.f, 0.f);
        const int self = valid ? (P.self_ids ? __ldg(P.self_ids + pid) : (int)pid) : -2;
        const unsigned vmask = __ballot_sync(TT_FULL, valid);

        bool lock = P.c.mode != TT_MODE_INDEPENDENT;
        if (P.c.mode == TT_MODE_AUTO && P.c.auto_min_depth > 0) {
            const int lv = min(P.c.auto_min_depth, 21);
            unsigned long long code = oct_path(b, P.c.root_center, P.c.root_side, lv);
            lock = warp_common_levels(code, vmask, 3, lv) >= P.c.auto_min_depth;
        }

        // fp64 accumulation of fp32 terms: the tree-order partial sums of a body
        // near the centre of mass cancel by 2-3 orders of magnitude, which fp32
        // accumulation turns into >1e-4 relative error.
        double ax = 0.0, ay = 0.0, az = 0.0;
        unsigned visits = 0, fetches = 0, steps = 0;
        if (lock) {
            int wait = valid ? INT_MAX : -1;
            int cur = 0;
            while (cur != TT_END) {
                float4 g;
                int4 t;
                ld_rec(s_top, g_rec, top, cur, g, t);
                if (STATS) ++steps;
                const int lvl = t.w;
                const bool active = lvl <= wait;
                const float dx = __fsub_rn(g.x, b.x);
                const float dy = __fsub_rn(g.y, b.y);
                const float dz = __fsub_rn(g.z, b.z);
                const float drsq = __fadd_rn(__fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)), __fmul_rn(dz, dz));
                const bool open = active && t.x >= 0 && drsq < s_dsq[lvl];
                if (active) {
                    if (STATS) ++visits;
                    wait = open ? INT_MAX : lvl;
                    if (!open && t.z != self) {
                        const float inv = rsqrtf(__fadd_rn(drsq, eps2));
                        const float f = g.w * inv * inv * inv;
                        ax += (double)(f * dx);
                        ay += (double)(f * dy);
                        az += (double)(f * dz);
                    }
                }
                cur = __any_sync(TT_FULL, open) ? t.x : t.y;
            }
            fetches = steps;
        } else {
            int cur = valid ? 0 : TT_END;
            while (cur != TT_END) {
                float4 g;
                int4 t;
                ld_rec(s_top, g_rec, top, cur, g, t);
                if (STATS) ++visits;
                const float dx = __fsub_rn(g.x, b.x);
                const float dy = __fsub_rn(g.y, b.y);
                const float dz = __fsub_rn(g.z, b.z);
                const float drsq = __fadd_rn(__fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)), __fmul_rn(dz, dz));
                const bool open = t.x >= 0 && drsq < s_dsq[t.w];
                if (!open && t.z != self) {
                    const float inv = rsqrtf(__fadd_rn(drsq, eps2));
                    const float f = g.w * inv * inv * inv;
                    ax += (double)(f * dx);
                    ay += (double)(f * dy);
                    az += (double)(f * dz);
                }
                cur = open ? t.x : t.y;
            }
            if (STATS) {
                fetches = warp_sum(visits);
                steps = __reduce_max_sync(TT_FULL, visits);
            }
        }
        if (valid) {
            P.acc[pid] = make_float4((float)ax, (float)ay, (float)az, 0.f);
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
    }
    cta_finish(P.c.counter);
}

template <bool STATS>
int launch(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * 32;
    auto kern = bh_kernel<STATS>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    int dev = 0, nsm = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, smem);
    if (e != cudaSuccess) return (int)e;
    if (cfg.ctas_per_sm > 0 && cfg.ctas_per_sm < occ) occ = cfg.ctas_per_sm;
    if (occ < 1) occ = 1;
    const long long ntiles = (p.c.n + 31) / 32;
    long long grid = (long long)nsm * occ;
    const long long need = (ntiles + kBlock / 32 - 1) / (kBlock / 32);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, kBlock, smem, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}

}  // namespace

int tt_launch_bh(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    const bool stats = p.c.st_visits || p.c.st_warp_fetches || p.c.st_warp_steps || p.c.st_warp_mode;
    return stats ? launch<true>(p, cfg) : launch<false>(p, cfg);
}
