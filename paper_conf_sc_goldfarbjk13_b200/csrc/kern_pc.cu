// kern_pc.cu -- 2-point correlation over a kd-tree (Fig.4 P:L425-438,
// autoroped Fig.6, lockstep Fig.8), sm_100a.
//
// Unguided (single call set: left then right), so the walk is
// stackless over the ropes: next = descend ? left : skip.  Lockstep uses the
// same level-wait rule as kern_bh.cu: a lane truncated or
// finished at node m re-activates at the first node whose level <= level[m],
// which is exactly skip[m].  Truncated lanes never update (Fig.8 line 13,
// reading R13).
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kSmemHdr = 128;

template <int DIM>
struct PcNode {
    float lo[DIM], hi[DIM];
    int4 t;  // left, right, skip, level
};

template <int DIM>
__device__ __forceinline__ void ld_node(const unsigned char *s_rec, const float *s_box, const tt_kd_rec *g_rec,
                                        const float *g_box, int dp, int top, int cur, PcNode<DIM> &nd) {
    if (cur < top) {
        nd.t = reinterpret_cast<const int4 *>(s_rec)[cur * 2];
        load_row_smem<DIM>(nd.lo, s_box + (size_t)cur * 2 * dp);
        load_row_smem<DIM>(nd.hi, s_box + (size_t)cur * 2 * dp + dp);
    } else {
        nd.t = __ldg(reinterpret_cast<const int4 *>(g_rec + cur));
        load_row_nc<DIM>(nd.lo, g_box + (size_t)cur * 2 * dp);
        load_row_nc<DIM>(nd.hi, g_box + (size_t)cur * 2 * dp + dp);
    }
}

// Leaf update (update_correlation): count the bucket's points within r.
// With one point per leaf the tight box IS the point and boxd2 == d2 exactly
// (both are the same pinned sequence on |q - p|), so nothing more is loaded.
template <int DIM>
__device__ __forceinline__ unsigned leaf_count(const tt_pc_params &P, const tt_kd_rec *g_rec, int cur,
                                               const float (&q)[DIM], int dp) {
    const int4 u = __ldg(reinterpret_cast<const int4 *>(g_rec + cur) + 1);
    const int pb = u.z, pc = u.w;
    if (pc == 1) return 1u;
    unsigned c = 0;
    for (int j = pb; j < pb + pc; ++j) {
        float p[DIM];
        load_row_nc<DIM>(p, P.c.tree.pts + (size_t)j * dp);
        c += pinned_d2<DIM>(q, p) <= P.r2;
    }
    return c;
}

template <int DIM, bool STATS>
__global__ void __launch_bounds__(kBlock) pc_kernel(const tt_pc_params P) {
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int DP = (DIM + 3) & ~3;
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    const int top = P.c.top_count;
    unsigned char *s_rec = smem + kSmemHdr;
    float *s_box = reinterpret_cast<float *>(s_rec + (size_t)top * 32);
    const tt_kd_rec *g_rec = static_cast<const tt_kd_rec *>(P.c.tree.rec);
    const float *g_box = P.c.tree.box;
    StageChunk ch[2] = {{s_rec, g_rec, (unsigned)top * 32u}, {s_box, g_box, (unsigned)top * 8u * DP}};
    stage_top(bar, ch);

    const int lane = threadIdx.x & 31;
    const long long n = P.c.n;
    const long long ntiles = (n + 31) >> 5;
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
        const unsigned vmask = __ballot_sync(TT_FULL, valid);

        bool lock = P.c.mode != TT_MODE_INDEPENDENT;
        if (P.c.mode == TT_MODE_AUTO && P.c.auto_min_depth > 0) {
            // descend the staged top levels by the split rule; path bits
            int cur = 0, lv = 0;
            unsigned long long code = 0;
            const int maxl = min(P.c.auto_min_depth, 60);
            while (lv < maxl && cur >= 0 && cur < top) {
                const int4 t = reinterpret_cast<const int4 *>(s_rec)[cur * 2];
                if (t.x < 0) break;
                const int4 u = reinterpret_cast<const int4 *>(s_rec)[cur * 2 + 1];
                const bool left = select_dim<DIM>(q, u.y) < __int_as_float(u.x);
                code = (code << 1) | (left ? 0u : 1u);
                cur = left ? t.x : t.y;
                ++lv;
            }
            lock = P.c.auto_min_depth < 64 && warp_key_changes(code << (maxl - lv), valid) < kAutoMaxChanges;
        }

        unsigned count = 0, visits = 0, fetches = 0, steps = 0, ptests = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        if (lock) {
            int wait = valid ? INT_MAX : -1;
            int cur = 0;
            while (cur != TT_END) {
                PcNode<DIM> nd;
                ld_node<DIM>(s_rec, s_box, g_rec, g_box, DP, top, cur, nd);
                if (STATS) ++steps;
                const bool active = nd.t.w <= wait;
                bool descend = false;
                if (active) {
                    if (STATS) {
                        ++visits;
                        if (hashing) vh.add(P.c.pre, cur);
                    }
                    if (pinned_boxd2<DIM>(q, nd.lo, nd.hi) > P.r2) {
                        wait = nd.t.w;                       // !can_correlate: truncate
                    } else if (nd.t.x < 0) {
                        count += leaf_count<DIM>(P, g_rec, cur, q, DP);  // update_correlation
                        if (STATS) ptests += (unsigned)__ldg(&g_rec[cur].pcount);
                        wait = nd.t.w;
                    } else {
                        descend = true;
                        wait = INT_MAX;
                    }
                }
                cur = __any_sync(TT_FULL, descend) ? nd.t.x : nd.t.z;
            }
            fetches = steps;
        } else {
            int cur = valid ? 0 : TT_END;
            while (cur != TT_END) {
                PcNode<DIM> nd;
                ld_node<DIM>(s_rec, s_box, g_rec, g_box, DP, top, cur, nd);
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, cur);
                }
                bool descend = false;
                if (pinned_boxd2<DIM>(q, nd.lo, nd.hi) <= P.r2) {
                    if (nd.t.x < 0) {
                        count += leaf_count<DIM>(P, g_rec, cur, q, DP);
                        if (STATS) ptests += (unsigned)__ldg(&g_rec[cur].pcount);
                    } else {
                        descend = true;
                    }
                }
                cur = descend ? nd.t.x : nd.t.z;
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
    cta_finish(P.c.counter);
}

template <int DIM, bool STATS>
int launch(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    constexpr int DP = (DIM + 3) & ~3;
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * (32 + 8 * DP);
    auto kern = pc_kernel<DIM, STATS>;
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

template <int DIM>
int launch_dim(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    return stats ? launch<DIM, true>(p, cfg) : launch<DIM, false>(p, cfg);
}

}  // namespace

int tt_launch_pc(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg) {
    switch (dim) {
    case 1: return launch_dim<1>(p, cfg);
    case 2: return launch_dim<2>(p, cfg);
    case 3: return launch_dim<3>(p, cfg);
    case 4: return launch_dim<4>(p, cfg);
    case 5: return launch_dim<5>(p, cfg);
    case 6: return launch_dim<6>(p, cfg);
    case 7: return launch_dim<7>(p, cfg);
    case 8: return launch_dim<8>(p, cfg);
    case 16: return launch_dim<16>(p, cfg);
    default: return -1;
    }
}
