// kern_pc_split.cu -- 2-point correlation with each point's traversal split
// over a group of 16 lanes (TT_VARIANT_SPLIT), sm_100a.
//
// configs[0] (10k points) is one 313-warp wave on 148 SMs: with one lane per
// point the kernel is the latency of the longest walks.  The
// count of Fig.4 is a sum over leaves, so a point's walk splits
// exactly by subtree: lane s of the point's 16-lane group descends the top 4
// levels along the bits of s, taking the truncation test of each node on the
// way (a truncated or leaf ancestor ends the lane; a node shared by several
// lanes is counted -- and a shared leaf updated -- by the lowest of them
// only), then walks the subtree below with the stackless rope walk of
// kern_pc.cu until it reaches that subtree's rope.  The group's counts are
// summed with a shuffle butterfly.  Every node the recursive walk tests is
// tested by exactly one lane (the ancestors by the representative lane), so
// counts and per-point visit counts equal the oracle's.
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kSmemHdr = 128;
#ifndef TT_PC_SPLIT_LEVELS
#define TT_PC_SPLIT_LEVELS 4  // configs[0], B200: 2/3/4/5 levels = 119/108/100/124 us
#endif
constexpr int kSplitLevels = TT_PC_SPLIT_LEVELS;  // 2^levels lanes per point
constexpr int kGroup = 1 << kSplitLevels;
constexpr int kPointsPerWarp = 32 / kGroup;

template <int DIM>
__device__ __forceinline__ void ld_node(const unsigned char *s_rec, const float *s_box, const tt_kd_rec *g_rec,
                                        const float *g_box, int dp, int top, int cur, int4 &t, float (&lo)[DIM],
                                        float (&hi)[DIM]) {
    if (cur < top) {
        t = reinterpret_cast<const int4 *>(s_rec)[cur * 2];
        load_row_smem<DIM>(lo, s_box + (size_t)cur * 2 * dp);
        load_row_smem<DIM>(hi, s_box + (size_t)cur * 2 * dp + dp);
    } else {
        t = __ldg(reinterpret_cast<const int4 *>(g_rec + cur));
        load_row_nc<DIM>(lo, g_box + (size_t)cur * 2 * dp);
        load_row_nc<DIM>(hi, g_box + (size_t)cur * 2 * dp + dp);
    }
}

// update_correlation at a leaf (as kern_pc.cu): a one-point leaf's box is the
// point, so passing the box test already counts it.
template <int DIM>
__device__ __forceinline__ unsigned leaf_count(const tt_pc_params &P, const tt_kd_rec *g_rec, int cur,
                                               const float (&q)[DIM], int dp) {
    const int4 u = __ldg(reinterpret_cast<const int4 *>(g_rec + cur) + 1);
    if (u.w == 1) return 1u;
    unsigned c = 0;
    for (int j = u.z; j < u.z + u.w; ++j) {
        float p[DIM];
        load_row_nc<DIM>(p, P.c.tree.pts + (size_t)j * dp);
        c += pinned_d2<DIM>(q, p) <= P.r2;
    }
    return c;
}

template <int DIM, bool STATS>
__global__ void __launch_bounds__(kBlock) pc_split_kernel(const tt_pc_params P) {
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
    const int sub = lane & (kGroup - 1);
    const long long n = P.c.n;
    const long long ntiles = (n + kPointsPerWarp - 1) / kPointsPerWarp;
    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        const long long pos = tile * kPointsPerWarp + (lane >> kSplitLevels);
        const bool valid = pos < n;
        const long long pid = valid ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
        float q[DIM];
        if (valid) load_query<DIM>(q, P.q, pid, P.ld);
        else
#pragma unroll
            for (int d = 0; d < DIM; ++d) q[d] = 0.f;

        unsigned count = 0, visits = 0, ptests = 0;
        unsigned long long vset = 0;  // set hash only: the lanes split the walk (reading R23)
        const bool hashing = STATS && P.c.pre;
        int cur = valid ? 0 : TT_END;
        // the top kSplitLevels levels along the bits of `sub`
#pragma unroll
        for (int l = 0; l < kSplitLevels; ++l) {
            if (cur == TT_END) break;
            const bool rep = (sub & ((kGroup >> l) - 1)) == 0;  // lowest lane sharing this node
            int4 t;
            float lo[DIM], hi[DIM];
            ld_node<DIM>(s_rec, s_box, g_rec, g_box, DP, top, cur, t, lo, hi);
            if (STATS && rep) {
                ++visits;
                if (hashing) vset += vh_mix64((unsigned long long)(unsigned)__ldg(P.c.pre + cur) + 1ull);
            }
            if (pinned_boxd2<DIM>(q, lo, hi) > P.r2) {
                cur = TT_END;                                    // !can_correlate
            } else if (t.x < 0) {
                if (rep) {
                    count += leaf_count<DIM>(P, g_rec, cur, q, DP);
                    if (STATS) ptests += (unsigned)__ldg(&g_rec[cur].pcount);
                }
                cur = TT_END;
            } else {
                cur = ((sub >> (kSplitLevels - 1 - l)) & 1) ? t.y : t.x;
            }
        }
        // the lane's subtree: rope walk until the subtree's own rope
        if (cur != TT_END) {
            const int end = __ldg(reinterpret_cast<const int *>(g_rec + cur) + 2);
            while (cur != end) {
                int4 t;
                float lo[DIM], hi[DIM];
                ld_node<DIM>(s_rec, s_box, g_rec, g_box, DP, top, cur, t, lo, hi);
                if (STATS) {
                    ++visits;
                    if (hashing) vset += vh_mix64((unsigned long long)(unsigned)__ldg(P.c.pre + cur) + 1ull);
                }
                bool descend = false;
                if (pinned_boxd2<DIM>(q, lo, hi) <= P.r2) {
                    if (t.x < 0) {
                        count += leaf_count<DIM>(P, g_rec, cur, q, DP);
                        if (STATS) ptests += (unsigned)__ldg(&g_rec[cur].pcount);
                    } else {
                        descend = true;
                    }
                }
                cur = descend ? t.x : t.z;
            }
        }
        // sum over the point's group
#pragma unroll
        for (int o = kGroup / 2; o > 0; o >>= 1) {
            count += __shfl_xor_sync(TT_FULL, count, o);
            if (STATS) {
                visits += __shfl_xor_sync(TT_FULL, visits, o);
                ptests += __shfl_xor_sync(TT_FULL, ptests, o);
                vset += __shfl_xor_sync(TT_FULL, vset, o);
            }
        }
        if (valid && sub == 0) {
            P.count[pid] = count;
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
            if (STATS && P.c.st_point_tests) P.c.st_point_tests[pid] = ptests;
            if (hashing) {
                if (P.c.st_hash) P.c.st_hash[pid] = 0ull;  // no per-point order
                if (P.c.st_set) P.c.st_set[pid] = vset;
            }
        }
    }
    cta_finish(P.c.counter);
}

template <int DIM, bool STATS>
int launch(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    constexpr int DP = (DIM + 3) & ~3;
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * (32 + 8 * DP);
    auto kern = pc_split_kernel<DIM, STATS>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    int dev = 0, nsm = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, smem);
    if (e != cudaSuccess) return (int)e;
    if (cfg.ctas_per_sm > 0 && cfg.ctas_per_sm < occ) occ = cfg.ctas_per_sm;
    if (occ < 1) occ = 1;
    const long long ntiles = (p.c.n + kPointsPerWarp - 1) / kPointsPerWarp;
    long long grid = (long long)nsm * occ;
    const long long need = (ntiles + kBlock / 32 - 1) / (kBlock / 32);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, kBlock, smem, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}

template <int DIM>
int launch_dim(const tt_pc_params &p, const tt_launch_cfg &cfg) {
    return stats_on(p.c) ? launch<DIM, true>(p, cfg) : launch<DIM, false>(p, cfg);
}

}  // namespace

int tt_launch_pc_split(const tt_pc_params &p, int dim, const tt_launch_cfg &cfg) {
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
