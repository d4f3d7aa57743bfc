// kern_nn.cu -- nearest neighbour over the point-per-node kd-tree of the
// paper's NN benchmark ("a variation of nearest neighbor search
// with a different implementation of the kd-tree structure"; build rule R21),
// guided with two call sets (near child first), sm_100a.  NEXT-3.
//
// Fig.5 pattern with the update at every node (each node holds a
// data point, Fig.1 line 9 before the children):
//   truncate iff boxd2(q, node's tight subtree box) > best d2 (can_correlate,
//     as R5a; strict: an equal distance can still win on id);
//   update with the node's point by (d2, id);
//   near = q[dim] < split ? left : right (R5), visited first.
// The test needs no argument from the parent, so rope-stack entries are bare
// node indices:
//   independent (N): per-lane stacks, lane-interleaved [depth][32] int32 in
//     shared memory (bank = lane);
//   lockstep (L): one {node, mask} stack per warp owned by lane 0
//     (P:L1015-1023); the call set is reduced by a majority vote of the
//     active lanes (§4.3, tie -> left first, R6).
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kWarps = kBlock / 32;
constexpr int kSmemHdr = 128;

// the node's tight box distance (can_correlate)
template <int DIM>
__device__ __forceinline__ float node_boxd2(const float *s_box, const float *g_box, int dp, int top, int cur,
                                            const float (&q)[DIM]) {
    float lo[DIM], hi[DIM];
    if (cur < top) {
        load_row_smem<DIM>(lo, s_box + (size_t)cur * 2 * dp);
        load_row_smem<DIM>(hi, s_box + (size_t)cur * 2 * dp + dp);
    } else {
        load_row_nc<DIM>(lo, g_box + (size_t)cur * 2 * dp);
        load_row_nc<DIM>(hi, g_box + (size_t)cur * 2 * dp + dp);
    }
    return pinned_boxd2<DIM>(q, lo, hi);
}

// record and point of node `cur`
template <int DIM>
__device__ __forceinline__ void ld_node(const unsigned char *s_rec, const float *s_pt, const tt_nn_rec *g_rec,
                                        const float *g_pt, int dp, int top, int cur, int4 &t, float (&v)[DIM]) {
    if (cur < top) {
        t = reinterpret_cast<const int4 *>(s_rec)[cur];
        load_row_smem<DIM>(v, s_pt + (size_t)cur * dp);
    } else {
        t = __ldg(reinterpret_cast<const int4 *>(g_rec + cur));
        load_row_nc<DIM>(v, g_pt + (size_t)cur * dp);
    }
}

template <int DIM, bool STATS>
__global__ void __launch_bounds__(kBlock) nn_kernel(const tt_nn_params P, int cap) {
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int DP = (DIM + 3) & ~3;
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    const int top = P.c.top_count;
    unsigned char *s_rec = smem + kSmemHdr;
    float *s_box = reinterpret_cast<float *>(s_rec + (size_t)top * 16);
    float *s_pt = s_box + (size_t)top * 2 * DP;
    unsigned char *s_stack = reinterpret_cast<unsigned char *>(s_pt + (size_t)top * DP);
    const tt_nn_rec *g_rec = static_cast<const tt_nn_rec *>(P.c.tree.rec);
    const float *g_box = P.c.tree.box;
    const float *g_pt = P.c.tree.vpt;
    StageChunk ch[3] = {{s_rec, g_rec, (unsigned)top * 16u},
                        {s_box, g_box, (unsigned)top * 8u * DP},
                        {s_pt, g_pt, (unsigned)top * 4u * DP}};
    stage_top(bar, ch);

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    // per-warp region of cap*32*4 bytes:
    //   N: node[cap][32]          (per-lane stacks, lane-interleaved)
    //   L: node[cap], mask[cap]   (warp-uniform, owned by lane 0)
    unsigned char *wreg = s_stack + (size_t)warp * cap * 32 * 4;
    int *n_node = reinterpret_cast<int *>(wreg);
    int *l_node = reinterpret_cast<int *>(wreg);
    unsigned *l_mask = reinterpret_cast<unsigned *>(l_node + cap);
    const long long n = P.c.n;
    const long long ntiles = (n + 31) >> 5;
    const float POS_INF = __int_as_float(0x7f800000);

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

        bool lock = P.c.mode == TT_MODE_LOCKSTEP;
        if (P.c.mode == TT_MODE_AUTO && P.c.auto_min_depth >= 0 && P.c.auto_min_depth < 64) {
            // per-warp coherence (R19): left/right descent through the staged top
            int cur = 0, lv = 0;
            unsigned long long code = 0;
            const int maxl = min(max(P.c.auto_min_depth, 1), 60);
            while (lv < maxl && cur >= 0 && cur < top) {
                const int4 t = reinterpret_cast<const int4 *>(s_rec)[cur];
                if (t.w < 0) break;
                const bool left = select_dim<DIM>(q, t.w) < __int_as_float(t.z);
                const int nx = left ? t.x : t.y;
                if (nx < 0) break;
                code = (code << 1) | (left ? 0u : 1u);
                cur = nx;
                ++lv;
            }
            lock = P.c.auto_min_depth == 0 || warp_key_changes(code << (maxl - lv), valid) < kAutoMaxChanges;
        }

        float best_d = POS_INF;
        unsigned best_i = 0xffffffffu;
        unsigned visits = 0, fetches = 0, steps = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        if (!lock) {
            int sp = 0;
            int cur = valid ? 0 : TT_END;
            while (cur != TT_END) {
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, cur);
                }
                if (!(node_boxd2<DIM>(s_box, g_box, DP, top, cur, q) > best_d)) {
                    int4 t;
                    float v[DIM];
                    ld_node<DIM>(s_rec, s_pt, g_rec, g_pt, DP, top, cur, t, v);
                    const float d2 = pinned_d2<DIM>(q, v);
                    if (d2 <= best_d) {
                        const unsigned id = (unsigned)__ldg(P.c.tree.pid + cur);
                        if (d2 < best_d || id < best_i) {
                            best_d = d2;
                            best_i = id;
                        }
                    }
                    if (t.w >= 0) {
                        const bool left_near = select_dim<DIM>(q, t.w) < __int_as_float(t.z);
                        const int nearc = left_near ? t.x : t.y, farc = left_near ? t.y : t.x;
                        if (farc != TT_END) n_node[sp++ * 32 + lane] = farc;
                        if (nearc != TT_END) {
                            cur = nearc;
                            continue;
                        }
                    }
                }
                cur = sp > 0 ? n_node[--sp * 32 + lane] : TT_END;
            }
            if (STATS) {
                fetches = warp_sum(visits);
                steps = __reduce_max_sync(TT_FULL, visits);
            }
        } else {
            int sp = 0;
            int cur = 0;
            unsigned mask = vmask;
            for (;;) {
                const bool in = (mask >> lane) & 1u;
                if (STATS) {
                    ++steps;
                    visits += in;
                    if (hashing) vh.add_if(in, P.c.pre, cur);
                }
                // one warp-uniform box fetch, tested by every lane of the mask
                const bool active = in && !(node_boxd2<DIM>(s_box, g_box, DP, top, cur, q) > best_d);
                const unsigned act = __ballot_sync(TT_FULL, active);
                if (act) {
                    if (STATS) ++fetches;
                    int4 t;
                    float v[DIM];
                    ld_node<DIM>(s_rec, s_pt, g_rec, g_pt, DP, top, cur, t, v);
                    if (active) {
                        const float d2 = pinned_d2<DIM>(q, v);
                        if (d2 <= best_d) {
                            const unsigned id = (unsigned)__ldg(P.c.tree.pid + cur);
                            if (d2 < best_d || id < best_i) {
                                best_d = d2;
                                best_i = id;
                            }
                        }
                    }
                    if (t.w >= 0) {
                        const bool left_near = select_dim<DIM>(q, t.w) < __int_as_float(t.z);
                        const int votes = __popc(__ballot_sync(TT_FULL, active && left_near));
                        const bool left_first = 2 * votes >= __popc(act);
                        const int first = left_first ? t.x : t.y, second = left_first ? t.y : t.x;
                        if (second != TT_END) {
                            if (lane == 0) {  // push second (warp-uniform entry)
                                l_node[sp] = second;
                                l_mask[sp] = act;
                            }
                            ++sp;
                        }
                        if (first != TT_END) {
                            cur = first;
                            mask = act;
                            continue;
                        }
                    }
                }
                if (sp == 0) break;
                --sp;
                // lane 0 owns the warp-uniform stack; its pop is broadcast
                int e_node = 0;
                unsigned e_mask = 0;
                if (lane == 0) {
                    e_node = l_node[sp];
                    e_mask = l_mask[sp];
                }
                cur = __shfl_sync(TT_FULL, e_node, 0);
                mask = __shfl_sync(TT_FULL, e_mask, 0);
            }
        }
        if (valid) {
            P.idx[pid] = best_i == 0xffffffffu ? -1 : (int)best_i;
            P.d2[pid] = best_d;
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
            if (hashing) vh.store(P.c, pid);
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
        __syncwarp();
    }
    cta_finish(P.c.counter);
}

template <int DIM, bool STATS>
int launch(const tt_nn_params &p, const tt_launch_cfg &cfg) {
    constexpr int DP = (DIM + 3) & ~3;
    const int cap = p.c.height + 2;
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * (16 + 12 * DP) + (size_t)kWarps * cap * 32 * 4;
    auto kern = nn_kernel<DIM, STATS>;
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
    const long long need = (ntiles + kWarps - 1) / kWarps;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, kBlock, smem, (cudaStream_t)cfg.stream>>>(p, cap);
    return (int)cudaGetLastError();
}

template <int DIM>
int launch_dim(const tt_nn_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    return stats ? launch<DIM, true>(p, cfg) : launch<DIM, false>(p, cfg);
}

}  // namespace

int tt_launch_nn(const tt_nn_params &p, int dim, const tt_launch_cfg &cfg) {
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
