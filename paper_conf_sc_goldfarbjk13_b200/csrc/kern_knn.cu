// kern_knn.cu -- k-nearest neighbours over a kd-tree (Fig.5 P:L440-458,
// autoroped Fig.7), sm_100a.
//
// Guided traversal with two call sets (near child first).  Autoropes with an
// explicit rope stack in shared memory:
//   independent (N): one stack per lane, lane-interleaved [depth][32] int32
//     (the shared-memory analogue of the paper's interleaved per-thread
//     stacks; bank = lane, conflict-free);
//   lockstep (L): one stack per warp of {node, mask} (Fig.8);
//     the call set is reduced per warp by a majority vote of the active lanes
//     (§4.3; tie -> left first, reading R6).
// Pushing the far child and continuing into the near one is the reverse-order
// push of §3.2.2 with its immediate pop folded away.
// can_correlate (reading R5a): prune iff the k-heap is full and the tight box
// distance exceeds the current k-th best -- conservative under the pinned
// arithmetic, so the result is exactly the brute-force definition.  The box
// distance of a child is computed while its parent is expanded (the blob
// stores both children's boxes with the parent, `cbox`) and travels on the
// rope stack with the node as Fig.7's non-invariant argument;
// the test itself is made when the node is popped, against the k-th best of
// that moment -- the same decision as testing at the visit, but a popped node
// that is pruned costs no memory access, and an expanded node is one
// independent load group (record + children's boxes).
// Per-lane k-best list: KT register slots kept sorted ascending on (d2, id);
// the first KT-k slots hold (-inf) sentinels, so the k-th best is always
// slot KT-1 (static register index).
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kWarps = kBlock / 32;
constexpr int kSmemHdr = 128;

__device__ __forceinline__ bool kless(float da, unsigned ia, float db, unsigned ib) {
    return da < db || (da == db && ia < ib);
}

template <int KT>
struct KBest {
    float d[KT];
    unsigned i[KT];
    __device__ __forceinline__ void init(int k) {
#pragma unroll
        for (int j = 0; j < KT; ++j) {
            const bool real = j >= KT - k;
            d[j] = real ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
            i[j] = 0xffffffffu;
        }
    }
    __device__ __forceinline__ float worst() const { return d[KT - 1]; }
    // caller guarantees (dd, ii) < (d[KT-1], i[KT-1])
    __device__ __forceinline__ void insert(float dd, unsigned ii) {
        d[KT - 1] = dd;
        i[KT - 1] = ii;
#pragma unroll
        for (int j = KT - 1; j > 0; --j) {
            const bool sw = kless(d[j], i[j], d[j - 1], i[j - 1]);
            const float td = d[j - 1];
            const unsigned ti = i[j - 1];
            d[j - 1] = sw ? d[j] : td;
            i[j - 1] = sw ? i[j] : ti;
            d[j] = sw ? td : d[j];
            i[j] = sw ? ti : i[j];
        }
    }
};

__device__ __forceinline__ void ld_rec(const unsigned char *s_rec, const tt_kd_rec *g_rec, int top, int cur,
                                       int4 &t, int4 &u) {
    if (cur < top) {
        t = reinterpret_cast<const int4 *>(s_rec)[cur * 2];
        u = reinterpret_cast<const int4 *>(s_rec)[cur * 2 + 1];
    } else {
        t = __ldg(reinterpret_cast<const int4 *>(g_rec + cur));
        u = __ldg(reinterpret_cast<const int4 *>(g_rec + cur) + 1);
    }
}

// box distances of node `cur`'s two children (from the parent's cbox row)
template <int DIM>
__device__ __forceinline__ void child_lbs(const float *s_cbox, const float *g_cbox, int dp, int top, int cur,
                                          const float (&q)[DIM], float &lb_left, float &lb_right) {
    float lo[DIM], hi[DIM];
    const float *row = (cur < top ? s_cbox : g_cbox) + (size_t)cur * 4 * dp;
    if (cur < top) {
        load_row_smem<DIM>(lo, row);
        load_row_smem<DIM>(hi, row + dp);
        lb_left = pinned_boxd2<DIM>(q, lo, hi);
        load_row_smem<DIM>(lo, row + 2 * dp);
        load_row_smem<DIM>(hi, row + 3 * dp);
        lb_right = pinned_boxd2<DIM>(q, lo, hi);
    } else {
        load_row_nc<DIM>(lo, row);
        load_row_nc<DIM>(hi, row + dp);
        lb_left = pinned_boxd2<DIM>(q, lo, hi);
        load_row_nc<DIM>(lo, row + 2 * dp);
        load_row_nc<DIM>(hi, row + 3 * dp);
        lb_right = pinned_boxd2<DIM>(q, lo, hi);
    }
}

// update_closest: every bucket point that beats the k-th best enters the list.
template <int DIM, int KT>
__device__ __forceinline__ void leaf_update(const tt_knn_params &P, int pb, int pc, int dp, const float (&q)[DIM],
                                            KBest<KT> &kb) {
#pragma unroll 2
    for (int j = pb; j < pb + pc; ++j) {
        float p[DIM];
        load_row_nc<DIM>(p, P.c.tree.pts + (size_t)j * dp);
        const float d2 = pinned_d2<DIM>(q, p);
        if (d2 <= kb.worst()) {
            const unsigned id = (unsigned)__ldg(P.c.tree.pid + j);
            if (kless(d2, id, kb.worst(), kb.i[KT - 1])) kb.insert(d2, id);
        }
    }
}

#ifndef TT_KNN_MINB
#define TT_KNN_MINB 4
#endif
// per-warp rope-stack bytes: INDEPENDENT launches keep {node, lb} per lane in
// shared memory ("wide"); AUTO / LOCKSTEP launches keep per-lane lb + the
// warp-uniform {node, mask} ("narrow"), and their independent warps put the
// lb half of a lane entry in a per-thread interleaved global scratch.
__host__ __device__ constexpr size_t knn_stack_bytes(int cap, bool wide) {
    return wide ? (size_t)cap * 32 * 8 : (size_t)cap * (32 * 4 + 8);
}

template <int DIM, int KT, bool STATS>
__global__ void __launch_bounds__(kBlock, TT_KNN_MINB) knn_kernel(const tt_knn_params P, int cap, float *g_lb) {
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int DP = (DIM + 3) & ~3;
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    const int top = P.c.top_count;
    unsigned char *s_rec = smem + kSmemHdr;
    float *s_cbox = reinterpret_cast<float *>(s_rec + (size_t)top * 32);
    unsigned char *s_stack = reinterpret_cast<unsigned char *>(s_cbox) + (size_t)top * 16 * DP;
    const tt_kd_rec *g_rec = static_cast<const tt_kd_rec *>(P.c.tree.rec);
    const float *g_cbox = P.c.tree.cbox;
    StageChunk ch[2] = {{s_rec, g_rec, (unsigned)top * 32u}, {s_cbox, g_cbox, (unsigned)top * 16u * DP}};
    stage_top(bar, ch);

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    // per-warp region of cap*32*8 bytes:
    //   N: node[cap][32], lb[cap][32]       (per-lane stacks, lane-interleaved)
    //   L: lb[cap][32], node[cap], mask[cap] (warp-uniform part owned by lane 0)
    const bool wide = g_lb == nullptr;
    unsigned char *wreg = s_stack + (size_t)warp * knn_stack_bytes(cap, wide);
    int *n_node = reinterpret_cast<int *>(wreg);
    // lb half of the independent stacks: shared (wide) or global scratch
    const size_t gtid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, gstride = (size_t)gridDim.x * blockDim.x;
    float *n_lbs = wide ? reinterpret_cast<float *>(wreg + (size_t)cap * 32 * 4) : g_lb + gtid;
    const size_t lbs_stride = wide ? 32 : gstride;
    const int lbs_lane = wide ? lane : 0;
    float *l_lb = reinterpret_cast<float *>(wreg);
    int *l_node = reinterpret_cast<int *>(wreg + (size_t)cap * 32 * 4);
    unsigned *l_mask = reinterpret_cast<unsigned *>(l_node + cap);
    const long long n = P.c.n;
    const long long ntiles = (n + 31) >> 5;
    const int k = P.k;
    const float INF = __int_as_float(0x7f800000);

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
            int cur = 0, lv = 0;
            unsigned long long code = 0;
            const int maxl = min(max(P.c.auto_min_depth, 1), 60);
            while (lv < maxl && cur >= 0 && cur < top) {
                const int4 t = reinterpret_cast<const int4 *>(s_rec)[cur * 2];
                if (t.x < 0) break;
                const int4 u = reinterpret_cast<const int4 *>(s_rec)[cur * 2 + 1];
                const bool left = select_dim<DIM>(q, u.y) < __int_as_float(u.x);
                code = (code << 1) | (left ? 0u : 1u);
                cur = left ? t.x : t.y;
                ++lv;
            }
            lock = P.c.auto_min_depth == 0 || warp_key_changes(code << (maxl - lv), valid) < kAutoMaxChanges;
        }

        KBest<KT> kb;
        kb.init(k);
        unsigned visits = 0, fetches = 0, steps = 0, ptests = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        // independent-walk state: the whole tile (N mode), or the rest of it
        // after a dynamic L->N switch
        int n_sp = 0;
        int n_cur = valid ? 0 : TT_END;
        float n_lb = 0.f;  // the root is never pruned: the list starts empty
        bool run_n = !lock;
        unsigned l_fetches = 0, l_steps = 0;
        if (lock) {
            int sp = 0;
            int cur = 0;
            unsigned mask = vmask;
            float lb = 0.f;
            const int switch_below = P.c.switch_below;
            for (;;) {
                const bool in = (mask >> lane) & 1u;
                if (STATS) {
                    ++steps;
                    visits += in;
                    if (hashing) vh.add_if(in, P.c.pre, cur);
                }
                const bool active = in && !(kb.worst() < INF && lb > kb.worst());
                const unsigned act = __ballot_sync(TT_FULL, active);
                if (act && __popc(act) < switch_below) {
                    // NEXT-3 dynamic L->N switch: each lane's rope stack is the
                    // warp entries whose mask holds it, in order (a lockstep
                    // lane visits exactly those), with its own bound.  The
                    // warp-uniform halves are read lane-distributed first; a
                    // lane's writes then only touch its own column of lb[][]
                    // (row j <= i, already consumed) and the node/mask region
                    // (already read).
                    int en0 = 0, en1 = 0;
                    unsigned em0 = 0, em1 = 0;
                    __syncwarp();  // lane 0's pushes visible to every lane
                    if (lane < sp) {
                        en0 = l_node[lane];
                        em0 = l_mask[lane];
                    }
                    if (lane + 32 < sp) {
                        en1 = l_node[lane + 32];
                        em1 = l_mask[lane + 32];
                    }
                    __syncwarp();
                    int j = 0;
                    for (int i = 0; i < sp; ++i) {
                        const int e_node = __shfl_sync(TT_FULL, i < 32 ? en0 : en1, i & 31);
                        const unsigned e_mask = __shfl_sync(TT_FULL, i < 32 ? em0 : em1, i & 31);
                        if ((e_mask >> lane) & 1u) {
                            const float v = l_lb[i * 32 + lane];
                            n_node[j * 32 + lane] = e_node;
                            n_lbs[j * lbs_stride + lbs_lane] = v;
                            ++j;
                        }
                    }
                    n_sp = j;
                    // lanes of the mask resume at `cur` (the N loop re-takes its
                    // truncation test, so it is not counted twice); the others
                    // pop their own stack
                    if (in) {
                        n_cur = cur;
                        n_lb = lb;
                        if (STATS) {
                            --visits;
                            if (hashing) {  // the N loop re-takes this test: undo its hash step
                                const unsigned long long v = (unsigned long long)(unsigned)__ldg(P.c.pre + cur) + 1ull;
                                vh.h = (vh.h - v) * 0xef7bdef7bdef7bdfull;  // * 31^-1 mod 2^64
                                vh.s -= vh_mix64(v);
                            }
                        }
                    } else if (n_sp > 0) {
                        --n_sp;
                        n_cur = n_node[n_sp * 32 + lane];
                        n_lb = n_lbs[n_sp * lbs_stride + lbs_lane];
                    } else {
                        n_cur = TT_END;
                    }
                    if (STATS) --steps;
                    run_n = true;
                    break;
                }
                if (act) {
                    if (STATS) ++fetches;
                    int4 t, u;
                    ld_rec(s_rec, g_rec, top, cur, t, u);
                    if (t.x < 0) {
                        if (active) {
                            leaf_update<DIM, KT>(P, u.z, u.w, DP, q, kb);
                            if (STATS) ptests += (unsigned)u.w;
                        }
                    } else {
                        float lbl, lbr;
                        child_lbs<DIM>(s_cbox, g_cbox, DP, top, cur, q, lbl, lbr);
                        const bool pref_left = active && select_dim<DIM>(q, u.y) < __int_as_float(u.x);
                        const int votes = __popc(__ballot_sync(TT_FULL, pref_left));
                        const bool left_first = 2 * votes >= __popc(act);
                        if (lane == 0) {  // push second (warp-uniform entry)
                            l_node[sp] = left_first ? t.y : t.x;
                            l_mask[sp] = act;
                        }
                        l_lb[sp * 32 + lane] = left_first ? lbr : lbl;
                        ++sp;
                        cur = left_first ? t.x : t.y;
                        lb = left_first ? lbl : lbr;
                        mask = act;
                        continue;
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
                lb = l_lb[sp * 32 + lane];
            }
            l_fetches = fetches;
            l_steps = steps;
        }
        if (run_n) {
            const unsigned v0 = visits;
            int sp = n_sp;
            int cur = n_cur;
            float lb = n_lb;
            while (cur != TT_END) {
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, cur);
                }
                if (!(kb.worst() < INF && lb > kb.worst())) {  // can_correlate
                    int4 t, u;
                    ld_rec(s_rec, g_rec, top, cur, t, u);
                    if (t.x < 0) {
                        leaf_update<DIM, KT>(P, u.z, u.w, DP, q, kb);
                        if (STATS) ptests += (unsigned)u.w;
                    } else {
                        float lbl, lbr;
                        child_lbs<DIM>(s_cbox, g_cbox, DP, top, cur, q, lbl, lbr);
                        const bool left_near = select_dim<DIM>(q, u.y) < __int_as_float(u.x);
                        n_node[sp * 32 + lane] = left_near ? t.y : t.x;  // push far with its bound
                        n_lbs[sp * lbs_stride + lbs_lane] = left_near ? lbr : lbl;
                        ++sp;
                        cur = left_near ? t.x : t.y;                     // visit near
                        lb = left_near ? lbl : lbr;
                        continue;
                    }
                }
                if (sp > 0) {
                    --sp;
                    cur = n_node[sp * 32 + lane];
                    lb = n_lbs[sp * lbs_stride + lbs_lane];
                } else {
                    cur = TT_END;
                }
            }
            if (STATS) {
                // N part: every lane visit is a fetch; a switched tile adds its
                // lockstep fetches / steps
                fetches = l_fetches + warp_sum(visits - v0);
                steps = l_steps + __reduce_max_sync(TT_FULL, visits - v0);
            }
        }
        if (valid) {
#pragma unroll
            for (int j = 0; j < KT; ++j) {
                const int slot = j - (KT - k);
                if (slot >= 0) {
                    const bool empty = kb.i[j] == 0xffffffffu;
                    P.idx[pid * k + slot] = empty ? -1 : (int)kb.i[j];
                    P.d2[pid * k + slot] = kb.d[j];
                }
            }
            if (STATS && P.c.st_visits) P.c.st_visits[pid] = visits;
            if (STATS && P.c.st_point_tests) P.c.st_point_tests[pid] = ptests;
            if (hashing) vh.store(P.c, pid);
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock, lock && run_n);
        __syncwarp();
    }
    cta_finish(P.c.counter);
}

template <int DIM, int KT, bool STATS>
int launch(const tt_knn_params &p, const tt_launch_cfg &cfg) {
    constexpr int DP = (DIM + 3) & ~3;
    const int cap = p.c.height + 2;
    const bool wide = p.c.mode == TT_MODE_INDEPENDENT;
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * (32 + 16 * DP) + (size_t)kWarps * knn_stack_bytes(cap, wide);
    auto kern = knn_kernel<DIM, KT, STATS>;
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
    float *g_lb = nullptr;
    const cudaStream_t s = (cudaStream_t)cfg.stream;
    if (!wide) {
        tt_keep_pool_memory();
        e = cudaMallocAsync((void **)&g_lb, sizeof(float) * (size_t)cap * (size_t)grid * kBlock, s);
        if (e != cudaSuccess) return (int)e;
    }
    kern<<<(unsigned)grid, kBlock, smem, s>>>(p, cap, g_lb);
    e = cudaGetLastError();
    if (g_lb) cudaFreeAsync(g_lb, s);
    return (int)e;
}

template <int DIM, int KT>
int launch_k(const tt_knn_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    return stats ? launch<DIM, KT, true>(p, cfg) : launch<DIM, KT, false>(p, cfg);
}

template <int DIM>
int launch_dim(const tt_knn_params &p, const tt_launch_cfg &cfg) {
    if (p.k <= 1) return launch_k<DIM, 1>(p, cfg);
    if (p.k <= 4) return launch_k<DIM, 4>(p, cfg);
    if (p.k <= 8) return launch_k<DIM, 8>(p, cfg);
    if (p.k <= 16) return launch_k<DIM, 16>(p, cfg);
    return launch_k<DIM, 32>(p, cfg);
}

}  // namespace

int tt_launch_knn(const tt_knn_params &p, int dim, const tt_launch_cfg &cfg) {
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
