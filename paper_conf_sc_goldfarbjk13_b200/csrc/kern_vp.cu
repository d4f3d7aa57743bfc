// kern_vp.cu -- nearest neighbour in a vantage-point tree (P:L1223-1226,
// [27] Yianilos), guided with two call sets (inside-first / outside-first),
// sm_100a.
//
// Every node holds a data point (its vantage point), so update() runs at
// every visited node before the children (Fig.1 line 9).  The
// non-invariant arguments of the recursive call -- the lower bound lb on the
// distance to any point of the child subtree and its scale sc -- travel on the
// rope stack with the node (Fig.7):
//   inside child:  lb = d - r_in_max,  sc = d + r_in_max
//   outside child: lb = r_out_min - d, sc = d + r_out_min
// and the truncation test at pop is lb - tau > eps_vp * (sc + tau) with
// tau = sqrt(best d2) (reading R12: conservative slack eps_vp = 2^-12).
// (lb, sc) are recomputed at pop from the lane's distance d to the parent's
// vantage point and the parent's radius on that side, with the same fp32
// operations as at push, so the arguments are bit-identical while an entry
// costs one float per lane:
//   L mode: per-warp entries {child << 1 | side, radius, mask} (lane 0 owns
//     them, pops are shuffled out) plus d[cap][32]; majority vote on the call
//     set (§4.3, tie -> inside first).
//   N mode, INDEPENDENT launches: per-lane {parent << 1 | side, d}; the child
//     and radius come from the parent's 16-B header at pop.
//   N mode inside an AUTO launch: per-lane {parent << 1 | side} in shared
//     memory, d in a per-thread interleaved global scratch [cap][threads]
//     (coalesced, L1/L2-resident; recomputing d from the parent's vantage
//     point instead made unsorted AUTO launches 870 vs 616 ms at 1M).
// The narrow layout halves the shared-memory stack of AUTO/LOCKSTEP launches,
// which the SM gives back to L1 for the (L2-resident) tree.
#include "kern_common.cuh"

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kWarps = kBlock / 32;
constexpr int kSmemHdr = 128;
#define TT_VP_EPS 0x1p-12f

// shared-memory rope stack bytes of one warp (see the header comment)
__host__ __device__ constexpr size_t vp_stack_bytes(int cap, bool wide) {
    return wide ? (size_t)cap * 32 * 8 : (size_t)cap * (32 * 4 + 16);
}

// tau = sqrt_rn(best d2) is kept in a register, recomputed only when the
// best improves (same value as recomputing it at every pop).
__device__ __forceinline__ bool vp_prune(float lb, float sc, float tau) {
    return __fsub_rn(lb, tau) > __fmul_rn(TT_VP_EPS, __fadd_rn(sc, tau));
}

template <int DIM>
__device__ __forceinline__ void ld_node(const unsigned char *s_rec, const float *s_vpt, const tt_vp_rec *g_rec,
                                        const float *g_vpt, int dp, int top, int cur, int4 &t, float (&v)[DIM]) {
    if (cur < top) {
        t = reinterpret_cast<const int4 *>(s_rec)[cur];
        load_row_smem<DIM>(v, s_vpt + (size_t)cur * dp);
    } else {
        t = __ldg(reinterpret_cast<const int4 *>(g_rec + cur));
        load_row_nc<DIM>(v, g_vpt + (size_t)cur * dp);
    }
}

// Child of `parent` on `side` (0 = inside, 1 = outside) and its (lb, sc).
__device__ __forceinline__ int child_args(int4 t, int side, float d, float &lb, float &sc) {
    const float rin = __int_as_float(t.z), rout = __int_as_float(t.w);
    lb = side ? __fsub_rn(rout, d) : __fsub_rn(d, rin);
    sc = side ? __fadd_rn(d, rout) : __fadd_rn(d, rin);
    return side ? t.y : t.x;
}

template <int DIM, bool STATS>
__global__ void __launch_bounds__(kBlock) vp_kernel(const tt_vp_params P, int cap, float *g_d) {
    extern __shared__ __align__(128) unsigned char smem[];
    constexpr int DP = (DIM + 3) & ~3;
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    const int top = P.c.top_count;
    unsigned char *s_rec = smem + kSmemHdr;
    float *s_vpt = reinterpret_cast<float *>(s_rec + (size_t)top * 16);
    unsigned char *s_stack = reinterpret_cast<unsigned char *>(s_vpt + (size_t)top * DP);
    const tt_vp_rec *g_rec = static_cast<const tt_vp_rec *>(P.c.tree.rec);
    const float *g_vpt = P.c.tree.vpt;
    StageChunk ch[2] = {{s_rec, g_rec, (unsigned)top * 16u}, {s_vpt, g_vpt, (unsigned)top * 4u * DP}};
    stage_top(bar, ch);

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const bool wide = P.c.mode == TT_MODE_INDEPENDENT;
    const size_t gtid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, gstride = (size_t)gridDim.x * blockDim.x;
    // per-warp region (vp_stack_bytes): wide: ent[cap][32], d[cap][32];
    // narrow: d (or N-mode ent)[cap][32], then int4 l_e[cap]
    unsigned char *wreg = s_stack + (size_t)warp * vp_stack_bytes(cap, wide);
    int *n_ent = reinterpret_cast<int *>(wreg);
    float *n_d = reinterpret_cast<float *>(wreg + (size_t)cap * 32 * 4);
    float *l_d = reinterpret_cast<float *>(wreg);
    int4 *l_e = reinterpret_cast<int4 *>(wreg + (size_t)cap * 32 * 4);
    const unsigned char *s_hdr_base = s_rec;
    const unsigned char *g_hdr_base = reinterpret_cast<const unsigned char *>(g_rec);
    auto hdr = [&](int node) -> int4 {
        const unsigned char *p = (node < top ? s_hdr_base : g_hdr_base) + (size_t)node * 16;
        return *reinterpret_cast<const int4 *>(p);
    };

    const long long n = P.c.n;
    const long long ntiles = (n + 31) >> 5;
    const float NEG_INF = __int_as_float(0xff800000), POS_INF = __int_as_float(0x7f800000);

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
            // inside/outside descent through the staged top levels
            int cur = 0, lv = 0;
            unsigned long long code = 0;
            const int maxl = min(max(P.c.auto_min_depth, 1), 60);
            while (lv < maxl && cur >= 0 && cur < top) {
                int4 t;
                float v[DIM];
                ld_node<DIM>(s_rec, s_vpt, g_rec, g_vpt, DP, top, cur, t, v);
                const float d = __fsqrt_rn(pinned_d2<DIM>(q, v));
                const bool inside = d <= __int_as_float(t.z);
                const int nx = inside ? t.x : t.y;
                if (nx < 0) break;
                code = (code << 1) | (inside ? 0u : 1u);
                cur = nx;
                ++lv;
            }
            lock = P.c.auto_min_depth == 0 || warp_key_changes(code << (maxl - lv), valid) < kAutoMaxChanges;
        }

        float best_d = POS_INF, tau = POS_INF;
        unsigned best_i = 0xffffffffu;
        unsigned visits = 0, fetches = 0, steps = 0;
        VHash vh;
        const bool hashing = STATS && P.c.pre;
        if (!lock) {
            int sp = 0;
            int cur = valid ? 0 : TT_END;
            float lb = NEG_INF, sc = 0.f;
            while (cur != TT_END) {
                if (STATS) {
                    ++visits;
                    if (hashing) vh.add(P.c.pre, cur);
                }
                if (!vp_prune(lb, sc, tau)) {
                    int4 t;
                    float v[DIM];
                    ld_node<DIM>(s_rec, s_vpt, g_rec, g_vpt, DP, top, cur, t, v);
                    const float d2 = pinned_d2<DIM>(q, v);
                    if (d2 <= best_d) {
                        const unsigned id = (unsigned)__ldg(P.c.tree.pid + cur);
                        if (d2 < best_d || id < best_i) {
                            best_d = d2;
                            best_i = id;
                            tau = __fsqrt_rn(d2);
                        }
                    }
                    const float d = __fsqrt_rn(d2);
                    const int first_side = d <= __int_as_float(t.z) ? 0 : 1;
                    const int second = first_side ? t.x : t.y;
                    if (second != TT_END) {
                        n_ent[sp * 32 + lane] = (cur << 1) | (first_side ^ 1);
                        if (wide) n_d[sp * 32 + lane] = d;
                        else g_d[(size_t)sp * gstride + gtid] = d;
                        ++sp;
                    }
                    const int first = child_args(t, first_side, d, lb, sc);
                    if (first != TT_END) {
                        cur = first;
                        continue;
                    }
                }
                if (sp > 0) {
                    --sp;
                    const int e = n_ent[sp * 32 + lane];
                    float d;
                    d = wide ? n_d[sp * 32 + lane] : g_d[(size_t)sp * gstride + gtid];
                    cur = child_args(hdr(e >> 1), e & 1, d, lb, sc);
                } else {
                    cur = TT_END;
                }
            }
            if (STATS) {
                fetches = warp_sum(visits);
                steps = __reduce_max_sync(TT_FULL, visits);
            }
        } else {
            int sp = 0;
            int cur = 0;
            unsigned mask = vmask;
            float lb = NEG_INF, sc = 0.f;
            for (;;) {
                const bool in = (mask >> lane) & 1u;
                if (STATS) {
                    ++steps;
                    visits += in;
                    if (hashing) vh.add_if(in, P.c.pre, cur);
                }
                const bool active = in && !vp_prune(lb, sc, tau);
                const unsigned act = __ballot_sync(TT_FULL, active);
                if (act) {
                    if (STATS) ++fetches;
                    int4 t;
                    float v[DIM];
                    ld_node<DIM>(s_rec, s_vpt, g_rec, g_vpt, DP, top, cur, t, v);
                    float d = 0.f;
                    bool pref_in = false;
                    if (active) {
                        const float d2 = pinned_d2<DIM>(q, v);
                        if (d2 <= best_d) {
                            const unsigned id = (unsigned)__ldg(P.c.tree.pid + cur);
                            if (d2 < best_d || id < best_i) {
                                best_d = d2;
                                best_i = id;
                                tau = __fsqrt_rn(d2);
                            }
                        }
                        d = __fsqrt_rn(d2);
                        pref_in = d <= __int_as_float(t.z);
                    }
                    const int votes = __popc(__ballot_sync(TT_FULL, pref_in));
                    const int first_side = 2 * votes >= __popc(act) ? 0 : 1;
                    const int second = first_side ? t.x : t.y;
                    if (second != TT_END) {
                        if (lane == 0)  // warp-uniform part: child|side, its radius, mask
                            l_e[sp] = make_int4((second << 1) | (first_side ^ 1), first_side ? t.z : t.w, (int)act, 0);
                        l_d[sp * 32 + lane] = d;
                        ++sp;
                    }
                    const int first = child_args(t, first_side, d, lb, sc);
                    if (first != TT_END) {
                        cur = first;
                        mask = act;
                        continue;
                    }
                }
                if (sp == 0) break;
                --sp;
                // lane 0 owns the warp-uniform part of the stack; broadcast its pop
                int4 e4 = make_int4(0, 0, 0, 0);
                if (lane == 0) e4 = l_e[sp];
                const int e = __shfl_sync(TT_FULL, e4.x, 0);
                const float r = __int_as_float(__shfl_sync(TT_FULL, e4.y, 0));
                mask = (unsigned)__shfl_sync(TT_FULL, e4.z, 0);
                const float dd = l_d[sp * 32 + lane];
                lb = (e & 1) ? __fsub_rn(r, dd) : __fsub_rn(dd, r);  // as child_args
                sc = __fadd_rn(dd, r);
                cur = e >> 1;
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
int launch(const tt_vp_params &p, const tt_launch_cfg &cfg) {
    constexpr int DP = (DIM + 3) & ~3;
    const int cap = p.c.height + 2;
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * (16 + 4 * DP) +
                        (size_t)kWarps * vp_stack_bytes(cap, p.c.mode == TT_MODE_INDEPENDENT);
    auto kern = vp_kernel<DIM, STATS>;
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
    // AUTO: d of the independent warps' stack entries (see the header comment)
    float *g_d = nullptr;
    const cudaStream_t s = (cudaStream_t)cfg.stream;
    if (p.c.mode == TT_MODE_AUTO) {
        tt_keep_pool_memory();
        e = cudaMallocAsync((void **)&g_d, sizeof(float) * (size_t)cap * (size_t)grid * kBlock, s);
        if (e != cudaSuccess) return (int)e;
    }
    kern<<<(unsigned)grid, kBlock, smem, s>>>(p, cap, g_d);
    e = cudaGetLastError();
    if (g_d) cudaFreeAsync(g_d, s);
    return (int)e;
}

template <int DIM>
int launch_dim(const tt_vp_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    return stats ? launch<DIM, true>(p, cfg) : launch<DIM, false>(p, cfg);
}

}  // namespace

int tt_launch_vp(const tt_vp_params &p, int dim, const tt_launch_cfg &cfg) {
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
