// kern_bh.cu -- Barnes-Hut force traversal (Fig.9), sm_100a:
// the per-node lockstep walk over stored ropes (TT_VARIANT_ROPES; round-1
// default).  BH's default path is now kern_bh_group.cu, whose lockstep warps
// expand whole cells per step (-6% at 1M sorted, -23% unsorted).
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
// Each lane therefore tests exactly its own recursive visit sequence: opening
// decisions, per-point visit counts and visit order are identical to the
// independent walk, and so are the results (the fp32 partials are flushed
// into fp64 per body after every kFlush of its own visits, as the
// independent walk does; an inactive step adds an exact +0).
#include <cfloat>
#include <cmath>

#include "kern_common.cuh"

// a negative self id means "no self leaf": -2 matches no record's body field
// (cells carry -1 there)
static __device__ __forceinline__ int tt_self_id(int s) { return s < 0 ? -2 : s; }

namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kSmemHdr = 384;  // [0,16) mbarrier, [16,272) dsq table (64 floats)

// Record fetch through one generic pointer: the staged top levels live in
// shared memory, the rest in global memory (L1/L2-cached); selecting the base
// costs one SEL instead of two predicated load pairs.
__device__ __forceinline__ void ld_rec(const unsigned char *s_base, const unsigned char *g_base, int top, int cur,
                                       float4 &gg, int4 &tt) {
    const unsigned char *p = (cur < top ? s_base : g_base) + (size_t)cur * 32u;
    gg = *reinterpret_cast<const float4 *>(p);
    tt = *reinterpret_cast<const int4 *>(p + 16);
}

// dsq_L = dsq_root * 0.25^L by exponent arithmetic: exact (a power-of-4
// scaling of a normal float), bit-identical to repeated "dsq*0.25" (Fig.9a
// line 4) -- the host checks dsq_root * 0.25^height stays normal, else the
// table path is used (also for theta = 0, dsq_root = +inf: every cell opens).
__device__ __forceinline__ float dsq_at(int dsq_bits, int lvl) { return __int_as_float(dsq_bits - (lvl << 24)); }

// Interaction (update(), Fig.9a line 6): a += m (c - x) / (|c - x|^2 + eps^2)^{3/2}.
// Terms go into fp32 partial sums that are flushed into fp64 every
// kFlush steps: the fp32 partials stay small, so the
// cancellation of a body near the centre of mass costs no accuracy.
constexpr int kFlush = 16;
struct Acc {
    float x = 0.f, y = 0.f, z = 0.f;
    double X = 0.0, Y = 0.0, Z = 0.0;
    __device__ __forceinline__ void add(float m, float dx, float dy, float dz, float drsq, float eps2) {
        const float inv = rsqrt_ftz(__fadd_rn(drsq, eps2));
        const float f = m * (inv * inv) * inv;
        x = fmaf(f, dx, x);
        y = fmaf(f, dy, y);
        z = fmaf(f, dz, z);
    }
    __device__ __forceinline__ void flush() {
        X += (double)x;
        Y += (double)y;
        Z += (double)z;
        x = y = z = 0.f;
    }
};

constexpr int kBPL = TT_BH_POINTS_PER_LANE;  // bodies per lane (2: -4% time vs 1)

struct Body {
    float4 b;
    long long pid;
    int self, wait;
    unsigned visits;
    bool valid;
    Acc acc;
};

// 4 CTAs (32 warps) per SM: <= 64 registers, no spills.  Measured on B200:
// forcing 5 or 6 CTAs (48 / 40 registers, with the fp64 sums moved to shared
// memory to avoid spills) was 2-4% slower -- more warps do not hide the L2
// latency of the dependent record loads better than the lost ILP.
template <bool STATS, bool EXP_DSQ>
__global__ void __launch_bounds__(kBlock, 4) bh_kernel(const tt_bh_params P) {
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
    const float eps2 = P.eps2;
    const unsigned char *s_base = reinterpret_cast<const unsigned char *>(s_top);
    const unsigned char *g_base = reinterpret_cast<const unsigned char *>(g_rec);
    const int dsq_bits = __float_as_int(P.dsq_root);
    auto dsq = [&](int lvl) { return EXP_DSQ ? dsq_at(dsq_bits, lvl) : s_dsq[lvl]; };

    // A warp tile is kBPL*32 consecutive points of the (sorted) order: lane l
    // owns points tile*64 + l and tile*64 + 32 + l.  In lockstep the warp walks
    // the union of all 64 traversals; the per-node fetch / vote / loop cost is
    // shared by two bodies per lane.
    const long long ntiles = (n + 32 * kBPL - 1) / (32 * kBPL);
    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        Body bd[kBPL];
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            const long long pos = tile * 32 * kBPL + 32 * j + lane;
            bd[j].valid = pos < n;
            bd[j].pid = bd[j].valid ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
            bd[j].b = bd[j].valid ? __ldg(P.bodies + bd[j].pid) : make_float4(0.f, 0.f, 0.f, 0.f);
            bd[j].self = bd[j].valid ? (P.self_ids ? tt_self_id(__ldg(P.self_ids + bd[j].pid)) : (int)bd[j].pid) : -2;
            bd[j].wait = bd[j].valid ? INT_MAX : -1;
            bd[j].visits = 0;
        }

        bool lock = P.c.mode != TT_MODE_INDEPENDENT;
        if (P.c.mode == TT_MODE_AUTO && P.c.auto_min_depth > 0) {
            // Coherence of the tile (reading R19): walk its kBPL*32 bodies in
            // launch order and count how often the level-T octree cell changes
            // (T = auto_min_depth, cells from 21-bit fixed-point coordinates in
            // the root cube).  A sorted tile is a Morton-contiguous run: a few
            // changes even where it straddles a cell face; an unsorted tile
            // changes at almost every body.  Lockstep iff fewer than
            // kAutoMaxChanges.  (A common-prefix test sent the few sorted tiles
            // that straddle a top-level face to independent mode, ~2x slower
            // per tile, and those set the kernel's tail.)  A heuristic only:
            // results do not depend on the mode.
            const int T = min(P.c.auto_min_depth, 10);  // (>= 64: never lockstep, below)
            const float lo_x = (float)(P.c.root_center[0] - 0.5 * P.c.root_side);
            const float lo_y = (float)(P.c.root_center[1] - 0.5 * P.c.root_side);
            const float lo_z = (float)(P.c.root_center[2] - 0.5 * P.c.root_side);
            const float sc = (float)((double)(1 << T) / P.c.root_side);
            const int cmax = (1 << T) - 1;
            unsigned cell[kBPL];
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                const unsigned cx = (unsigned)min(max(__float2int_rd((bd[j].b.x - lo_x) * sc), 0), cmax);
                const unsigned cy = (unsigned)min(max(__float2int_rd((bd[j].b.y - lo_y) * sc), 0), cmax);
                const unsigned cz = (unsigned)min(max(__float2int_rd((bd[j].b.z - lo_z) * sc), 0), cmax);
                cell[j] = (cx << (2 * T)) | (cy << T) | cz;
            }
            int changes = 0;
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                // predecessor in launch order: lane-1 of the same row, or the
                // last lane of the previous row
                const unsigned up = __shfl_up_sync(TT_FULL, cell[j], 1);
                const unsigned prev_row = j > 0 ? __shfl_sync(TT_FULL, cell[j > 0 ? j - 1 : 0], 31) : cell[j];
                const unsigned prev = lane > 0 ? up : prev_row;
                changes += __popc(__ballot_sync(TT_FULL, bd[j].valid && cell[j] != prev));
            }
            lock = P.c.auto_min_depth < 64 && changes < kAutoMaxChanges;
        }

        unsigned fetches = 0, steps = 0;
        if (lock) {
            // The warp's two bodies per lane run as one FP32x2 pair: every
            // per-body operation of a step (differences, squares, the pinned
            // sum, the softened inverse cube, the accumulation) is one packed
            // FADD2 / FMUL2 / FFMA2 for both bodies, each half rounded exactly
            // like the scalar op (rn(g - b) = rn(g + (-b)): negation is exact),
            // so results are bit-identical to the scalar form.
            static_assert(kBPL % 2 == 0, "packed lockstep loop is written for body pairs");
            constexpr int NP = kBPL / 2;
            // negated coordinate pairs, formed once per tile: rn(-0 + (-b)) = -b
            // exactly; the opaque -0 addend keeps ptxas from folding this into a
            // negate modifier that re-assembles the pairs every step
            const float nz = opaque_neg_zero(n);  // -0, see sqr2_rn
            const float2 nz2 = make_float2(nz, nz);
            float2 nbx[NP], nby[NP], nbz[NP], ax[NP], ay[NP], az[NP];
            int self[kBPL], w[kBPL];
#pragma unroll
            for (int p = 0; p < NP; ++p) {
                nbx[p] = add2_rn(nz2, make_float2(-bd[2 * p].b.x, -bd[2 * p + 1].b.x));
                nby[p] = add2_rn(nz2, make_float2(-bd[2 * p].b.y, -bd[2 * p + 1].b.y));
                nbz[p] = add2_rn(nz2, make_float2(-bd[2 * p].b.z, -bd[2 * p + 1].b.z));
                ax[p] = ay[p] = az[p] = make_float2(0.f, 0.f);
            }
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                self[j] = bd[j].self;
                w[j] = bd[j].wait;
            }
            int cur = 0;
            // kernel parameters pinned in registers for the hot loop (otherwise
            // re-read from the constant bank every iteration)
            // (through a shuffle: ptxas re-reads plain parameters from the
            // constant bank inside the loop, but cannot rematerialise a SHFL)
            const tt_oct_rec *grec =
                reinterpret_cast<const tt_oct_rec *>(__shfl_sync(TT_FULL, reinterpret_cast<long long>(g_rec), 0));
            const int dbits = __shfl_sync(TT_FULL, dsq_bits, 0);
            const float e2 = __shfl_sync(TT_FULL, eps2, 0);
            const float2 e22 = make_float2(e2, e2);

            // fp32 partials are flushed into fp64 per BODY after every kFlush
            // of its own visits -- the cadence of the independent walk, whose
            // terms are the same ops in the same order (an inactive step adds
            // an exact +0), so L and N results are bit-identical
            unsigned fc[kBPL];
#pragma unroll
            for (int j = 0; j < kBPL; ++j) fc[j] = 0;
            VHash vh[kBPL];
            const bool hashing = STATS && P.c.pre;
#pragma unroll 1
            for (;;) {
                // lockstep: one warp-uniform address, served by L1 (top levels
                // included -- they are also at [0, top) of the global array);
                // measured 2.7% faster than the smem/global select here
                float4 g;
                int4 t;
                ldg_rec256(grec + cur, g, t);
                if (STATS) ++steps;
                const int lvl = t.w;
                const float dl = EXP_DSQ ? dsq_at(dbits, lvl) : s_dsq[lvl];
                const bool cell = t.x >= 0;
                bool any_open = false;
#pragma unroll
                for (int p = 0; p < NP; ++p) {
                    const float2 dx = add2_rn(make_float2(g.x, g.x), nbx[p]);
                    const float2 dy = add2_rn(make_float2(g.y, g.y), nby[p]);
                    const float2 dz = add2_rn(make_float2(g.z, g.z), nbz[p]);
                    // rn(rn(rn(dx^2) + rn(dy^2)) + rn(dz^2)): the pinned order (R0)
                    const float2 drsq = fma2_rn(dz, dz, fma2_rn(dy, dy, sqr2_rn(dx, nz)));  // R8
                    const bool a0 = lvl <= w[2 * p], a1 = lvl <= w[2 * p + 1];
                    const bool o0 = a0 && cell && drsq.x < dl;
                    const bool o1 = a1 && cell && drsq.y < dl;
                    if (STATS) {
                        bd[2 * p].visits += a0;
                        bd[2 * p + 1].visits += a1;
                        if (hashing) {
                            vh[2 * p].add_if(a0, P.c.pre, cur);
                            vh[2 * p + 1].add_if(a1, P.c.pre, cur);
                        }
                    }
                    // active ? (open ? follow : wait at lvl) : keep -- as a min
                    // (an inactive lane has lvl > wait)
                    w[2 * p] = o0 ? INT_MAX : min(w[2 * p], lvl);
                    w[2 * p + 1] = o1 ? INT_MAX : min(w[2 * p + 1], lvl);
                    // branch-free update (some lane almost always interacts)
                    const bool k0 = a0 && !o0 && t.z != self[2 * p];
                    const bool k1 = a1 && !o1 && t.z != self[2 * p + 1];
                    const float2 mw = make_float2(k0 ? g.w : 0.f, k1 ? g.w : 0.f);
                    const float2 r = add2_rn(drsq, e22);
                    const float2 inv = make_float2(rsqrt_ftz(r.x), rsqrt_ftz(r.y));
                    float2 f = mul2_rn(mul2_rn(mw, mul2_rn(inv, inv)), inv);
                    // eps = 0: a skipped term at distance 0 has inv = inf (0 * inf)
                    f = make_float2(k0 ? f.x : 0.f, k1 ? f.y : 0.f);
                    ax[p] = fma2_rn(f, dx, ax[p]);
                    ay[p] = fma2_rn(f, dy, ay[p]);
                    az[p] = fma2_rn(f, dz, az[p]);
                    any_open = any_open || o0 || o1;
                    fc[2 * p] += a0;
                    fc[2 * p + 1] += a1;
                    if (fc[2 * p] == kFlush) {
                        bd[2 * p].acc.X += (double)ax[p].x;
                        bd[2 * p].acc.Y += (double)ay[p].x;
                        bd[2 * p].acc.Z += (double)az[p].x;
                        ax[p].x = ay[p].x = az[p].x = 0.f;
                        fc[2 * p] = 0;
                    }
                    if (fc[2 * p + 1] == kFlush) {
                        bd[2 * p + 1].acc.X += (double)ax[p].y;
                        bd[2 * p + 1].acc.Y += (double)ay[p].y;
                        bd[2 * p + 1].acc.Z += (double)az[p].y;
                        ax[p].y = ay[p].y = az[p].y = 0.f;
                        fc[2 * p + 1] = 0;
                    }
                }
                cur = __any_sync(TT_FULL, any_open) ? t.x : t.y;
                if (cur == TT_END) break;
            }
#pragma unroll
            for (int p = 0; p < NP; ++p) {
                bd[2 * p].acc.X += (double)ax[p].x;
                bd[2 * p].acc.Y += (double)ay[p].x;
                bd[2 * p].acc.Z += (double)az[p].x;
                bd[2 * p + 1].acc.X += (double)ax[p].y;
                bd[2 * p + 1].acc.Y += (double)ay[p].y;
                bd[2 * p + 1].acc.Z += (double)az[p].y;
            }
            if (hashing) {
#pragma unroll
                for (int j = 0; j < kBPL; ++j)
                    if (bd[j].valid) vh[j].store(P.c, bd[j].pid);
            }

            fetches = steps;
        } else {
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                int cur = bd[j].valid ? 0 : TT_END;
                VHash vh;
                while (cur != TT_END) {
#pragma unroll 1
                    for (int k = 0; k < kFlush; ++k) {
                        float4 g;
                        int4 t;
                        ld_rec(s_base, g_base, top, cur, g, t);
                        if (STATS) {
                            ++bd[j].visits;
                            if (P.c.pre) vh.add(P.c.pre, cur);
                        }
                        float dx, dy;
                        sub2_rn(g.x, g.y, bd[j].b.x, bd[j].b.y, dx, dy);
                        const float dz = __fsub_rn(g.z, bd[j].b.z);
                        const float drsq = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));  // R8
                        const bool open = t.x >= 0 && drsq < dsq(t.w);
                        const float inv = rsqrt_ftz(__fadd_rn(drsq, eps2));
                        const float f = (!open && t.z != bd[j].self) ? g.w * (inv * inv) * inv : 0.0f;
                        bd[j].acc.x = fmaf(f, dx, bd[j].acc.x);
                        bd[j].acc.y = fmaf(f, dy, bd[j].acc.y);
                        bd[j].acc.z = fmaf(f, dz, bd[j].acc.z);
                        cur = open ? t.x : t.y;
                        if (cur == TT_END) break;
                    }
                    bd[j].acc.flush();
                }
                if (STATS && P.c.pre && bd[j].valid) vh.store(P.c, bd[j].pid);
            }
            if (STATS) {
                unsigned v = 0, mx = 0;
#pragma unroll
                for (int j = 0; j < kBPL; ++j) {
                    v += bd[j].visits;
                    mx = max(mx, bd[j].visits);
                }
                fetches = warp_sum(v);
                steps = __reduce_max_sync(TT_FULL, mx);
            }
        }
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            if (bd[j].valid) {
                // the body's index is re-read rather than kept live across the walk
                const long long pos = tile * 32 * kBPL + 32 * j + lane;
                bd[j].pid = P.c.order ? (long long)__ldg(P.c.order + pos) : pos;
                P.acc[bd[j].pid] = make_float4((float)bd[j].acc.X, (float)bd[j].acc.Y, (float)bd[j].acc.Z, 0.f);
                if (STATS && P.c.st_visits) P.c.st_visits[bd[j].pid] = bd[j].visits;
            }
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
    }
    cta_finish(P.c.counter);
}

template <bool STATS, bool EXP_DSQ>
int launch(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    const size_t smem = kSmemHdr + (size_t)p.c.top_count * 32;
    auto kern = bh_kernel<STATS, EXP_DSQ>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    int dev = 0, nsm = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, smem);
    if (e != cudaSuccess) return (int)e;
    if (cfg.ctas_per_sm > 0 && cfg.ctas_per_sm < occ) occ = cfg.ctas_per_sm;
    if (occ < 1) occ = 1;
    const long long ntiles = (p.c.n + 32 * kBPL - 1) / (32 * kBPL);
    long long grid = (long long)nsm * occ;
    const long long need = (ntiles + kBlock / 32 - 1) / (kBlock / 32);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, kBlock, smem, (cudaStream_t)cfg.stream>>>(p);
    return (int)cudaGetLastError();
}

}  // namespace

int tt_launch_bh(const tt_bh_params &p, const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    // exponent-arithmetic dsq is exact iff dsq_root * 0.25^height is a normal float
    // (or dsq_root = +inf, theta = 0); otherwise use the shared-memory table
    const float r = p.dsq_root;
    const bool exp_ok = r < INFINITY && r > 0.f && std::ldexp((double)r, -2 * p.c.height) >= (double)FLT_MIN;
    if (stats) return exp_ok ? launch<true, true>(p, cfg) : launch<true, false>(p, cfg);
    return exp_ok ? launch<false, true>(p, cfg) : launch<false, false>(p, cfg);
}
