// kern_bh_group.cu -- Barnes-Hut lockstep walk by child groups
// (TT_VARIANT_GROUPS), sm_100a.
//
// The lockstep walk of kern_bh.cu makes one dependent L2 round trip per node
// (next = first child or rope of the record just loaded), and that latency is
// what binds it (0.58 of a pure pointer chase).  Here the warp
// expands a whole cell at once: when any of its bodies opens a cell, the
// cell's children -- stored contiguously in a group array built once per tree
// from the preorder blob -- are loaded together (independent loads, one round
// trip) and every active body tests each of them.  A child some body opens is
// pushed with the ballot of the bodies that opened it (Fig.8's per-entry
// mask, here one mask per body row of the 64-body tile).  Every body tests
// exactly the nodes its recursive walk tests (the children of the cells it
// opens), so per-body visit counts equal the oracle's and the warp fetches
// equal the Fig.8 union; only the order in which a body's terms are summed
// differs (within the 1e-4 bar: fp32 partials flushed to fp64).
//
// Group record (32 B, like tt_oct_rec): {com.xyz, mass} +
// {group offset of the node's children | -1, number of children, body | -1,
// level << 24 for a cell, kLeafLevel for a leaf}; entry 0 is the root, the
// children of a cell are contiguous.  kLeafLevel makes a leaf's opening
// distance negative (exponent path: dsq_bits - 0x7fffffff is a negative
// float for every finite dsq_root > 0; table path: entry 127 is -1), so
// `drsq < dl` alone is the opening test -- no separate "is a cell" compare.
#include <climits>
#include <cfloat>
#include <cmath>

#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <type_traits>
#include <unordered_map>
#include <vector>

#include "kern_common.cuh"
#include "tt_check.cuh"

// a negative self id means "no self leaf": -2 matches no record's body field
// (cells carry -1 there)
static __device__ __forceinline__ int tt_self_id(int s) { return s < 0 ? -2 : s; }


namespace {

using namespace tt;

constexpr int kBlock = 256;
constexpr int kSmemHdr = 640;          // mbarrier + dsq table of 128 levels (>= 64: leaves, -1)
constexpr int kLeafLevel = 0x7fffffff; // level field of a leaf group record
constexpr int kBPL = TT_BH_POINTS_PER_LANE;
constexpr int kStackPerWarp = 8 * 40;  // <= 8 children pushed per level, height <= 33 (R9) + slack
constexpr int kStackSmall = 8 * 24;    // height <= 22: the 1M / 16M configs (heights 18-20)
constexpr int kFlushEvery = 16;        // independent walk: steps between fp32 -> fp64 flushes
constexpr int kFlushEveryL = 32;       // lockstep group walk: >= children between flushes

struct GroupEntry {
    int off, nk;
    unsigned m0, m1;  // bodies (row 0 / row 1 of the tile) that opened the cell
};

// ------------------------------------------------------------ group build
__global__ void nkids_kernel(const tt_oct_rec *rec, long long nn, int *nk) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x) {
        int c = rec[v].first_child, k = 0;
        const int end = rec[v].skip;
        while (c >= 0 && c != end) {
            ++k;
            c = rec[c].skip;
        }
        nk[v] = k;
    }
}

__global__ void groups_fill_kernel(const tt_oct_rec *rec, long long nn, const int *nk, const int *goff,
                                   tt_oct_rec *grp, int *leaf_of, long long np, int *gsrc) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nn; v += (long long)gridDim.x * blockDim.x) {
        if (v == 0) {  // the root's own entry
            tt_oct_rec r = rec[0];
            r.first_child = nk[0] > 0 ? 1 + goff[0] : -1;
            r.skip = nk[0];
            r.level = r.first_child < 0 ? kLeafLevel : r.level << 24;
            grp[0] = r;
            gsrc[0] = 0;
            if (r.first_child < 0 && r.body >= 0 && r.body < np) leaf_of[r.body] = 0;
        }
        int c = rec[v].first_child, k = 0;
        const int end = rec[v].skip;
        while (c >= 0 && c != end) {
            tt_oct_rec r = rec[c];
            r.first_child = nk[c] > 0 ? 1 + goff[c] : -1;
            r.skip = nk[c];
            // the exponent step of dsq_L (level * 2^24): one IADD per child
            r.level = r.first_child < 0 ? kLeafLevel : r.level << 24;
            grp[1 + goff[v] + k] = r;
            gsrc[1 + goff[v] + k] = c;  // the device node (stats hashes map it to its preorder id)
            if (r.first_child < 0 && r.body >= 0 && r.body < np) leaf_of[r.body] = 1 + goff[v] + k;
            ++k;
            c = rec[c].skip;
        }
    }
}

__device__ __forceinline__ float dsq_at(int dsq_bits, int lvl) { return __int_as_float(dsq_bits - (lvl << 24)); }

#ifndef TT_BHG_MINB
#define TT_BHG_MINB 4
#endif
// WIDE: some node has more than 8 children (a depth-32 bucket of more than 8
// coincident bodies, R9, or a custom tree): groups are staged 8 at a time.
// Shared memory: header (mbarrier, dsq table) | per-warp group stacks of
// stk_cap entries (8 per level: sized by the tree height) | per-warp staging
// buffers (8 32-B records) | the first n_top group records -- the root's and
// the top levels' child groups, which every tile walks -- staged once per
// CTA by one bulk copy (TMA, UBLKCP) on an mbarrier (shallow
// data in fast shared memory).  A group lying inside the staged prefix is
// read in place; any other is staged from global memory by the warp.
template <bool STATS, bool EXP_DSQ, bool WIDE, int STK>
__global__ void __launch_bounds__(kBlock, TT_BHG_MINB) bh_group_kernel(const tt_bh_params P, const tt_oct_rec *grp,
                                                                                 const int *leaf_of, long long np,
                                                                                 const int *gsrc, int n_top,
                                                                                 long long n_groups) {
    constexpr int stk_cap = STK;  // compile-time stack stride
    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    float *s_dsq = reinterpret_cast<float *>(smem + 16);
    GroupEntry *s_stack = reinterpret_cast<GroupEntry *>(smem + kSmemHdr);
    float4 *s_stage = reinterpret_cast<float4 *>(s_stack + (kBlock / 32) * stk_cap);
    double *s_accb = reinterpret_cast<double *>(s_stage + (kBlock / 32) * 16);  // [6][kBlock]
    float4 *s_top = reinterpret_cast<float4 *>(s_accb + 6 * kBlock);
    if (threadIdx.x == 0) {
        float d = P.dsq_root;
        for (int l = 0; l < 64; ++l) {
            s_dsq[l] = d;
            d = __fmul_rn(d, 0.25f);
        }
        for (int l = 64; l < 128; ++l) s_dsq[l] = -1.f;  // kLeafLevel >> 24 = 127
    }
    StageChunk ch[1] = {{s_top, grp, (unsigned)n_top * 32u}};
    stage_top(bar, ch);

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    GroupEntry *stk = s_stack + warp * stk_cap;
    // per-warp staging buffer of one child group (<= 8 32-B records {g, t});
    // 32-bit shared addresses (no generic-address rebuild in the loop)
    // (warp-uniform by construction; the shuffles let the compiler keep them
    // in uniform registers, off the 64-register budget)
    const unsigned gbuf_a = __shfl_sync(TT_FULL, smem_addr(s_stage + warp * 16), 0);
    const unsigned top_a = smem_addr(s_top);
    const unsigned gbuf_l = gbuf_a + 32u * (unsigned)lane;  // this lane's staging slot
    const unsigned lbit = 1u << lane;
    const tt_oct_rec *g_rec = static_cast<const tt_oct_rec *>(P.c.tree.rec);
    const long long n = P.c.n;
    const int dsq_bits = __float_as_int(P.dsq_root);
    const float nz = opaque_neg_zero(n);
    const float2 e22 = make_float2(P.eps2, P.eps2);
    const long long ntiles = (n + 32 * kBPL - 1) / (32 * kBPL);
    for (;;) {
        const long long tile = next_tile(P.c.counter);
        if (tile >= ntiles) break;
        long long pid[kBPL];
        float4 b[kBPL];
        int self[kBPL];
        bool valid[kBPL];
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            const long long pos = tile * 32 * kBPL + 32 * j + lane;
            valid[j] = pos < n;
            pid[j] = valid[j] ? (P.c.order ? (long long)P.c.order[pos] : pos) : 0;
            b[j] = valid[j] ? __ldg(P.bodies + pid[j]) : make_float4(0.f, 0.f, 0.f, 0.f);
            self[j] = valid[j] ? (P.self_ids ? tt_self_id(__ldg(P.self_ids + pid[j])) : (int)pid[j]) : -2;
        }
        bool lock = P.c.mode != TT_MODE_INDEPENDENT;
        if (P.c.mode == TT_MODE_AUTO && P.c.auto_min_depth > 0) {
            // the coherence test of kern_bh.cu (reading R19)
            const int T = min(P.c.auto_min_depth, 10);
            const float lo_x = (float)(P.c.root_center[0] - 0.5 * P.c.root_side);
            const float lo_y = (float)(P.c.root_center[1] - 0.5 * P.c.root_side);
            const float lo_z = (float)(P.c.root_center[2] - 0.5 * P.c.root_side);
            const float sc = (float)((double)(1 << T) / P.c.root_side);
            const int cmax = (1 << T) - 1;
            unsigned cell[kBPL];
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                const unsigned cx = (unsigned)min(max(__float2int_rd((b[j].x - lo_x) * sc), 0), cmax);
                const unsigned cy = (unsigned)min(max(__float2int_rd((b[j].y - lo_y) * sc), 0), cmax);
                const unsigned cz = (unsigned)min(max(__float2int_rd((b[j].z - lo_z) * sc), 0), cmax);
                cell[j] = (cx << (2 * T)) | (cy << T) | cz;
            }
            int changes = 0;
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                const unsigned up = __shfl_up_sync(TT_FULL, cell[j], 1);
                const unsigned prev_row = j > 0 ? __shfl_sync(TT_FULL, cell[j > 0 ? j - 1 : 0], 31) : cell[j];
                const unsigned prev = lane > 0 ? up : prev_row;
                changes += __popc(__ballot_sync(TT_FULL, valid[j] && cell[j] != prev));
            }
            lock = P.c.auto_min_depth < 64 && changes < kAutoMaxChanges;
        }

        double X[kBPL], Y[kBPL], Z[kBPL];
        unsigned visits[kBPL];
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            X[j] = Y[j] = Z[j] = 0.0;
            visits[j] = 0;
        }
        unsigned fetches = 0, steps = 0;
        VHash vh[kBPL];
        const bool hashing = STATS && P.c.pre;
        // The self test (skip the leaf holding the body itself) only
        // matters where that leaf's term is not exactly zero: a leaf at
        // the body's own position contributes f * 0 = 0 whenever f is
        // finite (eps > 0).  A warp whose bodies all sit exactly on their
        // own leaves (the normal case: the tree was built from them)
        // walks without the per-child test; others keep it.
        // (eps = 0: every warp keeps the checked walk, whose select also
        // zeroes opened cells at distance 0 -- 0 * inf otherwise)
        const bool eps_ok = isfinite(rsqrt_ftz(__fadd_rn(0.f, P.eps2)));
        bool ok[kBPL];
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            ok[j] = !valid[j] || self[j] < 0 || (long long)self[j] >= np;
            if (!ok[j]) {
                const int lf = __ldg(leaf_of + self[j]);
                TT_DCHECK(lf < n_groups);
                if (lf < 0) {
                    ok[j] = true;  // no leaf is tested against this id
                } else {
                    const float4 c = __ldg(reinterpret_cast<const float4 *>(grp + lf));
                    const float inv = rsqrt_ftz(__fadd_rn(0.f, P.eps2));
                    const float f = __fmul_rn(__fmul_rn(c.w, __fmul_rn(inv, inv)), inv);
                    ok[j] = c.x == b[j].x && c.y == b[j].y && c.z == b[j].z && isfinite(f);
                }
            }
            ok[j] = ok[j] && eps_ok;
        }
        const bool need_self = __any_sync(TT_FULL, !(ok[0] && ok[1]));
        if (lock) {
            static_assert(kBPL == 2, "group walk is written for body pairs");
            const float2 nbx = add2_rn(make_float2(nz, nz), make_float2(-b[0].x, -b[1].x));
            const float2 nby = add2_rn(make_float2(nz, nz), make_float2(-b[0].y, -b[1].y));
            const float2 nbz = add2_rn(make_float2(nz, nz), make_float2(-b[0].z, -b[1].z));
            float2 ax = make_float2(0.f, 0.f), ay = ax, az = ax;
            int since_flush = 0;
            int sp = 0;
            // the fp64 sums of the walk live in shared memory (this thread's
            // column of s_acc[6][kBlock]): 12 registers fewer in the loop;
            // a flush (every >= kFlushEveryL children) is 6 read-add-writes
            double *s_acc = s_accb + threadIdx.x;
#pragma unroll
            for (int c = 0; c < 6; ++c) s_acc[c * kBlock] = 0.0;
            auto flush_s = [&]() {
                s_acc[0 * kBlock] += (double)ax.x;
                s_acc[1 * kBlock] += (double)ay.x;
                s_acc[2 * kBlock] += (double)az.x;
                s_acc[3 * kBlock] += (double)ax.y;
                s_acc[4 * kBlock] += (double)ay.y;
                s_acc[5 * kBlock] += (double)az.y;
            };
            // the root group: entry 0 alone, tested by every valid body
            int goff = 0, gnk = 1;
            unsigned m0 = __ballot_sync(TT_FULL, valid[0]), m1 = __ballot_sync(TT_FULL, valid[1]);
            auto walk = [&](auto self_chk) {
                constexpr bool SELF = decltype(self_chk)::value;
                for (;;) {
                    const bool in0 = (m0 & lbit) != 0u, in1 = (m1 & lbit) != 0u;
                    // the group's mask as the addend of the first square: +0 for
                    // a body in the mask (fma(dx, dx, +0) = rn(dx^2), R8's value),
                    // +inf outside it -- its |dr|^2 is then +inf, so it never
                    // opens a child (no mask predicate per child) and its r is
                    // +inf, inv = 0, f = 0 exactly
                    const float2 zm = make_float2(in0 ? 0.f : __int_as_float(0x7f800000),
                                                  in1 ? 0.f : __int_as_float(0x7f800000));
                    // stage the group: lane k loads child k (one request for the
                    // whole group, one round trip), the warp reads them back from
                    // shared memory with broadcast loads; the buffer holds 8
                    // records, so a WIDE tree stages larger groups 8 at a time
                    const int gall = gnk;
                    for (int c0 = 0;; c0 += 8) {
                    const int cn = WIDE ? min(gall - c0, 8) : gall;
                    TT_DCHECK(cn >= 1 && cn <= 8 && goff >= 0 && goff + c0 + cn <= n_groups);
                    // a group of the staged top levels is read in place
                    const bool staged = goff + c0 + cn <= n_top;
                    if (!staged) {
                        // lanes below cn: one 256-bit load, two 128-bit stores
                        // (predicated, no divergent branch).  32-bit record index:
                        // the launcher keeps groups to trees of < 2^27 nodes, so
                        // index * 32 B fits 32 bits
                        const unsigned gi = (unsigned)(goff + c0 + lane);
                        asm volatile(
                            "{\n\t.reg .pred p;\n\t.reg .b32 a<8>;\n\t"
                            "setp.lt.s32 p, %0, %1;\n\t"
                            "@p ld.global.nc.v8.b32 {a0, a1, a2, a3, a4, a5, a6, a7}, [%2];\n\t"
                            "@p st.shared.v4.b32 [%3], {a0, a1, a2, a3};\n\t"
                            "@p st.shared.v4.b32 [%3+16], {a4, a5, a6, a7};\n\t}"
                            :: "r"(lane), "r"(cn), "l"(reinterpret_cast<const char *>(grp) + gi * 32u), "r"(gbuf_l)
                            : "memory");
                        __syncwarp();
                    }
                    const unsigned rb = staged ? top_a + 32u * (unsigned)(goff + c0) : gbuf_a;
                    auto child = [&](unsigned a, int k) {
                        const float4 g = lds_f4(a);
                        const int4 t = lds_i4(a + 16u);
                        if (STATS) {
                            ++fetches;
                            ++steps;
                            visits[0] += in0;
                            visits[1] += in1;
                            if (hashing && (in0 || in1)) {
                                // the visited SET only: a body's tests are in DFS-over-
                                // groups order, not the recursive order (reading R23)
                                const unsigned long long m = vh_mix64(
                                    (unsigned long long)(unsigned)__ldg(P.c.pre + __ldg(gsrc + goff + c0 + k)) + 1ull);
                                if (in0) vh[0].s += m;
                                if (in1) vh[1].s += m;
                            }
                        }
                        // a leaf's dl is negative (kLeafLevel): drsq < dl is the whole test
                        const float dl = EXP_DSQ ? __int_as_float(dsq_bits - t.w) : s_dsq[t.w >> 24];
                        const float2 dx = add2_rn(make_float2(g.x, g.x), nbx);
                        const float2 dy = add2_rn(make_float2(g.y, g.y), nby);
                        const float2 dz = add2_rn(make_float2(g.z, g.z), nbz);
                        // |dr|^2 = fma(dz, dz, fma(dy, dy, dx * dx)) (R8), 3 instructions
                        // (masked: +inf for a body outside the group's mask)
                        const float2 drsq = fma2_rn(dz, dz, fma2_rn(dy, dy, SELF ? sqr2_rn(dx, nz) : fma2_rn(dx, dx, zm)));
                        const bool o0 = (!SELF || in0) && drsq.x < dl;
                        const bool o1 = (!SELF || in1) && drsq.y < dl;
                        float2 f;
                        if (SELF) {
                            const bool k0 = in0 && !o0 && t.z != self[0];
                            const bool k1 = in1 && !o1 && t.z != self[1];
                            const float2 mw = make_float2(k0 ? g.w : 0.f, k1 ? g.w : 0.f);
                            const float2 r = add2_rn(drsq, e22);
                            const float2 inv = make_float2(rsqrt_ftz(r.x), rsqrt_ftz(r.y));
                            f = mul2_rn(mul2_rn(mw, mul2_rn(inv, inv)), inv);
                            // the checked walk also serves eps = 0, where a skipped
                            // leaf at distance 0 has inv = inf (0 * inf): select
                            f = make_float2(k0 ? f.x : 0.f, k1 ? f.y : 0.f);
                        } else {
                            // a body outside the group's mask has r = inf, so inv = 0
                            // and f = 0 exactly (eps > 0 here: active inv is finite)
                            const float2 mw = make_float2(o0 ? 0.f : g.w, o1 ? 0.f : g.w);
                            const float2 r = add2_rn(drsq, e22);
                            const float2 inv = make_float2(rsqrt_ftz(r.x), rsqrt_ftz(r.y));
                            f = mul2_rn(mul2_rn(mw, mul2_rn(inv, inv)), inv);
                        }
                        ax = fma2_rn(f, dx, ax);
                        ay = fma2_rn(f, dy, ay);
                        az = fma2_rn(f, dz, az);
                        // one vote per child; the two ballots only when some body
                        // opens it (one vote: -1.5% vs two ballots per child)
                        if (__any_sync(TT_FULL, o0 || o1)) {
                            const unsigned om0 = __ballot_sync(TT_FULL, o0), om1 = __ballot_sync(TT_FULL, o1);
                            TT_DCHECK(sp < stk_cap && t.x >= 1 && t.y >= 1);
                            if (lane == 0) stk[sp] = GroupEntry{t.x, t.y, om0, om1};
                            ++sp;
                        }
                    };
                    // straight-line: enter the unrolled sequence of 8 at 8 - cn
                    // (one indirect jump per group, no per-child loop control;
                    // pushes stay in child order).  3.18 vs 3.20 ms for a loop
                    // of two children per trip, 3.32 for one.
                    {
                        const unsigned rb8 = rb - 32u * (unsigned)(8 - cn);
                        switch (8 - cn) {
                        case 0: child(rb8 + 0u, cn - 8); [[fallthrough]];
                        case 1: child(rb8 + 32u, cn - 7); [[fallthrough]];
                        case 2: child(rb8 + 64u, cn - 6); [[fallthrough]];
                        case 3: child(rb8 + 96u, cn - 5); [[fallthrough]];
                        case 4: child(rb8 + 128u, cn - 4); [[fallthrough]];
                        case 5: child(rb8 + 160u, cn - 3); [[fallthrough]];
                        case 6: child(rb8 + 192u, cn - 2); [[fallthrough]];
                        default: child(rb8 + 224u, cn - 1);
                        }
                    }
                    __syncwarp();  // the group buffer is reused by the next chunk / pop
                    if (!WIDE || c0 + 8 >= gall) break;
                    }
                    since_flush += gall;
                    if (since_flush >= kFlushEveryL) {  // warp-uniform cadence
                        flush_s();
                        ax = ay = az = make_float2(0.f, 0.f);
                        since_flush = 0;
                    }
                    if (sp == 0) break;
                    --sp;
                    __syncwarp();
                    // every lane reads the entry lane 0 pushed (one broadcast load);
                    // the group's offset and size pass through a shuffle so the
                    // compiler sees them warp-uniform (uniform loop control)
                    // (a plain C++ load: ordered after lane 0's plain-store push
                    // and the __syncwarp, which an asm load without a memory
                    // clobber is not)
                    const int4 e = *reinterpret_cast<const int4 *>(stk + sp);
                    goff = __shfl_sync(TT_FULL, e.x, 0);
                    gnk = __shfl_sync(TT_FULL, e.y, 0);
                    TT_DCHECK(sp >= 0 && gnk >= 1 && (WIDE || gnk <= 8) && goff >= 1 && goff + gnk <= n_groups &&
                              __shfl_sync(TT_FULL, e.z, 0) == e.z && __shfl_sync(TT_FULL, e.w, 0) == e.w);
                    m0 = (unsigned)e.z;
                    m1 = (unsigned)e.w;
                }
            };
            if (need_self) walk(std::true_type{});
            else walk(std::false_type{});
            flush_s();
            X[0] = s_acc[0 * kBlock];
            Y[0] = s_acc[1 * kBlock];
            Z[0] = s_acc[2 * kBlock];
            X[1] = s_acc[3 * kBlock];
            Y[1] = s_acc[4 * kBlock];
            Z[1] = s_acc[5 * kBlock];
        } else {
            // independent: the stackless rope walk of kern_bh.cu over the
            // preorder records (through L1/L2)
#pragma unroll
            for (int j = 0; j < kBPL; ++j) {
                int cur = valid[j] ? 0 : TT_END;
                float sx = 0.f, sy = 0.f, sz = 0.f;
                int cnt = 0;
                while (cur != TT_END) {
                    float4 g;
                    int4 t;
                    TT_DCHECK(cur >= 0 && cur < n_groups);
                    ldg_rec256(g_rec + cur, g, t);
                    if (STATS) {
                        ++visits[j];
                        if (hashing) vh[j].add(P.c.pre, cur);
                    }
                    const float dx = __fsub_rn(g.x, b[j].x), dy = __fsub_rn(g.y, b[j].y),
                                dz = __fsub_rn(g.z, b[j].z);
                    const float drsq = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));  // R8
                    const float dl = EXP_DSQ ? dsq_at(dsq_bits, t.w) : s_dsq[t.w];
                    const bool open = t.x >= 0 && drsq < dl;
                    const float inv = rsqrt_ftz(__fadd_rn(drsq, P.eps2));
                    const float f = (!open && t.z != self[j]) ? g.w * (inv * inv) * inv : 0.0f;
                    sx = fmaf(f, dx, sx);
                    sy = fmaf(f, dy, sy);
                    sz = fmaf(f, dz, sz);
                    if (++cnt == kFlushEvery) {
                        X[j] += (double)sx;
                        Y[j] += (double)sy;
                        Z[j] += (double)sz;
                        sx = sy = sz = 0.f;
                        cnt = 0;
                    }
                    cur = open ? t.x : t.y;
                }
                X[j] += (double)sx;
                Y[j] += (double)sy;
                Z[j] += (double)sz;
            }
            if (STATS) {
                fetches = warp_sum(visits[0] + visits[1]);
                steps = __reduce_max_sync(TT_FULL, max(visits[0], visits[1]));
            }
        }
#pragma unroll
        for (int j = 0; j < kBPL; ++j) {
            if (valid[j]) {
                P.acc[pid[j]] = make_float4((float)X[j], (float)Y[j], (float)Z[j], 0.f);
                if (STATS && P.c.st_visits) P.c.st_visits[pid[j]] = visits[j];
                if (hashing) vh[j].store(P.c, pid[j], !lock);  // lockstep: set only
            }
        }
        if (STATS) write_warp_stats(P.c, tile, fetches, steps, lock);
        __syncwarp();
    }
    cta_finish(P.c.counter);
}

template <bool STATS, bool EXP_DSQ, bool WIDE, bool BIG_STK>
int launch(const tt_bh_params &p, const tt_oct_rec *grp, const int *leaf_of, long long np, const int *gsrc,
           long long n_groups, const tt_launch_cfg &cfg) {
    // group stacks sized by the height: at most 8 cell children pushed per
    // level of the current path (oct_flags TT_OCT_FEW_CELL_KIDS)
    // (two compile-time sizes: 192 entries -- height <= 22, every config --
    // or the 33-level maximum)
    constexpr int STK = BIG_STK ? kStackPerWarp : kStackSmall;
    const int stk_cap = STK;
    const size_t base = kSmemHdr + (size_t)(kBlock / 32) * stk_cap * sizeof(GroupEntry) + (kBlock / 32) * 16 * 16 +
                        6 * kBlock * sizeof(double);
    // the staged top-level groups get what is left of the shared memory of
    // TT_BHG_MINB CTAs per SM (TT_STAGE_BYTES overrides: tuning sweeps)
    int dev = 0, nsm = 0, smem_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    long long budget = (long long)smem_sm / TT_BHG_MINB - 1024 - (long long)base;  // 1 KB reserved per CTA
    if (const char *ev = std::getenv("TT_STAGE_BYTES")) budget = std::atoll(ev);
    long long n_top = std::max(0LL, std::min(n_groups, budget / 32));
    const size_t smem = base + (size_t)n_top * 32;
    auto kern = bh_group_kernel<STATS, EXP_DSQ, WIDE, STK>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, smem);
    if (e != cudaSuccess) return (int)e;
    if (cfg.ctas_per_sm > 0 && cfg.ctas_per_sm < occ) occ = cfg.ctas_per_sm;
    if (occ < 1) occ = 1;
    const long long ntiles = (p.c.n + 32 * kBPL - 1) / (32 * kBPL);
    long long grid = (long long)nsm * occ;
    const long long need = (ntiles + kBlock / 32 - 1) / (kBlock / 32);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, kBlock, smem, (cudaStream_t)cfg.stream>>>(p, grp, leaf_of, np, gsrc, (int)n_top, n_groups);
    return (int)cudaGetLastError();
}

// Group arrays are recycled between trees: BH time stepping builds a tree,
// and so a group array, every step, and a fresh cudaMalloc per step costs
// milliseconds (pool allocations were fragmented by the sort's scratch).
// tt_tree_free returns the array here only after a successful device
// synchronisation, so a recycled array is never still in use; arrays are
// handed out again only on the device they were allocated on.
struct GrpInfo {
    size_t bytes;
    int device;
};
std::mutex g_grp_mu;
std::unordered_map<void *, GrpInfo> g_grp_info;  // every group array alive or free
std::vector<void *> g_grp_free;

void *grp_take(size_t bytes) {
    int dev = -1;
    cudaGetDevice(&dev);
    {
        std::lock_guard<std::mutex> lk(g_grp_mu);
        for (size_t i = 0; i < g_grp_free.size(); ++i) {
            void *p = g_grp_free[i];
            const GrpInfo &gi = g_grp_info[p];
            if (gi.device == dev && gi.bytes >= bytes && gi.bytes <= 2 * bytes) {
                g_grp_free.erase(g_grp_free.begin() + (long)i);
                return p;
            }
        }
    }
    // slack (1/8, in 2-MiB steps): the next time step's tree is a little
    // larger or smaller and should still fit [bytes, 2 * bytes]
    const size_t alloc = ((bytes + bytes / 8) + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
    void *p = nullptr;
    if (cudaMalloc(&p, alloc) != cudaSuccess) return nullptr;
    std::lock_guard<std::mutex> lk(g_grp_mu);
    g_grp_info[p] = GrpInfo{alloc, dev};
    return p;
}

}  // namespace

void tt_bh_groups_discard(void *grp) {
    if (!grp) return;
    {
        std::lock_guard<std::mutex> lk(g_grp_mu);
        g_grp_info.erase(grp);
    }
    cudaFree(grp);
}

void tt_bh_groups_release(void *grp) {
    if (!grp) return;
    std::lock_guard<std::mutex> lk(g_grp_mu);
    if (g_grp_free.size() >= 4) {  // keep a few
        g_grp_info.erase(grp);
        cudaFree(grp);
        return;
    }
    g_grp_free.push_back(grp);
}

// Child-group array of an oct tree (built once per tree, kept with it).
int tt_bh_groups_build(const void *rec, long long nn, long long np, void *stream, void **grp_out) {
    cudaStream_t s = (cudaStream_t)stream;
    const tt_oct_rec *r = static_cast<const tt_oct_rec *>(rec);
    int *nk = nullptr, *goff = nullptr;
    void *tmp = nullptr, *grp = nullptr;
    size_t tb = 0;
    cudaError_t e = cudaMallocAsync((void **)&nk, sizeof(int) * nn, s);
    if (!e) e = cudaMallocAsync((void **)&goff, sizeof(int) * nn, s);
    if (!e) e = cub::DeviceScan::ExclusiveSum(nullptr, tb, nk, goff, (int)nn, s);
    if (!e) e = cudaMallocAsync(&tmp, tb, s);
    if (!e) {
        // records, then leaf_of[np]: the group index of the leaf whose body
        // is each id (-1 for ids no leaf names first), then gsrc[nn]: the
        // device node of each group entry
        grp = grp_take(sizeof(tt_oct_rec) * (size_t)nn + sizeof(int) * (size_t)np + sizeof(int) * (size_t)nn);
        if (!grp) e = cudaErrorMemoryAllocation;
    }
    int *leaf_of = grp ? reinterpret_cast<int *>(static_cast<tt_oct_rec *>(grp) + nn) : nullptr;
    if (!e && np > 0) e = cudaMemsetAsync(leaf_of, 0xff, sizeof(int) * (size_t)np, s);
    const unsigned G = (unsigned)std::min<long long>((nn + 255) / 256, 148 * 8);
    if (!e) {
        nkids_kernel<<<G, 256, 0, s>>>(r, nn, nk);
        e = cub::DeviceScan::ExclusiveSum(tmp, tb, nk, goff, (int)nn, s);
    }
    if (!e) {
        groups_fill_kernel<<<G, 256, 0, s>>>(r, nn, nk, goff, static_cast<tt_oct_rec *>(grp), leaf_of, np,
                                             leaf_of + np);
        e = cudaGetLastError();
    }
    if (tmp) cudaFreeAsync(tmp, s);
    if (goff) cudaFreeAsync(goff, s);
    if (nk) cudaFreeAsync(nk, s);
    if (e) {
        if (grp) {
            cudaStreamSynchronize(s);
            tt_bh_groups_discard(grp);
        }
        return (int)e;
    }
    *grp_out = grp;
    return 0;
}

int tt_launch_bh_group(const tt_bh_params &p, const void *grp, long long nn, long long np, bool wide,
                       const tt_launch_cfg &cfg) {
    const bool stats = stats_on(p.c);
    const float r = p.dsq_root;
    const bool exp_ok = r < INFINITY && r > 0.f && std::ldexp((double)r, -2 * p.c.height) >= (double)FLT_MIN;
    const tt_oct_rec *g = static_cast<const tt_oct_rec *>(grp);
    const int *lf = reinterpret_cast<const int *>(g + nn);
    const int *gs = lf + np;
    const bool big = 8 * (p.c.height + 2) > kStackSmall;
    if (wide) {  // rare (buckets of > 8 coincident bodies): no specialisations beyond stats
        if (stats) return launch<true, false, true, true>(p, g, lf, np, gs, nn, cfg);
        return launch<false, false, true, true>(p, g, lf, np, gs, nn, cfg);
    }
    if (big) {
        if (stats) return launch<true, false, false, true>(p, g, lf, np, gs, nn, cfg);
        return launch<false, false, false, true>(p, g, lf, np, gs, nn, cfg);
    }
    if (stats) return exp_ok ? launch<true, true, false, false>(p, g, lf, np, gs, nn, cfg)
                             : launch<true, false, false, false>(p, g, lf, np, gs, nn, cfg);
    return exp_ok ? launch<false, true, false, false>(p, g, lf, np, gs, nn, cfg)
                  : launch<false, false, false, false>(p, g, lf, np, gs, nn, cfg);
}
