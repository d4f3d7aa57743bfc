// kern_common.cuh -- device helpers shared by the traversal kernels (sm_100a).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "tt_internal.h"

#define TT_FULL 0xffffffffu
#define TT_WARPS_PER_CTA_MAX 32

namespace tt {

// ------------------------------------------------------------------ TMA bulk
// One elected thread stages the top levels of the tree into shared memory with
// cp.async.bulk (SASS UBLKCP) completing on an mbarrier; every thread waits on
// the barrier's phase 0.  Sizes are multiples of 16 B, addresses 16-B aligned
// (blob sections are 256-B aligned).
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, unsigned bytes) {
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst_smem, const void *src_gmem, unsigned bytes, uint64_t *bar) {
    unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    unsigned b = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
        "l"(src_gmem), "r"(bytes), "r"(b)
        : "memory");
}
__device__ __forceinline__ void mbar_wait_phase0(uint64_t *bar) {
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t"
        "@!P1 bra WAIT_%=;\n}" ::"r"(a)
        : "memory");
}

struct StageChunk {
    void *dst;
    const void *src;
    unsigned bytes;
};

// Thread 0 arms the barrier with the total byte count and issues one bulk copy
// per chunk; all threads wait.  Must be called by every thread of the CTA.
template <int NCH>
__device__ __forceinline__ void stage_top(uint64_t *bar, const StageChunk (&ch)[NCH]) {
    unsigned total = 0;
#pragma unroll
    for (int i = 0; i < NCH; ++i) total += ch[i].bytes;
    if (threadIdx.x == 0) {
        mbar_init(bar, 1);
        mbar_arrive_expect_tx(bar, total);
#pragma unroll
        for (int i = 0; i < NCH; ++i)
            if (ch[i].bytes) bulk_g2s(ch[i].dst, ch[i].src, ch[i].bytes, bar);
    }
    __syncthreads();  // barrier initialised before anyone waits on it
    mbar_wait_phase0(bar);
}

// ------------------------------------------------------------ tile scheduler
// Persistent CTAs pull 32-point warp tiles from a global counter (dynamic load
// balance: clustered inputs give uneven traversal lengths).
__device__ __forceinline__ long long next_tile(uint32_t *ctr) {
    unsigned t = 0;
    if ((threadIdx.x & 31) == 0) t = atomicAdd(ctr, 1u);
    return (long long)__shfl_sync(TT_FULL, t, 0);
}

// Last CTA out resets the counters for the next launch on this slot.
__device__ __forceinline__ void cta_finish(uint32_t *ctr) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        unsigned done = atomicAdd(ctr + 1, 1u);
        if (done == gridDim.x - 1) {
            atomicExch(ctr, 0u);
            atomicExch(ctr + 1, 0u);
        }
    }
}

// ------------------------------------------------------ pinned fp32 arithmetic
// DESIGN.md R0: t_d = rn(q_d - p_d), s = rn(t_0 t_0), s = rn(s + rn(t_d t_d)),
// never contracted to FMA.  The independent per-dimension subtractions and
// squares run two at a time on Blackwell's packed FP32x2 pipe (FADD2 / FMUL2:
// sub.rn.f32x2 / mul.rn.f32x2, each lane rounded exactly like the scalar op);
// the sum stays sequential in dimension order.
__device__ __forceinline__ void sub2_rn(float a0, float a1, float b0, float b1, float &r0, float &r1) {
    asm("{\n\t.reg .b64 x, y, z;\n\tmov.b64 x, {%2, %3};\n\tmov.b64 y, {%4, %5};\n\t"
        "sub.rn.f32x2 z, x, y;\n\tmov.b64 {%0, %1}, z;\n\t}"
        : "=f"(r0), "=f"(r1)
        : "f"(a0), "f"(a1), "f"(b0), "f"(b1));
}
__device__ __forceinline__ void sqr2_rn(float a0, float a1, float &r0, float &r1) {
    asm("{\n\t.reg .b64 x, z;\n\tmov.b64 x, {%2, %3};\n\t"
        "mul.rn.f32x2 z, x, x;\n\tmov.b64 {%0, %1}, z;\n\t}"
        : "=f"(r0), "=f"(r1)
        : "f"(a0), "f"(a1));
}

// Packed FP32x2 pair ops on float2: one FADD2 / FMUL2 / FFMA2, each half
// rounded exactly like the scalar op.
__device__ __forceinline__ float2 add2_rn(float2 a, float2 b) {
    float2 r;
    asm("{\n\t.reg .b64 x, y, z;\n\tmov.b64 x, {%2, %3};\n\tmov.b64 y, {%4, %5};\n\t"
        "add.rn.f32x2 z, x, y;\n\tmov.b64 {%0, %1}, z;\n\t}"
        : "=f"(r.x), "=f"(r.y)
        : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
    return r;
}
__device__ __forceinline__ float2 mul2_rn(float2 a, float2 b) {
    float2 r;
    asm("{\n\t.reg .b64 x, y, z;\n\tmov.b64 x, {%2, %3};\n\tmov.b64 y, {%4, %5};\n\t"
        "mul.rn.f32x2 z, x, y;\n\tmov.b64 {%0, %1}, z;\n\t}"
        : "=f"(r.x), "=f"(r.y)
        : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
    return r;
}
__device__ __forceinline__ float2 fma2_rn(float2 a, float2 b, float2 c) {
    float2 r;
    asm("{\n\t.reg .b64 x, y, w, z;\n\tmov.b64 x, {%2, %3};\n\tmov.b64 y, {%4, %5};\n\t"
        "mov.b64 w, {%6, %7};\n\tfma.rn.f32x2 z, x, y, w;\n\tmov.b64 {%0, %1}, z;\n\t}"
        : "=f"(r.x), "=f"(r.y)
        : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(c.x), "f"(c.y));
    return r;
}

// rn(a*a) as fma.rn(a, a, z) with z = -0: exactly rn(a*a) (adding -0 changes
// nothing, +0 stays +0), and an FFMA2 result is never fused into the following
// add.  ptxas fuses mul.rn.f32x2 into a dependent add.rn.f32x2 despite the
// explicit rounding (seen in SASS, also with --fmad=false), and it folds a
// literal -0 addend back into a multiply -- so z must be a value it cannot
// prove is -0: callers pass opaque_neg_zero(), derived from a kernel parameter.
__device__ __forceinline__ float2 sqr2_rn(float2 a, float z) { return fma2_rn(a, a, make_float2(z, z)); }
__device__ __forceinline__ float opaque_neg_zero(long long never_negative) {
    return __int_as_float((int)(0x80000000u | (unsigned)(never_negative < 0)));
}

// max(a, b, c) in one FMNMX3 (sm_100 three-input min/max)
__device__ __forceinline__ float max3(float a, float b, float c) {
    float r;
    asm("max.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
    return r;
}

// per-dimension squared differences rn(rn(q_d - p_d)^2) into sq[]
template <int DIM>
__device__ __forceinline__ void sq_diffs(const float (&q)[DIM], const float *p, float (&sq)[DIM]) {
#pragma unroll
    for (int d = 0; d + 1 < DIM; d += 2) {
        float t0, t1;
        sub2_rn(q[d], q[d + 1], p[d], p[d + 1], t0, t1);
        sqr2_rn(t0, t1, sq[d], sq[d + 1]);
    }
    if (DIM & 1) {
        const float t = __fsub_rn(q[DIM - 1], p[DIM - 1]);
        sq[DIM - 1] = __fmul_rn(t, t);
    }
}

template <int DIM>
__device__ __forceinline__ float pinned_d2(const float (&q)[DIM], const float *p) {
    float sq[DIM];
    sq_diffs<DIM>(q, p, sq);
    float s = sq[0];
#pragma unroll
    for (int d = 1; d < DIM; ++d) s = __fadd_rn(s, sq[d]);
    return s;
}

// Box distance rn(max(lo - q, q - hi, 0))^2 summed in the same order.
template <int DIM>
__device__ __forceinline__ float pinned_boxd2(const float (&q)[DIM], const float *lo, const float *hi) {
    float sq[DIM];
#pragma unroll
    for (int d = 0; d + 1 < DIM; d += 2) {
        float a0, a1, b0, b1;
        sub2_rn(lo[d], lo[d + 1], q[d], q[d + 1], a0, a1);
        sub2_rn(q[d], q[d + 1], hi[d], hi[d + 1], b0, b1);
        sqr2_rn(max3(a0, b0, 0.0f), max3(a1, b1, 0.0f), sq[d], sq[d + 1]);
    }
    if (DIM & 1) {
        const int d = DIM - 1;
        const float t = max3(__fsub_rn(lo[d], q[d]), __fsub_rn(q[d], hi[d]), 0.0f);
        sq[d] = __fmul_rn(t, t);
    }
    float s = sq[0];
#pragma unroll
    for (int d = 1; d < DIM; ++d) s = __fadd_rn(s, sq[d]);
    return s;
}

// Load DIM floats from a 16-B aligned row (padded to a multiple of 4) with
// 128-bit loads.  `GLOBAL_NC` selects ld.global.nc (read-only path).
template <int DIM>
__device__ __forceinline__ void load_row_nc(float (&r)[DIM], const float *p) {
    constexpr int V = (DIM + 3) / 4;
    const float4 *p4 = reinterpret_cast<const float4 *>(p);
#pragma unroll
    for (int v = 0; v < V; ++v) {
        float4 x = __ldg(p4 + v);
        if (4 * v + 0 < DIM) r[4 * v + 0] = x.x;
        if (4 * v + 1 < DIM) r[4 * v + 1] = x.y;
        if (4 * v + 2 < DIM) r[4 * v + 2] = x.z;
        if (4 * v + 3 < DIM) r[4 * v + 3] = x.w;
    }
}
template <int DIM>
__device__ __forceinline__ void load_row_smem(float (&r)[DIM], const float *p) {
    constexpr int V = (DIM + 3) / 4;
    const float4 *p4 = reinterpret_cast<const float4 *>(p);
#pragma unroll
    for (int v = 0; v < V; ++v) {
        float4 x = p4[v];
        if (4 * v + 0 < DIM) r[4 * v + 0] = x.x;
        if (4 * v + 1 < DIM) r[4 * v + 1] = x.y;
        if (4 * v + 2 < DIM) r[4 * v + 2] = x.z;
        if (4 * v + 3 < DIM) r[4 * v + 3] = x.w;
    }
}
// Query rows have an arbitrary leading dimension: scalar loads.
template <int DIM>
__device__ __forceinline__ void load_query(float (&r)[DIM], const float *q, long long row, int ld) {
    const float *p = q + row * (long long)ld;
#pragma unroll
    for (int d = 0; d < DIM; ++d) r[d] = __ldg(p + d);
}

// q[dim] for a runtime dim without dynamic register indexing.
template <int DIM>
__device__ __forceinline__ float select_dim(const float (&q)[DIM], int dim) {
    float v = q[0];
#pragma unroll
    for (int d = 1; d < DIM; ++d) v = (dim == d) ? q[d] : v;
    return v;
}

// ------------------------------------------------ shared-space loads (LDS)
// 32-bit shared-window addresses kept in registers: generic pointers into
// dynamic shared memory make nvcc re-derive the window base (S2R CgaCtaId)
// inside every loop iteration.
__device__ __forceinline__ unsigned smem_addr(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float4 lds_f4(unsigned a) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ int4 lds_i4(unsigned a) {
    int4 v;
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ float lds_f(unsigned a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
// rsqrt without the denormal-input fixup (arguments are >= eps^2 > 0 or
// normal); the result only feeds the force magnitude, not a decision.
__device__ __forceinline__ float rsqrt_ftz(float x) {
    float y;
    asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// One 32-byte node record (one DRAM sector) in a single 256-bit load
// (ld.global.nc.v8, SASS LDG.E.ENL2.256 on sm_100): half the load
// instructions of two 128-bit loads.  p must be 32-B aligned.
__device__ __forceinline__ void ldg_rec256(const void *p, float4 &g, int4 &t) {
    asm("ld.global.nc.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
        : "=f"(g.x), "=f"(g.y), "=f"(g.z), "=f"(g.w), "=r"(t.x), "=r"(t.y), "=r"(t.z), "=r"(t.w)
        : "l"(p));
}

// L1 prefetch of a global line (the next nodes of a walk are known one step
// ahead: both children are in the current record).
__device__ __forceinline__ void prefetch_l1(const void *p) {
    asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}

// ------------------------------------------------------- warp-level helpers
// Number of leading tree levels on which all valid lanes agree, given a path
// code with `bits` bits per level packed in the low `bits*levels` bits.
__device__ __forceinline__ int warp_common_levels(unsigned long long code, unsigned vmask, int bits, int levels) {
    const int leader = __ffs(vmask) - 1;
    unsigned long long lead = __shfl_sync(TT_FULL, code, leader);
    unsigned long long diff = ((vmask >> (threadIdx.x & 31)) & 1u) ? (code ^ lead) : 0ull;
    unsigned hi = __reduce_or_sync(TT_FULL, (unsigned)(diff >> 32));
    unsigned lo = __reduce_or_sync(TT_FULL, (unsigned)diff);
    unsigned long long x = ((unsigned long long)hi << 32) | lo;
    if (x == 0) return levels;
    int lead_zero = __clzll((long long)x) - (64 - bits * levels);
    return lead_zero / bits;
}

// Per-warp coherence for the AUTO mode choice (reading R19): the number of
// launch-order neighbours (lane-1, lane) whose top-level path codes differ.
// A sorted tile is a run of consecutive leaves: a few changes even where it
// straddles a top-level split; an unsorted tile changes at almost every lane.
// (Invalid lanes only occur at the ragged end of the last tile.)
constexpr int kAutoMaxChanges = 8;
__device__ __forceinline__ int warp_key_changes(unsigned long long key, bool valid) {
    const unsigned long long up = __shfl_up_sync(TT_FULL, key, 1);
    return __popc(__ballot_sync(TT_FULL, valid && (threadIdx.x & 31) > 0 && key != up));
}

__device__ __forceinline__ unsigned warp_sum(unsigned v) { return __reduce_add_sync(TT_FULL, v); }

// any stats array requested -> the STATS instantiation
inline bool stats_on(const tt_common_params &c) {
    return c.st_visits || c.st_warp_fetches || c.st_warp_steps || c.st_warp_mode || c.st_hash || c.st_set ||
           c.st_point_tests;
}

// Per-point visit hashes (tt_stats.visit_hash / visit_set): the order hash
// h = h*31 + pre + 1 over the nodes the point tests, in the order it tests
// them (autoropes keep the recursive order, §3.3), and the set
// hash s = sum of mix64(pre + 1) (mix64 = the splitmix64 finaliser), where
// pre is the node's canonical preorder id.  Only the STATS instantiations
// compute them, and only when the caller asked (c.pre != nullptr).
__device__ __forceinline__ unsigned long long vh_mix64(unsigned long long z) {
    z ^= z >> 30;
    z *= 0xbf58476d1ce4e5b9ull;
    z ^= z >> 27;
    z *= 0x94d049bb133111ebull;
    z ^= z >> 31;
    return z;
}
struct VHash {
    unsigned long long h = 0, s = 0;
    __device__ __forceinline__ void add(const int32_t *pre, int node) {
        const unsigned long long v = (unsigned long long)(unsigned)__ldg(pre + node) + 1ull;
        h = h * 31ull + v;
        s += vh_mix64(v);
    }
    __device__ __forceinline__ void add_if(bool on, const int32_t *pre, int node) {
        if (on) add(pre, node);
    }
    // order = false: the walk keeps the visited set but not the order (the
    // order slot is written 0)
    __device__ __forceinline__ void store(const tt_common_params &c, long long pid, bool order = true) const {
        if (c.st_hash) c.st_hash[pid] = order ? h : 0ull;
        if (c.st_set) c.st_set[pid] = s;
    }
};

// Stats writer for the warp tile (lane 0).
__device__ __forceinline__ void write_warp_stats(const tt_common_params &c, long long tile, unsigned fetches,
                                                 unsigned steps, bool lock, bool switched = false) {
    if ((threadIdx.x & 31) == 0) {
        if (c.st_warp_fetches) c.st_warp_fetches[tile] = fetches;
        if (c.st_warp_steps) c.st_warp_steps[tile] = steps;
        if (c.st_warp_mode) c.st_warp_mode[tile] = switched ? 3 : lock ? 1 : 2;
    }
}

}  // namespace tt
