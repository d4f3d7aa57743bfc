// kern_integrate.cu -- kick-drift update of a Barnes-Hut time step (SURVEY
// NEXT-4: "build -> COM -> force pass -> leapfrog", the paper's BH input "ran
// ... for five timesteps").  v += a * dt_kick; x += v * dt_drift, in
// fp32 (explicit _rn: no contraction), mass untouched.  A leapfrog (KDK) step
// is kick(dt/2) [+ drift(dt)] before the force pass and kick(dt/2) after; the
// driver merges consecutive half kicks.
#include "kern_common.cuh"

namespace {
__global__ void kick_drift_kernel(float4 *x, float4 *v, const float4 *a, long long n, float dtk, float dtd) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        float4 p = x[i], u = v[i];
        const float4 g = a[i];
        u.x = __fadd_rn(u.x, __fmul_rn(g.x, dtk));
        u.y = __fadd_rn(u.y, __fmul_rn(g.y, dtk));
        u.z = __fadd_rn(u.z, __fmul_rn(g.z, dtk));
        p.x = __fadd_rn(p.x, __fmul_rn(u.x, dtd));
        p.y = __fadd_rn(p.y, __fmul_rn(u.y, dtd));
        p.z = __fadd_rn(p.z, __fmul_rn(u.z, dtd));
        v[i] = u;
        x[i] = p;
    }
}

// Gathering form for the sharded time step: lane j updates
// source row perm[j] and writes it to output row j, so a rank's shard of the
// sorted order comes out contiguous (ready for one all-gather) and the bodies
// travel in the order of the last point sort.  Same arithmetic as above.
__global__ void kick_drift_perm_kernel(const float4 *x, const float4 *v, const float4 *a, const int *perm,
                                       const int *ids, long long n, float dtk, float dtd, float4 *xo, float4 *vo,
                                       int *ido) {
    for (long long j = blockIdx.x * (long long)blockDim.x + threadIdx.x; j < n; j += (long long)gridDim.x * blockDim.x) {
        const int i = __ldg(perm + j);
        float4 p = __ldg(x + i), u = __ldg(v + i);
        const float4 g = __ldg(a + i);
        u.x = __fadd_rn(u.x, __fmul_rn(g.x, dtk));
        u.y = __fadd_rn(u.y, __fmul_rn(g.y, dtk));
        u.z = __fadd_rn(u.z, __fmul_rn(g.z, dtk));
        p.x = __fadd_rn(p.x, __fmul_rn(u.x, dtd));
        p.y = __fadd_rn(p.y, __fmul_rn(u.y, dtd));
        p.z = __fadd_rn(p.z, __fmul_rn(u.z, dtd));
        vo[j] = u;
        xo[j] = p;
        if (ids) ido[j] = __ldg(ids + i);
    }
}
}  // namespace

int tt_launch_kick_drift_permuted(const float *x, const float *v, const float *a, const int *perm, const int *ids,
                                  long long n, float dtk, float dtd, float *xo, float *vo, int *ido, void *stream) {
    long long g = (n + 255) / 256;
    if (g > 148 * 8) g = 148 * 8;
    kick_drift_perm_kernel<<<(unsigned)(g < 1 ? 1 : g), 256, 0, (cudaStream_t)stream>>>(
        reinterpret_cast<const float4 *>(x), reinterpret_cast<const float4 *>(v), reinterpret_cast<const float4 *>(a),
        perm, ids, n, dtk, dtd, reinterpret_cast<float4 *>(xo), reinterpret_cast<float4 *>(vo), ido);
    return (int)cudaGetLastError();
}

int tt_launch_kick_drift(float *x, float *v, const float *a, long long n, float dtk, float dtd, void *stream) {
    long long g = (n + 255) / 256;
    if (g > 148 * 8) g = 148 * 8;
    kick_drift_kernel<<<(unsigned)(g < 1 ? 1 : g), 256, 0, (cudaStream_t)stream>>>(
        reinterpret_cast<float4 *>(x), reinterpret_cast<float4 *>(v), reinterpret_cast<const float4 *>(a), n, dtk,
        dtd);
    return (int)cudaGetLastError();
}
