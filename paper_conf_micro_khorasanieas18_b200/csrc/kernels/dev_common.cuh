// Device helpers shared by the VPPS kernels (sm_100a).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace vpps {
namespace dev {
constexpr uint32_t FULLMASK = 0xFFFFFFFFu;

__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + expf(-x)); }
// Latency-short forms for the critical path of the dataflow / leaf kernels: MUFU.EX2-based exp and the
// approximate divide (a few ulp; the parity bar is 1e-4 relative, SURVEY R-22).  tanh x = 1 - 2/(1+e^{2x})
// saturates correctly at both ends (e^{2x} -> inf gives 1, -> 0 gives -1).
__device__ __forceinline__ float fsigm(float x) { return __fdividef(1.0f, 1.0f + __expf(-x)); }
__device__ __forceinline__ float ftanh(float x) { return 1.0f - __fdividef(2.0f, 1.0f + __expf(2.0f * x)); }
__device__ __forceinline__ float4 ld4cg(const float* p) { return __ldcg(reinterpret_cast<const float4*>(p)); }
__device__ __forceinline__ float4 f4zero() { return make_float4(0.f, 0.f, 0.f, 0.f); }


// Vectorised no-return float add in L2 (REDG.E.ADD.F32x4 on sm_90+): remote accumulation of the
// transposed matrix-vector product (fn4 L100).  The data is only read after a barrier.
template <int CG>
__device__ __forceinline__ void red_add(float* p, const float* v) {
    if constexpr (CG == 4) {
        asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v[0]), "f"(v[1]), "f"(v[2]),
                     "f"(v[3]));
    } else if constexpr (CG == 2) {
        asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" ::"l"(p), "f"(v[0]), "f"(v[1]));
    } else {
        atomicAdd(p, v[0]);
    }
}

template <int CG>
__device__ __forceinline__ void lds(const float* p, float* v) {
    if constexpr (CG == 4) {
        const float4 t = *reinterpret_cast<const float4*>(p);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    } else if constexpr (CG == 2) {
        const float2 t = *reinterpret_cast<const float2*>(p);
        v[0] = t.x; v[1] = t.y;
    } else {
        v[0] = *p;
    }
}

template <int CG>
__device__ __forceinline__ void sts_granule(float* p, const float (&v)[CG], bool keep) {
    if constexpr (CG == 4) {
        *reinterpret_cast<float4*>(p) = keep ? make_float4(v[0], v[1], v[2], v[3]) : f4zero();
    } else if constexpr (CG == 2) {
        *reinterpret_cast<float2*>(p) = keep ? make_float2(v[0], v[1]) : make_float2(0.f, 0.f);
    } else {
        *p = keep ? v[0] : 0.f;
    }
}


template <int CG, int NREG>
__device__ __forceinline__ void dot_acc(const float (&w)[NREG], int t, const float (&y)[CG], float2& a) {
    if constexpr (CG >= 2) {
#pragma unroll
        for (int q = 0; q < CG; q += 2)
            a = __ffma2_rn(make_float2(w[t * CG + q], w[t * CG + q + 1]), make_float2(y[q], y[q + 1]), a);
    } else {
        a.x = fmaf(w[t], y[0], a.x);
    }
}


__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
    for (int s = 16; s >= 1; s >>= 1) v += __shfl_xor_sync(FULLMASK, v, s);
    return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
    for (int s = 16; s >= 1; s >>= 1) v = fmaxf(v, __shfl_xor_sync(FULLMASK, v, s));
    return v;
}

// ---- asynchronous global -> shared copies (cp.async / LDGSTS): no registers, zero fill when
//      src_bytes < size ----
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cp_async16(void* dst, const void* src, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(void* dst, const void* src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Register layout of a K-long weight row over TU threads: CG-wide column granules, NT granules per thread.
template <int K, int TU>
struct Lay {
    static constexpr int CG = (K >= 4 * TU) ? 4 : ((K >= 2 * TU) ? 2 : 1);
    static constexpr int NT = (K + CG * TU - 1) / (CG * TU);
    static constexpr int NREG = NT * CG;
    static constexpr int KP = NT * CG * TU;
};

// Sum over a 16-lane group of four per-lane values (one per node): transposed halving at distances 8
// and 4, then a butterfly over the low two bits.  Lane l ends with node 2*bit3(l) + bit2(l).
__device__ __forceinline__ float treduce4_16(float v0, float v1, float v2, float v3, int lane) {
    const bool b3 = lane & 8, b2 = lane & 4;
    const float s0 = b3 ? v0 : v2, s1 = b3 ? v1 : v3;
    float k0 = b3 ? v2 : v0, k1 = b3 ? v3 : v1;
    k0 += __shfl_xor_sync(FULLMASK, s0, 8);
    k1 += __shfl_xor_sync(FULLMASK, s1, 8);
    const float s = b2 ? k0 : k1;
    float k = b2 ? k1 : k0;
    k += __shfl_xor_sync(FULLMASK, s, 4);
    k += __shfl_xor_sync(FULLMASK, k, 2);
    k += __shfl_xor_sync(FULLMASK, k, 1);
    return k;
}

__device__ __forceinline__ uint64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}


}  // namespace dev
}  // namespace vpps
