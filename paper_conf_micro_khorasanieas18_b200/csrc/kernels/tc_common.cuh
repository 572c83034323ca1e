// Shared building blocks of the tcgen05 kind::tf32 3xTF32 tiles (vpps_gemm.cu: the level paths' dense
// products; vpps_dwtc.cu: the dataflow path's gathered gradient GEMM).  One 128 x 128 FP32 accumulator in
// TMEM (128 columns) per CTA; K in chunks of 32 through two shared-memory stages, each operand staged by the
// threads through registers, split v = hi + lo (hi = v truncated to TF32, lo = v - hi exact in FP32) and
// stored K-major in the SWIZZLE_NONE canonical layout (core matrix 8 rows x 16 B, SBO 128 B between 8-row
// groups, LBO = 2064 B between 4-k slices: 16 B of padding keep both the 16-byte stores of K-contiguous
// operands and the 4-byte transposing stores of M/N-contiguous ones free of bank conflicts).  One thread issues
// D += A·B + A·B_lo + A_lo·B per k-step of 8 (the dropped A_lo·B_lo is ~2^-22 relative; tools/umma_test.cu
// pins the descriptors) and commits to the stage's mbarrier.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace tcc {
constexpr int BM = 128, BN = 128, BKC = 32, NT = 256;
constexpr uint32_t LBO = (BM / 8) * 128 + 16;                 // bytes between 4-k slices (padded)
constexpr int OP_F = (BKC / 4) * (LBO / 4);                    // floats of one operand copy (hi or lo)
constexpr int STAGE_F = 4 * OP_F;                              // A hi, A lo, B hi, B lo
constexpr size_t SMEM = (size_t)2 * STAGE_F * sizeof(float) + 128;
static_assert(BM == BN, "one staging geometry for both operands");

__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((LBO >> 4) & 0x3FFF) << 16) |
           ((uint64_t)(128 >> 4) << 32) | ((uint64_t)1 << 46);
}
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, int acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                 ::"r"(d), "l"(a), "l"(b), "r"(IDESC), "r"(acc));
}
__device__ __forceinline__ void mbar_wait(uint32_t mbar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(mbar), "r"(parity) : "memory");
}
__device__ __forceinline__ float tf32_hi(float v) { return __uint_as_float(__float_as_uint(v) & 0xFFFFE000u); }

// the register-staged pieces of one operand of a chunk: 4 x 16-byte pieces per thread.  KC (contiguous along
// k): piece g = threadIdx + 256 p covers row g / 8, k = 4 (g % 8) .. +3; otherwise (contiguous along the rows)
// lane = k, the piece covers rows 4 (g / 32) .. +3
__device__ __forceinline__ void piece_rk(bool kc, int p, int& r, int& k) {
    const int g = threadIdx.x + NT * p;
    r = kc ? g / 8 : 4 * (g / 32);
    k = kc ? 4 * (g % 8) : g % 32;
}
// element (r, k) of a stage copy: float offset (k / 4) (LBO / 4) + (r / 8) 32 + (r % 8) 4 + k % 4
template <bool KC>
__device__ __forceinline__ void store_chunk(float* hi, float* lo, const float4 (&v)[4]) {
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        const int g = threadIdx.x + NT * p;
        if (KC) {
            const int r = g / 8, k4 = g % 8;
            const int o = k4 * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4;
            const float4 h = make_float4(tf32_hi(v[p].x), tf32_hi(v[p].y), tf32_hi(v[p].z), tf32_hi(v[p].w));
            *reinterpret_cast<float4*>(hi + o) = h;
            *reinterpret_cast<float4*>(lo + o) = make_float4(v[p].x - h.x, v[p].y - h.y, v[p].z - h.z, v[p].w - h.w);
        } else {
            const int r0 = 4 * (g / 32), k = g % 32;
            const float e[4] = {v[p].x, v[p].y, v[p].z, v[p].w};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int r = r0 + q;
                const int o = (k >> 2) * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4 + (k & 3);
                const float h = tf32_hi(e[q]);
                hi[o] = h;
                lo[o] = e[q] - h;
            }
        }
    }
}


// TMEM allocation (warp 0) and the two stage mbarriers (one thread); call with every thread of the CTA
__device__ __forceinline__ void setup(uint32_t* tmem_base, uint64_t* mbar) {
    const int tid = threadIdx.x;
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base)), "r"(BN));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[0])));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[1])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void teardown(uint32_t tmem) {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(BN));
}
// after every thread stored a stage: make the generic-proxy writes visible to the tensor core and issue the
// chunk's 3 x 4 MMAs (first = the accumulator starts at 0), committing to the stage's mbarrier
__device__ __forceinline__ void issue_chunk(uint32_t tmem, const float* stage, uint64_t* mbar_st, bool first) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x == 0) {
        const uint32_t a0 = smem_u32(stage), al0 = a0 + 4 * OP_F, b0 = al0 + 4 * OP_F, bl0 = b0 + 4 * OP_F;
#pragma unroll
        for (int s = 0; s < BKC / 8; ++s) {
            const uint32_t o = 2 * s * LBO;
            mma(tmem, desc(a0 + o), desc(b0 + o), !first || s > 0);
            mma(tmem, desc(a0 + o), desc(bl0 + o), 1);
            mma(tmem, desc(al0 + o), desc(b0 + o), 1);
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                     ::"r"(smem_u32(mbar_st)) : "memory");
    }
}
// 16 accumulator columns (cb + 16 q ..) of this thread's TMEM lane 32 (warp & 3) + lane, columns half warp >> 2
__device__ __forceinline__ void load16(uint32_t tmem, int col, uint32_t (&r)[16]) {
    const int warp = threadIdx.x >> 5;
    const uint32_t ta = tmem + ((uint32_t)(32 * (warp & 3)) << 16) + col;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(ta));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

}  // namespace tcc
}  // namespace dev
}  // namespace vpps
