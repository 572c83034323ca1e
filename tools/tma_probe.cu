// Standalone check of the TMA-fed tcgen05 kind::tf32 building blocks for the leaf GEMM: one CTA computes
// D[128 leaves x 48 rows] = X[tok] · W[rows]ᵀ over K = 256 with
//   * the leaf rows gathered by token with cp.async.bulk.tensor.2d ... tile::gather4 (4 rows per copy),
//   * the W_iou rows as 2D TMA tiles (3 gates x 16 rows),
// both landing K-major in the SWIZZLE_128B layout (8-row x 128-byte atoms, SBO = 1024 B), UMMA descriptors
// advanced by 32 B per k-step of 8.  The TF32 operands are the raw FP32 tiles (the tensor core reads the
// top 19 bits); mode 1 adds A·B_lo + A_lo·B with lo = v - trunc_tf32(v), mode 2 with lo = v - rna_tf32(v).
// Prints the max relative error of each mode against an FP64 product (pins the hardware's TF32 conversion).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe tools/tma_probe.cu && /tmp/tma_probe
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include <random>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

constexpr int V = 4096, E = 256, H = 256, TL = 128, TR = 48, KC = 32;
constexpr int A_B = TL * KC * 4, B_B = TR * KC * 4;          // bytes of one raw chunk

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(TR >> 3) << 17) | ((uint32_t)(TL >> 4) << 24);
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

__global__ void __launch_bounds__(256, 1) probe(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmW,
                                                const int* tok, int j0, int mode, float* D) {
    extern __shared__ __align__(1024) uint8_t dsm[];
    uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(dsm) + 1023) & ~uintptr_t(1023));
    uint8_t* Ar = sm;                    // raw A chunk (16 KB), lo A (16 KB), raw B (6 KB), lo B (6 KB)
    uint8_t* Al = sm + A_B;
    uint8_t* Br = sm + 2 * A_B;
    uint8_t* Bl = sm + 2 * A_B + B_B;
    __shared__ __align__(8) uint64_t full, mdone;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(64));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full)));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mdone)));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmW)) : "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base;
    for (int c = 0; c < E / KC; ++c) {
        if (tid == 0) {
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full)), "r"(A_B + B_B) : "memory");
            for (int q = 0; q < TL / 4; ++q)
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                             " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                             ::"r"(smem_u32(Ar + q * 512)), "l"(reinterpret_cast<uint64_t>(&tmX)), "r"(c * KC),
                               "r"(tok[4 * q]), "r"(tok[4 * q + 1]), "r"(tok[4 * q + 2]), "r"(tok[4 * q + 3]),
                               "r"(smem_u32(&full)) : "memory");
            for (int g = 0; g < 3; ++g)
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                             " [%0], [%1, {%2, %3}], [%4];"
                             ::"r"(smem_u32(Br + g * 16 * 128)), "l"(reinterpret_cast<uint64_t>(&tmW)), "r"(c * KC),
                               "r"(g * H + j0), "r"(smem_u32(&full)) : "memory");
        }
        mbar_wait(smem_u32(&full), c & 1);
        // lo copies, element by element at the same offsets (the swizzle is a permutation of whole 16-byte
        // pieces, so an elementwise map keeps the layout)
        for (int i = tid; i < (A_B + B_B) / 16; i += 256) {
            const bool isA = i < A_B / 16;
            const float4 v = *reinterpret_cast<const float4*>((isA ? Ar : Br) + (isA ? i : i - A_B / 16) * 16);
            float e[4] = {v.x, v.y, v.z, v.w}, l[4];
            for (int k = 0; k < 4; ++k) {
                float hv;
                if (mode == 2) {
                    uint32_t r;
                    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(e[k]));
                    hv = __uint_as_float(r);
                } else {
                    hv = __uint_as_float(__float_as_uint(e[k]) & 0xFFFFE000u);
                }
                l[k] = e[k] - hv;
            }
            *reinterpret_cast<float4*>((isA ? Al : Bl) + (isA ? i : i - A_B / 16) * 16) = make_float4(l[0], l[1], l[2], l[3]);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (tid == 0) {
            for (int s = 0; s < KC / 8; ++s) {
                const uint32_t o = 32 * s;
                mma(tmem, desc_sw128(smem_u32(Ar) + o), desc_sw128(smem_u32(Br) + o), c > 0 || s > 0);
                if (mode) {
                    mma(tmem, desc_sw128(smem_u32(Ar) + o), desc_sw128(smem_u32(Bl) + o), 1);
                    mma(tmem, desc_sw128(smem_u32(Al) + o), desc_sw128(smem_u32(Br) + o), 1);
                }
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mdone)) : "memory");
        }
        mbar_wait(smem_u32(&mdone), c & 1);      // (probe: no overlap; the buffers are reused next chunk)
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    }
    if (warp < 4) {
        const int lane = tid & 31, row = 32 * warp + lane;
        for (int q = 0; q < 3; ++q) {
            uint32_t r[16];
            const uint32_t ta = tmem + ((uint32_t)(32 * warp) << 16) + 16 * q;
            asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                           "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                         : "r"(ta));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            for (int k = 0; k < 16; ++k) D[row * TR + 16 * q + k] = __uint_as_float(r[k]);
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(64));
}


// MMA throughput: `reps` MMAs of M = 128, N = n (K-major SWIZZLE_128B operands already in smem, contents
// irrelevant), issued back to back by one thread and committed once; cycles per MMA
template <int NN>
__global__ void __launch_bounds__(128, 1) mma_rate(int reps, long long* out) {
    extern __shared__ __align__(1024) uint8_t dsm[];
    uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(dsm) + 1023) & ~uintptr_t(1023));
    __shared__ __align__(8) uint64_t mdone;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x;
    for (int i = tid; i < (128 + NN) * 32; i += 128) reinterpret_cast<float*>(sm)[i] = 0.001f * (i % 97);
    if (tid < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(NN < 32 ? 32 : NN));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mdone)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (tid == 0) {
        constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NN >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
        const uint32_t a = smem_u32(sm), b = a + 128 * 128;
        const long long t0 = clock64();
        for (int r = 0; r < reps; ++r) {
            const uint32_t o = 32 * (r & 3);
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                         "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                         ::"r"(tmem_base), "l"(desc_sw128(a + o)), "l"(desc_sw128(b + o)), "r"(idesc), "r"(r > 0 ? 1 : 0));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mdone)) : "memory");
        const long long t1 = clock64();
        mbar_wait(smem_u32(&mdone), 0);
        const long long t2 = clock64();
        out[0] = t1 - t0; out[1] = t2 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(NN < 32 ? 32 : NN));
}

template <int NN>
static void rate(int reps) {
    long long* o;
    cudaMallocManaged(&o, 16);
    const size_t smem = (128 + NN) * 128 + 1024;
    cudaFuncSetAttribute(mma_rate<NN>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    mma_rate<NN><<<1, 128, smem>>>(reps, o);     // warm
    cudaDeviceSynchronize();
    mma_rate<NN><<<1, 128, smem>>>(reps, o);
    cudaError_t e = cudaDeviceSynchronize();
    printf("M=128 N=%3d K=8 tf32 x %d: issue %lld cycles, complete %lld cycles -> %.1f cycles/MMA, %.0f MAC/clk (%s)\n",
           NN, reps, o[0], o[1], (double)o[1] / reps, 128.0 * NN * 8 * reps / o[1], cudaGetErrorString(e));
    cudaFree(o);
}

// MN-major operand check: D[128 x 128] = Aᵀᵀ B with A stored transposed (At [K][M], M contiguous) loaded as
// SWIZZLE_128B MN-major atoms (32 M x 8 K, 1 KB) by 2D TMA boxes {32 M, 32 K}, and B [N][K] K-major
// (boxes {32 K, 128 N}).  UMMA: A MN-major (idesc bit 15), LBO = 4 KB between M atoms, SBO = 1 KB between
// K atoms, +1 KB per k-step of 8; B K-major as above.  Plain TF32 (relative error ~1e-4 expected).
__global__ void __launch_bounds__(128, 1) mn_probe(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                                                   int K, uint32_t lbo, uint32_t sbo, float* D) {
    extern __shared__ __align__(1024) uint8_t dsm[];
    uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(dsm) + 1023) & ~uintptr_t(1023));
    uint8_t* As = sm;              // 4 boxes x 4 KB
    uint8_t* Bs = sm + 16384;      // 16 KB
    __shared__ __align__(8) uint64_t full, mdone;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(128));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full)));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mdone)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base;
    constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    for (int c = 0; c < K / 32; ++c) {
        if (tid == 0) {
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full)), "r"(32768) : "memory");
            for (int i = 0; i < 4; ++i)
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                             ::"r"(smem_u32(As + 4096 * i)), "l"(reinterpret_cast<uint64_t>(&tmA)), "r"(32 * i), "r"(32 * c),
                               "r"(smem_u32(&full)) : "memory");
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         ::"r"(smem_u32(Bs)), "l"(reinterpret_cast<uint64_t>(&tmB)), "r"(32 * c), "r"(0), "r"(smem_u32(&full)) : "memory");
        }
        mbar_wait(smem_u32(&full), c & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (tid == 0) {
            for (int s = 0; s < 4; ++s) {
                const uint32_t a = smem_u32(As) + sbo * s;
                const uint64_t ad = (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
                                    ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                             "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                             ::"r"(tmem), "l"(ad), "l"(desc_sw128(smem_u32(Bs) + 32 * s)), "r"(idesc), "r"((c > 0 || s > 0) ? 1 : 0));
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mdone)) : "memory");
        }
        mbar_wait(smem_u32(&mdone), c & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        __syncthreads();
    }
    const int lane = tid & 31, row = 32 * warp + lane;
    for (int q = 0; q < 8; ++q) {
        uint32_t r[16];
        const uint32_t ta = tmem + ((uint32_t)(32 * warp) << 16) + 16 * q;
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                       "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                     : "r"(ta));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int k = 0; k < 16; ++k) D[row * 128 + 16 * q + k] = __uint_as_float(r[k]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(128));
}

static void mn_check(PFN_cuTensorMapEncodeTiled_v12000 enc) {
    const int M = 128, N = 128, K = 96;
    std::mt19937 rng(11);
    std::uniform_real_distribution<float> U(-1.f, 1.f);
    std::vector<float> At(K * M), B(N * K), D(M * N);
    for (auto& v : At) v = U(rng);
    for (auto& v : B) v = U(rng);
    float *dA, *dB, *dD;
    cudaMalloc(&dA, At.size() * 4); cudaMalloc(&dB, B.size() * 4); cudaMalloc(&dD, D.size() * 4);
    cudaMemcpy(dA, At.data(), At.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
    CUtensorMap ta, tb;
    cuuint64_t gda[2] = {(cuuint64_t)M, (cuuint64_t)K}, gsa[1] = {(cuuint64_t)M * 4};
    cuuint32_t ba[2] = {32, 32}, es[2] = {1, 1};
    enc(&ta, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dA, gda, gsa, ba, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cuuint64_t gdb[2] = {(cuuint64_t)K, (cuuint64_t)N}, gsb[1] = {(cuuint64_t)K * 4};
    cuuint32_t bb[2] = {32, 128};
    enc(&tb, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dB, gdb, gsb, bb, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    const size_t smem = 32768 + 1024;
    cudaFuncSetAttribute(mn_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const uint32_t cand[][2] = {{4096, 1024}, {1024, 4096}, {16, 1024}, {4096, 16}};
    for (auto& cd : cand) {
        cudaMemset(dD, 0, D.size() * 4);
        mn_probe<<<1, 128, smem>>>(ta, tb, K, cd[0], cd[1], dD);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
        double mx = 0;
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < N; ++n) {
                double sref = 0, sa = 0;
                for (int k = 0; k < K; ++k) { sref += (double)At[k * M + m] * B[n * K + k]; sa += fabs((double)At[k * M + m] * B[n * K + k]); }
                mx = std::max(mx, fabs(D[m * N + n] - sref) / sa);
            }
        printf("MN-major A (LBO %u, SBO %u): %s, max |err| / sum|terms| = %.3g\n", cd[0], cd[1], cudaGetErrorString(e), mx);
    }
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
}

int main() {
    std::mt19937 rng(7);
    std::uniform_real_distribution<float> U(-1.f, 1.f);
    std::vector<float> X(V * E), W(3 * H * E);
    for (auto& v : X) v = U(rng);
    for (auto& v : W) v = U(rng) * 0.1f;
    std::vector<int> tok(TL);
    for (auto& t : tok) t = rng() % V;
    float *dX, *dW, *dD;
    int* dtok;
    cudaMalloc(&dX, X.size() * 4); cudaMalloc(&dW, W.size() * 4); cudaMalloc(&dD, TL * TR * 4); cudaMalloc(&dtok, TL * 4);
    cudaMemcpy(dX, X.data(), X.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dW, W.data(), W.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dtok, tok.data(), TL * 4, cudaMemcpyHostToDevice);
    auto enc = get_encode();
    if (!enc) { printf("no cuTensorMapEncodeTiled\n"); return 1; }
    CUtensorMap tmX, tmW;
    cuuint64_t gdx[2] = {(cuuint64_t)E, (cuuint64_t)V}, gsx[1] = {(cuuint64_t)E * 4};
    cuuint32_t bx[2] = {KC, 1}, es[2] = {1, 1};
    CUresult r1 = enc(&tmX, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dX, gdx, gsx, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cuuint64_t gdw[2] = {(cuuint64_t)E, (cuuint64_t)(3 * H)}, gsw[1] = {(cuuint64_t)E * 4};
    cuuint32_t bw[2] = {KC, 16};
    CUresult r2 = enc(&tmW, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dW, gdw, gsw, bw, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode: X %d W %d\n", (int)r1, (int)r2);
    const int j0 = 80;
    const size_t smem = 2 * A_B + 2 * B_B + 1024;
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int* htok = tok.data();
    for (int mode = 0; mode < 3; ++mode) {
        // the kernel reads tok[] on the host side of the launch: pass the device copy's values via a kernel copy
        std::vector<float> Dh(TL * TR);
        int* tokd;
        cudaMallocManaged(&tokd, TL * 4);
        for (int i = 0; i < TL; ++i) tokd[i] = htok[i];
        probe<<<1, 256, smem>>>(tmX, tmW, tokd, j0, mode, dD);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(Dh.data(), dD, TL * TR * 4, cudaMemcpyDeviceToHost);
        double maxrel = 0, maxabs = 0, ref_scale = 0;
        for (int l = 0; l < TL; ++l)
            for (int r = 0; r < TR; ++r) {
                const int row = (r / 16) * H + j0 + r % 16;
                double s = 0, sa = 0;
                for (int k = 0; k < E; ++k) { s += (double)X[tok[l] * E + k] * W[row * E + k]; sa += fabs((double)X[tok[l] * E + k] * W[row * E + k]); }
                const double d = fabs(Dh[l * TR + r] - s);
                maxabs = std::max(maxabs, d);
                maxrel = std::max(maxrel, d / sa);
                ref_scale = std::max(ref_scale, fabs(s));
            }
        printf("mode %d (%s): err %s, max |err| / sum|terms| = %.3g, max |err| = %.3g (max |D| %.3g)\n", mode,
               mode == 0 ? "raw TF32" : (mode == 1 ? "3xTF32, lo = v - trunc(v)" : "3xTF32, lo = v - rna(v)"),
               cudaGetErrorString(e), maxrel, maxabs, ref_scale);
        cudaFree(tokd);
    }
    for (int reps : {12, 96, 384}) { rate<48>(reps); rate<128>(reps); rate<256>(reps); }
    mn_check(enc);
    return 0;
}
