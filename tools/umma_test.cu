// Standalone check of the tcgen05 (UMMA) building blocks used by the gradient GEMM: one CTA computes
// D[128 x N] = A[128 x K] B[K x N] with both operands MN-major in shared memory (the natural per-node
// layout of gate gradients and input vectors), SWIZZLE_NONE canonical layout, kind::tf32, accumulator in
// TMEM, as plain TF32 and as 3xTF32 (A·B + A·B_lo + A_lo·B, the split that keeps FP32 accuracy).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/umma tools/umma_test.cu && /tmp/umma
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include <random>
#include <cuda_runtime.h>

constexpr int M = 128, N = 64, K = 24;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// byte offset of element (mn, k) of an MN-major SWIZZLE_NONE operand with MN extent `mn_ext`:
// core matrix = 8 k-rows x 16 B (4 MN elements); SBO = 128 B between MN chunks, LBO = (mn_ext / 4) * 128 B
// between 8-groups of k
__host__ __device__ inline uint32_t mn_off(int mn, int k, int mn_ext) {
    return (uint32_t)((mn >> 2) * 128 + (k >> 3) * (mn_ext / 4) * 128 + (k & 7) * 16 + (mn & 3) * 4);
}

__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;                    // version 1 (Blackwell)
    return d;                                  // base offset 0, lbo mode 0, SWIZZLE_NONE
}

__host__ __device__ constexpr uint32_t make_idesc(int m, int n) {
    return (1u << 4)            // D format F32
         | (2u << 7)            // A format TF32
         | (2u << 10)           // B format TF32
         | (1u << 15)           // A MN-major
         | (1u << 16)           // B MN-major
         | ((uint32_t)(n >> 3) << 17)
         | ((uint32_t)(m >> 4) << 24);
}

__device__ __forceinline__ void mma_tf32(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, int acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
        ::"r"(d_tmem), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

// K-major SWIZZLE_NONE: core matrix = 8 MN-rows x 16 B (4 k), rows 16 B apart; LBO between k-chunks of 4,
// SBO between 8-row groups.  Here: SBO = 128 B, LBO = (mn_ext / 8) * 128 B
__host__ __device__ inline uint32_t k_off(int mn, int k, int mn_ext) {
    return (uint32_t)((mn >> 3) * 128 + (mn & 7) * 16 + (k >> 2) * (mn_ext / 8) * 128 + (k & 3) * 4);
}

__global__ void __launch_bounds__(128, 1) umma_kernel(const float* A, const float* B, float* D, int split) {
    const int mode = split / 10;
    split %= 10;
    __shared__ __align__(128) float As[M * K], Bs[N * K], Al[M * K], Bl[N * K];
    __shared__ __align__(8) uint64_t mbar;
    __shared__ uint32_t tbase;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    // operands: A[k][m], B[k][n] row-major in global (per-node vectors) -> MN-major canonical smem
    for (int i = tid; i < M * K; i += 128) {
        const int k = i / M, m = i % M;
        const float v = A[i];
        const float hi = __uint_as_float(__float_as_uint(v) & 0xFFFFE000u);
        const uint32_t o = mode == 2 ? k_off(m, k, M) : mn_off(m, k, M);
        As[o / 4] = v;
        Al[o / 4] = v - hi;
    }
    for (int i = tid; i < N * K; i += 128) {
        const int k = i / N, n = i % N;
        const float v = B[i];
        const float hi = __uint_as_float(__float_as_uint(v) & 0xFFFFE000u);
        const uint32_t o = mode == 2 ? k_off(n, k, N) : mn_off(n, k, N);
        Bs[o / 4] = v;
        Bl[o / 4] = v - hi;
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tbase)), "r"(64));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic-proxy smem writes -> async proxy
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tbase;
    if (split == 2) {   // TMEM addressing check: st then ld
        uint32_t v = 1000 + warp * 32 + lane;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(tmem + ((uint32_t)(warp * 32) << 16) + 5), "r"(v));
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        uint32_t r;
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(tmem + ((uint32_t)(warp * 32) << 16) + 5));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        D[warp * 32 + lane] = (float)r;
        if (tid == 0) D[200] = (float)tmem;
        __syncthreads();
        if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(64));
        return;
    }
    if (tid == 0) {
        const uint32_t idesc = mode == 2 ? (make_idesc(M, N) & ~((1u << 15) | (1u << 16))) : make_idesc(M, N);
        // per k-step of 8: MN-major advances by one LBO (8 k-rows); K-major by two LBOs (2 chunks of 4 k)
        const uint32_t la = mode == 2 ? (M / 8) * 128 : (M / 4) * 128, lb = mode == 2 ? (N / 8) * 128 : (N / 4) * 128;
        const uint32_t sa = mode == 2 ? 2 * la : la, sb = mode == 2 ? 2 * lb : lb;
        auto dsc = [&](const float* base, int s, uint32_t step, uint32_t l) {
            return mode == 1 ? make_desc(smem_u32(base) + s * step, 128, l) : make_desc(smem_u32(base) + s * step, l, 128);
        };
        for (int s = 0; s < K / 8; ++s) {
            const uint64_t a = dsc(As, s, sa, la), b = dsc(Bs, s, sb, lb);
            mma_tf32(tmem, a, b, idesc, s > 0);
            if (split) {
                const uint64_t al = dsc(Al, s, sa, la), bl = dsc(Bl, s, sb, lb);
                mma_tf32(tmem, a, bl, idesc, 1);
                mma_tf32(tmem, al, b, idesc, 1);
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&mbar)) : "memory");
    }
    {
        uint32_t done = 0;
        while (!done)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                         : "=r"(done) : "r"(smem_u32(&mbar)), "r"(0) : "memory");
    }
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int row = warp * 32 + lane;
    for (int c0 = 0; c0 < N; c0 += 16) {
        uint32_t r[16];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                       "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                     : "r"(tmem + ((uint32_t)(warp * 32) << 16) + c0));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int j = 0; j < 16; ++j) D[row * N + c0 + j] = __uint_as_float(r[j]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(64));
}

int main() {
    std::mt19937 g(1);
    std::uniform_real_distribution<float> u(-1.f, 1.f);
    std::vector<float> A(M * K), B(N * K), D(M * N);
    for (auto& x : A) x = u(g);
    for (auto& x : B) x = u(g);
    float *dA, *dB, *dD;
    cudaMalloc(&dA, A.size() * 4);
    cudaMalloc(&dB, B.size() * 4);
    cudaMalloc(&dD, D.size() * 4);
    cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
    {
        cudaMemset(dD, 0, D.size() * 4);
        umma_kernel<<<1, 128>>>(dA, dB, dD, 2);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
        printf("tmem check (%s): tbase %.0f, lanes 0,1,127 -> %.0f %.0f %.0f\n", cudaGetErrorString(e), D[200], D[0], D[1], D[127]);
    }
    for (int cfg = 0; cfg < 6; ++cfg) {
        const int split = cfg % 2, mode = cfg / 2;
        cudaMemset(dD, 0, D.size() * 4);
        umma_kernel<<<1, 128>>>(dA, dB, dD, mode * 10 + split);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("kernel error: %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
        double maxerr = 0, maxref = 0;
        for (int m = 0; m < M; ++m)
            for (int n = 0; n < N; ++n) {
                double ref = 0;
                for (int k = 0; k < K; ++k) ref += (double)A[k * M + m] * B[k * N + n];
                maxerr = fmax(maxerr, fabs(ref - D[m * N + n]));
                maxref = fmax(maxref, fabs(ref));
            }
        printf("mode %d %s: max |err| / max |ref| = %.3e   (D[0][0] %.6f, D[127][63] %.6f)\n", mode, split ? "3xTF32" : "TF32",
               maxerr / maxref, D[0], D[127 * N + 63]);
    }
    return 0;
}
