// DSMEM push throughput at the volumes of a VPPS level (B200, 16-CTA clusters):
// st.async v4 (h all-gather: 16 nodes x 16 peers x 64 B per CTA), plain remote v4 stores + fence,
// remote f32 reductions.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/cmb3.bin tools/cluster_mb3.cu && ./tools/cmb3.bin
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void arrive_rel() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void wait_acq() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ uint32_t rank() { uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ uint32_t smaddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
    uint32_t d; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(r)); return d;
}
__device__ __forceinline__ void st_async(uint32_t a, float4 v, uint32_t mbar) {
    asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1,%2,%3,%4}, [%5];"
                 :: "r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "r"(mbar) : "memory");
}
__device__ __forceinline__ void st_dsm(uint32_t a, float4 v) {
    asm volatile("st.shared::cluster.v4.f32 [%0], {%1,%2,%3,%4};" :: "r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ void red_dsm(uint32_t a, float v) {
    asm volatile("red.shared::cluster.add.f32 [%0], %1;" :: "r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void mbar_init(uint32_t m, uint32_t n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(m), "r"(n) : "memory"); }
__device__ __forceinline__ void mbar_expect(uint32_t m, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(m), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t m, uint32_t parity) {
    asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}"
                 :: "r"(m), "r"(parity) : "memory");
}

template <int PER>   // st.async v4 per thread per round
__device__ long long push_round(float* sm, uint64_t* mbar, uint32_t rk, int reps, int tid) {
    arrive_rel(); wait_acq();
    const long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        const int b = r & 1;
        const uint32_t mb_local = smaddr(&mbar[b]);
        if (tid == 0) mbar_expect(mb_local, 256 * PER * 16);
#pragma unroll
        for (int k = 0; k < PER; ++k) {
            const int e = tid + k * 256;                    // e: (node n = e / 64, peer = (e / 4) % 16, piece = e % 4)
            const uint32_t peer = (e >> 2) & 15, n = e >> 6;
            const uint32_t dst = mapa(smaddr(sm + b * 16384 + n * 256 + rk * 16 + (e & 3) * 4), peer);
            st_async(dst, make_float4(r, rk, n, 3), mapa(mb_local, peer));
        }
        mbar_wait(mb_local, (uint32_t)((r >> 1) & 1));
    }
    return (clock64() - t0) / reps;
}

__global__ void __launch_bounds__(256, 1) mb(long long* out, int reps) {
    extern __shared__ __align__(16) float sm[];
    __shared__ __align__(8) uint64_t mbar[2];
    const int tid = threadIdx.x;
    const uint32_t rk = rank();
    for (int i = tid; i < 40960; i += 256) sm[i] = 0.f;
    if (tid == 0) { mbar_init(smaddr(&mbar[0]), 1); mbar_init(smaddr(&mbar[1]), 1); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    arrive_rel(); wait_acq();
    long long res[8];
    res[0] = push_round<1>(sm, mbar, rk, reps, tid);     //  256 x 16 B (4 nodes)
    res[1] = push_round<4>(sm, mbar, rk, reps, tid);     // 1024 x 16 B (16 nodes)
    res[2] = push_round<8>(sm, mbar, rk, reps, tid);     // 2048 x 16 B (32 nodes)
    // plain remote v4 stores (4 per thread) + release cluster barrier
    arrive_rel(); wait_acq();
    long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const int e = tid + k * 256;
            const uint32_t peer = (e >> 2) & 15, n = e >> 6;
            st_dsm(mapa(smaddr(sm + 32768 + n * 256 + rk * 16 + (e & 3) * 4), peer), make_float4(r, rk, n, 3));
        }
        arrive_rel(); wait_acq();
    }
    res[3] = (clock64() - t0) / reps;
    // remote f32 reductions: 2 per thread (512 per CTA, the transposed product of one node) + release barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const int e = tid + k * 256, peer = e >> 5;
            red_dsm(mapa(smaddr(sm + 36864 + (e & 31) + 32 * (rk & 1)), peer), 1.f);
        }
        arrive_rel(); wait_acq();
    }
    res[4] = (clock64() - t0) / reps;
    // same with 32 per thread (16 nodes)
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
#pragma unroll 4
        for (int k = 0; k < 32; ++k) {
            const int e = tid + k * 256, peer = (e >> 5) & 15;
            red_dsm(mapa(smaddr(sm + 36864 + (e & 511)), peer), 1.f);
        }
        arrive_rel(); wait_acq();
    }
    res[5] = (clock64() - t0) / reps;
    // st.async of float partials for 16 nodes' transposed products: 16 nodes x 16 peers x 128 B per CTA
    res[6] = push_round<8>(sm, mbar, rk, reps, tid);
    arrive_rel(); wait_acq();
    if (tid == 0) for (int k = 0; k < 7; ++k) out[blockIdx.x * 8 + k] = res[k];
}

int main() {
    const int smem = 200 * 1024;
    cudaFuncSetAttribute(mb, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(mb, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    const int cs = 16, ncl = 7;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(cs * ncl);
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    long long* out;
    cudaMalloc(&out, cs * ncl * 8 * 8);
    cudaError_t e = cudaLaunchKernelEx(&cfg, mb, out, 100);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    printf("launch: %s\n", cudaGetErrorString(e));
    long long h[16 * 7 * 8];
    cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
    const char* names[7] = {"st.async 256 x 16 B/CTA + mbarrier", "st.async 1024 x 16 B/CTA + mbarrier",
                            "st.async 2048 x 16 B/CTA + mbarrier", "st.shared::cluster 1024 x 16 B + release bar",
                            "red.shared::cluster.f32 512/CTA + release bar", "red.shared::cluster.f32 8192/CTA + release bar",
                            "st.async 2048 x 16 B/CTA (repeat)"};
    for (int k = 0; k < 7; ++k) {
        double m = 0, mx = 0;
        for (int b = 0; b < cs * ncl; ++b) { m += h[b * 8 + k]; mx = h[b * 8 + k] > mx ? h[b * 8 + k] : mx; }
        printf("%-48s mean %7.0f  max %7.0f cycles\n", names[k], m / (cs * ncl), mx);
    }
    return 0;
}
