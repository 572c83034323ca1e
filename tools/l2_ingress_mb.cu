// Per-SM load throughput from L2 (measurement only): one CTA per SM (148 CTAs x 256 threads) moves
// `bytes` from an L2-resident buffer into shared memory or registers, four ways:
//   0: cp.async 16 B per thread (the staging of vpps_leaf_fwd / vpps_df / vpps_dw_gemm),
//   1: LDG.128 into registers (summed, so the loads are live),
//   2: cp.async.bulk (1D, TMA engine) 4 KB per copy, issued by one warp, one mbarrier,
//   3: as 0, but the source is a cold (never touched, DRAM) buffer.
// Prints cycles per CTA (mean / max over CTAs) and bytes per clock per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/l2mb tools/l2_ingress_mb.cu && /tmp/l2mb
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(256, 1) ingress(const float* __restrict__ src, int64_t per_cta_floats, int mode,
                                                  long long* cyc, float* sink) {
    extern __shared__ __align__(128) float sm[];
    __shared__ __align__(8) uint64_t bar;
    const int tid = threadIdx.x;
    const float* s = src + (int64_t)blockIdx.x * per_cta_floats;
    const int64_t n4 = per_cta_floats / 4;
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const long long t0 = clock64();
    float acc = 0.f;
    if (mode == 0 || mode == 3) {
        for (int64_t i = tid; i < n4; i += 256)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sm + 4 * i)), "l"(s + 4 * i) : "memory");
        asm volatile("cp.async.wait_all;" ::: "memory");
    } else if (mode == 1) {
        for (int64_t i = tid; i < n4; i += 256) {
            const float4 v = __ldcg(reinterpret_cast<const float4*>(s) + i);
            acc += v.x + v.y + v.z + v.w;
        }
    } else {
        const int64_t bytes = per_cta_floats * 4, chunk = 4096;
        if (tid < 32) {
            if (tid == 0) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar)), "r"((uint32_t)bytes) : "memory");
            __syncwarp();
            for (int64_t o = tid * chunk; o < bytes; o += 32 * chunk)
                asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(smem_u32(reinterpret_cast<char*>(sm) + o)), "l"(reinterpret_cast<const char*>(s) + o),
                               "r"((uint32_t)chunk), "r"(smem_u32(&bar)) : "memory");
        }
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                         : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
    }
    __syncthreads();
    const long long t1 = clock64();
    if (tid == 0) cyc[blockIdx.x] = t1 - t0;
    if (acc == 12345.f) sink[0] = acc + sm[tid];
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    float *warm, *cold, *sink;
    long long* cyc;
    const int64_t max_per = 192 * 1024 / 4;                                 // 192 KB per CTA
    cudaMalloc(&warm, (size_t)nsm * max_per * 4);
    cudaMalloc(&cold, (size_t)nsm * 1200 * 1024);
    cudaMalloc(&sink, 64);
    cudaMallocManaged(&cyc, nsm * sizeof(long long));
    cudaMemset(warm, 0, (size_t)nsm * max_per * 4);
    cudaFuncSetAttribute(ingress, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const char* names[] = {"cp.async 16B    ", "LDG.128 -> regs ", "bulk 4KB (TMA)  ", "cp.async 16B cold"};
    for (int kb : {32, 64, 128, 192}) {
        const int64_t per = (int64_t)kb * 1024 / 4;
        for (int mode = 0; mode < 4; ++mode) {
            const float* src = mode == 3 ? cold + (int64_t)kb * 1024 / 4 * nsm * (kb / 32 - 1) : warm;
            if (mode != 3) ingress<<<nsm, 256, 200 * 1024>>>(warm, per, mode, cyc, sink);   // warm L2
            cudaDeviceSynchronize();
            ingress<<<nsm, 256, 200 * 1024>>>(src, per, mode, cyc, sink);
            cudaError_t e = cudaDeviceSynchronize();
            std::vector<long long> c(cyc, cyc + nsm);
            double mean = 0;
            for (auto v : c) mean += v;
            mean /= nsm;
            const long long mx = *std::max_element(c.begin(), c.end());
            printf("%3d KB/CTA %s: mean %7.0f max %7lld cycles  -> %6.1f B/clk/SM (mean)  %s\n", kb, names[mode], mean, mx,
                   kb * 1024.0 / mean, cudaGetErrorString(e));
        }
    }
    return 0;
}
