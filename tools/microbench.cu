// Latency microbenchmarks of the primitives the VPPS interpreter uses per batch / per phase (B200).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb
// Every CTA (148 x 256 threads, one per SM) runs the same sequence; thread 0 of each CTA records clock64
// deltas; the host prints the mean / max over CTAs in cycles.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(256, 1) mb(const float* __restrict__ src, float* __restrict__ sink,
                                              unsigned* ctr, long long* out, int nseg, int seg_floats) {
    extern __shared__ __align__(16) float sm[];
    __shared__ __align__(8) uint64_t mbar;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    long long t[16];
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    // warm the source in L2
    for (int i = tid; i < nseg * seg_floats; i += 256) sink[blockIdx.x] += __ldcg(src + i) * 0.f;
    __syncthreads();
    uint32_t phase = 0;
    for (int rep = 0; rep < 3; ++rep) {
        __syncthreads();
        t[0] = clock64();
        __syncthreads();
        t[1] = clock64();                                          // (1) one __syncthreads
        // (2) warp 0 issues nseg bulk copies of seg_floats each, then all wait on the mbarrier
        if (warp == 0) {
            if (lane == 0)
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&mbar)),
                             "r"((uint32_t)(nseg * seg_floats * 4)));
            __syncwarp();
            for (int s = lane; s < nseg; s += 32)
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                                 smem_u32(sm + s * seg_floats)),
                             "l"(src + s * seg_floats), "r"((uint32_t)(seg_floats * 4)), "r"(smem_u32(&mbar)));
        }
        t[2] = clock64();                                          // issue done (thread 0)
        asm volatile(
            "{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
                smem_u32(&mbar)),
            "r"(phase));
        phase ^= 1;
        t[3] = clock64();                                          // copies landed
        // (3) one dependent L2 load per thread + store to smem + syncthreads
        const float v = __ldcg(src + ((tid * 97 + rep * 13) % (nseg * seg_floats)));
        sm[nseg * seg_floats + tid] = v;
        __syncthreads();
        t[4] = clock64();
        // (4) 16 independent float4 loads per thread, then stores (the old register staging)
        float4 r[16];
        const float4* s4 = reinterpret_cast<const float4*>(src);
#pragma unroll
        for (int i = 0; i < 16; ++i) r[i] = __ldcg(s4 + ((tid + 256 * i) % (nseg * seg_floats / 4)));
#pragma unroll
        for (int i = 0; i < 16; ++i) reinterpret_cast<float4*>(sm)[tid + 256 * i % 4096] = r[i];
        __syncthreads();
        t[5] = clock64();
        // (5) grid barrier: bar.sync + red.release / ld.acquire spin + bar.sync
        __syncthreads();
        if (tid == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr + rep) : "memory");
        t[6] = clock64();
        if (tid == 0) {
            unsigned c;
            do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(c) : "l"(ctr + rep) : "memory"); } while (c < gridDim.x);
        }
        __syncthreads();
        t[7] = clock64();
        // (6) 64 red.global.add.v4 per thread to distinct addresses (no contention) + bar.sync
        float* dst = sink + 1024 + (size_t)blockIdx.x * 256 * 64 * 4;
        for (int i = 0; i < 64; ++i)
            asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(dst + (i * 256 + tid) * 4), "f"(1.f), "f"(1.f),
                         "f"(1.f), "f"(1.f));
        __syncthreads();
        t[8] = clock64();
        if (tid == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr + 8 + rep) : "memory");
        t[9] = clock64();                                          // release after many reds
        if (tid == 0 && rep == 2)
            for (int k = 0; k < 9; ++k) out[blockIdx.x * 16 + k] = t[k + 1] - t[k];
    }
}

// FP32 FMA throughput: 8 independent accumulators per thread, plain FFMA vs packed FFMA2.
template <bool PACKED>
__global__ void __launch_bounds__(256, 1) fma_tp(float* out, long long* cyc, int iters) {
    float a[16];
    for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3f + i;
    const float b = 0.999f, c = 1e-4f;
    __syncthreads();
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        if constexpr (PACKED) {
#pragma unroll
            for (int i = 0; i < 16; i += 2) {
                float2 r = __ffma2_rn(make_float2(a[i], a[i + 1]), make_float2(b, b), make_float2(c, c));
                a[i] = r.x; a[i + 1] = r.y;
            }
        } else {
#pragma unroll
            for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], b, c);
        }
    }
    __syncthreads();
    const long long t1 = clock64();
    float s = 0.f;
    for (int i = 0; i < 16; ++i) s += a[i];
    out[blockIdx.x * 256 + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    {
        float* o;
        long long* cy;
        cudaMalloc(&o, 148 * 256 * 4);
        cudaMalloc(&cy, 148 * 8);
        const int iters = 4096;
        for (int packed = 0; packed < 2; ++packed) {
            if (packed) fma_tp<true><<<148, 256>>>(o, cy, iters);
            else fma_tp<false><<<148, 256>>>(o, cy, iters);
            cudaDeviceSynchronize();
            long long h[148];
            cudaMemcpy(h, cy, sizeof(h), cudaMemcpyDeviceToHost);
            double mean = 0;
            for (int i = 0; i < 148; ++i) mean += h[i] / 148.0;
            printf("%s: %.1f FMA/clk/SM (256 threads, 16 independent accumulators)\n", packed ? "FFMA2" : "FFMA ",
                   256.0 * 16 * iters / mean);
        }
    }
    const int nseg = 64, segf = 256;
    float *src, *sink;
    unsigned* ctr;
    long long* out;
    cudaMalloc(&src, 1 << 24);
    cudaMalloc(&sink, 1 << 28);
    cudaMalloc(&ctr, 64 * 4);
    cudaMalloc(&out, 148 * 16 * 8);
    cudaMemset(src, 0, 1 << 24);
    cudaMemset(sink, 0, 1 << 28);
    cudaMemset(ctr, 0, 64 * 4);
    const int smem = (nseg * segf + 4096 * 4 + 1024) * 4;
    cudaFuncSetAttribute(mb, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    void* args[] = {&src, &sink, &ctr, &out, (void*)&nseg, (void*)&segf};
    int ns = nseg, sf = segf;
    args[4] = &ns;
    args[5] = &sf;
    cudaError_t e = cudaLaunchCooperativeKernel((void*)mb, 148, 256, args, smem, 0);
    cudaDeviceSynchronize();
    printf("launch: %s\n", cudaGetErrorString(e ? e : cudaGetLastError()));
    std::vector<long long> h(148 * 16);
    cudaMemcpy(h.data(), out, h.size() * 8, cudaMemcpyDeviceToHost);
    const char* names[9] = {"syncthreads", "issue 64x1KB bulk copies (warp 0)", "wait for the copies (mbarrier)",
                            "1 dependent L2 load/thread + sts + sync", "16 float4 L2 loads/thread + sts + sync",
                            "sync + red.release (signal)", "acquire spin until all 148 arrived + sync",
                            "64 red.v4/thread + sync", "red.release after reds"};
    for (int k = 0; k < 9; ++k) {
        double s = 0, mx = 0;
        for (int c = 0; c < 148; ++c) { s += h[c * 16 + k]; mx = mx > h[c * 16 + k] ? mx : h[c * 16 + k]; }
        printf("%-45s mean %8.0f  max %8.0f cycles\n", names[k], s / 148, mx);
    }
    return 0;
}
