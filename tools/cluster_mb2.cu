// Cluster-barrier cost under pending memory traffic + DSMEM exchange options (B200, 16-CTA clusters).
// Answers: how much of the cluster kernel's per-level "arrive" time is the release waiting for global stores,
// and what a DSMEM pull / st.async push costs instead of the L2 round trip.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/cmb2.bin tools/cluster_mb2.cu && ./tools/cmb2.bin
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void arrive_rel() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void arrive_rlx() { asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory"); }
__device__ __forceinline__ void wait_acq() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ uint32_t rank() { uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ uint32_t smaddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
    uint32_t d; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(r)); return d;
}
__device__ __forceinline__ float4 ld_dsm(uint32_t a) {
    float4 v;
    asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void st_dsm(uint32_t a, float4 v) {
    asm volatile("st.shared::cluster.v4.f32 [%0], {%1,%2,%3,%4};" :: "r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ void st_async(uint32_t a, float4 v, uint32_t mbar) {
    asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1,%2,%3,%4}, [%5];"
                 :: "r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "r"(mbar) : "memory");
}
__device__ __forceinline__ void red_async_u64(uint32_t a, unsigned long long v, uint32_t mbar) {
    asm volatile("red.async.relaxed.cluster.shared::cluster.mbarrier::complete_tx::bytes.add.u64 [%0], %1, [%2];"
                 :: "r"(a), "l"(v), "r"(mbar) : "memory");
}
__device__ __forceinline__ void mbar_init(uint32_t m, uint32_t n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(m), "r"(n) : "memory"); }
__device__ __forceinline__ void mbar_expect(uint32_t m, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(m), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t m, uint32_t parity) {
    asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}"
                 :: "r"(m), "r"(parity) : "memory");
}

__global__ void __launch_bounds__(256, 1) mb(float* gbuf, long long* out, int reps) {
    extern __shared__ __align__(16) float sm[];
    __shared__ __align__(8) uint64_t mbar[2];
    const int tid = threadIdx.x;
    const uint32_t rk = rank();
    for (int i = tid; i < 16384; i += 256) sm[i] = rk + i * 1e-3f;
    if (tid == 0) { mbar_init(smaddr(&mbar[0]), 1); mbar_init(smaddr(&mbar[1]), 1); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    arrive_rel(); wait_acq();
    float* g = gbuf + (size_t)blockIdx.x * 65536;
    long long res[10];
    long long t0;
    float sink = 0.f;
    // 0: bare barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) { arrive_rel(); wait_acq(); }
    res[0] = (clock64() - t0) / reps;
    // 1: 64 threads x 7 scattered st.global (cell update), then release barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        if (tid % 4 == 0) for (int k = 0; k < 7; ++k) g[k * 4096 + tid + r] = sink + k;
        arrive_rel(); wait_acq();
    }
    res[1] = (clock64() - t0) / reps;
    // 2: same stores, relaxed arrive (no ordering)
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        if (tid % 4 == 0) for (int k = 0; k < 7; ++k) g[k * 4096 + tid + r] = sink + k;
        arrive_rlx(); wait_acq();
    }
    res[2] = (clock64() - t0) / reps;
    // 3: 256 threads x 2 red.global.add.v4 (transposed product), release barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        for (int k = 0; k < 2; ++k)
            asm volatile("red.global.add.v4.f32 [%0], {%1,%1,%1,%1};" :: "l"(g + 32768 + k * 1024 + tid * 4), "f"(1.f) : "memory");
        arrive_rel(); wait_acq();
    }
    res[3] = (clock64() - t0) / reps;
    // 4: remote DSMEM stores: 256 threads write 16 B each to one peer (16 peers covered) then release barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        st_dsm(mapa(smaddr(sm + 8192 + rk * 64 + (tid & 15) * 4), tid >> 4), make_float4(r, 1, 2, 3));
        arrive_rel(); wait_acq();
    }
    res[4] = (clock64() - t0) / reps;
    // 5: DSMEM pull: 8 remote float4 loads per thread (16 nodes x 512 floats), sum, syncthreads
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        float4 s = make_float4(0, 0, 0, 0);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const float4 v = ld_dsm(mapa(smaddr(sm + ((tid * 8 + k) & 4095) * 4), (tid + k + r) & 15));
            s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
        }
        sm[12288 + tid] = s.x + s.y + s.z + s.w;
        __syncthreads();
    }
    res[5] = (clock64() - t0) / reps;
    // 6: L2 pull for comparison: 8 ld.global.cg float4 per thread of another CTA's region, syncthreads
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        const float* o = gbuf + (size_t)((blockIdx.x + 1 + r) % gridDim.x) * 65536;
        float4 s = make_float4(0, 0, 0, 0);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const float4 v = __ldcg(reinterpret_cast<const float4*>(o) + ((tid * 8 + k) & 4095));
            s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
        }
        sm[12288 + tid] = s.x + s.y + s.z + s.w;
        __syncthreads();
    }
    res[6] = (clock64() - t0) / reps;
    // 7: st.async push + mbarrier: each CTA sends 64 B to each of 16 peers (threads 0..63: 16 B each),
    //    then waits until 16 x 64 B have landed in its own buffer (alternating mbarriers / buffers)
    arrive_rel(); wait_acq();
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        const int b = r & 1;
        const uint32_t mb_local = smaddr(&mbar[b]);
        if (tid == 0) mbar_expect(mb_local, 16 * 64);
        if (tid < 64) {
            const uint32_t peer = tid >> 2;
            const uint32_t dst = mapa(smaddr(sm + 8192 + b * 1024 + rk * 16 + (tid & 3) * 4), peer);
            st_async(dst, make_float4(r, rk, 2, 3), mapa(mb_local, peer));
        }
        mbar_wait(mb_local, (uint32_t)((r >> 1) & 1));
    }
    res[7] = (clock64() - t0) / reps;
    // 8: st.async after 7 global stores (does the global traffic slow the push path?)
    t0 = clock64();
    for (int r = reps; r < 2 * reps; ++r) {
        const int b = r & 1;
        const uint32_t mb_local = smaddr(&mbar[b]);
        if (tid % 4 == 0) for (int k = 0; k < 7; ++k) g[k * 4096 + tid + r] = sink + k;
        if (tid == 0) mbar_expect(mb_local, 16 * 64);
        if (tid < 64) {
            const uint32_t peer = tid >> 2;
            const uint32_t dst = mapa(smaddr(sm + 8192 + b * 1024 + rk * 16 + (tid & 3) * 4), peer);
            st_async(dst, make_float4(r, rk, 2, 3), mapa(mb_local, peer));
        }
        mbar_wait(mb_local, (uint32_t)((r >> 1) & 1));
    }
    res[8] = (clock64() - t0) / reps;
    arrive_rel(); wait_acq();
    // 9: release barrier after 16 st.global (float4) per thread -> measures drain of a larger store burst
    t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        for (int k = 0; k < 16; ++k) reinterpret_cast<float4*>(g)[k * 256 + tid] = make_float4(r, k, 0, 0);
        arrive_rel(); wait_acq();
    }
    res[9] = (clock64() - t0) / reps;
    // 10: red.async.add.u64 fixed-point reduction: every CTA adds 32 values into each of the 16 peers'
    //     accumulators (2 per thread), receiver expects 16 x 32 x 8 B; checks the sums
    unsigned long long* acc = reinterpret_cast<unsigned long long*>(sm + 12288);   // 512 u64
    for (int i = tid; i < 512; i += 256) acc[i] = 0ull;
    arrive_rel(); wait_acq();
    t0 = clock64();
    long long bad = 0;
    for (int r = 0; r < reps; ++r) {
        const int b = r & 1;
        const uint32_t mb_local = smaddr(&mbar[b]);
        if (tid == 0) mbar_expect(mb_local, 16 * 32 * 8);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int e = tid + h * 256, peer = e >> 5, slot = (e & 31) + 32 * b;
            const uint32_t dst = mapa(smaddr(acc + slot * 8 + (rk & 7)), peer);   // 8 u64 lanes per slot
            red_async_u64(dst, (unsigned long long)(rk + 1), mapa(mb_local, peer));
        }
        mbar_wait(mb_local, (uint32_t)((r >> 1) & 1));
    }
    res[8] = res[8];
    const long long red_t = (clock64() - t0) / reps;
    // every slot s: lane (k & 7) received (k+1) from ranks k and k+8, reps/2 times per parity
    for (int i = tid; i < 512; i += 256) {
        const int lane8 = i & 7;
        const unsigned long long want = (unsigned long long)((lane8 + 1) + (lane8 + 9)) * (reps / 2);
        if (acc[i] != want) ++bad;
    }
    arrive_rel(); wait_acq();
    if (tid == 0) for (int k = 0; k < 10; ++k) out[blockIdx.x * 12 + k] = res[k];
    if (tid == 0) out[blockIdx.x * 12 + 10] = red_t;
    bad = __syncthreads_count(bad > 0);
    if (tid == 0) out[blockIdx.x * 12 + 11] = bad;
}

int main() {
    const int smem = 80 * 1024;
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
    float* g;
    long long* out;
    cudaMalloc(&g, (size_t)cs * ncl * 65536 * 4);
    cudaMemset(g, 0, (size_t)cs * ncl * 65536 * 4);
    cudaMalloc(&out, cs * ncl * 12 * 8);
    cudaError_t e = cudaLaunchKernelEx(&cfg, mb, g, out, 200);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    printf("launch: %s\n", cudaGetErrorString(e));
    long long h[16 * 7 * 12];
    cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
    const char* names[10] = {"bare arrive.release+wait", "7 st.global (64 thr) + release barrier",
                             "7 st.global (64 thr) + relaxed barrier", "2 red.v4 (256 thr) + release barrier",
                             "1 remote st.shared::cluster + release barrier", "DSMEM pull 8 x v4/thread + syncthreads",
                             "L2 pull 8 x v4/thread (ld.cg) + syncthreads", "st.async 16 peers x 64 B + mbarrier wait",
                             "7 st.global + st.async push + mbarrier wait", "16 st.global.v4 (256 thr) + release barrier"};
    for (int k = 0; k < 11; ++k) {
        double m = 0, mx = 0;
        for (int b = 0; b < cs * ncl; ++b) { m += h[b * 12 + k]; mx = h[b * 12 + k] > mx ? h[b * 12 + k] : mx; }
        printf("%-48s mean %7.0f  max %7.0f cycles\n", k < 10 ? names[k] : "red.async.add.u64 16 peers x 32 + mbarrier wait", m / (cs * ncl), mx);
    }
    long long nbad = 0;
    for (int b = 0; b < cs * ncl; ++b) nbad += h[b * 12 + 11];
    printf("red.async sums: %s (%lld threads saw a wrong sum)\n", nbad ? "WRONG" : "correct", nbad);
    return 0;
}
