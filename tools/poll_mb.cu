// Microbenchmark: latency of the dataflow kernel's slot polls (17 independent 8-byte loads per thread from
// L2-resident memory) in the load flavours the kernel can use, with and without preceding stores.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pmb tools/poll_mb.cu && /tmp/pmb
// 148 CTAs x 256 threads; per test the max over the CTA's threads of (clock after consuming the loads -
// clock before issuing them), mean / max over CTAs, in cycles.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

typedef unsigned long long u64;
template <int K>
__device__ __forceinline__ u64 ld(const u64* p) {
    u64 v;
    if constexpr (K == 0) asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    else if constexpr (K == 1) asm volatile("ld.global.cg.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    else if constexpr (K == 2) asm volatile("ld.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    else if constexpr (K == 3) asm volatile("ld.volatile.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    else asm volatile("ld.global.cg.b64 %0, [%1];" : "=l"(v) : "l"(p));   // no memory clobber
    return v;
}

template <int K, int NL>
__device__ __forceinline__ u64 poll(const u64* base, int tid) {
    u64 v[NL];
#pragma unroll
    for (int k = 0; k < NL; ++k) v[k] = ld<K>(base + tid + k * 32 * 148 * 4);
    u64 s = 0;
#pragma unroll
    for (int k = 0; k < NL; ++k) s += v[k];
    return s;
}

constexpr int NT = 16;
__global__ void __launch_bounds__(256, 1) pmb(const u64* src, float* junk, u64* sink, long long* out) {
    __shared__ int mx[NT];
    const int tid = threadIdx.x;
    if (tid < NT) mx[tid] = 0;
    const u64* base = src + blockIdx.x * 256;
    u64 acc = 0;
    for (int rep = 0; rep < 4; ++rep) {
        long long d[NT];
        long long t0, t1;
#define MEAS(i, ...)                          \
    __syncthreads();                           \
    t0 = clock64();                            \
    acc += (__VA_ARGS__);                      \
    t1 = clock64();                            \
    d[i] = t1 - t0;
        MEAS(0, poll<0, 17>(base, tid));
        MEAS(1, poll<1, 17>(base, tid));
        MEAS(2, poll<2, 17>(base, tid));
        MEAS(3, poll<3, 17>(base, tid));
        MEAS(4, poll<4, 17>(base, tid));
        MEAS(5, poll<0, 1>(base, tid));
        MEAS(6, poll<1, 1>(base, tid));
        MEAS(7, (tid < 16 ? poll<0, 17>(base, tid) : 0ull));
        MEAS(8, (tid < 16 ? poll<1, 17>(base, tid) : 0ull));
        // preceded by 8 global stores per thread (a batch's record writes)
        __syncthreads();
        for (int k = 0; k < 8; ++k) junk[(blockIdx.x * 8 + k) * 256 + tid] = (float)acc;
        MEAS(9, poll<1, 17>(base, tid));
        __syncthreads();
        for (int k = 0; k < 8; ++k) junk[(blockIdx.x * 8 + k) * 256 + tid] = (float)acc;
        MEAS(10, poll<0, 17>(base, tid));
        // 4 dependent rounds of 17 (LEAF_B loop)
        __syncthreads();
        t0 = clock64();
        {
            u64 s = 0;
            for (int r = 0; r < 4; ++r) s += poll<1, 17>(base + (s & 1), tid);
            acc += s;
        }
        t1 = clock64();
        d[11] = t1 - t0;
        __syncthreads();
        t0 = clock64();
        {
            u64 s = 0;
            for (int r = 0; r < 4; ++r) s += poll<0, 17>(base + (s & 1), tid);
            acc += s;
        }
        t1 = clock64();
        d[12] = t1 - t0;
        if (rep == 3)
            for (int i = 0; i < 13; ++i) atomicMax(&mx[i], (int)d[i]);
    }
    __syncthreads();
    if (tid < 13) out[blockIdx.x * NT + tid] = mx[tid];
    if (acc == 12345) sink[0] = acc;
}

int main() {
    const int n = 148 * 256 + 17 * 32 * 148 * 4 + 64;
    u64* src;
    float* junk;
    u64* sink;
    long long* out;
    cudaMalloc(&src, n * sizeof(u64));
    cudaMemset(src, 1, n * sizeof(u64));
    cudaMalloc(&junk, 148 * 8 * 256 * sizeof(float));
    cudaMalloc(&sink, 8);
    cudaMalloc(&out, 148 * NT * sizeof(long long));
    pmb<<<148, 256>>>(src, junk, sink, out);
    pmb<<<148, 256>>>(src, junk, sink, out);
    cudaError_t e = cudaDeviceSynchronize();
    printf("launch: %s\n", cudaGetErrorString(e));
    std::vector<long long> h(148 * NT);
    cudaMemcpy(h.data(), out, h.size() * 8, cudaMemcpyDeviceToHost);
    const char* names[13] = {"17 x ld.relaxed.gpu.b64 (256 thr)", "17 x ld.global.cg.b64", "17 x ld.global.b64 (.ca)",
                             "17 x ld.volatile.global.b64", "17 x ld.cg.b64 (no memory clobber)", "1 x ld.relaxed.gpu",
                             "1 x ld.cg", "17 x ld.relaxed.gpu (16 threads)", "17 x ld.cg (16 threads)",
                             "8 st.global + 17 x ld.cg", "8 st.global + 17 x ld.relaxed.gpu",
                             "4 dependent rounds of 17 ld.cg", "4 dependent rounds of 17 ld.relaxed.gpu"};
    for (int i = 0; i < 13; ++i) {
        double s = 0, m = 0;
        for (int b = 0; b < 148; ++b) { s += h[b * NT + i]; m = h[b * NT + i] > m ? h[b * NT + i] : m; }
        printf("%-44s mean %8.0f  max %8.0f cycles\n", names[i], s / 148, m);
    }
    return 0;
}
