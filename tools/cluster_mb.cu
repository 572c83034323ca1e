// Cluster feasibility + latency microbenchmark on B200: max active clusters of size 8/16 at the VPPS
// kernel's resources, hardware cluster barrier latency, DSMEM load / store latency.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/cmb.bin tools/cluster_mb.cu && ./tools/cmb.bin
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__global__ void __launch_bounds__(256, 1) cmb(long long* out, int reps) {
    extern __shared__ __align__(16) float sm[];
    cg::cluster_group cl = cg::this_cluster();
    const int rank = cl.block_rank(), n = cl.num_blocks();
    const int tid = threadIdx.x;
    for (int i = tid; i < 4096; i += 256) sm[i] = rank * 10000 + i;
    cl.sync();
    long long t0, t1, acc = 0;
    // (1) cluster barrier
    t0 = clock64();
    for (int r = 0; r < reps; ++r) cl.sync();
    t1 = clock64();
    const long long bar = (t1 - t0) / reps;
    // (2) DSMEM dependent load latency (thread 0 chases one remote float)
    float v = 0.f;
    if (tid == 0) {
        float* remote = cl.map_shared_rank(sm, (rank + 1) % n);
        t0 = clock64();
        int idx = 0;
        for (int r = 0; r < reps; ++r) { v += remote[idx]; idx = ((int)v) & 1023; }
        t1 = clock64();
        acc = (t1 - t0) / reps;
    }
    cl.sync();
    // (3) all-gather: every thread reads 16 B from each of the n ranks (n * 4 KB per CTA), then cluster.sync
    t0 = clock64();
    float4 s = make_float4(0, 0, 0, 0);
    for (int r = 0; r < n; ++r) {
        const float4* rem = reinterpret_cast<const float4*>(cl.map_shared_rank(sm, r));
        float4 x = rem[tid];
        s.x += x.x; s.y += x.y; s.z += x.z; s.w += x.w;
    }
    sm[8192 + tid] = s.x + s.y + s.z + s.w;
    cl.sync();
    t1 = clock64();
    const long long gather = t1 - t0;
    // (4) reduce-scatter style: every thread writes 16 B into each rank's slot, then cluster.sync
    t0 = clock64();
    for (int r = 0; r < n; ++r) {
        float4* rem = reinterpret_cast<float4*>(cl.map_shared_rank(sm + 4096, r));
        rem[rank * 256 / n + (tid % (256 / n)) + 0] = make_float4(1, 2, 3, 4);
    }
    cl.sync();
    t1 = clock64();
    if (tid == 0) {
        out[blockIdx.x * 4 + 0] = bar;
        out[blockIdx.x * 4 + 1] = acc + (long long)v * 0;
        out[blockIdx.x * 4 + 2] = gather;
        out[blockIdx.x * 4 + 3] = t1 - t0;
    }
}

int main() {
    const int smem = 200 * 1024;
    cudaFuncSetAttribute(cmb, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(cmb, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    for (int cs : {4, 8, 16}) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(cs * 8);
        cfg.blockDim = dim3(256);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = cs;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        int ncl = 0;
        cudaError_t e = cudaOccupancyMaxActiveClusters(&ncl, cmb, &cfg);
        printf("cluster %2d: max active clusters %d (%s)\n", cs, ncl, cudaGetErrorString(e));
        if (ncl <= 0) continue;
        cfg.gridDim = dim3(cs * ncl);
        long long* out;
        cudaMalloc(&out, cs * ncl * 4 * 8);
        e = cudaLaunchKernelEx(&cfg, cmb, out, 100);
        cudaDeviceSynchronize();
        if (e == cudaSuccess) e = cudaGetLastError();
        long long h[16 * 16 * 4];
        cudaMemcpy(h, out, cs * ncl * 4 * 8, cudaMemcpyDeviceToHost);
        double m[4] = {0, 0, 0, 0};
        for (int b = 0; b < cs * ncl; ++b)
            for (int k = 0; k < 4; ++k) m[k] += h[b * 4 + k] / double(cs * ncl);
        printf("   launch %s: cluster.sync %.0f cyc, DSMEM dependent load %.0f cyc, all-gather %d x 4KB + sync %.0f cyc,"
               " scatter-store + sync %.0f cyc\n",
               cudaGetErrorString(e), m[0], m[1] * 148 / 148, cs, m[2], m[3]);
        cudaFree(out);
    }
    return 0;
}
