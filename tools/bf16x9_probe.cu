// Probe: does the loaded cuBLAS accept the FP32-emulation math mode (BF16x9, CUBLAS_FP32_EMULATED_BF16X9_MATH)
// and how do its accuracy and speed compare with pedantic FP32 SGEMM on a level-path-sized product?
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/bf16x9_probe.cu -lcublas -o /tmp/bf9 && /tmp/bf9
#include <cublas_v2.h>
#include <cstdio>
#include <cmath>
#include <vector>
#include <random>
int main() {
    int ver = 0;
    cublasHandle_t h;
    cublasCreate(&h);
    cublasGetVersion(h, &ver);
    printf("cuBLAS version %d\n", ver);
    const int M = 1024, N = 3072, K = 2048;   // rows = nodes of a level, N = 3H gates, K = 2H (C5)
    std::vector<float> A((size_t)M * K), B((size_t)K * N);
    std::mt19937 g(1);
    std::uniform_real_distribution<float> u(-1.f, 1.f);
    for (auto& x : A) x = u(g);
    for (auto& x : B) x = u(g) * 0.03f;
    float *dA, *dB, *dC;
    cudaMalloc(&dA, A.size() * 4); cudaMalloc(&dB, B.size() * 4); cudaMalloc(&dC, (size_t)M * N * 4);
    cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
    std::vector<double> ref((size_t)M * N);
    for (int i = 0; i < 64; ++i)          // reference rows (FP64) for the accuracy check
        for (int j = 0; j < N; ++j) {
            double s = 0;
            for (int k = 0; k < K; ++k) s += (double)A[(size_t)i * K + k] * B[(size_t)k * N + j];
            ref[(size_t)i * N + j] = s;
        }
    const float one = 1.f, zero = 0.f;
    cublasMath_t modes[2] = {CUBLAS_PEDANTIC_MATH, CUBLAS_FP32_EMULATED_BF16X9_MATH};
    const char* names[2] = {"pedantic FP32", "BF16x9 emulation"};
    for (int m = 0; m < 2; ++m) {
        cublasStatus_t st = cublasSetMathMode(h, modes[m]);
        // row-major C[M][N] = A[M][K] B[K][N]  ==  column-major Cᵀ = Bᵀ Aᵀ
        auto run = [&]() { return cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, N, M, K, &one, dB, N, dA, K, &zero, dC, N); };
        cublasStatus_t st2 = run();
        cudaDeviceSynchronize();
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        for (int r = 0; r < 20; ++r) run();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        std::vector<float> C((size_t)64 * N);
        cudaMemcpy(C.data(), dC, C.size() * 4, cudaMemcpyDeviceToHost);
        double maxerr = 0, maxref = 0;
        for (size_t i = 0; i < C.size(); ++i) { maxerr = fmax(maxerr, fabs(C[i] - ref[i])); maxref = fmax(maxref, fabs(ref[i])); }
        printf("%-18s setMathMode %d gemm %d: %.3f ms, %.1f TFLOP/s, max rel err %.2e\n", names[m], (int)st, (int)st2,
               ms / 20, 2.0 * M * N * K / (ms / 20 * 1e-3) / 1e12, maxerr / maxref);
    }
    return 0;
}
