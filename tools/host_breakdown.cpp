// Fig.10-style host breakdown: per-phase time of the script builder over the bench's
// batches.  Built and run by tools/host_breakdown.py (links csrc/host/script.cpp with -DVPPS_HOST_PHASES).
#include <chrono>
#include <cstdio>
#include <cstdint>
#include <fstream>
#include <string>
#include <vector>
#include "host.h"
using namespace vpps;
extern double vpps_host_phase_us[8];
int main(int argc, char** argv) {
    std::ifstream f(argv[1], std::ios::binary);
    int32_t nb = 0;
    f.read((char*)&nb, 4);
    std::vector<std::vector<int32_t>> arr[5];
    for (int k = 0; k < 5; ++k) arr[k].resize(nb);
    for (int b = 0; b < nb; ++b)
        for (int k = 0; k < 5; ++k) {
            int32_t n = 0;
            f.read((char*)&n, 4);
            arr[k][b].resize(n);
            f.read((char*)arr[k][b].data(), 4 * n);
        }
    Plan p{};
    p.cell = CELL_BINARY; p.H = 256; p.E = 256; p.C = 5; p.G = 9; p.n_act = 16; p.by_graph = true;
    const int reps = argc > 2 ? atoi(argv[2]) : 20;
    std::string err;
    double total = 0;
    for (int r = 0; r < reps + 1; ++r) {
        if (r == 1) { for (double& x : vpps_host_phase_us) x = 0; total = 0; }
        for (int b = 0; b < nb; ++b) {
            BatchIn bi{(int32_t)arr[0][b].size() - 1, arr[0][b].data(), arr[1][b].data(), arr[2][b].data(),
                       arr[3][b].data(), arr[4][b].data()};
            Script s;
            const auto t0 = std::chrono::steady_clock::now();
            if (build_script(p, bi, INT64_MAX, &s, &err) != 0) { printf("error: %s\n", err.c_str()); return 1; }
            total += std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
        }
    }
    const double n = (double)reps * nb;
    const char* names[7] = {"S1/S2 super-graph (L205)", "S3 level sort (L139)", "per-node cost, FLOPs", "S4-S6 schedule + S/W (L141-167)",
                            "encode: header, GEMM node lists (L169)", "level-path lists", "dataflow lowering (vpps_df program)"};
    for (int k = 0; k < 7; ++k) printf("%-40s %8.1f us\n", names[k], vpps_host_phase_us[k] / n);
    printf("%-40s %8.1f us per batch of 16 trees (one core)\n", "total build_script", total / n);
    return 0;
}
