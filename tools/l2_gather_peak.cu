// l2_gather_peak.cu — measured ceiling for k_call_tile's dominant access: random 80-byte rows
// (5 x 16-byte loads) gathered from an L2-resident table of the score-table's size.
// Prints one JSON line: {"l2_gather_gbs": ..., "rows_per_s": ..., "table_bytes": ...}.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/l2_gather_peak tools/l2_gather_peak.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) gather(const double2* __restrict__ T, uint32_t rows,
                                              uint32_t iters, uint32_t seed, double* out) {
    uint32_t x = seed ^ (blockIdx.x * 256u + threadIdx.x) * 2654435761u;
    double a0 = 0, a1 = 0, a2 = 0, a3 = 0, a4 = 0, a5 = 0, a6 = 0, a7 = 0, a8 = 0, a9 = 0;
#pragma unroll 4
    for (uint32_t i = 0; i < iters; ++i) {
        x = x * 1664525u + 1013904223u;
        const double2* r = T + (size_t)(x % rows) * 5;
        double2 v0 = __ldg(r), v1 = __ldg(r + 1), v2 = __ldg(r + 2), v3 = __ldg(r + 3),
                v4 = __ldg(r + 4);
        a0 += v0.x; a1 += v0.y; a2 += v1.x; a3 += v1.y; a4 += v2.x;
        a5 += v2.y; a6 += v3.x; a7 += v3.y; a8 += v4.x; a9 += v4.y;
    }
    double s = a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 + a8 + a9;
    if (s == 12345.678) out[0] = s;  // keep the loads alive
}

int main(int argc, char** argv) {
    const uint32_t rows = argc > 1 ? (uint32_t)atoi(argv[1]) : 64 * 100 * 4;   // 2 MB table
    const uint32_t iters = 4096;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double2* T;
    double* out;
    cudaMalloc(&T, (size_t)rows * 80);
    cudaMemset(T, 0, (size_t)rows * 80);
    cudaMalloc(&out, 8);
    double best = 0;
    for (int occ = 4; occ <= 8; occ += 4) {
        const unsigned grid = (unsigned)(sms * occ);
        gather<<<grid, 256>>>(T, rows, 64, 1, out);
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(a);
            gather<<<grid, 256>>>(T, rows, iters, 7 + rep, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms = 0;
            cudaEventElapsedTime(&ms, a, b);
            const double nrows = (double)grid * 256 * iters;
            const double gbs = nrows * 80 / (ms * 1e-3) / 1e9;
            if (gbs > best) best = gbs;
        }
    }
    printf("{\"l2_gather_gbs\": %.1f, \"rows_per_s\": %.4g, \"row_bytes\": 80, \"table_bytes\": %llu, "
           "\"how\": \"random 80-byte rows (5 x LDG.128) from an L2-resident table, best of 5 x 2 grids\"}\n",
           best, best * 1e9 / 80, (unsigned long long)rows * 80);
    return 0;
}
