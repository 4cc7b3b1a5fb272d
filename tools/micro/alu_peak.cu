// ALU ceiling for the bit-algebra tail: the rate of the tail's unit of
// work, one 64-bit "word-op" = AND of two row words + 64-bit POPC + accumulate, with
// operands in registers (no memory), 8 independent chains per thread, every SM full.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o alu_peak alu_peak.cu && ./alu_peak
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) k_wordops(uint64_t seed, int iters, unsigned long long* out) {
    uint64_t a[8], acc[8];
    const uint64_t t = seed ^ (blockIdx.x * 256ull + threadIdx.x) * 0x9E3779B97F4A7C15ull;
#pragma unroll
    for (int i = 0; i < 8; ++i) { a[i] = t * (2 * i + 1) + i; acc[i] = 0; }
    uint64_t b = t ^ 0xD1B54A32D192ED03ull;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] += __popcll(a[i] & b);
        b = b * 6364136223846793005ull + 1442695040888963407ull;   // defeats hoisting (1 IMAD.WIDE per 8 word-ops)
    }
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s += acc[i];
    if (s == 0x123456789ull) out[0] = s;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long* d;
    cudaMalloc(&d, 8);
    const int blocks = sms * 8, iters = 1 << 14;
    k_wordops<<<blocks, 256>>>(1, 16, d);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
        cudaEventRecord(e0);
        k_wordops<<<blocks, 256>>>(r + 2, iters, d);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    const double ops = (double)blocks * 256 * iters * 8;
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("{\"sms\": %d, \"word_ops_per_s\": %.4e, \"ms\": %.3f, \"per_sm_per_clk_at_max\": %.2f, \"clock_khz\": %d}\n",
           sms, ops / (best * 1e-3), best, ops / (best * 1e-3) / sms / (clk * 1e3), clk);
    return 0;
}
