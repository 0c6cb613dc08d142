// gather_ceiling.cu -- the practical ceiling of k_find's access pattern on this GPU:
// N random 8-byte probes into an L2-resident table (C4: 150 M query positions into the
// 16 MB rank-word directory), 8 independent probes per thread as in k_find, no other
// work. Reports probes/s and global-load sectors per SM clock, to set against k_find's
// 198 M sectors in its measured kernel time.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o gather_ceiling gather_ceiling.cu
//   ./gather_ceiling [n_probes=150000000] [table_MB=16]
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint64_t x) {  // splitmix-style hash -> word index
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return uint32_t(x ^ (x >> 31));
}

template <int kPer>
__global__ void __launch_bounds__(256) k_gather(const unsigned long long *__restrict__ t, uint32_t mask, uint64_t n,
                                                unsigned long long *sink) {
    unsigned long long acc = 0;
    for (uint64_t base = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) * kPer; base < n;
         base += uint64_t(gridDim.x) * blockDim.x * kPer) {
        unsigned long long v[kPer];
#pragma unroll
        for (int j = 0; j < kPer; ++j) v[j] = base + j < n ? __ldg(t + (mix(base + j) & mask)) : 0ull;
#pragma unroll
        for (int j = 0; j < kPer; ++j) acc ^= v[j];
    }
    if (acc == 0x123456789ull) *sink = acc;  // keep the loads
}

int main(int argc, char **argv) {
    const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 10) : 150000000ull;
    const uint64_t mb = argc > 2 ? strtoull(argv[2], 0, 10) : 16;
    const uint64_t words = (mb << 20) / 8;  // power of two
    unsigned long long *t, *sink;
    cudaMalloc(&t, words * 8);
    cudaMalloc(&sink, 8);
    cudaMemset(t, 1, words * 8);
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);  // kHz (max)
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_gather<8>, 256, 0);
    const int grid = per_sm * sms;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int it = 0; it < 8; ++it) {
        cudaEventRecord(a);
        k_gather<8><<<grid, 256>>>(t, uint32_t(words - 1), n, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        if (it >= 2 && ms < best) best = ms;
    }
    const double sec = best / 1e3;
    printf("{\"probes\": %llu, \"table_MB\": %llu, \"ms\": %.4f, \"probes_per_s\": %.4g, "
           "\"sectors_per_sm_clk_at_max_clock\": %.3f, \"grid\": %d}\n",
           (unsigned long long)n, (unsigned long long)mb, best, n / sec, n / (sec * sms * clk * 1e3), grid);
    return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
