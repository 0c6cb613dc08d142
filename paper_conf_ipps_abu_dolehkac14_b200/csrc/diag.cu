// diag.cu -- instrumentation, not the method: the gather ceiling that bounds k_find.
// k_find is limited by the rate at which SMs request random 32-byte sectors from L2
// (one rank-word probe per query position). This kernel does nothing but
// such probes -- 8 independent random 8-byte loads per thread into an L2-resident table,
// as k_find issues them -- so bench.py can report k_find's sector rate against the rate
// this GPU actually sustains for the pattern, measured in the same process.
#include "internal.h"

namespace gm {
namespace {

__device__ __forceinline__ uint32_t mix32(uint64_t x) {  // splitmix64 finaliser -> word index
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return uint32_t(x ^ (x >> 31));
}

__global__ void __launch_bounds__(256) k_gather_ceiling(const unsigned long long *__restrict__ t, uint32_t mask,
                                                        uint64_t n, unsigned long long *sink) {
    pdl_wait();
    constexpr int kPer = 8;
    unsigned long long acc = 0;
    for (uint64_t base = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) * kPer; base < n;
         base += uint64_t(gridDim.x) * blockDim.x * kPer) {
        unsigned long long v[kPer];
#pragma unroll
        for (int j = 0; j < kPer; ++j) v[j] = base + j < n ? __ldg(t + (mix32(base + j) & mask)) : 0ull;
#pragma unroll
        for (int j = 0; j < kPer; ++j) acc ^= v[j];
    }
    if (acc == 0x123456789ull) *sink = acc;  // keeps the loads
}

}  // namespace

cudaError_t gather_ceiling(uint64_t n_probes, uint64_t table_bytes, cudaStream_t s, float *best_ms) {
    uint64_t words = 1;
    while (words * 16 <= table_bytes) words <<= 1;  // power of two <= table_bytes / 8
    unsigned long long *t = nullptr, *sink = nullptr;
    cudaError_t e = cudaMalloc(&t, words * 8);
    if (e == cudaSuccess) e = cudaMalloc(&sink, 8);
    if (e == cudaSuccess) e = cudaMemsetAsync(t, 1, words * 8, s);
    int per_sm = 0;
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_gather_ceiling, 256, 0);
    cudaEvent_t a = nullptr, b = nullptr;
    if (e == cudaSuccess) e = cudaEventCreate(&a);
    if (e == cudaSuccess) e = cudaEventCreate(&b);
    float best = 1e30f;
    for (int it = 0; e == cudaSuccess && it < 6; ++it) {
        cudaEventRecord(a, s);
        k_gather_ceiling<<<(per_sm > 0 ? per_sm : 1) * num_sms(), 256, 0, s>>>(t, uint32_t(words - 1), n_probes, sink);
        cudaEventRecord(b, s);
        e = cudaEventSynchronize(b);
        float ms = 0.f;
        if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, a, b);
        if (it >= 2 && ms < best) best = ms;  // the first runs warm the table into L2
    }
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    cudaFree(t);
    cudaFree(sink);
    *best_ms = best;
    return e;
}

}  // namespace gm
