// sort.cu -- K8 helpers around the radix sort: packed (r << qbits | q, len) keys
// <-> gpumem_triple AoS (output sorted by (r, q); len is
// determined by (r, q) so it never breaks a tie, reading R16).
#include "internal.h"

namespace gm {
namespace {

constexpr int kT = 256;

__global__ void __launch_bounds__(kT) k_keys_to_triples(const uint64_t *__restrict__ keys,
                                                        const uint32_t *__restrict__ lens, uint64_t n,
                                                        uint32_t qbits, gpumem_triple *__restrict__ out,
                                                        const unsigned long long *__restrict__ dn) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (dn) {  // device-resident count, n is the capacity
        const unsigned long long x = *dn;
        if (x < n) n = x;
    }
    if (i >= n) return;
    const uint64_t k = keys[i];
    const uint64_t qmask = (1ull << qbits) - 1;
    gpumem_triple t;
    t.r = uint32_t(k >> qbits);
    t.q = uint32_t(k & qmask);
    t.len = lens[i];
    out[i] = t;
}

__global__ void __launch_bounds__(kT) k_triples_to_keys(const gpumem_triple *__restrict__ in, uint64_t n,
                                                        uint32_t qbits, uint64_t *__restrict__ keys,
                                                        uint32_t *__restrict__ lens) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    const gpumem_triple t = in[i];
    keys[i] = (uint64_t(t.r) << qbits) | t.q;
    lens[i] = t.len;
}

}  // namespace

cudaError_t launch_keys_to_triples(const uint64_t *keys, const uint32_t *lens, uint64_t n, uint32_t qbits,
                                   gpumem_triple *out, cudaStream_t s, const unsigned long long *dn) {
    if (!n) return cudaSuccess;
    pdl_launch(k_keys_to_triples, unsigned((n + kT - 1) / kT), kT, 0, s, keys, lens, n, qbits, out, dn);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_triples_to_keys(const gpumem_triple *in, uint64_t n, uint32_t qbits, uint64_t *keys,
                                   uint32_t *lens, cudaStream_t s) {
    if (!n) return cudaSuccess;
    pdl_launch(k_triples_to_keys, unsigned((n + kT - 1) / kT), kT, 0, s, in, n, qbits, keys, lens);
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
