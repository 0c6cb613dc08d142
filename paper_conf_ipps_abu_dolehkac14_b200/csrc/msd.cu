// msd.cu -- MSD bucket sort for unique 64-bit keys (+ optional 32-bit values).
//
// Used where the keys are unique, so stability is irrelevant:
//  * the index: keys (seed code << 32 | location) -- sorting them groups the sampled
//    locations by seed with ascending locations inside each seed, i.e. Alg. 1 steps
//    1-4 in one sort;
//  * the output: keys (r << qbits | q) with len as value.
// One pass scatters every key into one of 2^B buckets by its top B bits (an atomic
// cursor per bucket; order inside a bucket is arbitrary), then each bucket is sorted
// by one CTA: in shared memory (bitonic) when it holds <= kLocal keys, otherwise by a
// CTA-level LSD radix over the bucket in global memory. B is chosen so that buckets
// average ~1K keys, which keeps a 13M-key sort to two passes over the data.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;
constexpr int kWarps = kT / 32;
constexpr uint32_t kLocal = 4096;   // keys sorted in shared memory per bucket
constexpr int kMaxB = 14;

__global__ void __launch_bounds__(kT) k_msd_hist(const uint64_t *__restrict__ keys, uint64_t n, int shift,
                                                 uint32_t nb, uint32_t *__restrict__ counts) {
    extern __shared__ uint32_t h[];
    for (uint32_t i = threadIdx.x; i < nb; i += kT) h[i] = 0;
    __syncthreads();
    for (uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x; i < n; i += uint64_t(gridDim.x) * kT)
        atomicAdd(&h[uint32_t(keys[i] >> shift)], 1u);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < nb; i += kT)
        if (h[i]) atomicAdd(counts + i, h[i]);
}

// exclusive scan of counts[0..nb) -> offs[0..nb] and a copy in cursor[0..nb)
__global__ void __launch_bounds__(kT) k_msd_scan(const uint32_t *__restrict__ counts, uint32_t nb,
                                                 uint32_t *__restrict__ offs, uint32_t *__restrict__ cursor) {
    __shared__ uint32_t ws[kWarps];
    __shared__ uint32_t carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint32_t base = 0; base < nb; base += kT) {
        const uint32_t i = base + threadIdx.x;
        const uint32_t x = i < nb ? counts[i] : 0;
        uint32_t inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) ws[w] = inc;
        __syncthreads();
        uint32_t pre = carry, tot = carry;
        for (int k = 0; k < kWarps; ++k) {
            if (k < w) pre += ws[k];
            tot += ws[k];
        }
        if (i < nb) offs[i] = cursor[i] = pre + inc - x;
        __syncthreads();
        if (threadIdx.x == 0) carry = tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) offs[nb] = carry;
}

__global__ void __launch_bounds__(kT) k_msd_scatter(const uint64_t *__restrict__ keys,
                                                    const uint32_t *__restrict__ vals, uint64_t n, int shift,
                                                    uint32_t *__restrict__ cursor, uint64_t *__restrict__ ok,
                                                    uint32_t *__restrict__ ov) {
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    const uint64_t k = keys[i];
    const uint32_t slot = atomicAdd(cursor + uint32_t(k >> shift), 1u);
    ok[slot] = k;
    if (vals) ov[slot] = vals[i];
}

// One CTA per bucket: shared-memory bitonic sort when it fits, else defer to k_msd_big.
__global__ void __launch_bounds__(kT) k_msd_local(const uint32_t *__restrict__ offs, uint32_t nb, uint64_t *keys,
                                                  uint32_t *vals, uint32_t *big, unsigned int *n_big) {
    extern __shared__ __align__(16) unsigned char smem[];
    uint64_t *sk = reinterpret_cast<uint64_t *>(smem);
    uint32_t *sv = reinterpret_cast<uint32_t *>(sk + kLocal);
    for (uint32_t b = blockIdx.x; b < nb; b += gridDim.x) {
        const uint32_t lo = offs[b], m = offs[b + 1] - lo;
        if (m <= 1) continue;
        if (m > kLocal) {
            if (threadIdx.x == 0) big[atomicAdd(n_big, 1u)] = b;
            continue;
        }
        uint32_t P = 2;
        while (P < m) P <<= 1;
        for (uint32_t j = threadIdx.x; j < P; j += kT) {
            sk[j] = j < m ? keys[lo + j] : ~0ull;
            if (vals) sv[j] = j < m ? vals[lo + j] : 0u;
        }
        __syncthreads();
        for (uint32_t size = 2; size <= P; size <<= 1) {
            for (uint32_t stride = size >> 1; stride; stride >>= 1) {
                for (uint32_t j = threadIdx.x; j < P / 2; j += kT) {
                    const uint32_t a = 2 * stride * (j / stride) + (j % stride), c = a + stride;
                    const bool up = (a & size) == 0;
                    const uint64_t x = sk[a], y = sk[c];
                    if ((x > y) == up) {
                        sk[a] = y;
                        sk[c] = x;
                        if (vals) {
                            const uint32_t t = sv[a];
                            sv[a] = sv[c];
                            sv[c] = t;
                        }
                    }
                }
                __syncthreads();
            }
        }
        for (uint32_t j = threadIdx.x; j < m; j += kT) {
            keys[lo + j] = sk[j];
            if (vals) vals[lo + j] = sv[j];
        }
        __syncthreads();
    }
}

// One CTA per oversized bucket: LSD radix (8-bit digits) over its low `bits` key bits,
// ping-ponging with the same range of (tk, tv).
__global__ void __launch_bounds__(kT) k_msd_big(const uint32_t *__restrict__ offs, const uint32_t *__restrict__ big,
                                                const unsigned int *__restrict__ n_big, uint64_t *keys,
                                                uint32_t *vals, uint64_t *tk, uint32_t *tv, int bits) {
    __shared__ uint32_t hist[256];
    __shared__ uint32_t wcnt[kWarps][256];
    __shared__ uint32_t ws[kWarps];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const unsigned nbig = *n_big;
    const int passes = (bits + 7) / 8;
    for (unsigned li = blockIdx.x; li < nbig; li += gridDim.x) {
        const uint32_t b = big[li];
        const uint32_t lo = offs[b], m = offs[b + 1] - lo;
        uint64_t *sk = keys + lo, *dk = tk + lo;
        uint32_t *sv = vals ? vals + lo : nullptr, *dv = vals ? tv + lo : nullptr;
        for (int pass = 0; pass < passes; ++pass) {
            const int sh = 8 * pass;
            for (int i = tid; i < 256; i += kT) hist[i] = 0;
            __syncthreads();
            for (uint32_t j = tid; j < m; j += kT) atomicAdd(&hist[uint32_t(sk[j] >> sh) & 255u], 1u);
            __syncthreads();
            {
                const uint32_t x = hist[tid];
                uint32_t inc = x;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                    if (lane >= o) inc += y;
                }
                if (lane == 31) ws[w] = inc;
                __syncthreads();
                uint32_t pre = 0;
                for (int i = 0; i < w; ++i) pre += ws[i];
                hist[tid] = pre + inc - x;
                __syncthreads();
            }
            for (uint32_t base = 0; base < m; base += kT) {  // stable, kT keys per round
                const uint32_t j = base + tid;
                const bool valid = j < m;
                const uint64_t x = valid ? sk[j] : 0ull;
                const uint32_t xv = (valid && sv) ? sv[j] : 0u;
                const uint32_t d = uint32_t(x >> sh) & 255u;
                unsigned peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
                for (int bit = 0; bit < 8; ++bit) {
                    const bool bb = (d >> bit) & 1u;
                    const unsigned mm = __ballot_sync(0xffffffffu, bb);
                    peers &= bb ? mm : ~mm;
                }
                for (int i = tid; i < kWarps * 256; i += kT) (&wcnt[0][0])[i] = 0;
                __syncthreads();
                if (valid && lane == __ffs(peers) - 1) wcnt[w][d] = __popc(peers);
                __syncthreads();
                uint32_t run = 0;
                for (int ww = 0; ww < kWarps; ++ww) {
                    const uint32_t c = wcnt[ww][tid];
                    wcnt[ww][tid] = run;
                    run += c;
                }
                __syncthreads();
                if (valid) {
                    const uint32_t pos = hist[d] + wcnt[w][d] + __popc(peers & lanemask_lt());
                    dk[pos] = x;
                    if (dv) dv[pos] = xv;
                }
                __syncthreads();
                hist[tid] += run;
                __syncthreads();
            }
            uint64_t *t = sk;
            sk = dk;
            dk = t;
            uint32_t *t2 = sv;
            sv = dv;
            dv = t2;
            __syncthreads();
        }
        if (passes & 1) {
            for (uint32_t j = tid; j < m; j += kT) {
                keys[lo + j] = tk[lo + j];
                if (vals) vals[lo + j] = tv[lo + j];
            }
        }
        __syncthreads();
    }
}

int choose_b(uint64_t n, int bits) {
    int B = 4;
    while (B < kMaxB && (n >> (B + 10)) > 0) ++B;  // ~1K keys per bucket
    return B < bits ? B : bits;
}

}  // namespace

size_t msd_scratch_bytes(uint64_t n) {
    const uint64_t nb = 1ull << kMaxB;
    return n * 8 + n * 4 + (nb + 1) * 4 * 3 + nb * 4 + 1024;
}

// Sorts (keys, vals) (vals may be null) of n unique keys whose significant bits are the
// low `bits`. The result lands in (keys, vals) in place. `scratch` >= msd_scratch_bytes(n).
cudaError_t msd_sort(uint64_t *keys, uint32_t *vals, uint64_t n, int bits, void *scratch, cudaStream_t s) {
    if (n <= 1) return cudaSuccess;
    if (bits < 1) bits = 1;
    const int B = choose_b(n, bits);
    const uint32_t nb = 1u << B;
    const int shift = bits - B;
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t c = align(reinterpret_cast<uintptr_t>(scratch));
    uint64_t *tk = reinterpret_cast<uint64_t *>(c);
    c = align(c + n * 8);
    uint32_t *tv = reinterpret_cast<uint32_t *>(c);
    c = align(c + n * 4);
    uint32_t *counts = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb + 1) * 4);
    uint32_t *offs = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb + 1) * 4);
    uint32_t *cursor = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb + 1) * 4);
    uint32_t *big = reinterpret_cast<uint32_t *>(c);
    c = align(c + nb * 4);
    unsigned int *n_big = reinterpret_cast<unsigned int *>(c);
    cudaError_t e = cudaMemsetAsync(counts, 0, (nb + 1) * 4, s);
    if (e != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(n_big, 0, 4, s)) != cudaSuccess) return e;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_msd_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, (1 << kMaxB) * 4);
        cudaFuncSetAttribute(k_msd_local, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kLocal * 12));
        attr = true;
    }
    const int sms = num_sms();
    const uint64_t hblocks = (n + kT * 16 - 1) / (kT * 16);
    k_msd_hist<<<unsigned(hblocks < uint64_t(sms * 4) ? hblocks : uint64_t(sms * 4)), kT, nb * 4, s>>>(
        keys, n, shift, nb, counts);
    k_msd_scan<<<1, kT, 0, s>>>(counts, nb, offs, cursor);
    k_msd_scatter<<<unsigned((n + kT - 1) / kT), kT, 0, s>>>(keys, vals, n, shift, cursor, tk, vals ? tv : nullptr);
    // sorted-by-bucket data now in (tk, tv); sort each bucket in place there, then copy back
    k_msd_local<<<nb < 65535u ? nb : 65535u, kT, kLocal * 12, s>>>(offs, nb, tk, vals ? tv : nullptr, big, n_big);
    k_msd_big<<<sms, kT, 0, s>>>(offs, big, n_big, tk, vals ? tv : nullptr, keys, vals, shift);
    note_launch(5);
    if ((e = cudaMemcpyAsync(keys, tk, n * 8, cudaMemcpyDeviceToDevice, s)) != cudaSuccess) return e;
    if (vals && (e = cudaMemcpyAsync(vals, tv, n * 4, cudaMemcpyDeviceToDevice, s)) != cudaSuccess) return e;
    return cudaGetLastError();
}

}  // namespace gm
