// radix.cu -- stable LSD radix sort (counting sort per 8-bit digit: histogram,
// device-wide exclusive scan, stable scatter). Used twice on the hot path:
//  * index build: the counting sort of sampled seeds over 4^ls buckets
//    (Alg. 1 steps 1-3) done digit by digit; stability makes
//    every bucket come out in ascending location order, which is what Alg. 1
//    step 4 (:102-106, per-seed sort) achieves, without a per-bucket sort;
//  * output: MEM triples into (r, q) order.
//
// Per pass over a tile of kTile = 256 x 16 items:
//   k_hist    per-tile digit counts (warp-aggregated with __match_any_sync)
//   scan      exclusive scan of the digit-major count matrix [digit][tile]
//   k_scatter stable local ranks (per-warp running counters + match_any peers),
//             then global position = scanned offset + warp offset + rank.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;                 // threads per CTA
constexpr int kItems = 16;              // items per thread
constexpr int kTile = kT * kItems;      // 4096
constexpr int kBins = 256;
constexpr int kWarps = kT / 32;
constexpr int kScanChunk = 4096;

template <class K>
__global__ void __launch_bounds__(kT) k_hist(const K *__restrict__ keys, uint64_t n, int shift,
                                             uint32_t *__restrict__ counts, uint32_t n_tiles) {
    __shared__ uint32_t h[kBins];
    for (int i = threadIdx.x; i < kBins; i += kT) h[i] = 0;
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kTile;
    const int lane = threadIdx.x & 31;
#pragma unroll 4
    for (int j = 0; j < kItems; ++j) {
        const uint64_t idx = base + uint64_t(j) * kT + threadIdx.x;
        const bool valid = idx < n;
        const unsigned act = __ballot_sync(0xffffffffu, valid);
        if (valid) {
            const uint32_t d = uint32_t(keys[idx] >> shift) & (kBins - 1);
            const unsigned peers = __match_any_sync(act, d);
            if (lane == __ffs(peers) - 1) atomicAdd(&h[d], __popc(peers));
        }
    }
    __syncthreads();
    for (int d = threadIdx.x; d < kBins; d += kT) counts[uint64_t(d) * n_tiles + blockIdx.x] = h[d];
}

template <class K, class V>
__global__ void __launch_bounds__(kT) k_scatter(const K *__restrict__ kin, const V *__restrict__ vin,
                                                K *__restrict__ kout, V *__restrict__ vout, uint64_t n,
                                                int shift, const uint32_t *__restrict__ offs,
                                                uint32_t n_tiles) {
    __shared__ uint32_t wcnt[kWarps][kBins];
    __shared__ uint32_t boff[kBins];
    for (int i = threadIdx.x; i < kWarps * kBins; i += kT) (&wcnt[0][0])[i] = 0;
    for (int d = threadIdx.x; d < kBins; d += kT) boff[d] = offs[uint64_t(d) * n_tiles + blockIdx.x];
    __syncthreads();
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t wbase = uint64_t(blockIdx.x) * kTile + uint64_t(w) * 32 * kItems;
    K k[kItems];
    V v[kItems];
    uint32_t rank[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t idx = wbase + uint64_t(j) * 32 + lane;
        const bool valid = idx < n;
        const unsigned act = __ballot_sync(0xffffffffu, valid);
        rank[j] = 0;
        if (valid) {
            k[j] = kin[idx];
            v[j] = vin[idx];
            const uint32_t d = uint32_t(k[j] >> shift) & (kBins - 1);
            const unsigned peers = __match_any_sync(act, d);
            const uint32_t base = wcnt[w][d];
            rank[j] = base + __popc(peers & lanemask_lt());
            __syncwarp(act);
            if (lane == __ffs(peers) - 1) wcnt[w][d] = base + __popc(peers);
            __syncwarp(act);
        }
    }
    __syncthreads();
    for (int d = threadIdx.x; d < kBins; d += kT) {  // exclusive scan over warps, per digit
        uint32_t run = 0;
#pragma unroll
        for (int ww = 0; ww < kWarps; ++ww) {
            const uint32_t c = wcnt[ww][d];
            wcnt[ww][d] = run;
            run += c;
        }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t idx = wbase + uint64_t(j) * 32 + lane;
        if (idx < n) {
            const uint32_t d = uint32_t(k[j] >> shift) & (kBins - 1);
            const uint64_t pos = uint64_t(boff[d]) + wcnt[w][d] + rank[j];
            kout[pos] = k[j];
            vout[pos] = v[j];
        }
    }
}

// ---- device-wide exclusive scan of uint32 (reduce, scan partials, downsweep)
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t x, uint32_t *total) {
    __shared__ uint32_t ws[kWarps];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) ws[w] = inc;
    __syncthreads();
    uint32_t wpre = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < kWarps; ++i) {
        const uint32_t c = ws[i];
        if (i < w) wpre += c;
        tot += c;
    }
    __syncthreads();
    *total = tot;
    return wpre + inc - x;
}

__global__ void __launch_bounds__(kT) k_scan_reduce(const uint32_t *__restrict__ in, uint64_t n,
                                                    uint32_t *__restrict__ part) {
    const uint64_t base = uint64_t(blockIdx.x) * kScanChunk;
    uint32_t s = 0;
    for (int i = threadIdx.x; i < kScanChunk; i += kT) {
        const uint64_t idx = base + i;
        if (idx < n) s += in[idx];
    }
    uint32_t tot;
    block_excl_scan(s, &tot);
    if (threadIdx.x == 0) part[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kT) k_scan_partials(uint32_t *part, uint64_t m) {
    // single CTA: scan m partials in place (exclusive), kT*kItems at a time
    uint32_t carry = 0;
    for (uint64_t base = 0; base < m; base += uint64_t(kT) * kItems) {
        uint32_t v[kItems];
        uint32_t s = 0;
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            const uint64_t idx = base + uint64_t(threadIdx.x) * kItems + j;
            v[j] = idx < m ? part[idx] : 0;
            s += v[j];
        }
        uint32_t tot;
        uint32_t pre = block_excl_scan(s, &tot) + carry;
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            const uint64_t idx = base + uint64_t(threadIdx.x) * kItems + j;
            if (idx < m) part[idx] = pre;
            pre += v[j];
        }
        carry += tot;
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kT) k_scan_down(const uint32_t *__restrict__ in, uint32_t *__restrict__ out,
                                                  uint64_t n, const uint32_t *__restrict__ part) {
    constexpr int per = kScanChunk / kT;  // 16 consecutive per thread
    const uint64_t base = uint64_t(blockIdx.x) * kScanChunk + uint64_t(threadIdx.x) * per;
    uint32_t v[per];
    uint32_t s = 0;
#pragma unroll
    for (int j = 0; j < per; ++j) {
        v[j] = base + j < n ? in[base + j] : 0;
        s += v[j];
    }
    uint32_t tot;
    uint32_t pre = block_excl_scan(s, &tot) + part[blockIdx.x];
#pragma unroll
    for (int j = 0; j < per; ++j) {
        if (base + j < n) out[base + j] = pre;
        pre += v[j];
    }
}

cudaError_t excl_scan(const uint32_t *in, uint32_t *out, uint64_t n, uint32_t *part, cudaStream_t s) {
    const uint64_t chunks = (n + kScanChunk - 1) / kScanChunk;
    k_scan_reduce<<<unsigned(chunks), kT, 0, s>>>(in, n, part);
    k_scan_partials<<<1, kT, 0, s>>>(part, chunks);
    k_scan_down<<<unsigned(chunks), kT, 0, s>>>(in, out, n, part);
    note_launch(3);
    return cudaGetLastError();
}

template <class K>
cudaError_t radix_sort(K *k0, uint32_t *v0, K *k1, uint32_t *v1, uint64_t n, int bits, void *scratch,
                       cudaStream_t s, bool *in_alt) {
    *in_alt = false;
    if (n <= 1 || bits <= 0) return cudaSuccess;
    const uint64_t tiles = (n + kTile - 1) / kTile;
    const uint64_t m = tiles * kBins;
    if (!scratch) return cudaErrorInvalidValue;
    uint32_t *counts = static_cast<uint32_t *>(scratch);
    uint32_t *offs = counts + m;
    uint32_t *part = offs + m;
    K *ka = k0, *kb = k1;
    uint32_t *va = v0, *vb = v1;
    for (int shift = 0; shift < bits; shift += 8) {
        k_hist<K><<<unsigned(tiles), kT, 0, s>>>(ka, n, shift, counts, uint32_t(tiles));
        note_launch();
        cudaError_t e = excl_scan(counts, offs, m, part, s);
        if (e != cudaSuccess) return e;
        k_scatter<K, uint32_t><<<unsigned(tiles), kT, 0, s>>>(ka, va, kb, vb, n, shift, offs, uint32_t(tiles));
        note_launch();
        std::swap(ka, kb);
        std::swap(va, vb);
        *in_alt = !*in_alt;
    }
    return cudaGetLastError();
}

}  // namespace

size_t radix_scratch_bytes(uint64_t n) {
    const uint64_t tiles = (n + kTile - 1) / kTile;
    const uint64_t m = tiles * kBins;
    const uint64_t chunks = (m + kScanChunk - 1) / kScanChunk;
    return (m + m + chunks + 64) * sizeof(uint32_t);
}

cudaError_t radix_sort_u32(uint32_t *k0, uint32_t *v0, uint32_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt) {
    return radix_sort<uint32_t>(k0, v0, k1, v1, n, bits, scratch, s, in_alt);
}

cudaError_t radix_sort_u64(uint64_t *k0, uint32_t *v0, uint64_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt) {
    return radix_sort<uint64_t>(k0, v0, k1, v1, n, bits, scratch, s, in_alt);
}

}  // namespace gm
