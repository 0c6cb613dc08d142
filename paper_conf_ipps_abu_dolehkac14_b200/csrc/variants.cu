// variants.cu -- NEXT-F3: maximal unique matches (MUMs) from the MEM set.
//
// PAPER.md:23 defines a MUM as a match that "appears only once in both sequences
// (i.e., unique) and cannot be extended to either directions" -- the paper's future
// work (:286). Reading used here (R21): a MUM is a MEM (r, q, len) whose
// string S = R[r, r+len) occurs exactly once in R and exactly once in Q.
//
// From the MEM set alone: if S also occurs in R at r' != r, the diagonal r' - q matches
// Q[q, q+len) for len >= L bases, so the maximal run through those cells is a MEM
// (r'', q'', len'') on a different diagonal with q'' <= q and q'' + len'' >= q + len.
// Conversely such a MEM yields another occurrence. So S is unique in R iff no other MEM's
// query interval contains [q, q+len), and unique in Q iff no other MEM's reference
// interval contains [r, r+len). (Two MEMs on one diagonal never nest: maximal runs on a
// diagonal are disjoint.)
//
// Per axis: sort (start asc, len desc) with the radix sort; interval i is contained in
// another iff the running maximum of the ends of the intervals before it reaches its own
// end, or the next interval is identical. Prefix maxima: per-block maxima, a scan of the
// block maxima, then a block-wide exclusive max-scan. The kept MEMs are compacted in
// their original (r, q) order.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;
constexpr int kPer = 8;
constexpr int kBlock = kT * kPer;  // items per CTA in the scans

__global__ void __launch_bounds__(kT) k_interval_keys(const gpumem_triple *__restrict__ t, uint64_t n, int axis,
                                                      uint64_t *__restrict__ keys, uint32_t *__restrict__ vals) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    const gpumem_triple x = t[i];
    const uint32_t start = axis ? x.r : x.q;
    keys[i] = (uint64_t(start) << 32) | uint32_t(~x.len);  // start ascending, len descending
    vals[i] = uint32_t(i);
}

__device__ __forceinline__ uint64_t end_of(uint64_t key) {
    return (key >> 32) + uint64_t(~uint32_t(key));  // start + len
}

__global__ void __launch_bounds__(kT) k_block_max(const uint64_t *__restrict__ keys, uint64_t n,
                                                  uint64_t *__restrict__ bmax) {
    pdl_wait();
    __shared__ uint64_t ws[kT / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kBlock;
    uint64_t m = 0;
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + uint64_t(j) * kT + threadIdx.x;
        if (i < n) m = max(m, end_of(keys[i]));
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) m = max(m, __shfl_down_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t r = 0;
        for (int w = 0; w < kT / 32; ++w) r = max(r, ws[w]);
        bmax[blockIdx.x] = r;
    }
}

// exclusive running maximum of bmax[0..m) in place (single CTA, sequential over chunks)
__global__ void __launch_bounds__(kT) k_scan_max(uint64_t *bmax, uint64_t m) {
    pdl_wait();
    __shared__ uint64_t ws[kT / 32];
    __shared__ uint64_t carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t base = 0; base < m; base += kT) {
        const uint64_t i = base + threadIdx.x;
        const uint64_t x = i < m ? bmax[i] : 0;
        uint64_t inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc = max(inc, y);
        }
        if (lane == 31) ws[w] = inc;
        __syncthreads();
        uint64_t pre = carry;
        for (int k = 0; k < w; ++k) pre = max(pre, ws[k]);
        const uint64_t up = __shfl_up_sync(0xffffffffu, inc, 1);
        const uint64_t excl = lane ? max(pre, up) : pre;
        uint64_t tot = carry;
        for (int k = 0; k < kT / 32; ++k) tot = max(tot, ws[k]);
        __syncthreads();
        if (i < m) bmax[i] = excl;
        if (threadIdx.x == 0) carry = tot;
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kT) k_contained(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ vals,
                                                  uint64_t n, const uint64_t *__restrict__ bprefix,
                                                  uint8_t *__restrict__ flags) {
    pdl_wait();
    __shared__ uint64_t ws[kT / 32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t base = uint64_t(blockIdx.x) * kBlock + uint64_t(threadIdx.x) * kPer;  // blocked
    uint64_t e[kPer];
    uint64_t m = 0;
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        e[j] = base + j < n ? end_of(keys[base + j]) : 0;
        m = max(m, e[j]);
    }
    uint64_t inc = m;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc = max(inc, y);
    }
    if (lane == 31) ws[w] = inc;
    __syncthreads();
    uint64_t run = bprefix[blockIdx.x];
    for (int k = 0; k < w; ++k) run = max(run, ws[k]);
    const uint64_t up = __shfl_up_sync(0xffffffffu, inc, 1);
    if (lane) run = max(run, up);
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + j;
        if (i < n) {
            bool c = run >= e[j] && i > 0;
            if (!c && i + 1 < n && keys[i + 1] == keys[i]) c = true;  // identical interval follows
            if (c) flags[vals[i]] = 1;
            run = max(run, e[j]);
        }
    }
}

__global__ void __launch_bounds__(kT) k_count_kept(const uint8_t *__restrict__ fq, const uint8_t *__restrict__ fr,
                                                   uint64_t n, uint32_t *__restrict__ counts) {
    pdl_wait();
    __shared__ uint32_t ws[kT / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kBlock;
    uint32_t c = 0;
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + uint64_t(j) * kT + threadIdx.x;
        if (i < n && !fq[i] && !fr[i]) ++c;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t r = 0;
        for (int w = 0; w < kT / 32; ++w) r += ws[w];
        counts[blockIdx.x] = r;
    }
}

// exclusive sum of counts[0..m) in place; total -> *total
__global__ void __launch_bounds__(kT) k_scan_sum(uint32_t *counts, uint64_t m, unsigned long long *total) {
    pdl_wait();
    __shared__ uint32_t ws[kT / 32];
    __shared__ unsigned long long carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t base = 0; base < m; base += kT) {
        const uint64_t i = base + threadIdx.x;
        const uint32_t x = i < m ? counts[i] : 0;
        uint32_t inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) ws[w] = inc;
        __syncthreads();
        uint32_t pre = 0, tot = 0;
        for (int k = 0; k < kT / 32; ++k) {
            if (k < w) pre += ws[k];
            tot += ws[k];
        }
        if (i < m) counts[i] = uint32_t(carry) + pre + inc - x;
        __syncthreads();
        if (threadIdx.x == 0) carry += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) *total = carry;
}

// order-preserving compaction of the kept triples (same striped order as k_count_kept)
__global__ void __launch_bounds__(kT) k_compact(const gpumem_triple *__restrict__ in, const uint8_t *__restrict__ fq,
                                                const uint8_t *__restrict__ fr, uint64_t n,
                                                const uint32_t *__restrict__ offs, gpumem_triple *__restrict__ out) {
    pdl_wait();
    __shared__ uint32_t ws[kT / 32];
    __shared__ uint32_t s_base;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_base = offs[blockIdx.x];
    __syncthreads();
    const uint64_t base = uint64_t(blockIdx.x) * kBlock;
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + uint64_t(j) * kT + threadIdx.x;
        const bool keep = i < n && !fq[i] && !fr[i];
        const unsigned bal = __ballot_sync(0xffffffffu, keep);
        if (lane == 0) ws[w] = __popc(bal);
        __syncthreads();
        uint32_t pre = 0, tot = 0;
        for (int k = 0; k < kT / 32; ++k) {
            if (k < w) pre += ws[k];
            tot += ws[k];
        }
        if (keep) out[s_base + pre + __popc(bal & lanemask_lt())] = in[i];
        __syncthreads();
        if (threadIdx.x == 0) s_base += tot;
        __syncthreads();
    }
}

unsigned nblk(uint64_t n, uint64_t per) { return unsigned((n + per - 1) / per); }

}  // namespace

size_t mum_scratch_bytes(uint64_t n) {
    const uint64_t nb = (n + kBlock - 1) / kBlock + 1;
    return n * 8 * 2 + n * 4 * 2 + n * 2 + nb * 8 + nb * 4 + radix_scratch_bytes(n) + 8 * 256;
}

cudaError_t mum_filter(const gpumem_triple *in, uint64_t n, gpumem_triple *out, unsigned long long *d_count,
                       void *scratch, cudaStream_t s) {
    cudaError_t e;
    if (n == 0) return cudaMemsetAsync(d_count, 0, 8, s);
    const uint64_t nb = (n + kBlock - 1) / kBlock;
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t c = align(reinterpret_cast<uintptr_t>(scratch));
    uint64_t *k0 = reinterpret_cast<uint64_t *>(c);
    c = align(c + n * 8);
    uint64_t *k1 = reinterpret_cast<uint64_t *>(c);
    c = align(c + n * 8);
    uint32_t *v0 = reinterpret_cast<uint32_t *>(c);
    c = align(c + n * 4);
    uint32_t *v1 = reinterpret_cast<uint32_t *>(c);
    c = align(c + n * 4);
    uint8_t *flags = reinterpret_cast<uint8_t *>(c);  // [axis][n]
    c = align(c + n * 2);
    uint64_t *bmax = reinterpret_cast<uint64_t *>(c);
    c = align(c + (nb + 1) * 8);
    uint32_t *counts = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb + 1) * 4);
    void *rs = reinterpret_cast<void *>(c);
    if ((e = cudaMemsetAsync(flags, 0, n * 2, s)) != cudaSuccess) return e;
    for (int axis = 0; axis < 2; ++axis) {  // 0: query intervals (uniqueness in R), 1: reference (in Q)
        pdl_launch(k_interval_keys, nblk(n, kT), kT, 0, s, in, n, axis, k0, v0);
        bool alt = false;
        if ((e = radix_sort_u64(k0, v0, k1, v1, n, 64, rs, s, &alt)) != cudaSuccess) return e;
        const uint64_t *ks = alt ? k1 : k0;
        const uint32_t *vs = alt ? v1 : v0;
        pdl_launch(k_block_max, unsigned(nb), kT, 0, s, ks, n, bmax);
        pdl_launch(k_scan_max, 1, kT, 0, s, bmax, nb);
        pdl_launch(k_contained, unsigned(nb), kT, 0, s, ks, vs, n, bmax, flags + uint64_t(axis) * n);
        note_launch(4);
    }
    pdl_launch(k_count_kept, unsigned(nb), kT, 0, s, flags, flags + n, n, counts);
    pdl_launch(k_scan_sum, 1, kT, 0, s, counts, nb, d_count);
    pdl_launch(k_compact, unsigned(nb), kT, 0, s, in, flags, flags + n, n, counts, out);
    note_launch(3);
    return cudaGetLastError();
}

}  // namespace gm
