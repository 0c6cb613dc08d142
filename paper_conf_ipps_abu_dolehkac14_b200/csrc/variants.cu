// variants.cu -- NEXT-F3: maximal rare matches (MEMs whose string occurs at most k times
// in R and at most k times in Q) and, as k = 1, maximal unique matches (MUMs).
//
// PAPER.md:23 defines a MUM as a match that "appears only once in both sequences (i.e.,
// unique) and cannot be extended to either directions" and mentions "maximal rare
// matches"; :286 lists "unique and rare exact match extraction" as future work.
// Reading used here (R21/R23): a rare MEM for k >= 1 is a MEM (r, q, len)
// whose string S = R[r, r+len) occurs (overlapping occurrences counted) at most k times
// in R and at most k times in Q; k = 1 gives the MUMs.
//
// Counting from the MEM set alone: an occurrence of S in R at r' != r is a match of
// length len >= L on the diagonal r' - q covering the query interval [q, q+len), so the
// maximal run through it is a MEM (r'', q'', len'') on that diagonal with q'' <= q and
// q'' + len'' >= q + len; different occurrences lie on different diagonals, and a
// diagonal's maximal runs are disjoint, so
//     occ_R(S) = #MEMs whose query interval contains [q, q+len)   (itself included),
//     occ_Q(S) = #MEMs whose reference interval contains [r, r+len).
// Per axis: sort the intervals by (start asc, len desc) (radix.cu); the intervals that
// contain interval i are exactly the earlier ones with end >= end_i plus the identical
// ones after it. A prefix scan whose running value is the top-K ends seen so far (K a
// power of two > k; the union-of-two-top-K merge is associative) gives, for every i,
// min(K, #earlier ends >= end_i) exactly. The kept MEMs are compacted in (r, q) order.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;
constexpr int kPer = 8;
constexpr int kBlock = kT * kPer;  // items per CTA in the scans

// The K largest interval ends seen, descending; 0 = empty (every end is >= L >= 1).
template <int K>
struct TopK {
    uint32_t v[K];
};

template <int K>
__device__ __forceinline__ TopK<K> topk_empty() {
    TopK<K> t;
#pragma unroll
    for (int i = 0; i < K; ++i) t.v[i] = 0;
    return t;
}

// Top K of the union of two descending lists: max(a[i], b[K-1-i]) is a bitonic sequence
// holding the K largest; a bitonic merge network sorts it descending.
template <int K>
__device__ __forceinline__ TopK<K> topk_merge(const TopK<K> &a, const TopK<K> &b) {
    TopK<K> c;
#pragma unroll
    for (int i = 0; i < K; ++i) c.v[i] = max(a.v[i], b.v[K - 1 - i]);
#pragma unroll
    for (int j = K / 2; j > 0; j >>= 1) {
#pragma unroll
        for (int i = 0; i < K; ++i) {
            if ((i & j) == 0) {
                const uint32_t x = c.v[i], y = c.v[i + j];
                c.v[i] = max(x, y);
                c.v[i + j] = min(x, y);
            }
        }
    }
    return c;
}

template <int K>
__device__ __forceinline__ TopK<K> topk_one(uint32_t x) {
    TopK<K> t = topk_empty<K>();
    t.v[0] = x;
    return t;
}

template <int K>
__device__ __forceinline__ TopK<K> topk_shfl_up(const TopK<K> &a, int o) {
    TopK<K> t;
#pragma unroll
    for (int i = 0; i < K; ++i) t.v[i] = __shfl_up_sync(0xffffffffu, a.v[i], o);
    return t;
}

template <int K>
__device__ __forceinline__ uint32_t topk_count_ge(const TopK<K> &a, uint32_t e) {
    uint32_t c = 0;
#pragma unroll
    for (int i = 0; i < K; ++i) c += a.v[i] >= e ? 1u : 0u;
    return c;
}

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

__device__ __forceinline__ uint32_t end_of(uint64_t key) {
    return uint32_t(key >> 32) + ~uint32_t(key);  // start + len (< 2^32: a position in a sequence)
}

// Block-wide inclusive scan of per-thread top-K lists (warp shuffles, then the warp
// totals through shared memory). Returns the exclusive prefix of this thread; *total =
// the block's aggregate.
template <int K>
__device__ __forceinline__ TopK<K> block_excl_scan(const TopK<K> &mine, TopK<K> *ws, TopK<K> *total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    TopK<K> inc = mine;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const TopK<K> y = topk_shfl_up(inc, o);
        if (lane >= o) inc = topk_merge(inc, y);
    }
    if (lane == 31) ws[w] = inc;
    __syncthreads();
    TopK<K> pre = topk_empty<K>(), tot = topk_empty<K>();
    for (int k = 0; k < kT / 32; ++k) {
        if (k < w) pre = topk_merge(pre, ws[k]);
        tot = topk_merge(tot, ws[k]);
    }
    const TopK<K> up = topk_shfl_up(inc, 1);
    if (lane) pre = topk_merge(pre, up);
    *total = tot;
    __syncthreads();
    return pre;
}

template <int K>
__global__ void __launch_bounds__(kT) k_block_topk(const uint64_t *__restrict__ keys, uint64_t n,
                                                   TopK<K> *__restrict__ bagg) {
    pdl_wait();
    __shared__ TopK<K> ws[kT / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kBlock + uint64_t(threadIdx.x) * kPer;
    TopK<K> m = topk_empty<K>();
    for (int j = 0; j < kPer; ++j)
        if (base + j < n) m = topk_merge(m, topk_one<K>(end_of(keys[base + j])));
    TopK<K> tot;
    block_excl_scan(m, ws, &tot);
    if (threadIdx.x == 0) bagg[blockIdx.x] = tot;
}

// exclusive scan of the block aggregates in place (one CTA, kT blocks per round)
template <int K>
__global__ void __launch_bounds__(kT) k_scan_topk(TopK<K> *bagg, uint64_t m) {
    pdl_wait();
    __shared__ TopK<K> ws[kT / 32];
    TopK<K> carry = topk_empty<K>();
    for (uint64_t base = 0; base < m; base += kT) {
        const uint64_t i = base + threadIdx.x;
        const TopK<K> x = i < m ? bagg[i] : topk_empty<K>();
        TopK<K> tot;
        const TopK<K> pre = block_excl_scan(x, ws, &tot);
        if (i < m) bagg[i] = topk_merge(carry, pre);
        carry = topk_merge(carry, tot);
    }
}

// occ[vals[i]] = min(255, 1 + #intervals containing interval i other than itself), exact
// up to K: the earlier ends >= end_i (from the top-K prefix) + identical intervals after i.
template <int K>
__global__ void __launch_bounds__(kT) k_occurrences(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ vals,
                                                    uint64_t n, const TopK<K> *__restrict__ bprefix,
                                                    uint8_t *__restrict__ occ) {
    pdl_wait();
    __shared__ TopK<K> ws[kT / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kBlock + uint64_t(threadIdx.x) * kPer;  // blocked
    uint32_t e[kPer];
    TopK<K> m = topk_empty<K>();
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        e[j] = base + j < n ? end_of(keys[base + j]) : 0;
        if (base + j < n) m = topk_merge(m, topk_one<K>(e[j]));
    }
    TopK<K> tot;
    TopK<K> run = topk_merge(bprefix[blockIdx.x], block_excl_scan(m, ws, &tot));
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + j;
        if (i < n) {
            uint32_t c = 1 + topk_count_ge(run, e[j]);
            for (uint64_t x = i + 1; x < n && c <= uint32_t(K) && keys[x] == keys[i]; ++x) ++c;
            occ[vals[i]] = uint8_t(c < 255 ? c : 255);
            run = topk_merge(run, topk_one<K>(e[j]));
        }
    }
}

__global__ void __launch_bounds__(kT) k_count_kept(const uint8_t *__restrict__ oq, const uint8_t *__restrict__ orr,
                                                   uint64_t n, uint32_t k, uint32_t *__restrict__ counts) {
    pdl_wait();
    __shared__ uint32_t ws[kT / 32];
    const uint64_t base = uint64_t(blockIdx.x) * kBlock;
    uint32_t c = 0;
    for (int j = 0; j < kPer; ++j) {
        const uint64_t i = base + uint64_t(j) * kT + threadIdx.x;
        if (i < n && oq[i] <= k && orr[i] <= k) ++c;
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
__global__ void __launch_bounds__(kT) k_compact(const gpumem_triple *__restrict__ in, const uint8_t *__restrict__ oq,
                                                const uint8_t *__restrict__ orr, uint64_t n, uint32_t k,
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
        const bool keep = i < n && oq[i] <= k && orr[i] <= k;
        const unsigned bal = __ballot_sync(0xffffffffu, keep);
        if (lane == 0) ws[w] = __popc(bal);
        __syncthreads();
        uint32_t pre = 0, tot = 0;
        for (int x = 0; x < kT / 32; ++x) {
            if (x < w) pre += ws[x];
            tot += ws[x];
        }
        if (keep) out[s_base + pre + __popc(bal & lanemask_lt())] = in[i];
        __syncthreads();
        if (threadIdx.x == 0) s_base += tot;
        __syncthreads();
    }
}

unsigned nblk(uint64_t n, uint64_t per) { return unsigned((n + per - 1) / per); }

template <int K>
void launch_occurrences(const uint64_t *ks, const uint32_t *vs, uint64_t n, void *bagg, uint8_t *occ, cudaStream_t s) {
    const uint64_t nb = (n + kBlock - 1) / kBlock;
    auto *b = static_cast<TopK<K> *>(bagg);
    pdl_launch(k_block_topk<K>, unsigned(nb), kT, 0, s, ks, n, b);
    pdl_launch(k_scan_topk<K>, 1, kT, 0, s, b, nb);
    pdl_launch(k_occurrences<K>, unsigned(nb), kT, 0, s, ks, vs, n, static_cast<const TopK<K> *>(b), occ);
}

}  // namespace

size_t rare_scratch_bytes(uint64_t n) {
    const uint64_t nb = (n + kBlock - 1) / kBlock + 1;
    return n * 8 * 2 + n * 4 * 2 + n * 2 + nb * sizeof(TopK<kRareMaxK + 1>) + nb * 4 + radix_scratch_bytes(n) +
           8 * 256;
}

cudaError_t rare_filter(const gpumem_triple *in, uint64_t n, uint32_t k, gpumem_triple *out,
                        unsigned long long *d_count, void *scratch, cudaStream_t s) {
    cudaError_t e;
    if (k < 1 || k > uint32_t(kRareMaxK)) return cudaErrorInvalidValue;
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
    uint8_t *occ = reinterpret_cast<uint8_t *>(c);  // [axis][n]
    c = align(c + n * 2);
    void *bagg = reinterpret_cast<void *>(c);
    c = align(c + (nb + 1) * sizeof(TopK<kRareMaxK + 1>));
    uint32_t *counts = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb + 1) * 4);
    void *rs = reinterpret_cast<void *>(c);
    for (int axis = 0; axis < 2; ++axis) {  // 0: query intervals (occurrences in R), 1: reference (in Q)
        pdl_launch(k_interval_keys, nblk(n, kT), kT, 0, s, in, n, axis, k0, v0);
        bool alt = false;
        if ((e = radix_sort_u64(k0, v0, k1, v1, n, 64, rs, s, &alt)) != cudaSuccess) return e;
        const uint64_t *ks = alt ? k1 : k0;
        const uint32_t *vs = alt ? v1 : v0;
        uint8_t *o = occ + uint64_t(axis) * n;
        if (k + 1 <= 2) launch_occurrences<2>(ks, vs, n, bagg, o, s);
        else if (k + 1 <= 4) launch_occurrences<4>(ks, vs, n, bagg, o, s);
        else if (k + 1 <= 8) launch_occurrences<8>(ks, vs, n, bagg, o, s);
        else launch_occurrences<16>(ks, vs, n, bagg, o, s);
        note_launch(4);
    }
    pdl_launch(k_count_kept, unsigned(nb), kT, 0, s, occ, occ + n, n, k, counts);
    pdl_launch(k_scan_sum, 1, kT, 0, s, counts, nb, d_count);
    pdl_launch(k_compact, unsigned(nb), kT, 0, s, in, occ, occ + n, n, k, counts, out);
    note_launch(3);
    return cudaGetLastError();
}

}  // namespace gm
