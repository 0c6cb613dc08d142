// index.cu -- GPUMEM's lightweight index of R (Sec. III-A, Alg. 1 :102-106).
//
// Built in three steps:
//  k_seed_codes  for every sampled location p = k*step (Eq. 1, :86-90; reading R6):
//                the seed integer s = code(R, p) (2*ls bits, first base most
//                significant, A0 C1 G2 T3, :92) and the location itself.
//  radix sort    the (s, p) pairs by s, stable (radix.cu): the counting sort of
//                Alg. 1 steps 1-3 done digit by digit. Stability leaves each
//                bucket in ascending p order = Alg. 1 step 4, so `locs` is the
//                sorted value array (deterministic, checkable word for word).
//  k_ptrs_fill   over the 4^ls buckets in chunks of kChunk: per-chunk seed
//                histogram from the sorted codes (a binary search bounds the
//                chunk's slice) and a block-wide exclusive scan ->
//                ptrs[s] = #locations with seed < s (:84), ptrs[4^ls] = n_locs;
//                the same pass writes the 4^ls-bit occupancy bitmap that the
//                lookup probes first (an L2-resident filter, 8 MB at ls = 13).
// Algorithmic bytes: n_locs * (8 B codes/locs written + 16 B per radix pass read+
// write) + 4 * (4^ls + 1) B ptrs written + 4^ls / 8 B bitmap written.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kCodeThreads = 256;
constexpr int kFillThreads = 256;
constexpr int kChunk = 8192;                    // buckets per CTA in k_ptrs_fill
constexpr int kPer = kChunk / kFillThreads;     // 32 consecutive buckets per thread

__global__ void __launch_bounds__(kCodeThreads) k_seed_codes(const uint64_t *__restrict__ R, uint32_t ls,
                                                             uint32_t step, uint64_t n_locs,
                                                             uint32_t *__restrict__ codes,
                                                             uint32_t *__restrict__ locs) {
    const uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (k >= n_locs) return;
    const uint64_t p = k * step;
    codes[k] = uint32_t(win_fwd(R, p) >> (64 - 2 * ls));
    locs[k] = uint32_t(p);
}

__device__ __forceinline__ uint64_t lower_bound(const uint32_t *__restrict__ a, uint64_t n, uint64_t x) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (uint64_t(a[mid]) < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kFillThreads) k_ptrs_fill(const uint32_t *__restrict__ codes, uint64_t n,
                                                            uint64_t n_buckets, uint32_t *__restrict__ ptrs,
                                                            uint32_t *__restrict__ bitmap) {
    __shared__ uint32_t cnt[kChunk + kChunk / 32];   // one pad word per 32: conflict-free rows
    __shared__ uint64_t range[2];
    __shared__ uint32_t wsum[kFillThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    for (uint64_t s0 = uint64_t(blockIdx.x) * kChunk; s0 < n_buckets; s0 += uint64_t(gridDim.x) * kChunk) {
        for (int i = tid; i < kChunk + kChunk / 32; i += kFillThreads) cnt[i] = 0;
        if (tid == 0) range[0] = lower_bound(codes, n, s0);
        if (tid == 32) range[1] = lower_bound(codes, n, s0 + kChunk);
        __syncthreads();
        const uint64_t lo = range[0], hi = range[1];
        // Alg. 1 step 1 for this chunk: seed counts (sorted input: equal runs aggregate per warp)
        for (uint64_t b = lo; b < hi; b += kFillThreads) {
            const uint64_t i = b + tid;
            const bool valid = i < hi;
            const unsigned act = __ballot_sync(0xffffffffu, valid);
            if (valid) {
                const uint32_t d = uint32_t(codes[i] - s0);
                const unsigned peers = __match_any_sync(act, d);
                if (lane == __ffs(peers) - 1) atomicAdd(&cnt[d + (d >> 5)], __popc(peers));
            }
        }
        __syncthreads();
        // Alg. 1 step 2: block-wide exclusive scan; thread t owns buckets [32t, 32t+32)
        uint32_t v[kPer];
        uint32_t sum = 0, occ = 0;
#pragma unroll
        for (int j = 0; j < kPer; ++j) {
            v[j] = cnt[tid * (kPer + 1) + j];
            sum += v[j];
            occ |= (v[j] ? 1u : 0u) << j;
        }
        uint32_t inc = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) wsum[w] = inc;
        __syncthreads();
        uint32_t pre = uint32_t(lo);
        for (int i = 0; i < w; ++i) pre += wsum[i];
        pre += inc - sum;
#pragma unroll
        for (int j = 0; j < kPer; ++j) {
            cnt[tid * (kPer + 1) + j] = pre;
            pre += v[j];
        }
        const uint64_t bw = (s0 >> 5) + tid;                     // bitmap word of my 32 buckets
        if (s0 + uint64_t(tid) * kPer < n_buckets) bitmap[bw] = occ;
        __syncthreads();
        // coalesced write-out of the chunk's ptrs
        const uint64_t lim = n_buckets - s0 < uint64_t(kChunk) ? n_buckets - s0 : uint64_t(kChunk);
        for (int i = tid; i < int(lim); i += kFillThreads) ptrs[s0 + i] = cnt[i + (i >> 5)];
        if (blockIdx.x == 0 && tid == 0 && s0 == 0) ptrs[n_buckets] = uint32_t(n);
        __syncthreads();
    }
}

// Seed records (lookup acceleration, not part of the paper's index): for each slot k
// of locs, {p, bases R[p-16, p) with base p-1 in the low bits (00 before position 0),
// bases R[p+ls, p+ls+32) first base highest (00 past the end)} -- 16 bytes, one
// sector, so the find kernel decides a random seed hit without gathering R.
__global__ void __launch_bounds__(kCodeThreads) k_seed_recs(const uint64_t *__restrict__ R, uint32_t ls,
                                                            const uint32_t *__restrict__ locs, uint64_t n_locs,
                                                            uint4 *__restrict__ recs) {
    const uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (k >= n_locs) return;
    const uint32_t p = locs[k];
    const uint32_t left = uint32_t(win_back(R, p));
    const uint64_t right = win_fwd(R, uint64_t(p) + ls);
    recs[k] = make_uint4(p, left, uint32_t(right), uint32_t(right >> 32));
}

}  // namespace

cudaError_t launch_seed_recs(const uint64_t *R, uint32_t ls, const uint32_t *locs, uint64_t n_locs, uint4 *recs,
                             cudaStream_t s) {
    if (n_locs == 0) return cudaSuccess;
    const uint64_t blocks = (n_locs + kCodeThreads - 1) / kCodeThreads;
    k_seed_recs<<<unsigned(blocks), kCodeThreads, 0, s>>>(R, ls, locs, n_locs, recs);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_seed_codes(const uint64_t *R, uint64_t nR, uint32_t ls, uint32_t step, uint64_t n_locs,
                              uint32_t *codes, uint32_t *locs, cudaStream_t s) {
    (void)nR;
    if (n_locs == 0) return cudaSuccess;
    const uint64_t blocks = (n_locs + kCodeThreads - 1) / kCodeThreads;
    k_seed_codes<<<unsigned(blocks), kCodeThreads, 0, s>>>(R, ls, step, n_locs, codes, locs);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_ptrs_fill(const uint32_t *sorted_codes, uint64_t n_locs, uint32_t ls, uint32_t *ptrs,
                             uint32_t *bitmap, cudaStream_t s) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    const int grid = int(chunks < 65535ull ? chunks : 65535ull);
    k_ptrs_fill<<<grid, kFillThreads, 0, s>>>(sorted_codes, n_locs, nb, ptrs, bitmap);
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
