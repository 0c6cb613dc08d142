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
//                ptrs[s] = #locations with seed < s (:84), ptrs[4^ls] = n_locs.
//                The same pass writes the lookup structures (not in the paper):
//                rank words, one u64 per 32 seeds = {occupancy bits, number of
//                occupied seeds before the word} (16 MB at ls = 13, L2-resident),
//                and the compact table {ptrs[s], count} of the occupied seeds in
//                seed order (8 B each). A chunk's first rank comes from a
//                decoupled look-back over earlier chunks. The lookup then costs
//                one 8-byte probe per query position plus one 8-byte read per
//                occupied seed, both L2-resident, instead of two reads of the
//                HBM-resident 4^ls-entry ptrs.
// Algorithmic bytes: n_locs * (8 B codes/locs written + 16 B per radix pass read+
// write) + 4 * (4^ls + 1) B ptrs written + 4^ls / 4 B rank words + 8 B per
// occupied seed.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kCodeThreads = 256;
constexpr int kFillThreads = 256;
constexpr int kChunk = 8192;                    // buckets per CTA in k_ptrs_fill
constexpr int kPer = kChunk / kFillThreads;     // 32 consecutive buckets per thread

__global__ void __launch_bounds__(kCodeThreads) k_seed_codes(const uint64_t *__restrict__ R, uint32_t ls,
                                                             uint32_t step, uint64_t k0, uint64_t n_locs,
                                                             uint32_t *__restrict__ codes,
                                                             uint32_t *__restrict__ locs) {
    const uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (k >= n_locs) return;
    const uint64_t p = (k0 + k) * step;
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

// chunk_first[c] = first index i of the sorted codes with codes[i] >= c * kChunk, for
// c in [0, n_chunks]; written by the element at each chunk boundary (no searches).
__global__ void __launch_bounds__(kCodeThreads) k_chunk_bounds(const uint32_t *__restrict__ codes, uint64_t n,
                                                               uint64_t n_chunks, uint32_t *__restrict__ first) {
    const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i > n) return;
    const uint64_t c_prev = i == 0 ? 0 : uint64_t(codes[i - 1]) / kChunk + 1;  // chunks after codes[i-1]'s
    const uint64_t c_this = i == n ? n_chunks : uint64_t(codes[i]) / kChunk;    // ... up to codes[i]'s
    for (uint64_t c = (i == 0 ? 0 : c_prev); c <= c_this && c <= n_chunks; ++c) first[c] = uint32_t(i);
}

constexpr uint64_t kStAgg = 1ull << 62;
constexpr uint64_t kStInc = 2ull << 62;
constexpr uint64_t kStMask = (1ull << 62) - 1;

// Exclusive prefix of `agg` over chunks 0..chunk-1 by decoupled look-back (warp 0 only;
// 32 predecessors per step). Chunks are numbered in launch order by a ticket.
__device__ __forceinline__ unsigned long long chunk_lookback(unsigned long long *status, uint64_t chunk,
                                                             unsigned long long agg) {
    const int lane = threadIdx.x & 31;
    volatile unsigned long long *st = status;
    if (chunk == 0) {
        if (lane == 0) st[0] = kStInc | agg;
        return 0;
    }
    if (lane == 0) st[chunk] = kStAgg | agg;
    unsigned long long excl = 0;
    int64_t c = int64_t(chunk) - 1;
    for (;;) {
        const int64_t idx = c - lane;
        const unsigned long long sv = idx >= 0 ? st[idx] : kStInc;
        const unsigned long long f = sv & ~kStMask;
        const unsigned inc_m = __ballot_sync(0xffffffffu, f == kStInc);
        const unsigned zero_m = __ballot_sync(0xffffffffu, f == 0);
        const int first_inc = inc_m ? __ffs(int(inc_m)) - 1 : 32;
        const unsigned need = first_inc >= 31 ? 0xffffffffu : ((2u << first_inc) - 1u);
        if (zero_m & need) continue;  // a predecessor has not published yet
        unsigned long long part = (lane <= first_inc) ? (sv & kStMask) : 0ull;
#pragma unroll
        for (int o = 16; o; o >>= 1) part += __shfl_down_sync(0xffffffffu, part, o);
        excl += __shfl_sync(0xffffffffu, part, 0);
        if (first_inc < 32) break;
        c -= 32;
    }
    if (lane == 0) st[chunk] = kStInc | (excl + agg);
    return excl;
}

__global__ void __launch_bounds__(kFillThreads) k_ptrs_fill(const uint32_t *__restrict__ codes, uint64_t n,
                                                            uint64_t n_buckets, uint32_t *__restrict__ ptrs,
                                                            unsigned long long *__restrict__ rankw,
                                                            uint2 *__restrict__ buckets,
                                                            const uint32_t *__restrict__ chunk_first,
                                                            unsigned long long *status, unsigned int *ticket) {
    __shared__ uint32_t cnt[kChunk + kChunk / 32];   // one pad word per 32: conflict-free rows
    __shared__ uint64_t range[2];
    __shared__ uint32_t wsum[kFillThreads / 32];
    __shared__ uint32_t wocc[kFillThreads / 32];
    __shared__ unsigned long long s_rank0;
    __shared__ unsigned int s_chunk;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid == 0) s_chunk = atomicAdd(ticket, 1u);
    __syncthreads();
    {
        const uint64_t s0 = uint64_t(s_chunk) * kChunk;
        for (int i = tid; i < kChunk + kChunk / 32; i += kFillThreads) cnt[i] = 0;
        if (tid == 0) range[0] = chunk_first[s_chunk];
        if (tid == 32) range[1] = chunk_first[s_chunk + 1];
        __syncthreads();
        const uint64_t lo = range[0], hi = range[1];
        // Alg. 1 step 1 for this chunk: seed counts
        for (uint64_t i = lo + tid; i < hi; i += kFillThreads) {
            const uint32_t d = uint32_t(codes[i] - s0);
            atomicAdd(&cnt[d + (d >> 5)], 1u);
        }
        __syncthreads();
        // Alg. 1 step 2: block-wide exclusive scan; thread t owns buckets [32t, 32t+32)
        uint32_t sum = 0, occ = 0;
#pragma unroll
        for (int j = 0; j < kPer; ++j) {
            const uint32_t c = cnt[tid * (kPer + 1) + j];
            sum += c;
            occ |= (c ? 1u : 0u) << j;
        }
        // block scans of (counts, occupied buckets) per thread
        const uint32_t nocc = __popc(occ);
        uint32_t inc = sum, inco = nocc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            const uint32_t z = __shfl_up_sync(0xffffffffu, inco, o);
            if (lane >= o) {
                inc += y;
                inco += z;
            }
        }
        if (lane == 31) {
            wsum[w] = inc;
            wocc[w] = inco;
        }
        __syncthreads();
        uint32_t pre = uint32_t(lo), preo = 0, tot_occ = 0;
        for (int i = 0; i < kFillThreads / 32; ++i) {
            if (i < w) {
                pre += wsum[i];
                preo += wocc[i];
            }
            tot_occ += wocc[i];
        }
        pre += inc - sum;
        preo += inco - nocc;
        // rank of the chunk's first occupied bucket among all occupied buckets
        if (w == 0) {
            const unsigned long long r0 = chunk_lookback(status, s_chunk, tot_occ);
            if (lane == 0) s_rank0 = r0;
        }
        __syncthreads();
        // counts -> ptrs (in place), rank words {occupancy bits, occupied buckets before
        // this word} and the compact {first slot, count} table, in bucket order
        const uint64_t rank = s_rank0 + preo;
        uint64_t r = rank;
#pragma unroll 4
        for (int j = 0; j < kPer; ++j) {
            const uint32_t c = cnt[tid * (kPer + 1) + j];
            cnt[tid * (kPer + 1) + j] = pre;
            if (c) buckets[r++] = make_uint2(pre, c);
            pre += c;
        }
        if (s0 + uint64_t(tid) * kPer < n_buckets) rankw[(s0 >> 5) + tid] = (rank << 32) | occ;
        __syncthreads();
        // coalesced write-out of the chunk's ptrs
        const uint64_t lim = n_buckets - s0 < uint64_t(kChunk) ? n_buckets - s0 : uint64_t(kChunk);
        for (int i = tid; i < int(lim); i += kFillThreads) ptrs[s0 + i] = cnt[i + (i >> 5)];
        if (s0 == 0 && tid == 0) ptrs[n_buckets] = uint32_t(n);
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

cudaError_t launch_seed_codes(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                              uint32_t *codes, uint32_t *locs, cudaStream_t s) {
    if (n_locs == 0) return cudaSuccess;
    const uint64_t blocks = (n_locs + kCodeThreads - 1) / kCodeThreads;
    k_seed_codes<<<unsigned(blocks), kCodeThreads, 0, s>>>(R, ls, step, k0, n_locs, codes, locs);
    note_launch();
    return cudaGetLastError();
}

size_t ptrs_fill_scratch_bytes(uint32_t ls) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    return chunks * 8 + 64 + (chunks + 1) * 4 + 256;
}

cudaError_t launch_ptrs_fill(const uint32_t *sorted_codes, uint64_t n_locs, uint32_t ls, uint32_t *ptrs,
                             unsigned long long *rankw, uint2 *buckets, void *scratch, cudaStream_t s) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    cudaError_t e = cudaMemsetAsync(scratch, 0, chunks * 8 + 64, s);
    if (e != cudaSuccess) return e;
    auto *status = static_cast<unsigned long long *>(scratch);
    auto *ticket = reinterpret_cast<unsigned int *>(status + chunks);
    auto *first = reinterpret_cast<uint32_t *>(reinterpret_cast<char *>(scratch) + chunks * 8 + 64);
    k_chunk_bounds<<<unsigned((n_locs + 1 + kCodeThreads - 1) / kCodeThreads), kCodeThreads, 0, s>>>(
        sorted_codes, n_locs, chunks, first);
    k_ptrs_fill<<<unsigned(chunks), kFillThreads, 0, s>>>(sorted_codes, n_locs, nb, ptrs, rankw, buckets, first,
                                                         status, ticket);
    note_launch(2);
    return cudaGetLastError();
}

}  // namespace gm
