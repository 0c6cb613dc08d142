// index.cu -- GPUMEM's lightweight index of R (Sec. III-A, Alg. 1 :102-106).
//
// Built in three steps:
//  k_seed_codes  for every sampled location p = k*step (Eq. 1, :86-90; reading R6):
//                the seed integer s = code(R, p) (2*ls bits, first base most
//                significant, A0 C1 G2 T3, :92); the location itself only when no radix
//                pass runs (the first pass generates the locations from the key index).
//  radix sort    the (s, p) pairs by s, stable (radix.cu): the counting sort of
//                Alg. 1 steps 1-3 done digit by digit. Stability leaves each
//                bucket in ascending p order = Alg. 1 step 4, so `locs` is the
//                sorted value array (deterministic, checkable word for word).
//  k_ptrs_fill   over the 4^ls buckets in chunks of kChunk: per-chunk seed
//                histogram from the sorted codes (a binary search bounds the
//                chunk's slice) and a block-wide exclusive scan ->
//                ptrs[s] = #locations with seed < s (:84), ptrs[4^ls] = n_locs.
//                The same pass writes the lookup structures (not in the paper): the
//                compact table {ptrs[s], count} of the occupied seeds in seed order
//                (8 B each) and a directory over the 4^ls seeds, either
//                rank words, 8 B per 32 seeds = {occupancy bits, occupied seeds before}
//                (16 MB at ls = 13) -- the lookup is one 8-byte probe per query
//                position + one 8-byte table read per occupied seed, both L2-resident
//                when the table is small -- or, when the compact table would not stay
//                in L2, rank sectors, 16 B per 32 seeds = {records before the group,
//                occupied seeds before the group, a 2-bit saturating count per seed}:
//                the probe alone gives {first, count} unless a count in the group up
//                to the seed saturates (>= 3), so most HBM table reads disappear.
//                The table is gapped: a chunk's entries start at its first slot (entries
//                past its occupied seeds are gaps {next chunk's first slot, 0}), so no
//                scan of occupancy counts across chunks is needed (Alg. 1 as written,
//                index_alg1, keeps the dense table). Either replaces two reads of the
//                HBM-resident 4^ls-entry ptrs.
// Algorithmic bytes: n_locs * (8 B codes/locs written + 16 B per radix pass read+
// write) + 4 * (4^ls + 1) B ptrs written + 4^ls / 2 B rank sectors + 8 B per
// occupied seed.
#include <algorithm>
#include <type_traits>

#include "internal.h"
#include "device.cuh"
#include "index_common.cuh"

namespace gm {
namespace {

constexpr int kCodeThreads = 256;
#ifndef GM_DIR_CHUNK
#define GM_DIR_CHUNK 8192  // measured: 8192 vs 16384 C4 1.221 vs 1.231 ms, C5 L = 20 5.468 vs 5.499; 4096 between
#endif
constexpr int kChunk = GM_DIR_CHUNK;            // buckets per CTA in k_ptrs_fill / k_dir_fill
constexpr int kFillThreads = kChunk / 32;       // one group of 32 seeds per thread
constexpr int kPer = kChunk / kFillThreads;     // 32 consecutive buckets per thread
static_assert(kPer == 32, "k_ptrs_fill: one seed group per thread");

// four consecutive sampled locations per thread (16-byte stores), grid-stride: one
// thread per location left the GPU block-scheduling-bound (C5 L = 20: 31 M locations)
__global__ void __launch_bounds__(kCodeThreads) k_seed_codes(const uint64_t *__restrict__ R, uint32_t ls,
                                                             uint32_t step, uint64_t k0, uint64_t n_locs,
                                                             uint32_t *__restrict__ codes,
                                                             uint32_t *__restrict__ locs) {
    pdl_wait();
    const uint32_t sh = 64 - 2 * ls;
    const uint64_t n4 = (n_locs + 3) / 4;
    for (uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; g < n4; g += uint64_t(gridDim.x) * blockDim.x) {
        const uint64_t k = 4 * g;
        uint32_t c[4], p[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            p[j] = uint32_t((k0 + k + j) * step);
            c[j] = k + j < n_locs ? uint32_t(win_fwd(R, p[j]) >> sh) : 0u;
        }
        if (k + 4 <= n_locs) {
            reinterpret_cast<uint4 *>(codes)[g] = make_uint4(c[0], c[1], c[2], c[3]);
            if (locs) reinterpret_cast<uint4 *>(locs)[g] = make_uint4(p[0], p[1], p[2], p[3]);
        } else {
            for (int j = 0; j < 4 && k + j < n_locs; ++j) {
                codes[k + j] = c[j];
                if (locs) locs[k + j] = p[j];
            }
        }
    }
}

// chunk_first[c] = first index i of the sorted codes with codes[i] >= c * kChunk, for
// c in [0, n_chunks]; written by the element at each chunk boundary (no searches).
__global__ void __launch_bounds__(kCodeThreads) k_chunk_bounds(const uint32_t *__restrict__ codes, uint64_t n,
                                                               uint64_t n_chunks, uint32_t *__restrict__ first,
                                                               uint2 *__restrict__ buckets, unsigned int *hv_cnt) {
    pdl_wait();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        buckets[n] = make_uint2(uint32_t(n), 0u);  // the table's closing entry
        if (hv_cnt) hv_cnt[0] = 0;                 // the heavy-bucket list, filled by the directory fill
    }
    // element i in [0, n]: four per thread, grid-stride
    for (uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; 4 * g <= n;
         g += uint64_t(gridDim.x) * blockDim.x) {
        const uint64_t i0 = 4 * g;
        uint32_t prev = i0 ? codes[i0 - 1] : 0u;
        for (uint64_t i = i0; i < i0 + 4 && i <= n; ++i) {
            const uint32_t cur = i < n ? codes[i] : 0u;
            const uint64_t c_prev = i == 0 ? 0 : uint64_t(prev) / kChunk + 1;  // chunks after codes[i-1]'s
            const uint64_t c_this = i == n ? n_chunks : uint64_t(cur) / kChunk;  // ... up to codes[i]'s
            for (uint64_t c = (i == 0 ? 0 : c_prev); c <= c_this && c <= n_chunks; ++c) first[c] = uint32_t(i);
            prev = cur;
        }
    }
}

// rank0[c] = exclusive prefix of occ over the chunks (one CTA, contiguous runs per thread)
__global__ void __launch_bounds__(1024) k_occ_scan(const uint32_t *__restrict__ occ, uint32_t n,
                                                   uint32_t *__restrict__ rank0) {
    pdl_wait();
    __shared__ uint32_t ws[32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint32_t per = (n + 1023) / 1024;
    const uint32_t i0 = threadIdx.x * per, i1 = min(i0 + per, n);
    uint32_t sum = 0;
    for (uint32_t i = i0; i < i1; ++i) sum += occ[i];
    uint32_t inc = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) ws[w] = inc;
    __syncthreads();
    uint32_t run = inc - sum;
    for (int k = 0; k < w; ++k) run += ws[k];
    for (uint32_t i = i0; i < i1; ++i) {
        rank0[i] = run;
        run += occ[i];
    }
}

// kCounts: `codes` is instead the dense per-seed count array (Alg. 1 step 1 done with
// atomics by k_alg1_count) and chunk_first the records before each chunk.
template <bool kSect, bool kCounts = false>
__global__ void __launch_bounds__(kFillThreads) k_ptrs_fill(const uint32_t *__restrict__ codes, uint64_t n,
                                                            uint64_t n_buckets, uint32_t *__restrict__ ptrs,
                                                            unsigned long long *__restrict__ rankw,
                                                            uint4 *__restrict__ rsect,
                                                            uint2 *__restrict__ buckets,
                                                            const uint32_t *__restrict__ chunk_first,
                                                            const uint32_t *__restrict__ rank0, uint32_t rot_ls,
                                                            uint2 *__restrict__ hv_list, unsigned int *hv_cnt) {
    pdl_wait();
    extern __shared__ uint32_t cnt[];                // kChunk + kChunk / 32: a pad word per 32 (conflict-free rows)
    __shared__ uint32_t wsum[kFillThreads / 32];
    __shared__ uint32_t wocc[kFillThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t c = blockIdx.x;
    const uint64_t s0 = uint64_t(c) * kChunk;
    const uint64_t lo = chunk_first[c], hi = kCounts ? lo : chunk_first[c + 1];
    if (kCounts) {  // the chunk's counts, coalesced
        for (int i = tid; i < kChunk; i += kFillThreads)
            cnt[i + (i >> 5)] = s0 + uint64_t(i) < n_buckets ? codes[s0 + i] : 0u;
    } else {
        for (int i = tid; i < kChunk + kChunk / 32; i += kFillThreads) cnt[i] = 0;
    }
    __syncthreads();
    // Alg. 1 step 1 for this chunk: seed counts. The codes are sorted, so equal codes are
    // runs of lanes: one shared atomic per run (a hot seed, e.g. poly-A, would otherwise
    // serialise thousands of atomics on one counter)
    for (uint64_t base = lo; base < hi; base += kFillThreads) {
        const uint64_t i = base + tid;
        const bool valid = i < hi;
        const uint32_t code = valid ? codes[i] : 0xffffffffu;
        const uint32_t prev = __shfl_up_sync(0xffffffffu, code, 1);
        const bool start = valid && (lane == 0 || prev != code);
        const unsigned starts = __ballot_sync(0xffffffffu, start), vmask = __ballot_sync(0xffffffffu, valid);
        if (start) {
            const unsigned later = starts & ~((2u << lane) - 1u);
            const unsigned run = (later ? ((1u << (__ffs(int(later)) - 1)) - 1u) : 0xffffffffu) & ~((1u << lane) - 1u);
            const uint32_t d = code - uint32_t(s0);
            atomicAdd(&cnt[d + (d >> 5)], uint32_t(__popc(run & vmask)));
        }
    }
    __syncthreads();
    // Alg. 1 step 2: block-wide exclusive scan; thread t owns buckets [32t, 32t+32)
    uint32_t sum = 0, occ = 0;
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        const uint32_t x = cnt[tid * (kPer + 1) + j];
        sum += x;
        occ |= (x ? 1u : 0u) << j;
    }
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
    uint32_t pre = uint32_t(lo), preo = 0;
    for (int i = 0; i < w; ++i) {
        pre += wsum[i];
        preo += wocc[i];
    }
    pre += inc - sum;
    preo += inco - nocc;
    // counts -> ptrs (in place) and rank words {occupancy bits, occupied buckets before this
    // word} (or rank sectors)
    const uint64_t rank = uint64_t(rank0[c]) + preo;
    const uint32_t group_first = pre;
    uint64_t c2 = 0;  // 2-bit saturating count per seed of the group
#pragma unroll 4
    for (int j = 0; j < kPer; ++j) {
        const uint32_t x = cnt[tid * (kPer + 1) + j];
        cnt[tid * (kPer + 1) + j] = pre;
        if (hv_cnt && x > kHvT) {  // a heavy bucket: listed for k_hv_part
            const unsigned slot = atomicAdd(hv_cnt, 1u);
            if (slot < kHvCap) hv_list[slot] = make_uint2(pre, x);
        }
        if (!kSect && x) set_rot_occ(rankw, uint32_t(s0) + uint32_t(tid) * kPer + j, rot_ls);
        if (kSect) c2 |= uint64_t(x < 3 ? x : 3u) << (2 * j);
        pre += x;
    }
    if (s0 + uint64_t(tid) * kPer < n_buckets) {
        if (kSect) rsect[(s0 >> 5) + tid] = make_uint4(group_first, uint32_t(rank), uint32_t(c2), uint32_t(c2 >> 32));
        else rankw[2 * ((s0 >> 5) + tid)] = (rank << 32) | occ;
    }
    __syncthreads();
    // the compact {first slot, count} table in seed order, coalesced: warp w's seeds (the 32
    // groups of its lanes) take consecutive entries from its first lane's rank; lane j walks
    // seed j of each group (consecutive seeds across the lanes, consecutive entries)
    {
        uint32_t chunk_end = uint32_t(lo);
        for (int i = 0; i < kFillThreads / 32; ++i) chunk_end += wsum[i];
        uint64_t wr = __shfl_sync(0xffffffffu, rank, 0);
        const uint32_t wseed = uint32_t(w) * 32 * kPer;
        for (int g = 0; g < 32; ++g) {  // group g of the warp = lane g's seeds
            const uint32_t sl = wseed + uint32_t(g) * kPer + uint32_t(lane);  // chunk-local seed
            const uint32_t f = cnt[sl + (sl >> 5)];
            const uint32_t nx = sl + 1 < uint32_t(kChunk) ? cnt[(sl + 1) + ((sl + 1) >> 5)] : chunk_end;
            const uint32_t x = s0 + sl < n_buckets ? nx - f : 0u;
            const unsigned ob = __ballot_sync(0xffffffffu, x != 0);
            if (x) buckets[wr + __popc(ob & lanemask_lt())] = make_uint2(f, x);
            wr += __popc(ob);
        }
        // gapped table (the radix path): the chunk's entries start at its first slot and
        // run up to the next chunk's as gaps {its first slot, 0} (see tindex.cu)
        if (!kCounts) {
            uint32_t nocc = 0;
            for (int i = 0; i < kFillThreads / 32; ++i) nocc += wocc[i];
            for (uint32_t i = uint32_t(lo) + nocc + tid; i < chunk_end; i += kFillThreads)
                buckets[i] = make_uint2(chunk_end, 0u);
        }
    }
    // coalesced write-out of the chunk's ptrs, 16 bytes per store (skipped when the dense
    // table is not wanted: the lookup uses the rank directory + compact table, and
    // gpumem_index_view expands ptrs from them on demand, k_ptrs_expand)
    if (!ptrs) return;
    const uint64_t lim = n_buckets - s0 < uint64_t(kChunk) ? n_buckets - s0 : uint64_t(kChunk);
    if (lim == uint64_t(kChunk)) {
        uint4 *dst = reinterpret_cast<uint4 *>(ptrs + s0);
        for (int i = tid; i < kChunk / 4; i += kFillThreads) {
            const int b = 4 * i;  // 4 | 32: the four buckets share one padded row
            const int sp = b + (b >> 5);
            dst[i] = make_uint4(cnt[sp], cnt[sp + 1], cnt[sp + 2], cnt[sp + 3]);
        }
    } else {
        for (int i = tid; i < int(lim); i += kFillThreads) ptrs[s0 + i] = cnt[i + (i >> 5)];
    }
    if (s0 == 0 && tid == 0) ptrs[n_buckets] = uint32_t(n);
}

// The lookup directory of one chunk (kChunk seeds = kGroups groups of 32) driven by
// the chunk's sorted codes instead of its seeds: work O(elements + groups) per CTA
// rather than O(kChunk), so a sparse index (C4: ~350 sampled seeds per 8K-seed chunk)
// is not dominated by zeroing and scanning 16K empty counters (k_ptrs_fill).
//  elements  run heads (first of each distinct code) get their in-chunk rank by a
//            block scan; a run's length is the distance to the next head (runs never
//            cross a chunk), the last run of a block is finished by the next block
//            (or the chunk end). Each run -> buckets[rank0 + rank] = {first, count},
//            its occupancy bit, its 2-bit saturating count (rank sectors) and its
//            element count per group (records before the group, rank sectors);
//  groups    a block scan over the chunk's kGroups groups gives occupied seeds (and
//            records) before each group -> one rank word / rank sector per group.
constexpr int kGroups = kChunk / 32;           // 512
constexpr int kDirThreads = kGroups;
static_assert(kGroups == kDirThreads, "one group per thread in the group phase");

template <bool kSect>
__global__ void __launch_bounds__(kDirThreads) k_dir_fill(const uint32_t *__restrict__ codes, uint64_t n_buckets,
                                                          unsigned long long *__restrict__ rankw,
                                                          uint4 *__restrict__ rsect, uint2 *__restrict__ buckets,
                                                          const uint32_t *__restrict__ chunk_first,
                                                          const uint32_t *__restrict__ rank0, uint32_t rot_ls,
                                                          uint2 *__restrict__ hv_list, unsigned int *hv_cnt) {
    pdl_wait();
    __shared__ uint32_t occ[kGroups], ecnt[kGroups], c2lo[kGroups], c2hi[kGroups];
    __shared__ uint32_t hpos[kDirThreads + 1];
    __shared__ uint32_t wsum[kDirThreads / 32];
    __shared__ uint32_t s_carry, s_pend_first, s_pend_code, s_pend_rank, s_pend;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t c = blockIdx.x;
    const uint64_t s0 = uint64_t(c) * kChunk;
    const uint32_t lo = chunk_first[c], hi = chunk_first[c + 1];
    const uint32_t r0 = rank0[c];
    occ[tid] = 0;
    ecnt[tid] = 0;
    if (kSect) {
        c2lo[tid] = 0;
        c2hi[tid] = 0;
    }
    if (tid == 0) {
        s_carry = 0;
        s_pend = 0;
    }
    __syncthreads();
    // one finished run (code, first slot, count, in-chunk rank) into every structure
    auto run_out = [&](uint32_t code, uint32_t first, uint32_t count, uint32_t rank) {
        buckets[r0 + rank] = make_uint2(first, count);
        if (hv_cnt && count > kHvT) {  // a heavy bucket: listed for k_hv_part
            const unsigned slot = atomicAdd(hv_cnt, 1u);
            if (slot < kHvCap) hv_list[slot] = make_uint2(first, count);
        }
        const uint32_t sd = code - uint32_t(s0), g = sd >> 5, b = sd & 31;
        atomicOr(&occ[g], 1u << b);
        if (!kSect) set_rot_occ(rankw, code, rot_ls);
        if (kSect) {
            atomicAdd(&ecnt[g], count);
            const uint32_t sat = count < 3 ? count : 3u;
            if (b < 16) atomicOr(&c2lo[g], sat << (2 * b));
            else atomicOr(&c2hi[g], sat << (2 * (b - 16)));
        }
    };
    for (uint32_t base = lo; base < hi; base += kDirThreads) {
        const uint32_t i = base + tid;
        const bool valid = i < hi;
        const uint32_t code = valid ? codes[i] : 0u;
        const bool head = valid && (i == 0 || codes[i - 1] != code);
        const unsigned hb = __ballot_sync(0xffffffffu, head);
        if (lane == 0) wsum[w] = __popc(hb);
        __syncthreads();
        uint32_t before = 0, total = 0;
        for (int k = 0; k < kDirThreads / 32; ++k) {
            const uint32_t x = wsum[k];
            before += k < w ? x : 0u;
            total += x;
        }
        const uint32_t hr = before + __popc(hb & ((1u << lane) - 1u));  // head rank in this block
        if (head) hpos[hr] = i;
        if (tid == 0) hpos[total] = base + kDirThreads < hi ? 0xffffffffu : hi;  // block end sentinel
        __syncthreads();
        const uint32_t carry = s_carry;
        // the previous block's last run ends at this block's first head (or the chunk end)
        if (tid == 0 && s_pend) {
            const uint32_t end = total ? hpos[0] : (base + kDirThreads < hi ? 0xffffffffu : hi);
            if (end != 0xffffffffu) {
                run_out(s_pend_code, s_pend_first, end - s_pend_first, s_pend_rank);
                s_pend = 0;
            }
        }
        __syncthreads();  // the old pending run is settled before a new one is recorded
        if (head) {
            const uint32_t nxt = hpos[hr + 1];
            if (nxt != 0xffffffffu) run_out(code, i, nxt - i, carry + hr);
            else {  // the last head of a non-final block: finished later
                s_pend = 1;
                s_pend_code = code;
                s_pend_first = i;
                s_pend_rank = carry + hr;
            }
        }
        __syncthreads();
        if (tid == 0) s_carry = carry + total;
        __syncthreads();
    }
    if (tid == 0 && s_pend) run_out(s_pend_code, s_pend_first, hi - s_pend_first, s_pend_rank);
    __syncthreads();
    // gapped table: entries from the chunk's first slot (rank0 = first), gaps {hi, 0} after
    // its occupied seeds up to the next chunk's first slot (see tindex.cu)
    for (uint32_t i = r0 + s_carry + tid; i < hi; i += kDirThreads) buckets[i] = make_uint2(hi, 0u);
    // group phase: thread tid owns group tid of the chunk
    const uint32_t o = occ[tid], no = __popc(o), ne = kSect ? ecnt[tid] : 0u;
    uint32_t inc = no, ince = ne;
#pragma unroll
    for (int k = 1; k < 32; k <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, k);
        const uint32_t z = __shfl_up_sync(0xffffffffu, ince, k);
        if (lane >= k) {
            inc += y;
            ince += z;
        }
    }
    __shared__ uint32_t wo[kDirThreads / 32], we[kDirThreads / 32];
    if (lane == 31) {
        wo[w] = inc;
        we[w] = ince;
    }
    __syncthreads();
    uint32_t po = inc - no, pe = ince - ne;
    for (int k = 0; k < w; ++k) {
        po += wo[k];
        pe += we[k];
    }
    if (s0 + uint64_t(tid) * 32 < n_buckets) {
        const uint64_t g = (s0 >> 5) + tid;
        if (kSect) rsect[g] = make_uint4(lo + pe, r0 + po, c2lo[tid], c2hi[tid]);
        else rankw[2 * g] = (uint64_t(r0 + po) << 32) | o;
    }
}

// ---------------------------------------------------------------- Alg. 1 for dense indexes
// PAPER.md Alg. 1 (:102-106) as written -- per-seed counts by atomics (step 1), prefix
// sums (step 2), placement through per-seed cursors (step 3), a sort of every bucket
// (step 4). Option index_alg1; measured slower than the radix path even where the index
// is dense (C5 L = 20: 2.9 vs 1.4 ms; the counting atomics and the placement stores go
// to random 4-byte cells of the DRAM-resident 4^ls table / locs, ~1 ms each), so it is
// not the default. The arrival order of the atomics is made deterministic by step 4
// (most buckets hold 1-3 locations; a bucket over kFixMax goes to k_bucket_big).
// code(R, p) for the sampled location k; warp-aggregated atomics per equal code (hot
// seeds -- poly-A, (AC)^n -- come in runs of consecutive k).
__global__ void __launch_bounds__(kCodeThreads) k_alg1_count(const uint64_t *__restrict__ R, uint32_t ls, uint32_t step,
                                                             uint64_t k0, uint64_t n_locs, uint32_t *__restrict__ cnt,
                                                             uint32_t *__restrict__ codes, uint32_t *__restrict__ arr) {
    pdl_wait();
    const uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const bool valid = k < n_locs;
    const uint32_t code = valid ? uint32_t(win_fwd(R, (k0 + k) * step) >> (64 - 2 * ls)) : 0xffffffffu;
    const unsigned active = __ballot_sync(0xffffffffu, valid);
    if (!valid) return;
    const unsigned peers = __match_any_sync(active, code);
    const int leader = __ffs(int(peers)) - 1;
    uint32_t base = 0;
    if ((threadIdx.x & 31) == leader) base = atomicAdd(cnt + code, uint32_t(__popc(peers)));
    base = __shfl_sync(peers, base, leader);
    codes[k] = code;
    arr[k] = base + __popc(peers & lanemask_lt());
}

// per chunk of kChunk seeds: records and occupied seeds (one CTA per chunk)
__global__ void __launch_bounds__(kCodeThreads) k_cnt_chunk_sums(const uint32_t *__restrict__ cnt, uint64_t nb,
                                                                 uint32_t *__restrict__ rec, uint32_t *__restrict__ occ) {
    pdl_wait();
    __shared__ uint32_t ws[2][kCodeThreads / 32];
    const uint64_t s0 = uint64_t(blockIdx.x) * kChunk;
    uint32_t r = 0, o = 0;
    for (uint64_t i = s0 + threadIdx.x; i < s0 + kChunk && i < nb; i += kCodeThreads) {
        const uint32_t x = cnt[i];
        r += x;
        o += x ? 1u : 0u;
    }
#pragma unroll
    for (int d = 16; d; d >>= 1) {
        r += __shfl_xor_sync(0xffffffffu, r, d);
        o += __shfl_xor_sync(0xffffffffu, o, d);
    }
    if ((threadIdx.x & 31) == 0) {
        ws[0][threadIdx.x >> 5] = r;
        ws[1][threadIdx.x >> 5] = o;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tr = 0, to = 0;
        for (int k = 0; k < kCodeThreads / 32; ++k) {
            tr += ws[0][k];
            to += ws[1][k];
        }
        rec[blockIdx.x] = tr;
        occ[blockIdx.x] = to;
    }
}

// Alg. 1 step 3: locs[first(code) + arrival rank] = p, first(code) from the directory
// just built (rank sector: records before the group + the 2-bit counts below the seed,
// exact unless one saturates; rank word / saturation: the compact table).
template <bool kSect>
__global__ void __launch_bounds__(kCodeThreads) k_alg1_place(const uint32_t *__restrict__ codes,
                                                             const uint32_t *__restrict__ arr, uint64_t n_locs,
                                                             uint64_t k0, uint32_t step,
                                                             const unsigned long long *__restrict__ rankw,
                                                             const uint4 *__restrict__ rsect,
                                                             const uint2 *__restrict__ buckets,
                                                             uint32_t *__restrict__ locs) {
    pdl_wait();
    const uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (k >= n_locs) return;
    const uint32_t code = codes[k], b = code & 31;
    uint32_t first;
    if (kSect) {
        constexpr uint64_t kLo = 0x5555555555555555ull;
        const uint4 rs = __ldg(rsect + (code >> 5));
        const uint64_t c2 = (uint64_t(rs.w) << 32) | rs.z;
        const uint64_t below = b ? c2 & ((1ull << (2 * b)) - 1ull) : 0ull;
        if ((below & (below >> 1) & kLo) == 0) {  // no saturated count below: exact from the sector
            first = rs.x + uint32_t(__popcll(below & kLo) + 2 * __popcll(below & ~kLo));
        } else {
            first = __ldg(buckets + rs.y + __popcll((below | (below >> 1)) & kLo)).x;
        }
    } else {
        const unsigned long long rw = __ldg(rankw + 2 * (code >> 5));
        const uint32_t rank = uint32_t(rw >> 32) + __popc(uint32_t(rw) & ((1u << b) - 1u));
        first = __ldg(buckets + rank).x;
    }
    locs[first + arr[k]] = uint32_t((k0 + k) * step);
}

// Alg. 1 step 4: each bucket ascending. One thread per occupied seed: insertion sort up
// to kFixMax locations (nearly all); larger buckets are listed for k_bucket_big.
constexpr uint32_t kFixMax = 32;
__global__ void __launch_bounds__(kCodeThreads) k_bucket_fix(const uint2 *__restrict__ buckets,
                                                             const unsigned long long *__restrict__ rankw,
                                                             const uint4 *__restrict__ rsect, uint64_t nb,
                                                             uint32_t *__restrict__ locs, uint32_t *__restrict__ big,
                                                             unsigned int *__restrict__ n_big) {
    pdl_wait();
    // occupied seeds in total, from the last directory group
    const uint64_t g = (nb - 1) >> 5;
    uint64_t n_occ;
    if (rsect) {
        const uint4 rs = rsect[g];
        const uint64_t c2 = (uint64_t(rs.w) << 32) | rs.z;
        n_occ = rs.y + __popcll((c2 | (c2 >> 1)) & 0x5555555555555555ull);
    } else {
        const unsigned long long rw = rankw[2 * g];
        n_occ = uint32_t(rw >> 32) + __popc(uint32_t(rw));
    }
    for (uint64_t r = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < n_occ; r += uint64_t(gridDim.x) * blockDim.x) {
        const uint2 bk = buckets[r];
        if (bk.y < 2) continue;
        if (bk.y > kFixMax) {
            big[atomicAdd(n_big, 1u)] = uint32_t(r);
            continue;
        }
        uint32_t *a = locs + bk.x;
        for (uint32_t x = 1; x < bk.y; ++x) {
            const uint32_t v = a[x];
            uint32_t y = x;
            while (y > 0 && a[y - 1] > v) {
                a[y] = a[y - 1];
                --y;
            }
            a[y] = v;
        }
    }
}

constexpr uint32_t kBigSmem = 16384;
// One CTA per listed bucket: the sorting network net_sort (index_common.cuh), in shared
// memory up to kBigSmem locations, in place in global memory beyond.
__global__ void __launch_bounds__(1024) k_bucket_big(const uint2 *__restrict__ buckets, const uint32_t *__restrict__ big,
                                                     const unsigned int *__restrict__ n_big, uint32_t *__restrict__ locs) {
    pdl_wait();
    extern __shared__ uint32_t sm[];
    const unsigned nbig = *n_big;
    for (unsigned li = blockIdx.x; li < nbig; li += gridDim.x) {
        const uint2 bk = buckets[big[li]];
        uint32_t *a = locs + bk.x;
        if (bk.y <= kBigSmem) {
            for (uint32_t i = threadIdx.x; i < bk.y; i += blockDim.x) sm[i] = a[i];
            __syncthreads();
            net_sort(sm, bk.y);
            for (uint32_t i = threadIdx.x; i < bk.y; i += blockDim.x) a[i] = sm[i];
        } else {
            net_sort(a, bk.y);  // global memory: visible to the block after each barrier
        }
        __syncthreads();
    }
}

// kRecsPT records per thread (their R gathers in flight together), grid-stride
constexpr int kRecsPT = 4;
template <bool kRec8>
__global__ void __launch_bounds__(kCodeThreads) k_seed_recs(const uint64_t *__restrict__ R, uint32_t ls,
                                                            const uint32_t *__restrict__ locs, uint64_t n_locs,
                                                            void *__restrict__ recs) {
    pdl_wait();
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    for (uint64_t k0 = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; k0 < n_locs; k0 += stride * kRecsPT) {
        uint32_t p[kRecsPT];
#pragma unroll
        for (int j = 0; j < kRecsPT; ++j) {
            const uint64_t k = k0 + uint64_t(j) * stride;
            p[j] = k < n_locs ? locs[k] : 0u;
        }
#pragma unroll
        for (int j = 0; j < kRecsPT; ++j) {
            const uint64_t k = k0 + uint64_t(j) * stride;
            if (k < n_locs) seed_rec<kRec8>(R, ls, p[j], recs, k);
        }
    }
}

// ---------------------------------------------------------------- heavy buckets
// A hit whose record's left flank (kL bases before p) equals the query's (kL bases before
// q) is non-canonical whenever step <= kL and p, q >= step (decide_rec drops it: the left
// extension reaches step). A hot seed (poly-A, (AC)^n) has one left flank on nearly all
// of its locations, so for a query position with that same flank only the other records
// can give a MEM. k_hv_part finds each heavy bucket's majority flank (from 32 evenly
// spaced records) and reorders the bucket's records minority first (the records of
// p < step count as minority); k_find then spills only that prefix for such positions.
// Only the records move (find never reads locs); the MEM set is unchanged.
constexpr int kHvT_ = 512;  // threads of k_hv_part
template <bool kRec8>
__device__ __forceinline__ uint32_t rec_flank(const void *recs, uint64_t k) {
    return kRec8 ? (static_cast<const uint2 *>(recs)[k].y & 0xffffu) : static_cast<const uint4 *>(recs)[k].y;
}
template <bool kRec8>
__global__ void __launch_bounds__(kHvT_) k_hv_part(void *__restrict__ recs, uint32_t step,
                                                   const uint2 *__restrict__ hv_list, const unsigned int *hv_cnt,
                                                   uint4 *__restrict__ hv_info) {
    pdl_wait();
    using Rec = typename std::conditional<kRec8, uint2, uint4>::type;
    extern __shared__ __align__(16) unsigned char hsm[];
    Rec *buf = reinterpret_cast<Rec *>(hsm);
    const uint32_t cap = (kRec8 ? 16384u : 8192u);
    __shared__ uint32_t s_m, s_min, s_maj;
    const uint32_t n = min(hv_cnt[0], kHvCap);
    Rec *R = static_cast<Rec *>(recs);
    for (uint32_t li = blockIdx.x; li < n; li += gridDim.x) {
        const uint2 e = hv_list[li];  // {first slot, count}
        if (threadIdx.x < 32) {       // the majority flank among 32 evenly spaced records
            const uint32_t f = rec_flank<kRec8>(recs, e.x + uint64_t(e.y) * threadIdx.x / 32);
            uint32_t votes = 0;
            for (int k = 0; k < 32; ++k) votes += __shfl_sync(0xffffffffu, f, k) == f ? 1u : 0u;
            uint32_t best = (votes << 5) | (31u - threadIdx.x);  // most votes, then the lowest lane
#pragma unroll
            for (int o = 16; o; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
            const uint32_t src = 31u - (best & 31u);
            const uint32_t m = __shfl_sync(0xffffffffu, f, src);
            if (threadIdx.x == 0) {
                s_m = m;
                s_min = 0;
                s_maj = 0;
            }
        }
        __syncthreads();
        const uint32_t m = s_m;
        if (e.y > cap) {  // too large to reorder here: no skipping for this bucket
            if (threadIdx.x == 0) hv_info[li] = make_uint4(e.x, e.y, m, e.y);
            __syncthreads();
            continue;
        }
        for (uint32_t i = threadIdx.x; i < e.y; i += kHvT_) buf[i] = R[e.x + i];
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < e.y; i += kHvT_) {
            const Rec r = buf[i];
            const uint32_t f = kRec8 ? (uint32_t(r.y) & 0xffffu) : uint32_t(r.y);
            const bool minority = f != m || r.x < step;
            const uint32_t pos = minority ? atomicAdd(&s_min, 1u) : e.y - 1u - atomicAdd(&s_maj, 1u);
            GM_CHECK(pos < e.y);
            R[e.x + pos] = r;
        }
        __syncthreads();
        if (threadIdx.x == 0) hv_info[li] = make_uint4(e.x, e.y, m, s_min);
        __syncthreads();
    }
}

// one CTA: hv_info[0, n) sorted by first slot (a bitonic network in shared memory);
// hv_cnt[1] = n, or 0 when the list overflowed kHvCap (no skipping at all then)
__global__ void __launch_bounds__(1024) k_hv_sort(uint4 *__restrict__ hv_info, unsigned int *hv_cnt) {
    pdl_wait();
    __shared__ uint4 a[kHvCap];
    const uint32_t raw = hv_cnt[0];
    const uint32_t n = raw > kHvCap ? 0u : raw;
    uint32_t N = 1;
    while (N < n) N <<= 1;
    for (uint32_t i = threadIdx.x; i < N; i += 1024) a[i] = i < n ? hv_info[i] : make_uint4(~0u, 0u, 0u, 0u);
    __syncthreads();
    for (uint32_t k = 2; k <= N; k <<= 1) {
        for (uint32_t j = k >> 1; j > 0; j >>= 1) {
            for (uint32_t t = threadIdx.x; t < N / 2; t += 1024) {
                const uint32_t i = ((t & ~(j - 1)) << 1) | (t & (j - 1)), p = i + j;
                const uint4 x = a[i], y = a[p];
                if ((x.x > y.x) == ((i & k) == 0)) {
                    a[i] = y;
                    a[p] = x;
                }
            }
            __syncthreads();
        }
    }
    for (uint32_t i = threadIdx.x; i < n; i += 1024) hv_info[i] = a[i];
    if (threadIdx.x == 0) hv_cnt[1] = n;
}

}  // namespace

cudaError_t launch_seed_recs(const uint64_t *R, uint32_t ls, const uint32_t *locs, uint64_t n_locs, void *recs,
                             int rec8, cudaStream_t s) {
    if (n_locs == 0) return cudaSuccess;
    uint64_t blocks = (n_locs + kCodeThreads * kRecsPT - 1) / (kCodeThreads * kRecsPT);
    if (blocks > uint64_t(num_sms()) * 16) blocks = uint64_t(num_sms()) * 16;
    if (rec8) pdl_launch(k_seed_recs<true>, unsigned(blocks), kCodeThreads, 0, s, R, ls, locs, n_locs, recs);
    else pdl_launch(k_seed_recs<false>, unsigned(blocks), kCodeThreads, 0, s, R, ls, locs, n_locs, recs);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_seed_codes(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                              uint32_t *codes, uint32_t *locs, cudaStream_t s) {
    if (n_locs == 0) return cudaSuccess;
    uint64_t blocks = ((n_locs + 3) / 4 + kCodeThreads - 1) / kCodeThreads;
    if (blocks > uint64_t(num_sms()) * 16) blocks = uint64_t(num_sms()) * 16;
    pdl_launch(k_seed_codes, unsigned(blocks), kCodeThreads, 0, s, R, ls, step, k0, n_locs, codes, locs);
    note_launch();
    return cudaGetLastError();
}

// The paper's dense ptrs (ptrs[s] = number of sampled locations with seed
// < s, ptrs[4^ls] = n_locs) expanded from the rank directory and the compact table:
// ptrs[s] = first slot of the first occupied seed >= s = buckets[rank(s)].first, where
// rank(s) = occupied seeds below s, or n_locs past the last occupied seed.
template <bool kSect>
__global__ void __launch_bounds__(256) k_ptrs_expand(const unsigned long long *__restrict__ rankw,
                                                     const uint4 *__restrict__ rsect,
                                                     const uint2 *__restrict__ buckets, uint64_t nb, uint64_t n_locs,
                                                     uint32_t *__restrict__ ptrs) {
    pdl_wait();
    constexpr uint64_t kLo = 0x5555555555555555ull;
    auto rank_of = [&](uint64_t s, bool &in) -> uint64_t {  // occupied seeds in [0, s) (+ s's own occupancy)
        const uint32_t b = uint32_t(s & 31);
        if (kSect) {
            const uint4 r = rsect[s >> 5];
            const uint64_t c2 = (uint64_t(r.w) << 32) | r.z;
            const uint64_t below = b ? c2 & ((1ull << (2 * b)) - 1ull) : 0ull;
            in = ((c2 >> (2 * b)) & 3u) != 0;
            return r.y + __popcll((below | (below >> 1)) & kLo);
        }
        const unsigned long long r = rankw[2 * (s >> 5)];
        const uint32_t bits = uint32_t(r);
        in = (bits >> b) & 1u;
        return uint32_t(r >> 32) + __popc(bits & ((1u << b) - 1u));
    };
    bool in_last = false;
    const uint64_t n_occ = nb ? rank_of(nb - 1, in_last) + (in_last ? 1 : 0) : 0;
    for (uint64_t s = uint64_t(blockIdx.x) * 256 + threadIdx.x; s <= nb; s += uint64_t(gridDim.x) * 256) {
        uint32_t v = uint32_t(n_locs);
        if (s < nb) {
            bool in = false;
            const uint64_t r = rank_of(s, in);
            if (r < n_occ) v = buckets[r].x;
        }
        ptrs[s] = v;
    }
}

cudaError_t launch_ptrs_expand(const unsigned long long *rankw, const uint4 *rsect, const uint2 *buckets, uint32_t ls,
                               uint64_t n_locs, uint32_t *ptrs, cudaStream_t s) {
    const uint64_t nb = 1ull << (2 * ls);
    const unsigned grid = unsigned(std::min<uint64_t>((nb + 1 + 255) / 256, uint64_t(num_sms()) * 16));
    if (rsect) pdl_launch(k_ptrs_expand<true>, grid, 256, 0, s, rankw, rsect, buckets, nb, n_locs, ptrs);
    else pdl_launch(k_ptrs_expand<false>, grid, 256, 0, s, rankw, rsect, buckets, nb, n_locs, ptrs);
    note_launch();
    return cudaGetLastError();
}

size_t alg1_scratch_bytes(uint32_t ls, uint64_t n_locs) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    return nb * 4 + n_locs * 8 + (chunks + 1) * 4 * 4 + (n_locs / kFixMax + 1) * 4 + 16 * 256;
}

// Alg. 1 on packed R: codes + counts, directory + compact table (+ chunk sums and
// scans), placement, per-bucket sort. locs out; scratch >= alg1_scratch_bytes.
cudaError_t launch_index_alg1(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                              unsigned long long *rankw, uint4 *rsect, uint2 *buckets, uint32_t *locs, void *scratch,
                              cudaStream_t s) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t a = align(reinterpret_cast<uintptr_t>(scratch));
    auto *cnt = reinterpret_cast<uint32_t *>(a);
    a = align(a + nb * 4);
    auto *codes = reinterpret_cast<uint32_t *>(a);
    a = align(a + n_locs * 4);
    auto *arr = reinterpret_cast<uint32_t *>(a);
    a = align(a + n_locs * 4);
    auto *rec = reinterpret_cast<uint32_t *>(a);
    a = align(a + (chunks + 1) * 4);
    auto *occ = reinterpret_cast<uint32_t *>(a);
    a = align(a + (chunks + 1) * 4);
    auto *first = reinterpret_cast<uint32_t *>(a);
    a = align(a + (chunks + 1) * 4);
    auto *rank0 = reinterpret_cast<uint32_t *>(a);
    a = align(a + (chunks + 1) * 4);
    auto *n_big = reinterpret_cast<unsigned int *>(a);
    a = align(a + 256);
    auto *big = reinterpret_cast<uint32_t *>(a);  // occupied seeds over kFixMax (<= n_locs / kFixMax)
    cudaError_t e = cudaMemsetAsync(cnt, 0, nb * 4, s);
    if (e == cudaSuccess) e = cudaMemsetAsync(n_big, 0, 4, s);
    if (e == cudaSuccess && rankw) e = cudaMemsetAsync(rankw, 0, ((nb + 31) / 32) * 16, s);
    if (e != cudaSuccess) return e;
    const unsigned grid_k = unsigned((n_locs + kCodeThreads - 1) / kCodeThreads);
    pdl_launch(k_alg1_count, grid_k, kCodeThreads, 0, s, R, ls, step, k0, n_locs, cnt, codes, arr);
    pdl_launch(k_cnt_chunk_sums, unsigned(chunks), kCodeThreads, 0, s, cnt, nb, rec, occ);
    pdl_launch(k_occ_scan, 1, 1024, 0, s, rec, uint32_t(chunks), first);
    pdl_launch(k_occ_scan, 1, 1024, 0, s, occ, uint32_t(chunks), rank0);
    constexpr int smem = (kChunk + kChunk / 32) * 4;
    static bool attr = false;
    if (!attr) {
        e = cudaFuncSetAttribute(k_ptrs_fill<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e == cudaSuccess) e = cudaFuncSetAttribute(k_ptrs_fill<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e == cudaSuccess) e = cudaFuncSetAttribute(k_bucket_big, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kBigSmem * 4));
        if (e != cudaSuccess) return e;
        attr = true;
    }
    if (rsect)
        pdl_launch(k_ptrs_fill<true, true>, unsigned(chunks), kFillThreads, smem, s, cnt, n_locs, nb, (uint32_t *)nullptr,
                   rankw, rsect, buckets, first, rank0, ls, (uint2 *)nullptr, (unsigned int *)nullptr);
    else
        pdl_launch(k_ptrs_fill<false, true>, unsigned(chunks), kFillThreads, smem, s, cnt, n_locs, nb, (uint32_t *)nullptr,
                   rankw, rsect, buckets, first, rank0, ls, (uint2 *)nullptr, (unsigned int *)nullptr);
    if (rsect) pdl_launch(k_alg1_place<true>, grid_k, kCodeThreads, 0, s, codes, arr, n_locs, k0, step, rankw, rsect, buckets, locs);
    else pdl_launch(k_alg1_place<false>, grid_k, kCodeThreads, 0, s, codes, arr, n_locs, k0, step, rankw, rsect, buckets, locs);
    pdl_launch(k_bucket_fix, unsigned(num_sms() * 8), kCodeThreads, 0, s, buckets, rankw, rsect, nb, locs, big, n_big);
    pdl_launch(k_bucket_big, unsigned(num_sms()), 1024, size_t(kBigSmem * 4), s, buckets, big, n_big, locs);
    note_launch(9);
    return cudaGetLastError();
}

cudaError_t launch_heavy_prep(void *recs, int rec8, uint32_t step, const uint2 *hv_list, unsigned int *hv_cnt,
                              uint4 *hv_info, cudaStream_t s) {
    const size_t sm = rec8 ? 16384 * sizeof(uint2) : 8192 * sizeof(uint4);
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_hv_part<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sm));
        if (!e) e = cudaFuncSetAttribute(k_hv_part<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sm));
        if (e) return e;
        attr = true;
    }
    const unsigned grid = unsigned(num_sms());
    if (rec8) pdl_launch(k_hv_part<true>, grid, kHvT_, sm, s, recs, step, hv_list, hv_cnt, hv_info);
    else pdl_launch(k_hv_part<false>, grid, kHvT_, sm, s, recs, step, hv_list, hv_cnt, hv_info);
    pdl_launch(k_hv_sort, 1, 1024, 0, s, hv_info, hv_cnt);
    note_launch(2);
    return cudaGetLastError();
}

size_t ptrs_fill_scratch_bytes(uint32_t ls) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    return (chunks + 1) * 4 * 3 + 3 * 256;
}

cudaError_t launch_ptrs_fill(const uint32_t *sorted_codes, uint64_t n_locs, uint32_t ls, uint32_t *ptrs,
                             unsigned long long *rankw, uint4 *rsect, uint2 *buckets, void *scratch,
                             cudaStream_t s, uint2 *hv_list, unsigned int *hv_cnt) {
    const uint64_t nb = 1ull << (2 * ls);
    const uint64_t chunks = (nb + kChunk - 1) / kChunk;
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t a = align(reinterpret_cast<uintptr_t>(scratch));
    auto *first = reinterpret_cast<uint32_t *>(a);
    cudaError_t e = cudaSuccess;
    if (rankw) {  // 16 B per group: rank word + rotated occupancy (ORed in by the fill)
        e = fill_async(rankw, 0u, ((nb + 31) / 32) * 16, s);
        if (e != cudaSuccess) return e;
    }
    uint64_t bblocks = ((n_locs + 1 + 3) / 4 + kCodeThreads - 1) / kCodeThreads;
    if (bblocks > uint64_t(num_sms()) * 16) bblocks = uint64_t(num_sms()) * 16;
    pdl_launch(k_chunk_bounds, unsigned(bblocks), kCodeThreads, 0, s, sorted_codes, n_locs, chunks, first, buckets,
               hv_cnt);
    // the compact table is gapped (indexed from each chunk's first slot), so a chunk's
    // first entry is its first slot: no occupancy count and scan across chunks
    const uint32_t *rank0 = first;
    constexpr int smem = (kChunk + kChunk / 32) * 4;
    static bool attr = false;
    if (!attr) {
        e = cudaFuncSetAttribute(k_ptrs_fill<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_ptrs_fill<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    // directory + compact table only (the default): element-driven while the index is
    // sparse (C4: 0.086 -> 0.053 ms); a dense one (C5 at L = 20: 7.6K seeds per chunk,
    // 0.33 vs 0.46 ms) keeps the seed-driven fill with its ptrs write-out skipped
    if (!ptrs && n_locs * 4 < nb) {
        if (rsect)
            pdl_launch(k_dir_fill<true>, unsigned(chunks), kDirThreads, 0, s, sorted_codes, nb, rankw, rsect, buckets, first,
                       rank0, ls, hv_list, hv_cnt);
        else
            pdl_launch(k_dir_fill<false>, unsigned(chunks), kDirThreads, 0, s, sorted_codes, nb, rankw, rsect, buckets, first,
                       rank0, ls, hv_list, hv_cnt);
    } else if (rsect) {
        pdl_launch(k_ptrs_fill<true>, unsigned(chunks), kFillThreads, smem, s, sorted_codes, n_locs, nb, ptrs, rankw, rsect,
                   buckets, first, rank0, ls, hv_list, hv_cnt);
    } else {
        pdl_launch(k_ptrs_fill<false>, unsigned(chunks), kFillThreads, smem, s, sorted_codes, n_locs, nb, ptrs, rankw, rsect,
                   buckets, first, rank0, ls, hv_list, hv_cnt);
    }
    note_launch(2);
    return cudaGetLastError();
}


}  // namespace gm
