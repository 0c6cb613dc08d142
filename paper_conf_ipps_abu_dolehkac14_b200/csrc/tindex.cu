// tindex.cu -- GPUMEM's index of R (Sec. III-A, Alg. 1 :102-106) built as Alg. 1
// tiled over the seed space. The 4^ls seeds are cut into 2^H bins of 2^b consecutive
// seeds (the top H bits of a code pick its bin; b = 10: 32 groups of 32 seeds); every bin
// then runs Alg. 1 on its own, on chip:
//
//  k_seed_codes  Eq. 1 sampling (p = (k0 + k) * step, :86-90) and the seed code of every
//                sampled location (index.cu);
//  radix sort    stable LSD passes over the top H code bits only (radix.cu; 2 passes for
//                ls = 13 instead of 3 over all 2 ls bits): the locations grouped by bin,
//                ascending inside each bin;
//  k_tx_bounds   the first slot of every bin (one pass over the bin-sorted codes);
//  k_tx_warp     one warp per bin of <= Cap locations (Cap 128-512 by the mean density),
//                Alg. 1 steps 1-4 for the bin (a count per seed, exclusive scan = the bin's
//                slice of ptrs :84, placement, each seed's locations ascending): a bin of
//                <= 32 locations (nearly all of a sparse index) by a radix rank from one
//                ballot per seed bit; a larger one by two stable 5-bit counting passes
//                (lane l = digit l). The bin's directory groups, {first, count} entries and
//                locs come out of the same ranks, each written once;
//  k_tx_bins     the same by a CTA (shared counters per seed, block scans) for the bins
//                past Cap (hot seeds), concurrently with k_tx_warp; a bin past kBCap runs
//                steps 3-4 in global memory;
//  k_seed_recs   the seed records in slot order (index.cu).
// Used by default for sparse indexes up to 2^20 locations (measured faster there: C1,
// C2); larger or dense ones take the radix path.
//
// The compact {first, count} table is indexed from each bin's FIRST SLOT: bin j's
// occupied seeds take table entries [off_j, off_j + occupied_j), and entries up to
// off_{j+1} are gaps {off_{j+1}, 0}; so a group's "occupied seeds before" is local to its
// bin (no scan across bins) and the dense ptrs expand exactly as before (a seed after a
// bin's last occupied one reads a gap or the next bin's first entry: its first slot).
// The table has n_locs + 1 entries (the last = {n_locs, 0}).
//
// Compared with the radix path (index.cu: all 2 ls bits sorted, then chunk bounds,
// occupancy counts and scan, the directory fill and the seed records as separate passes)
// the directory, table, locs and records are written once, by the warp/CTA owning the bin.
#include <algorithm>

#include "internal.h"
#include "device.cuh"
#include "index_common.cuh"

namespace gm {
namespace {

constexpr int kMaxH = 16;         // at most 2^16 bins (two radix passes)
constexpr int kWT = 128;          // threads of k_tx_warp (4 warps, one bin each)
constexpr int kBT = 512;          // threads of k_tx_bins
constexpr uint32_t kBCap = 4096;  // locations a k_tx_bins CTA holds in shared memory
constexpr int kRunT = 32;         // buckets up to this size: insertion sort by one thread

__host__ __device__ __forceinline__ uint32_t pad(uint32_t i) { return i + (i >> 5); }  // a pad word per 32
constexpr uint32_t kFlag = 0x80000000u;  // a first slot marked: long bucket, placed in input order

// binoff[b] = first i with codes[i] >> bbits >= b, b in [0, nbins]; written by the element
// at each bin boundary. Also: the table's closing entry {n, 0}.
__global__ void __launch_bounds__(256) k_tx_bounds(const uint32_t *__restrict__ codes, uint64_t n, uint32_t bbits,
                                                   uint32_t nbins, uint32_t *__restrict__ binoff,
                                                   uint2 *__restrict__ buckets) {
    pdl_wait();
    const uint64_t g0 = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g0 == 0) buckets[n] = make_uint2(uint32_t(n), 0u);
    for (uint64_t i = g0; i <= n; i += uint64_t(gridDim.x) * blockDim.x) {
        const uint32_t cur = i < n ? codes[i] >> bbits : nbins;
        const uint32_t b0 = i ? (codes[i - 1] >> bbits) + 1 : 0u;
        GM_CHECK(cur <= nbins);
        for (uint32_t b = b0; b <= cur; ++b) binoff[b] = uint32_t(i);
    }
}

// k_tx_warp: a bin of at most 2^10 seeds = 32 groups of 32 and at most Cap locations,
// by one warp, with work proportional to its locations (a sparse index has many more
// seeds than locations: C4 ~24 per location). The bin's locations arrive ascending
// (stable radix passes), so two stable counting passes over 5-bit digits of the
// bin-local seed -- low digit, then the group -- leave them in seed order, ascending in
// each seed: Alg. 1 steps 1-4 for the bin. Lane l holds the count / running offset of
// digit l; five ballots (one per digit bit) give every lane both its digit's lanes
// (counts) and its own element's peers (stable ranks).
template <uint32_t Cap>
struct alignas(16) WarpSmem {
    uint32_t ic[2][Cap + 8];  // a bin's codes and locations, bulk-copied (16-byte aligned
    uint32_t il[2][Cap + 8];  // superset of the range; the next bin's into the other half)
    uint32_t al[Cap];         // after pass 1: locations
    uint16_t ac[Cap];         //               their bin-local seeds
    uint32_t occ[32], c2lo[32], c2hi[32];
    unsigned long long bar[2];
};

__device__ __forceinline__ uint32_t smem_addr(const void *p) { return uint32_t(__cvta_generic_to_shared(p)); }
// lane 0: bulk-copy the bin [lo, lo + m) of codes and lin (16-byte aligned superset) into
// stage `st`, completing on its mbarrier; returns the bin's offset inside the stage
template <uint32_t Cap>
__device__ __forceinline__ uint32_t bin_fetch(WarpSmem<Cap> &S, int st, const uint32_t *codes, const uint32_t *lin,
                                              uint32_t lo, uint32_t m) {
    const uint32_t a0 = lo & ~3u, a1 = (lo + m + 3) & ~3u, bytes = (a1 - a0) * 4;
    GM_CHECK(a1 - a0 <= Cap + 8);
    if ((threadIdx.x & 31) == 0 && m) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(&S.bar[st])), "r"(2 * bytes)
                     : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         smem_addr(S.ic[st])),
                     "l"(codes + a0), "r"(bytes), "r"(smem_addr(&S.bar[st]))
                     : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         smem_addr(S.il[st])),
                     "l"(lin + a0), "r"(bytes), "r"(smem_addr(&S.bar[st]))
                     : "memory");
    }
    return lo - a0;
}
__device__ __forceinline__ void bar_wait(unsigned long long *bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(ok)
                     : "r"(smem_addr(bar)), "r"(parity)
                     : "memory");
}

// lanes whose digit equals `mine` (the caller's own digit) and whose digit equals the
// lane number, from the five digit-bit ballots
struct Match5 {
    unsigned lanes_of_lane;  // elements with digit == this lane's number
    unsigned peers;          // elements with digit == this lane's element's digit
};
__device__ __forceinline__ Match5 match5(uint32_t d, bool valid) {
    const unsigned v = __ballot_sync(0xffffffffu, valid);
    unsigned byl = v, byd = v;
    const uint32_t lane = threadIdx.x & 31;
#pragma unroll
    for (int b = 0; b < 5; ++b) {
        const unsigned bb = __ballot_sync(0xffffffffu, valid && ((d >> b) & 1u));
        byl &= ((lane >> b) & 1u) ? bb : ~bb;
        byd &= ((d >> b) & 1u) ? bb : ~bb;
    }
    return Match5{byl, byd};
}

// A bin of m <= 32 locations, one per lane (lane i: the i-th, ascending): Alg. 1 steps 1-4
// as a radix rank over the bin-local seed bits (ballots from the top bit down keep the
// lanes still equal to mine and count the smaller ones), so location i goes to slot
// rank_i; the same rank over the run heads only (one per occupied seed) gives its
// {first, count} entry, and over a lane's own number (as a group) the directory counts.
constexpr int kTB = 10;  // bin-local seed bits at most (bins of <= 2^10 seeds)
template <bool kSect>
__device__ void bin_warp_round(uint32_t bin, uint32_t lo, uint32_t m, uint32_t *occw, uint32_t *c2lo,
                               uint32_t *c2hi, const uint32_t *ic, const uint32_t *il, uint32_t bbits, uint32_t ls,
                               uint32_t *__restrict__ locs, unsigned long long *__restrict__ rankw,
                               uint4 *__restrict__ rsect, uint2 *__restrict__ buckets) {
    const uint32_t lane = threadIdx.x & 31, lt = lanemask_lt();
    const uint32_t bmask = (1u << bbits) - 1, ng = bbits >= 5 ? (1u << bbits) >> 5 : 1u;
    const bool valid = lane < m;
    const uint32_t c = valid ? ic[lane] & bmask : 0u;
    const unsigned vm = __ballot_sync(0xffffffffu, valid);
    unsigned bal[kTB];
#pragma unroll
    for (int b = 0; b < kTB; ++b) bal[b] = __ballot_sync(0xffffffffu, valid && ((c >> b) & 1u));
    // rank of value v among the lanes of `set`: (lanes with a smaller value, lanes equal)
    auto rank = [&](uint32_t v, unsigned set, int lowest, uint32_t &smaller) -> unsigned {
        smaller = 0;
#pragma unroll
        for (int b = kTB - 1; b >= 0; --b) {
            if (b < int(bbits) && b >= lowest) {
                if ((v >> b) & 1u) {
                    smaller += __popc(set & ~bal[b]);
                    set &= bal[b];
                } else {
                    set &= ~bal[b];
                }
            }
        }
        return set;
    };
    uint32_t less, hless;
    const unsigned eq = rank(c, vm, 0, less);             // my seed's locations
    const bool head = valid && (eq & lt) == 0;            // the first of them
    const unsigned hm = __ballot_sync(0xffffffffu, head);
    rank(c, hm, 0, hless);                                // occupied seeds before mine
    GM_CHECK(!valid || less + __popc(eq & lt) < m);
    if (valid) locs[lo + less + __popc(eq & lt)] = il[lane];
    const uint32_t g = c >> 5, bb = c & 31, len = __popc(eq);
    if (head) {
        GM_CHECK(hless < m && g < 32);
        buckets[lo + hless] = make_uint2(lo + less, len);
        atomicOr(&occw[g], 1u << bb);
        if (kSect) {
            const uint32_t sat = len < 3 ? len : 3u;
            if (bb < 16) atomicOr(&c2lo[g], sat << (2 * bb));
            else atomicOr(&c2hi[g], sat << (2 * (bb - 16)));
        } else {
            set_rot_occ(rankw, uint32_t(((uint64_t(bin) << bbits) >> 5) << 5) + c, ls);
        }
    }
    const uint32_t n_occ = __popc(hm);
    if (lane >= n_occ && lane < m) buckets[lo + lane] = make_uint2(lo + m, 0u);  // gaps
    __syncwarp();
    // directory: lane q = group q; locations / occupied seeds in groups before it
    uint32_t pe, po;
    rank(lane << 5, vm, 5, pe);
    rank(lane << 5, hm, 5, po);
    if (lane < ng) {
        const uint64_t gq = ((uint64_t(bin) << bbits) >> 5) + lane;
        if (kSect) rsect[gq] = make_uint4(lo + pe, lo + po, c2lo[lane], c2hi[lane]);
        else rankw[2 * gq] = (uint64_t(lo + po) << 32) | occw[lane];
    }
}

template <bool kSect, uint32_t Cap>
__device__ void bin_warp(uint32_t bin, uint32_t lo, uint32_t m, WarpSmem<Cap> &S, const uint32_t *ic, const uint32_t *il,
                         uint32_t bbits, uint32_t ls, uint32_t *__restrict__ locs,
                         unsigned long long *__restrict__ rankw, uint4 *__restrict__ rsect,
                         uint2 *__restrict__ buckets) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t bmask = (1u << bbits) - 1, ng = bbits >= 5 ? (1u << bbits) >> 5 : 1u;
    const uint32_t lt = lanemask_lt();
    S.occ[lane] = 0;
    if (kSect) {
        S.c2lo[lane] = 0;
        S.c2hi[lane] = 0;
    }
    if (m <= 32) {  // one round: ranks straight from ballots (most bins of a sparse index)
        bin_warp_round<kSect>(bin, lo, m, S.occ, S.c2lo, S.c2hi, ic, il, bbits, ls, locs, rankw, rsect, buckets);
        return;
    }
    // pass 1 (low digit), from the staged bin: count sweep, scan, placement sweep
    uint32_t cnt = 0;
    for (uint32_t r0 = 0; r0 < m; r0 += 32) {
        const uint32_t i = r0 + lane;
        const uint32_t c = i < m ? ic[i] & bmask : 0u;
        cnt += __popc(match5(c & 31, i < m).lanes_of_lane);
    }
    uint32_t inc = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= uint32_t(o)) inc += y;
    }
    uint32_t run = inc - cnt;
    for (uint32_t r0 = 0; r0 < m; r0 += 32) {
        const uint32_t i = r0 + lane;
        const bool valid = i < m;
        const uint32_t c = valid ? ic[i] & bmask : 0u;
        const Match5 mt = match5(c & 31, valid);
        const uint32_t base = __shfl_sync(0xffffffffu, run, c & 31);
        if (valid) {
            const uint32_t pos = base + __popc(mt.peers & lt);
            GM_CHECK(pos < m && m <= Cap);
            S.al[pos] = il[i];
            S.ac[pos] = uint16_t(c);
        }
        run += __popc(mt.lanes_of_lane);
    }
    __syncwarp();
    uint16_t *bc = reinterpret_cast<uint16_t *>(const_cast<uint32_t *>(ic));  // the staged codes are consumed
    // pass 2 (the group), from shared memory: lane g ends with group g's records
    // (cnt) and the records before it (pe) -- the directory's record counts
    cnt = 0;
    for (uint32_t r0 = 0; r0 < m; r0 += 32) {
        const uint32_t i = r0 + lane;
        const uint32_t c = i < m ? S.ac[i] : 0u;
        cnt += __popc(match5(c >> 5, i < m).lanes_of_lane);
    }
    inc = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= uint32_t(o)) inc += y;
    }
    const uint32_t pe = inc - cnt;
    run = pe;
    for (uint32_t r0 = 0; r0 < m; r0 += 32) {
        const uint32_t i = r0 + lane;
        const bool valid = i < m;
        const uint32_t c = valid ? S.ac[i] : 0u;
        const Match5 mt = match5(c >> 5, valid);
        const uint32_t base = __shfl_sync(0xffffffffu, run, c >> 5);
        if (valid) {
            const uint32_t pos = base + __popc(mt.peers & lt);
            GM_CHECK(pos < m);
            locs[lo + pos] = S.al[i];
            bc[pos] = uint16_t(c);
        }
        run += __popc(mt.lanes_of_lane);
    }
    __syncwarp();
    // runs of equal seeds: the last location of a run finds its head (the latest head at
    // or before it: this round's heads by ballot, else the carried one)
    uint32_t carry_rank = 0, carry_head = 0;
    const uint64_t gb = (uint64_t(bin) << bbits) >> 5;  // the bin's first directory group
    for (uint32_t r0 = 0; r0 < m; r0 += 32) {
        const uint32_t i = r0 + lane;
        const bool valid = i < m;
        const uint32_t c = valid ? bc[i] : 0u;
        const bool head = valid && (i == 0 || bc[i - 1] != c);
        const bool last = valid && (i + 1 == m || bc[i + 1] != c);
        const unsigned hb = __ballot_sync(0xffffffffu, head);
        if (last) {
            const unsigned mine = hb & (0xffffffffu >> (31 - lane));  // heads at lanes <= lane
            uint32_t h, rank;
            if (mine) {
                const int hl = 31 - __clz(int(mine));
                h = r0 + hl;
                rank = carry_rank + __popc(hb & ((1u << hl) - 1u));
            } else {
                h = carry_head;
                rank = carry_rank - 1;
            }
            const uint32_t len = i - h + 1, g = c >> 5, b = c & 31;
            GM_CHECK(rank < m && h <= i && g < 32);
            buckets[lo + rank] = make_uint2(lo + h, len);
            atomicOr(&S.occ[g], 1u << b);
            if (kSect) {
                const uint32_t sat = len < 3 ? len : 3u;
                if (b < 16) atomicOr(&S.c2lo[g], sat << (2 * b));
                else atomicOr(&S.c2hi[g], sat << (2 * (b - 16)));
            } else {
                set_rot_occ(rankw, uint32_t(gb << 5) + c, ls);
            }
        }
        if (hb) carry_head = r0 + 31 - __clz(int(hb));
        carry_rank += __popc(hb);
    }
    for (uint32_t i = carry_rank + lane; i < m; i += 32) buckets[lo + i] = make_uint2(lo + m, 0u);  // gaps
    __syncwarp();
    // directory: lane g = group g; occupied seeds before it by a warp scan
    const uint32_t occ = S.occ[lane], no = __popc(occ);
    inc = no;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= uint32_t(o)) inc += y;
    }
    if (lane < ng) {
        const uint32_t po = inc - no;
        if (kSect) rsect[gb + lane] = make_uint4(lo + pe, lo + po, S.c2lo[lane], S.c2hi[lane]);
        else rankw[2 * (gb + lane)] = (uint64_t(lo + po) << 32) | occ;
    }
    __syncwarp();  // shared memory reused by the warp's next bin
}

// Bins b = warp, warp + warps, ...: the next bin's codes / locations are bulk-copied into
// the other stage while the current one is processed (bins past Cap: k_tx_bins).
template <bool kSect, uint32_t Cap>
__global__ void __launch_bounds__(kWT, 4) k_tx_warp(const uint32_t *__restrict__ codes, const uint32_t *__restrict__ lin,
                                                    const uint32_t *__restrict__ binoff, uint32_t nbins, uint32_t bbits,
                                                    uint32_t ls, uint32_t *__restrict__ locs,
                                                    unsigned long long *__restrict__ rankw, uint4 *__restrict__ rsect,
                                                    uint2 *__restrict__ buckets) {
    pdl_wait();
    extern __shared__ __align__(16) unsigned char wsm[];
    WarpSmem<Cap> &S = reinterpret_cast<WarpSmem<Cap> *>(wsm)[threadIdx.x >> 5];
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t warps = gridDim.x * (kWT / 32);
    uint32_t bin = blockIdx.x * (kWT / 32) + (threadIdx.x >> 5);
    if (lane == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&S.bar[0])) : "memory");
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&S.bar[1])) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t lo = 0, m = 0, off = 0, uses = 0;  // uses: bit st = parity of stage st's next wait
    if (bin < nbins) {
        lo = binoff[bin];
        m = binoff[bin + 1] - lo;
        if (m <= Cap) off = bin_fetch(S, 0, codes, lin, lo, m);
    }
    for (int st = 0; bin < nbins; bin += warps, st ^= 1) {
        // the next bin's range, and its copy into the other stage (consumed two bins ago)
        const uint32_t nb = bin + warps;
        uint32_t nlo = 0, nm = 0, noff = 0;
        if (nb < nbins) {
            nlo = binoff[nb];
            nm = binoff[nb + 1] - nlo;
            __syncwarp();
            if (nm <= Cap) noff = bin_fetch(S, st ^ 1, codes, lin, nlo, nm);
        }
        if (m <= Cap) {
            if (m) {
                bar_wait(&S.bar[st], (uses >> st) & 1u);
                uses ^= 1u << st;
            }
            bin_warp<kSect, Cap>(bin, lo, m, S, S.ic[st] + off, S.il[st] + off, bbits, ls, locs, rankw, rsect,
                                 buckets);
        }
        lo = nlo;
        m = nm;
        off = noff;
    }
}

// Shared memory of a bins CTA: counters (padded), the placed locations, long buckets.
struct BinSmem {
    uint32_t *cnt;   // pad(2^b) words: counts, then first slots (after the scan), then cursors
    uint32_t *out;   // cap words: the bin's locations in seed order
};

// Alg. 1 on one bin: the m locations lin[lo, lo + m) (codes[lo, lo + m)) of the bin.
// In shared memory when m <= cap, else steps 3-4 in locs directly.
template <int kT, bool kSect>
__device__ void bin_alg1(uint32_t bin, uint32_t lo, uint32_t m, uint32_t cap, const BinSmem &S,
                         const uint32_t *__restrict__ codes, const uint32_t *__restrict__ lin, uint32_t bbits,
                         uint32_t ls, uint32_t *__restrict__ locs, unsigned long long *__restrict__ rankw,
                         uint4 *__restrict__ rsect, uint2 *__restrict__ buckets) {
    __shared__ uint32_t ws_e[kT / 32], ws_o[kT / 32], s_nlong;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t S_ = 1u << bbits;                  // seeds per bin (>= 32)
    const uint32_t kPer = S_ > uint32_t(kT) ? S_ / kT : 1u;  // consecutive seeds per thread (<= 16, | 32)
    const uint32_t bmask = S_ - 1;
    const bool in_smem = m <= cap;
    // ---- step 1: counts
    for (uint32_t i = tid; i < pad(S_); i += kT) S.cnt[i] = 0;
    __syncthreads();
    for (uint32_t i = tid; i < m; i += kT) atomicAdd(&S.cnt[pad(codes[lo + i] & bmask)], 1u);
    __syncthreads();
    // ---- step 2: exclusive scan (thread t owns seeds [t kPer, (t+1) kPer)); occupancy
    const uint32_t s0 = uint32_t(tid) * kPer;
    const uint32_t own = s0 < S_ ? kPer : 0u;  // seeds this thread owns
    uint32_t sum = 0, nocc = 0, occ = 0, todo = 0;  // todo bit j: seed s0 + j is a long bucket
    uint64_t c2 = 0;
    for (uint32_t j = 0; j < own; ++j) {
        const uint32_t x = S.cnt[pad(s0 + j)];
        sum += x;
        nocc += x ? 1u : 0u;
        const uint32_t bit = (s0 + j) & 31;
        occ |= (x ? 1u : 0u) << bit;
        c2 |= uint64_t(x < 3 ? x : 3u) << (2 * bit);
        todo |= (x > uint32_t(kRunT) ? 1u : 0u) << j;
    }
    uint32_t ie = sum, io = nocc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t ye = __shfl_up_sync(0xffffffffu, ie, o), yo = __shfl_up_sync(0xffffffffu, io, o);
        if (lane >= o) {
            ie += ye;
            io += yo;
        }
    }
    if (lane == 31) {
        ws_e[w] = ie;
        ws_o[w] = io;
    }
    __syncthreads();
    uint32_t pe = ie - sum, po = io - nocc, tot_o = 0;
    for (int k = 0; k < kT / 32; ++k) {
        pe += k < w ? ws_e[k] : 0u;
        po += k < w ? ws_o[k] : 0u;
        tot_o += ws_o[k];
    }
    // ---- the lookup directory of the bin's groups of 32 seeds: lanes [g L, g L + L) own
    //      one group (L = 32 / kPer); OR-reduce the group's bits, its first lane writes
    const uint32_t L = 32u / kPer;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        if (uint32_t(o) < L) {
            occ |= __shfl_xor_sync(0xffffffffu, occ, o);
            c2 |= __shfl_xor_sync(0xffffffffu, c2, o);
        }
    }
    const uint64_t seed0 = (uint64_t(bin) << bbits) + s0;  // global seed of this thread's first counter
    if (own && (s0 & 31) == 0) {
        const uint64_t g = seed0 >> 5;
        if (kSect) rsect[g] = make_uint4(lo + pe, lo + po, uint32_t(c2), uint32_t(c2 >> 32));
        else rankw[2 * g] = (uint64_t(lo + po) << 32) | occ;
    }
    // ---- the bin's {first, count} entries (from its first slot; gaps {lo + m, 0} after
    //      its occupied seeds) and the first slots in place of the counts (long buckets
    //      marked: placed in input order below)
    {
        uint32_t f = pe, r = lo + po;
        for (uint32_t j = 0; j < own; ++j) {
            const uint32_t x = S.cnt[pad(s0 + j)];
            S.cnt[pad(s0 + j)] = f | (x > uint32_t(kRunT) ? kFlag : 0u);
            if (x) {
                buckets[r++] = make_uint2(lo + f, x);
                if (!kSect) set_rot_occ(rankw, uint32_t(seed0) + j, ls);
            }
            f += x;
        }
        for (uint32_t i = tot_o + tid; i < m; i += kT) buckets[lo + i] = make_uint2(lo + m, 0u);
    }
    __syncthreads();
    // ---- step 3: short buckets through their cursors (first slots; each ends at the next seed's)
    uint32_t *dst = in_smem ? S.out : locs + lo;
    for (uint32_t i = tid; i < m; i += kT) {
        const uint32_t k = pad(codes[lo + i] & bmask);
        if (!(S.cnt[k] & kFlag)) {
            const uint32_t pos = atomicAdd(&S.cnt[k], 1u);
            GM_CHECK(pos < m);
            dst[pos] = lin[lo + i];
        }
    }
    // long buckets: the bin's locations arrive ascending (stable radix passes), so each is
    // placed in input order -- rank = same-seed locations before it (block-wide ballot scan)
    while (__syncthreads_or(todo != 0)) {
        if (tid == 0) s_nlong = 0xffffffffu;
        __syncthreads();
        if (todo) atomicMin(&s_nlong, s0 + uint32_t(__ffs(int(todo)) - 1));
        __syncthreads();
        const uint32_t sd = s_nlong;
        if (own && sd >= s0 && sd < s0 + own) todo &= ~(1u << (sd - s0));
        const uint32_t first = S.cnt[pad(sd)] & ~kFlag;
        uint32_t run = 0;
        for (uint32_t r0 = 0; r0 < m; r0 += kT) {
            const uint32_t i = r0 + tid;
            const bool mine = i < m && (codes[lo + i] & bmask) == sd;
            const unsigned bb = __ballot_sync(0xffffffffu, mine);
            if (lane == 0) ws_e[w] = __popc(bb);
            __syncthreads();
            uint32_t before = 0, tot = 0;
            for (int k = 0; k < kT / 32; ++k) {
                before += k < w ? ws_e[k] : 0u;
                tot += ws_e[k];
            }
            GM_CHECK(!mine || first + run + before + __popc(bb & lanemask_lt()) < m);
            if (mine) dst[first + run + before + __popc(bb & lanemask_lt())] = lin[lo + i];
            run += tot;
            __syncthreads();
        }
        if (tid == 0) S.cnt[pad(sd)] = first + run;  // a cursor at its end, like the short ones
    }
    __syncthreads();
    // ---- step 4: short buckets ascending (one thread each, insertion sort)
    {
        uint32_t f = pe;
        for (uint32_t j = 0; j < own; ++j) {
            const uint32_t end = S.cnt[pad(s0 + j)], c = end - f;
            if (c >= 2 && c <= uint32_t(kRunT)) {
                uint32_t *a = dst + f;
                for (uint32_t u = 1; u < c; ++u) {
                    const uint32_t v = a[u];
                    uint32_t y = u;
                    while (y > 0 && a[y - 1] > v) {
                        a[y] = a[y - 1];
                        --y;
                    }
                    a[y] = v;
                }
            }
            f = end;
        }
    }
    __syncthreads();
    // ---- locs of the bin, coalesced (the seed records follow in k_seed_recs)
    if (in_smem) {
        for (uint32_t i = tid; i < m; i += kT) locs[lo + i] = S.out[i];
    }
    __syncthreads();  // shared memory reused by the next bin
}

// The bins past the warps' capacity (hot seeds): each CTA picks them from its share of
// binoff and runs Alg. 1 on each in shared memory (<= kBCap locations), else with steps 3-4
// in global memory. Runs concurrently with k_tx_warp (disjoint bins).
template <bool kSect>
__global__ void __launch_bounds__(kBT, 2) k_tx_bins(const uint32_t *__restrict__ codes, const uint32_t *__restrict__ lin,
                                                    const uint32_t *__restrict__ binoff, uint32_t nbins, uint32_t bbits,
                                                    uint32_t wcap, uint32_t ls, uint32_t *__restrict__ locs,
                                                    unsigned long long *__restrict__ rankw, uint4 *__restrict__ rsect,
                                                    uint2 *__restrict__ buckets) {
    pdl_wait();
    extern __shared__ uint32_t smem[];
    __shared__ uint32_t lst[kBT], s_n;
    const uint32_t S_ = 1u << bbits;
    BinSmem S{smem, smem + pad(S_)};
    for (uint32_t base = blockIdx.x * kBT; base < nbins; base += gridDim.x * kBT) {
        if (threadIdx.x == 0) s_n = 0;
        __syncthreads();
        const uint32_t b = base + threadIdx.x;
        if (b < nbins && binoff[b + 1] - binoff[b] > wcap) lst[atomicAdd(&s_n, 1u)] = b;
        __syncthreads();
        const uint32_t n = s_n;
        for (uint32_t k = 0; k < n; ++k) {
            const uint32_t bin = lst[k];
            const uint32_t lo = binoff[bin], m = binoff[bin + 1] - lo;
            bin_alg1<kBT, kSect>(bin, lo, m, kBCap, S, codes, lin, bbits, ls, locs, rankw, rsect, buckets);
        }
        __syncthreads();
    }
}

template <bool kSect>
cudaError_t launch_warp(uint32_t cap, cudaStream_t s, const uint32_t *codes, const uint32_t *lin,
                        const uint32_t *binoff, uint32_t nbins, uint32_t bbits, uint32_t ls, uint32_t *locs,
                        unsigned long long *rankw, uint4 *rsect, uint2 *buckets) {
    auto go = [&](auto kern, size_t sm) -> cudaError_t {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sm));
        int per = 1;
        if (!e) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, kWT, sm);
        if (e) return e;
        const unsigned grid = unsigned(std::min<uint64_t>((nbins + kWT / 32 - 1) / (kWT / 32),
                                                          uint64_t(std::max(per, 1)) * num_sms()));
        return pdl_launch(kern, grid, kWT, sm, s, codes, lin, binoff, nbins, bbits, ls, locs, rankw, rsect, buckets);
    };
    if (cap == 128) return go(k_tx_warp<kSect, 128>, sizeof(WarpSmem<128>) * (kWT / 32));
    if (cap == 256) return go(k_tx_warp<kSect, 256>, sizeof(WarpSmem<256>) * (kWT / 32));
    return go(k_tx_warp<kSect, 512>, sizeof(WarpSmem<512>) * (kWT / 32));
}

}  // namespace

TiledPlan tiled_plan(uint32_t ls, uint64_t n_locs) {
    TiledPlan p{};
    const int nbits = int(2 * ls);
    // sparse indexes only (dense ones: the radix path), < 2^32 locations
    if (n_locs == 0 || n_locs >= (1ull << 32) - 1 || n_locs * 4 >= (1ull << nbits)) return p;
    // bins of 2^10 seeds = 32 groups of 32 (C2: ~8 locations per bin, C4: ~43); tiny seed
    // spaces: one bin. (2^9-seed bins, nearly all within one warp round at C4, measured
    // slower: 2^17 bins' fetch latency)
    const int b = nbits < 10 ? nbits : 10;
    if (nbits - b > kMaxH) return p;
    p.bbits = uint32_t(b);
    p.H = uint32_t(nbits - b);
    const uint64_t avg = n_locs >> p.H;  // warp capacity ~3x the mean bin
    p.wcap = avg * 3 <= 128 ? 128u : (avg * 3 <= 256 ? 256u : 512u);
    p.ok = 1;
    return p;
}

size_t tiled_scratch_bytes(const TiledPlan &p, uint64_t n_locs) {
    const uint64_t nbins = 1ull << p.H;
    return (nbins + 1) * 4 + 4 * 256 + (n_locs + 8) * 4 * 3 + radix_scratch_bytes(n_locs) + 256;
}

// One build: locs[n_locs], the directory (rankw or rsect), buckets[n_locs + 1] and the seed
// records from packed R. `scratch` >= tiled_scratch_bytes(p, n_locs).
cudaError_t launch_index_tiled(const TiledPlan &p, const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0,
                               uint64_t n_locs, unsigned long long *rankw, uint4 *rsect, uint2 *buckets, uint32_t *locs,
                               void *recs, int rec8, void *scratch, cudaStream_t s, cudaStream_t side,
                               cudaEvent_t ev_fork, cudaEvent_t ev_join) {
    if (!p.ok) return cudaErrorInvalidValue;
    const uint32_t nbins = 1u << p.H, S_ = 1u << p.bbits;
    auto align = [](uintptr_t a) { return (a + 255) & ~uintptr_t(255); };
    uintptr_t a = align(reinterpret_cast<uintptr_t>(scratch));
    auto *binoff = reinterpret_cast<uint32_t *>(a);
    a = align(a + uint64_t(nbins + 1) * 4);
    auto *c0 = reinterpret_cast<uint32_t *>(a);  // + 8 words: bulk copies read 16-byte aligned supersets
    a = align(a + (n_locs + 8) * 4);
    auto *c1 = reinterpret_cast<uint32_t *>(a);
    a = align(a + (n_locs + 8) * 4);
    auto *l1 = reinterpret_cast<uint32_t *>(a);
    a = align(a + (n_locs + 8) * 4);
    void *rscratch = reinterpret_cast<void *>(a);
    const size_t bsm = (size_t(pad(S_)) + kBCap) * 4;
    cudaError_t e = cudaSuccess;
    static bool attr = false;
    if (!attr) {
        const int maxb = int((size_t(pad(1u << 10)) + kBCap) * 4);
        e = cudaFuncSetAttribute(k_tx_bins<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, maxb);
        if (!e) e = cudaFuncSetAttribute(k_tx_bins<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, maxb);
        if (e) return e;
        attr = true;
    }
    if (rankw) {  // rank words are stored per group; the rotated-occupancy words are ORed in
        e = fill_async(rankw, 0u, ((uint64_t(1) << (2 * ls)) + 31) / 32 * 16, s);
        if (e) return e;
    }
    // codes and locations, bins by radix; the first location buffer is picked so that the
    // bin-sorted locations do not land in locs (the final ones are written there)
    const int np = radix_passes(int(2 * ls - p.bbits), n_locs);
    const bool odd = np & 1;
    uint32_t *la = odd ? locs : l1, *lb = odd ? l1 : locs;  // the result: la after even passes, lb after odd
    // the first pass generates the locations (p = (k0 + i) * step); written here only
    // when no pass runs
    e = launch_seed_codes(R, ls, step, k0, n_locs, c0, np ? nullptr : la, s);
    if (e) return e;
    bool alt = false;
    e = radix_sort_u32(c0, la, c1, lb, n_locs, int(2 * ls), rscratch, s, &alt, int(p.bbits), np ? k0 : 0,
                       np ? step : 0u);
    if (e) return e;
    const uint32_t *codes = alt ? c1 : c0;
    const uint32_t *lin = alt ? lb : la;
    if (lin == locs) return cudaErrorUnknown;  // radix_passes disagrees with the sort
    uint64_t bblocks = (n_locs + 1 + 255) / 256;
    if (bblocks > uint64_t(num_sms()) * 8) bblocks = uint64_t(num_sms()) * 8;
    pdl_launch(k_tx_bounds, unsigned(bblocks), 256, 0, s, codes, n_locs, p.bbits, nbins, binoff, buckets);
    // the hot bins (k_tx_bins) beside the warps' bins (k_tx_warp): a fork when a side
    // stream is given (pipeline capture), else one after the other
    const bool sect = rsect != nullptr;
    cudaStream_t sb = s;
    if (side && ev_fork && ev_join) {
        e = cudaEventRecord(ev_fork, s);
        if (!e) e = cudaStreamWaitEvent(side, ev_fork, 0);
        if (e) return e;
        sb = side;
    }
    int per_sm = 1;
    auto kb = sect ? k_tx_bins<true> : k_tx_bins<false>;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kb, kBT, bsm);
    if (e) return e;
    const uint32_t grid = uint32_t(std::min<uint64_t>((nbins + kBT - 1) / kBT, uint64_t(num_sms())));
    pdl_launch(kb, grid, kBT, bsm, sb, codes, lin, binoff, nbins, p.bbits, p.wcap, ls, locs, rankw, rsect, buckets);
    e = sect ? launch_warp<true>(p.wcap, s, codes, lin, binoff, nbins, p.bbits, ls, locs, rankw, rsect, buckets)
             : launch_warp<false>(p.wcap, s, codes, lin, binoff, nbins, p.bbits, ls, locs, rankw, rsect, buckets);
    if (e) return e;
    if (sb != s) {
        e = cudaEventRecord(ev_join, sb);
        if (!e) e = cudaStreamWaitEvent(s, ev_join, 0);
        if (e) return e;
    }
    e = launch_seed_recs(R, ls, locs, n_locs, recs, rec8, s);  // records in slot order
    if (e) return e;
    note_launch(3);  // k_tx_bounds, k_tx_bins, k_tx_warp (the others count themselves)
    return cudaGetLastError();
}

}  // namespace gm
