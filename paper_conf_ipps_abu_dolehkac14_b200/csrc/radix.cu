// radix.cu -- stable LSD radix sort (counting sort per 8-, 9- or 10-bit digit), one
// contiguous chunk of the input per resident CTA.
// Used twice on the hot path:
//  * index build: the counting sort of sampled seeds over 4^ls buckets (Alg. 1
//    steps 1-3) done digit by digit; stability leaves every
//    bucket in ascending location order, which is what Alg. 1 step 4 (:102-106,
//    per-seed sort) achieves, without a per-bucket sort;
//  * output: MEM triples into (r, q) order.
//
// Per digit pass, three launches:
//  k_chunk_hist  -- one CTA per chunk (a contiguous run of tiles; as many chunks as the
//                   GPU holds resident scatter CTAs) counts the chunk's digits into
//                   counts[d][c] and adds them to the pass's digit totals;
//  k_chunk_scan  -- exact global offsets of every (digit, chunk):
//                   offs[d][c] = sum_{d'<d} total[d'] + sum_{c'<c} counts[d][c'];
//  k_scatter     -- same grid; CTA c walks its chunk's tiles in order with the next
//                   tile's keys/values already in flight (TMA bulk copy into the second
//                   shared-memory stage), ranks each tile stably (per-warp running digit
//                   counters + ballot peers), reorders it through shared memory and
//                   writes every digit run contiguously at its running chunk offset.
// No CTA ever waits on another (no look-back chain); the cost is one extra read of
// the keys per pass for the chunk histogram.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;  // threads per CTA of the histogram / scan kernels
constexpr int kWarps = kT / 32;
#ifndef GM_RADIX_ST
#define GM_RADIX_ST 256
#endif
constexpr int kST = GM_RADIX_ST;  // threads per CTA of k_scatter (512 x 8 items measured slower)
constexpr int kSW = kST / 32;

#ifndef GM_RADIX_ITEMS32
#define GM_RADIX_ITEMS32 16
#endif
#ifndef GM_RADIX_ITEMS64
#define GM_RADIX_ITEMS64 16
#endif
#ifndef GM_RADIX_MINB
#define GM_RADIX_MINB 2
#endif
template <class K>
struct Cfg;
template <>
struct Cfg<uint32_t> {
    static constexpr int kItems = GM_RADIX_ITEMS32;
};
template <>
struct Cfg<uint64_t> {
    static constexpr int kItems = GM_RADIX_ITEMS64;
};

template <class K>
constexpr uint64_t tile_items() {
    return uint64_t(kST) * Cfg<K>::kItems;  // one k_scatter tile
}

// Lanes of the warp holding the same digit (among lanes with valid == true), built
// from one ballot per digit bit -- full-rate, unlike __match_any_sync.
template <int RB>
__device__ __forceinline__ unsigned match_digit(uint32_t d, bool valid, int bits) {
    unsigned peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < RB; ++b) {
        if (b < bits) {
            const bool bit = (d >> b) & 1u;
            const unsigned m = __ballot_sync(0xffffffffu, bit);
            peers &= bit ? m : ~m;
        }
    }
    return peers;
}

// Chunk c of a pass: tiles [c * tpc, min((c + 1) * tpc, tiles)). With a device-resident
// count (dn != null: the sort inside a captured pipeline) n is the capacity on the host
// and live() re-derives n, tiles and tiles-per-chunk from min(*dn, capacity) on the
// device; the chunk count (the grid) stays fixed and trailing chunks may be empty.
struct Chunking {
    uint64_t n, tiles, tpc;
    uint32_t chunks;
    const unsigned long long *dn;
    __device__ Chunking live(uint64_t tile) const {
        if (!dn) return *this;
        Chunking c = *this;
        const unsigned long long x = *dn;
        c.n = x < n ? x : n;
        c.tiles = (c.n + tile - 1) / tile;
        c.tpc = (c.tiles + chunks - 1) / chunks;
        if (!c.tpc) c.tpc = 1;
        return c;
    }
    __host__ __device__ uint64_t begin(uint32_t c, uint64_t tile) const {
        const uint64_t b = uint64_t(c) * tpc * tile;
        return b < n ? b : n;
    }
    __host__ __device__ uint64_t end(uint32_t c, uint64_t tile) const {
        const uint64_t e = (uint64_t(c) + 1) * tpc * tile;
        return e < n ? e : n;
    }
};

template <class K, int RB>
__global__ void __launch_bounds__(kT) k_chunk_hist(const K *__restrict__ keys, Chunking ch0, int shift, int bits,
                                                   uint32_t *__restrict__ counts, uint32_t *__restrict__ totals) {
    pdl_wait();
    constexpr int kBins = 1 << RB;
    constexpr int DPT = kBins / kT;
    __shared__ uint32_t h[kWarps][kBins];
    const int tid = threadIdx.x, w = tid >> 5;
    const uint32_t dmask = (1u << bits) - 1;
    for (int i = tid; i < kWarps * kBins; i += kT) (&h[0][0])[i] = 0;
    __syncthreads();
    const uint32_t c = blockIdx.x;
    const Chunking ch = ch0.live(tile_items<K>());
    const uint64_t b = ch.begin(c, tile_items<K>()), e = ch.end(c, tile_items<K>());
    for (uint64_t i = b + tid; i < e; i += kT) atomicAdd(&h[w][uint32_t(keys[i] >> shift) & dmask], 1u);
    __syncthreads();
#pragma unroll
    for (int dd = 0; dd < DPT; ++dd) {
        const int d = dd * kT + tid;
        uint32_t s = 0;
#pragma unroll
        for (int ww = 0; ww < kWarps; ++ww) s += h[ww][d];
        counts[uint64_t(d) * ch.chunks + c] = s;  // digit-major
        if (s) atomicAdd(totals + d, s);
    }
}

// offs[d][c] = sum_{d' < d} totals[d'] + sum_{c' < c} counts[d][c']: every CTA scans the
// (small) digit totals, then each warp scans one digit's row of chunk counts.
template <int RB>
__global__ void __launch_bounds__(kT) k_chunk_scan(const uint32_t *__restrict__ counts,
                                                   const uint32_t *__restrict__ totals, uint32_t chunks,
                                                   uint32_t *__restrict__ offs) {
    pdl_wait();
    constexpr int kBins = 1 << RB;
    constexpr int DPT = kBins / kT;
    __shared__ uint32_t dbase[kBins];
    __shared__ uint32_t ws[kWarps * DPT];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    uint32_t tot[DPT], inc[DPT];
#pragma unroll
    for (int dd = 0; dd < DPT; ++dd) tot[dd] = inc[dd] = totals[dd * kT + tid];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
        for (int dd = 0; dd < DPT; ++dd) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc[dd], o);
            if (lane >= o) inc[dd] += y;
        }
    }
    if (lane == 31) {
#pragma unroll
        for (int dd = 0; dd < DPT; ++dd) ws[dd * kWarps + w] = inc[dd];
    }
    __syncthreads();
    uint32_t carry = 0;
#pragma unroll
    for (int dd = 0; dd < DPT; ++dd) {
        uint32_t pre = 0, seg = 0;
#pragma unroll
        for (int i = 0; i < kWarps; ++i) {
            const uint32_t x = ws[dd * kWarps + i];
            pre += i < w ? x : 0u;
            seg += x;
        }
        dbase[dd * kT + tid] = carry + pre + inc[dd] - tot[dd];
        carry += seg;
    }
    __syncthreads();
    const uint32_t d = blockIdx.x * kWarps + w;
    const uint32_t *row = counts + uint64_t(d) * chunks;
    uint32_t *orow = offs + uint64_t(d) * chunks;
    uint32_t run = dbase[d];
    for (uint32_t c0 = 0; c0 < chunks; c0 += 32) {
        const uint32_t c = c0 + lane;
        const uint32_t x = c < chunks ? row[c] : 0u;
        uint32_t s = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
            if (lane >= o) s += y;
        }
        if (c < chunks) orow[c] = run + s - x;
        run += __shfl_sync(0xffffffffu, s, 31);
    }
}

// Shared memory of k_scatter: two stage buffers, each first the TMA destination of
// one tile's keys/values and then, once they sit in registers, that tile's reorder
// buffer.
template <class K, class V, int RB>
struct alignas(128) ScatterSmem {
    K k[2][kST * Cfg<K>::kItems];
    V v[2][kST * Cfg<K>::kItems];
    uint32_t wcnt[kSW][1 << RB];
    uint32_t gofs[1 << RB];  // per digit: global position of the tile's slot 0 (mod 2^32)
    uint32_t ws[kSW * (((1 << RB) + kST - 1) / kST)];
    unsigned long long bar[2];
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return uint32_t(__cvta_generic_to_shared(p));
}

// One thread: bulk-copy `bytes` (multiple of 16) from global to shared, completing on `bar`.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, unsigned long long *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long *bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
}

template <class K, class V, int RB, bool kGen = false>
__global__ void __launch_bounds__(kST, GM_RADIX_MINB) k_scatter(const K *__restrict__ kin, const V *__restrict__ vin,
                                                  K *__restrict__ kout, V *__restrict__ vout, Chunking ch0,
                                                  int shift, int bits, const uint32_t *__restrict__ offs,
                                                  uint64_t vg_base, uint32_t vg_step) {
    // kGen: the values are generated, value of item i = (vg_base + i) * vg_step, vin unread
    // (the index sort's first pass: the sampled locations in input order)
    pdl_wait();
    constexpr int kBins = 1 << RB;
    constexpr int DPT = (kBins + kST - 1) / kST;  // digits owned per thread: tid, tid + kST, ... (< kBins)
    constexpr int kItems = Cfg<K>::kItems;
    constexpr int kTile = kST * kItems;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    ScatterSmem<K, V, RB> &S = *reinterpret_cast<ScatterSmem<K, V, RB> *>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t dmask = (1u << bits) - 1;
    const uint32_t c = blockIdx.x;
    const Chunking ch = ch0.live(kTile);
    const uint64_t cb = ch.begin(c, kTile), ce = ch.end(c, kTile);
    const uint32_t n_t = uint32_t((ce - cb + kTile - 1) / kTile);
    const uint32_t n_full = uint32_t((ce - cb) / kTile);  // tiles moved by TMA; a ragged tail is loaded directly

    auto issue = [&](uint32_t t, int stage) {  // thread 0
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                     :: "r"(smem_u32(&S.bar[stage])), "r"(uint32_t(kTile * (sizeof(K) + (kGen ? 0 : sizeof(V)))))
                     : "memory");
        bulk_g2s(S.k[stage], kin + cb + uint64_t(t) * kTile, kTile * sizeof(K), &S.bar[stage]);
        if (!kGen) bulk_g2s(S.v[stage], vin + cb + uint64_t(t) * kTile, kTile * sizeof(V), &S.bar[stage]);
    };
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&S.bar[0])) : "memory");
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&S.bar[1])) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        if (n_full > 0) issue(0, 0);
    }
    uint32_t gbase[DPT];  // running global offset of each owned digit in this chunk
#pragma unroll
    for (int dd = 0; dd < DPT; ++dd)
        gbase[dd] = dd * kST + tid < kBins ? offs[uint64_t(dd * kST + tid) * ch.chunks + c] : 0u;
    __syncthreads();

    for (uint32_t t = 0; t < n_t; ++t) {
        const int sg = t & 1;
        if (tid == 0 && t + 1 < n_full) issue(t + 1, sg ^ 1);  // buffer sg^1 was released at the end of tile t-1
        for (int i = tid; i < kSW * kBins; i += kST) (&S.wcnt[0][0])[i] = 0;
        const uint64_t base = cb + uint64_t(t) * kTile;
        const uint32_t tile_n = uint32_t(min(uint64_t(kTile), ce - base));

        // ---- items into registers (warp-striped rounds keep input order = (warp, round, lane))
        K k[kItems];
        V v[kItems];
        uint32_t rank[kItems];
        const uint32_t wofs = uint32_t(w) * 32 * kItems;
        if (t < n_full) {
            mbar_wait(&S.bar[sg], (t >> 1) & 1);
#pragma unroll
            for (int j = 0; j < kItems; ++j) {
                k[j] = S.k[sg][wofs + j * 32 + lane];
                v[j] = kGen ? V((vg_base + base + wofs + j * 32 + lane) * vg_step) : S.v[sg][wofs + j * 32 + lane];
            }
        } else {
#pragma unroll
            for (int j = 0; j < kItems; ++j) {
                const uint32_t li = wofs + j * 32 + lane;
                k[j] = li < tile_n ? kin[base + li] : K(0);
                v[j] = li < tile_n ? (kGen ? V((vg_base + base + li) * vg_step) : vin[base + li]) : V(0);
            }
        }
        __syncthreads();  // wcnt zeroed

        // ---- stable ranks: per-warp running digit counters + ballot peers (all ballots
        //      first: they are independent, only the counter updates are sequential)
        unsigned peers[kItems];
#pragma unroll
        for (int j = 0; j < kItems; ++j)
            peers[j] = match_digit<RB>(uint32_t(k[j] >> shift) & dmask, wofs + j * 32 + lane < tile_n, bits);
#ifndef GM_RADIX_ATOMIC_RANK
#define GM_RADIX_ATOMIC_RANK 1
#endif
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            const bool valid = wofs + j * 32 + lane < tile_n;
            const uint32_t d = uint32_t(k[j] >> shift) & dmask;
#if GM_RADIX_ATOMIC_RANK
            // the leader of each digit group reserves the group's slots with one shared
            // atomicAdd (rounds of one warp issue in program order: ranks stay stable) and
            // hands the base to its peers
            const int leader = __ffs(peers[j]) - 1;
            uint32_t b0 = 0;
            if (valid && lane == leader) b0 = atomicAdd(&S.wcnt[w][d], uint32_t(__popc(peers[j])));
            b0 = __shfl_sync(0xffffffffu, b0, valid ? leader : lane);
            rank[j] = b0 + __popc(peers[j] & lanemask_lt());
#else
            const uint32_t b0 = valid ? S.wcnt[w][d] : 0u;
            rank[j] = b0 + __popc(peers[j] & lanemask_lt());
            __syncwarp();
            if (valid && lane == __ffs(peers[j]) - 1) S.wcnt[w][d] = b0 + __popc(peers[j]);
            __syncwarp();
#endif
        }
        __syncthreads();

        // ---- per digit: tile count, tile-local exclusive offset (block scan); then each
        //      warp's slot base in the reorder buffer and the tile-to-global offset
        uint32_t cnt[DPT], inc[DPT];
#pragma unroll
        for (int dd = 0; dd < DPT; ++dd) {
            uint32_t c0 = 0;
            if (dd * kST + tid < kBins) {
#pragma unroll
                for (int ww = 0; ww < kSW; ++ww) c0 += S.wcnt[ww][dd * kST + tid];
            }
            cnt[dd] = inc[dd] = c0;
        }
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
            for (int dd = 0; dd < DPT; ++dd) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, inc[dd], o);
                if (lane >= o) inc[dd] += y;
            }
        }
        if (lane == 31) {
#pragma unroll
            for (int dd = 0; dd < DPT; ++dd) S.ws[dd * kSW + w] = inc[dd];
        }
        __syncthreads();
        {
            uint32_t carry = 0;
#pragma unroll
            for (int dd = 0; dd < DPT; ++dd) {
                uint32_t pre = 0, seg = 0;
#pragma unroll
                for (int i = 0; i < kSW; ++i) {
                    const uint32_t x = S.ws[dd * kSW + i];
                    pre += i < w ? x : 0u;
                    seg += x;
                }
                const uint32_t excl = carry + pre + inc[dd] - cnt[dd];
                carry += seg;
                const uint32_t d = dd * kST + tid;
                if (d < kBins) {
                    uint32_t run = excl;
#pragma unroll
                    for (int ww = 0; ww < kSW; ++ww) {
                        const uint32_t x = S.wcnt[ww][d];
                        S.wcnt[ww][d] = run;
                        run += x;
                    }
                    S.gofs[d] = gbase[dd] - excl;  // slot i of digit d goes to gofs[d] + i (mod 2^32)
                    gbase[dd] += cnt[dd];
                }
            }
        }
        __syncthreads();

        // ---- reorder into digit order through this tile's (consumed) stage buffer
        K *rk = S.k[sg];
        V *rv = S.v[sg];
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            if (wofs + j * 32 + lane < tile_n) {
                const uint32_t lp = S.wcnt[w][uint32_t(k[j] >> shift) & dmask] + rank[j];
                rk[lp] = k[j];
                rv[lp] = v[j];
            }
        }
        __syncthreads();
        // ---- coalesced write-out: consecutive slots of one digit go to consecutive addresses
        auto put = [&](uint32_t i) {
            const K kk = rk[i];
            const uint32_t g = S.gofs[uint32_t(kk >> shift) & dmask] + i;
            kout[g] = kk;
            vout[g] = rv[i];
        };
        if (tile_n == kTile) {
#pragma unroll
            for (int j = 0; j < kItems; ++j) put(j * kST + tid);
        } else {
            for (uint32_t i = tid; i < tile_n; i += kST) put(i);
        }
        __syncthreads();  // buffer sg, wcnt and gofs free for the next tiles
    }
}

// Digit width: 9 bits when that saves a pass over 8 (26-bit seed codes: 3 passes
// instead of 4), else 8; 10-bit digits measured slower (more ballots, shorter digit
// runs per tile) and are used only when g_opt.radix_bits pins them.
int pick_digit_bits(int bits, uint64_t n) {
    if (g_opt.radix_bits >= 8 && g_opt.radix_bits <= 10) return int(g_opt.radix_bits);
    if (n > (16u << 20)) return 8;  // large sorts: longer digit runs per tile beat the saved pass
                                    // (C5 L = 20 index, 31 M keys: 0.998 vs 1.039 ms)
    return (bits + 8) / 9 < (bits + 7) / 8 ? 9 : 8;
}

constexpr int kMaxChunks = 148 * 8;  // >= SMs x resident scatter CTAs

template <class K, int RB>
cudaError_t radix_sort_rb(K *k0, uint32_t *v0, K *k1, uint32_t *v1, uint64_t n, int lo, int bits, void *scratch,
                          cudaStream_t s, bool *in_alt, const unsigned long long *dn, uint64_t vg_base = 0,
                          uint32_t vg_step = 0) {
    constexpr int kBins = 1 << RB;
    const int passes = (bits - lo + RB - 1) / RB;
    const size_t smem = sizeof(ScatterSmem<K, uint32_t, RB>);
    static int grid_cap = 0;  // per instantiation: resident scatter CTAs on the whole GPU
    cudaError_t e;
    if (!grid_cap) {
        e = cudaFuncSetAttribute(k_scatter<K, uint32_t, RB>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_scatter<K, uint32_t, RB>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_scatter<K, uint32_t, RB, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 int(smem));
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_scatter<K, uint32_t, RB, true>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        if (e != cudaSuccess) return e;
        int per_sm = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_scatter<K, uint32_t, RB>, kST, smem);
        if (e != cudaSuccess) return e;
        grid_cap = (per_sm > 0 ? per_sm : 1) * num_sms();
    }
    // large sorts: two chunks per resident CTA (shorter chunks balance better; C5 L = 20:
    // index sort 1.00 -> 0.955 ms, output sort 1.05 -> 1.01 ms); small ones: one (C4: 0.116
    // vs 0.122 ms)
    int cap_chunks = grid_cap * (n > (8u << 20) ? 2 : 1);
    if (cap_chunks > kMaxChunks) cap_chunks = kMaxChunks;
    Chunking ch;
    ch.dn = dn;
    ch.n = n;
    ch.tiles = (n + tile_items<K>() - 1) / tile_items<K>();
    ch.chunks = uint32_t(ch.tiles < uint64_t(cap_chunks) ? ch.tiles : uint64_t(cap_chunks));
    ch.tpc = (ch.tiles + ch.chunks - 1) / ch.chunks;
    ch.chunks = uint32_t((ch.tiles + ch.tpc - 1) / ch.tpc);  // no empty chunk
    uint32_t *totals = static_cast<uint32_t *>(scratch);  // [passes][kBins]
    uint32_t *counts = totals + size_t(passes) * kBins;     // [kBins][chunks]
    uint32_t *offs = counts + size_t(ch.chunks) * kBins;    // [kBins][chunks]
    e = fill_async(totals, 0u, size_t(passes) * kBins * sizeof(uint32_t), s);
    if (e != cudaSuccess) return e;
    K *ka = k0, *kb = k1;
    uint32_t *va = v0, *vb = v1;
    for (int p = 0; p < passes; ++p) {
        const int sh = lo + RB * p;
        const int dbits = (p == passes - 1) ? bits - sh : RB;
        uint32_t *tot = totals + size_t(p) * kBins;
        pdl_launch(k_chunk_hist<K, RB>, ch.chunks, kT, 0, s, ka, ch, sh, dbits, counts, tot);
        pdl_launch(k_chunk_scan<RB>, kBins / kWarps, kT, 0, s, counts, tot, ch.chunks, offs);
        // pass 0 with generated values (vg_step != 0): v0 is not read
        if (p == 0 && vg_step)
            pdl_launch(k_scatter<K, uint32_t, RB, true>, ch.chunks, kST, smem, s, ka, va, kb, vb, ch, sh, dbits, offs,
                       vg_base, vg_step);
        else
            pdl_launch(k_scatter<K, uint32_t, RB>, ch.chunks, kST, smem, s, ka, va, kb, vb, ch, sh, dbits, offs,
                       vg_base, vg_step);
        note_launch(3);
        std::swap(ka, kb);
        std::swap(va, vb);
        *in_alt = !*in_alt;
    }
    return cudaGetLastError();
}

template <class K>
cudaError_t radix_sort(K *k0, uint32_t *v0, K *k1, uint32_t *v1, uint64_t n, int lo, int bits, void *scratch,
                       cudaStream_t s, bool *in_alt, const unsigned long long *dn = nullptr, uint64_t vg_base = 0,
                       uint32_t vg_step = 0) {
    *in_alt = false;
    if (bits > int(8 * sizeof(K))) bits = int(8 * sizeof(K));
    if ((n <= 1 && !dn) || n == 0 || bits <= lo) return cudaSuccess;
    if (!scratch) return cudaErrorInvalidValue;
    if (uint64_t(n) >= (uint64_t(1) << 32)) return cudaErrorInvalidValue;  // 32-bit offsets
    switch (pick_digit_bits(bits - lo, n)) {
        case 9: return radix_sort_rb<K, 9>(k0, v0, k1, v1, n, lo, bits, scratch, s, in_alt, dn, vg_base, vg_step);
        case 10: return radix_sort_rb<K, 10>(k0, v0, k1, v1, n, lo, bits, scratch, s, in_alt, dn, vg_base, vg_step);
        default: return radix_sort_rb<K, 8>(k0, v0, k1, v1, n, lo, bits, scratch, s, in_alt, dn, vg_base, vg_step);
    }
}

}  // namespace

int radix_passes(int bits, uint64_t n) {  // as radix_sort runs them (none for n <= 1)
    if (bits <= 0 || n <= 1) return 0;
    const int rb = pick_digit_bits(bits, n);
    return (bits + rb - 1) / rb;
}

size_t radix_scratch_bytes(uint64_t n) {  // totals of every pass + counts + offsets, at the widest digit
    (void)n;
    return size_t(8 * 1024 + 2 * size_t(kMaxChunks) * 1024) * sizeof(uint32_t);
}

cudaError_t radix_sort_u32(uint32_t *k0, uint32_t *v0, uint32_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt, int lo, uint64_t vg_base, uint32_t vg_step) {
    return radix_sort<uint32_t>(k0, v0, k1, v1, n, lo, bits, scratch, s, in_alt, nullptr, vg_base, vg_step);
}

cudaError_t radix_sort_u64(uint64_t *k0, uint32_t *v0, uint64_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt, int lo, const unsigned long long *dn) {
    return radix_sort<uint64_t>(k0, v0, k1, v1, n, lo, bits, scratch, s, in_alt, dn);
}

}  // namespace gm
