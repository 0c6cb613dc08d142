// radix.cu -- stable LSD radix sort, onesweep style (counting sort per 8-bit digit).
// Used twice on the hot path:
//  * index build: the counting sort of sampled seeds over 4^ls buckets (Alg. 1
//    steps 1-3) done digit by digit; stability leaves every
//    bucket in ascending location order, which is what Alg. 1 step 4 (:102-106,
//    per-seed sort) achieves, without a per-bucket sort;
//  * output: MEM triples into (r, q) order.
//
// Launches per sort: one memset, k_hist_all (histograms of every digit in one
// read of the keys), k_hist_scan (exclusive scan of each digit histogram), then
// one k_onesweep per digit: the tile's stable local ranks (per-warp running
// counters + __match_any_sync peers), its digit counts published to a status
// array and the global prefix found by decoupled look-back over earlier tiles,
// then a reorder through shared memory so each digit run is written out
// contiguously (coalesced).
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;                 // threads per CTA
constexpr int kWarps = kT / 32;
constexpr int kBins = 256;
constexpr uint32_t kFlagAgg = 1u << 30;
constexpr uint32_t kFlagInc = 2u << 30;
constexpr uint32_t kValMask = (1u << 30) - 1;

template <class K>
struct Cfg;
template <>
struct Cfg<uint32_t> {
    static constexpr int kItems = 12;
};
template <>
struct Cfg<uint64_t> {
    static constexpr int kItems = 8;
};
constexpr int kLookWin = 16;  // predecessors read per look-back step

// Lanes of the warp holding the same digit (among lanes with valid == true), built
// from one ballot per digit bit -- full-rate, unlike __match_any_sync.
__device__ __forceinline__ unsigned match_digit(uint32_t d, bool valid, int bits) {
    unsigned peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < 8; ++b) {
        if (b < bits) {
            const bool bit = (d >> b) & 1u;
            const unsigned m = __ballot_sync(0xffffffffu, bit);
            peers &= bit ? m : ~m;
        }
    }
    return peers;
}

// Histograms of every digit position in one read of the keys. Each warp owns
// private counters (no shared-memory atomics, which serialise per lane): the
// leader of each group of equal digits adds the group's size.
constexpr int kHT = 128;
constexpr int kHWarps = kHT / 32;

template <class K>
__global__ void __launch_bounds__(kHT) k_hist_all(const K *__restrict__ keys, uint64_t n, int passes,
                                                  uint32_t *__restrict__ hist) {
    __shared__ uint32_t h[kHWarps][8][kBins];  // 32 KB
    for (int i = threadIdx.x; i < kHWarps * 8 * kBins; i += kHT) (&h[0][0][0])[i] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t stride = uint64_t(gridDim.x) * kHT;
    for (uint64_t base = uint64_t(blockIdx.x) * kHT + uint64_t(w) * 32; base < n; base += stride) {
        const uint64_t idx = base + lane;
        const bool valid = idx < n;
        const K k = valid ? keys[idx] : K(0);
        if (valid) {
            for (int p = 0; p < passes; ++p) atomicAdd(&h[w][p][uint32_t(k >> (8 * p)) & (kBins - 1)], 1u);
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < passes * kBins; i += kHT) {
        uint32_t c = 0;
#pragma unroll
        for (int ww = 0; ww < kHWarps; ++ww) c += (&h[ww][0][0])[i];
        if (c) atomicAdd(hist + i, c);
    }
}

__global__ void __launch_bounds__(kT) k_hist_scan(uint32_t *hist, int passes) {
    __shared__ uint32_t ws[kWarps];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int p = 0; p < passes; ++p) {
        const uint32_t x = hist[p * kBins + threadIdx.x];
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
        hist[p * kBins + threadIdx.x] = pre + inc - x;  // exclusive
        __syncthreads();
    }
}

template <class K, class V>
struct alignas(16) SweepSmem {
    K k[kT * Cfg<K>::kItems];
    V v[kT * Cfg<K>::kItems];
    uint32_t wcnt[kWarps][kBins];
    uint32_t local_excl[kBins];
    uint32_t global_base[kBins];
    uint32_t ws[kWarps];
    uint32_t tile;
};

template <class K, class V>
__global__ void __launch_bounds__(kT, 3) k_onesweep(const K *__restrict__ kin, const V *__restrict__ vin,
                                                 K *__restrict__ kout, V *__restrict__ vout, uint64_t n,
                                                 int shift, int bits, const uint32_t *__restrict__ digit_off,
                                                 uint32_t *status, unsigned int *tile_ctr) {
    constexpr int kItems = Cfg<K>::kItems;
    constexpr int kTile = kT * kItems;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SweepSmem<K, V> &S = *reinterpret_cast<SweepSmem<K, V> *>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t dmask = (1u << bits) - 1;
    if (tid == 0) S.tile = atomicAdd(tile_ctr, 1u);
    for (int i = tid; i < kWarps * kBins; i += kT) (&S.wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = S.tile;
    const uint64_t base = uint64_t(tile) * kTile;
    const uint32_t tile_n = uint32_t(min(uint64_t(kTile), n - base));

    // ---- load (warp-striped rounds keep input order = (warp, round, lane)) and rank
    K k[kItems];
    V v[kItems];
    uint32_t rank[kItems];
    const uint64_t wbase = base + uint64_t(w) * 32 * kItems;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t idx = wbase + uint64_t(j) * 32 + lane;
        const bool valid = idx < n;
        k[j] = valid ? kin[idx] : K(0);
        v[j] = valid ? vin[idx] : 0u;
        const uint32_t d = uint32_t(k[j] >> shift) & dmask;
        const unsigned peers = match_digit(d, valid, bits);
        const uint32_t b0 = valid ? S.wcnt[w][d] : 0u;
        rank[j] = b0 + __popc(peers & lanemask_lt());
        __syncwarp();
        if (valid && lane == __ffs(peers) - 1) S.wcnt[w][d] = b0 + __popc(peers);
        __syncwarp();
    }
    __syncthreads();

    // ---- per digit: tile count, warp offsets, publish + decoupled look-back
    const uint32_t d = tid;  // kT == kBins
    uint32_t cnt = 0;
#pragma unroll
    for (int ww = 0; ww < kWarps; ++ww) {
        const uint32_t c = S.wcnt[ww][d];
        S.wcnt[ww][d] = cnt;
        cnt += c;
    }
    volatile uint32_t *st = status;
    if (tile == 0) {
        st[d] = kFlagInc | cnt;
        S.global_base[d] = digit_off[d];
    } else {
        st[uint64_t(tile) * kBins + d] = kFlagAgg | cnt;
        // decoupled look-back in windows of kLookWin predecessors (independent loads)
        uint32_t excl = 0;
        int64_t t = int64_t(tile) - 1;
        for (bool done = false; !done;) {
            uint32_t s[kLookWin];
#pragma unroll
            for (int i = 0; i < kLookWin; ++i)
                s[i] = (t - i >= 0) ? st[uint64_t(t - i) * kBins + d] : uint32_t(2u << 30);
            int i = 0;
#pragma unroll
            for (int ii = 0; ii < kLookWin; ++ii) {
                if (i != ii || done) continue;
                const uint32_t f = s[ii] & ~kValMask;
                if (f == 0) continue;  // not published yet: re-poll from here
                excl += s[ii] & kValMask;
                if (f == kFlagInc) done = true; else ++i;
            }
            t -= i;
        }
        st[uint64_t(tile) * kBins + d] = kFlagInc | (excl + cnt);
        S.global_base[d] = digit_off[d] + excl;
    }
    {  // tile-local exclusive digit offsets (block scan over the 256 digits)
        uint32_t inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) S.ws[w] = inc;
        __syncthreads();
        uint32_t pre = 0;
        for (int i = 0; i < w; ++i) pre += S.ws[i];
        S.local_excl[d] = pre + inc - cnt;
    }
    __syncthreads();

    // ---- reorder into digit order in shared memory
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t idx = wbase + uint64_t(j) * 32 + lane;
        if (idx < n) {
            const uint32_t dd = uint32_t(k[j] >> shift) & dmask;
            const uint32_t lp = S.local_excl[dd] + S.wcnt[w][dd] + rank[j];
            S.k[lp] = k[j];
            S.v[lp] = v[j];
        }
    }
    __syncthreads();
    // ---- coalesced write-out: consecutive slots of one digit go to consecutive addresses
    for (uint32_t i = tid; i < tile_n; i += kT) {
        const K kk = S.k[i];
        const uint32_t dd = uint32_t(kk >> shift) & dmask;
        const uint64_t g = uint64_t(S.global_base[dd]) + (i - S.local_excl[dd]);
        kout[g] = kk;
        vout[g] = S.v[i];
    }
}

template <class K>
constexpr uint64_t tile_items() {
    return uint64_t(kT) * Cfg<K>::kItems;
}

template <class K>
size_t scratch_bytes(uint64_t n, int passes) {
    const uint64_t tiles = (n + tile_items<K>() - 1) / tile_items<K>();
    return (size_t(passes) * kBins + 16 + size_t(passes) * tiles * kBins) * sizeof(uint32_t);
}

template <class K>
cudaError_t radix_sort(K *k0, uint32_t *v0, K *k1, uint32_t *v1, uint64_t n, int bits, void *scratch,
                       cudaStream_t s, bool *in_alt) {
    *in_alt = false;
    if (n <= 1 || bits <= 0) return cudaSuccess;
    if (!scratch) return cudaErrorInvalidValue;
    if (bits > int(8 * sizeof(K))) bits = int(8 * sizeof(K));
    const int passes = (bits + 7) / 8;
    const uint64_t tiles = (n + tile_items<K>() - 1) / tile_items<K>();
    uint32_t *hist = static_cast<uint32_t *>(scratch);
    unsigned int *ctr = hist + passes * kBins;  // one tile counter per pass
    uint32_t *status = ctr + 16;
    cudaError_t e = cudaMemsetAsync(scratch, 0, scratch_bytes<K>(n, passes), s);
    if (e != cudaSuccess) return e;
    const uint64_t hblocks = (n + kHT * 8 - 1) / (kHT * 8);  // >= 8 items per thread
    const int hgrid = int(hblocks < uint64_t(num_sms() * 6) ? hblocks : uint64_t(num_sms() * 6));
    k_hist_all<K><<<hgrid, kHT, 0, s>>>(k0, n, passes, hist);
    k_hist_scan<<<1, kT, 0, s>>>(hist, passes);
    note_launch(2);
    const size_t smem = sizeof(SweepSmem<K, uint32_t>);
    static bool attr_set = false;  // per instantiation
    if (!attr_set) {
        e = cudaFuncSetAttribute(k_onesweep<K, uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_onesweep<K, uint32_t>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    K *ka = k0, *kb = k1;
    uint32_t *va = v0, *vb = v1;
    for (int p = 0; p < passes; ++p) {
        const int dbits = (p == passes - 1) ? bits - 8 * p : 8;
        k_onesweep<K, uint32_t><<<unsigned(tiles), kT, smem, s>>>(ka, va, kb, vb, n, 8 * p, dbits, hist + p * kBins,
                                                                  status + uint64_t(p) * tiles * kBins, ctr + p);
        note_launch();
        std::swap(ka, kb);
        std::swap(va, vb);
        *in_alt = !*in_alt;
    }
    return cudaGetLastError();
}

}  // namespace

size_t radix_scratch_bytes(uint64_t n) {
    const size_t a = scratch_bytes<uint32_t>(n, 8), b = scratch_bytes<uint64_t>(n, 8);
    return a > b ? a : b;
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
