// msd.cu -- MSD bucket sort for unique 64-bit keys (+ optional 32-bit values).
//
// Used where the keys are unique, so stability is irrelevant: the output, keys
// (r << qbits | q) with len as value, up to 2 M MEMs; the last
// kernel writes gpumem_triple {r, q, len} directly.
// Two passes over the data:
//  k_bp_hist     chunk c (one CTA per SM, a contiguous run of the input) counts the
//                top B key bits (2^B <= 16384 buckets) in a shared-memory histogram;
//  k_bp_colscan  per bucket: exclusive prefix over the chunks + the bucket total;
//  k_bp_scatter  every CTA scans the bucket totals (CTA 0 publishes the offsets); chunk c
//                moves its keys to its private range of each bucket (order
//                inside a chunk's range arbitrary: shared-memory atomic cursors; the
//                keys are unique and get fully sorted next);
//  k_bs_local    CTA s sorts the buckets that start in slots [s * kSeg, (s + 1) * kSeg)
//                -- a contiguous segment of whole buckets, so sorting the segment by
//                the full key sorts each of them -- with an LSD radix sort in shared
//                memory (digits that are equal across the segment are skipped), and
//                writes the result (keys/values, or triples);
//  k_bs_big      buckets too large for shared memory (adversarial inputs: e.g. one
//                r with 10^5 MEMs) get a CTA-level LSD radix in global memory.
// No per-element global atomics anywhere. B is chosen so that buckets average ~512 keys.
// The key count n may live in device memory (msd_sort_dev: the find kernel's output
// counter, so a captured CUDA graph needs no host round trip): every kernel derives n,
// B, the bucket count and its chunk bounds from it on the device; grids are sized for
// the capacity and idle blocks exit (k_bs_local loops over segments).
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;                          // threads of k_bs_big
constexpr int kWarps = kT / 32;
constexpr int kPT = 1024;                        // threads of the chunk kernels
constexpr int kLT = 512;                         // threads of k_bs_local
constexpr int kLWarps = kLT / 32;
#ifndef GM_MSD_ITEMS
#define GM_MSD_ITEMS 8
#endif
#ifndef GM_MSD_CTAS
#define GM_MSD_CTAS 2
#endif
constexpr int kItems = GM_MSD_ITEMS;             // keys per thread in k_bs_local
constexpr int kLocalCtas = GM_MSD_CTAS;          // resident k_bs_local CTAs per SM (grid size)
constexpr uint32_t kLocal = kLT * kItems;        // most keys one CTA sorts in shared memory (4096)
constexpr uint32_t kSeg = kLocal / 2;            // segment spacing (slots) for the grid size
#ifndef GM_MSD_SEGMAX
#define GM_MSD_SEGMAX (kLocal * 7 / 8)           // largest segment spacing k_bs_local picks (measured
                                                 // 2048 / 3072 / 3584 / 4096: C4 0.149 / 0.113 / 0.113 / 0.113 ms,
                                                 // C5 L = 50 0.437 / 0.400 / 0.380 / 0.381 ms)
#endif
constexpr int kMaxB = 14;                        // 16384 buckets: a 64 KB shared histogram

__host__ __device__ __forceinline__ int choose_b(uint64_t n, int bits) {
    int B = 1;
    while (B < kMaxB && (n >> (B + 9)) > 0) ++B;  // ~512 keys per bucket
    return B < bits ? B : bits;
}

// The number of keys: *dn clamped to cap when the count is device-resident, else cap.
struct NSpec {
    const unsigned long long *dn;
    uint64_t cap;
    int bits;                                    // significant key bits
    __device__ __forceinline__ int B(uint64_t n) const { return choose_b(n, bits); }
    __device__ __forceinline__ uint64_t n() const {
        if (!dn) return cap;
        const unsigned long long x = *dn;
        return x < cap ? x : cap;
    }
};

// chunk c = elements [c * cs, min((c + 1) * cs, n))
__global__ void __launch_bounds__(kPT) k_bp_hist(const uint64_t *__restrict__ keys, NSpec ns,
                                                 uint32_t *__restrict__ counts, unsigned int *__restrict__ n_big) {
    pdl_wait();
    if (blockIdx.x == 0 && threadIdx.x == 0) *n_big = 0;  // k_bs_local's list of oversized buckets
    extern __shared__ uint32_t h[];
    const uint64_t n = ns.n();
    const int B = choose_b(n, ns.bits), shift = ns.bits - B;
    const uint32_t nb = 1u << B;
    const uint64_t cs = (n + gridDim.x - 1) / gridDim.x;
    for (uint32_t i = threadIdx.x; i < nb; i += kPT) h[i] = 0;
    __syncthreads();
    const uint64_t b = uint64_t(blockIdx.x) * cs, e = min(b + cs, n);
    for (uint64_t i = b + threadIdx.x; i < e; i += kPT) atomicAdd(&h[uint32_t(keys[i] >> shift)], 1u);
    __syncthreads();
    uint32_t *row = counts + uint64_t(blockIdx.x) * nb;  // chunk-major
    for (uint32_t i = threadIdx.x; i < nb; i += kPT) row[i] = h[i];
}

// per bucket b (one warp): counts[c][b] -> exclusive prefix over c (in place); totals[b].
// Lane l owns a contiguous run of chunks; a warp scan joins the runs.
__global__ void __launch_bounds__(256) k_bp_colscan(uint32_t *__restrict__ counts, uint32_t chunks, NSpec ns,
                                                    uint32_t *__restrict__ totals) {
    pdl_wait();
    const uint32_t nb = 1u << choose_b(ns.n(), ns.bits);
    const uint32_t b = blockIdx.x * 8 + (threadIdx.x >> 5);
    const int lane = threadIdx.x & 31;
    if (b >= nb) return;
    const uint32_t per = (chunks + 31) / 32;
    const uint32_t c0 = min(uint32_t(lane) * per, chunks), c1 = min(c0 + per, chunks);
    uint32_t x[8], sum = 0;  // per <= 8 (chunks <= 256)
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        x[j] = c0 + j < c1 ? counts[uint64_t(c0 + j) * nb + b] : 0u;
        sum += x[j];
    }
    uint32_t inc = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    uint32_t run = inc - sum;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        if (c0 + j < c1) counts[uint64_t(c0 + j) * nb + b] = run;
        run += x[j];
    }
    if (lane == 31) totals[b] = inc;
}

// Every CTA scans the bucket totals itself (<= 16 K of them: one run of 16 per thread),
// so no separate scan launch sits between the column scan and the scatter; CTA 0 writes
// the bucket offsets (offs[0, nb]) for k_bs_local / k_bs_big.
__global__ void __launch_bounds__(kPT) k_bp_scatter(const uint64_t *__restrict__ keys,
                                                    const uint32_t *__restrict__ vals, NSpec ns,
                                                    const uint32_t *__restrict__ rel,
                                                    const uint32_t *__restrict__ totals, uint32_t *__restrict__ offs,
                                                    uint64_t *__restrict__ ok, uint32_t *__restrict__ ov) {
    pdl_wait();
    extern __shared__ uint32_t cur[];
    __shared__ uint32_t ws[kPT / 32];
    const uint64_t n = ns.n();
    const int B = choose_b(n, ns.bits), shift = ns.bits - B;
    const uint32_t nb = 1u << B;
    const uint64_t cs = (n + gridDim.x - 1) / gridDim.x;
    const uint32_t *row = rel + uint64_t(blockIdx.x) * nb;
    {
        const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
        const uint32_t per = (nb + kPT - 1) / kPT;
        const uint32_t i0 = min(threadIdx.x * per, nb), i1 = min(i0 + per, nb);
        uint32_t sum = 0;
        for (uint32_t i = i0; i < i1; ++i) sum += totals[i];
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
            if (blockIdx.x == 0) offs[i] = run;
            cur[i] = run + row[i];
            run += totals[i];
        }
        if (blockIdx.x == 0 && threadIdx.x == kPT - 1) offs[nb] = run;
    }
    __syncthreads();
    const uint64_t b = uint64_t(blockIdx.x) * cs, e = min(b + cs, n);
    for (uint64_t i = b + threadIdx.x; i < e; i += kPT) {
        const uint64_t k = keys[i];
        const uint32_t slot = atomicAdd(&cur[uint32_t(k >> shift)], 1u);
        ok[slot] = k;
        if (vals) ov[slot] = vals[i];
    }
}

struct Out {
    uint64_t *keys;          // generic result (in place of the input)
    uint32_t *vals;          // may be null
    gpumem_triple *trip;     // if set: triples {key >> qbits, key & qmask, val} instead
    uint32_t qbits;
    __device__ __forceinline__ void put(uint64_t i, uint64_t k, uint32_t v) const {
        if (trip) {
            gpumem_triple t;
            t.r = uint32_t(k >> qbits);
            t.q = uint32_t(k & ((1ull << qbits) - 1));
            t.len = v;
            trip[i] = t;
        } else {
            keys[i] = k;
            if (vals) vals[i] = v;
        }
    }
};

// first bucket b in [0, nb] with offs[b] >= x
__device__ __forceinline__ uint32_t first_at(const uint32_t *__restrict__ offs, uint32_t nb, uint64_t x) {
    uint32_t lo = 0, hi = nb;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (uint64_t(offs[mid]) < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// Shared memory of k_bs_local: a ping-pong pair of key/value buffers and the per-warp
// digit counters of one LSD pass.
struct LocalSmem {
    uint64_t k[2][kLocal];
    uint32_t v[2][kLocal];
    uint32_t wcnt[kLWarps][256];
    uint32_t ws[kLWarps];
    unsigned long long kor, kand;  // OR / AND of the keys: digits equal in all keys are skipped
};

// Lanes of the warp holding the same 8-bit digit (among valid lanes): one ballot per bit.
__device__ __forceinline__ unsigned match8(uint32_t d, bool valid) {
    unsigned peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < 8; ++b) {
        const bool bit = (d >> b) & 1u;
        const unsigned m = __ballot_sync(0xffffffffu, bit);
        peers &= bit ? m : ~m;
    }
    return peers;
}

// One stable LSD pass in shared memory over the 8-bit digit at `sh`: buffer cur -> cur ^ 1
// (stable ranks from per-warp digit counters + ballot peers). Rows of 32 slots wholly past
// m are skipped warp-uniformly (a segment rarely fills the CTA's kLocal slots).
__device__ __forceinline__ void smem_pass(LocalSmem &S, uint32_t m, int sh, int &cur) {
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t wofs = uint32_t(w) * 32 * kItems;  // warp w owns slots [wofs, wofs + 32 kItems)
#pragma unroll
    for (int ww = 0; ww < kLWarps; ++ww) S.wcnt[ww][tid & 255] = 0;
    __syncthreads();
    uint64_t k[kItems];
    uint32_t v[kItems], rank[kItems];
    unsigned peers[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint32_t i = wofs + j * 32 + lane;
        const bool valid = i < m;
        k[j] = valid ? S.k[cur][i] : 0ull;
        v[j] = valid ? S.v[cur][i] : 0u;
        peers[j] = wofs + j * 32 < m ? match8(uint32_t(k[j] >> sh) & 255u, valid) : 0u;
    }
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (wofs + j * 32 >= m) break;  // warp-uniform
        const bool valid = wofs + j * 32 + lane < m;
        const uint32_t d = uint32_t(k[j] >> sh) & 255u;
        const uint32_t b0 = valid ? S.wcnt[w][d] : 0u;
        rank[j] = b0 + __popc(peers[j] & lanemask_lt());
        __syncwarp();
        if (valid && lane == __ffs(peers[j]) - 1) S.wcnt[w][d] = b0 + __popc(peers[j]);
        __syncwarp();
    }
    __syncthreads();
    // digit-major, warp-minor exclusive offsets (thread tid < 256 owns digit tid)
    uint32_t xw[kLWarps], c = 0;
    if (tid < 256) {
#pragma unroll
        for (int ww = 0; ww < kLWarps; ++ww) {
            xw[ww] = S.wcnt[ww][tid];
            c += xw[ww];
        }
    }
    uint32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) S.ws[w] = inc;
    __syncthreads();
    if (tid < 256) {
        uint32_t run = inc - c;
        for (int i = 0; i < w; ++i) run += S.ws[i];
#pragma unroll
        for (int ww = 0; ww < kLWarps; ++ww) {
            S.wcnt[ww][tid] = run;
            run += xw[ww];
        }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (wofs + j * 32 + lane < m) {
            const uint32_t pos = S.wcnt[w][uint32_t(k[j] >> sh) & 255u] + rank[j];
            S.k[cur ^ 1][pos] = k[j];
            S.v[cur ^ 1][pos] = v[j];
        }
    }
    cur ^= 1;
    __syncthreads();
}

// Sorts the m <= kLocal keys (with values) of [tk + lo, tk + lo + m) by their low `bits`
// bits with LSD passes in shared memory (digits equal in every key skipped) and writes
// them to out[lo, lo + m).
__device__ void smem_sort_write(LocalSmem &S, const uint64_t *__restrict__ tk, const uint32_t *__restrict__ tv,
                                uint32_t lo, uint32_t m, int bits, const Out &out) {
    const int tid = threadIdx.x, lane = tid & 31;
    if (tid == 0) {
        S.kor = 0ull;
        S.kand = ~0ull;
    }
    __syncthreads();
    unsigned long long kor = 0ull, kand = ~0ull;
    for (uint32_t i = tid; i < m; i += kLT) {
        const uint64_t x = tk[lo + i];
        S.k[0][i] = x;
        S.v[0][i] = tv[lo + i];
        kor |= x;
        kand &= x;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        kor |= __shfl_xor_sync(0xffffffffu, kor, o);
        kand &= __shfl_xor_sync(0xffffffffu, kand, o);
    }
    if (lane == 0) {
        atomicOr(&S.kor, kor);
        atomicAnd(&S.kand, kand);
    }
    __syncthreads();
    const uint64_t diff = S.kor ^ S.kand;
    int cur = 0;
    for (int sh = 0; sh < bits; sh += 8)
        if ((diff >> sh) & 255u) smem_pass(S, m, sh, cur);  // same digit in every key: the pass is the identity
    for (uint32_t i = tid; i < m; i += kLT) out.put(uint64_t(lo) + i, S.k[cur][i], S.v[cur][i]);
    __syncthreads();
}

__global__ void __launch_bounds__(kLT, kLocalCtas) k_bs_local(const uint32_t *__restrict__ offs, NSpec ns,
                                                 const uint64_t *__restrict__ tk, const uint32_t *__restrict__ tv,
                                                 Out out, uint32_t *__restrict__ big, unsigned int *n_big) {
    pdl_wait();
    extern __shared__ __align__(16) unsigned char smem[];
    LocalSmem &S = *reinterpret_cast<LocalSmem *>(smem);
    __shared__ uint32_t s_b[2];
    const uint64_t n = ns.n();
    const int bits = ns.bits;
    const uint32_t nb = 1u << ns.B(n);
    // segment spacing: an even share of n over the grid in as few rounds as possible, a
    // segment's cost being nearly independent of its size (every thread walks kItems
    // slots per pass): up to kSegMax slots, leaving room below kLocal for the whole
    // buckets that start in the segment (C4: 0.81 M keys over 296 blocks -> one round of
    // 2.7 K-slot segments instead of 1-2 rounds of 2 K)
    constexpr uint64_t kSegMax = GM_MSD_SEGMAX;
    const uint64_t rounds = (n + uint64_t(gridDim.x) * kSegMax - 1) / (uint64_t(gridDim.x) * kSegMax);
    const uint64_t seg_w = rounds ? (n + uint64_t(gridDim.x) * rounds - 1) / (uint64_t(gridDim.x) * rounds) : kSeg;
    for (uint64_t seg = blockIdx.x; seg * seg_w < n; seg += gridDim.x) {
        __syncthreads();  // the previous segment's readers of s_b are done
        if (threadIdx.x == 0) s_b[0] = first_at(offs, nb, seg * seg_w);
        if (threadIdx.x == 32) s_b[1] = first_at(offs, nb, (seg + 1) * seg_w);
        __syncthreads();
        const uint32_t b0 = s_b[0], b1 = s_b[1];
        if (b0 >= b1) continue;
        const uint32_t lo = offs[b0], m = offs[b1] - lo;
        if (m <= kLocal) {
            // the segment's keys share no common prefix below the bucket bits in general:
            // sort by all key bits (the bucket prefix bits then sort the buckets among themselves)
            smem_sort_write(S, tk, tv, lo, m, bits, out);
            continue;
        }
        // a large bucket in the segment: runs of consecutive buckets of <= kLocal keys in
        // all, each sorted as one (buckets are ordered by their prefix); a bucket past
        // kLocal alone goes to k_bs_big
        for (uint32_t b = b0; b < b1;) {
            const uint32_t blo = offs[b];
            if (offs[b + 1] - blo > kLocal) {
                if (threadIdx.x == 0) big[atomicAdd(n_big, 1u)] = b;
                ++b;
                continue;
            }
            uint32_t e = b + 1;
            while (e < b1 && offs[e + 1] - blo <= kLocal) ++e;
            if (offs[e] > blo) smem_sort_write(S, tk, tv, blo, offs[e] - blo, bits, out);
            b = e;
        }
    }
}

// One CTA per oversized bucket: LSD radix (8-bit digits) over the low `bits` key bits,
// ping-ponging between (tk, tv) and (sk, sv) over the bucket's range; then written out.
__global__ void __launch_bounds__(kT) k_bs_big(const uint32_t *__restrict__ offs, const uint32_t *__restrict__ big,
                                               const unsigned int *__restrict__ n_big, uint64_t *tk, uint32_t *tv,
                                               uint64_t *xk, uint32_t *xv, NSpec ns, Out out) {
    pdl_wait();
    __shared__ uint32_t hist[256];
    __shared__ uint32_t wcnt[kWarps][256];
    __shared__ uint32_t ws[kWarps];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const unsigned nbig = *n_big;
    const int bits = ns.bits - ns.B(ns.n());  // the bits below the bucket prefix
    const int passes = (bits + 7) / 8;
    for (unsigned li = blockIdx.x; li < nbig; li += gridDim.x) {
        const uint32_t b = big[li];
        const uint32_t lo = offs[b], m = offs[b + 1] - lo;
        uint64_t *sk = tk + lo, *dk = xk + lo;
        uint32_t *sv = tv + lo, *dv = xv + lo;
        for (int pass = 0; pass < passes; ++pass) {
            const int sh = 8 * pass;
            hist[tid] = 0;
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
                const uint32_t xv2 = valid ? sv[j] : 0u;
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
                    dv[pos] = xv2;
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
        for (uint32_t j = tid; j < m; j += kT) out.put(uint64_t(lo) + j, sk[j], sv[j]);
        __syncthreads();
    }
}

uint32_t n_chunks(uint64_t n) {
    const uint64_t c = (n + 4095) / 4096;  // >= 4K keys per chunk
    const uint64_t cap = uint64_t(num_sms());
    return uint32_t(c < cap ? (c ? c : 1) : cap);
}

}  // namespace

size_t msd_scratch_bytes(uint64_t n) {
    const uint64_t nb = 1ull << kMaxB;
    const uint64_t chunks = 1024;  // >= SMs
    return n * 8 + n * 4 * 2 + chunks * nb * 4 + (nb + 1) * 4 * 2 + nb * 4 + 1024 + 8 * 256;
}

static cudaError_t msd_run(uint64_t *keys, uint32_t *vals, NSpec ns, void *scratch, cudaStream_t s,
                           gpumem_triple *trip, uint32_t qbits) {
    Out out{keys, vals, trip, qbits};
    const uint64_t cap = ns.cap;
    const uint32_t nb_max = 1u << choose_b(ns.dn ? (1ull << 62) : cap, ns.bits);  // device count: any B
    const uint32_t chunks = n_chunks(cap);
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t c = align(reinterpret_cast<uintptr_t>(scratch));
    uint64_t *tk = reinterpret_cast<uint64_t *>(c);
    c = align(c + cap * 8);
    uint32_t *tv = reinterpret_cast<uint32_t *>(c);
    c = align(c + cap * 4);
    uint32_t *xv = vals ? vals : reinterpret_cast<uint32_t *>(c);  // value ping-pong of k_bs_big
    c = align(c + cap * 4);
    uint32_t *counts = reinterpret_cast<uint32_t *>(c);  // [chunks][nb]
    c = align(c + uint64_t(chunks) * nb_max * 4);
    uint32_t *totals = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb_max + 1) * 4);
    uint32_t *offs = reinterpret_cast<uint32_t *>(c);
    c = align(c + (nb_max + 1) * 4);
    uint32_t *big = reinterpret_cast<uint32_t *>(c);
    c = align(c + nb_max * 4);
    unsigned int *n_big = reinterpret_cast<unsigned int *>(c);
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_bp_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, (1 << kMaxB) * 4);
        cudaFuncSetAttribute(k_bp_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (1 << kMaxB) * 4);
        cudaFuncSetAttribute(k_bs_local, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sizeof(LocalSmem)));
        attr = true;
    }
    pdl_launch(k_bp_hist, chunks, kPT, nb_max * 4, s, keys, ns, counts, n_big);
    pdl_launch(k_bp_colscan, (nb_max + 7) / 8, 256, 0, s, counts, chunks, ns, totals);
    pdl_launch(k_bp_scatter, chunks, kPT, nb_max * 4, s, keys, vals, ns, counts, totals, offs, tk, tv);
    uint64_t segs = (cap + kSeg - 1) / kSeg;
    if (segs > uint64_t(kLocalCtas * num_sms())) segs = kLocalCtas * num_sms();  // blocks loop over the segments
    pdl_launch(k_bs_local, unsigned(segs ? segs : 1), kLT, sizeof(LocalSmem), s, offs, ns, tk, tv, out, big, n_big);
    // oversized buckets: ping-pong with the input's range of the bucket (free: the scatter
    // consumed it and the local pass wrote only other buckets' ranges)
    pdl_launch(k_bs_big, num_sms(), kT, 0, s, offs, big, n_big, tk, tv, keys, xv, ns, out);
    note_launch(5);
    return cudaGetLastError();
}

// Sorts n unique keys whose significant bits are the low `bits` (+ values, may be null).
// Result: in place in (keys, vals), or as triples {key >> qbits, key & qmask, val} in
// `trip` when trip != null. `scratch` >= msd_scratch_bytes(n).
cudaError_t msd_sort(uint64_t *keys, uint32_t *vals, uint64_t n, int bits, void *scratch, cudaStream_t s,
                     gpumem_triple *trip, uint32_t qbits) {
    if (n == 0) return cudaSuccess;
    return msd_run(keys, vals, NSpec{nullptr, n, bits < 1 ? 1 : bits}, scratch, s, trip, qbits);
}

// The same with the key count in device memory: n = min(*d_n, cap); nothing is read on
// the host, so the launch sequence is fixed (CUDA-graph capturable).
cudaError_t msd_sort_dev(uint64_t *keys, uint32_t *vals, const unsigned long long *d_n, uint64_t cap, int bits,
                         void *scratch, cudaStream_t s, gpumem_triple *trip, uint32_t qbits) {
    if (cap == 0) return cudaSuccess;
    return msd_run(keys, vals, NSpec{d_n, cap, bits < 1 ? 1 : bits}, scratch, s, trip, qbits);
}

}  // namespace gm
