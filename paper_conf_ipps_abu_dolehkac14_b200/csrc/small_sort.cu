// small_sort.cu -- stable LSD radix sort in ONE cooperative launch, for inputs whose
// per-SM chunk fits in shared memory (<= 148 x 20K u32 keys, 148 x 12K u64 keys).
//
// The multi-launch LSD (radix.cu) spends most of its time at these sizes on launch
// gaps and per-tile barriers, not on bytes (C4: 2.8M seed codes, 0.8M MEM keys). Here
// every CTA owns a contiguous chunk for the whole sort (held in shared memory during a
// pass); a digit pass is
//   load chunk (pass 0: from the source functor, else from the previous pass's output)
//   -> per-warp digit counts (shared atomics) -> publish the CTA's 256 digit counts
//   -> grid barrier -> digit base = (keys with smaller digit anywhere) + (same digit in
//   earlier CTAs) + (same digit in earlier warps of this CTA)
//   -> stable positions in input order (ballot peers + per-warp running counters)
//   -> scatter (last pass: through the sink functor) -> grid barrier.
// Two grid barriers per pass and no kernel boundaries. Used by
//  * the index (Alg. 1): the source computes the seed code of every
//    sampled location from packed R (no separate codes kernel); the sink writes the
//    sorted codes, `locs` and the seed records, so stability = ascending locations
//    inside each seed = Alg. 1 step 4;
//  * the output sort: keys (r << qbits | q) + len -> triples.
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 1024;
constexpr int kWarps = kT / 32;
constexpr int kBins = 256;

// Grid-wide barrier for a cooperative launch: the counter only grows; barrier number b
// completes when every CTA has arrived b times.
__device__ __forceinline__ void grid_barrier(unsigned int *ctr, unsigned int &target) {
    __syncthreads();
    target += gridDim.x;
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(ctr, 1u);
        unsigned int v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
            if (v < target) __nanosleep(64);
        } while (v < target);
    }
    __syncthreads();
}

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

template <class K>
__device__ __forceinline__ K ld_cg(const K *p) {
    return __ldcg(p);
}

// ---- sources / sinks
struct SrcKV64 {  // keys + values in memory
    const uint64_t *k;
    const uint32_t *v;
    __device__ __forceinline__ void load(uint64_t i, uint64_t &key, uint32_t &val) const {
        key = k[i];
        val = v[i];
    }
};
struct SinkTriples {  // (r << qbits | q, len) -> gpumem_triple
    gpumem_triple *out;
    uint32_t qbits;
    __device__ __forceinline__ void store(uint64_t i, uint64_t key, uint32_t val) const {
        gpumem_triple t;
        t.r = uint32_t(key >> qbits);
        t.q = uint32_t(key & ((1ull << qbits) - 1));
        t.len = val;
        out[i] = t;
    }
};
struct SrcSeeds {  // sampled location k -> (code(R, p), p), p = (k0 + k) * step
    const uint64_t *R;
    uint32_t ls, step;
    uint64_t k0;
    __device__ __forceinline__ void load(uint64_t i, uint32_t &key, uint32_t &val) const {
        const uint64_t p = (k0 + i) * step;
        key = uint32_t(win_fwd(R, p) >> (64 - 2 * ls));
        val = uint32_t(p);
    }
};
struct SinkIndex {  // sorted (code, p) -> codes, locs and the seed record of p
    const uint64_t *R;
    uint32_t ls;
    uint32_t *codes, *locs;
    uint4 *recs;
    __device__ __forceinline__ void store(uint64_t i, uint32_t code, uint32_t p) const {
        codes[i] = code;
        locs[i] = p;
        uint32_t left;
        uint64_t right;
        if (p >= 16) {  // bases [p - 16, p + ls + 32) lie in the 3 words from (p - 16) / 32
            const uint64_t x = p - 16, w = x >> 5;
            const uint64_t w0 = __ldg(R + w), w1 = __ldg(R + w + 1), w2 = __ldg(R + w + 2);
            const uint32_t sx = uint32_t(x & 31) * 2;
            left = uint32_t(((w0 << sx) | ((w1 >> 1) >> (63 - sx))) >> 32);
            const uint32_t o = uint32_t(x & 31) + 16 + ls;
            const uint32_t so = (o & 31) * 2;
            const uint64_t a = o < 32 ? w0 : w1, b = o < 32 ? w1 : w2;
            right = (a << so) | ((b >> 1) >> (63 - so));
        } else {
            left = uint32_t(win_back(R, p));
            right = win_fwd(R, uint64_t(p) + ls);
        }
        recs[i] = make_uint4(p, left, uint32_t(right), uint32_t(right >> 32));
    }
};

template <class K, int kCap>
struct SmallSmem {
    K k[kCap];                     // this CTA's chunk
    uint32_t v[kCap];
    uint32_t wcnt[kWarps][kBins];  // per-warp digit counters, then running positions
    uint32_t base[kBins];          // global position of digit d's first key from this CTA
    uint32_t ws[8];
};

template <class K, int kCap, class Src, class Sink>
__global__ void __launch_bounds__(kT, 1) k_small_sort(Src src, Sink sink, uint64_t n, int bits, K *kb0, uint32_t *vb0,
                                                      K *kb1, uint32_t *vb1, uint32_t *counts, unsigned int *bar) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SmallSmem<K, kCap> &S = *reinterpret_cast<SmallSmem<K, kCap> *>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t G = gridDim.x, c = blockIdx.x;
    const uint64_t cs = (n + G - 1) / G;
    const uint64_t cb = min(uint64_t(c) * cs, n), ce = min(cb + cs, n);
    const uint32_t m = uint32_t(ce - cb);
    const uint32_t per_w = (m + kWarps - 1) / kWarps;  // warp w: chunk slots [w * per_w, (w + 1) * per_w)
    const uint32_t w_lo = min(uint32_t(w) * per_w, m), w_hi = min(w_lo + per_w, m);
    unsigned int target = 0;
    const int passes = (bits + 7) / 8;
    for (int pass = 0; pass < passes; ++pass) {
        const int sh = pass * 8;
        const K *kin = (pass & 1) ? kb1 : kb0;
        const uint32_t *vin = (pass & 1) ? vb1 : vb0;
        K *kout = (pass & 1) ? kb0 : kb1;
        uint32_t *vout = (pass & 1) ? vb0 : vb1;
        for (uint32_t i = tid; i < m; i += kT) {
            if (pass == 0) {
                src.load(cb + i, S.k[i], S.v[i]);
            } else {
                S.k[i] = ld_cg(kin + cb + i);
                S.v[i] = ld_cg(vin + cb + i);
            }
        }
        for (int i = tid; i < kWarps * kBins; i += kT) (&S.wcnt[0][0])[i] = 0;
        __syncthreads();
        // sweep 1: per-warp digit counts
        for (uint32_t i = w_lo + lane; i < w_hi; i += 32) atomicAdd(&S.wcnt[w][uint32_t(S.k[i] >> sh) & 255u], 1u);
        __syncthreads();
        // per digit: warp offsets inside the CTA, CTA count published
        if (tid < kBins) {
            uint32_t run = 0;
#pragma unroll 8
            for (int ww = 0; ww < kWarps; ++ww) {
                const uint32_t x = S.wcnt[ww][tid];
                S.wcnt[ww][tid] = run;
                run += x;
            }
            counts[(uint64_t(pass) * G + c) * kBins + tid] = run;
        }
        grid_barrier(bar, target);
        // digit bases: keys of smaller digits anywhere + same digit in earlier CTAs
        if (tid < kBins) {
            const uint32_t *col = counts + uint64_t(pass) * G * kBins + tid;
            uint32_t before = 0, tot = 0;
            uint32_t g = 0;
            for (; g + 8 <= G; g += 8) {
                uint32_t x[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) x[u] = __ldcg(col + uint64_t(g + u) * kBins);
#pragma unroll
                for (int u = 0; u < 8; ++u) {
                    before += (g + u < c) ? x[u] : 0u;
                    tot += x[u];
                }
            }
            for (; g < G; ++g) {
                const uint32_t x = __ldcg(col + uint64_t(g) * kBins);
                before += g < c ? x : 0u;
                tot += x;
            }
            uint32_t inc = tot;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += y;
            }
            if (lane == 31) S.ws[w] = inc;
            S.base[tid] = inc - tot + before;  // + the totals of earlier warps' digits, below
        }
        __syncthreads();
        if (tid < kBins) {
            uint32_t pre = 0;
            for (int i = 0; i < (tid >> 5); ++i) pre += S.ws[i];
            const uint32_t b = S.base[tid] + pre;
#pragma unroll 8
            for (int ww = 0; ww < kWarps; ++ww) S.wcnt[ww][tid] += b;  // running global positions
        }
        __syncthreads();
        // sweep 2: stable positions in input order (warp, round, lane); scatter
        const bool last = pass == passes - 1;
        for (uint32_t r0 = w_lo; r0 < w_hi; r0 += 32) {
            const uint32_t i = r0 + lane;
            const bool valid = i < w_hi;
            const K key = valid ? S.k[i] : K(0);
            const uint32_t d = uint32_t(key >> sh) & 255u;
            const unsigned peers = match8(d, valid);
            const uint32_t b0 = valid ? S.wcnt[w][d] : 0u;
            __syncwarp();
            if (valid && lane == __ffs(peers) - 1) S.wcnt[w][d] = b0 + __popc(peers);
            __syncwarp();
            if (valid) {
                const uint64_t pos = uint64_t(b0) + __popc(peers & lanemask_lt());
                if (last) {
                    sink.store(pos, key, S.v[i]);
                } else {
                    kout[pos] = key;
                    vout[pos] = S.v[i];
                }
            }
        }
        if (!last) grid_barrier(bar, target);
    }
}

int g_ctas = 0;

template <class K, int kCap, class Src, class Sink>
cudaError_t launch_small(const Src &src, const Sink &sink, uint64_t n, int bits, void *scratch, cudaStream_t s) {
    auto kern = k_small_sort<K, kCap, Src, Sink>;
    const int smem = int(sizeof(SmallSmem<K, kCap>));
    static int ctas = 0;
    cudaError_t e;
    if (!ctas) {
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        int per_sm = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kT, smem);
        if (e != cudaSuccess) return e;
        if (per_sm < 1) return cudaErrorLaunchOutOfResources;
        ctas = num_sms();  // one CTA per SM (all co-resident: the launch is cooperative)
    }
    const int passes = (bits + 7) / 8;
    auto align = [](uintptr_t p) { return (p + 255) & ~uintptr_t(255); };
    uintptr_t a = align(reinterpret_cast<uintptr_t>(scratch));
    auto *bar = reinterpret_cast<unsigned int *>(a);
    a = align(a + 256);
    auto *counts = reinterpret_cast<uint32_t *>(a);
    a = align(a + uint64_t(passes) * ctas * kBins * 4);
    K *kb0 = reinterpret_cast<K *>(a);
    a = align(a + n * sizeof(K));
    K *kb1 = reinterpret_cast<K *>(a);
    a = align(a + n * sizeof(K));
    auto *vb0 = reinterpret_cast<uint32_t *>(a);
    a = align(a + n * 4);
    auto *vb1 = reinterpret_cast<uint32_t *>(a);
    if ((e = cudaMemsetAsync(bar, 0, 4, s)) != cudaSuccess) return e;
    void *args[] = {const_cast<Src *>(&src), const_cast<Sink *>(&sink), &n, &bits, &kb0, &vb0, &kb1, &vb1,
                    &counts, &bar};
    e = cudaLaunchCooperativeKernel(reinterpret_cast<const void *>(kern), dim3(ctas), dim3(kT), args, smem, s);
    note_launch();
    return e;
}

}  // namespace

constexpr int kCap32 = 20 * 1024, kCap64 = 12 * 1024;  // keys per CTA: shared memory holds the chunk

uint64_t small_sort_max_n(int key_bytes) {
    return uint64_t(num_sms()) * (key_bytes == 4 ? kCap32 : kCap64);
}

size_t small_sort_scratch_bytes(uint64_t n, int key_bytes) {
    return 256 * 8 + uint64_t(8) * num_sms() * kBins * 4 + 2 * n * (key_bytes + 4);
}

cudaError_t small_sort_index(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                             uint32_t *codes, uint32_t *locs, uint4 *recs, void *scratch, cudaStream_t s) {
    if (n_locs == 0) return cudaSuccess;
    if (n_locs > small_sort_max_n(4)) return cudaErrorInvalidValue;
    return launch_small<uint32_t, kCap32>(SrcSeeds{R, ls, step, k0}, SinkIndex{R, ls, codes, locs, recs}, n_locs,
                                             int(2 * ls), scratch, s);
}

cudaError_t small_sort_triples(const uint64_t *keys, const uint32_t *lens, uint64_t n, int bits, uint32_t qbits,
                               gpumem_triple *out, void *scratch, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    if (n > small_sort_max_n(8)) return cudaErrorInvalidValue;
    return launch_small<uint64_t, kCap64>(SrcKV64{keys, lens}, SinkTriples{out, qbits}, n, bits, scratch, s);
}

}  // namespace gm
