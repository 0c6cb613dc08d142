// merge.cu -- K9: rank-0 merge of G sorted, disjoint runs of (r, q, len) triples into
// one run sorted by (r, q) (it replaces the host merge-sort of
// the paper's out-tile triplets, §III-C2). One read and one write
// of every triple, instead of re-sorting the concatenation:
//
//  prep    (1 thread) the largest r over the runs (their last triples: runs are
//          sorted by r first) -> the bucket shift, so that r >> shift spreads the
//          triples over 2^nb_log buckets of ~kAvg triples;
//  dir     D[h][b] = first index of run h whose r >> shift >= b, a binary search
//          per (run, bucket) boundary: every bucket is a contiguous slice of every
//          run, and bucket b's slice of the output starts at sum_h D[h][b];
//  bucket  one CTA per bucket: the G slices (<= kCap triples together) go to shared
//          memory as 64-bit keys (r << 32 | q); each triple's place in the bucket is
//          its index in its own slice + the number of smaller keys in every other
//          slice (binary search in shared memory; keys are unique across runs); the
//          bucket is written back coalesced. A bucket over kCap (many MEMs with one r:
//          low-complexity repeats) is ranked the same way with the searches in global
//          memory.
//
// The runs may live in other GPUs' memory (CUDA IPC mappings of the ranks' result
// buffers, dist.py): then this kernel is the gather and the merge in one pass, each
// triple crossing NVLink once, read directly by the CTA that places it.
#include "internal.h"

namespace gm {
namespace {

constexpr int kT = 256;
constexpr int kCap = 2048;            // triples per bucket held in shared memory
constexpr int kAvg = 512;             // target mean bucket size (kCap / 4: headroom for skew)
constexpr int kMaxLog = 20;           // at most 2^20 buckets

struct MergeRuns {
    const gpumem_triple *run[kMergeMaxRuns];
    uint64_t n[kMergeMaxRuns];
    int g;
};

__device__ __forceinline__ uint64_t key_of(const gpumem_triple &t) { return (uint64_t(t.r) << 32) | t.q; }

__global__ void k_merge_prep(const MergeRuns runs, int nb_log, uint32_t *__restrict__ shift_out) {
    pdl_wait();
    if (threadIdx.x || blockIdx.x) return;
    uint32_t maxr = 0;
    for (int h = 0; h < runs.g; ++h)
        if (runs.n[h]) maxr = max(maxr, runs.run[h][runs.n[h] - 1].r);
    const uint32_t rbits = maxr ? 32u - uint32_t(__clz(int(maxr))) : 1u;  // bits to hold maxr
    *shift_out = rbits > uint32_t(nb_log) ? rbits - uint32_t(nb_log) : 0u;
}

// D[h * (nb + 1) + b], b in [0, nb]: first index of run h with (r >> shift) >= b
__global__ void __launch_bounds__(kT) k_merge_dir(const MergeRuns runs, uint32_t nb, const uint32_t *__restrict__ shift_p,
                                                   uint32_t *__restrict__ D) {
    pdl_wait();
    const uint32_t shift = *shift_p;
    const uint64_t total = uint64_t(runs.g) * (nb + 1);
    for (uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x; i < total; i += uint64_t(gridDim.x) * kT) {
        const int h = int(i / (nb + 1));
        const uint32_t b = uint32_t(i % (nb + 1));
        const gpumem_triple *t = runs.run[h];
        uint64_t lo = 0, hi = runs.n[h];
        if (b == nb) lo = hi;
        while (lo < hi) {
            const uint64_t mid = (lo + hi) >> 1;
            if ((uint64_t(t[mid].r) >> shift) < b) lo = mid + 1; else hi = mid;
        }
        D[i] = uint32_t(lo);
    }
}

struct BucketSmem {
    uint64_t key[kCap];
    uint32_t len[kCap];
    gpumem_triple out[kCap];
    uint32_t off[kMergeMaxRuns + 1];   // slice h of the bucket: [off[h], off[h+1]) in key[]
    uint32_t lo[kMergeMaxRuns];        // ... = run h's [lo[h], lo[h] + off[h+1] - off[h])
};

// number of keys < k in a[0, n)
template <class F>
__device__ __forceinline__ uint32_t count_less(F at, uint32_t n, uint64_t k) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (at(mid) < k) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kT) k_merge_bucket(const MergeRuns runs, uint32_t nb, const uint32_t *__restrict__ D,
                                                      gpumem_triple *__restrict__ out) {
    pdl_wait();
    extern __shared__ __align__(16) unsigned char smem_raw[];
    BucketSmem &s = *reinterpret_cast<BucketSmem *>(smem_raw);
    const uint32_t b = blockIdx.x;
    const int G = runs.g;
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (int h = 0; h < G; ++h) {
            const uint32_t a = D[uint64_t(h) * (nb + 1) + b], z = D[uint64_t(h) * (nb + 1) + b + 1];
            s.lo[h] = a;
            s.off[h] = acc;
            acc += z - a;
        }
        s.off[G] = acc;
    }
    __syncthreads();
    uint64_t base = 0;  // the bucket's first output slot: triples of all runs in earlier buckets
    for (int h = 0; h < G; ++h) base += D[uint64_t(h) * (nb + 1) + b];
    const uint32_t nbk = s.off[G];
    if (nbk == 0) return;
    if (nbk <= uint32_t(kCap)) {
        for (uint32_t i = threadIdx.x; i < nbk; i += kT) {
            int g = 0;
            while (s.off[g + 1] <= i) ++g;
            const gpumem_triple t = runs.run[g][s.lo[g] + (i - s.off[g])];
            s.key[i] = key_of(t);
            s.len[i] = t.len;
        }
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < nbk; i += kT) {
            int g = 0;
            while (s.off[g + 1] <= i) ++g;
            const uint64_t k = s.key[i];
            uint32_t rank = i - s.off[g];
            for (int h = 0; h < G; ++h) {
                if (h == g) continue;
                const uint32_t o = s.off[h];
                rank += count_less([&](uint32_t j) { return s.key[o + j]; }, s.off[h + 1] - o, k);
            }
            s.out[rank] = gpumem_triple{uint32_t(k >> 32), uint32_t(k), s.len[i]};
        }
        __syncthreads();
        // coalesced write-back: the bucket's triples as 32-bit words
        const uint32_t *src = reinterpret_cast<const uint32_t *>(s.out);
        uint32_t *dst = reinterpret_cast<uint32_t *>(out + base);
        for (uint32_t w = threadIdx.x; w < nbk * 3; w += kT) dst[w] = src[w];
        return;
    }
    // oversized bucket: the same ranks, searched in global memory
    for (uint32_t i = threadIdx.x; i < nbk; i += kT) {
        int g = 0;
        while (s.off[g + 1] <= i) ++g;
        const gpumem_triple t = runs.run[g][s.lo[g] + (i - s.off[g])];
        const uint64_t k = key_of(t);
        uint64_t rank = i - s.off[g];
        for (int h = 0; h < G; ++h) {
            if (h == g) continue;
            const gpumem_triple *th = runs.run[h] + s.lo[h];
            rank += count_less([&](uint32_t j) { return key_of(th[j]); }, s.off[h + 1] - s.off[h], k);
        }
        out[base + rank] = t;
    }
}

}  // namespace

static int merge_nb_log(uint64_t total) {  // buckets of ~kAvg triples
    int nb_log = 0;
    while (nb_log < kMaxLog && (uint64_t(kAvg) << nb_log) < total) ++nb_log;
    return nb_log;
}

size_t merge_scratch_bytes(int n_runs, uint64_t total) {
    return (size_t(n_runs) * ((size_t(1) << merge_nb_log(total)) + 1) + 64) * 4;
}

cudaError_t merge_runs(const gpumem_triple *const *runs, const uint64_t *counts, int n_runs, gpumem_triple *out,
                       void *scratch, cudaStream_t s) {
    if (n_runs < 1 || n_runs > kMergeMaxRuns) return cudaErrorInvalidValue;
    MergeRuns mr{};
    uint64_t total = 0;
    for (int h = 0; h < n_runs; ++h) {
        mr.run[h] = runs[h];
        mr.n[h] = counts[h];
        total += counts[h];
    }
    mr.g = n_runs;
    if (total == 0) return cudaSuccess;
    const int nb_log = merge_nb_log(total);
    const uint32_t nb = 1u << nb_log;
    auto *shift = static_cast<uint32_t *>(scratch);
    uint32_t *D = shift + 64;
    static bool attr = false;
    if (!attr) {
        const cudaError_t e = cudaFuncSetAttribute(k_merge_bucket, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                   int(sizeof(BucketSmem)));
        if (e != cudaSuccess) return e;
        attr = true;
    }
    pdl_launch(k_merge_prep, 1, 32, 0, s, mr, nb_log, shift);
    const uint64_t dir_n = uint64_t(n_runs) * (nb + 1);
    const uint64_t dir_blocks = (dir_n + kT - 1) / kT;
    pdl_launch(k_merge_dir, unsigned(dir_blocks < 4096 ? dir_blocks : 4096), kT, 0, s, mr, nb,
               static_cast<const uint32_t *>(shift), D);
    pdl_launch(k_merge_bucket, nb, kT, sizeof(BucketSmem), s, mr, nb, static_cast<const uint32_t *>(D), out);
    note_launch(3);
    return cudaGetLastError();
}

}  // namespace gm
