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
//          bucket is written back coalesced. A bucket over kCap (many MEMs in a narrow
//          r range: low-complexity repeats) is split evenly over its key range into
//          sub-buckets merged the same way; one still over kCap (keys that do not
//          spread) is ranked with the searches in global memory.
//
// The runs may live in other GPUs' memory (CUDA IPC mappings of the ranks' result
// buffers, dist.py): then this kernel is the gather and the merge in one pass, each
// triple crossing NVLink once, read directly by the CTA that places it.
#include "internal.h"

namespace gm {
namespace {

constexpr int kT = 256;
#ifndef GM_MERGE_BT
#define GM_MERGE_BT 512
#endif
#ifndef GM_MERGE_CAP
#define GM_MERGE_CAP 4096
#endif
constexpr int kBT = GM_MERGE_BT;      // threads of the bucket kernel
constexpr int kCap = GM_MERGE_CAP;    // triples per bucket held in shared memory
constexpr int kAvg = kCap / 4;        // target mean bucket size (headroom for skew)
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

constexpr int kSubB = 32;            // sub-buckets of an oversized bucket handled per batch

struct BucketSmem {
    uint64_t key[kCap];
    uint32_t len[kCap];
    uint16_t perm[kCap];               // perm[rank] = the triple's slot in key[] / len[]
    uint32_t off[kMergeMaxRuns + 1];   // the slices being merged: slice h is key[off[h], off[h+1])
    uint32_t lo[kMergeMaxRuns];        // ... = run h's [lo[h], lo[h] + off[h+1] - off[h])
    uint32_t blo[kMergeMaxRuns];       // the bucket's slices (oversized buckets: split further)
    uint32_t bhi[kMergeMaxRuns];
    uint32_t sb[kMergeMaxRuns * (kSubB + 1)];  // sub-bucket boundaries, [h][j]
    uint64_t kmin, kmax;
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

// Merge the slices in s.lo / s.off (n <= kCap triples together) into out[0, n): keys to
// shared memory, each triple's rank = its index in its slice + the smaller keys of every
// other slice (binary searches in shared memory), coalesced write-back. All threads.
__device__ void merge_in_smem(BucketSmem &s, const MergeRuns &runs, gpumem_triple *__restrict__ out) {
    const int G = runs.g;
    const uint32_t n = s.off[G];
    for (uint32_t i = threadIdx.x; i < n; i += kBT) {
        int g = 0;
        while (s.off[g + 1] <= i) ++g;
        const gpumem_triple t = runs.run[g][s.lo[g] + (i - s.off[g])];
        s.key[i] = key_of(t);
        s.len[i] = t.len;
    }
    __syncthreads();
    // rank of a triple = its index in its slice + the smaller keys of every other slice
    for (uint32_t i = threadIdx.x; i < n; i += kBT) {
        int g = 0;
        while (s.off[g + 1] <= i) ++g;
        const uint64_t k = s.key[i];
        uint32_t rank = i - s.off[g];
        for (int h = 0; h < G; ++h) {
            if (h == g) continue;
            const uint32_t o = s.off[h];
            rank += count_less([&](uint32_t j) { return s.key[o + j]; }, s.off[h + 1] - o, k);
        }
        s.perm[rank] = uint16_t(i);
    }
    __syncthreads();
    uint32_t *dst = reinterpret_cast<uint32_t *>(out);  // coalesced write-back: consecutive triples
    for (uint32_t e = threadIdx.x; e < n; e += kBT) {
        const uint32_t src = s.perm[e];
        const uint64_t k = s.key[src];
        dst[3 * e] = uint32_t(k >> 32);
        dst[3 * e + 1] = uint32_t(k);
        dst[3 * e + 2] = s.len[src];
    }
    __syncthreads();
}

// The same ranks with the searches in global memory (a slice set over kCap whose keys
// could not be split further). All threads.
__device__ void merge_in_global(BucketSmem &s, const MergeRuns &runs, gpumem_triple *__restrict__ out) {
    const int G = runs.g;
    const uint32_t n = s.off[G];
    for (uint32_t i = threadIdx.x; i < n; i += kBT) {
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
        out[rank] = t;
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kBT) k_merge_bucket(const MergeRuns runs, uint32_t nb, const uint32_t *__restrict__ D,
                                                       gpumem_triple *__restrict__ out) {
    pdl_wait();
    extern __shared__ __align__(16) unsigned char smem_raw[];
    BucketSmem &s = *reinterpret_cast<BucketSmem *>(smem_raw);
    const uint32_t b = blockIdx.x;
    const int G = runs.g;
    if (int(threadIdx.x) < G) {  // the bucket's slice of every run, loaded in parallel
        const uint64_t r0 = uint64_t(threadIdx.x) * (nb + 1) + b;
        s.lo[threadIdx.x] = s.blo[threadIdx.x] = D[r0];
        s.bhi[threadIdx.x] = D[r0 + 1];
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (int h = 0; h < G; ++h) {
            s.off[h] = acc;
            acc += s.bhi[h] - s.blo[h];
        }
        s.off[G] = acc;
    }
    __syncthreads();
    uint64_t base = 0;  // the bucket's first output slot: triples of all runs in earlier buckets
    for (int h = 0; h < G; ++h) base += s.blo[h];
    const uint32_t nbk = s.off[G];
    if (nbk == 0) return;
    if (nbk <= uint32_t(kCap)) {
        merge_in_smem(s, runs, out + base);
        return;
    }
    // Oversized bucket (many MEMs in a narrow r range: low-complexity repeats): split its
    // key range [kmin, kmax] evenly into sub-buckets of ~kCap/2 expected triples, slice
    // boundaries by binary search in each run, each sub-bucket merged like a bucket.
    if (threadIdx.x == 0) {
        uint64_t mn = ~0ull, mx = 0;
        for (int h = 0; h < G; ++h) {
            if (s.bhi[h] == s.blo[h]) continue;
            mn = min(mn, key_of(runs.run[h][s.blo[h]]));
            mx = max(mx, key_of(runs.run[h][s.bhi[h] - 1]));
        }
        s.kmin = mn;
        s.kmax = mx;
    }
    __syncthreads();
    const uint64_t kmin = s.kmin, span = s.kmax - s.kmin;  // keys in [kmin, kmin + span]
    uint32_t nsub = (nbk + kCap / 2 - 1) / (kCap / 2);
    if (uint64_t(nsub) > span + 1) nsub = uint32_t(span + 1);
    const uint64_t w = span / nsub + 1;                       // nsub * w > span
    uint64_t sbase = base;
    for (uint32_t j0 = 0; j0 < nsub; j0 += kSubB) {
        const uint32_t jn = min(uint32_t(kSubB), nsub - j0);
        for (uint32_t x = threadIdx.x; x < uint32_t(G) * (jn + 1); x += kBT) {
            const int h = int(x / (jn + 1));
            const uint32_t j = x % (jn + 1);
            uint32_t v = s.bhi[h];
            if (j0 + j < nsub) {  // first index of run h's slice with key >= kmin + (j0 + j) * w
                const gpumem_triple *th = runs.run[h] + s.blo[h];
                v = s.blo[h] + count_less([&](uint32_t i) { return key_of(th[i]); }, s.bhi[h] - s.blo[h],
                                          kmin + uint64_t(j0 + j) * w);
            }
            s.sb[h * (kSubB + 1) + j] = v;
        }
        __syncthreads();
        for (uint32_t j = 0; j < jn; ++j) {
            if (threadIdx.x == 0) {
                uint32_t acc = 0;
                for (int h = 0; h < G; ++h) {
                    const uint32_t a = s.sb[h * (kSubB + 1) + j], z = s.sb[h * (kSubB + 1) + j + 1];
                    s.lo[h] = a;
                    s.off[h] = acc;
                    acc += z - a;
                }
                s.off[G] = acc;
            }
            __syncthreads();
            const uint32_t n = s.off[G];
            if (n && n <= uint32_t(kCap)) merge_in_smem(s, runs, out + sbase);
            else if (n) merge_in_global(s, runs, out + sbase);
            sbase += n;
        }
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
    pdl_launch(k_merge_bucket, nb, kBT, sizeof(BucketSmem), s, mr, nb, static_cast<const uint32_t *>(D), out);
    note_launch(3);
    return cudaGetLastError();
}

}  // namespace gm
