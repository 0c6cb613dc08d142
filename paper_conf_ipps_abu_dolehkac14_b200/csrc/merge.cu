// merge.cu -- K9: rank-0 merge of G sorted, disjoint runs of (r, q, len) triples into
// one run sorted by (r, q) (it replaces the host merge-sort of the
// paper's out-tile triplets, §III-C2).
//
// A tree of two-way merge-path merges: ceil(log2 G) levels, each one pair of launches
// that merges every pair of runs of the level (an odd last run is copied along). Per
// level every triple is read once and written once, whatever the key distribution (no
// bucket can be skewed):
//  k_merge_split  for every output tile of kTile triples of every pair, the merge-path
//                 co-rank -- how many of the tile's first outputs come from run A -- by a
//                 binary search along the tile's starting cross diagonal;
//  k_merge_tile   one CTA per tile: its A and B slices (kTile triples together) go to
//                 shared memory as 64-bit keys (r << 32 | q) + lengths, each thread finds
//                 its kItems outputs' co-rank inside the tile by the same search and
//                 merges them sequentially; the tile is written back coalesced.
// Keys are unique across runs (the query shards are disjoint), so there are no ties.
// The runs may live in other GPUs' memory (CUDA IPC mappings of the ranks' results,
// dist.py): the first level then reads every peer's run over NVLink exactly once.
#include <vector>

#include "internal.h"

namespace gm {
namespace {

constexpr int kT = 256;
constexpr int kItems = 8;
constexpr int kTile = kT * kItems;  // outputs per CTA
constexpr int kMaxPairs = kMergeMaxRuns / 2;

__device__ __forceinline__ uint64_t key_of(const gpumem_triple &t) { return (uint64_t(t.r) << 32) | t.q; }

// One level: pair p merges (a[p], na[p]) and (b[p], nb[p]) into out[p]; tile_base[p] =
// the level's first tile of pair p (tile_base[n_pairs] = the level's tiles).
struct Level {
    const gpumem_triple *a[kMaxPairs];
    const gpumem_triple *b[kMaxPairs];
    gpumem_triple *out[kMaxPairs];
    uint32_t na[kMaxPairs], nb[kMaxPairs];
    uint32_t tile_base[kMaxPairs + 1];
    int n_pairs;
};

__device__ __forceinline__ int pair_of(const Level &L, uint32_t tile) {
    int p = 0;
    while (p + 1 < L.n_pairs && L.tile_base[p + 1] <= tile) ++p;
    return p;
}

// merge-path co-rank: the number of A elements among the first d outputs of merge(A, B)
template <class FA, class FB>
__device__ __forceinline__ uint32_t co_rank(FA a, FB b, uint32_t na, uint32_t nb, uint32_t d) {
    uint32_t lo = d > nb ? d - nb : 0, hi = d < na ? d : na;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (a(mid) < b(d - 1 - mid)) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// split[t] = the A elements before tile t's first output, for every tile of the level
__global__ void __launch_bounds__(kT) k_merge_split(const Level L, uint32_t *__restrict__ split) {
    pdl_wait();
    const uint32_t t = blockIdx.x * kT + threadIdx.x;
    if (t >= L.tile_base[L.n_pairs]) return;
    const int p = pair_of(L, t);
    const uint32_t d = (t - L.tile_base[p]) * uint32_t(kTile);
    const gpumem_triple *A = L.a[p], *B = L.b[p];
    split[t] = co_rank([&](uint32_t i) { return key_of(A[i]); }, [&](uint32_t j) { return key_of(B[j]); }, L.na[p],
                       L.nb[p], d);
}

struct TileSmem {
    uint64_t key[kTile];
    uint32_t len[kTile];
    gpumem_triple out[kTile];
};

__global__ void __launch_bounds__(kT) k_merge_tile(const Level L, const uint32_t *__restrict__ split) {
    pdl_wait();
    __shared__ TileSmem s;
    const uint32_t t = blockIdx.x;
    const int p = pair_of(L, t);
    const uint32_t na = L.na[p], nb = L.nb[p], n = na + nb;
    const uint32_t d0 = (t - L.tile_base[p]) * uint32_t(kTile), d1 = min(d0 + uint32_t(kTile), n);
    const uint32_t a0 = split[t], a1 = t + 1 == L.tile_base[p + 1] ? na : split[t + 1];
    const uint32_t ma = a1 - a0, m = d1 - d0, mb = m - ma;
    const gpumem_triple *A = L.a[p] + a0, *B = L.b[p] + (d0 - a0);
    // the tile's inputs: the A slice at [0, ma), the B slice at [ma, m)
    for (uint32_t i = threadIdx.x; i < m; i += kT) {
        const gpumem_triple x = i < ma ? A[i] : B[i - ma];
        s.key[i] = key_of(x);
        s.len[i] = x.len;
    }
    __syncthreads();
    const uint32_t dt = min(uint32_t(threadIdx.x) * kItems, m);
    uint32_t i = co_rank([&](uint32_t x) { return s.key[x]; }, [&](uint32_t y) { return s.key[ma + y]; }, ma, mb, dt);
    uint32_t j = dt - i;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        const uint32_t o = dt + k;
        if (o >= m) break;
        const bool take_a = j >= mb || (i < ma && s.key[i] < s.key[ma + j]);
        const uint32_t src = take_a ? i : ma + j;
        const uint64_t key = s.key[src];
        s.out[o] = gpumem_triple{uint32_t(key >> 32), uint32_t(key), s.len[src]};
        if (take_a) ++i; else ++j;
    }
    __syncthreads();
    const uint32_t *src = reinterpret_cast<const uint32_t *>(s.out);
    uint32_t *dst = reinterpret_cast<uint32_t *>(L.out[p] + d0);
    for (uint32_t w = threadIdx.x; w < m * 3; w += kT) dst[w] = src[w];
}

uint32_t tiles_of(uint64_t n) { return uint32_t((n + kTile - 1) / kTile); }

}  // namespace

size_t merge_scratch_bytes(int n_runs, uint64_t total) {
    (void)n_runs;  // two ping-pong levels of triples + the split table of the largest level
    return size_t(2) * (total ? total : 1) * sizeof(gpumem_triple) + size_t(tiles_of(total) + kMaxPairs + 1) * 4 +
           1024;
}

cudaError_t merge_runs(const gpumem_triple *const *runs, const uint64_t *counts, int n_runs, gpumem_triple *out,
                       void *scratch, cudaStream_t s) {
    if (n_runs < 1 || n_runs > kMergeMaxRuns) return cudaErrorInvalidValue;
    uint64_t total = 0;
    std::vector<std::pair<const gpumem_triple *, uint64_t>> cur;
    for (int h = 0; h < n_runs; ++h) {
        total += counts[h];
        if (counts[h]) cur.push_back({runs[h], counts[h]});
    }
    if (total == 0) return cudaSuccess;
    if (total >= (1ull << 32)) return cudaErrorInvalidValue;
    if (cur.size() == 1)
        return cudaMemcpyAsync(out, cur[0].first, total * sizeof(gpumem_triple), cudaMemcpyDeviceToDevice, s);
    auto align = [](uintptr_t x) { return (x + 255) & ~uintptr_t(255); };
    uintptr_t c = align(reinterpret_cast<uintptr_t>(scratch));
    gpumem_triple *buf[2];
    buf[0] = reinterpret_cast<gpumem_triple *>(c);
    c = align(c + total * sizeof(gpumem_triple));
    buf[1] = reinterpret_cast<gpumem_triple *>(c);
    c = align(c + total * sizeof(gpumem_triple));
    auto *split = reinterpret_cast<uint32_t *>(c);
    for (int level = 0; cur.size() > 1; ++level) {
        // every run of the next level lands in this level's buffer (the last level: out),
        // so a level never writes the buffer it reads
        gpumem_triple *dst = cur.size() == 2 ? out : buf[level & 1];
        Level L{};
        std::vector<std::pair<const gpumem_triple *, uint64_t>> nxt;
        uint64_t off = 0;
        uint32_t tiles = 0;
        size_t k = 0;
        for (; k + 1 < cur.size(); k += 2) {
            const int p = L.n_pairs++;
            const uint64_t n = cur[k].second + cur[k + 1].second;
            L.a[p] = cur[k].first;
            L.b[p] = cur[k + 1].first;
            L.na[p] = uint32_t(cur[k].second);
            L.nb[p] = uint32_t(cur[k + 1].second);
            L.out[p] = dst + off;
            L.tile_base[p] = tiles;
            tiles += tiles_of(n);
            nxt.push_back({dst + off, n});
            off += n;
        }
        L.tile_base[L.n_pairs] = tiles;
        if (k < cur.size()) {  // the odd last run: copied along
            const cudaError_t e = cudaMemcpyAsync(dst + off, cur[k].first, cur[k].second * sizeof(gpumem_triple),
                                                  cudaMemcpyDeviceToDevice, s);
            if (e != cudaSuccess) return e;
            nxt.push_back({dst + off, cur[k].second});
        }
        pdl_launch(k_merge_split, (tiles + kT - 1) / kT, kT, 0, s, L, split);
        pdl_launch(k_merge_tile, tiles, kT, 0, s, L, static_cast<const uint32_t *>(split));
        note_launch(2);
        cur.swap(nxt);
    }
    return cudaGetLastError();
}

}  // namespace gm
