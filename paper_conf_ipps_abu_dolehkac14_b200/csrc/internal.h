// internal.h -- host-side declarations shared by the .cu files of libgpumem.so.
// Not part of the ABI (see include/gpumem.h). No torch types anywhere.
#pragma once
#include <cstdint>
#include <string>
#include <utility>
#include <vector>
#include <cuda_runtime.h>

#include "gpumem.h"

// A parsed multi-FASTA (fasta.cu): records concatenated with one masked separator base,
// non-ACGT letters masked (read as 'A'); masked positions as sorted half-open intervals.
struct gpumem_fasta {
    uint32_t magic;
    std::string seq;                          // concatenated ASCII (A C G T only)
    std::vector<std::string> names;
    std::vector<uint64_t> start, len;         // record i: seq[start[i], start[i] + len[i])
    std::vector<uint64_t> mask;               // masked intervals [mask[2j], mask[2j+1])
};

namespace gm {

constexpr uint32_t kMagicFasta = 0x47464153u;

// ---------------------------------------------------------------- runtime
struct Options {
    int64_t find_grid = 0;       // 0 = SMs x occupancy
    int64_t find_spill = 64;     // bucket sizes above this go to the heavy queue
    int64_t out_capacity = 0;    // 0 = automatic
    int64_t use_bitmap = 1;      // 1: rank-word probe + compact bucket table; 0: read the dense ptrs
    int64_t static_lb = 0;       // 1: each lane processes its own positions' hits (LB ablation)
    int64_t sort_impl = 0;       // output sort: 0 = auto (MSD below kMsdMaxN keys, else LSD), 1 = stable LSD radix
                                 // (radix.cu), 2 = MSD bucket sort (msd.cu)
    int64_t rec8 = -1;           // seed records: -1 auto (8-byte when step <= 8), 0 16-byte, 1 8-byte
    int64_t rank_sectors = -1;   // lookup directory: -1 auto (sectors when the compact table exceeds L2/4),
                                 // 0 rank words, 1 rank sectors
    int64_t radix_bits = 0;      // LSD digit width: 0 = 9 bits if that saves a pass else 8; or pinned 8, 9, 10
    int64_t pdl = 1;             // programmatic dependent launch between consecutive kernels
    int64_t find_hints = -1;     // k_find L2 cache-policy loads: -1 auto (seed records > L2 / 2), 0 off, 1 on
    int64_t q_chunks = 8;        // host-input pipelines: Q copied, packed and searched in this many pieces
                                 // (read at gpumem_pipeline_create; 1 = the whole Q after its copy)
    int64_t pipe_events = 0;     // stage event nodes in a pipeline graph: 0 none (fastest), 2 find only, 1 every
                                 // stage (each node costs a few us: C4 1.263 / 1.280 / 1.311 ms per step)
    int64_t index_alg1 = 0;      // Alg. 1 literally (atomic counts, scan, placement, bucket sort): 1 always,
                                 // -1 for dense indexes (n_locs >= 4^ls / 4), 0 never (default: measured
                                 // slower everywhere -- C5 L = 20 2.9 vs 1.4 ms, C4 0.40 vs 0.21 ms)
    int64_t index_tiled = -1;    // index build: 1 Alg. 1 tiled over the seed space (tindex.cu) where it
                                 // applies (sparse: n_locs < 4^ls / 4, ls <= 13), 0 the radix-sort path
                                 // (index.cu + radix.cu), -1 auto: tiled up to 2^20 locations (measured
                                 // faster at C1/C2, slower at C3-C5: DESIGN.md)
    int64_t l2_persist = 0;      // MB of L2 set aside for persisting lines (cudaLimitPersistingL2CacheSize);
                                 // 0 = none (default)
    int64_t l2_window = 0;       // k_find / k_heavy access-policy window over: 0 nothing, 1 the lookup
                                 // directory, 2 the compact table, 3 the seed records (hit ratio = set-aside
                                 // / window bytes)
};
extern Options g_opt;
// L2 access-policy window of the launches being issued (num_bytes == 0: none)
extern thread_local cudaAccessPolicyWindow g_l2win;

// Kernel launch with programmatic dependent launch (PDL): the next kernel on the stream
// may be scheduled while this one drains (its CTAs fill the SMs freed by finished
// ones); every kernel of the library begins with pdl_wait() (griddepcontrol.wait),
// which blocks until the preceding grid has completed and its writes are visible, so
// the overlap covers only launch latency and CTA ramp-up. In a captured graph the
// attribute becomes a programmatic dependency edge. g_opt.pdl = 0: ordinary launches.
template <typename... KArgs, typename... Args>
inline cudaError_t pdl_launch(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args &&...args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = g_opt.pdl ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (g_l2win.num_bytes) {  // set around the find launches only (launch_find / launch_heavy)
        attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[1].val.accessPolicyWindow = g_l2win;
        cfg.numAttrs = 2;
    }
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}
#ifdef __CUDACC__
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
#endif

void *dalloc(size_t bytes, cudaStream_t s);   // nullptr on failure (error text set)
void dfree(void *p, cudaStream_t s);
void note_launch(int n = 1);                  // launch counter
// bytes / 4 words of value v at p, as a (PDL) kernel instead of a memset node (pack.cu)
cudaError_t fill_async(void *p, uint32_t v, size_t bytes, cudaStream_t s);
int num_sms();

gpumem_status fail(gpumem_status st, const char *fmt, ...);
gpumem_status cuda_fail(cudaError_t e, const char *what);

// Brackets one stage with CUDA events when profiling is enabled.
// Inside a pipeline capture the events go to the pipeline instead (re-recorded by
// every graph launch).
struct Stage {
    Stage(const char *name, cudaStream_t s);
    ~Stage();
    int slot;
    cudaStream_t s;
    void *vec;
};

// ---------------------------------------------------------------- kernels (launchers)
// K1: ASCII -> 2-bit words (pack.cu): in[0, n) into words[0, n_words_alloc) (words past
// the data zero); an invalid byte at in[i] records pos_base + i (atomicMin) in *bad_pos.
// A chunk of a longer sequence starting at base 32j: in + 32j, words + j, pos_base 32j.
cudaError_t launch_pack(const uint8_t *in, uint64_t n, uint64_t *words, uint64_t n_words_alloc,
                        unsigned long long *bad_pos, cudaStream_t s, uint64_t pos_base = 0);

// Reverse complement of packed words (pack.cu).
cudaError_t launch_revcomp(const uint64_t *in, uint64_t n, uint64_t *out, uint64_t n_words_alloc, cudaStream_t s);

// Radix sort (radix.cu): stable LSD on bits [lo, bits) of the keys, values ride along.
// Ping-pongs between (k0,v0) and (k1,v1); returns true when the result is in (k1,v1).
// `scratch` must hold radix_scratch_bytes(n) bytes (digit counts + scan partials).
// vg_step != 0: v0 is not read -- the values are generated, value of key i = (vg_base + i) * vg_step
cudaError_t radix_sort_u32(uint32_t *k0, uint32_t *v0, uint32_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt, int lo = 0, uint64_t vg_base = 0,
                           uint32_t vg_step = 0);
// radix_sort_u64 with dn != null: n is a capacity, the count is min(*dn, n) on the device.
cudaError_t radix_sort_u64(uint64_t *k0, uint32_t *v0, uint64_t *k1, uint32_t *v1, uint64_t n, int bits,
                           void *scratch, cudaStream_t s, bool *in_alt, int lo = 0,
                           const unsigned long long *dn = nullptr);
size_t radix_scratch_bytes(uint64_t n);
int radix_passes(int bits, uint64_t n);  // LSD passes a sort of `bits` key bits of n keys runs

// MSD bucket sort of unique u64 keys (+ optional u32 values), in place, or written as
// triples {key >> qbits, key & qmask, val} when trip != null (msd.cu).
size_t msd_scratch_bytes(uint64_t n);
cudaError_t msd_sort(uint64_t *keys, uint32_t *vals, uint64_t n, int bits, void *scratch, cudaStream_t s,
                     gpumem_triple *trip = nullptr, uint32_t qbits = 0);
// The same with the key count in device memory (n = min(*d_n, cap)); capturable.
cudaError_t msd_sort_dev(uint64_t *keys, uint32_t *vals, const unsigned long long *d_n, uint64_t cap, int bits,
                         void *scratch, cudaStream_t s, gpumem_triple *trip, uint32_t qbits);
// Index (index.cu)
// sampled locations p = (k0 + k) * step for k in [0, n_locs)
cudaError_t launch_seed_codes(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                              uint32_t *codes, uint32_t *locs, cudaStream_t s);
size_t ptrs_fill_scratch_bytes(uint32_t ls);
// Alg. 1 tiled over the seed space (tindex.cu): partition the sampled locations into 2^H
// bins of 2^bbits seeds, then Alg. 1 steps 1-4 + directory + table + seed records per bin
// in shared memory. ok == 0: not applicable (ls > 13), use the radix path.
struct TiledPlan {
    uint32_t ok, H, bbits, wcap;  // 2^H bins of 2^bbits seeds; locations a warp takes per bin
};
TiledPlan tiled_plan(uint32_t ls, uint64_t n_locs);
size_t tiled_scratch_bytes(const TiledPlan &p, uint64_t n_locs);
// buckets must hold n_locs + 1 entries (gapped per bin, see tindex.cu)
cudaError_t launch_index_tiled(const TiledPlan &p, const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0,
                               uint64_t n_locs, unsigned long long *rankw, uint4 *rsect, uint2 *buckets, uint32_t *locs,
                               void *recs, int rec8, void *scratch, cudaStream_t s, cudaStream_t side = nullptr,
                               cudaEvent_t ev_fork = nullptr, cudaEvent_t ev_join = nullptr);
// Alg. 1 as written for dense indexes (index.cu): counts by atomics, prefix sums +
// directory, placement, per-bucket sort -> locs, directory, compact table.
size_t alg1_scratch_bytes(uint32_t ls, uint64_t n_locs);
cudaError_t launch_index_alg1(const uint64_t *R, uint32_t ls, uint32_t step, uint64_t k0, uint64_t n_locs,
                              unsigned long long *rankw, uint4 *rsect, uint2 *buckets, uint32_t *locs, void *scratch,
                              cudaStream_t s);
cudaError_t launch_ptrs_fill(const uint32_t *sorted_codes, uint64_t n_locs, uint32_t ls, uint32_t *ptrs,
                             unsigned long long *rankw, uint4 *rsect, uint2 *buckets, void *scratch,
                             cudaStream_t s, uint2 *hv_list = nullptr, unsigned int *hv_cnt = nullptr);
// Heavy buckets (> kHvT locations), listed by the directory fill into hv_list (hv_cnt[0]):
// each one's records reordered minority-left-flank first, hv_info sorted by first slot,
// hv_cnt[1] = how many (0 if more than kHvCap). Valid when step <= the records' left flank.
constexpr uint32_t kHvT = 64, kHvCap = 2048;
cudaError_t launch_heavy_prep(void *recs, int rec8, uint32_t step, const uint2 *hv_list, unsigned int *hv_cnt,
                              uint4 *hv_info, cudaStream_t s);
// Dense ptrs[0 .. 4^ls] from the rank directory (rankw or rsect) + compact table (index.cu).
cudaError_t launch_ptrs_expand(const unsigned long long *rankw, const uint4 *rsect, const uint2 *buckets, uint32_t ls,
                               uint64_t n_locs, uint32_t *ptrs, cudaStream_t s);
// Seed records for the lookup: rec[k] = {locs[k], 16 bases left of it, 32 bases right of its seed}
// (uint4), or with rec8 {locs[k], 8 bases left | 8 bases right << 16} (uint2).
cudaError_t launch_seed_recs(const uint64_t *R, uint32_t ls, const uint32_t *locs, uint64_t n_locs, void *recs,
                             int rec8, cudaStream_t s);

// Find (find.cu)
struct FindParams {
    const uint64_t *R;
    uint64_t nR;
    const uint64_t *Q;
    uint64_t nQ;
    uint64_t nQw;                // allocated words of Q (incl. padding)
    uint64_t q_avail;            // Q bases present (== nQ unless Q is streamed in chunks)
    const uint32_t *ptrs;
    const void *recs;            // seed records, parallel to locs: uint4 {p, R[p-16,p), R[p+ls,p+ls+32)}, or
    int rec8;                    // (rec8) uint2 {p, R[p-8,p) | R[p+ls,p+ls+8) << 16}
    const unsigned long long *rankw;  // per 32 seeds: {occupancy bits (low 32), occupied seeds before (high 32)}
    const uint4 *rsect;          // or (large indexes) per 32 seeds: {records before, occupied seeds before,
                                 // 2-bit saturating counts lo, hi}; exactly one of rankw / rsect is set
    const uint2 *buckets;        // per occupied seed, in seed order: {first slot in locs, count}
    uint32_t ls, L, step, qbits;
    uint64_t scan_lo, scan_hi;   // query seed positions scanned
    uint64_t own_lo, own_hi;     // MEM start q kept
    uint64_t *out_key;           // (r << qbits) | q
    uint32_t *out_len;
    uint64_t capacity;
    unsigned long long *out_count;
    unsigned int *tile_ctr;
    uint64_t n_tiles;
    uint32_t spill_t;
    uint4 *spill;                // {q, beg, len, 0}
    uint64_t spill_cap;
    unsigned long long *spill_count;
    unsigned long long *stats;   // [0] entries kept local, [1] hits kept local, [2] hits spilled, [3] entries spilled
    uint2 *coopq;                // hits whose extension exceeds kLaneCap: {p, q}
    uint64_t coop_cap;
    unsigned long long *coop_count;
    int use_bitmap;
    int static_lb;               // ablation: no hit redistribution across lanes
    int recs_stream;             // seed records too large to stay in L2: load them evict_first
    unsigned long long *work;    // [0] most hits one warp dealt locally, [1] warps (D5 balance)
    const uint4 *hv_info;        // heavy buckets sorted by first slot: {first, count, majority left flank,
                                 // minority count}; their records minority first (index.cu, k_hv_part)
    const unsigned int *hv_n;    // how many (null: none built)
    cudaAccessPolicyWindow l2win;  // persisting-L2 window of k_find / k_heavy (num_bytes 0: none)
};
uint64_t find_tile_positions(bool rank_sectors);  // query positions per scheduler chunk
cudaError_t launch_find(const FindParams &p, int grid, cudaStream_t s);
cudaError_t launch_heavy(const FindParams &p, cudaStream_t s);
cudaError_t launch_coop(const FindParams &p, cudaStream_t s);
cudaError_t launch_open_fix(const FindParams &p, cudaStream_t s);  // after streamed-Q finds
// pipeline report: counters, alphabet flags and balance stats into pinned host memory
cudaError_t launch_collect(const unsigned long long *ctr, const unsigned long long *rbad,
                           const unsigned long long *qbad, unsigned long long *host, cudaStream_t s);
int find_default_grid(bool rank_sectors);

// Instrumentation (diag.cu): best-of-4 time of n random 8-byte probes into a table of
// table_bytes (rounded down to a power of two), 8 independent probes per thread.
cudaError_t gather_ceiling(uint64_t n_probes, uint64_t table_bytes, cudaStream_t s, float *best_ms);

// Rare-MEM filter (variants.cu): the MEMs whose string occurs at most k times in R and
// at most k times in Q (1 <= k <= kRareMaxK; k = 1: MUMs), order kept; the kept count is
// written to *d_count (device).
constexpr int kRareMaxK = 15;
size_t rare_scratch_bytes(uint64_t n);
cudaError_t rare_filter(const gpumem_triple *in, uint64_t n, uint32_t k, gpumem_triple *out,
                        unsigned long long *d_count, void *scratch, cudaStream_t s);

// K9 merge (merge.cu): G <= kMergeMaxRuns runs, each sorted by (r, q), pairwise disjoint
// -> out (sum of counts triples) sorted by (r, q). The runs may be peer (IPC) memory.
constexpr int kMergeMaxRuns = 64;
size_t merge_scratch_bytes(int n_runs, uint64_t total);
cudaError_t merge_runs(const gpumem_triple *const *runs, const uint64_t *counts, int n_runs, gpumem_triple *out,
                       void *scratch, cudaStream_t s);

// Multi-record split (fasta.cu): the pieces (length >= L) of the MEMs `in` cut at the
// masked intervals of R (mr, nmr intervals) and Q (mq, nmq), as keys (r << qbits | q) and
// lengths at off[i] (exclusive scan of the per-MEM piece counts cnt); *d_total = pieces.
// Two phases: count + scan, then (keys, lens sized by *d_total) emit -- keys == nullptr
// runs the first phase only.
cudaError_t split_masked(const gpumem_triple *in, uint64_t n, const uint64_t *mr, uint64_t nmr, const uint64_t *mq,
                         uint64_t nmq, uint32_t L, uint32_t qbits, uint32_t *cnt, uint32_t *off,
                         unsigned long long *d_total, uint64_t *keys, uint32_t *lens, cudaStream_t s);

// Band sweep (band.cu): place a band's local triples (global r = r + w0) into the closed
// or open list, and continue carried open MEMs in the next window.
cudaError_t band_place(const gpumem_triple *in, uint64_t n, uint64_t w0, uint64_t wlen, int more,
                       gpumem_triple *closed, unsigned long long *n_closed, gpumem_triple *open,
                       unsigned long long *n_open, cudaStream_t s);
cudaError_t band_continue(const gpumem_triple *in, uint64_t n, const uint64_t *W, uint64_t w0, uint64_t wlen,
                          int more, const uint64_t *Q, uint64_t nQ, gpumem_triple *closed,
                          unsigned long long *n_closed, gpumem_triple *open, unsigned long long *n_open,
                          cudaStream_t s);

// Triples (sort.cu)
cudaError_t launch_keys_to_triples(const uint64_t *keys, const uint32_t *lens, uint64_t n, uint32_t qbits,
                                   gpumem_triple *out, cudaStream_t s, const unsigned long long *dn = nullptr);
cudaError_t launch_triples_to_keys(const gpumem_triple *in, uint64_t n, uint32_t qbits, uint64_t *keys,
                                   uint32_t *lens, cudaStream_t s);

inline uint32_t bits_for(uint64_t n) {  // bits needed to hold values in [0, n)
    uint32_t b = 0;
    while (b < 64 && (n >> b) > 0) ++b;
    return b ? b : 1;
}

}  // namespace gm
