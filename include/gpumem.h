/*
 * include/gpumem.h -- C ABI of libgpumem.so, the B200 (sm_100a) MEM finder.
 *
 * Problem (Sec. II): given a reference R, a query Q over
 * Sigma = {A,C,G,T} (:58) and an integer L, report every maximal exact match
 * (r, q, len): R[r+i] == Q[q+i] for i < len, len >= L, R[r-1] != Q[q-1] and
 * R[r+len] != Q[q+len], where a sequence end counts as a mismatch
 * (reading R3). Positions are 0-based; sequences hold < 2^32 bases
 * (32-bit locations).
 *
 * Method (GPUMEM, Sec. III): index every step-th seed of length
 * seed_len of R with step = L - seed_len + 1 (Eq. 1, :86-90), look up the seed
 * at every query position, extend each hit both ways, keep len >= L and report
 * each MEM once (:151-153, :171-173). Every step runs in hand-written CUDA
 * kernels on the caller's device; there is no CPU fallback.
 *
 * Conventions for every call:
 *  - Device: the calling thread's current CUDA device (cudaSetDevice). All
 *    handles passed to one call must live on that device.
 *  - Streams: `cuda_stream` is a cudaStream_t passed as void* (NULL = the legacy
 *    default stream). Work is enqueued on it; calls documented "async" return
 *    before the GPU finishes. Handles are immutable after creation, so several
 *    streams may read one handle concurrently; the caller orders creation,
 *    use and gpumem_free across streams (free is enqueued on the handle's
 *    creation stream).
 *  - Memory: the library allocates device memory through the allocator hook
 *    (default: cudaMallocAsync / cudaFreeAsync on the stream, pool kept cached).
 *    Every handle is owned by the caller and released with gpumem_free.
 *  - Errors: every call returns gpumem_status. On failure *out is set to NULL,
 *    nothing leaks, and gpumem_last_error() (thread-local) says why. CUDA
 *    errors map to GPUMEM_ERR_CUDA with cudaGetErrorString's text. No call
 *    aborts or exits.
 */
#ifndef GPUMEM_H
#define GPUMEM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GPUMEM_OK = 0,
    GPUMEM_ERR_ARG = 1,         /* bad argument (NULL, ls/L/step out of range, wrong handle type) */
    GPUMEM_ERR_ALPHABET = 2,    /* a byte outside {A,C,G,T,a,c,g,t} (Sigma; reading R4) */
    GPUMEM_ERR_RANGE = 3,       /* length >= 2^32, q range outside Q, host buffer too small */
    GPUMEM_ERR_NOMEM = 4,       /* allocator returned NULL */
    GPUMEM_ERR_CUDA = 5,        /* a CUDA runtime error (message in gpumem_last_error) */
    GPUMEM_ERR_UNSUPPORTED = 6  /* no sm_100 device / unsupported request */
} gpumem_status;

typedef struct gpumem_seq gpumem_seq;     /* 2-bit packed sequence resident on one device        */
typedef struct gpumem_index gpumem_index; /* locs[n_locs] + lookup directory (ptrs on demand); refs R */
typedef struct gpumem_mems gpumem_mems;   /* MEM set sorted by (r, q), device-resident            */
typedef struct gpumem_pipeline gpumem_pipeline; /* the whole path captured as one CUDA graph        */

/* One MEM (Table I :34-35): R[r .. r+len) == Q[q .. q+len). 12 bytes, AoS. */
typedef struct {
    uint32_t r, q, len;
} gpumem_triple;

/*
 * gpumem_pack -- 2-bit encode a sequence (A=00, C=01, G=10, T=11).
 *  bases            n ASCII bytes; lowercase is folded; anything else is an alphabet error.
 *  bases_on_device  1: `bases` is a device pointer on the current device (read in place);
 *                   0: `bases` is host memory, copied to the device inside the call
 *                      (async if pinned) -- the copy is part of this call's stream work.
 *  Layout of the result: uint64 words, base i in bits [63-2(i%32), 62-2(i%32)] of
 *  word i/32 (first base most significant), 4 zero words of padding after the last.
 *  Async. Alphabet validation runs on the GPU; its verdict is reported by
 *  gpumem_seq_check() and by gpumem_find_mems() (which synchronises anyway).
 *  n == 0 is allowed (empty sequence). n >= 2^32 -> GPUMEM_ERR_RANGE.
 */
gpumem_status gpumem_pack(const char *bases, uint64_t n, int bases_on_device,
                          void *cuda_stream, gpumem_seq **out);

/* Reverse complement of a packed sequence (NEXT-F4; the paper's problem is forward-only,
 * reading R17): base i of the result is the complement of base n-1-i (A<->T, C<->G).
 * MEMs on the reverse strand are gpumem_find_mems(idx, revcomp(Q)); their q is a position
 * in the reverse-complemented query (the forward-strand interval is [|Q|-q-len, |Q|-q)).
 * The alphabet verdict of the input is carried over. Async. */
gpumem_status gpumem_revcomp(const gpumem_seq *in, void *cuda_stream, gpumem_seq **out);

/* Synchronises `cuda_stream`; GPUMEM_ERR_ALPHABET (with the first bad position in the
 * message) if the packed input held a byte outside the alphabet, else GPUMEM_OK. */
gpumem_status gpumem_seq_check(const gpumem_seq *s, void *cuda_stream);

/* Length in bases and the device pointer to the packed words (borrowed). */
gpumem_status gpumem_seq_info(const gpumem_seq *s, uint64_t *n_bases, const uint64_t **dev_words,
                              uint64_t *n_words);

/*
 * gpumem_index_build -- GPUMEM's lightweight index of R (Sec. III-A, Alg. 1 :102-106).
 *  seed_len (ls) in [1, 15], min_len (L) >= ls, step = L - ls + 1 (the maximum allowed by
 *  Eq. 1, :88-90). Indexed locations: p = 0, step, 2*step, ... <= |R| - ls (reading R6).
 *  Result: locs (n_locs uint32, sorted ascending inside each seed, Alg. 1 step 4) and the
 *  lookup directory: per 32 seeds an occupancy/rank word (or rank sector), plus the
 *  compact table {first slot, count} of the occupied seeds (one entry per sampled
 *  location at most: each chunk of seeds indexes its entries from its first slot) -- an
 *  exact, compressed form of the paper's ptrs (4^ls + 1 uint32, ptrs[s] = first slot of
 *  seed s, ptrs[4^ls] = n_locs, :84; 268 MB at ls = 13), which is expanded from it only on demand
 *  (gpumem_index_view, or find with option use_bitmap = 0). The index references R: R
 *  must outlive it. Async.
 */
gpumem_status gpumem_index_build(const gpumem_seq *R, uint32_t seed_len, uint32_t min_len,
                                 void *cuda_stream, gpumem_index **out);

/* Test-only: same with an explicit step in [1, L - ls + 1] (the MEM set does not depend on it). */
gpumem_status gpumem_index_build_step(const gpumem_seq *R, uint32_t seed_len, uint32_t min_len,
                                      uint32_t step, void *cuda_stream, gpumem_index **out);

/*
 * gpumem_index_build_range -- partial index of one band of R (the paper's tile-row
 *  index: "only a partial index is created for l_tile base pairs of
 *  reference"): only sampled locations p with r_begin <= p < r_end are indexed (same
 *  stride, same phase as the whole index, reading R6). Extensions still read the whole
 *  of R, so gpumem_find_mems on a band index returns exactly the MEMs whose canonical
 *  (leftmost sampled) seed lies in the band; the bands of a partition of [0, |R|) give
 *  disjoint MEM sets whose union is the whole set. r_begin > r_end -> GPUMEM_ERR_RANGE.
 */
gpumem_status gpumem_index_build_range(const gpumem_seq *R, uint32_t seed_len, uint32_t min_len,
                                       uint64_t r_begin, uint64_t r_end, void *cuda_stream,
                                       gpumem_index **out);

/*
 * gpumem_find_mems_banded -- the paper's reference row sweep (NEXT-F2; PAPER.md:76-80
 *  §III "only a partial index is created for l_tile base pairs of reference", :92 §III-A)
 *  for an R that need not fit in device memory: r_bases_host (ASCII, host, r_len bases)
 *  is processed in bands of band_len bases (0 = one band; rounded up to a multiple of the
 *  step). Only one window of R is resident at a time: the band plus `step` bases before
 *  it and max(L, 1024) after it, copied, packed and indexed over the band's sampled seeds
 *  (gpumem_index_build_range on the window), then searched against all of Q (resident,
 *  packed). A MEM cut by its window's right end is carried to the next band and its
 *  extension continued there (replacing the out-tile combining of PAPER.md:179-185).
 *  *out: the same set as gpumem_find_mems on the whole of R, sorted by (r, q). stats
 *  (optional): bands, band_len used, largest window in bytes, MEMs carried across
 *  windows, MEMs. Synchronises once per band. Errors as gpumem_index_build /
 *  gpumem_find_mems; *out NULL on error, nothing leaked.
 */
typedef struct {
    uint64_t bands, band_len, window_bytes, carried, mems;
} gpumem_band_stats;
gpumem_status gpumem_find_mems_banded(const char *r_bases_host, uint64_t r_len, const gpumem_seq *Q, uint32_t seed_len,
                                      uint32_t min_len, uint64_t band_len, void *cuda_stream, gpumem_mems **out,
                                      gpumem_band_stats *stats);

/* Borrowed device pointers to ptrs (4^ls + 1 entries) and locs (n_locs entries). The first
 * request for ptrs expands it on the index's stream and synchronises that stream. */
gpumem_status gpumem_index_view(const gpumem_index *idx, const uint32_t **dev_ptrs,
                                const uint32_t **dev_locs, uint64_t *n_locs);

/*
 * gpumem_find_mems -- every MEM of (R, Q, L) whose query start q lies in [q_begin, q_end)
 *  (q_end clamped to |Q|; 0, UINT64_MAX = all of Q), sorted ascending by (r, q), each
 *  exactly once (PAPER.md:153 "not to extract a MEM more than once", :185). The set is
 *  independent of ls and step. q_begin > |Q| -> GPUMEM_ERR_RANGE.
 *  Synchronises the stream once (the output size is data-dependent) and reports an
 *  alphabet error of R or Q here. Edge cases: |R| < ls or |Q| < L -> OK with 0 MEMs;
 *  R == Q includes (0, 0, |R|). Forward strand only.
 */
gpumem_status gpumem_find_mems(const gpumem_index *idx, const gpumem_seq *Q, uint64_t q_begin,
                               uint64_t q_end, void *cuda_stream, gpumem_mems **out);

/* Work counters of the find call that produced `m` (diagnostics; the bench derives the
 * find kernel's algorithmic bytes from them). */
typedef struct {
    uint64_t positions;      /* query seed positions scanned                                 */
    uint64_t occupied;       /* of those, positions whose seed occurs in the index           */
    uint64_t hits;           /* (sampled r, q) pairs with equal seeds that were examined      */
    uint64_t spilled_chunks; /* heavy-bucket chunks drained by the heavy kernel               */
    uint64_t mems;           /* MEMs reported                                                */
    uint32_t attempts;       /* 1, or 2 after an output-capacity overflow                     */
    uint64_t max_warp_hits;  /* D5 balance: the most hits one warp of the search dealt itself  */
    uint64_t warps;          /* ... over this many warps (mean = (hits - spilled hits) / warps) */
} gpumem_find_stats;
gpumem_status gpumem_mems_stats(const gpumem_mems *m, gpumem_find_stats *out);

/*
 * gpumem_mums -- maximal unique matches (NEXT-F3; PAPER.md:23 defines a MUM, :286 lists
 *  it as future work): the MEMs of `m` whose string occurs exactly once in R and once in
 *  Q (reading R21), in the same (r, q) order. `m` must be a complete MEM set of
 *  (R, Q, L) (a q-range or band subset is not enough to decide uniqueness).
 *  Synchronises once (the result size is data-dependent).
 */
gpumem_status gpumem_mums(const gpumem_mems *m, void *cuda_stream, gpumem_mems **out);

/*
 * gpumem_rare -- maximal rare matches (NEXT-F3; PAPER.md:23 "maximal rare matches", :286
 *  "unique and rare exact match extraction" as future work): the MEMs of `m` whose
 *  string occurs (overlapping occurrences counted) at most k times in R and at most k
 *  times in Q (reading R23), in the same (r, q) order; k = 1 is gpumem_mums.
 *  1 <= k <= 15, else GPUMEM_ERR_ARG. `m` must be a complete MEM set of (R, Q, L): the
 *  counts come from the containment of the MEMs' query / reference intervals. New
 *  handle on *out (NULL on error). Synchronises once (the result size is data-dependent).
 */
gpumem_status gpumem_rare(const gpumem_mems *m, uint32_t k, void *cuda_stream, gpumem_mems **out);

/* Borrowed device pointer to the sorted triples and their count. */
gpumem_status gpumem_mems_view(const gpumem_mems *m, const gpumem_triple **dev_ptr, uint64_t *count);

/* Copy the triples to host memory (synchronous); capacity < count -> GPUMEM_ERR_RANGE. */
gpumem_status gpumem_mems_to_host(const gpumem_mems *m, gpumem_triple *host_buf, uint64_t capacity);

/*
 * gpumem_merge_sorted -- K9, the rank-0 merge of the query shards (it
 *  replaces the host merge-sort of out-tile triplets, §III-C2).
 *  dev_runs[i]: device pointer to counts[i] triples (host array of n_runs <= 64
 *  pointers / host counts), each run sorted by (r, q) and no (r, q) in two runs (the
 *  query shards are disjoint by the ownership rule). The runs may be peer memory
 *  mapped with gpumem_ipc_open: the kernel then reads them over NVLink directly, the
 *  gather and the merge in one pass. *out: the union sorted by (r, q) (a tree of
 *  two-way merge-path merges: one read and one write per triple per level).
 *  Asynchronous on cuda_stream (the runs must stay valid until it completes).
 *  Errors: n_runs > 64 or a NULL run with a count -> GPUMEM_ERR_ARG; a run of 2^32 or
 *  more triples -> GPUMEM_ERR_RANGE. Runs that are unsorted or overlap give an
 *  unspecified order (not checked).
 */
gpumem_status gpumem_merge_sorted(const gpumem_triple *const *dev_runs, const uint64_t *counts,
                                  int n_runs, void *cuda_stream, gpumem_mems **out);

/*
 * Pipeline: the whole path (pack R, pack Q, index R, find, sort -- the same kernels
 * and the same result as gpumem_pack + gpumem_index_build + gpumem_find_mems) for
 * fixed sizes, captured once as a CUDA graph and replayed with one launch and no host
 * round trip in between (find's output count stays on the device; the output sort is
 * sized by it there). Intended for repeated work of one shape (benchmarks, batches of
 * equally long queries) where host launch latency would otherwise show between stages.
 *
 * gpumem_pipeline_create -- sizes |R| = r_len, |Q| = q_len, seed_len (ls), min_len (L)
 *  and the MEM start range [q_begin, q_end) as in gpumem_find_mems (0, UINT64_MAX = all).
 *  Argument rules as gpumem_index_build / gpumem_find_mems. Stream: runs are ordered
 *  after the caller's prior work on `cuda_stream` and before its later work (events);
 *  the graph itself runs on streams the pipeline owns (a captured graph cannot live on
 *  the legacy default stream), which also own its workspaces. Allocates those streams
 *  and a pinned 128-byte counter buffer; device memory (one arena holding the packed
 *  sequences, the index and the result) is allocated at the first run.
 *
 * gpumem_pipeline_run -- async. r_bases_dev / q_bases_dev: device pointers to r_len and
 *  q_len ASCII bases (read, not modified; must stay valid until the run completes).
 *  The first call, and any call with different input pointers, measures and captures
 *  the graph (one ordinary synchronous pass + capture; option settings are taken at
 *  capture time); later calls are one cudaGraphLaunch. The previous run's result is
 *  invalidated.
 *
 * gpumem_pipeline_run_host -- the same from host memory (pinned for full speed): R and Q
 *  are copied on a copy stream into pipeline-owned device buffers (allocated on the
 *  first call, through the allocator hook), R first; the graph packs and indexes R while
 *  Q is still in flight. Q crosses PCIe in q_chunks pieces (option "q_chunks", read at
 *  gpumem_pipeline_create; pieces >= max(1 Mbp, 8 L) bases; whole-Q pipelines only):
 *  piece j is packed as soon as it has arrived and searched for the MEMs starting in it
 *  (shifted back by max(L, step + ls) + 64 bases), extensions stopping at the data present;
 *  the few matches cut there are finished after the last piece. Same
 *  result as gpumem_pipeline_run. Async: the host buffers must stay valid and
 *  unmodified until the run completes (gpumem_pipeline_result).
 *
 * gpumem_pipeline_result -- synchronises the stream, then checks the alphabet flags
 *  (GPUMEM_ERR_ALPHABET as gpumem_find_mems) and the output capacity: on overflow the
 *  MEMs are recomputed with gpumem_find_mems on the pipeline's packed sequences and
 *  index (stats.attempts > 1). *dev_ptr / *count: the sorted triples, borrowed, valid
 *  until the next run or gpumem_free(pl).
 *
 * gpumem_pipeline_stats -- find statistics of the last result.
 * gpumem_pipeline_profile -- per-stage device time of the last completed run (the
 *  stage events are event-record nodes of the graph, present per option "pipe_events"),
 *  aggregated by name as gpumem_profile_read;
 *  synchronises those events. Returns the number of entries written.
 * gpumem_free(pl) synchronises the stream and releases everything.
 */
gpumem_status gpumem_pipeline_create(uint64_t r_len, uint64_t q_len, uint32_t seed_len, uint32_t min_len,
                                     uint64_t q_begin, uint64_t q_end, void *cuda_stream, gpumem_pipeline **out);
gpumem_status gpumem_pipeline_run(gpumem_pipeline *pl, const char *r_bases_dev, const char *q_bases_dev);
gpumem_status gpumem_pipeline_run_host(gpumem_pipeline *pl, const char *r_bases_host, const char *q_bases_host);
gpumem_status gpumem_pipeline_result(gpumem_pipeline *pl, const gpumem_triple **dev_ptr, uint64_t *count);
gpumem_status gpumem_pipeline_stats(const gpumem_pipeline *pl, gpumem_find_stats *out);
int gpumem_pipeline_profile(const gpumem_pipeline *pl, const char **names, double *ms, uint64_t *launches,
                            int max_stages);

/*
 * Multi-GPU export of a pipeline's result (dist.py's fused gather + merge):
 * gpumem_pipeline_set_exportable(pl, 1) -- before the first run (or it recaptures):
 *  the arena is allocated with cudaMalloc (IPC-capable; bypasses the allocator hook).
 * gpumem_pipeline_export -- after a run: a CUDA IPC handle of the arena, the byte
 *  offset of the result triples inside it, and the capture generation (a recapture,
 *  e.g. on new input pointers, moves the arena: re-export; handle may be NULL to read
 *  only offset and generation). The triples there are the
 *  graph's result; after an overflow fallback (stats.attempts > 1) they are not.
 * gpumem_ipc_open / gpumem_ipc_close -- map / unmap another process's exported arena
 *  on the current device (peer access enabled lazily); dev_base + offset are the
 *  triples. The exporting pipeline must outlive the mapping.
 */
typedef struct { unsigned char bytes[64]; } gpumem_ipc_handle;
gpumem_status gpumem_pipeline_set_exportable(gpumem_pipeline *pl, int on);
gpumem_status gpumem_pipeline_export(const gpumem_pipeline *pl, gpumem_ipc_handle *handle, uint64_t *offset,
                                     uint64_t *generation);
gpumem_status gpumem_ipc_open(const gpumem_ipc_handle *handle, void **dev_base);
gpumem_status gpumem_ipc_close(void *dev_base);

/*
 * Multi-FASTA input and MUMmer-style output (NEXT-F4; PAPER.md:64 §II-A MUMmer, :226
 * §IV-B: I/O is outside the paper's timings). Host-side parsing and formatting; the
 * record-boundary split runs on the GPU.
 *
 * gpumem_fasta_parse -- text[0, n): one or more records ">name[ description]\n" + sequence
 *  lines (whitespace ignored; a leading run of blank lines allowed). The records are
 *  concatenated with ONE masked separator base between consecutive records, and every
 *  letter outside {A,C,G,T,a,c,g,t} (N, IUPAC codes) becomes a masked 'A' (DESIGN.md
 *  reading R24: a masked position matches nothing). Errors: no '>' where a header must
 *  start -> GPUMEM_ERR_ARG; a non-printable byte -> GPUMEM_ERR_ALPHABET; more than
 *  2^32-1 bases in total -> GPUMEM_ERR_RANGE. *out: new handle (gpumem_free), NULL on error.
 * gpumem_fasta_info -- the record count, the concatenated sequence (host, borrowed; pass
 *  it to gpumem_pack / a pipeline), its length, the number of masked intervals.
 * gpumem_fasta_record -- record i's name (borrowed) and its [start, start + len) in the
 *  concatenated sequence.
 * gpumem_split_masked -- the MEMs of the multi-record problem from the MEMs `m` of the
 *  concatenated sequences (same L): every MEM cut at the masked positions of R and of Q,
 *  the pieces of length >= min_len kept, sorted by (r, q) in concatenated coordinates.
 *  q_reverse = 1 when m was computed against gpumem_revcomp(Q) (Q's masks mirrored).
 *  Synchronises once. New handle on *out.
 * gpumem_write_mummer -- writes host triples (concatenated coordinates, from
 *  gpumem_split_masked: no match may cross a record, else GPUMEM_ERR_ARG) as MUMmer text to
 *  `path`: per query record in input order "> qname" then "  rname\trpos\tqpos\tlen"
 *  lines (1-based positions inside the records), ordered by query position, reference
 *  record, reference position; if rev != NULL also "> qname Reverse" and the reverse-strand
 *  matches (query positions relative to the reverse complement of the query record).
 */
typedef struct gpumem_fasta gpumem_fasta;
gpumem_status gpumem_fasta_parse(const char *text, uint64_t n, gpumem_fasta **out);
gpumem_status gpumem_fasta_info(const gpumem_fasta *f, uint64_t *n_records, const char **seq, uint64_t *seq_len,
                                uint64_t *n_masked);
gpumem_status gpumem_fasta_record(const gpumem_fasta *f, uint64_t i, const char **name, uint64_t *start,
                                  uint64_t *len);
gpumem_status gpumem_split_masked(const gpumem_mems *m, const gpumem_fasta *R, const gpumem_fasta *Q, uint32_t min_len,
                                  int q_reverse, void *cuda_stream, gpumem_mems **out);
gpumem_status gpumem_write_mummer(const gpumem_triple *fwd, uint64_t n_fwd, const gpumem_triple *rev, uint64_t n_rev,
                                  const gpumem_fasta *R, const gpumem_fasta *Q, const char *path);

/* Release any handle above (seq, index, mems, pipeline, fasta). NULL is a no-op. */
void gpumem_free(void *handle);

/* Temporaries (find buffers, sort and index scratch) live in a grow-only workspace per
 * (device, stream) so repeated calls do not allocate. gpumem_trim synchronises those
 * streams and releases every workspace. Handles are unaffected. */
gpumem_status gpumem_trim(void);

/* Thread-local text of the last failure ("" if none). */
const char *gpumem_last_error(void);

/* Allocator hook (e.g. the torch caching allocator). Both NULL restores the default. */
gpumem_status gpumem_set_allocator(void *(*alloc_fn)(size_t bytes, void *cuda_stream, void *ctx),
                                   void (*free_fn)(void *ptr, void *cuda_stream, void *ctx), void *ctx);

/* ---- instrumentation and tuning (not part of the method) ---------------------------- */

/* Tuning knobs; the MEM set never depends on them. Names:
 *  "find_grid"        CTAs of the find kernel (0 = SMs x occupancy)
 *  "find_spill"       bucket size above which hits are spilled to the heavy queue
 *  "out_capacity"     initial output capacity in triples (0 = automatic; small values
 *                     force the overflow-and-retry path in tests)
 *  "use_bitmap"       1 (default) probe the rank words + bucket table, 0 probe ptrs only
 *  "static_lb"        1: no hit redistribution across lanes (load-balancing ablation)
 *  "sort_impl"        output sort: 0 (default) auto by size, 1 stable LSD radix sort,
 *                     2 MSD bucket sort; in a pipeline 0 picks MSD or LSD by the MEM
 *                     count of its measuring run
 *  "rec8"             seed records: -1 (default) auto (8-byte when step <= 8), 0 16-byte, 1 8-byte
 *  "rank_sectors"     lookup directory: -1 (default) auto, 0 rank words, 1 rank sectors
 *  "index_tiled"      1: a sparse index (n_locs < 4^ls / 4, seed_len <= 13) is Alg. 1
 *                     tiled over the seed space (the sampled locations put into bins of
 *                     1024 consecutive seeds by a radix sort of the top code bits, then
 *                     Alg. 1 steps 1-4, the directory and the table per bin on chip);
 *                     0: the stable LSD radix sort of all code bits; -1 (default): tiled
 *                     for sparse indexes up to 2^20 sampled locations
 *  "index_alg1"       1: PAPER.md Alg. 1 as written over the whole 4^ls table (atomic
 *                     counts, prefix sums, placement, per-bucket sort); -1: only for
 *                     dense indexes (n_locs >= 4^ls / 4); 0 (default): never (measured
 *                     slower: random atomics/stores into the 4^ls table)
 *  "pipe_events"      stage event nodes captured into a pipeline graph (read at capture):
 *                     0 (default) none, 2 around the find kernel only, 1 at every stage
 *                     boundary (gpumem_pipeline_profile; each node costs a few us per run)
 *  "pdl"              1 (default): programmatic dependent launch between consecutive
 *                     kernels (each waits for its predecessor with griddepcontrol.wait);
 *                     0: ordinary launches
 *  "q_chunks"         host-input pipelines: pieces Q is copied, packed and searched in
 *                     (default 8; 1 = search after the whole Q has arrived); read at create
 *  "radix_bits"       LSD digit width: 0 (default) = 9 bits when that saves a pass, else 8;
 *                     or pinned to 8, 9, 10; anything else is GPUMEM_ERR_ARG
 *  "l2_persist"       MB of L2 set aside for persisting lines (device-wide
 *                     cudaLimitPersistingL2CacheSize, clamped to the device maximum);
 *                     0 (default) none. Not a stream operation: set outside capture
 *  "l2_window"        access-policy window of k_find / k_heavy (with l2_persist > 0):
 *                     0 (default) none, 1 the lookup directory, 2 the compact table,
 *                     3 the seed records; hit ratio = set-aside / window bytes.
 *                     Measured no gain (profiles/r2_l2_persist.json), kept as the probe
 *                     of SURVEY.md §7's persisting-window suggestion
 * Unknown names are GPUMEM_ERR_ARG. */
gpumem_status gpumem_set_option(const char *name, int64_t value);

/* Per-stage device time: when enabled, CUDA events bracket each stage on its stream.
 * gpumem_profile_read synchronises those events, writes up to max_stages
 * (name, total ms, launches) entries and resets the accumulators. */
gpumem_status gpumem_profile_enable(int on);
int gpumem_profile_read(const char **names, double *ms, uint64_t *launches, int max_stages);

/* The ceiling of k_find's access pattern on this GPU (not part of the method):
 * *ms = best time of n_probes random 8-byte loads into a device table of table_bytes
 * (rounded down to a power of two; L2-resident when small), 8 independent loads per
 * thread as the find kernel issues its probes. Synchronous; allocates and frees its
 * own table. bench.py sets k_find's sector rate against it. */
gpumem_status gpumem_gather_ceiling(uint64_t n_probes, uint64_t table_bytes, void *cuda_stream, double *ms);

/* Kernels this library has launched in this process (monotone counter). */
uint64_t gpumem_launch_count(void);

/* Library version string. */
const char *gpumem_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GPUMEM_H */
