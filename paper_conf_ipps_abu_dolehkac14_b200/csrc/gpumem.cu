// gpumem.cu -- the C ABI of libgpumem.so (include/gpumem.h): handles, allocation,
// streams, status codes, the overflow-and-retry protocol of find, and stage
// instrumentation. All compute is in pack.cu / index.cu / radix.cu / find.cu /
// sort.cu; this file only orchestrates launches.
#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

#define GPUMEM_VERSION "0.2.0"

// output sort: the MSD bucket sort up to this many MEMs, the LSD radix sort beyond
// (measured in the pipeline: MSD 0.115 vs LSD 0.173 ms at 0.81 M keys (C4), 0.50 vs 0.31 ms
// at 2.98 M (C5 L = 50): its shared-memory segment sorts grow with the key count)
constexpr uint64_t kMsdMaxN = 2u << 20;

enum : uint32_t { kMagicSeq = 0x47534551u, kMagicIdx = 0x47494458u, kMagicMems = 0x474d454du,
                  kMagicPipe = 0x47504950u };

struct gpumem_seq {
    uint32_t magic;
    int device;
    cudaStream_t stream;
    uint64_t n;
    uint64_t n_words;
    uint64_t *words;
    unsigned long long *bad;  // first invalid position (ULLONG_MAX if none)
};

struct gpumem_index {
    uint32_t magic;
    int device;
    cudaStream_t stream;
    const gpumem_seq *R;
    uint32_t ls, L, step;
    uint64_t n_locs;
    uint32_t *ptrs;
    uint32_t *locs;
    unsigned long long *rankw;   // rank words + rotated occupancy, 16 B per 32 seeds (index.cu), or
    uint4 *rsect;                // rank sectors, 16 B per 32 seeds (index.cu); one of the two is null
    uint2 *buckets;
    void *recs;                  // uint4 records, or uint2 when rec8
    int rec8;
    uint4 *hv_info = nullptr;    // heavy buckets (index.cu k_hv_part), or null
    unsigned int *hv_cnt = nullptr;  // [0] listed, [1] usable (sorted) entries of hv_info
    uint2 *hv_list = nullptr;
};

struct gpumem_mems {
    uint32_t magic;
    int device;
    cudaStream_t stream;
    uint64_t count;
    gpumem_triple *dev;
    gpumem_find_stats stats;
};

namespace gm {

Options g_opt;
thread_local cudaAccessPolicyWindow g_l2win = {};

namespace {
thread_local std::string t_err;
std::atomic<uint64_t> g_launches{0};
void *(*g_alloc_fn)(size_t, void *, void *) = nullptr;
void (*g_free_fn)(void *, void *, void *) = nullptr;
void *g_alloc_ctx = nullptr;
std::mutex g_pool_mu;
uint64_t g_pool_done = 0;  // bitmask of devices whose default pool was configured

struct StageRec {
    const char *name;
    cudaEvent_t a, b;
    uint64_t l0, l1;
};
std::mutex g_prof_mu;
bool g_prof = false;
std::vector<StageRec> g_recs;
std::vector<cudaEvent_t> g_ev_free;

// Pipeline capture context (gpumem_pipeline_*). mode 1 = measuring run: real
// allocations, their bytes summed; mode 2 = capture: handle/scratch allocations are
// bump-allocated from the pipeline's arena (frees of arena memory are no-ops), so the
// captured graph holds no allocation nodes and can be relaunched. `deferred` makes
// find_mems skip its host synchronisation: the output sort reads the MEM count from
// device memory and the counters are copied to pinned host memory at the end.
struct CapCtx {
    int mode = 0;
    cudaError_t err = cudaSuccess;
    char *arena = nullptr;
    size_t off = 0, cap = 0, need = 0;
    bool deferred = false;
    std::vector<StageRec> *recs = nullptr;
    unsigned long long *host = nullptr;   // pinned: [0, 8) find counters, [8] R flag, [9] Q flag
    uint64_t out_cap = 0, coop_cap = 0, spill_cap = 0, span = 0;
    uint64_t expect_n = 0;                // capture: the measuring run's MEM count (sort choice)
    cudaStream_t side = nullptr;          // pipeline: the seed records are built here, next to the
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;  // directory fill on the main stream (fork / join)
    gpumem_mems *mems = nullptr;
    // The pipeline's own workspaces (never the per-stream global ones, which ordinary
    // calls and gpumem_trim may grow or free while the graph still points into them):
    // the measuring run allocates and sizes them (ws_need), the capture bump-allocates
    // each from the arena at that size, so they live and die with the arena.
    void *ws_priv = nullptr;              // WsSet *
    // streamed query (host-input pipeline): Q in q_chunks pieces at q_bnd[0..q_chunks]
    // (multiples of 32); piece j is packed once its copy has arrived and q_packed[j] is
    // recorded; find over the MEM starts of piece i runs once pieces <= i + 1 are packed
    int q_chunks = 1;
    const uint64_t *q_bnd = nullptr;
    const cudaEvent_t *q_packed = nullptr;
};
thread_local CapCtx *t_cap = nullptr;
thread_local bool t_ws_alloc = false;     // workspace growth: never from the arena

cudaEvent_t take_event() {
    if (!g_ev_free.empty()) {
        cudaEvent_t e = g_ev_free.back();
        g_ev_free.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

int current_device() {
    int d = -1;
    if (cudaGetDevice(&d) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    return d;
}
}  // namespace

gpumem_status fail(gpumem_status st, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    t_err = buf;
    return st;
}

gpumem_status cuda_fail(cudaError_t e, const char *what) {
    cudaGetLastError();  // clear sticky non-fatal state
    return fail(GPUMEM_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
}

void note_launch(int n) { g_launches.fetch_add(uint64_t(n), std::memory_order_relaxed); }

int num_sms() {
    static int cached[64] = {0};
    const int d = current_device();
    if (d < 0) return 148;
    if (d < 64 && cached[d]) return cached[d];
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    if (v <= 0) v = 148;
    if (d < 64) cached[d] = v;
    return v;
}

void *dalloc(size_t bytes, cudaStream_t s) {
    if (bytes == 0) bytes = 256;
    bytes = (bytes + 255) & ~size_t(255);
    if (t_cap && !t_ws_alloc) {
        if (t_cap->mode == 2) {
            if (t_cap->off + bytes > t_cap->cap) {
                fail(GPUMEM_ERR_NOMEM, "pipeline arena exhausted (%zu + %zu > %zu bytes)", t_cap->off, bytes,
                     t_cap->cap);
                return nullptr;
            }
            void *p = t_cap->arena + t_cap->off;
            t_cap->off += bytes;
            return p;
        }
        t_cap->need += bytes;
    }
    if (g_alloc_fn) {
        void *p = g_alloc_fn(bytes, s, g_alloc_ctx);
        if (!p) fail(GPUMEM_ERR_NOMEM, "allocator hook returned NULL for %zu bytes", bytes);
        return p;
    }
    const int d = current_device();
    if (d >= 0 && d < 64) {
        std::lock_guard<std::mutex> g(g_pool_mu);
        if (!(g_pool_done >> d & 1)) {  // keep freed memory cached in the pool
            cudaMemPool_t pool;
            if (cudaDeviceGetDefaultMemPool(&pool, d) == cudaSuccess) {
                uint64_t thr = UINT64_MAX;
                cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
            }
            cudaGetLastError();
            g_pool_done |= 1ull << d;
        }
    }
    void *p = nullptr;
    const cudaError_t e = cudaMallocAsync(&p, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(GPUMEM_ERR_NOMEM, "cudaMallocAsync(%zu bytes): %s", bytes, cudaGetErrorString(e));
        return nullptr;
    }
    return p;
}

void dfree(void *p, cudaStream_t s) {
    if (!p) return;
    if (t_cap && t_cap->mode == 2 && static_cast<char *>(p) >= t_cap->arena &&
        static_cast<char *>(p) < t_cap->arena + t_cap->cap)
        return;  // arena memory lives as long as the pipeline
    if (g_free_fn) {
        g_free_fn(p, s, g_alloc_ctx);
        return;
    }
    cudaFreeAsync(p, s);
}

Stage::Stage(const char *name, cudaStream_t st) : slot(-1), s(st), vec(nullptr) {
    std::vector<StageRec> *v = (t_cap && t_cap->recs) ? t_cap->recs : (g_prof ? &g_recs : nullptr);
    if (!v) return;
    if (t_cap && t_cap->recs && g_opt.pipe_events == 0) return;                       // no stage events
    if (t_cap && t_cap->recs && g_opt.pipe_events == 2 && strcmp(name, "find")) return;  // find's only
    std::lock_guard<std::mutex> g(g_prof_mu);
    StageRec r{name, take_event(), take_event(), g_launches.load(), 0};
    // in a capture: an event record node of the graph (timed on every launch)
    if (t_cap && t_cap->recs) cudaEventRecordWithFlags(r.a, s, cudaEventRecordExternal);
    else cudaEventRecord(r.a, s);
    v->push_back(r);
    slot = int(v->size()) - 1;
    vec = v;
}

Stage::~Stage() {
    if (slot < 0) return;
    std::lock_guard<std::mutex> g(g_prof_mu);
    auto &v = *static_cast<std::vector<StageRec> *>(vec);
    if (slot < int(v.size())) {
        if (t_cap && t_cap->recs) cudaEventRecordWithFlags(v[slot].b, s, cudaEventRecordExternal);
        else cudaEventRecord(v[slot].b, s);
        v[slot].l1 = g_launches.load();
    }
}

}  // namespace gm

using namespace gm;

namespace {

// RAII bundle of device allocations freed (async) on scope exit unless released.
struct Scratch {
    cudaStream_t s;
    std::vector<void *> ptrs;
    explicit Scratch(cudaStream_t st) : s(st) {}
    void *get(size_t bytes) {
        void *p = dalloc(bytes, s);
        if (p) ptrs.push_back(p);
        return p;
    }
    void keep(void *p) {
        for (auto &q : ptrs)
            if (q == p) q = nullptr;
    }
    ~Scratch() {
        for (void *p : ptrs) dfree(p, s);
    }
};

gpumem_status check_device(int *dev) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
        cudaGetLastError();
        return fail(GPUMEM_ERR_UNSUPPORTED, "no CUDA device visible");
    }
    int d = 0;
    cudaGetDevice(&d);
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, d);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, d);
    if (major != 10 || minor != 0)
        return fail(GPUMEM_ERR_UNSUPPORTED, "libgpumem.so is built for sm_100a (B200); device %d is sm_%d%d", d,
                    major, minor);
    *dev = d;
    return GPUMEM_OK;
}

#define CK(call, what)                                \
    do {                                              \
        const cudaError_t _e = (call);                \
        if (_e != cudaSuccess) return cuda_fail(_e, what); \
    } while (0)

// Per-(device, stream) grow-only workspace for temporaries: successive calls on one
// stream are ordered, so a slot can be reused without synchronisation, and the hot
// loop does no allocation at all once warm. gpumem_trim() releases everything.
enum WsSlot {
    kWsCtr, kWsSpill, kWsKeys, kWsLens, kWsSortK, kWsSortL, kWsSortScratch, kWsCodes0, kWsCodes1,
    kWsRadix, kWsFill, kWsMergeK, kWsFasta, kWsPackTmp, kWsCoop, kWsMums, kWsAlg1, kWsTiled,
    kWsCount
};
struct Workspace {
    void *p[kWsCount] = {};
    size_t sz[kWsCount] = {};
};
std::mutex g_ws_mu;
std::vector<std::pair<std::pair<int, cudaStream_t>, Workspace *>> g_ws;

// A pipeline's private workspaces, per stream of its path.
struct WsSet {
    std::vector<std::pair<cudaStream_t, Workspace>> w;
    Workspace &of(cudaStream_t s) {
        for (auto &e : w)
            if (e.first == s) return e.second;
        w.push_back({s, Workspace{}});
        return w.back().second;
    }
    size_t bytes() const {  // arena bytes the capture will bump-allocate for them
        size_t t = 0;
        for (auto &e : w)
            for (int k = 0; k < kWsCount; ++k) t += (e.second.sz[k] + 255) & ~size_t(255);
        return t;
    }
    void release() {  // measuring run only (capture workspaces are arena memory)
        for (auto &e : w)
            for (int k = 0; k < kWsCount; ++k)
                if (e.second.p[k]) dfree(e.second.p[k], e.first);
        w.clear();
    }
};

void *ws_get_priv(WsSet &set, int slot, size_t bytes, cudaStream_t s) {
    Workspace &w = set.of(s);
    if (w.sz[slot] >= bytes && w.p[slot]) return w.p[slot];
    if (t_cap->mode == 2) {  // one arena slice per workspace, at the measured size
        if (w.p[slot] || bytes > w.sz[slot]) {
            fail(GPUMEM_ERR_NOMEM, "workspace %d would grow during a pipeline capture", slot);
            return nullptr;
        }
        w.p[slot] = dalloc(w.sz[slot], s);  // bump allocation from the arena
        return w.p[slot];
    }
    t_ws_alloc = true;  // measuring run: real allocations, not counted as handle bytes
    if (w.p[slot]) dfree(w.p[slot], s);
    w.p[slot] = dalloc(bytes, s);
    w.sz[slot] = w.p[slot] ? bytes : 0;
    t_ws_alloc = false;
    return w.p[slot];
}

void *ws_get(int slot, size_t bytes, cudaStream_t s) {
    if (t_cap && t_cap->ws_priv) return ws_get_priv(*static_cast<WsSet *>(t_cap->ws_priv), slot, bytes, s);
    int d = 0;
    cudaGetDevice(&d);
    std::lock_guard<std::mutex> g(g_ws_mu);
    Workspace *w = nullptr;
    for (auto &e : g_ws)
        if (e.first.first == d && e.first.second == s) w = e.second;
    if (!w) {
        w = new Workspace();
        g_ws.push_back({{d, s}, w});
    }
    if (w->sz[slot] < bytes) {
        t_ws_alloc = true;
        if (w->p[slot]) dfree(w->p[slot], s);
        const size_t want = bytes + bytes / 8 + 4096;
        w->p[slot] = dalloc(want, s);
        w->sz[slot] = w->p[slot] ? want : 0;
        t_ws_alloc = false;
    }
    return w->p[slot];
}

// Free one stream's workspace (the stream is about to be destroyed).
void ws_release_stream(int d, cudaStream_t s) {
    std::lock_guard<std::mutex> g(g_ws_mu);
    for (size_t i = 0; i < g_ws.size(); ++i) {
        if (g_ws[i].first.first != d || g_ws[i].first.second != s) continue;
        cudaStreamSynchronize(s);
        for (int k = 0; k < kWsCount; ++k)
            if (g_ws[i].second->p[k]) dfree(g_ws[i].second->p[k], s);
        cudaStreamSynchronize(s);
        delete g_ws[i].second;
        g_ws.erase(g_ws.begin() + long(i));
        return;
    }
}

unsigned long long *pinned_slots() {  // 16 per thread, never freed
    thread_local unsigned long long *p = nullptr;
    if (!p) {
        if (cudaMallocHost(&p, 16 * sizeof(unsigned long long)) != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
        }
    }
    return p;
}

}  // namespace

// ---------------------------------------------------------------- pipeline (CUDA graph)
constexpr int kMaxQChunks = 16;
struct gpumem_pipeline {
    uint32_t magic;
    int device;
    cudaStream_t user;                     // the caller's stream (runs are ordered on it by events)
    cudaStream_t stream;                   // the pipeline's own stream: capture, launches, fallback
    cudaStream_t side;                     // runs pack Q next to the index build
    cudaStream_t side2;                    // runs the seed records next to the directory fill
    cudaEvent_t ev_in, ev_out, ev_join;
    uint64_t nR, nQ, q_begin, q_end;
    uint32_t ls, L;
    const char *inR, *inQ;                 // the device inputs the graph was captured with
    char *arena;                           // every allocation of the captured path (allocator hook)
    size_t arena_bytes;
    WsSet *ws;                             // the graph's workspaces, slices of the arena
    cudaGraph_t graph;                     // the captured path (one launch per run)
    cudaGraphExec_t exec;
    cudaEvent_t ev_fork;                   // side-stream fork inside the graph
    cudaEvent_t ev_ra, ev_rb;              // fork / join of the seed-record build (index)
    char *stage;                           // host-input runs: device copies of R and Q (nR + nQ bytes)
    cudaStream_t copy;                     // ... copied on this stream
    cudaEvent_t ev_r, ev_q;                // R / Q copied
    gpumem_seq *R, *Q;
    gpumem_index *idx;
    gpumem_mems *mems;                     // the graph's result buffer (count set by _result)
    gpumem_mems *fallback;                 // overflow rerun through gpumem_find_mems
    unsigned long long *host;              // pinned counters written by the graph
    uint64_t out_cap, coop_cap, spill_cap, span;
    std::vector<StageRec> recs;
    uint64_t launches;                     // kernels per graph launch
    int q_chunks;                          // host-input runs: Q copied, packed, searched in this many pieces
    uint64_t q_bnd[kMaxQChunks + 1];       // ... at these boundaries (multiples of 32)
    int cap_chunks;                        // pieces of the captured graph (1 = whole Q at once)
    cudaEvent_t ev_qc[kMaxQChunks];        // piece j copied (recorded on `copy`, waited on by the graph)
    cudaEvent_t ev_pk[kMaxQChunks];        // piece j packed (inside the graph)
    int exportable;                        // arena from cudaMalloc, so its IPC handle can be exported
    uint64_t generation;                   // captures so far (an exported handle is valid for one)
    int ran;
    gpumem_find_stats stats;
};

namespace {

// The whole path on the pipeline's stream: pack R, pack Q, index R, find (deferred).
// Where the path waits for the host copy of R (1) or Q (2): an external event wait
// node in the captured graph (device-input runs record both events just before the
// launch, so the waits are free). Nothing to do outside a capture.
void pipeline_wait_mark(gpumem_pipeline *pl, cudaStream_t s, int which) {
    if (t_cap && t_cap->recs) cudaStreamWaitEvent(s, which == 1 ? pl->ev_r : pl->ev_q, cudaEventWaitExternal);
}

// Q in pieces (host-input pipeline, cap_chunks > 1): piece j is packed on stream s once
// its copy has arrived (external event wait in the graph), into one packed sequence;
// ev_pk[j] marks it packed for the find launches of gpumem_find_mems.
gpumem_status pack_q_pieces(gpumem_pipeline *pl, const char *Q, cudaStream_t s, gpumem_seq **out) {
    *out = nullptr;
    const uint64_t n = pl->nQ, n_words = (n + 31) / 32 + 4;
    Scratch sc(s);
    auto *words = static_cast<uint64_t *>(sc.get(n_words * 8));
    auto *bad = static_cast<unsigned long long *>(sc.get(8));
    if (!words || !bad) return GPUMEM_ERR_NOMEM;
    CK(fill_async(bad, 0xffffffffu, 8, s), "flag init");
    const int K = pl->cap_chunks;
    for (int j = 0; j < K; ++j) {
        const uint64_t a = pl->q_bnd[j], b = pl->q_bnd[j + 1];
        if (t_cap && t_cap->recs) CK(cudaStreamWaitEvent(s, pl->ev_qc[j], cudaEventWaitExternal), "wait piece");
        const uint64_t nw = j + 1 < K ? (b - a) / 32 : n_words - a / 32;
        Stage stage("pack", s);
        CK(launch_pack(reinterpret_cast<const uint8_t *>(Q) + a, b - a, words + a / 32, nw, bad, s, a), "pack piece");
        CK(cudaEventRecord(pl->ev_pk[j], s), "piece packed");
    }
    sc.keep(words);
    sc.keep(bad);
    *out = new gpumem_seq{kMagicSeq, pl->device, s, n, n_words, words, bad};
    return GPUMEM_OK;
}

gpumem_status pipeline_path(gpumem_pipeline *pl, const char *R, const char *Q, gpumem_seq **hR, gpumem_seq **hQ,
                            gpumem_index **hI, gpumem_mems **hM) {
    *hR = *hQ = nullptr;
    *hI = nullptr;
    *hM = nullptr;
    // R's part first: with host inputs the index is built while Q is still crossing PCIe
    // pack Q runs on the side stream, concurrently with the (latency-bound) index build
    gpumem_status st = GPUMEM_OK;
    if (cudaEventRecord(pl->ev_fork, pl->stream) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "fork");
    if (!st && cudaStreamWaitEvent(pl->side, pl->ev_fork, 0) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "fork");
    if (pl->cap_chunks > 1) {  // streamed query: pieces packed as they arrive; find joins per piece
        if (!st) st = pack_q_pieces(pl, Q, pl->side, hQ);
        if (!st) pipeline_wait_mark(pl, pl->stream, 1);
        if (!st) st = gpumem_pack(R, pl->nR, 1, pl->stream, hR);
        if (!st) st = gpumem_index_build(*hR, pl->ls, pl->L, pl->stream, hI);
        if (!st) st = gpumem_find_mems(*hI, *hQ, pl->q_begin, pl->q_end, pl->stream, hM);
        return st;
    }
    if (!st) pipeline_wait_mark(pl, pl->side, 2);
    if (!st) st = gpumem_pack(Q, pl->nQ, 1, pl->side, hQ);
    if (!st && cudaEventRecord(pl->ev_join, pl->side) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "join");
    if (!st) pipeline_wait_mark(pl, pl->stream, 1);
    if (!st) st = gpumem_pack(R, pl->nR, 1, pl->stream, hR);
    if (!st) st = gpumem_index_build(*hR, pl->ls, pl->L, pl->stream, hI);
    if (!st && cudaStreamWaitEvent(pl->stream, pl->ev_join, 0) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "join");
    if (!st) st = gpumem_find_mems(*hI, *hQ, pl->q_begin, pl->q_end, pl->stream, hM);
    return st;
}

void pipeline_release(gpumem_pipeline *pl) {  // graph, arena and the arena-backed handles
    if (pl->exec) cudaGraphExecDestroy(pl->exec);
    if (pl->graph) cudaGraphDestroy(pl->graph);
    pl->exec = nullptr;
    pl->graph = nullptr;
    if (pl->R) { pl->R->magic = 0; delete pl->R; }
    if (pl->Q) { pl->Q->magic = 0; delete pl->Q; }
    if (pl->idx) { pl->idx->magic = 0; delete pl->idx; }
    if (pl->mems) { pl->mems->magic = 0; delete pl->mems; }
    pl->R = pl->Q = nullptr;
    pl->idx = nullptr;
    pl->mems = nullptr;
    if (pl->arena) {
        if (pl->exportable) cudaFree(pl->arena);
        else dfree(pl->arena, pl->stream);
    }
    pl->arena = nullptr;
    pl->arena_bytes = 0;
    delete pl->ws;  // its buffers were arena slices
    pl->ws = nullptr;
    {
        std::lock_guard<std::mutex> g(g_prof_mu);
        for (auto &r : pl->recs) {
            g_ev_free.push_back(r.a);
            g_ev_free.push_back(r.b);
        }
    }
    pl->recs.clear();
    pl->inR = pl->inQ = nullptr;
    cudaGetLastError();
}

gpumem_status pipeline_capture(gpumem_pipeline *pl, const char *R, const char *Q, bool host_inputs) {
    cudaStream_t s = pl->stream;
    CK(cudaStreamSynchronize(s), "sync");
    pipeline_release(pl);
    pl->cap_chunks = host_inputs ? pl->q_chunks : 1;
    // 1) measuring run: sizes every workspace, sums the handle/scratch bytes
    WsSet mws;
    CapCtx m;
    m.mode = 1;
    m.ws_priv = &mws;
    m.deferred = true;
    m.q_chunks = pl->cap_chunks;
    m.q_bnd = pl->q_bnd;
    m.q_packed = pl->ev_pk;
    m.host = pl->host;
    m.side = pl->side2;
    m.ev_a = pl->ev_ra;
    m.ev_b = pl->ev_rb;
    gpumem_seq *hR, *hQ;
    gpumem_index *hI;
    gpumem_mems *hM;
    t_cap = &m;
    gpumem_status st = pipeline_path(pl, R, Q, &hR, &hQ, &hI, &hM);
    t_cap = nullptr;
    const cudaError_t se = cudaStreamSynchronize(s);
    for (void *h : {(void *)hM, (void *)hI, (void *)hQ, (void *)hR}) gpumem_free(h);
    pl->ws = new WsSet();  // the capture's workspaces: the measured sizes, no memory yet
    for (auto &e : mws.w) {
        Workspace &w = pl->ws->of(e.first);
        for (int k = 0; k < kWsCount; ++k) w.sz[k] = e.second.sz[k];
    }
    mws.release();
    if (st) return st;
    CK(se, "measuring run");
    CK(cudaStreamSynchronize(s), "sync");
    // 2) capture into the arena (one allocation, through the allocator hook if set)
    pl->arena_bytes = m.need + pl->ws->bytes() + (1u << 20);
    if (pl->exportable) {  // IPC-capable memory (stream-ordered pool memory cannot be exported)
        if (cudaMalloc(&pl->arena, pl->arena_bytes) != cudaSuccess) {
            cudaGetLastError();
            fail(GPUMEM_ERR_NOMEM, "cudaMalloc");
            pl->arena = nullptr;
        }
    } else {
        pl->arena = static_cast<char *>(dalloc(pl->arena_bytes, s));
    }
    if (!pl->arena) {
        const std::string why = t_err;
        const size_t want = pl->arena_bytes;
        pipeline_release(pl);
        return fail(GPUMEM_ERR_NOMEM, "pipeline arena of %zu bytes: %s", want, why.c_str());
    }
    CapCtx c;
    c.mode = 2;
    c.ws_priv = pl->ws;
    c.q_chunks = pl->cap_chunks;
    c.q_bnd = pl->q_bnd;
    c.q_packed = pl->ev_pk;
    c.arena = pl->arena;
    c.cap = pl->arena_bytes;
    c.deferred = true;
    c.host = pl->host;
    c.side = pl->side2;
    c.ev_a = pl->ev_ra;
    c.ev_b = pl->ev_rb;
    c.recs = &pl->recs;
    c.expect_n = pl->host[0];
    CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed), "begin capture");
    const uint64_t l0 = g_launches.load();
    t_cap = &c;
    st = pipeline_path(pl, R, Q, &pl->R, &pl->Q, &pl->idx, &pl->mems);
    t_cap = nullptr;
    pl->launches = g_launches.load() - l0;
    g_launches.fetch_sub(pl->launches);      // captured, not launched
    const cudaError_t ce = cudaStreamEndCapture(s, &pl->graph);
    if (st) {
        pipeline_release(pl);
        return st;
    }
    if (ce != cudaSuccess) {
        pipeline_release(pl);
        return cuda_fail(ce, "pipeline capture");
    }
    const cudaError_t ie = cudaGraphInstantiate(&pl->exec, pl->graph, 0);
    if (ie != cudaSuccess) {
        pipeline_release(pl);
        return cuda_fail(ie, "graph instantiate");
    }
    pl->out_cap = c.out_cap;
    pl->coop_cap = c.coop_cap;
    pl->spill_cap = c.spill_cap;
    pl->span = c.span;
    pl->inR = R;
    pl->inQ = Q;
    ++pl->generation;
    return GPUMEM_OK;
}

// One run = one graph launch. Device-input runs record the copy events first so the
// graph's external waits on them are satisfied at once.
cudaError_t pipeline_launch(gpumem_pipeline *pl, bool host_inputs) {
    cudaError_t e = cudaSuccess;
    if (!host_inputs) {
        e = cudaEventRecord(pl->ev_r, pl->stream);
        if (e == cudaSuccess) e = cudaEventRecord(pl->ev_q, pl->stream);
        for (int j = 0; j < pl->cap_chunks && e == cudaSuccess; ++j) e = cudaEventRecord(pl->ev_qc[j], pl->stream);
        if (e != cudaSuccess) return e;
    }
    return cudaGraphLaunch(pl->exec, pl->stream);
}

}  // namespace

extern "C" {

const char *gpumem_version(void) { return GPUMEM_VERSION; }

const char *gpumem_last_error(void) { return t_err.c_str(); }

gpumem_status gpumem_trim(void) {
    std::lock_guard<std::mutex> g(g_ws_mu);
    int prev = -1;
    cudaGetDevice(&prev);
    for (auto &e : g_ws) {
        cudaSetDevice(e.first.first);
        cudaStreamSynchronize(e.first.second);
        for (int i = 0; i < kWsCount; ++i)
            if (e.second->p[i]) dfree(e.second->p[i], e.first.second);
        cudaStreamSynchronize(e.first.second);
        delete e.second;
    }
    g_ws.clear();
    if (prev >= 0) cudaSetDevice(prev);
    const cudaError_t err = cudaGetLastError();
    return err == cudaSuccess ? GPUMEM_OK : cuda_fail(err, "trim");
}

uint64_t gpumem_launch_count(void) { return g_launches.load(); }

gpumem_status gpumem_gather_ceiling(uint64_t n_probes, uint64_t table_bytes, void *cuda_stream, double *ms) {
    if (!ms || n_probes == 0 || table_bytes < 16) return fail(GPUMEM_ERR_ARG, "need ms, n_probes > 0, table >= 16 B");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    float best = 0.f;
    CK(gather_ceiling(n_probes, table_bytes, static_cast<cudaStream_t>(cuda_stream), &best), "gather ceiling");
    *ms = best;
    return GPUMEM_OK;
}

gpumem_status gpumem_set_allocator(void *(*alloc_fn)(size_t, void *, void *), void (*free_fn)(void *, void *, void *),
                                   void *ctx) {
    if ((alloc_fn == nullptr) != (free_fn == nullptr)) return fail(GPUMEM_ERR_ARG, "set both hooks or neither");
    g_alloc_fn = alloc_fn;
    g_free_fn = free_fn;
    g_alloc_ctx = ctx;
    return GPUMEM_OK;
}

gpumem_status gpumem_set_option(const char *name, int64_t value) {
    if (!name) return fail(GPUMEM_ERR_ARG, "NULL option name");
    if (!strcmp(name, "find_grid")) g_opt.find_grid = value < 0 ? 0 : value;
    else if (!strcmp(name, "find_spill")) g_opt.find_spill = value < 1 ? 1 : value;
    else if (!strcmp(name, "out_capacity")) g_opt.out_capacity = value < 0 ? 0 : value;
    else if (!strcmp(name, "use_bitmap")) g_opt.use_bitmap = value ? 1 : 0;
    else if (!strcmp(name, "static_lb")) g_opt.static_lb = value ? 1 : 0;
    else if (!strcmp(name, "sort_impl")) {
        if (value < 0 || value > 2) return fail(GPUMEM_ERR_ARG, "sort_impl must be 0, 1 or 2");
        g_opt.sort_impl = value;
    }
    else if (!strcmp(name, "pdl")) g_opt.pdl = value ? 1 : 0;
    else if (!strcmp(name, "find_hints")) g_opt.find_hints = value < 0 ? -1 : (value ? 1 : 0);
    else if (!strcmp(name, "q_chunks")) g_opt.q_chunks = value < 1 ? 1 : value;
    else if (!strcmp(name, "pipe_events")) g_opt.pipe_events = value < 0 ? 0 : (value > 2 ? 2 : value);
    else if (!strcmp(name, "index_alg1")) g_opt.index_alg1 = value < 0 ? -1 : (value ? 1 : 0);
    else if (!strcmp(name, "index_tiled")) g_opt.index_tiled = value < 0 ? -1 : (value ? 1 : 0);
    else if (!strcmp(name, "rec8")) g_opt.rec8 = value < 0 ? -1 : (value ? 1 : 0);
    else if (!strcmp(name, "rank_sectors")) g_opt.rank_sectors = value < 0 ? -1 : (value ? 1 : 0);
    else if (!strcmp(name, "l2_window")) {
        if (value < 0 || value > 3) return fail(GPUMEM_ERR_ARG, "l2_window must be 0..3");
        g_opt.l2_window = value;
    }
    else if (!strcmp(name, "l2_persist")) {  // MB of persisting L2 (device-wide limit), clamped to the maximum
        int dev = 0, mx = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, dev);
        uint64_t b = value < 0 ? 0 : uint64_t(value) << 20;
        if (b > uint64_t(mx)) b = uint64_t(mx);
        const cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, size_t(b));
        if (e != cudaSuccess) return cuda_fail(e, "persisting L2 limit");
        if (!b) cudaCtxResetPersistingL2Cache();
        g_opt.l2_persist = int64_t(b >> 20);
    }
    else if (!strcmp(name, "radix_bits")) {
        if (value != 0 && (value < 8 || value > 10)) return fail(GPUMEM_ERR_ARG, "radix_bits must be 0 or 8..10");
        g_opt.radix_bits = value;
    }
    else return fail(GPUMEM_ERR_ARG, "unknown option '%s'", name);
    return GPUMEM_OK;
}

gpumem_status gpumem_profile_enable(int on) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    g_prof = on != 0;
    return GPUMEM_OK;
}

int gpumem_profile_read(const char **names, double *ms, uint64_t *launches, int max_stages) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    int n = 0;
    for (auto &r : g_recs) {
        float t = 0.f;
        cudaEventSynchronize(r.b);
        cudaEventElapsedTime(&t, r.a, r.b);
        int i = 0;
        for (; i < n; ++i)
            if (!strcmp(names[i], r.name)) break;
        if (i == n) {
            if (n >= max_stages) continue;
            names[n] = r.name;
            ms[n] = 0;
            launches[n] = 0;
            ++n;
        }
        ms[i] += t;
        launches[i] += r.l1 - r.l0;
        g_ev_free.push_back(r.a);
        g_ev_free.push_back(r.b);
    }
    g_recs.clear();
    cudaGetLastError();
    return n;
}

void gpumem_free(void *handle) {
    if (!handle) return;
    const uint32_t magic = *static_cast<uint32_t *>(handle);
    int prev = -1;
    cudaGetDevice(&prev);
    if (magic == kMagicSeq) {
        auto *s = static_cast<gpumem_seq *>(handle);
        cudaSetDevice(s->device);
        dfree(s->words, s->stream);
        dfree(s->bad, s->stream);
        s->magic = 0;
        delete s;
    } else if (magic == kMagicIdx) {
        auto *x = static_cast<gpumem_index *>(handle);
        cudaSetDevice(x->device);
        dfree(x->ptrs, x->stream);
        dfree(x->locs, x->stream);
        dfree(x->rankw, x->stream);
        dfree(x->rsect, x->stream);
        dfree(x->buckets, x->stream);
        dfree(x->recs, x->stream);
        if (x->hv_info) dfree(x->hv_info, x->stream);
        if (x->hv_cnt) dfree(x->hv_cnt, x->stream);
        if (x->hv_list) dfree(x->hv_list, x->stream);
        x->magic = 0;
        delete x;
    } else if (magic == kMagicPipe) {
        auto *pl = static_cast<gpumem_pipeline *>(handle);
        cudaSetDevice(pl->device);
        cudaStreamSynchronize(pl->stream);
        if (pl->fallback) gpumem_free(pl->fallback);
        pipeline_release(pl);
        cudaStreamSynchronize(pl->stream);
        cudaFreeHost(pl->host);
        cudaEventDestroy(pl->ev_in);
        cudaEventDestroy(pl->ev_out);
        if (pl->copy) {
            cudaStreamSynchronize(pl->copy);
            if (pl->stage) dfree(pl->stage, pl->copy);
            cudaStreamSynchronize(pl->copy);
            ws_release_stream(pl->device, pl->copy);
            cudaStreamDestroy(pl->copy);
        }
        cudaEventDestroy(pl->ev_r);
        cudaEventDestroy(pl->ev_q);
        for (int j = 0; j < kMaxQChunks; ++j) {
            cudaEventDestroy(pl->ev_qc[j]);
            cudaEventDestroy(pl->ev_pk[j]);
        }
        cudaEventDestroy(pl->ev_fork);
        cudaEventDestroy(pl->ev_ra);
        cudaEventDestroy(pl->ev_rb);
        ws_release_stream(pl->device, pl->stream);
        for (cudaStream_t x : {pl->side, pl->side2}) {
            cudaStreamSynchronize(x);
            ws_release_stream(pl->device, x);
            cudaStreamDestroy(x);
        }
        cudaEventDestroy(pl->ev_join);
        cudaStreamDestroy(pl->stream);
        pl->magic = 0;
        delete pl;
    } else if (magic == kMagicFasta) {
        auto *f = static_cast<gpumem_fasta *>(handle);
        f->magic = 0;
        delete f;
    } else if (magic == kMagicMems) {
        auto *m = static_cast<gpumem_mems *>(handle);
        cudaSetDevice(m->device);
        dfree(m->dev, m->stream);
        m->magic = 0;
        delete m;
    }
    if (prev >= 0) cudaSetDevice(prev);
    cudaGetLastError();
}

gpumem_status gpumem_pack(const char *bases, uint64_t n, int bases_on_device, void *cuda_stream,
                          gpumem_seq **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!bases && n) return fail(GPUMEM_ERR_ARG, "bases is NULL");
    if (n >= (1ull << 32)) return fail(GPUMEM_ERR_RANGE, "sequence of %llu bases exceeds 2^32-1 (32-bit locations)",
                                       (unsigned long long)n);
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    Stage stage("pack", s);
    Scratch sc(s);
    const uint64_t n_words = (n + 31) / 32 + 4;  // 4 zero words: multi-word extension rounds
    auto *words = static_cast<uint64_t *>(sc.get(n_words * 8));
    auto *bad = static_cast<unsigned long long *>(sc.get(8));
    if (!words || !bad) return GPUMEM_ERR_NOMEM;
    CK(fill_async(bad, 0xffffffffu, 8, s), "flag init");
    const uint8_t *in = reinterpret_cast<const uint8_t *>(bases);
    if (!bases_on_device && n) {
        auto *tmp = static_cast<uint8_t *>(ws_get(kWsPackTmp, n, s));
        if (!tmp) return GPUMEM_ERR_NOMEM;
        CK(cudaMemcpyAsync(tmp, bases, n, cudaMemcpyHostToDevice, s), "H2D copy of bases");
        in = tmp;
    }
    CK(launch_pack(in, n, words, n_words, bad, s), "pack kernel");
    sc.keep(words);
    sc.keep(bad);
    auto *h = new gpumem_seq{kMagicSeq, dev, s, n, n_words, words, bad};
    *out = h;
    return GPUMEM_OK;
}

gpumem_status gpumem_revcomp(const gpumem_seq *in, void *cuda_stream, gpumem_seq **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!in || in->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "not a gpumem_seq");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    Stage stage("revcomp", s);
    Scratch sc(s);
    auto *words = static_cast<uint64_t *>(sc.get(in->n_words * 8));
    auto *bad = static_cast<unsigned long long *>(sc.get(8));
    if (!words || !bad) return GPUMEM_ERR_NOMEM;
    CK(cudaMemcpyAsync(bad, in->bad, 8, cudaMemcpyDeviceToDevice, s), "copy flag");
    CK(launch_revcomp(in->words, in->n, words, in->n_words, s), "revcomp kernel");
    sc.keep(words);
    sc.keep(bad);
    *out = new gpumem_seq{kMagicSeq, dev, s, in->n, in->n_words, words, bad};
    return GPUMEM_OK;
}

gpumem_status gpumem_seq_check(const gpumem_seq *sq, void *cuda_stream) {
    if (!sq || sq->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "not a gpumem_seq");
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    unsigned long long *h = pinned_slots();
    if (!h) return fail(GPUMEM_ERR_NOMEM, "pinned host buffer");
    CK(cudaMemcpyAsync(h, sq->bad, 8, cudaMemcpyDeviceToHost, s), "D2H");
    CK(cudaStreamSynchronize(s), "sync");
    if (h[0] != ~0ull)
        return fail(GPUMEM_ERR_ALPHABET, "byte at position %llu is not in {A,C,G,T,a,c,g,t}", h[0]);
    return GPUMEM_OK;
}

gpumem_status gpumem_seq_info(const gpumem_seq *sq, uint64_t *n_bases, const uint64_t **dev_words,
                              uint64_t *n_words) {
    if (!sq || sq->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "not a gpumem_seq");
    if (n_bases) *n_bases = sq->n;
    if (dev_words) *dev_words = sq->words;
    if (n_words) *n_words = sq->n_words;
    return GPUMEM_OK;
}

static gpumem_status index_build_impl(const gpumem_seq *R, uint32_t ls, uint32_t L, uint32_t step,
                                      uint64_t r_begin, uint64_t r_end, void *cuda_stream, gpumem_index **out);

gpumem_status gpumem_index_build_step(const gpumem_seq *R, uint32_t ls, uint32_t L, uint32_t step,
                                      void *cuda_stream, gpumem_index **out) {
    return index_build_impl(R, ls, L, step, 0, UINT64_MAX, cuda_stream, out);
}

gpumem_status gpumem_index_build_range(const gpumem_seq *R, uint32_t ls, uint32_t L, uint64_t r_begin,
                                       uint64_t r_end, void *cuda_stream, gpumem_index **out) {
    if (ls < 1 || ls > 15 || L < ls) {
        if (out) *out = nullptr;
        return fail(GPUMEM_ERR_ARG, "need 1 <= seed_len <= 15 and seed_len <= min_len (got %u, %u)", ls, L);
    }
    return index_build_impl(R, ls, L, L - ls + 1, r_begin, r_end, cuda_stream, out);
}

static gpumem_status index_build_impl(const gpumem_seq *R, uint32_t ls, uint32_t L, uint32_t step,
                                      uint64_t r_begin, uint64_t r_end, void *cuda_stream, gpumem_index **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!R || R->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "R is not a gpumem_seq");
    if (ls < 1 || ls > 15) return fail(GPUMEM_ERR_ARG, "seed_len %u outside [1, 15]", ls);
    if (L < ls) return fail(GPUMEM_ERR_ARG, "min_len %u < seed_len %u (Eq. 1 needs ls <= L)", L, ls);
    if (step < 1 || step > L - ls + 1)
        return fail(GPUMEM_ERR_ARG, "step %u outside [1, L - ls + 1 = %u] (Eq. 1)", step, L - ls + 1);
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    if (dev != R->device) return fail(GPUMEM_ERR_ARG, "R lives on device %d, current is %d", R->device, dev);
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    const uint64_t nb = 1ull << (2 * ls);
    // sampled locations p = k * step with r_begin <= p < r_end and p <= |R| - ls
    if (r_begin > r_end) return fail(GPUMEM_ERR_RANGE, "r_begin > r_end");
    const uint64_t k_all = R->n >= ls ? (R->n - ls) / step + 1 : 0;
    const uint64_t k0 = (r_begin + step - 1) / step;
    const uint64_t k1_band = r_end >= UINT64_MAX - step ? UINT64_MAX : (r_end + step - 1) / step;
    const uint64_t k1 = k1_band < k_all ? k1_band : k_all;
    const uint64_t n_locs = k1 > k0 ? k1 - k0 : 0;
    Scratch sc(s);
    uint32_t *ptrs = nullptr;  // the dense ptrs table is expanded on demand (index_ptrs)
    // lookup directory: rank sectors when the compact table {first, count} (<= 8 B per
    // sampled seed) would not stay in L2 next to the rest, else the smaller rank words
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    const bool use_sect = g_opt.rank_sectors < 0 ? n_locs * 8 > uint64_t(l2) / 4 : g_opt.rank_sectors != 0;
    unsigned long long *rankw = nullptr;
    uint4 *rsect = nullptr;
    if (use_sect) rsect = static_cast<uint4 *>(sc.get(((nb + 31) / 32) * 16));
    else rankw = static_cast<unsigned long long *>(sc.get(((nb + 31) / 32) * 16));  // + rotated occupancy
    const bool alg1 = n_locs && (g_opt.index_alg1 > 0 || (g_opt.index_alg1 < 0 && n_locs * 4 >= nb));
    const bool tiled = g_opt.index_tiled > 0 || (g_opt.index_tiled < 0 && n_locs <= (1u << 20));
    const TiledPlan tp = (tiled && !alg1) ? tiled_plan(ls, n_locs) : TiledPlan{};
    // compact table: per location, gapped per chunk / bin (radix and tiled builds), or one
    // entry per occupied seed (Alg. 1 as written)
    const uint64_t max_occ = (alg1 ? (n_locs < nb ? n_locs : nb) : n_locs) + 1;
    auto *buckets = static_cast<uint2 *>(sc.get(max_occ * sizeof(uint2)));
    void *fill_scratch = ws_get(kWsFill, ptrs_fill_scratch_bytes(ls), s);
    auto *locs0 = static_cast<uint32_t *>(sc.get((n_locs ? n_locs : 1) * 4));
    if (!(rsect || rankw) || !buckets || !fill_scratch || !locs0) return GPUMEM_ERR_NOMEM;
    uint32_t *locs = locs0;
    const uint32_t *codes_sorted = nullptr;
    // 8-byte seed records when the left extension is capped at <= 8 bases (step <= 8)
    const int rec8 = g_opt.rec8 < 0 ? (step <= 8 ? 1 : 0) : int(g_opt.rec8 != 0);
    void *recs = sc.get((n_locs ? n_locs : 1) * (rec8 ? sizeof(uint2) : sizeof(uint4)));
    if (!recs) return GPUMEM_ERR_NOMEM;
    // heavy buckets reordered minority-left-flank first (k_hv_part) when the record's left
    // flank decides canonicity (step <= its width); radix-path directory fills list them
    const bool hv_ok = n_locs && !tp.ok && !alg1 && step <= (rec8 ? 8u : 16u);
    uint2 *hv_list = nullptr;
    uint4 *hv_info = nullptr;
    unsigned int *hv_cnt = nullptr;
    if (hv_ok) {
        hv_list = static_cast<uint2 *>(sc.get(kHvCap * sizeof(uint2)));
        hv_info = static_cast<uint4 *>(sc.get(kHvCap * sizeof(uint4)));
        hv_cnt = static_cast<unsigned int *>(sc.get(2 * sizeof(unsigned int)));
        if (!hv_list || !hv_info || !hv_cnt) return GPUMEM_ERR_NOMEM;
    }
    bool recs_done = false, fill_done = false;
    if (tp.ok) {
        // Alg. 1 tiled over the seed space: partition, then every bin in shared memory
        void *scratch = ws_get(kWsTiled, tiled_scratch_bytes(tp, n_locs), s);
        if (!scratch) return GPUMEM_ERR_NOMEM;
        {
            Stage g("index.tiled", s);
            const bool side = t_cap && t_cap->side;  // hot bins beside the warps' bins
            CK(launch_index_tiled(tp, R->words, ls, step, k0, n_locs, rankw, rsect, buckets, locs0, recs, rec8, scratch, s,
                                  side ? t_cap->side : nullptr, side ? t_cap->ev_a : nullptr,
                                  side ? t_cap->ev_b : nullptr),
               "index (tiled Alg. 1)");
        }
        fill_done = recs_done = true;
    } else if (alg1) {
        // dense index: Alg. 1 literally (atomic counts, prefix sums, placement, bucket sort)
        void *scratch = ws_get(kWsAlg1, alg1_scratch_bytes(ls, n_locs), s);
        if (!scratch) return GPUMEM_ERR_NOMEM;
        {
            Stage g("index.alg1", s);
            CK(launch_index_alg1(R->words, ls, step, k0, n_locs, rankw, rsect, buckets, locs0, scratch, s),
               "index (Alg. 1)");
        }
        fill_done = true;
    } else if (n_locs) {
        auto *codes0 = static_cast<uint32_t *>(ws_get(kWsCodes0, n_locs * 4, s));
        auto *codes1 = static_cast<uint32_t *>(ws_get(kWsCodes1, n_locs * 4, s));
        auto *locs1 = static_cast<uint32_t *>(sc.get(n_locs * 4));
        void *scratch = ws_get(kWsRadix, radix_scratch_bytes(n_locs), s);
        if (!codes0 || !codes1 || !locs1 || !scratch) return GPUMEM_ERR_NOMEM;
        // the first radix pass generates the locations (p = (k0 + i) * step) instead of
        // reading them: the codes pass writes them only when no pass runs
        const bool gen = radix_passes(int(2 * ls), n_locs) > 0;
        {
            Stage g("index.codes", s);
            CK(launch_seed_codes(R->words, ls, step, k0, n_locs, codes0, gen ? nullptr : locs0, s), "seed codes");
        }
        bool alt = false;
        {
            Stage g("index.sort", s);
            CK(radix_sort_u32(codes0, locs0, codes1, locs1, n_locs, int(2 * ls), scratch, s, &alt, 0, gen ? k0 : 0,
                              gen ? step : 0u),
               "seed counting sort");
        }
        codes_sorted = alt ? codes1 : codes0;
        locs = alt ? locs1 : locs0;
    }
    // the directory (from the sorted codes) and the seed records (from locs and R) are
    // independent: in a pipeline the records are built on its side stream meanwhile
    const bool fork = t_cap && t_cap->side && n_locs && !recs_done && !fill_done;
    if (fork) {
        CK(cudaEventRecord(t_cap->ev_a, s), "fork");
        CK(cudaStreamWaitEvent(t_cap->side, t_cap->ev_a, 0), "fork");
        {
            Stage g("index.recs", t_cap->side);
            CK(launch_seed_recs(R->words, ls, locs, n_locs, recs, rec8, t_cap->side), "seed records");
        }
        CK(cudaEventRecord(t_cap->ev_b, t_cap->side), "join");
        recs_done = true;
    }
    if (!fill_done) {
        Stage g("index.ptrs", s);
        CK(launch_ptrs_fill(codes_sorted, n_locs, ls, ptrs, rankw, rsect, buckets, fill_scratch, s, hv_list, hv_cnt),
           "ptrs fill");
    }
    if (fork) CK(cudaStreamWaitEvent(s, t_cap->ev_b, 0), "join");
    if (n_locs && !recs_done) {
        Stage g("index.recs", s);
        CK(launch_seed_recs(R->words, ls, locs, n_locs, recs, rec8, s), "seed records");
    }
    if (hv_ok) {
        Stage g("index.heavy", s);
        CK(launch_heavy_prep(recs, rec8, step, hv_list, hv_cnt, hv_info, s), "heavy buckets");
        sc.keep(hv_list);
        sc.keep(hv_info);
        sc.keep(hv_cnt);
    }
    if (rankw) sc.keep(rankw);
    if (rsect) sc.keep(rsect);
    sc.keep(buckets);
    sc.keep(locs);
    sc.keep(recs);
    auto *h = new gpumem_index{kMagicIdx, dev, s, R, ls, L, step, n_locs, ptrs, locs, rankw, rsect, buckets, recs, rec8};
    h->hv_info = hv_info;
    h->hv_cnt = hv_cnt;
    h->hv_list = hv_list;
    *out = h;
    return GPUMEM_OK;
}

gpumem_status gpumem_index_build(const gpumem_seq *R, uint32_t ls, uint32_t L, void *cuda_stream,
                                 gpumem_index **out) {
    if (out) *out = nullptr;
    if (ls < 1 || ls > 15 || L < ls) {
        if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
        return fail(GPUMEM_ERR_ARG, "need 1 <= seed_len <= 15 and seed_len <= min_len (got %u, %u)", ls, L);
    }
    return gpumem_index_build_step(R, ls, L, L - ls + 1, cuda_stream, out);
}

// The paper's dense ptrs[4^ls + 1], expanded once from the rank directory
// and the compact table on first use (index_view, or find with use_bitmap = 0), on
// stream s. The fast lookup never reads it, so the index build does not write it.
static std::mutex g_ptrs_mu;
static gpumem_status index_ptrs(const gpumem_index *cidx, cudaStream_t s) {
    auto *idx = const_cast<gpumem_index *>(cidx);
    std::lock_guard<std::mutex> g(g_ptrs_mu);
    if (idx->ptrs) return GPUMEM_OK;
    const uint64_t nb = 1ull << (2 * idx->ls);
    auto *p = static_cast<uint32_t *>(dalloc((nb + 1) * 4, s));
    if (!p) return GPUMEM_ERR_NOMEM;
    const cudaError_t e = launch_ptrs_expand(idx->rankw, idx->rsect, idx->buckets, idx->ls, idx->n_locs, p, s);
    if (e != cudaSuccess) {
        dfree(p, s);
        return cuda_fail(e, "ptrs expand");
    }
    if (s != idx->stream && !(t_cap && t_cap->mode == 2)) {  // freed on the index's stream later
        const cudaError_t e2 = cudaStreamSynchronize(s);
        if (e2 != cudaSuccess) return cuda_fail(e2, "ptrs expand");
    }
    idx->ptrs = p;
    return GPUMEM_OK;
}

gpumem_status gpumem_index_view(const gpumem_index *idx, const uint32_t **dev_ptrs, const uint32_t **dev_locs,
                                uint64_t *n_locs) {
    if (!idx || idx->magic != kMagicIdx) return fail(GPUMEM_ERR_ARG, "not a gpumem_index");
    if (dev_ptrs) {
        gpumem_status st = index_ptrs(idx, idx->stream);
        if (st) return st;
        CK(cudaStreamSynchronize(idx->stream), "ptrs expand");
    }
    if (dev_ptrs) *dev_ptrs = idx->ptrs;
    if (dev_locs) *dev_locs = idx->locs;
    if (n_locs) *n_locs = idx->n_locs;
    return GPUMEM_OK;
}

static gpumem_status sort_into_triples(uint64_t *keys, uint32_t *lens, uint64_t n, uint32_t key_bits,
                                       uint32_t qbits, int dev, cudaStream_t s, gpumem_mems **out) {
    Scratch sc(s);
    auto *trip = static_cast<gpumem_triple *>(sc.get((n ? n : 1) * sizeof(gpumem_triple)));
    if (!trip) return GPUMEM_ERR_NOMEM;
    if (n) {
        Stage g("sort", s);
        // MSD bucket sort (keys are unique): two passes over the data; measured faster than
        // the 7-pass LSD radix up to a few million keys, slower beyond (its 16K-way scatter)
        if (g_opt.sort_impl == 2 || (g_opt.sort_impl == 0 && n <= kMsdMaxN)) {
            void *scratch = ws_get(kWsSortScratch, msd_scratch_bytes(n), s);
            if (!scratch) return GPUMEM_ERR_NOMEM;
            CK(msd_sort(keys, lens, n, int(key_bits), scratch, s, trip, qbits), "triple sort");
        } else {  // stable LSD onesweep radix
            auto *k1 = static_cast<uint64_t *>(ws_get(kWsSortK, n * 8, s));
            auto *l1 = static_cast<uint32_t *>(ws_get(kWsSortL, n * 4, s));
            void *scratch = ws_get(kWsSortScratch, radix_scratch_bytes(n), s);
            if (!k1 || !l1 || !scratch) return GPUMEM_ERR_NOMEM;
            bool alt = false;
            CK(radix_sort_u64(keys, lens, k1, l1, n, int(key_bits), scratch, s, &alt), "triple sort");
            CK(launch_keys_to_triples(alt ? k1 : keys, alt ? l1 : lens, n, qbits, trip, s), "keys to triples");
        }
    }
    sc.keep(trip);
    *out = new gpumem_mems{kMagicMems, dev, s, n, trip, gpumem_find_stats{}};
    (*out)->stats.mems = n;
    return GPUMEM_OK;
}

gpumem_status gpumem_find_mems(const gpumem_index *idx, const gpumem_seq *Q, uint64_t q_begin, uint64_t q_end,
                               void *cuda_stream, gpumem_mems **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!idx || idx->magic != kMagicIdx) return fail(GPUMEM_ERR_ARG, "idx is not a gpumem_index");
    if (!Q || Q->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "Q is not a gpumem_seq");
    const gpumem_seq *R = idx->R;
    if (!R || R->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "the index's R was freed");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    if (Q->device != dev || idx->device != dev) return fail(GPUMEM_ERR_ARG, "handles on another device");
    const uint64_t nQ = Q->n, nR = R->n;
    if (q_end > nQ) q_end = nQ;
    if (q_begin > nQ) return fail(GPUMEM_ERR_RANGE, "q_begin %llu > |Q| = %llu", (unsigned long long)q_begin,
                                  (unsigned long long)nQ);
    if (q_begin > q_end) q_end = q_begin;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    const uint32_t ls = idx->ls, L = idx->L, step = idx->step;

    FindParams P{};
    P.R = R->words;
    P.nR = nR;
    P.Q = Q->words;
    P.nQ = nQ;
    P.nQw = Q->n_words;
    P.q_avail = nQ;
    if (!g_opt.use_bitmap) {  // the paper's lookup reads the dense ptrs
        st = index_ptrs(idx, s);
        if (st) return st;
    }
    P.ptrs = idx->ptrs;
    P.recs = idx->recs;
    P.rec8 = idx->rec8;
    P.rankw = idx->rankw;
    P.rsect = idx->rsect;
    P.buckets = idx->buckets;
    P.hv_info = idx->hv_info;
    P.hv_n = idx->hv_cnt ? idx->hv_cnt + 1 : nullptr;
    P.ls = ls;
    P.L = L;
    P.step = step;
    P.qbits = bits_for(nQ);
    P.own_lo = q_begin;
    P.own_hi = q_end;
    P.scan_lo = q_begin;
    P.scan_hi = q_begin;
    if (nQ >= ls && nR >= ls && nQ >= L && nR >= L && q_begin < q_end) {
        const uint64_t hi = q_end + step - 1;  // the canonical seed lies < step right of the MEM start
        P.scan_hi = hi < nQ - ls + 1 ? hi : nQ - ls + 1;
        if (P.scan_hi < P.scan_lo) P.scan_hi = P.scan_lo;
    }
    const uint64_t span = P.scan_hi - P.scan_lo;
    const uint64_t tile = find_tile_positions(idx->rsect != nullptr);
    P.n_tiles = (span + tile - 1) / tile;
    P.spill_t = uint32_t(g_opt.find_spill);
    P.use_bitmap = int(g_opt.use_bitmap);
    P.static_lb = int(g_opt.static_lb);
    {  // records that cannot share L2 with the lookup tables are streamed
        int l2 = 0;
        cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
        P.recs_stream = idx->n_locs * (idx->rec8 ? 8 : 16) > uint64_t(l2) / 2 ? 1 : 0;
        if (g_opt.find_hints >= 0) P.recs_stream = int(g_opt.find_hints);
        // optional persisting-L2 window over one lookup structure (l2_window / l2_persist)
        if (g_opt.l2_window && g_opt.l2_persist) {
            const uint64_t groups = ((1ull << (2 * ls)) + 31) / 32;
            void *base = nullptr;
            uint64_t bytes = 0;
            if (g_opt.l2_window == 1) {
                base = idx->rsect ? static_cast<void *>(idx->rsect) : static_cast<void *>(idx->rankw);
                bytes = groups * 16;
            } else if (g_opt.l2_window == 2) {
                base = idx->buckets;
                bytes = idx->n_locs * sizeof(uint2);
            } else {
                base = idx->recs;
                bytes = idx->n_locs * (idx->rec8 ? 8 : 16);
            }
            int wmax = 0;
            cudaDeviceGetAttribute(&wmax, cudaDevAttrMaxAccessPolicyWindowSize, dev);
            if (bytes > uint64_t(wmax)) bytes = uint64_t(wmax);
            if (base && bytes) {
                const double set_aside = double(g_opt.l2_persist) * (1 << 20);
                P.l2win.base_ptr = base;
                P.l2win.num_bytes = size_t(bytes);
                P.l2win.hitRatio = float(set_aside >= double(bytes) ? 1.0 : set_aside / double(bytes));
                P.l2win.hitProp = cudaAccessPropertyPersisting;
                P.l2win.missProp = cudaAccessPropertyStreaming;
            }
        }
    }
    uint64_t cap = g_opt.out_capacity ? uint64_t(g_opt.out_capacity) : (span / 8 + 4096);

    Scratch sc(s);
    // [16, 24): per-piece tile counters (u32), [24, 40): per-piece heavy-queue counters
    auto *ctr = static_cast<unsigned long long *>(ws_get(kWsCtr, 320, s));
    const uint64_t spill_cap = span / 8 + 4096;
    auto *spill = static_cast<uint4 *>(ws_get(kWsSpill, spill_cap * sizeof(uint4), s));
    uint64_t coop_cap = span / 64 + 4096;
    if (!ctr || !spill) return GPUMEM_ERR_NOMEM;
    P.out_count = ctr;
    P.spill_count = ctr + 1;
    P.tile_ctr = reinterpret_cast<unsigned int *>(ctr + 2);
    P.stats = ctr + 3;
    P.coop_count = ctr + 7;
    P.work = ctr + 8;  // [8] max hits per warp, [9] warps
    P.spill = spill;
    P.spill_cap = spill_cap;
    unsigned long long *h = pinned_slots();
    if (!h) return fail(GPUMEM_ERR_NOMEM, "pinned host buffer");

    if (t_cap && t_cap->deferred) {
        // pipeline: one pass with the automatic capacity, no host round trip. The sort
        // takes the MEM count from the device counter; the counters and alphabet flags go
        // to the pipeline's pinned buffer, checked by gpumem_pipeline_result (which reruns
        // this call the ordinary way in the rare overflow case).
        auto *keys = static_cast<uint64_t *>(ws_get(kWsKeys, cap * 8, s));
        auto *lens = static_cast<uint32_t *>(ws_get(kWsLens, cap * 4, s));
        P.coopq = static_cast<uint2 *>(ws_get(kWsCoop, coop_cap * sizeof(uint2), s));
        // output sort by the device-resident count; which one: sort_impl if pinned, else by
        // the MEM count of the pipeline's measuring run (MSD up to kMsdMaxN, LSD beyond)
        int impl = int(g_opt.sort_impl);
        if (impl == 0) impl = (t_cap->mode == 2 && t_cap->expect_n > kMsdMaxN) ? 1 : 2;
        size_t sbytes = msd_scratch_bytes(cap);
        if (radix_scratch_bytes(cap) > sbytes) sbytes = radix_scratch_bytes(cap);
        void *scratch = ws_get(kWsSortScratch, sbytes, s);  // sized for every choice: the measuring
        auto *k1 = static_cast<uint64_t *>(ws_get(kWsSortK, cap * 8, s));  // run and the capture agree
        auto *l1 = static_cast<uint32_t *>(ws_get(kWsSortL, cap * 4, s));
        auto *trip = static_cast<gpumem_triple *>(sc.get(cap * sizeof(gpumem_triple)));
        if (!keys || !lens || !P.coopq || !scratch || !trip || !k1 || !l1) return GPUMEM_ERR_NOMEM;
        P.out_key = keys;
        P.out_len = lens;
        P.capacity = cap;
        P.coop_cap = coop_cap;
        CK(fill_async(ctr, 0u, 320, s), "zero counters");
        const int K = t_cap->q_chunks > 1 && q_begin == 0 && q_end == nQ ? t_cap->q_chunks : 1;
        if (K == 1) {
            Stage g("find", s);
            CK(launch_find(P, int(g_opt.find_grid), s), "find kernel");
        } else {
            // streamed query: piece i's search starts once piece i is packed. It owns the MEM
            // starts [B[i] - X, B[i+1] - X) (X = 0 at the ends of Q), so its seeds (up to
            // step - 1 bases past a start, ls long) lie in the data present; extensions
            // stop at q_avail = B[i+1], and a match cut there starts >= X >= L before it
            const uint64_t *B = t_cap->q_bnd;
            const uint64_t X = std::max<uint64_t>(L, step + ls) + 64;
            Stage g("find", s);
            for (int i = 0; i < K && P.n_tiles; ++i) {
                CK(cudaStreamWaitEvent(s, t_cap->q_packed[i], 0), "wait for query piece");
                FindParams Pi = P;
                Pi.q_avail = B[i + 1];
                Pi.own_lo = i == 0 ? 0 : B[i] - X;
                Pi.own_hi = i + 1 == K ? nQ : B[i + 1] - X;
                Pi.scan_lo = Pi.own_lo;
                const uint64_t hi = Pi.own_hi + step - 1;
                Pi.scan_hi = hi < nQ - ls + 1 ? hi : nQ - ls + 1;
                if (Pi.scan_hi < Pi.scan_lo) Pi.scan_hi = Pi.scan_lo;
                Pi.n_tiles = (Pi.scan_hi - Pi.scan_lo + tile - 1) / tile;
                Pi.tile_ctr = reinterpret_cast<unsigned int *>(ctr + 16) + i;
                // the piece's own heavy queue (its counter; the buffer is reused piece after
                // piece): its hits are decided with the piece's ownership range and data end
                Pi.spill_count = ctr + 24 + i;
                CK(launch_find(Pi, int(g_opt.find_grid), s), "find kernel");
                CK(launch_heavy(Pi, s), "heavy kernel");
            }
            CK(cudaStreamWaitEvent(s, t_cap->q_packed[K - 1], 0), "join the query pieces");
        }
        if (P.n_tiles) {
            Stage g("find.heavy", s);
            if (K == 1) CK(launch_heavy(P, s), "heavy kernel");
            CK(launch_coop(P, s), "coop kernel");
            if (K > 1) CK(launch_open_fix(P, s), "open-match fix");
        }
        {
            Stage g("sort", s);
            const int kb = int(bits_for(nR) + P.qbits);
            if (impl == 2) {
                CK(msd_sort_dev(keys, lens, ctr, cap, kb, scratch, s, trip, P.qbits), "triple sort");
            } else {
                bool alt = false;
                CK(radix_sort_u64(keys, lens, k1, l1, cap, kb, scratch, s, &alt, 0, ctr), "triple sort");
                CK(launch_keys_to_triples(alt ? k1 : keys, alt ? l1 : lens, cap, P.qbits, trip, s, ctr),
                   "keys to triples");
            }
        }
        CK(launch_collect(ctr, R->bad, Q->bad, t_cap->host, s), "report");
        sc.keep(trip);
        *out = new gpumem_mems{kMagicMems, dev, s, 0, trip, gpumem_find_stats{}};
        t_cap->out_cap = cap;
        t_cap->coop_cap = coop_cap;
        t_cap->spill_cap = spill_cap;
        t_cap->span = span;
        t_cap->mems = *out;
        return GPUMEM_OK;
    }

    uint64_t count = 0;
    int attempts = 0;
    uint64_t *keys = nullptr;
    uint32_t *lens = nullptr;
    for (int attempt = 0; attempt < 3; ++attempt) {
        keys = static_cast<uint64_t *>(ws_get(kWsKeys, cap * 8, s));
        lens = static_cast<uint32_t *>(ws_get(kWsLens, cap * 4, s));
        if (!keys || !lens) return GPUMEM_ERR_NOMEM;
        P.out_key = keys;
        P.out_len = lens;
        P.capacity = cap;
        P.coopq = static_cast<uint2 *>(ws_get(kWsCoop, coop_cap * sizeof(uint2), s));
        P.coop_cap = coop_cap;
        if (!P.coopq) return GPUMEM_ERR_NOMEM;
        CK(fill_async(ctr, 0u, 128, s), "zero counters");
        {
            Stage g("find", s);
            CK(launch_find(P, int(g_opt.find_grid), s), "find kernel");
        }
        if (P.n_tiles) {
            Stage g("find.heavy", s);
            CK(launch_heavy(P, s), "heavy kernel");
            CK(launch_coop(P, s), "coop kernel");
        }
        ++attempts;
        CK(cudaMemcpyAsync(h, ctr, 64, cudaMemcpyDeviceToHost, s), "D2H counters");
        CK(cudaMemcpyAsync(h + 10, ctr + 8, 16, cudaMemcpyDeviceToHost, s), "D2H balance");
        CK(cudaMemcpyAsync(h + 8, R->bad, 8, cudaMemcpyDeviceToHost, s), "D2H flag");
        CK(cudaMemcpyAsync(h + 9, Q->bad, 8, cudaMemcpyDeviceToHost, s), "D2H flag");
        CK(cudaStreamSynchronize(s), "find sync");
        if (h[8] != ~0ull) return fail(GPUMEM_ERR_ALPHABET, "R: byte at position %llu is not in {A,C,G,T,a,c,g,t}", h[8]);
        if (h[9] != ~0ull) return fail(GPUMEM_ERR_ALPHABET, "Q: byte at position %llu is not in {A,C,G,T,a,c,g,t}", h[9]);
        count = h[0];
        if (count <= cap && h[7] <= coop_cap) break;
        if (attempt == 2) return fail(GPUMEM_ERR_CUDA, "output count changed between runs (%llu > %llu)",
                                      (unsigned long long)count, (unsigned long long)cap);
        // overflow: rerun with exact capacities. The count of a run whose coop queue
        // overflowed leaves out the dropped entries' MEMs (each entry yields at most one)
        const uint64_t dropped = h[7] > coop_cap ? h[7] - coop_cap : 0;
        if (count + dropped > cap) cap = count + dropped;
        if (h[7] > coop_cap) coop_cap = h[7];
    }
    gpumem_find_stats fs{};
    fs.positions = span;
    fs.occupied = h[3] + h[6];
    fs.hits = h[4] + h[5];
    fs.spilled_chunks = h[1] < spill_cap ? h[1] : spill_cap;
    fs.attempts = uint32_t(attempts);
    fs.max_warp_hits = h[10];
    fs.warps = h[11];
    const uint32_t key_bits = bits_for(nR) + P.qbits;
    const gpumem_status st2 = sort_into_triples(keys, lens, count, key_bits, P.qbits, dev, s, out);
    if (st2 == GPUMEM_OK) {
        fs.mems = count;
        (*out)->stats = fs;
    }
    return st2;
}

gpumem_status gpumem_pipeline_create(uint64_t r_len, uint64_t q_len, uint32_t seed_len, uint32_t min_len,
                                     uint64_t q_begin, uint64_t q_end, void *cuda_stream, gpumem_pipeline **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (seed_len < 1 || seed_len > 15 || min_len < seed_len)
        return fail(GPUMEM_ERR_ARG, "need 1 <= seed_len <= 15 and seed_len <= min_len (got %u, %u)", seed_len,
                    min_len);
    if (r_len >= (1ull << 32) || q_len >= (1ull << 32))
        return fail(GPUMEM_ERR_RANGE, "sequences must be shorter than 2^32 bases");
    if (q_begin > q_len) return fail(GPUMEM_ERR_RANGE, "q_begin > |Q|");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    auto *pl = new gpumem_pipeline{};
    pl->magic = kMagicPipe;
    pl->device = dev;
    pl->user = static_cast<cudaStream_t>(cuda_stream);
    // the legacy default stream cannot be captured: the graph runs on a stream of its
    // own, ordered after / before the caller's stream by events
    if (cudaStreamCreateWithFlags(&pl->stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&pl->side, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&pl->side2, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_join, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_ra, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_rb, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_r, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_q, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_in, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&pl->ev_out, cudaEventDisableTiming) != cudaSuccess) {
        const cudaError_t e = cudaGetLastError();
        delete pl;
        return cuda_fail(e, "pipeline stream");
    }
    pl->nR = r_len;
    pl->nQ = q_len;
    pl->q_begin = q_begin;
    pl->q_end = q_end;
    pl->ls = seed_len;
    pl->L = min_len;
    // streamed query for host-input runs (option q_chunks): pieces of >= max(1 Mbp, 8 L)
    // bases on 32-base boundaries (a piece's search then owns a non-empty start range and
    // a cut match is already >= L long)
    {
        int K = int(g_opt.q_chunks < 1 ? 1 : (g_opt.q_chunks > kMaxQChunks ? kMaxQChunks : g_opt.q_chunks));
        const uint64_t min_piece = std::max<uint64_t>(uint64_t(1) << 20, 8ull * min_len + 256);
        while (K > 1 && q_len / uint64_t(K) < 2 * min_piece) --K;
        if (q_begin != 0 || q_end < q_len) K = 1;  // a sharded pipeline keeps the whole-Q path
        if (min_len - seed_len + 1 > 4000) K = 1;   // left extensions past one lane's reach defer
                                                    // before their ownership is known
        pl->q_chunks = K;
        // the last piece small (its search is the part of the run after the copy): the
        // first K-1 pieces share the rest evenly
        const uint64_t last = K > 1 ? std::max<uint64_t>(min_piece, q_len / 32) : q_len;
        const uint64_t head = q_len - last;
        for (int j = 0; j < K; ++j) pl->q_bnd[j] = K > 1 ? (head * uint64_t(j) / uint64_t(K - 1)) / 32 * 32 : 0;
        pl->q_bnd[K] = q_len;
        pl->cap_chunks = 1;
        for (int j = 0; j < kMaxQChunks; ++j) {
            if (cudaEventCreateWithFlags(&pl->ev_qc[j], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&pl->ev_pk[j], cudaEventDisableTiming) != cudaSuccess) {
                cudaGetLastError();
                gpumem_free(pl);
                return fail(GPUMEM_ERR_CUDA, "pipeline events");
            }
        }
    }
    if (cudaMallocHost(&pl->host, 16 * sizeof(unsigned long long)) != cudaSuccess) {
        cudaGetLastError();
        delete pl;
        return fail(GPUMEM_ERR_NOMEM, "pinned host buffer");
    }
    *out = pl;
    return GPUMEM_OK;
}

gpumem_status gpumem_pipeline_run(gpumem_pipeline *pl, const char *r_bases_dev, const char *q_bases_dev) {
    if (!pl || pl->magic != kMagicPipe) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    if ((!r_bases_dev && pl->nR) || (!q_bases_dev && pl->nQ)) return fail(GPUMEM_ERR_ARG, "NULL input");
    int dev = -1;
    cudaGetDevice(&dev);
    if (dev != pl->device) return fail(GPUMEM_ERR_ARG, "pipeline lives on device %d, current is %d", pl->device, dev);
    if (pl->fallback) {
        gpumem_free(pl->fallback);
        pl->fallback = nullptr;
    }
    CK(cudaEventRecord(pl->ev_in, pl->user), "event");  // inputs written on the caller's stream
    CK(cudaStreamWaitEvent(pl->stream, pl->ev_in, 0), "wait");
    if (!pl->exec || pl->inR != r_bases_dev || pl->inQ != q_bases_dev) {
        const gpumem_status st = pipeline_capture(pl, r_bases_dev, q_bases_dev, false);
        if (st) return st;
    }
    CK(pipeline_launch(pl, false), "graph launch");
    note_launch(int(pl->launches));
    CK(cudaEventRecord(pl->ev_out, pl->stream), "event");  // the caller's later work sees the result
    CK(cudaStreamWaitEvent(pl->user, pl->ev_out, 0), "wait");
    pl->ran = 1;
    return GPUMEM_OK;
}

gpumem_status gpumem_pipeline_run_host(gpumem_pipeline *pl, const char *r_bases_host, const char *q_bases_host) {
    if (!pl || pl->magic != kMagicPipe) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    if ((!r_bases_host && pl->nR) || (!q_bases_host && pl->nQ)) return fail(GPUMEM_ERR_ARG, "NULL input");
    int dev = -1;
    cudaGetDevice(&dev);
    if (dev != pl->device) return fail(GPUMEM_ERR_ARG, "pipeline lives on device %d, current is %d", pl->device, dev);
    if (pl->fallback) {
        gpumem_free(pl->fallback);
        pl->fallback = nullptr;
    }
    if (!pl->copy) CK(cudaStreamCreateWithFlags(&pl->copy, cudaStreamNonBlocking), "copy stream");
    if (!pl->stage) {  // device copies of R and Q (allocator hook if set)
        pl->stage = static_cast<char *>(dalloc(pl->nR + pl->nQ + 256, pl->copy));
        if (!pl->stage) return GPUMEM_ERR_NOMEM;
        CK(cudaStreamSynchronize(pl->copy), "input staging");
    }
    char *dR = pl->stage, *dQ = pl->stage + pl->nR;
    // the copies start after the caller's prior work and after the previous run (which
    // read the staging buffers); R, then Q, each announced by an event
    CK(cudaEventRecord(pl->ev_in, pl->user), "event");
    CK(cudaStreamWaitEvent(pl->copy, pl->ev_in, 0), "wait");
    CK(cudaStreamWaitEvent(pl->copy, pl->ev_out, 0), "wait");
    if (pl->nR) CK(cudaMemcpyAsync(dR, r_bases_host, pl->nR, cudaMemcpyHostToDevice, pl->copy), "H2D R");
    CK(cudaEventRecord(pl->ev_r, pl->copy), "event");
    for (int j = 0; j < pl->q_chunks; ++j) {  // Q in pieces, each announced by its event
        const uint64_t a = pl->q_bnd[j], b = pl->q_bnd[j + 1];
        if (b > a) CK(cudaMemcpyAsync(dQ + a, q_bases_host + a, b - a, cudaMemcpyHostToDevice, pl->copy), "H2D Q");
        CK(cudaEventRecord(pl->ev_qc[j], pl->copy), "event");
    }
    CK(cudaEventRecord(pl->ev_q, pl->copy), "event");
    CK(cudaStreamWaitEvent(pl->stream, pl->ev_in, 0), "wait");
    if (!pl->exec || pl->inR != dR || pl->inQ != dQ) {
        CK(cudaStreamWaitEvent(pl->stream, pl->ev_q, 0), "wait");  // the measuring run reads both
        const gpumem_status st = pipeline_capture(pl, dR, dQ, true);
        if (st) return st;
    }
    CK(pipeline_launch(pl, true), "graph launch");
    note_launch(int(pl->launches));
    CK(cudaEventRecord(pl->ev_out, pl->stream), "event");
    CK(cudaStreamWaitEvent(pl->user, pl->ev_out, 0), "wait");
    pl->ran = 1;
    return GPUMEM_OK;
}

gpumem_status gpumem_pipeline_result(gpumem_pipeline *pl, const gpumem_triple **dev_ptr, uint64_t *count) {
    if (!pl || pl->magic != kMagicPipe) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    if (!pl->ran) return fail(GPUMEM_ERR_ARG, "gpumem_pipeline_run has not been called");
    CK(cudaStreamSynchronize(pl->stream), "pipeline sync");
    const unsigned long long *h = pl->host;
    if (h[8] != ~0ull) return fail(GPUMEM_ERR_ALPHABET, "R: byte at position %llu is not in {A,C,G,T,a,c,g,t}", h[8]);
    if (h[9] != ~0ull) return fail(GPUMEM_ERR_ALPHABET, "Q: byte at position %llu is not in {A,C,G,T,a,c,g,t}", h[9]);
    gpumem_find_stats fs{};
    fs.positions = pl->span;
    fs.occupied = h[3] + h[6];
    fs.hits = h[4] + h[5];
    fs.spilled_chunks = h[1] < pl->spill_cap ? h[1] : pl->spill_cap;
    fs.attempts = 1;
    fs.max_warp_hits = h[10];
    fs.warps = h[11];
    const gpumem_mems *res = pl->mems;
    uint64_t n = h[0];
    if (!pl->fallback && (h[0] > pl->out_cap || h[7] > pl->coop_cap)) {
        // output or coop queue overflow: the ordinary call (exact-capacity retry) on the
        // pipeline's packed sequences and index
        const gpumem_status st = gpumem_find_mems(pl->idx, pl->Q, pl->q_begin, pl->q_end, pl->stream, &pl->fallback);
        if (st) return st;
        fs.attempts = 2;
        CK(cudaEventRecord(pl->ev_out, pl->stream), "event");
        CK(cudaStreamWaitEvent(pl->user, pl->ev_out, 0), "wait");
    }
    if (pl->fallback) {
        res = pl->fallback;
        n = pl->fallback->count;
        fs = pl->fallback->stats;
        fs.attempts += 1;
    } else {
        pl->mems->count = n;
    }
    fs.mems = n;
    pl->stats = fs;
    if (dev_ptr) *dev_ptr = res->dev;
    if (count) *count = n;
    return GPUMEM_OK;
}

gpumem_status gpumem_pipeline_stats(const gpumem_pipeline *pl, gpumem_find_stats *out) {
    if (!pl || pl->magic != kMagicPipe || !out) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    *out = pl->stats;
    return GPUMEM_OK;
}

int gpumem_pipeline_profile(const gpumem_pipeline *pl, const char **names, double *ms, uint64_t *launches,
                            int max_stages) {
    if (!pl || pl->magic != kMagicPipe) return 0;
    int n = 0;
    for (auto &r : pl->recs) {
        float t = 0.f;
        cudaEventSynchronize(r.b);
        cudaEventElapsedTime(&t, r.a, r.b);
        int i = 0;
        for (; i < n; ++i)
            if (!strcmp(names[i], r.name)) break;
        if (i == n) {
            if (n >= max_stages) continue;
            names[n] = r.name;
            ms[n] = 0;
            launches[n] = 0;
            ++n;
        }
        ms[i] += t;
        launches[i] += r.l1 - r.l0;
    }
    cudaGetLastError();
    return n;
}

gpumem_status gpumem_pipeline_set_exportable(gpumem_pipeline *pl, int on) {
    if (!pl || pl->magic != kMagicPipe) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    if ((on != 0) != (pl->exportable != 0)) {
        CK(cudaStreamSynchronize(pl->stream), "sync");
        pipeline_release(pl);  // the next run recaptures into the other kind of arena
        pl->exportable = on != 0;
        pl->ran = 0;
    }
    return GPUMEM_OK;
}

gpumem_status gpumem_pipeline_export(const gpumem_pipeline *pl, gpumem_ipc_handle *handle, uint64_t *offset,
                                     uint64_t *generation) {
    if (!pl || pl->magic != kMagicPipe) return fail(GPUMEM_ERR_ARG, "not a gpumem_pipeline");
    if (!offset) return fail(GPUMEM_ERR_ARG, "offset is NULL");
    if (!pl->exportable) return fail(GPUMEM_ERR_ARG, "pipeline is not exportable (gpumem_pipeline_set_exportable)");
    if (!pl->exec || !pl->mems) return fail(GPUMEM_ERR_ARG, "pipeline has not run yet");
    static_assert(sizeof(cudaIpcMemHandle_t) <= sizeof(gpumem_ipc_handle), "IPC handle size");
    if (handle) {  // NULL: offset and generation only
        cudaIpcMemHandle_t h;
        CK(cudaIpcGetMemHandle(&h, pl->arena), "IPC handle");
        memset(handle, 0, sizeof *handle);
        memcpy(handle->bytes, &h, sizeof h);
    }
    *offset = uint64_t(reinterpret_cast<char *>(pl->mems->dev) - pl->arena);
    if (generation) *generation = pl->generation;
    return GPUMEM_OK;
}

gpumem_status gpumem_ipc_open(const gpumem_ipc_handle *handle, void **dev_base) {
    if (!handle || !dev_base) return fail(GPUMEM_ERR_ARG, "handle / dev_base is NULL");
    *dev_base = nullptr;
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle->bytes, sizeof h);
    CK(cudaIpcOpenMemHandle(dev_base, h, cudaIpcMemLazyEnablePeerAccess), "IPC open");
    return GPUMEM_OK;
}

gpumem_status gpumem_ipc_close(void *dev_base) {
    if (!dev_base) return GPUMEM_OK;
    CK(cudaIpcCloseMemHandle(dev_base), "IPC close");
    return GPUMEM_OK;
}

gpumem_status gpumem_rare(const gpumem_mems *m, uint32_t k, void *cuda_stream, gpumem_mems **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!m || m->magic != kMagicMems) return fail(GPUMEM_ERR_ARG, "not a gpumem_mems");
    if (k < 1 || k > uint32_t(kRareMaxK)) return fail(GPUMEM_ERR_ARG, "k = %u outside [1, %d]", k, kRareMaxK);
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    Stage g(k == 1 ? "mums" : "rare", s);
    Scratch sc(s);
    auto *res = static_cast<gpumem_triple *>(sc.get((m->count ? m->count : 1) * sizeof(gpumem_triple)));
    void *scratch = ws_get(kWsMums, rare_scratch_bytes(m->count), s);
    auto *dcount = static_cast<unsigned long long *>(ws_get(kWsCtr, 64, s));
    unsigned long long *h = pinned_slots();
    if (!res || !scratch || !dcount || !h) return GPUMEM_ERR_NOMEM;
    CK(rare_filter(m->dev, m->count, k, res, dcount, scratch, s), "rare filter");
    CK(cudaMemcpyAsync(h, dcount, 8, cudaMemcpyDeviceToHost, s), "D2H count");
    CK(cudaStreamSynchronize(s), "sync");
    sc.keep(res);
    *out = new gpumem_mems{kMagicMems, dev, s, h[0], res, m->stats};
    (*out)->stats.mems = h[0];
    return GPUMEM_OK;
}

gpumem_status gpumem_mums(const gpumem_mems *m, void *cuda_stream, gpumem_mems **out) {
    return gpumem_rare(m, 1, cuda_stream, out);
}

gpumem_status gpumem_split_masked(const gpumem_mems *m, const gpumem_fasta *R, const gpumem_fasta *Q, uint32_t L,
                                  int q_reverse, void *cuda_stream, gpumem_mems **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!m || m->magic != kMagicMems) return fail(GPUMEM_ERR_ARG, "not a gpumem_mems");
    if (!R || R->magic != kMagicFasta || !Q || Q->magic != kMagicFasta)
        return fail(GPUMEM_ERR_ARG, "R and Q must be gpumem_fasta handles");
    if (L < 1) return fail(GPUMEM_ERR_ARG, "min_len must be >= 1");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    Stage g("split", s);
    const uint64_t n = m->count, nQ = Q->seq.size();
    std::vector<uint64_t> mq = Q->mask;
    if (q_reverse) {  // the path ran on the reverse complement of the concatenated query
        const size_t k = mq.size() / 2;
        for (size_t j = 0; j < k; ++j) {
            mq[2 * j] = nQ - Q->mask[2 * (k - 1 - j) + 1];
            mq[2 * j + 1] = nQ - Q->mask[2 * (k - 1 - j)];
        }
    }
    const size_t mbytes = (R->mask.size() + mq.size() + 2) * 8;
    auto *dm = static_cast<uint64_t *>(ws_get(kWsFasta, mbytes, s));
    auto *cnt = static_cast<uint32_t *>(ws_get(kWsMergeK, (n + 1) * 8, s));
    auto *ctr = static_cast<unsigned long long *>(ws_get(kWsCtr, 64, s));
    unsigned long long *h = pinned_slots();
    if (!dm || !cnt || !ctr || !h) return GPUMEM_ERR_NOMEM;
    uint32_t *off = cnt + (n + 1);
    if (!R->mask.empty())
        CK(cudaMemcpyAsync(dm, R->mask.data(), R->mask.size() * 8, cudaMemcpyHostToDevice, s), "H2D masks");
    if (!mq.empty())
        CK(cudaMemcpyAsync(dm + R->mask.size(), mq.data(), mq.size() * 8, cudaMemcpyHostToDevice, s), "H2D masks");
    const uint32_t qbits = bits_for(nQ ? nQ : 1);
    const uint64_t nmr = R->mask.size() / 2, nmq = mq.size() / 2;
    CK(split_masked(m->dev, n, dm, nmr, dm + R->mask.size(), nmq, L, qbits, cnt, off, ctr, nullptr, nullptr, s),
       "split count");
    CK(cudaMemcpyAsync(h, ctr, 8, cudaMemcpyDeviceToHost, s), "D2H count");
    CK(cudaStreamSynchronize(s), "sync");
    const uint64_t total = h[0];
    auto *keys = static_cast<uint64_t *>(ws_get(kWsKeys, (total ? total : 1) * 8, s));
    auto *lens = static_cast<uint32_t *>(ws_get(kWsLens, (total ? total : 1) * 4, s));
    if (!keys || !lens) return GPUMEM_ERR_NOMEM;
    CK(split_masked(m->dev, n, dm, nmr, dm + R->mask.size(), nmq, L, qbits, cnt, off, ctr, keys, lens, s),
       "split emit");
    const uint32_t key_bits = bits_for(R->seq.size() ? R->seq.size() : 1) + qbits;
    st = sort_into_triples(keys, lens, total, key_bits, qbits, dev, s, out);
    if (st == GPUMEM_OK) (*out)->stats = m->stats, (*out)->stats.mems = total;
    return st;
}

gpumem_status gpumem_find_mems_banded(const char *r_bases_host, uint64_t r_len, const gpumem_seq *Q, uint32_t seed_len,
                                      uint32_t min_len, uint64_t band_len, void *cuda_stream, gpumem_mems **out,
                                      gpumem_band_stats *stats) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!r_bases_host && r_len) return fail(GPUMEM_ERR_ARG, "r_bases_host is NULL");
    if (!Q || Q->magic != kMagicSeq) return fail(GPUMEM_ERR_ARG, "Q is not a gpumem_seq");
    if (seed_len < 1 || seed_len > 15 || min_len < seed_len)
        return fail(GPUMEM_ERR_ARG, "need 1 <= seed_len <= 15 and seed_len <= min_len (got %u, %u)", seed_len, min_len);
    if (r_len >= (1ull << 32)) return fail(GPUMEM_ERR_RANGE, "sequences must be shorter than 2^32 bases");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    if (Q->device != dev) return fail(GPUMEM_ERR_ARG, "Q lives on another device");
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    const uint64_t step = min_len - seed_len + 1;
    if (band_len == 0 || band_len > r_len) band_len = r_len ? r_len : 1;
    band_len = (band_len + step - 1) / step * step;        // bands start on the sampling grid
    const uint64_t halo = min_len > 1024 ? min_len : 1024;  // >= L: a cut MEM is still reported
    uint64_t max_w = 0;
    for (uint64_t b0 = 0; b0 < r_len; b0 += band_len) {
        const uint64_t w0 = b0 >= step ? b0 - step : 0, b1 = min(b0 + band_len, r_len);
        max_w = max(max_w, min(b1 + halo, r_len) - w0);
    }
    Scratch sc(s);
    // two window buffers: the next band's window crosses PCIe on a copy stream while the
    // current band is searched (double buffering; full overlap needs pinned host memory)
    char *dwin[2] = {static_cast<char *>(sc.get(max_w ? max_w : 1)), static_cast<char *>(sc.get(max_w ? max_w : 1))};
    auto *ctr = static_cast<unsigned long long *>(sc.get(64));
    unsigned long long *h = pinned_slots();
    if (!dwin[0] || !dwin[1] || !ctr || !h) return GPUMEM_ERR_NOMEM;
    struct CopyLane {  // copy stream + "window copied" / "window consumed" events, released on exit
        cudaStream_t cs = nullptr;
        cudaEvent_t copied[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr};
        bool ok = true;
        CopyLane() {
            ok = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) == cudaSuccess;
            for (int i = 0; i < 2 && ok; ++i)
                ok = cudaEventCreateWithFlags(&copied[i], cudaEventDisableTiming) == cudaSuccess &&
                     cudaEventCreateWithFlags(&freed[i], cudaEventDisableTiming) == cudaSuccess;
        }
        ~CopyLane() {
            if (cs) cudaStreamSynchronize(cs);
            for (int i = 0; i < 2; ++i) {
                if (copied[i]) cudaEventDestroy(copied[i]);
                if (freed[i]) cudaEventDestroy(freed[i]);
            }
            if (cs) cudaStreamDestroy(cs);
        }
    } lane;
    if (!lane.ok) return cuda_fail(cudaGetLastError(), "band copy stream");
    auto window = [&](uint64_t b0, uint64_t &w0, uint64_t &w1) {
        const uint64_t b1 = min(b0 + band_len, r_len);
        w0 = b0 >= step ? b0 - step : 0;
        w1 = min(b1 + halo, r_len);
    };
    auto issue_copy = [&](uint64_t b0, int buf, bool wait_free) -> cudaError_t {
        uint64_t w0, w1;
        window(b0, w0, w1);
        cudaError_t e = wait_free ? cudaStreamWaitEvent(lane.cs, lane.freed[buf], 0) : cudaSuccess;
        if (e == cudaSuccess) e = cudaMemcpyAsync(dwin[buf], r_bases_host + w0, w1 - w0, cudaMemcpyHostToDevice, lane.cs);
        if (e == cudaSuccess) e = cudaEventRecord(lane.copied[buf], lane.cs);
        return e;
    };
    if (r_len && issue_copy(0, 0, false) != cudaSuccess) return cuda_fail(cudaGetLastError(), "H2D band window");
    std::vector<std::pair<gpumem_triple *, uint64_t>> chunks;  // closed MEMs per band (global r)
    gpumem_triple *open = nullptr;
    uint64_t n_open = 0, bands = 0, carried = 0;
    auto release = [&]() {
        for (auto &c : chunks) dfree(c.first, s);
        chunks.clear();
        if (open) dfree(open, s);
        open = nullptr;
    };
    for (uint64_t b0 = 0; b0 < r_len; b0 += band_len, ++bands) {
        const uint64_t b1 = min(b0 + band_len, r_len);
        const uint64_t w0 = b0 >= step ? b0 - step : 0, w1 = min(b1 + halo, r_len), wlen = w1 - w0;
        const int more = w1 < r_len ? 1 : 0;
        Stage g("band", s);
        const int buf = int(bands & 1);
        cudaError_t ce = cudaSuccess;
        if (b0 + band_len < r_len) ce = issue_copy(b0 + band_len, buf ^ 1, bands >= 1);  // the next window
        if (ce == cudaSuccess) ce = cudaStreamWaitEvent(s, lane.copied[buf], 0);
        if (ce != cudaSuccess) {
            release();
            return cuda_fail(ce, "H2D band window");
        }
        gpumem_seq *W = nullptr;
        gpumem_index *idx = nullptr;
        gpumem_mems *m = nullptr;
        st = gpumem_pack(dwin[buf], wlen, 1, s, &W);
        if (!st && cudaEventRecord(lane.freed[buf], s) != cudaSuccess) st = cuda_fail(cudaGetLastError(), "event");
        if (!st) st = gpumem_index_build_range(W, seed_len, min_len, b0 - w0, b1 - w0, s, &idx);
        if (!st) st = gpumem_find_mems(idx, Q, 0, UINT64_MAX, s, &m);
        const uint64_t cap = (m ? m->count : 0) + n_open;
        gpumem_triple *closed = st ? nullptr : static_cast<gpumem_triple *>(dalloc((cap ? cap : 1) * 12, s));
        gpumem_triple *open2 = st ? nullptr : static_cast<gpumem_triple *>(dalloc((cap ? cap : 1) * 12, s));
        if (!st && (!closed || !open2)) st = GPUMEM_ERR_NOMEM;
        cudaError_t e = cudaSuccess;
        if (!st) e = cudaMemsetAsync(ctr, 0, 16, s);
        if (!st && e == cudaSuccess)  // carried MEMs first: continue their right extension here
            e = band_continue(open, n_open, W->words, w0, wlen, more, Q->words, Q->n, closed, ctr, open2, ctr + 1, s);
        if (!st && e == cudaSuccess) e = band_place(m->dev, m->count, w0, wlen, more, closed, ctr, open2, ctr + 1, s);
        if (!st && e == cudaSuccess) e = cudaMemcpyAsync(h, ctr, 16, cudaMemcpyDeviceToHost, s);
        if (!st && e == cudaSuccess) e = cudaStreamSynchronize(s);
        for (void *x : {(void *)m, (void *)idx, (void *)W}) gpumem_free(x);
        if (!st && e != cudaSuccess) st = cuda_fail(e, "band");
        if (st) {
            if (closed) dfree(closed, s);
            if (open2) dfree(open2, s);
            release();
            return st;
        }
        carried += n_open;
        if (open) dfree(open, s);
        open = open2;
        n_open = h[1];
        chunks.push_back({closed, h[0]});
    }
    // every MEM is closed after the last band (no R follows it)
    uint64_t total = 0;
    for (auto &c : chunks) total += c.second;
    const uint32_t qbits = bits_for(Q->n ? Q->n : 1);
    auto *keys = static_cast<uint64_t *>(ws_get(kWsKeys, (total ? total : 1) * 8, s));
    auto *lens = static_cast<uint32_t *>(ws_get(kWsLens, (total ? total : 1) * 4, s));
    if (!keys || !lens) {
        release();
        return GPUMEM_ERR_NOMEM;
    }
    uint64_t off = 0;
    for (auto &c : chunks) {
        const cudaError_t e = launch_triples_to_keys(c.first, c.second, qbits, keys + off, lens + off, s);
        if (e != cudaSuccess) {
            release();
            return cuda_fail(e, "band keys");
        }
        off += c.second;
    }
    st = sort_into_triples(keys, lens, total, bits_for(r_len ? r_len : 1) + qbits, qbits, dev, s, out);
    release();
    if (st) return st;
    (*out)->stats.mems = total;
    if (stats) {
        stats->bands = bands;
        stats->band_len = band_len;
        stats->window_bytes = max_w;
        stats->carried = carried;
        stats->mems = total;
    }
    return GPUMEM_OK;
}

gpumem_status gpumem_mems_view(const gpumem_mems *m, const gpumem_triple **dev_ptr, uint64_t *count) {
    if (!m || m->magic != kMagicMems) return fail(GPUMEM_ERR_ARG, "not a gpumem_mems");
    if (dev_ptr) *dev_ptr = m->dev;
    if (count) *count = m->count;
    return GPUMEM_OK;
}

gpumem_status gpumem_mems_stats(const gpumem_mems *m, gpumem_find_stats *out) {
    if (!m || m->magic != kMagicMems) return fail(GPUMEM_ERR_ARG, "not a gpumem_mems");
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = m->stats;
    return GPUMEM_OK;
}

gpumem_status gpumem_mems_to_host(const gpumem_mems *m, gpumem_triple *host_buf, uint64_t capacity) {
    if (!m || m->magic != kMagicMems) return fail(GPUMEM_ERR_ARG, "not a gpumem_mems");
    if (capacity < m->count) return fail(GPUMEM_ERR_RANGE, "host buffer holds %llu < %llu triples",
                                         (unsigned long long)capacity, (unsigned long long)m->count);
    if (!m->count) return GPUMEM_OK;
    if (!host_buf) return fail(GPUMEM_ERR_ARG, "host_buf is NULL");
    CK(cudaMemcpyAsync(host_buf, m->dev, m->count * sizeof(gpumem_triple), cudaMemcpyDeviceToHost, m->stream),
       "D2H triples");
    CK(cudaStreamSynchronize(m->stream), "sync");
    return GPUMEM_OK;
}

gpumem_status gpumem_merge_sorted(const gpumem_triple *const *dev_runs, const uint64_t *counts, int n_runs,
                                  void *cuda_stream, gpumem_mems **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (n_runs < 0 || (n_runs > 0 && (!dev_runs || !counts))) return fail(GPUMEM_ERR_ARG, "bad runs");
    int dev;
    gpumem_status st = check_device(&dev);
    if (st) return st;
    cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
    if (n_runs > kMergeMaxRuns) return fail(GPUMEM_ERR_ARG, "at most %d runs (got %d)", kMergeMaxRuns, n_runs);
    uint64_t total = 0;
    for (int i = 0; i < n_runs; ++i) {
        if (counts[i] && !dev_runs[i]) return fail(GPUMEM_ERR_ARG, "run %d is NULL", i);
        if (counts[i] >= (1ull << 32)) return fail(GPUMEM_ERR_RANGE, "run %d holds 2^32 or more triples", i);
        total += counts[i];
    }
    Scratch sc(s);
    auto *trip = static_cast<gpumem_triple *>(sc.get((total ? total : 1) * sizeof(gpumem_triple)));
    void *scratch = ws_get(kWsMergeK, merge_scratch_bytes(n_runs > 0 ? n_runs : 1, total), s);
    if (!trip || !scratch) return GPUMEM_ERR_NOMEM;
    if (total) {
        Stage g("merge", s);
        CK(merge_runs(dev_runs, counts, n_runs, trip, scratch, s), "merge kernel");
    }
    sc.keep(trip);
    *out = new gpumem_mems{kMagicMems, dev, s, total, trip, gpumem_find_stats{}};
    (*out)->stats.mems = total;
    return GPUMEM_OK;
}

}  // extern "C"
