// find.cu -- K6/K7: seed lookup + bidirectional extension + canonical-seed
// duplicate elimination + compaction.
//
// Work decomposition (the tile scheduler, A6). The 2D search space (PAPER.md:78-80:
// R on one axis, Q on the other) is cut into query chunks of kChunk positions x
// the sampled-R hits of those positions. Every warp of a persistent grid is an
// independent worker: it grabs kGrab chunks at a time from an atomic counter and
// never waits on other warps (no CTA barriers). Per chunk:
//  stage   the chunk's packed Q words (+ halo) go to the warp's shared memory (loaded
//          into a register while the previous chunk was processed);
//  A5      each lane cuts kQPT consecutive seeds out of one 64-bit window, probes
//          the rank word of each seed (occupancy bit + running rank, 8 B per 32
//          seeds, 16 MB at ls = 13, L2-resident) and, for occupied seeds, reads
//          {first slot, count} of the bucket from the compact table -- the range
//          [ptrs[s], ptrs[s+1]). When that table is too large to stay
//          in L2 (many sampled seeds: C5 L = 20, 50) the index carries rank sectors
//          instead (16 B per 32 seeds: records and occupied seeds before the group +
//          a 2-bit saturating count per seed), which alone give {first, count}
//          unless a count in the group up to the seed saturates; only then is the
//          compact table read. use_bitmap = 0 reads the dense ptrs. Buckets of
//          more than spill_t hits are cut into kSpillHits-hit pieces and pushed to
//          a global queue drained by k_heavy (reference-axis tiles of the hot
//          seeds, Fig. 6 :268-270); the rest become (q, bucket) entries with a
//          warp-scanned prefix of their hit counts;
//  A6      the chunk's hits are dealt 32 at a time to the lanes (hit h -> its entry
//          from an OR-reduction of the entry starts inside the round), replacing
//          Alg. 2's proactive load balancing (:120-149) and Alg. 3's combine
//          (:155-169);
//  A7      left extension capped at step. The seed record carries the 16 bases
//          left of p and the 32 bases right of the seed (index.cu), so a random
//          hit is decided without touching R. e == step means the sampled seed at
//          p - step is on the same diagonal inside the same match, and that hit
//          owns the MEM: drop. Exactly one sampled seed per MEM has e < step
//          (DESIGN.md "canonical seed"): each MEM is emitted once (:153);
//  A8      right extension from the seed's end to the first mismatch or end;
//  A9      keep len = e + ls + f >= L (:53-56), maximal by construction;
//  A10     ballot/popc into a per-warp shared buffer, flushed 32+ at a time with
//          one atomicAdd; writes past `capacity` are counted, not stored.
// Extensions past the record run per lane up to kLaneCap bases; longer ones (R == Q,
// long repeats) are queued and finished by k_coop with the whole warp, 1024 bases
// per step, so no single lane walks a megabase-long match.
// Compares are 2-bit packed words: XOR, then clz (rightwards) / ffs (leftwards)
// finds the first mismatching base exactly (reading R11).
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;                   // threads per CTA
constexpr int kWarps = kT / 32;
#ifndef GM_FIND_QPT
#define GM_FIND_QPT 8
#endif
constexpr int kQPT = GM_FIND_QPT;         // query positions per lane per chunk
constexpr int kChunk = 32 * kQPT;         // 256 positions per warp chunk
#ifndef GM_HEAVY_CTAS
#define GM_HEAVY_CTAS 8  // k_heavy CTAs per SM (8 vs 4: C5 L = 20 0.517 vs 0.536 ms)
#endif
#ifndef GM_FIND_GRAB
#define GM_FIND_GRAB 2
#endif
constexpr uint32_t kGrab = GM_FIND_GRAB;  // chunks per scheduler grab
constexpr int kQW = kChunk / 32 + 6;      // staged Q words (chunk + left/right halo)
constexpr uint32_t kSpillHits = 32;       // hits per heavy-queue piece (one per lane)
constexpr int kOutBuf = 64;
constexpr uint32_t kUnresolved = 0xffffffffu;
constexpr uint32_t kLaneCap = 4096;       // bases one lane extends before the warp takes over

constexpr int kDQ = 64;                   // deferred-extension queue entries per warp

// per-warp shared memory of k_find for chunks of kC query positions (sized to the chunk:
// shared memory the kernel does not need is L1 its record and window loads rely on)
template <int kC>
struct WarpSmemT {
    uint4 dq[kDQ];                        // {p, q, e (or kUnresolved), known right}: hits needing global extension
    uint64_t qw[kC / 32 + 6];
    uint32_t e_beg[kC];
    uint32_t e_off[kC + 1];
    uint64_t okey[kOutBuf];
    uint32_t olen[kOutBuf];
    uint8_t e_q[kC];
};

// k_heavy / k_coop: only the output buffer of warp_emit
struct EmitSmem {
    uint64_t okey[kOutBuf];
    uint32_t olen[kOutBuf];
};

// staged Q: word i of the smem copy is Q word (wbase + i)
struct QStage {
    const uint64_t *w;
    uint32_t wbase;
    __device__ __forceinline__ uint64_t fwd(uint32_t x) const {  // bases [x, x+32)
        const uint32_t i = (x >> 5) - wbase;
        const uint32_t sh = (x & 31) * 2;
        const uint64_t a = w[i];
        return sh ? (a << sh) | (w[i + 1] >> (64 - sh)) : a;
    }
    __device__ __forceinline__ uint32_t back16(uint32_t x) const {  // bases [x-16, x), base x-1 lowest
        if (x >= 32) return uint32_t(fwd(x - 32));
        return x ? uint32_t(w[0] >> (64 - 2 * x)) : 0u;  // x < 32 implies wbase == 0
    }
};

struct Hit {
    uint64_t key;
    uint32_t len;
};

enum : int { kDrop = 0, kDefer = 1, kEmit = 2 };

// Extension rounds: kRW consecutive 32-base windows per round, so a round loads kRW + 1
// words of each sequence at once (independent loads, one memory latency) instead of one
// dependent pair of loads per 32 bases. The first mismatching window decides.
#ifndef GM_KRW
#define GM_KRW 2
#endif
constexpr int kRW = GM_KRW;

__device__ __forceinline__ uint64_t funnel(uint64_t hi, uint64_t lo, uint32_t sh) {  // sh even, 0..62
    return (hi << sh) | ((lo >> 1) >> (63 - sh));
}

// Equal bases of R[a + f ..) and Q[b + f ..), the first f known equal; clamped to lim.
// kUnresolved when the run passes `cap` (the lane hands it to the warp).
__device__ __forceinline__ uint32_t ext_right(const uint64_t *__restrict__ R, const uint64_t *__restrict__ Q,
                                              uint64_t a, uint64_t b, uint32_t f, uint32_t lim, uint32_t cap) {
    while (f < lim) {
        if (f >= cap) return kUnresolved;
        const uint64_t x = a + f, y = b + f;  // x < |R|, y < |Q|: words x/32 + kRW are padding at worst
        const uint64_t *pr = R + (x >> 5), *pq = Q + (y >> 5);
        const uint32_t sr = uint32_t(x & 31) * 2, sq = uint32_t(y & 31) * 2;
        uint64_t wr[kRW + 1], wq[kRW + 1];
#pragma unroll
        for (int k = 0; k <= kRW; ++k) {
            wr[k] = __ldg(pr + k);
            wq[k] = __ldg(pq + k);
        }
        uint32_t run = 32 * kRW;
#pragma unroll
        for (int k = kRW - 1; k >= 0; --k) {  // nearest mismatching window assigned last
            const uint64_t d = funnel(wr[k], wr[k + 1], sr) ^ funnel(wq[k], wq[k + 1], sq);
            if (d) run = 32u * k + (uint32_t(__clzll(d)) >> 1);
        }
        f += run;
        if (run < 32 * kRW) break;
    }
    return min(f, lim);
}

// Equal bases leftwards of the exclusive ends a - e (R) and b - e (Q), the first e known
// equal; clamped to lim (lim <= min(a, b), so no base before 0 is ever counted).
__device__ __forceinline__ uint32_t ext_left(const uint64_t *__restrict__ R, const uint64_t *__restrict__ Q,
                                             uint64_t a, uint64_t b, uint32_t e, uint32_t lim, uint32_t cap) {
    while (e < lim) {
        if (e >= cap) return kUnresolved;
        const uint64_t x = a - e, y = b - e;
        uint32_t run;
        if (x >= 32 * kRW && y >= 32 * kRW) {
            const uint64_t xs = x - 32 * kRW, ys = y - 32 * kRW;  // window k covers [xs + 32k, xs + 32k + 32)
            const uint64_t *pr = R + (xs >> 5), *pq = Q + (ys >> 5);
            const uint32_t sr = uint32_t(xs & 31) * 2, sq = uint32_t(ys & 31) * 2;
            uint64_t wr[kRW + 1], wq[kRW + 1];
#pragma unroll
            for (int k = 0; k <= kRW; ++k) {
                wr[k] = __ldg(pr + k);
                wq[k] = __ldg(pq + k);
            }
            run = 32 * kRW;
#pragma unroll
            for (int k = 0; k < kRW; ++k) {  // nearest (k = kRW - 1) mismatching window assigned last
                const uint64_t d = funnel(wr[k], wr[k + 1], sr) ^ funnel(wq[k], wq[k + 1], sq);
                if (d) run = 32u * (kRW - 1 - k) + ((uint32_t(__ffsll(d)) - 1) >> 1);
            }
            e += run;
            if (run < 32 * kRW) break;
        } else {  // near the start of R or Q: one window at a time (zero-filled before 0)
            run = trail_eq(win_back(R, x) ^ win_back(Q, y));
            e += run;
            if (run < 32) break;
        }
    }
    return min(e, lim);
}

// Streamed query (host-input pipeline, Q arriving in chunks): extensions stop at the
// end of the query data present, q_avail. A match whose right extension was cut there
// (more of Q follows, R does not end at the same point) is emitted with kOpenBit set in
// its length and finished by k_open_fix once all of Q is present. Its length is already
// >= L: its start lies a whole chunk (>= L bases) before q_avail.
constexpr uint32_t kOpenBit = 0x80000000u;
__device__ __forceinline__ uint32_t open_bit(const FindParams &P, uint32_t a, uint32_t b, uint32_t f) {
    return (uint64_t(b) + f == P.q_avail && P.q_avail < P.nQ && uint64_t(a) + f < P.nR) ? kOpenBit : 0u;
}

// The record-only part of decide(): kDrop / kEmit when the kL + kR flank bases of the
// record (16 + 32 for 16-byte records, 8 + 8 for 8-byte records) settle the hit, else
// kExt with e_out = the left extension if the record settled it, or kUnresolved. kExt
// hits are queued per warp and finished 32 at a time by decide_deferred(), so the
// (rare, long) global-memory extensions run with all lanes busy instead of stalling a
// whole warp round for one lane.
enum : int { kExt = 3 };
template <int kL, int kR>
__device__ __forceinline__ int decide_rec(const FindParams &P, uint32_t p, uint32_t rleft, uint64_t rright,
                                          uint32_t q, uint32_t qleft, uint64_t qright, Hit &out, uint32_t &e_out,
                                          uint32_t &f_out) {
    const uint32_t lim = min(P.step, min(p, q));
    const uint32_t lmask = kL >= 16 ? 0xffffffffu : ((1u << (2 * kL)) - 1u);  // kL bases, base p-1 lowest
    const uint32_t xl = (rleft ^ qleft) & lmask;
    uint32_t e = xl ? uint32_t(__ffs(int(xl)) - 1) >> 1 : uint32_t(kL);
    if (e == kL && lim > kL) {
        e_out = kUnresolved;
        f_out = 0;
        return kExt;
    }
    e = min(e, lim);
    if (e == P.step) return kDrop;
    const uint32_t qs = q - e;
    if (qs < P.own_lo || qs >= P.own_hi) return kDrop;
    const uint32_t a = p + P.ls, b = q + P.ls;
    const uint32_t lim_r = min(uint32_t(P.nR) - a, uint32_t(P.q_avail) - b);
    const uint64_t rmask = kR >= 32 ? ~0ull : ~(~0ull >> (2 * kR));  // kR bases, first base highest
    const uint64_t xr = (rright ^ qright) & rmask;
    uint32_t f = xr ? uint32_t(__clzll(xr)) >> 1 : uint32_t(kR);
    if (f == kR && lim_r > kR) {
        e_out = e;
        f_out = kR;  // the record's right flank matched: the global extension starts past it
        return kExt;
    }
    f = min(f, lim_r);
    const uint32_t lam = e + P.ls + f;
    if (lam < P.L) return kDrop;
    out.key = (uint64_t(p - e) << P.qbits) | qs;
    out.len = lam | open_bit(P, a, b, f);
    return kEmit;
}

// The rest of decide() for a queued hit, from global memory (kL left bases already known
// equal when e_in == kUnresolved; f0 right bases known equal).
template <int kL>
__device__ __forceinline__ int decide_deferred(const FindParams &P, uint32_t p, uint32_t q, uint32_t e_in, uint32_t f0,
                                               Hit &out) {
    const uint32_t lim = min(P.step, min(p, q));
    uint32_t e = e_in;
    if (e == kUnresolved) {
        e = ext_left(P.R, P.Q, p, q, kL, lim, kLaneCap);
        if (e == kUnresolved) return kDefer;
    }
    e = min(e, lim);
    if (e == P.step) return kDrop;
    const uint32_t qs = q - e;
    if (qs < P.own_lo || qs >= P.own_hi) return kDrop;
    const uint32_t a = p + P.ls, b = q + P.ls;
    const uint32_t lim_r = min(uint32_t(P.nR) - a, uint32_t(P.q_avail) - b);
    uint32_t f = ext_right(P.R, P.Q, a, b, f0, lim_r, kLaneCap);
    if (f == kUnresolved) return kDefer;
    const uint32_t lam = e + P.ls + f;
    if (lam < P.L) return kDrop;
    out.key = (uint64_t(p - e) << P.qbits) | qs;
    out.len = lam | open_bit(P, a, b, f);
    return kEmit;
}

// Warp-cooperative extensions (uniform arguments): lane i compares the i-th 32-base
// window, 1024 bases per step; the first mismatching window decides.
__device__ __forceinline__ uint32_t warp_ext_right(const FindParams &P, uint64_t a, uint64_t b, uint32_t f,
                                                   uint32_t lim) {
    const int lane = threadIdx.x & 31;
    while (f < lim) {
        const uint32_t o = f + 32u * lane;
        const bool in = o < lim;
        const uint64_t x = in ? (win_fwd(P.R, a + o) ^ win_fwd(P.Q, b + o)) : 0ull;
        const unsigned bad = __ballot_sync(0xffffffffu, !in || x != 0);
        if (bad) {
            const int first = __ffs(int(bad)) - 1;
            const uint32_t run = __shfl_sync(0xffffffffu, in ? lead_eq(x) : 0u, first);
            return min(f + 32u * first + run, lim);
        }
        f += 1024;
    }
    return min(f, lim);
}

__device__ __forceinline__ uint32_t warp_ext_left(const FindParams &P, uint64_t a, uint64_t b, uint32_t e,
                                                  uint32_t lim) {
    const int lane = threadIdx.x & 31;
    while (e < lim) {
        const uint32_t o = e + 32u * lane;
        const bool in = o < lim;
        const uint64_t x = in ? (win_back(P.R, a - o) ^ win_back(P.Q, b - o)) : 0ull;
        const unsigned bad = __ballot_sync(0xffffffffu, !in || x != 0);
        if (bad) {
            const int first = __ffs(int(bad)) - 1;
            const uint32_t run = __shfl_sync(0xffffffffu, in ? trail_eq(x) : 0u, first);
            return min(e + 32u * first + run, lim);
        }
        e += 1024;
    }
    return min(e, lim);
}

// Resolve deferred hits, one per lane (all 32 lanes call it; `valid` marks real ones):
// the full decision again from global windows, per lane up to kLaneCap bases per
// direction, longer extensions handed to the whole warp.
__device__ __forceinline__ bool resolve_deferred(const FindParams &P, bool valid, uint32_t p, uint32_t q,
                                              uint32_t es, Hit &out) {
    // ---- left
    const uint32_t lim = valid ? min(P.step, min(p, q)) : 0u;
    uint32_t e = 0;
    bool need = false;
    if (valid) {
        if (es == kUnresolved) {
            e = 0;  // recomputed from the sequences (rare path)
            const uint32_t cap = min(lim, kLaneCap);
            bool done = false;
            while (e < cap) {
                const uint32_t run = trail_eq(win_back(P.R, p - e) ^ win_back(P.Q, q - e));
                e += run;
                if (run < 32) {
                    done = true;
                    break;
                }
            }
            need = !done && e < lim;
        } else {
            e = es;
        }
    }
    for (unsigned m = __ballot_sync(0xffffffffu, need); m; m &= m - 1) {
        const int src = __ffs(int(m)) - 1;
        const uint32_t sp = __shfl_sync(0xffffffffu, p, src), sq = __shfl_sync(0xffffffffu, q, src);
        const uint32_t se = __shfl_sync(0xffffffffu, e, src), sl = __shfl_sync(0xffffffffu, lim, src);
        const uint32_t r = warp_ext_left(P, sp, sq, se, sl);
        if (lane_id() == src) e = r;
    }
    e = min(e, lim);
    bool alive = valid && e != P.step;
    const uint32_t qs = q - e;
    alive = alive && qs >= P.own_lo && qs < P.own_hi;
    // ---- right
    const uint32_t a = p + P.ls, b = q + P.ls;
    const uint32_t lim_r = alive ? min(uint32_t(P.nR) - a, uint32_t(P.q_avail) - b) : 0u;
    uint32_t f = 0;
    need = false;
    if (alive) {
        const uint32_t cap = min(lim_r, kLaneCap);
        bool done = false;
        while (f < cap) {
            const uint32_t run = lead_eq(win_fwd(P.R, uint64_t(a) + f) ^ win_fwd(P.Q, uint64_t(b) + f));
            f += run;
            if (run < 32) {
                done = true;
                break;
            }
        }
        need = !done && f < lim_r;
    }
    for (unsigned m = __ballot_sync(0xffffffffu, need); m; m &= m - 1) {
        const int src = __ffs(int(m)) - 1;
        const uint32_t sa = __shfl_sync(0xffffffffu, a, src), sb = __shfl_sync(0xffffffffu, b, src);
        const uint32_t sf = __shfl_sync(0xffffffffu, f, src), sl = __shfl_sync(0xffffffffu, lim_r, src);
        const uint32_t r = warp_ext_right(P, sa, sb, sf, sl);
        if (lane_id() == src) f = r;
    }
    f = min(f, lim_r);
    const uint32_t lam = e + P.ls + f;
    if (!alive || lam < P.L) return false;
    out.key = (uint64_t(p - e) << P.qbits) | qs;
    out.len = lam | open_bit(P, a, b, f);
    return true;
}

// Deferred hits (extension longer than kLaneCap) go to the coop queue, drained by
// k_coop after the find kernels; rare, so one atomic per hit is fine.
__device__ __forceinline__ void push_coop(const FindParams &P, int &verdict, uint32_t p, uint32_t q) {
    if (verdict != kDefer) return;
    verdict = kDrop;
    const unsigned long long slot = atomicAdd(P.coop_count, 1ull);
    if (slot < P.coop_cap) P.coopq[slot] = make_uint2(p, q);
}

// A10: warp-aggregated append into the warp's buffer; flush when >= 32 are pending.
template <class WarpSmem>
__device__ __forceinline__ void warp_emit(const FindParams &P, WarpSmem &s, uint32_t &nbuf, bool emit,
                                          const Hit &h, bool force_flush) {
    const int lane = threadIdx.x & 31;
    const unsigned bal = __ballot_sync(0xffffffffu, emit);
    if (emit) {
        const uint32_t pos = nbuf + __popc(bal & lanemask_lt());
        s.okey[pos] = h.key;
        s.olen[pos] = h.len;
    }
    nbuf += __popc(bal);
    if (nbuf >= 32 || (force_flush && nbuf)) {
        __syncwarp();
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(P.out_count, (unsigned long long)nbuf);
        base = __shfl_sync(0xffffffffu, base, 0);
        for (uint32_t i = lane; i < nbuf; i += 32) {
            if (base + i < P.capacity) {
                P.out_key[base + i] = s.okey[i];
                P.out_len[base + i] = s.olen[i];
            }
        }
        __syncwarp();
        nbuf = 0;
    }
}

// Seed record k: 16-byte {p, R[p-16, p), R[p+ls, p+ls+32)} or, for 8-byte records,
// {p, R[p-8, p) | R[p+ls, p+ls+8) << 16}; left flank base p-1 lowest, right flank first
// base highest (the layout decide_rec<kL, kR> expects).
template <bool kRec8>
__device__ __forceinline__ void load_rec(const FindParams &P, uint64_t k, uint32_t &p, uint32_t &left,
                                         uint64_t &right, int stream) {
    if (kRec8) {
        const uint2 *r8 = reinterpret_cast<const uint2 *>(P.recs);
        const uint2 r = stream < 0 ? __ldg(r8 + k) : ld_hint_u2(r8 + k, stream != 0);
        p = r.x;
        left = r.y & 0xffffu;
        right = uint64_t(r.y >> 16) << 48;
    } else {
        const uint4 *r16 = reinterpret_cast<const uint4 *>(P.recs);
        const uint4 r = stream < 0 ? __ldg(r16 + k) : ld_hint_u4(r16 + k, stream != 0);
        p = r.x;
        left = r.y;
        right = (uint64_t(r.w) << 32) | r.z;
    }
}

// One converged extension round: the last `take` (<= 32) queued hits, one per lane.
template <int kL, class WarpSmem>
__device__ __forceinline__ void drain_deferred(const FindParams &P, WarpSmem &s, uint32_t &nq, uint32_t &nbuf,
                                               uint32_t take) {
    const int lane = threadIdx.x & 31;
    int verdict = kDrop;
    Hit out{0, 0};
    uint32_t p = 0, q = 0;
    if (uint32_t(lane) < take) {
        const uint4 d = s.dq[nq - take + lane];
        p = d.x;
        q = d.y;
        verdict = decide_deferred<kL>(P, p, q, d.z, d.w, out);
    }
    __syncwarp();
    nq -= take;
    push_coop(P, verdict, p, q);
    warp_emit(P, s, nbuf, verdict == kEmit, out, false);
}

#ifndef GM_FIND_MINB
#define GM_FIND_MINB 4
#endif
#ifndef GM_FIND_MINB_SECT
#define GM_FIND_MINB_SECT 6
#endif
#ifndef GM_FIND_QPT_SECT
#define GM_FIND_QPT_SECT 4
#endif
// Rank-sector indexes (large: C5 at L = 20, 50) run 4 positions per lane and 6 CTAs per SM
// (their find is DRAM-bound: more warps in flight, C5 L = 20 2.66 -> 2.53 ms); rank-word
// indexes 8 positions per lane and 4 CTAs per SM (probe pairs; C4 0.78 vs 0.81 ms).
template <bool kSect>
struct FindShape {
    static constexpr int kQPT = kSect ? GM_FIND_QPT_SECT : GM_FIND_QPT;
    static constexpr int kChunk = 32 * kQPT;
    static constexpr int kQW = kChunk / 32 + 6;
    static constexpr int kMinB = kSect ? GM_FIND_MINB_SECT : GM_FIND_MINB;
};
static_assert(FindShape<true>::kChunk <= 256 && FindShape<false>::kChunk <= 256, "e_q holds 8-bit slots");

template <bool kStatic, bool kHints, bool kSect, bool kRec8>
__global__ void __launch_bounds__(kT, FindShape<kSect>::kMinB) k_find(const FindParams P) {
    pdl_wait();
    constexpr int kQPT = FindShape<kSect>::kQPT, kChunk = FindShape<kSect>::kChunk, kQW = FindShape<kSect>::kQW;
    using WarpSmem = WarpSmemT<kChunk>;
    constexpr int kL = kRec8 ? 8 : 16, kR = kRec8 ? 8 : 32;  // record flank widths (bases)
    __shared__ WarpSmem smem[kWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    WarpSmem &s = smem[wid];
    const uint32_t sh = 64 - 2 * P.ls;
    uint32_t nbuf = 0, nq = 0;
    unsigned long long st_e = 0, st_h = 0;
    QStage qs{s.qw, 0};
    const uint32_t hvn = P.hv_n ? *P.hv_n : 0u;  // heavy buckets with a minority prefix
    // L2 priorities: lookup tables stay, streamed data goes first (records only when
    // they cannot stay resident anyway, P.recs_stream)

    // chunks in scheduler order; the next chunk (and, at a grab's end, the next grab) is
    // claimed and its packed Q words loaded into a register before the current chunk is
    // processed, so that load's latency hides behind the current chunk's work
    auto grab_next = [&](uint64_t &c, uint64_t &c_end) {
        uint32_t g = 0;
        if (lane == 0) g = atomicAdd(P.tile_ctr, 1u);
        g = __shfl_sync(0xffffffffu, g, 0);
        c = uint64_t(g) * kGrab;
        c_end = min(c + kGrab, P.n_tiles);
    };
    auto q_words = [&](uint64_t c) -> uint64_t {  // lane's staged word of chunk c
        const uint32_t q0 = uint32_t(P.scan_lo + c * kChunk);
        const uint32_t wb = (q0 >> 5) ? (q0 >> 5) - 1 : 0;
        if (lane >= kQW || wb + lane >= P.nQw) return 0ull;
        return kHints ? ld_first_u64(reinterpret_cast<const unsigned long long *>(P.Q) + wb + lane)
                      : __ldg(P.Q + wb + lane);
    };
    uint64_t c, c_end;
    grab_next(c, c_end);
    uint64_t qpre = c < P.n_tiles ? q_words(c) : 0ull;
    while (c < P.n_tiles) {
        uint64_t cn = c + 1, cn_end = c_end;
        if (cn >= c_end) grab_next(cn, cn_end);
        {
            const uint32_t q0 = uint32_t(P.scan_lo + c * kChunk);
            // ---- stage the chunk's Q words (+ halo) in shared memory
            const uint32_t wb = (q0 >> 5) ? (q0 >> 5) - 1 : 0;
            qs.wbase = wb;
            if (lane < kQW) s.qw[lane] = qpre;
            __syncwarp();
            qpre = cn < P.n_tiles ? q_words(cn) : 0ull;  // the next chunk's words, in flight

            // ---- A5: seeds -> bitmap -> bucket ranges
            uint32_t beg[kQPT], cnt[kQPT];
            const uint32_t qa = q0 + uint32_t(lane) * kQPT;
#pragma unroll
            for (int j = 0; j < kQPT; ++j) beg[j] = cnt[j] = 0;
            if (qa < P.scan_hi) {
                const uint64_t win = qs.fwd(qa);
                uint32_t code[kQPT];
                bool occ[kQPT];
#pragma unroll
                for (int j = 0; j < kQPT; ++j) {
                    code[j] = uint32_t((win << (2 * j)) >> sh);
                    occ[j] = qa + j < P.scan_hi;
                }
                if (P.use_bitmap && !kSect) {
                    // rank-word probes in pairs (q, q+1): one 16-byte entry of group code(q+1) >> 5
                    // holds q+1's rank word and the occupancy of the rotated code of q (same
                    // group, index.cu); q's own rank word only when it is occupied. Then the
                    // compact {first, count} of each occupied seed.
                    const uint32_t nbits = 2 * P.ls;
                    const uint32_t cmask = nbits >= 32 ? 0xffffffffu : ((1u << nbits) - 1u);
                    uint32_t rank[kQPT];
                    bool own[kQPT];  // rank word of the position's own group still needed
#pragma unroll
                    for (int j = 0; j < kQPT; j += 2) {
                        rank[j] = rank[j + 1] = 0;
                        own[j] = false;
                        own[j + 1] = false;
                        if (occ[j + 1]) {  // both positions in range
                            const uint4 *ep = reinterpret_cast<const uint4 *>(P.rankw + 2 * (code[j + 1] >> 5));
                            const uint4 e = kHints ? ld_last_u4(ep) : __ldg(ep);
                            const uint32_t b1 = code[j + 1] & 31;
                            occ[j + 1] = (e.x >> b1) & 1u;
                            rank[j + 1] = e.y + __popc(e.x & ((1u << b1) - 1u));
                            const uint32_t rot = ((code[j] << 2) | (code[j] >> (nbits - 2))) & cmask;
                            occ[j] = (e.z >> (rot & 31)) & 1u;
                            own[j] = occ[j];
                        } else if (occ[j]) {
                            own[j] = true;
                        }
                    }
#pragma unroll
                    for (int j = 0; j < kQPT; j += 2) {
                        if (own[j]) {
                            const unsigned long long rw = kHints ? ld_last_u64(P.rankw + 2 * (code[j] >> 5))
                                                                 : __ldg(P.rankw + 2 * (code[j] >> 5));
                            const uint32_t bit = code[j] & 31, bits = uint32_t(rw);
                            occ[j] = (bits >> bit) & 1u;
                            rank[j] = uint32_t(rw >> 32) + __popc(bits & ((1u << bit) - 1u));
                        }
                    }
#pragma unroll
                    for (int j = 0; j < kQPT; ++j) {
                        if (occ[j]) {
                            const uint2 b = kHints ? ld_last_u2(P.buckets + rank[j]) : __ldg(P.buckets + rank[j]);
                            beg[j] = b.x;
                            cnt[j] = b.y;
                        }
                    }
                } else if (P.use_bitmap) {
                    // rank-sector probe: {records before the group, occupied seeds before
                    // the group, 2-bit saturating count per seed}. Counts <= 2 all the way
                    // up to the seed give {first, count} directly; otherwise the compact
                    // {first, count} table is read at the seed's rank.
                    uint32_t rank[kQPT];
                    bool need[kQPT];
#pragma unroll
                    for (int j = 0; j < kQPT; ++j) {
                        need[j] = false;
                        rank[j] = 0;
                        if (occ[j]) {
                            const uint4 rs = kHints ? ld_last_u4(P.rsect + (code[j] >> 5)) : __ldg(P.rsect + (code[j] >> 5));
                            const uint32_t b = code[j] & 31;
                            const uint64_t c2 = (uint64_t(rs.w) << 32) | rs.z;
                            const uint32_t f = uint32_t(c2 >> (2 * b)) & 3u;
                            const uint64_t below = c2 & ((1ull << (2 * b)) - 1ull);
                            constexpr uint64_t kLo = 0x5555555555555555ull;
                            occ[j] = f != 0;
                            need[j] = f != 0 && (f == 3u || (below & (below >> 1) & kLo) != 0);
                            beg[j] = rs.x + __popcll(below & kLo) + 2 * __popcll(below & ~kLo);
                            cnt[j] = occ[j] ? f : 0u;
                            rank[j] = rs.y + __popcll((below | (below >> 1)) & kLo);
                        }
                    }
#pragma unroll
                    for (int j = 0; j < kQPT; ++j) {
                        if (need[j]) {
                            const uint2 b = kHints ? ld_last_u2(P.buckets + rank[j]) : __ldg(P.buckets + rank[j]);
                            beg[j] = b.x;
                            cnt[j] = b.y;
                        }
                    }
                } else {  // the paper's lookup: ptrs[s], ptrs[s+1]
#pragma unroll
                    for (int j = 0; j < kQPT; ++j) {
                        if (occ[j]) {
                            beg[j] = __ldg(P.ptrs + code[j]);
                            cnt[j] = __ldg(P.ptrs + code[j] + 1) - beg[j];
                        }
                    }
                }
#pragma unroll
                for (int j = 0; j < kQPT; ++j) {
                    if (cnt[j] > P.spill_t) {  // heavy bucket -> reference-axis pieces on the queue
                        // a bucket reordered minority-left-flank first (index.cu, k_hv_part): a
                        // query position with the majority flank spills only the minority
                        // (the others are non-canonical: equal flanks over >= step bases)
                        uint32_t ncnt = cnt[j];
                        if (hvn && qa + j >= P.step) {
                            uint32_t lo2 = 0, hi2 = hvn;
                            while (lo2 < hi2) {
                                const uint32_t mid = (lo2 + hi2) >> 1;
                                if (__ldg(&P.hv_info[mid].x) < beg[j]) lo2 = mid + 1; else hi2 = mid;
                            }
                            if (lo2 < hvn) {
                                const uint4 hv = __ldg(P.hv_info + lo2);
                                constexpr uint32_t lmask = kL >= 16 ? 0xffffffffu : ((1u << (2 * kL)) - 1u);
                                if (hv.x == beg[j] && (qs.back16(qa + j) & lmask) == hv.z) ncnt = hv.w;
                            }
                        }
                        GM_CHECK(ncnt <= cnt[j]);
                        if (ncnt == 0) {  // every location of the bucket is non-canonical here
                            atomicAdd(&P.stats[2], (unsigned long long)cnt[j]);  // hits (decided here)
                            atomicAdd(&P.stats[3], 1ull);
                            cnt[j] = 0;
                            continue;
                        }
                        const uint32_t npc = (ncnt + kSpillHits - 1) / kSpillHits;
                        const unsigned long long slot = atomicAdd(P.spill_count, (unsigned long long)npc);
                        if (slot + npc <= P.spill_cap) {
                            for (uint32_t c2 = 0; c2 < npc; ++c2) {
                                const uint32_t off = c2 * kSpillHits;
                                P.spill[slot + c2] = make_uint4(qa + j, beg[j] + off, min(kSpillHits, ncnt - off), 0u);
                            }
                            atomicAdd(&P.stats[2], (unsigned long long)cnt[j]);  // hits: the skipped majority
                            atomicAdd(&P.stats[3], 1ull);                          // is decided here too
                            cnt[j] = 0;
                        } else {
                            for (unsigned long long s2 = slot; s2 < P.spill_cap; ++s2)
                                P.spill[s2] = make_uint4(0u, 0u, 0u, 0u);  // neutralised; processed here
                        }
                    }
                }
            }
            uint32_t n_e = 0, n_h = 0;
#pragma unroll
            for (int j = 0; j < kQPT; ++j) {
                n_e += cnt[j] ? 1u : 0u;
                n_h += cnt[j];
            }
            uint32_t ie = n_e, ih = n_h;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t a = __shfl_up_sync(0xffffffffu, ie, o);
                const uint32_t b = __shfl_up_sync(0xffffffffu, ih, o);
                if (lane >= o) {
                    ie += a;
                    ih += b;
                }
            }
            const uint32_t E = __shfl_sync(0xffffffffu, ie, 31);
            const uint32_t H = __shfl_sync(0xffffffffu, ih, 31);
            if (H) {
                uint32_t pe = ie - n_e, ph = ih - n_h;
#pragma unroll
                for (int j = 0; j < kQPT; ++j) {
                    if (cnt[j]) {
                        s.e_q[pe] = uint8_t(lane * kQPT + j);
                        s.e_beg[pe] = beg[j];
                        s.e_off[pe] = ph;
                        ++pe;
                        ph += cnt[j];
                    }
                }
                __syncwarp();
                st_e += E;
                st_h += H;
                // ---- A6-A10: hits dealt 32 at a time
                // default: hits dealt 32 per round across the warp (A6). static_lb (the
                // Fig. 7 ablation, "without load balancing"): every lane walks
                // the hits of its own query positions, rounds = the warp's largest count.
                uint32_t rounds = (H + 31) / 32;
                const uint32_t h0 = ih - n_h;
                if (kStatic) {
                    rounds = n_h;
#pragma unroll
                    for (int o = 16; o; o >>= 1) rounds = max(rounds, __shfl_xor_sync(0xffffffffu, rounds, o));
                }
                uint32_t ent0 = 0;  // entry holding the round's first hit (entries hold >= 1 hit each)
                for (uint32_t rd = 0; rd < rounds; ++rd) {
                    const uint32_t h = kStatic ? h0 + rd : rd * 32 + lane;
                    const bool has = kStatic ? rd < n_h : h < H;
                    int verdict = kDrop;
                    Hit out{0, 0};
                    uint32_t p = 0, q = 0, e_rec = 0, f_rec = 0;
                    uint32_t ent = 0;
                    if (!kStatic) {
                        // the entries starting inside this round's 32 hits are among the next
                        // 32: one shared load per lane, an OR-reduction of their start bits,
                        // and each lane's entry is ent0 + the starts at or before it
                        const uint32_t hb = rd * 32, cand = ent0 + 1 + lane;
                        uint32_t bit = 0;
                        if (cand < E) {
                            const uint32_t off = s.e_off[cand];
                            if (off < hb + 32) bit = 1u << (off - hb);
                        }
                        const uint32_t starts = __reduce_or_sync(0xffffffffu, bit);
                        ent = ent0 + __popc(starts & ((2u << lane) - 1u));
                        const uint32_t last = ent0 + __popc(starts);  // entry of hit hb + 31
                        ent0 = (last + 1 < E && s.e_off[last + 1] <= hb + 32) ? last + 1 : last;
                    }
                    if (has) {
                        uint32_t lo = ent;
                        if (kStatic) {
                            uint32_t lo2 = 0, hi = E;  // largest entry i with e_off[i] <= h
                            while (hi - lo2 > 1) {
                                const uint32_t mid = (lo2 + hi) >> 1;
                                if (s.e_off[mid] <= h) lo2 = mid; else hi = mid;
                            }
                            lo = lo2;
                        }
                        q = q0 + s.e_q[lo];
                        uint32_t rl;
                        uint64_t rr;
                        load_rec<kRec8>(P, s.e_beg[lo] + (h - s.e_off[lo]), p, rl, rr, kHints ? 1 : -1);
                        verdict = decide_rec<kL, kR>(P, p, rl, rr, q, qs.back16(q), qs.fwd(q + P.ls), out, e_rec,
                                                     f_rec);
                    }
                    // hits the records cannot settle wait in the warp's queue
                    const unsigned need = __ballot_sync(0xffffffffu, verdict == kExt);
                    if (need) {
                        if (verdict == kExt) s.dq[nq + __popc(need & lanemask_lt())] = make_uint4(p, q, e_rec, f_rec);
                        nq += __popc(need);
                        __syncwarp();
                    }
                    warp_emit(P, s, nbuf, verdict == kEmit, out, false);
                    if (nq >= 32) drain_deferred<kL>(P, s, nq, nbuf, 32);
                }
            }
            __syncwarp();
        }
        c = cn;
        c_end = cn_end;
    }
    if (nq) drain_deferred<kL>(P, s, nq, nbuf, nq);
    warp_emit(P, s, nbuf, false, Hit{0, 0}, true);
    if (lane == 0 && st_e) {
        atomicAdd(&P.stats[0], st_e);
        atomicAdd(&P.stats[1], st_h);
    }
    if (lane == 0 && P.work) {  // D5: the tile scheduler's balance -- the busiest warp's hits
        atomicMax(P.work, st_h);
        atomicAdd(P.work + 1, 1ull);
    }
}

// K7: drain the heavy-bucket queue, one 32-hit piece per warp iteration.
template <bool kRec8>
__global__ void __launch_bounds__(kT) k_heavy(const FindParams P) {
    pdl_wait();
    constexpr int kL = kRec8 ? 8 : 16, kR = kRec8 ? 8 : 32;
    __shared__ EmitSmem smem[kWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    EmitSmem &s = smem[wid];
    uint32_t nbuf = 0;
    const unsigned long long sc = *P.spill_count;
    const unsigned long long n = sc < P.spill_cap ? sc : P.spill_cap;
    const unsigned long long gw = (unsigned long long)blockIdx.x * kWarps + wid;
    const unsigned long long nw = (unsigned long long)gridDim.x * kWarps;
    uint4 next = gw < n ? P.spill[gw] : make_uint4(0u, 0u, 0u, 0u);
    for (unsigned long long c = gw; c < n; c += nw) {
        const uint4 piece = next;
        if (c + nw < n) next = P.spill[c + nw];  // the warp's next piece, in flight meanwhile
        int verdict = kDrop;
        Hit out{0, 0};
        uint32_t p = 0;
        const uint32_t q = piece.x;
        if (uint32_t(lane) < piece.z) {
            uint32_t rl, e_rec = 0, f_rec = 0;
            uint64_t rr;
            load_rec<kRec8>(P, piece.y + lane, p, rl, rr, P.recs_stream);
            verdict = decide_rec<kL, kR>(P, p, rl, rr, q, uint32_t(win_back(P.Q, q)), win_fwd(P.Q, uint64_t(q) + P.ls),
                                         out, e_rec, f_rec);
            if (verdict == kExt) verdict = decide_deferred<kL>(P, p, q, e_rec, f_rec, out);
        }
        push_coop(P, verdict, p, q);
        warp_emit(P, s, nbuf, verdict == kEmit, out, false);
    }
    warp_emit(P, s, nbuf, false, Hit{0, 0}, true);
}

// Drain the coop queue: 32 deferred hits per warp iteration, decided from scratch
// with per-lane extension up to kLaneCap and warp-cooperative extension beyond.
__global__ void __launch_bounds__(kT) k_coop(const FindParams P) {
    pdl_wait();
    __shared__ EmitSmem smem[kWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    EmitSmem &s = smem[wid];
    uint32_t nbuf = 0;
    const unsigned long long cc = *P.coop_count;
    const unsigned long long n = cc < P.coop_cap ? cc : P.coop_cap;
    const unsigned long long gw = (unsigned long long)blockIdx.x * kWarps + wid;
    const unsigned long long nw = (unsigned long long)gridDim.x * kWarps;
    for (unsigned long long base = gw * 32; base < n; base += nw * 32) {
        const unsigned long long i = base + lane;
        const bool valid = i < n;
        const uint2 x = valid ? P.coopq[i] : make_uint2(0u, 0u);
        Hit h{0, 0};
        const bool em = resolve_deferred(P, valid, x.x, x.y, kUnresolved, h);
        warp_emit(P, s, nbuf, em, h, false);
    }
    warp_emit(P, s, nbuf, false, Hit{0, 0}, true);
}

// Finish the right extension of the matches emitted open (kOpenBit) while Q was still
// arriving: all of Q is present now. One thread per output slot; open matches are rare
// (those reaching a chunk end), a long one is walked 32 bases per step.
__global__ void __launch_bounds__(kT) k_open_fix(uint64_t *__restrict__ keys, uint32_t *__restrict__ lens,
                                                 const unsigned long long *__restrict__ count, uint64_t cap,
                                                 const uint64_t *__restrict__ R, uint64_t nR,
                                                 const uint64_t *__restrict__ Q, uint64_t nQ, uint32_t qbits) {
    pdl_wait();
    const unsigned long long c = *count;
    const uint64_t n = c < cap ? c : cap;
    for (uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x; i < n; i += uint64_t(gridDim.x) * kT) {
        const uint32_t l0 = lens[i];
        if (!(l0 & kOpenBit)) continue;
        const uint64_t k = keys[i];
        const uint64_t r = k >> qbits, q = k & ((1ull << qbits) - 1);
        uint64_t f = l0 & ~kOpenBit;
        const uint64_t lim = min(nR - r, nQ - q);
        while (f < lim) {
            const uint32_t run = lead_eq(win_fwd(R, r + f) ^ win_fwd(Q, q + f));
            f += run;
            if (run < 32) break;
        }
        lens[i] = uint32_t(min(f, lim));
    }
}

int g_default_grid[2] = {0, 0};

}  // namespace

uint64_t find_tile_positions(bool sect) { return sect ? FindShape<true>::kChunk : FindShape<false>::kChunk; }

int find_default_grid(bool sect) {
    int &g = g_default_grid[sect ? 1 : 0];
    if (!g) {
        int per_sm = 0;
        if (sect) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_find<false, false, true, false>, kT, 0);
        else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_find<false, false, false, false>, kT, 0);
        if (per_sm < 1) per_sm = 1;
        g = per_sm * num_sms();
    }
    return g;
}

cudaError_t launch_find(const FindParams &p, int grid, cudaStream_t s) {
    if (p.n_tiles == 0) return cudaSuccess;
    if (grid <= 0) grid = find_default_grid(p.rsect != nullptr);
    const uint64_t max_useful = (p.n_tiles + kGrab - 1) / kGrab;
    if (uint64_t(grid) * kWarps > max_useful) grid = int((max_useful + kWarps - 1) / kWarps);
    if (grid < 1) grid = 1;
    g_l2win = p.l2win;
    // kHints: the seed records exceed half of L2 -> cache-policy loads (lookup tables
    // evict_last, streams evict_first); otherwise plain loads (measured faster there)
    const bool sect = p.rsect != nullptr;
#define GM_FIND_LAUNCH(ST, HI)                                                              \
    do {                                                                                    \
        if (sect) {                                                                         \
            if (p.rec8) pdl_launch(k_find<ST, HI, true, true>, grid, kT, 0, s, p);                  \
            else pdl_launch(k_find<ST, HI, true, false>, grid, kT, 0, s, p);                        \
        } else {                                                                            \
            if (p.rec8) pdl_launch(k_find<ST, HI, false, true>, grid, kT, 0, s, p);                 \
            else pdl_launch(k_find<ST, HI, false, false>, grid, kT, 0, s, p);                       \
        }                                                                                   \
    } while (0)
    if (p.static_lb) GM_FIND_LAUNCH(true, false);
    else if (p.recs_stream) GM_FIND_LAUNCH(false, true);
    else GM_FIND_LAUNCH(false, false);
#undef GM_FIND_LAUNCH
    g_l2win = cudaAccessPolicyWindow{};
    note_launch();
    return cudaGetLastError();
}

// The pipeline's end-of-run report, written straight into its pinned host buffer (mapped
// under unified addressing) by one launch instead of four small D2H copy nodes:
// host[0, 8) = counters, [8] / [9] = R / Q alphabet flags, [10, 12) = balance stats.
__global__ void k_collect(const unsigned long long *__restrict__ ctr, const unsigned long long *__restrict__ rbad,
                          const unsigned long long *__restrict__ qbad, unsigned long long *host) {
    pdl_wait();
    const int t = threadIdx.x;
    if (t < 8) host[t] = ctr[t];
    else if (t == 8) host[8] = *rbad;
    else if (t == 9) host[9] = *qbad;
    else if (t < 12) host[t] = ctr[t - 2];
}

cudaError_t launch_collect(const unsigned long long *ctr, const unsigned long long *rbad,
                           const unsigned long long *qbad, unsigned long long *host, cudaStream_t s) {
    pdl_launch(k_collect, 1, 32, 0, s, ctr, rbad, qbad, host);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_open_fix(const FindParams &p, cudaStream_t s) {
    pdl_launch(k_open_fix, num_sms() * 4, kT, 0, s, p.out_key, p.out_len, static_cast<const unsigned long long *>(p.out_count),
               p.capacity, p.R, p.nR, p.Q, p.nQ, p.qbits);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_coop(const FindParams &p, cudaStream_t s) {
    pdl_launch(k_coop, num_sms() * 2, kT, 0, s, p);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_heavy(const FindParams &p, cudaStream_t s) {
    g_l2win = p.l2win;
    if (p.rec8) pdl_launch(k_heavy<true>, num_sms() * GM_HEAVY_CTAS, kT, 0, s, p);
    else pdl_launch(k_heavy<false>, num_sms() * GM_HEAVY_CTAS, kT, 0, s, p);
    g_l2win = cudaAccessPolicyWindow{};
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
