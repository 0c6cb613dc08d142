// find.cu -- K6/K7: seed lookup + bidirectional extension + canonical-seed
// duplicate elimination + compaction.
//
// The 2D search space (R on one axis, Q on the other) is cut into
// query tiles of kFTile positions x the sampled-R hits of those positions. A
// persistent grid pulls tiles from an atomic counter (the tile scheduler, A6).
// Per tile:
//  phase 1 (A5)  each thread takes kQPT consecutive query positions, cuts their
//                seeds out of one 64-bit window of packed Q, probes the occupancy
//                bitmap (L2-resident) and, for occupied seeds, reads the bucket
//                range [ptrs[s], ptrs[s+1]). Buckets larger than
//                `spill_t` are cut into kSpillChunk-hit chunks and pushed to a
//                global queue drained by k_heavy (reference-axis tiles of the hot
//                seeds, Fig. 6 :268-270); the rest become (q, bucket) entries in
//                shared memory with an exclusive prefix of their hit counts.
//  phase 2 (A6)  the tile's H hits are dealt evenly to the CTA's threads (hit h
//                -> entry by binary search over the prefix), replacing the paper's
//                proactive load-balancing heuristic (Alg. 2, :120-149) and its
//                combine step (Alg. 3, :155-169):
//   A7 left extension, capped at step: e = equal bases left of (p, q), stopping at
//      a mismatch, at either sequence start, or at e == step. e == step means the
//      sampled seed at p - step lies on the same diagonal inside the same match,
//      so that hit (further left) owns the MEM: drop. Exactly one sampled seed per
//      MEM has e < step, so each MEM is emitted once
//      (:153 "not to extract a MEM more than once").
//   A8 right extension from the seed's end to the first mismatch or end, unbounded.
//   A9 keep len = e + ls + f >= L (:53-56); maximal on both sides by construction.
//   A10 block-aggregated compaction: ballot/popc per warp, one atomicAdd per CTA
//      round on the global counter; writes past `capacity` are counted, not stored.
// All compares are 2-bit packed words: XOR, then __clzll (rightwards) or __ffsll
// (leftwards) finds the first mismatching base exactly (reading R11).
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kFT = 256;                  // threads per CTA
constexpr int kWarps = kFT / 32;
constexpr int kQPT = 8;                   // query positions per thread per tile
constexpr int kFTile = kFT * kQPT;        // 2048 query positions per tile
constexpr uint32_t kSpillChunk = kFT;     // hits per heavy chunk (one per thread)

// Four consecutive words starting at i0 = max(p/32 - 1, 0): cover the first left
// window [p-32, p) and the first right window [p+ls, p+ls+32) for ls <= 15.
struct Win4 {
    uint64_t w0, w1, w2, w3;
    uint64_t i0;
    __device__ __forceinline__ uint64_t get(uint32_t k) const {
        return k == 0 ? w0 : k == 1 ? w1 : k == 2 ? w2 : w3;
    }
    __device__ __forceinline__ void load(const uint64_t *__restrict__ W, uint64_t p) {
        i0 = (p >> 5) ? (p >> 5) - 1 : 0;
        w0 = __ldg(W + i0);
        w1 = __ldg(W + i0 + 1);
        w2 = __ldg(W + i0 + 2);
        w3 = __ldg(W + i0 + 3);
    }
    // bases [p-32, p) (zeros before position 0)
    __device__ __forceinline__ uint64_t back(uint64_t p) const {
        if (p < 32) return p ? (w0 >> (64 - 2 * p)) : 0ull;
        const uint32_t sh = uint32_t(p & 31) * 2;  // (p-32)/32 == i0
        return sh ? (w0 << sh) | (w1 >> (64 - sh)) : w0;
    }
    // bases [x, x+32) for x in [p, p+15]
    __device__ __forceinline__ uint64_t fwd(uint64_t x) const {
        const uint32_t k = uint32_t((x >> 5) - i0);
        const uint32_t sh = uint32_t(x & 31) * 2;
        const uint64_t a = get(k), b = get(k + 1);
        return sh ? (a << sh) | (b >> (64 - sh)) : a;
    }
};

// One hit (p in R, q in Q, seeds equal). Returns true and the packed triple if
// this hit is the MEM's canonical seed, the MEM is owned and len >= L.
__device__ __forceinline__ bool process_hit(const FindParams &P, uint64_t p, uint64_t q, uint64_t &key,
                                            uint32_t &len) {
    Win4 wr, wq;
    wr.load(P.R, p);
    wq.load(P.Q, q);
    // A7: left extension, capped at step
    const uint64_t lim = min(uint64_t(P.step), min(p, q));
    uint64_t e = trail_eq(wr.back(p) ^ wq.back(q));
    if (e == 32) {
        while (e < lim) {
            const uint32_t run = trail_eq(win_back(P.R, p - e) ^ win_back(P.Q, q - e));
            e += run;
            if (run < 32) break;
        }
    }
    if (e > lim) e = lim;
    if (e == P.step) return false;                         // not the canonical (leftmost) seed
    const uint64_t qs = q - e;
    if (qs < P.own_lo || qs >= P.own_hi) return false;     // another shard owns it
    // A8: right extension from the end of the seed
    const uint64_t a = p + P.ls, b = q + P.ls;
    const uint64_t lim_r = min(P.nR - a, P.nQ - b);
    uint64_t f = lead_eq(wr.fwd(a) ^ wq.fwd(b));
    if (f == 32) {
        while (f < lim_r) {
            const uint32_t run = lead_eq(win_fwd(P.R, a + f) ^ win_fwd(P.Q, b + f));
            f += run;
            if (run < 32) break;
        }
    }
    if (f > lim_r) f = lim_r;
    const uint64_t lam = e + P.ls + f;
    if (lam < P.L) return false;                           // A9
    key = ((p - e) << P.qbits) | qs;
    len = uint32_t(lam);
    return true;
}

// A10: CTA-aggregated append. Must be reached by every thread of the CTA.
__device__ __forceinline__ void block_emit(const FindParams &P, bool emit, uint64_t key, uint32_t len,
                                           uint32_t *s_wcnt, unsigned long long *s_base) {
    if (!__syncthreads_or(emit)) return;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned bal = __ballot_sync(0xffffffffu, emit);
    if (lane == 0) s_wcnt[w] = __popc(bal);
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tot = 0;
#pragma unroll
        for (int i = 0; i < kWarps; ++i) {
            const uint32_t c = s_wcnt[i];
            s_wcnt[i] = tot;
            tot += c;
        }
        *s_base = atomicAdd(P.out_count, (unsigned long long)tot);
    }
    __syncthreads();
    if (emit) {
        const unsigned long long pos = *s_base + s_wcnt[w] + __popc(bal & lanemask_lt());
        if (pos < P.capacity) {
            P.out_key[pos] = key;
            P.out_len[pos] = len;
        }
    }
}

__global__ void __launch_bounds__(kFT) k_find(const FindParams P) {
    __shared__ uint32_t s_eq[kFTile];       // entry -> query offset in tile
    __shared__ uint32_t s_ebeg[kFTile];     // entry -> first slot of its bucket in locs
    __shared__ uint32_t s_eoff[kFTile + 1]; // entry -> exclusive prefix of hit counts
    __shared__ uint32_t s_ws[2][kWarps];
    __shared__ uint32_t s_wcnt[kWarps];
    __shared__ unsigned long long s_base;
    __shared__ unsigned int s_tile;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint32_t sh = 64 - 2 * P.ls;

    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(P.tile_ctr, 1u);
        __syncthreads();
        const uint64_t tile = s_tile;
        if (tile >= P.n_tiles) break;
        const uint64_t t0 = P.scan_lo + tile * kFTile;
        const uint64_t q0 = t0 + uint64_t(threadIdx.x) * kQPT;

        // ---- phase 1: seeds -> bitmap -> bucket ranges
        uint32_t beg[kQPT], cnt[kQPT];
#pragma unroll
        for (int j = 0; j < kQPT; ++j) beg[j] = cnt[j] = 0;
        if (q0 < P.scan_hi) {
            const uint64_t win = win_fwd(P.Q, q0);  // bases q0 .. q0+31 cover kQPT seeds
            uint32_t code[kQPT];
            bool occ[kQPT];
#pragma unroll
            for (int j = 0; j < kQPT; ++j) {
                code[j] = uint32_t((win << (2 * j)) >> sh);
                occ[j] = q0 + j < P.scan_hi;
            }
            if (P.use_bitmap) {
#pragma unroll
                for (int j = 0; j < kQPT; ++j)
                    if (occ[j]) occ[j] = (__ldg(P.bitmap + (code[j] >> 5)) >> (code[j] & 31)) & 1u;
            }
#pragma unroll
            for (int j = 0; j < kQPT; ++j) {
                if (occ[j]) {
                    beg[j] = __ldg(P.ptrs + code[j]);
                    cnt[j] = __ldg(P.ptrs + code[j] + 1) - beg[j];
                }
            }
#pragma unroll
            for (int j = 0; j < kQPT; ++j) {
                if (cnt[j] > P.spill_t) {  // heavy bucket: reference-axis chunks to the queue
                    const uint32_t nch = (cnt[j] + kSpillChunk - 1) / kSpillChunk;
                    const unsigned long long slot = atomicAdd(P.spill_count, (unsigned long long)nch);
                    if (slot + nch <= P.spill_cap) {
                        for (uint32_t c = 0; c < nch; ++c) {
                            const uint32_t off = c * kSpillChunk;
                            P.spill[slot + c] = make_uint4(uint32_t(q0 + j), beg[j] + off,
                                                           min(kSpillChunk, cnt[j] - off), 0u);
                        }
                        cnt[j] = 0;
                    } else {
                        for (unsigned long long s2 = slot; s2 < P.spill_cap; ++s2)
                            P.spill[s2] = make_uint4(0u, 0u, 0u, 0u);  // neutralise; processed here
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
        // block exclusive scan of (n_e, n_h)
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
        if (lane == 31) {
            s_ws[0][w] = ie;
            s_ws[1][w] = ih;
        }
        __syncthreads();
        uint32_t pe = ie - n_e, ph = ih - n_h, E = 0, H = 0;
#pragma unroll
        for (int i = 0; i < kWarps; ++i) {
            const uint32_t a = s_ws[0][i], b = s_ws[1][i];
            if (i < w) {
                pe += a;
                ph += b;
            }
            E += a;
            H += b;
        }
#pragma unroll
        for (int j = 0; j < kQPT; ++j) {
            if (cnt[j]) {
                s_eq[pe] = uint32_t(threadIdx.x) * kQPT + j;
                s_ebeg[pe] = beg[j];
                s_eoff[pe] = ph;
                ++pe;
                ph += cnt[j];
            }
        }
        __syncthreads();

        // ---- phase 2: hits dealt evenly over the CTA
        for (uint32_t hb = 0; hb < H; hb += kFT) {
            const uint32_t h = hb + threadIdx.x;
            bool emit = false;
            uint64_t key = 0;
            uint32_t len = 0;
            if (h < H) {
                uint32_t lo = 0, hi = E;  // largest entry i with s_eoff[i] <= h
                while (hi - lo > 1) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if (s_eoff[mid] <= h) lo = mid; else hi = mid;
                }
                const uint64_t q = t0 + s_eq[lo];
                const uint64_t p = __ldg(P.locs + s_ebeg[lo] + (h - s_eoff[lo]));
                emit = process_hit(P, p, q, key, len);
            }
            block_emit(P, emit, key, len, s_wcnt, &s_base);
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kFT) k_heavy(const FindParams P) {
    __shared__ uint32_t s_wcnt[kWarps];
    __shared__ unsigned long long s_base;
    const unsigned long long sc = *P.spill_count;
    const unsigned long long n = sc < P.spill_cap ? sc : P.spill_cap;
    for (unsigned long long c = blockIdx.x; c < n; c += gridDim.x) {
        const uint4 ch = P.spill[c];
        bool emit = false;
        uint64_t key = 0;
        uint32_t len = 0;
        if (threadIdx.x < ch.z) {
            const uint64_t p = __ldg(P.locs + ch.y + threadIdx.x);
            emit = process_hit(P, p, ch.x, key, len);
        }
        block_emit(P, emit, key, len, s_wcnt, &s_base);
    }
}

int g_default_grid = 0;

}  // namespace

uint64_t find_tile_positions() { return kFTile; }

int find_default_grid() {
    if (!g_default_grid) {
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_find, kFT, 0);
        if (per_sm < 1) per_sm = 1;
        g_default_grid = per_sm * num_sms();
    }
    return g_default_grid;
}

cudaError_t launch_find(const FindParams &p, int grid, cudaStream_t s) {
    if (p.n_tiles == 0) return cudaSuccess;
    if (grid <= 0) grid = find_default_grid();
    if (uint64_t(grid) > p.n_tiles) grid = int(p.n_tiles);
    k_find<<<grid, kFT, 0, s>>>(p);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_heavy(const FindParams &p, cudaStream_t s) {
    k_heavy<<<num_sms() * 4, kFT, 0, s>>>(p);
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
