// index_common.cuh -- device helpers shared by the two index builders (index.cu: the
// radix-sort path; tindex.cu: Alg. 1 tiled over the seed space).
#pragma once
#include <cstdint>

#include "device.cuh"

namespace gm {
namespace {

// Rank-word directory entries are 16 bytes per group g of 32 seeds: word 2g = {occupancy
// bits, occupied seeds before the group} (the rank word), word 2g+1 = occupancy of the 32
// seeds whose codes ROTATED left by one base (the first base moved to the end) fall in
// group g. Rotating code(Q, q) gives the same top bits as code(Q, q+1) (both start with
// bases q+1 ...), so one 16-byte probe of group code(q+1) >> 5 answers "is the seed at q
// occupied?" and "at q+1?" -- k_find probes query positions in pairs.
// The rotated bits are ORed in here (the directory is zeroed first) for every occupied seed.
__device__ __forceinline__ void set_rot_occ(unsigned long long *rankw, uint32_t code, uint32_t ls) {
    const uint32_t nbits = 2 * ls;
    const uint32_t mask = nbits >= 32 ? 0xffffffffu : ((1u << nbits) - 1u);
    const uint32_t rot = ((code << 2) | (code >> (nbits - 2))) & mask;
    atomicOr(reinterpret_cast<unsigned int *>(rankw + 2 * (rot >> 5) + 1), 1u << (rot & 31));
}

// Seed records (lookup acceleration, not part of the paper's index): for each slot k
// of locs, {p, bases R[p-16, p) with base p-1 in the low bits (00 before position 0),
// bases R[p+ls, p+ls+32) first base highest (00 past the end)} -- 16 bytes, one
// sector, so the find kernel decides a random seed hit without gathering R. With
// step <= 8 the left extension never passes 8 bases, and 8-byte records {p, R[p-8, p)
// | R[p+ls, p+ls+8) << 16} halve the record traffic of the (then numerous) hits.
// the record of location p = locs[k] (16-byte or 8-byte layout, see above)
template <bool kRec8>
__device__ __forceinline__ void seed_rec(const uint64_t *__restrict__ R, uint32_t ls, uint32_t p, void *recs,
                                         uint64_t k) {
    uint32_t left;
    uint64_t right;
    if (kRec8 && p >= 8) {  // bases [p - 8, p + ls + 8) (<= 31 bases) lie in the 2 words from (p - 8) / 32
        const uint64_t x = p - 8, w = x >> 5;
        const uint64_t w0 = __ldg(R + w), w1 = __ldg(R + w + 1);
        const uint32_t sx = uint32_t(x & 31) * 2;
        const uint64_t win = sx ? (w0 << sx) | (w1 >> (64 - sx)) : w0;  // bases [p - 8, p + 24)
        left = uint32_t(win >> 48);                                       // R[p - 8, p), base p-1 lowest
        right = (win << (2 * (8 + ls))) & 0xffff000000000000ull;          // R[p + ls, p + ls + 8) on top
    } else if (p >= 16) {  // bases [p - 16, p + ls + 32) lie in the 3 words from (p - 16) / 32: one gather
        const uint64_t x = p - 16, w = x >> 5;
        const uint64_t w0 = __ldg(R + w), w1 = __ldg(R + w + 1), w2 = __ldg(R + w + 2);
        const uint32_t sx = uint32_t(x & 31) * 2;
        left = uint32_t(((w0 << sx) | ((w1 >> 1) >> (63 - sx))) >> 32);
        const uint32_t o = uint32_t(x & 31) + 16 + ls;  // right window start, bases from word w
        const uint32_t so = (o & 31) * 2;
        const uint64_t a = o < 32 ? w0 : w1, b = o < 32 ? w1 : w2;
        right = (a << so) | ((b >> 1) >> (63 - so));
    } else {
        left = uint32_t(win_back(R, p));
        right = win_fwd(R, uint64_t(p) + ls);
    }
    if (kRec8) static_cast<uint2 *>(recs)[k] = make_uint2(p, (left & 0xffffu) | uint32_t(right >> 48) << 16);
    else static_cast<uint4 *>(recs)[k] = make_uint4(p, left, uint32_t(right), uint32_t(right >> 32));
}

// Ascending in-place sort of a[0, n) by all threads of the block (a bitonic-type network
// with ascending compare-exchanges only: the first stage of every merge pairs i with the
// mirror element, so indices past n act as +infinity and need no padding). a may be
// shared or global memory (global: visible to the block after each barrier).
__device__ __forceinline__ void cmpswap(uint32_t *a, uint32_t i, uint32_t j) {
    const uint32_t x = a[i], y = a[j];
    if (x > y) {
        a[i] = y;
        a[j] = x;
    }
}
__device__ void net_sort(uint32_t *a, uint32_t n) {
    uint32_t N = 1;
    while (N < n) N <<= 1;
    for (uint32_t k = 2; k <= N; k <<= 1) {
        for (uint32_t t = threadIdx.x; t < N / 2; t += blockDim.x) {  // mirror stage
            const uint32_t blk = t / (k / 2), j = t % (k / 2);
            const uint32_t i0 = blk * k + j, i1 = blk * k + k - 1 - j;
            if (i1 < n) cmpswap(a, i0, i1);
        }
        __syncthreads();
        for (uint32_t d = k / 4; d >= 1; d >>= 1) {  // half-cleaners
            for (uint32_t t = threadIdx.x; t < N / 2; t += blockDim.x) {
                const uint32_t blk = t / d, j = t % d;
                const uint32_t i0 = blk * 2 * d + j, i1 = i0 + d;
                if (i1 < n) cmpswap(a, i0, i1);
            }
            __syncthreads();
        }
    }
}

}  // namespace
}  // namespace gm
