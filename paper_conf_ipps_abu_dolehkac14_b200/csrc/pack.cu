// pack.cu -- K1: ASCII -> 2-bit packed words.
//
// One thread per kWPT output words = 32 input bytes each, read as two 128-bit vector
// loads when the input is 16-byte aligned (scalar bytes otherwise and for the tail).
// Per 4 bytes (SWAR): code = ((c>>1) ^ (c>>2)) & 3 maps A/a->0 C/c->1 G/g->2
// T/t->3; validity is checked exactly by rebuilding the expected upper-case
// byte from the code with one PRMT and comparing. The first invalid position
// is recorded with atomicMin (alphabet error, reading R4).
// Algorithmic bytes: 1 B read + 0.25 B written per base (HBM-bound).
#include "internal.h"

namespace gm {
namespace {

constexpr int kPackThreads = 256;

// 4 ASCII bytes -> 8 bits of codes (first byte most significant), valid flag.
__device__ __forceinline__ uint32_t pack4(uint32_t x, bool &ok) {
    const uint32_t c = ((x >> 1) ^ (x >> 2)) & 0x03030303u;          // per-byte code
    const uint32_t y = c | (c >> 4);
    const uint32_t sel = (y & 0xFFu) | ((y >> 8) & 0xFF00u);         // codes -> PRMT nibbles
    const uint32_t expect = __byte_perm(0x54474341u, 0u, sel);       // 'T''G''C''A'
    ok = ok && (expect == (x & 0xDFDFDFDFu));                        // exact, upper-cased
    return (c * 0x40100401u) >> 24;                                  // c0<<6|c1<<4|c2<<2|c3
}

// word w from 32 ASCII bytes (the scalar path handles unaligned input and the tail)
__device__ __forceinline__ uint64_t pack_word_scalar(const uint8_t *__restrict__ in, uint64_t n, uint64_t w,
                                                     unsigned long long *bad_pos, uint64_t pos_base) {
    uint64_t word = 0;
    const uint64_t base = w * 32;
    for (int i = 0; i < 32; ++i) {
        const uint64_t pos = base + i;
        if (pos >= n) break;  // padding bases stay 00
        const uint32_t ch = in[pos];
        const uint32_t c = ((ch >> 1) ^ (ch >> 2)) & 3u;
        const uint32_t up = ch & 0xDFu;
        if (up != 'A' && up != 'C' && up != 'G' && up != 'T') atomicMin(bad_pos, (unsigned long long)(pos_base + pos));
        word |= uint64_t(c) << (62 - 2 * i);
    }
    return word;
}

__device__ __noinline__ void report_bad(const uint8_t *__restrict__ in, uint64_t w, unsigned long long *bad_pos,
                                       uint64_t pos_base) {
    for (int i = 0; i < 32; ++i) {  // locate the first bad byte of this word
        const uint32_t up = in[w * 32 + i] & 0xDFu;
        if (up != 'A' && up != 'C' && up != 'G' && up != 'T') {
            atomicMin(bad_pos, (unsigned long long)(pos_base + w * 32 + i));
            break;
        }
    }
}

// Aligned input: thread t of a CTA takes the 16-byte halves t, t + T, ... (T = threads;
// kHPT of them, all loads in flight first), so every warp load instruction reads 512
// contiguous bytes; a half packs to 32 bits and the even lane of each pair assembles
// the 64-bit word with its odd neighbour's half (one shuffle) and stores it -- each
// input sector is requested exactly once. Words from n_full on (the partial last word
// and the zero padding) and unaligned inputs take the scalar path.
#ifndef GM_PACK_HPT
#define GM_PACK_HPT 8
#endif
constexpr int kHPT = GM_PACK_HPT;  // halves per thread

__device__ __forceinline__ uint32_t pack16(const uint4 v, bool &ok) {
    return (pack4(v.x, ok) << 24) | (pack4(v.y, ok) << 16) | (pack4(v.z, ok) << 8) | pack4(v.w, ok);
}

__global__ void __launch_bounds__(kPackThreads) k_pack(const uint8_t *__restrict__ in, uint64_t n,
                                                       uint64_t *__restrict__ words, uint64_t n_full,
                                                       uint64_t n_words_alloc, unsigned long long *bad_pos,
                                                       int aligned, uint64_t pos_base) {
    pdl_wait();
    const int lane = threadIdx.x & 31;
    if (aligned) {
        const uint64_t n_halves = 2 * n_full;
        const uint64_t h0 = uint64_t(blockIdx.x) * kPackThreads * kHPT + threadIdx.x;
        uint4 v[kHPT];
#pragma unroll
        for (int k = 0; k < kHPT; ++k) {
            const uint64_t h = h0 + uint64_t(k) * kPackThreads;
            if (h < n_halves) v[k] = __ldcs(reinterpret_cast<const uint4 *>(in) + h);  // streamed once
        }
#pragma unroll
        for (int k = 0; k < kHPT; ++k) {
            const uint64_t h = h0 + uint64_t(k) * kPackThreads;  // h's parity = the lane's parity
            bool ok = true;
            const uint32_t half = h < n_halves ? pack16(v[k], ok) : 0u;
            const uint32_t odd = __shfl_down_sync(0xffffffffu, half, 1);
            if (h < n_halves) {
                if (!ok) report_bad(in, h >> 1, bad_pos, pos_base);  // the word's first bad byte (either half)
                if (!(lane & 1)) words[h >> 1] = (uint64_t(half) << 32) | odd;
            }
        }
    }
    // scalar words: [n_full, n_words_alloc) always, all words for unaligned input
    const uint64_t first = aligned ? n_full : 0;
    const uint64_t tail = n_words_alloc - first;
    const uint64_t per_cta = uint64_t(kPackThreads);
    for (uint64_t i = uint64_t(blockIdx.x) * per_cta + threadIdx.x; i < tail; i += uint64_t(gridDim.x) * per_cta)
        words[first + i] = pack_word_scalar(in, n, first + i, bad_pos, pos_base);
}

// Reverse complement of a packed sequence (NEXT-F4): rc[i] = 3 - s[n-1-i] (A<->T, C<->G
// is XOR 3 in the A0 C1 G2 T3 code). Output word w holds rc bases [32w, 32w+32): the
// 32 bases of s ending at n - 32w, reversed pairwise, complemented, tail kept 00.
__global__ void __launch_bounds__(kPackThreads) k_revcomp(const uint64_t *__restrict__ in, uint64_t n,
                                                          uint64_t *__restrict__ out, uint64_t n_words_alloc) {
    pdl_wait();
    const uint64_t w = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (w >= n_words_alloc) return;
    const uint64_t first = w * 32;
    if (first >= n) {
        out[w] = 0;
        return;
    }
    const uint64_t end = n - first;  // s bases [end-32, end) -> rc bases [first, first+32)
    uint64_t x;
    if (end >= 32) {
        const uint64_t a = end - 32, wi = a >> 5;
        const uint32_t sh = uint32_t(a & 31) * 2;
        x = sh ? (in[wi] << sh) | (in[wi + 1] >> (64 - sh)) : in[wi];
    } else {
        x = in[0] >> (64 - 2 * end);  // s bases [0, end) in the low bits
    }
    uint64_t y = __brevll(x);                                                  // bit order reversed
    y = ((y >> 1) & 0x5555555555555555ull) | ((y & 0x5555555555555555ull) << 1);  // fix pairs
    y = ~y;                                                                    // complement (XOR 3)
    const uint64_t valid = end >= 32 ? 32 : end;
    if (valid < 32) y &= ~0ull << (64 - 2 * valid);                            // padding stays 00
    out[w] = y;
}

// Fill `words` 32-bit words with v (16-byte stores when aligned), grid-stride. A kernel
// rather than a memset node, so it keeps the PDL chain between the kernels around it.
__global__ void __launch_bounds__(256) k_fill(uint32_t *__restrict__ p, uint64_t words, uint32_t v) {
    pdl_wait();
    const uint64_t t0 = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x, nt = uint64_t(gridDim.x) * blockDim.x;
    uint64_t head = 0;
    if ((reinterpret_cast<uintptr_t>(p) & 15) == 0) {
        const uint64_t n4 = words / 4;
        uint4 *q = reinterpret_cast<uint4 *>(p);
        for (uint64_t i = t0; i < n4; i += nt) q[i] = make_uint4(v, v, v, v);
        head = n4 * 4;
    }
    for (uint64_t i = head + t0; i < words; i += nt) p[i] = v;
}

}  // namespace

cudaError_t fill_async(void *p, uint32_t v, size_t bytes, cudaStream_t s) {
    const uint64_t words = bytes / 4;
    if (!words) return cudaSuccess;
    uint64_t blocks = (words / 4 + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > uint64_t(num_sms()) * 8) blocks = uint64_t(num_sms()) * 8;
    pdl_launch(k_fill, unsigned(blocks), 256, 0, s, static_cast<uint32_t *>(p), words, v);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_revcomp(const uint64_t *in, uint64_t n, uint64_t *out, uint64_t n_words_alloc, cudaStream_t s) {
    const uint64_t blocks = (n_words_alloc + kPackThreads - 1) / kPackThreads;
    pdl_launch(k_revcomp, unsigned(blocks), kPackThreads, 0, s, in, n, out, n_words_alloc);
    note_launch();
    return cudaGetLastError();
}

cudaError_t launch_pack(const uint8_t *in, uint64_t n, uint64_t *words, uint64_t n_words_alloc,
                        unsigned long long *bad_pos, cudaStream_t s, uint64_t pos_base) {
    const int aligned = (reinterpret_cast<uintptr_t>(in) & 15) == 0;
    const uint64_t n_full = n / 32;
    const uint64_t per = uint64_t(kPackThreads) * kHPT;  // halves per CTA
    uint64_t blocks = aligned ? (2 * n_full + per - 1) / per : (n_words_alloc + kPackThreads - 1) / kPackThreads;
    if (blocks == 0) blocks = 1;
    pdl_launch(k_pack, unsigned(blocks), kPackThreads, 0, s, in, n, words, n_full, n_words_alloc, bad_pos, aligned,
               pos_base);
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
