// device.cuh -- device helpers on 2-bit packed sequences (sm_100a).
//
// Packed layout ("each base is represented by 2 bits", A=00 C=01
// G=10 T=11): base i sits in bits [63-2(i%32), 62-2(i%32)] of word i/32, so the
// first base of a word is its most significant pair and a 64-bit window of 32
// consecutive bases starting anywhere is a funnel shift of two words. Every
// sequence carries four zero words of padding after its last word; bases past
// the end read as 'A' (00), so every compare is clamped by the caller to the
// sequence ends (an end counts as a mismatch, reading R3).
#pragma once
#include <cstdint>

namespace gm {

// Bounds checks of the debug variant (tools/variants.py dbg=-DGM_DEBUG_BOUNDS=1): a failed
// check traps the kernel (the call returns GPUMEM_ERR_CUDA); compiled out by default.
#ifndef GM_DEBUG_BOUNDS
#define GM_DEBUG_BOUNDS 0
#endif
#if GM_DEBUG_BOUNDS
#define GM_CHECK(c) \
    do {            \
        if (!(c)) __trap(); \
    } while (0)
#else
#define GM_CHECK(c) \
    do {            \
    } while (0)
#endif

// 32 bases starting at position i (i may be up to n; padding makes it safe).
__device__ __forceinline__ uint64_t win_fwd(const uint64_t *__restrict__ W, uint64_t i) {
    const uint64_t wi = i >> 5;
    const uint32_t sh = uint32_t(i & 31) * 2;
    const uint64_t w0 = __ldg(W + wi);
    const uint64_t w1 = __ldg(W + wi + 1);
    return sh ? (w0 << sh) | (w1 >> (64 - sh)) : w0;
}

// 32 bases ending at position a (exclusive): bases [a-32, a), base a-1 in the
// low two bits. Positions before 0 read as 00 (callers clamp with min(p, q)).
__device__ __forceinline__ uint64_t win_back(const uint64_t *__restrict__ W, uint64_t a) {
    if (a >= 32) return win_fwd(W, a - 32);
    return a ? (__ldg(W) >> (64 - 2 * a)) : 0ull;
}

// Number of equal leading bases of two forward windows (32 if identical).
__device__ __forceinline__ uint32_t lead_eq(uint64_t x) { return x ? uint32_t(__clzll(x)) >> 1 : 32u; }
// Number of equal trailing bases of two backward windows (32 if identical).
__device__ __forceinline__ uint32_t trail_eq(uint64_t x) { return x ? uint32_t(__ffsll(x) - 1) >> 1 : 32u; }

__device__ __forceinline__ int lane_id() { return int(threadIdx.x & 31); }

// Loads with an L2 eviction priority (PTX createpolicy + ld.L2::cache_hint): the small,
// hot lookup tables stay (evict_last) while one-pass streams go first (evict_first).
// The policy is created inside each asm block so it never occupies a live register.
#define GM_LD_HINT(PRIO, TYPE, MOD, OUTS, ...)                                                     \
    asm("{ .reg .b64 pol; createpolicy.fractional.L2::" PRIO ".b64 pol, 1.0;\n\t"                 \
        "ld.global.nc" MOD ".L2::cache_hint" TYPE " " OUTS ", pol; }" __VA_ARGS__)
__device__ __forceinline__ unsigned long long ld_last_u64(const unsigned long long *a) {
    unsigned long long v;
    GM_LD_HINT("evict_last", ".u64", "", "%0, [%1]", : "=l"(v) : "l"(a));
    return v;
}
__device__ __forceinline__ unsigned long long ld_first_u64(const unsigned long long *a) {
    unsigned long long v;
    GM_LD_HINT("evict_first", ".u64", "", "%0, [%1]", : "=l"(v) : "l"(a));
    return v;
}
__device__ __forceinline__ uint2 ld_last_u2(const uint2 *a) {
    uint2 v;
    GM_LD_HINT("evict_last", ".v2.u32", "", "{%0, %1}, [%2]", : "=r"(v.x), "=r"(v.y) : "l"(a));
    return v;
}
__device__ __forceinline__ uint4 ld_last_u4(const uint4 *a) {
    uint4 v;
    GM_LD_HINT("evict_last", ".v4.u32", "", "{%0, %1, %2, %3}, [%4]", : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a));
    return v;
}
__device__ __forceinline__ uint2 ld_hint_u2(const uint2 *a, bool stream) {
    uint2 v;
    if (stream)
        GM_LD_HINT("evict_first", ".v2.u32", ".L1::no_allocate", "{%0, %1}, [%2]", : "=r"(v.x), "=r"(v.y) : "l"(a));
    else
        GM_LD_HINT("evict_last", ".v2.u32", ".L1::no_allocate", "{%0, %1}, [%2]", : "=r"(v.x), "=r"(v.y) : "l"(a));
    return v;
}
__device__ __forceinline__ uint4 ld_hint_u4(const uint4 *a, bool stream) {
    uint4 v;
    if (stream)
        GM_LD_HINT("evict_first", ".v4.u32", ".L1::no_allocate", "{%0, %1, %2, %3}, [%4]",
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a));
    else
        GM_LD_HINT("evict_last", ".v4.u32", ".L1::no_allocate", "{%0, %1, %2, %3}, [%4]",
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a));
    return v;
}

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

}  // namespace gm
