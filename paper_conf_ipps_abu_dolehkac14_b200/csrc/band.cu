// band.cu -- NEXT-F2: the paper's reference row sweep with a band-local R
// (§III: "only a partial index is created for l_tile base pairs of
// reference ... used until all the tiles in that row are processed"; :92 §III-A), so R
// need not fit in device memory: only one window of R (ASCII on the host) is resident.
//
// Band k owns the sampled seed locations p in [b0, b1) (b0 a multiple of the step, so
// the global sampling phase is kept). Its window W = R[w0, w1) with
//   w0 = b0 - step (clamped at 0): the canonical rule reads at most `step` bases left of
//        a seed (e <= step, DESIGN.md canonical seed), so left extensions never leave W;
//   w1 = b1 + H, H = max(L, kHalo): a MEM whose canonical seed is in the band starts at
//        r <= p < b1, so when its right extension is cut at w1 its length is already
//        >= H >= L -- it is reported, and recognised as "open" (r + len == w1 < |R|).
// The window is packed, indexed over [b0, b1) (gpumem_index_build_range on the window)
// and searched against the whole of Q (gpumem_find_mems); every MEM is reported by
// exactly one band (its canonical seed's). Open MEMs are carried to the next band,
// whose window starts at b1 - step < w1, and their right extension is continued there
// (k_band_continue) until a mismatch, the end of R or Q, or the next window's end (open
// again). This replaces the paper's out-tile combining. The final set
// is re-sorted by (r, q) (bands overlap by < step in r).
#include "internal.h"
#include "device.cuh"

namespace gm {
namespace {

constexpr int kT = 256;

// Local triples of band k -> global (r + w0). open: r_local + len == wlen and more R
// follows (w1 < |R|): the right extension was cut at the window's end.
__global__ void __launch_bounds__(kT) k_band_place(const gpumem_triple *__restrict__ in, uint64_t n, uint64_t w0,
                                                   uint64_t wlen, int more, gpumem_triple *__restrict__ closed,
                                                   unsigned long long *__restrict__ n_closed,
                                                   gpumem_triple *__restrict__ open,
                                                   unsigned long long *__restrict__ n_open) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    gpumem_triple t = in[i];
    const bool is_open = more && uint64_t(t.r) + t.len == wlen;
    t.r = uint32_t(t.r + w0);
    if (is_open) open[atomicAdd(n_open, 1ull)] = t;
    else closed[atomicAdd(n_closed, 1ull)] = t;
}

// Continue the right extension of carried MEMs (global r, q, len so far) in the window
// W = words of R[w0, w0 + wlen): compare from (r + len, q + len) on; still open when the
// window's end is reached and more R follows.
__global__ void __launch_bounds__(kT) k_band_continue(const gpumem_triple *__restrict__ in, uint64_t n,
                                                      const uint64_t *__restrict__ W, uint64_t w0, uint64_t wlen,
                                                      int more, const uint64_t *__restrict__ Q, uint64_t nQ,
                                                      gpumem_triple *__restrict__ closed,
                                                      unsigned long long *__restrict__ n_closed,
                                                      gpumem_triple *__restrict__ open,
                                                      unsigned long long *__restrict__ n_open) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    gpumem_triple t = in[i];
    const uint64_t x = uint64_t(t.r) + t.len - w0;  // local start of the continuation (<= wlen)
    const uint64_t y = uint64_t(t.q) + t.len;
    const uint64_t lim_w = wlen - x, lim_q = nQ - y;
    const uint64_t lim = lim_w < lim_q ? lim_w : lim_q;
    uint64_t f = 0;
    while (f < lim) {
        const uint32_t run = lead_eq(win_fwd(W, x + f) ^ win_fwd(Q, y + f));
        f += run;
        if (run < 32) break;
    }
    if (f > lim) f = lim;
    t.len = uint32_t(t.len + f);
    const bool still_open = more && f == lim_w && lim_w <= lim_q;
    if (still_open) open[atomicAdd(n_open, 1ull)] = t;
    else closed[atomicAdd(n_closed, 1ull)] = t;
}

}  // namespace

cudaError_t band_place(const gpumem_triple *in, uint64_t n, uint64_t w0, uint64_t wlen, int more,
                       gpumem_triple *closed, unsigned long long *n_closed, gpumem_triple *open,
                       unsigned long long *n_open, cudaStream_t s) {
    if (!n) return cudaSuccess;
    pdl_launch(k_band_place, unsigned((n + kT - 1) / kT), kT, 0, s, in, n, w0, wlen, more, closed, n_closed, open,
               n_open);
    note_launch();
    return cudaGetLastError();
}

cudaError_t band_continue(const gpumem_triple *in, uint64_t n, const uint64_t *W, uint64_t w0, uint64_t wlen,
                          int more, const uint64_t *Q, uint64_t nQ, gpumem_triple *closed,
                          unsigned long long *n_closed, gpumem_triple *open, unsigned long long *n_open,
                          cudaStream_t s) {
    if (!n) return cudaSuccess;
    pdl_launch(k_band_continue, unsigned((n + kT - 1) / kT), kT, 0, s, in, n, W, w0, wlen, more, Q, nQ, closed,
               n_closed, open, n_open);
    note_launch();
    return cudaGetLastError();
}

}  // namespace gm
