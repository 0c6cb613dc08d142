// fasta.cu -- NEXT-F4 I/O around the path: multi-FASTA input whose record boundaries
// (and non-ACGT letters) break matches, and MUMmer-style 1-based text output
// (PAPER.md:64 §II-A MUMmer, :226 §IV-B "the I/O time is excluded").
//
// Input. gpumem_fasta_parse turns a multi-FASTA text into one ASCII sequence the MEM
// path can pack: the records in order, one separator base between consecutive records,
// and every non-ACGT letter (N, IUPAC codes) replaced by 'A'. The separators and the
// replaced letters are "masked" positions, kept as sorted half-open intervals. A match
// of the multi-record problem may not contain a masked position (a record end counts as
// a mismatch, reading R3; an N matches nothing, as in MUMmer).
//
// Why the path still finds them: a maximal run of the multi-record problem (a diagonal
// run of equal bases avoiding masked positions, bounded by a mismatch, a masked
// position or a sequence end) lies inside a maximal run of the concatenated sequences
// (masked letters read as 'A' may extend it), and is one of the pieces that cutting
// that run at every masked position leaves. A piece of length >= L lies in a run of
// length >= L, which the path reports. So the multi-record MEM set = the pieces >= L
// of the concatenation's MEMs cut at the masked positions of R and of Q
// (k_split_count / k_split_emit), re-sorted by (r, q).
//
// Output. gpumem_write_mummer prints, per query record in input order, a header line
// "> name" (and "> name Reverse" for reverse-strand matches) followed by one line per
// match "  ref_name  ref_pos  query_pos  len", positions 1-based inside their records,
// ordered by query position then reference record and position (MUMmer's mummer
// -maxmatch layout with several reference records; reverse-strand query positions are
// relative to the reverse complement of the query record, MUMmer's default).
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "internal.h"

namespace gm {
namespace {

constexpr int kT = 256;

struct Masks {
    const uint64_t *r, *q;   // [2i] begin, [2i+1] end, sorted, disjoint
    uint64_t nr, nq;         // interval counts
};

// first interval of m (n intervals) whose end > x
__device__ __forceinline__ uint64_t first_ending_after(const uint64_t *m, uint64_t n, uint64_t x) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (m[2 * mid + 1] <= x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// Walk the pieces of MEM t: cut at the masked intervals of R (on r + o) and of Q (on
// q + o), o in [0, len). emit(r, q, len) is called for every piece of length >= L.
template <class F>
__device__ __forceinline__ void pieces(const gpumem_triple &t, const Masks &M, uint32_t L, F emit) {
    uint64_t ir = first_ending_after(M.r, M.nr, t.r), iq = first_ending_after(M.q, M.nq, t.q);
    uint64_t o = 0;  // current piece starts at offset o
    const uint64_t end = t.len;
    while (o < end) {
        // next masked offset >= o on either axis (end if none)
        uint64_t cut = end, resume = end;
        if (ir < M.nr && M.r[2 * ir] < t.r + end) {
            const uint64_t b = M.r[2 * ir] > t.r + o ? M.r[2 * ir] - t.r : o;
            if (b < cut) { cut = b; resume = M.r[2 * ir + 1] - t.r; }
        }
        if (iq < M.nq && M.q[2 * iq] < t.q + end) {
            const uint64_t b = M.q[2 * iq] > t.q + o ? M.q[2 * iq] - t.q : o;
            if (b < cut) { cut = b; resume = M.q[2 * iq + 1] - t.q; }
            else if (b == cut) resume = max(resume, M.q[2 * iq + 1] - t.q);
        }
        if (cut - o >= L) emit(uint32_t(t.r + o), uint32_t(t.q + o), uint32_t(cut - o));
        if (cut >= end) break;
        o = min(resume, end);
        while (ir < M.nr && M.r[2 * ir + 1] <= t.r + o) ++ir;
        while (iq < M.nq && M.q[2 * iq + 1] <= t.q + o) ++iq;
    }
}

__global__ void __launch_bounds__(kT) k_split_count(const gpumem_triple *__restrict__ in, uint64_t n, Masks M,
                                                    uint32_t L, uint32_t *__restrict__ cnt) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    uint32_t c = 0;
    pieces(in[i], M, L, [&](uint32_t, uint32_t, uint32_t) { ++c; });
    cnt[i] = c;
}

__global__ void __launch_bounds__(kT) k_split_emit(const gpumem_triple *__restrict__ in, uint64_t n, Masks M,
                                                   uint32_t L, const uint32_t *__restrict__ off, uint32_t qbits,
                                                   uint64_t *__restrict__ keys, uint32_t *__restrict__ lens) {
    pdl_wait();
    const uint64_t i = uint64_t(blockIdx.x) * kT + threadIdx.x;
    if (i >= n) return;
    uint32_t o = off[i];
    pieces(in[i], M, L, [&](uint32_t r, uint32_t q, uint32_t len) {
        keys[o] = (uint64_t(r) << qbits) | q;
        lens[o] = len;
        ++o;
    });
}

// exclusive scan of cnt[0, n) into off (single CTA, kT items per round); total -> *tot
__global__ void __launch_bounds__(kT) k_split_scan(const uint32_t *__restrict__ cnt, uint64_t n,
                                                   uint32_t *__restrict__ off, unsigned long long *tot) {
    pdl_wait();
    __shared__ uint32_t ws[kT / 32];
    __shared__ unsigned long long carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t base = 0; base < n; base += kT) {
        const uint64_t i = base + threadIdx.x;
        const uint32_t x = i < n ? cnt[i] : 0;
        uint32_t inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31) ws[w] = inc;
        __syncthreads();
        uint32_t pre = 0, sum = 0;
        for (int k = 0; k < kT / 32; ++k) {
            if (k < w) pre += ws[k];
            sum += ws[k];
        }
        if (i < n) off[i] = uint32_t(carry) + pre + inc - x;
        __syncthreads();
        if (threadIdx.x == 0) carry += sum;
        __syncthreads();
    }
    if (threadIdx.x == 0) *tot = carry;
}

bool is_acgt(unsigned char c) {
    switch (c) {
        case 'A': case 'C': case 'G': case 'T': case 'a': case 'c': case 'g': case 't': return true;
        default: return false;
    }
}

// record index of concatenated position x (records sorted by start)
size_t record_of(const gpumem_fasta *f, uint64_t x) {
    return size_t(std::upper_bound(f->start.begin(), f->start.end(), x) - f->start.begin()) - 1;
}

}  // namespace

cudaError_t split_masked(const gpumem_triple *in, uint64_t n, const uint64_t *mr, uint64_t nmr, const uint64_t *mq,
                         uint64_t nmq, uint32_t L, uint32_t qbits, uint32_t *cnt, uint32_t *off,
                         unsigned long long *d_total, uint64_t *keys, uint32_t *lens, cudaStream_t s) {
    const Masks M{mr, mq, nmr, nmq};
    const unsigned blocks = unsigned((n + kT - 1) / kT);
    if (!n) return keys ? cudaSuccess : cudaMemsetAsync(d_total, 0, 8, s);
    if (!keys) {
        pdl_launch(k_split_count, blocks, kT, 0, s, in, n, M, L, cnt);
        pdl_launch(k_split_scan, 1, kT, 0, s, static_cast<const uint32_t *>(cnt), n, off, d_total);
        note_launch(2);
    } else {
        pdl_launch(k_split_emit, blocks, kT, 0, s, in, n, M, L, static_cast<const uint32_t *>(off), qbits, keys, lens);
        note_launch(1);
    }
    return cudaGetLastError();
}

}  // namespace gm

using namespace gm;

extern "C" {

gpumem_status gpumem_fasta_parse(const char *text, uint64_t n, gpumem_fasta **out) {
    if (!out) return fail(GPUMEM_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (!text && n) return fail(GPUMEM_ERR_ARG, "text is NULL");
    auto *f = new gpumem_fasta{};
    f->magic = kMagicFasta;
    uint64_t i = 0;
    bool any = false;
    while (i < n) {
        // header line
        while (i < n && (text[i] == '\n' || text[i] == '\r')) ++i;
        if (i >= n) break;
        if (text[i] != '>') {
            delete f;
            return fail(GPUMEM_ERR_ARG, "FASTA: expected '>' at byte %llu", (unsigned long long)i);
        }
        uint64_t e = i + 1;
        while (e < n && text[e] != '\n' && text[e] != '\r') ++e;
        std::string name(text + i + 1, text + e);
        const size_t sp = name.find_first_of(" \t");  // the name is the first word
        if (sp != std::string::npos) name.resize(sp);
        if (any) {  // one masked separator base between records
            const uint64_t p = f->seq.size();
            if (!f->mask.empty() && f->mask.back() == p) f->mask.back() = p + 1;
            else {
                f->mask.push_back(p);
                f->mask.push_back(p + 1);
            }
            f->seq.push_back('A');
        }
        any = true;
        f->names.push_back(name);
        f->start.push_back(f->seq.size());
        i = e;
        // sequence lines up to the next header
        while (i < n && text[i] != '>') {
            const unsigned char c = static_cast<unsigned char>(text[i]);
            if (c == '\n' || c == '\r' || c == ' ' || c == '\t') {
                ++i;
                continue;
            }
            if (c < 33 || c > 126) {
                delete f;
                return fail(GPUMEM_ERR_ALPHABET, "FASTA: byte %u at %llu is not a sequence letter", unsigned(c),
                            (unsigned long long)i);
            }
            const uint64_t p = f->seq.size();
            if (is_acgt(c)) {
                f->seq.push_back(char(c & 0xDF));
            } else {  // N / IUPAC: masked, matches nothing
                if (!f->mask.empty() && f->mask.back() == p) f->mask.back() = p + 1;
                else {
                    f->mask.push_back(p);
                    f->mask.push_back(p + 1);
                }
                f->seq.push_back('A');
            }
            ++i;
        }
        f->len.push_back(f->seq.size() - f->start.back());
    }
    if (f->seq.size() >= (1ull << 32)) {
        delete f;
        return fail(GPUMEM_ERR_RANGE, "FASTA: %llu bases in total exceed 2^32-1", (unsigned long long)f->seq.size());
    }
    *out = f;
    return GPUMEM_OK;
}

gpumem_status gpumem_fasta_info(const gpumem_fasta *f, uint64_t *n_records, const char **seq, uint64_t *seq_len,
                                uint64_t *n_masked) {
    if (!f || f->magic != kMagicFasta) return fail(GPUMEM_ERR_ARG, "not a gpumem_fasta");
    if (n_records) *n_records = f->names.size();
    if (seq) *seq = f->seq.data();
    if (seq_len) *seq_len = f->seq.size();
    if (n_masked) *n_masked = f->mask.size() / 2;
    return GPUMEM_OK;
}

gpumem_status gpumem_fasta_record(const gpumem_fasta *f, uint64_t i, const char **name, uint64_t *start,
                                  uint64_t *len) {
    if (!f || f->magic != kMagicFasta) return fail(GPUMEM_ERR_ARG, "not a gpumem_fasta");
    if (i >= f->names.size()) return fail(GPUMEM_ERR_RANGE, "record %llu of %zu", (unsigned long long)i,
                                          f->names.size());
    if (name) *name = f->names[i].c_str();
    if (start) *start = f->start[i];
    if (len) *len = f->len[i];
    return GPUMEM_OK;
}

gpumem_status gpumem_write_mummer(const gpumem_triple *fwd, uint64_t n_fwd, const gpumem_triple *rev, uint64_t n_rev,
                                  const gpumem_fasta *R, const gpumem_fasta *Q, const char *path) {
    if (!R || R->magic != kMagicFasta || !Q || Q->magic != kMagicFasta)
        return fail(GPUMEM_ERR_ARG, "R and Q must be gpumem_fasta handles");
    if (!path) return fail(GPUMEM_ERR_ARG, "path is NULL");
    if ((n_fwd && !fwd) || (n_rev && !rev)) return fail(GPUMEM_ERR_ARG, "NULL triples");
    struct Row {
        size_t qrec;
        uint64_t qpos;
        size_t rrec;
        uint64_t rpos, len;
    };
    auto rows_of = [&](const gpumem_triple *t, uint64_t n, bool reverse, std::vector<Row> &rows) -> bool {
        const uint64_t qlen_all = Q->seq.size();
        for (uint64_t i = 0; i < n; ++i) {
            // reverse strand: the path ran on the reverse complement of the whole
            // concatenated query; map back to the record and the position inside the
            // reverse complement of that record
            const uint64_t qg = reverse ? qlen_all - (uint64_t(t[i].q) + t[i].len) : t[i].q;
            const size_t qr = record_of(Q, qg), rr = record_of(R, t[i].r);
            const uint64_t qoff = qg - Q->start[qr], roff = t[i].r - R->start[rr];
            if (qoff + t[i].len > Q->len[qr] || roff + t[i].len > R->len[rr]) return false;  // crosses a record
            const uint64_t qpos = reverse ? Q->len[qr] - (qoff + t[i].len) : qoff;
            rows.push_back(Row{qr, qpos, rr, roff, t[i].len});
        }
        std::sort(rows.begin(), rows.end(), [](const Row &a, const Row &b) {
            if (a.qrec != b.qrec) return a.qrec < b.qrec;
            if (a.qpos != b.qpos) return a.qpos < b.qpos;
            if (a.rrec != b.rrec) return a.rrec < b.rrec;
            return a.rpos < b.rpos;
        });
        return true;
    };
    std::vector<Row> f, r;
    if (!rows_of(fwd, n_fwd, false, f) || !rows_of(rev, n_rev, true, r))
        return fail(GPUMEM_ERR_ARG, "a match crosses a record boundary (split with gpumem_split_masked first)");
    FILE *fp = fopen(path, "w");
    if (!fp) return fail(GPUMEM_ERR_ARG, "cannot open %s for writing", path);
    size_t fi = 0, ri = 0;
    for (size_t qr = 0; qr < Q->names.size(); ++qr) {
        fprintf(fp, "> %s\n", Q->names[qr].c_str());
        for (; fi < f.size() && f[fi].qrec == qr; ++fi)
            fprintf(fp, "  %s\t%llu\t%llu\t%llu\n", R->names[f[fi].rrec].c_str(), (unsigned long long)(f[fi].rpos + 1),
                    (unsigned long long)(f[fi].qpos + 1), (unsigned long long)f[fi].len);
        if (rev) {
            fprintf(fp, "> %s Reverse\n", Q->names[qr].c_str());
            for (; ri < r.size() && r[ri].qrec == qr; ++ri)
                fprintf(fp, "  %s\t%llu\t%llu\t%llu\n", R->names[r[ri].rrec].c_str(),
                        (unsigned long long)(r[ri].rpos + 1), (unsigned long long)(r[ri].qpos + 1),
                        (unsigned long long)r[ri].len);
        }
    }
    const bool ok = fclose(fp) == 0;
    return ok ? GPUMEM_OK : fail(GPUMEM_ERR_ARG, "write error on %s", path);
}

}  // extern "C"
