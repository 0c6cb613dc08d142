// oracle/mem_oracle.cpp -- CPU ORACLE. TEST INFRASTRUCTURE ONLY.
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
// --impl reference legs may load this library. The product path
// (paper_conf_ipps_abu_dolehkac14_b200/, libgpumem.so) never links, imports
// or calls it, and this file shares no code, header, table or helper with
// the CUDA path. It works on ASCII bytes, std::string_view hash keys and
// char-by-char loops: no 2-bit packing, no word XOR, no canonical-seed rule.
//
// Functions and the passages they follow (PAPER.md = /root/reference/PAPER.md):
//
//  oracle_mems   GPUMEM's method as the paper states it, step by step
//                (SURVEY.md §8(c) C2):
//                  1. validate, step = L - ls + 1                (Eq. 1, :86-90)
//                  2. index every step-th ls-mer of R            (:84-90, Alg 1 :102)
//                  3. for every query position q, every indexed r with the
//                     same ls-mer: extend left and right char by char until a
//                     mismatch or a sequence end                 (:151-153, :171-173)
//                  4. keep length >= L                            (:53-56, :173)
//                  5. duplicate elimination by sort + unique      (:153 "not to
//                     extract a MEM more than once"; :185 final MEMs)
//                Pinned by: brute force (below), hand-worked examples in
//                tests/golden/, homopolymer closed form, R/Q swap symmetry,
//                planted ground truth, random-MEM expectation.
//  brute_mems    The MEM definition (with sequence ends
//                counting as mismatches, reading R3) written out:
//                walk every diagonal r - q and emit each maximal run of equal
//                characters of length >= L. O(|R||Q|). Pinned by the
//                hand-worked examples and the homopolymer closed form.
//  oracle_index  Algorithm 1 as a sequential counting
//                sort: count each sampled seed into ptrs[s+1], prefix-sum,
//                place locations in increasing order (so step 4's per-seed
//                sort is satisfied by construction). Seed integer: A=00, C=01,
//                G=10, T=11 (:92), first base most significant (reading R5).
//                Pinned by the hand-worked W2 index in tests/golden/ and the
//                invariants of :84 (ptrs monotone, last == |locs|, bucket s
//                holds exactly the sampled locations whose ls-mer is s).
//
// Errors: return value < 0: -1 bad argument, -2 alphabet, -3 range/alloc.

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <string>
#include <string_view>
#include <unordered_map>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

struct Triple {
    uint32_t r, q, len;
    bool operator<(const Triple& o) const {
        return r != o.r ? r < o.r : (q != o.q ? q < o.q : len < o.len);
    }
    bool operator==(const Triple& o) const { return r == o.r && q == o.q && len == o.len; }
};

// Alphabet Sigma = {A,C,G,T}; lowercase folded (reading R4).
bool normalise(const char* s, uint64_t n, std::string& out) {
    out.resize(n);
    for (uint64_t i = 0; i < n; ++i) {
        char c = s[i];
        if (c >= 'a' && c <= 'z') c = char(c - 'a' + 'A');
        if (c != 'A' && c != 'C' && c != 'G' && c != 'T') return false;
        out[i] = c;
    }
    return true;
}

int set_threads(int threads) {
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
    return omp_get_max_threads();
#else
    (void)threads;
    return 1;
#endif
}

uint32_t* export_triples(const std::vector<Triple>& v) {
    uint32_t* out = static_cast<uint32_t*>(std::malloc(sizeof(uint32_t) * 3 * (v.size() ? v.size() : 1)));
    if (!out) return nullptr;
    for (size_t i = 0; i < v.size(); ++i) {
        out[3 * i] = v[i].r;
        out[3 * i + 1] = v[i].q;
        out[3 * i + 2] = v[i].len;
    }
    return out;
}

}  // namespace

extern "C" {

int oracle_num_threads(int threads) { return set_threads(threads); }

void oracle_free(void* p) { std::free(p); }

// MEMs (r, q, len) with len >= L whose query start q lies in [q_begin, q_end),
// sorted by (r, q). step == 0 means the paper's maximum step L - ls + 1.
int64_t oracle_mems(const char* Rs, uint64_t nR, const char* Qs, uint64_t nQ,
                    uint32_t L, uint32_t ls, uint32_t step,
                    uint64_t q_begin, uint64_t q_end, int threads, uint32_t** out) {
    *out = nullptr;
    if (L < 1 || ls < 1 || ls > L) return -1;                       // Eq. (1) needs ls <= L
    if (step == 0) step = L - ls + 1;                                // max step, :90
    if (step > L - ls + 1) return -1;                                // Eq. (1), :88
    if (nR >= (1ull << 32) || nQ >= (1ull << 32)) return -3;         // 32-bit locations, :86
    std::string R, Q;
    if (!normalise(Rs, nR, R) || !normalise(Qs, nQ, Q)) return -2;
    if (q_end > nQ) q_end = nQ;
    std::vector<Triple> all;
    if (nR >= ls && nQ >= ls && q_begin < q_end) {
        // Step 2: hash index of every step-th ls-mer of R.
        std::unordered_map<std::string_view, std::vector<uint32_t>> H;
        H.reserve((nR - ls) / step + 1);
        const std::string_view Rv(R), Qv(Q);
        for (uint64_t p = 0; p + ls <= nR; p += step) H[Rv.substr(p, ls)].push_back(uint32_t(p));
        // Step 3: every query position whose seed could lie in a MEM starting in
        // [q_begin, q_end): a MEM of length >= L contains a sampled seed within
        // its first `step` seed positions (Eq. 1), so scan up to q_end + step - 1.
        const uint64_t q_lo = q_begin;
        const uint64_t q_hi = std::min<uint64_t>(q_end + step - 1, nQ - ls + 1);
        set_threads(threads);
        std::vector<std::vector<Triple>> parts;
#pragma omp parallel
        {
#ifdef _OPENMP
            const int nt = omp_get_num_threads(), tid = omp_get_thread_num();
#else
            const int nt = 1, tid = 0;
#endif
#pragma omp single
            parts.resize(nt);
            std::vector<Triple>& mine = parts[tid];
#pragma omp for schedule(dynamic, 4096)
            for (int64_t qi = int64_t(q_lo); qi < int64_t(q_hi); ++qi) {
                const uint64_t q = uint64_t(qi);
                auto it = H.find(Qv.substr(q, ls));
                if (it == H.end()) continue;
                for (uint32_t p : it->second) {
                    uint64_t a = 0;  // left: R[p-k] == Q[q-k], k = 1..
                    while (a < p && a < q && R[p - a - 1] == Q[q - a - 1]) ++a;
                    uint64_t b = ls; // right: seed matches by construction, then extend
                    while (p + b < nR && q + b < nQ && R[p + b] == Q[q + b]) ++b;
                    const uint64_t len = a + b;
                    const uint64_t qs = q - a;
                    if (len >= L && qs >= q_begin && qs < q_end)
                        mine.push_back(Triple{uint32_t(p - a), uint32_t(qs), uint32_t(len)});
                }
            }
        }
        size_t tot = 0;
        for (auto& v : parts) tot += v.size();
        all.reserve(tot);
        for (auto& v : parts) all.insert(all.end(), v.begin(), v.end());
    }
    // Step 5: a MEM is found once per sampled seed inside it; keep one copy.
    std::sort(all.begin(), all.end());
    all.erase(std::unique(all.begin(), all.end()), all.end());
    *out = export_triples(all);
    if (!*out) return -3;
    return int64_t(all.size());
}

// Brute force over the definition: every diagonal, every maximal run.
int64_t brute_mems(const char* Rs, uint64_t nR, const char* Qs, uint64_t nQ, uint32_t L,
                   int threads, uint32_t** out) {
    *out = nullptr;
    if (L < 1) return -1;
    if (nR >= (1ull << 32) || nQ >= (1ull << 32)) return -3;
    std::string R, Q;
    if (!normalise(Rs, nR, R) || !normalise(Qs, nQ, Q)) return -2;
    std::vector<Triple> all;
    if (nR > 0 && nQ > 0) {
        set_threads(threads);
        const int64_t dmin = -int64_t(nQ) + 1, dmax = int64_t(nR) - 1;  // d = r - q
        std::vector<std::vector<Triple>> parts;
#pragma omp parallel
        {
#ifdef _OPENMP
            const int nt = omp_get_num_threads(), tid = omp_get_thread_num();
#else
            const int nt = 1, tid = 0;
#endif
#pragma omp single
            parts.resize(nt);
            std::vector<Triple>& mine = parts[tid];
#pragma omp for schedule(dynamic, 64)
            for (int64_t d = dmin; d <= dmax; ++d) {
                uint64_t r = d >= 0 ? uint64_t(d) : 0, q = d >= 0 ? 0 : uint64_t(-d);
                uint64_t run = 0;  // length of the current run of equal characters
                for (; r < nR && q < nQ; ++r, ++q) {
                    if (R[r] == Q[q]) {
                        ++run;
                    } else {
                        if (run >= L) mine.push_back(Triple{uint32_t(r - run), uint32_t(q - run), uint32_t(run)});
                        run = 0;
                    }
                }
                if (run >= L) mine.push_back(Triple{uint32_t(r - run), uint32_t(q - run), uint32_t(run)});
            }
        }
        for (auto& v : parts) all.insert(all.end(), v.begin(), v.end());
    }
    std::sort(all.begin(), all.end());
    *out = export_triples(all);
    if (!*out) return -3;
    return int64_t(all.size());
}

// Algorithm 1 (whole R, one "tile row"): ptrs has 4^ls + 1 entries, locs
// n_locs = ceil((nR - ls + 1) / step) entries (0 if nR < ls).
int64_t oracle_index(const char* Rs, uint64_t nR, uint32_t ls, uint32_t step,
                     uint32_t* ptrs, uint32_t* locs) {
    if (ls < 1 || ls > 15 || step < 1) return -1;
    std::string R;
    if (!normalise(Rs, nR, R)) return -2;
    const uint64_t nb = 1ull << (2 * ls);
    auto enc = [](char c) -> uint64_t {  // A=00 C=01 G=10 T=11
        return c == 'A' ? 0 : c == 'C' ? 1 : c == 'G' ? 2 : 3;
    };
    auto seed = [&](uint64_t l) {        // s <- (R_l, ..., R_{l+ls-1}), first base most significant
        uint64_t s = 0;
        for (uint32_t i = 0; i < ls; ++i) s = s * 4 + enc(R[l + i]);
        return s;
    };
    // Step 1: counts into ptrs[s+1]
    for (uint64_t s = 0; s <= nb; ++s) ptrs[s] = 0;
    uint64_t n = 0;
    for (uint64_t l = 0; l + ls <= nR; l += step, ++n) ptrs[seed(l) + 1] += 1;
    // Step 2: prefix sum
    for (uint64_t s = 1; s <= nb; ++s) ptrs[s] += ptrs[s - 1];
    // Step 3 (+4): fill with a cursor copy, locations visited in increasing order
    std::vector<uint32_t> temp(ptrs, ptrs + nb);
    for (uint64_t l = 0; l + ls <= nR; l += step) locs[temp[seed(l)]++] = uint32_t(l);
    return int64_t(n);
}

}  // extern "C"

// MUMs (a match that "appears only once in both sequences ... and cannot be
// extended to either directions"): the MEMs of oracle_mems whose string occurs exactly
// once in R and exactly once in Q, counted by plain substring search (std::string::find,
// overlapping occurrences). Pinned by the hand-worked W2 MUM fixture and the Python twin.
extern "C" int64_t oracle_mums(const char* Rs, uint64_t nR, const char* Qs, uint64_t nQ, uint32_t L,
                               uint32_t ls, int threads, uint32_t** out) {
    uint32_t* mem = nullptr;
    const int64_t n = oracle_mems(Rs, nR, Qs, nQ, L, ls, 0, 0, nQ, threads, &mem);
    *out = nullptr;
    if (n < 0) return n;
    std::string R, Q;
    normalise(Rs, nR, R);
    normalise(Qs, nQ, Q);
    auto occurs_once = [](const std::string& T, const std::string& S) {
        size_t pos = T.find(S);
        if (pos == std::string::npos) return false;
        return T.find(S, pos + 1) == std::string::npos;
    };
    std::vector<Triple> keep;
    for (int64_t i = 0; i < n; ++i) {
        const Triple t{mem[3 * i], mem[3 * i + 1], mem[3 * i + 2]};
        const std::string S = R.substr(t.r, t.len);
        if (occurs_once(R, S) && occurs_once(Q, S)) keep.push_back(t);
    }
    std::free(mem);
    *out = export_triples(keep);
    return *out ? int64_t(keep.size()) : -3;
}

// Rare MEMs (PAPER.md:23 "maximal rare matches"; :286 "unique and rare exact match
// extraction", future work; reading R23): the MEMs of oracle_mems whose string
// occurs at most k times in R and at most k times in Q, occurrences counted by plain
// substring search (std::string::find from every position, overlapping occurrences).
// k = 1 is oracle_mums. Pinned by the hand-worked W3 fixture (tests/golden/w3_rare.txt),
// the homopolymer closed form and the Python twin.
extern "C" int64_t oracle_rare(const char* Rs, uint64_t nR, const char* Qs, uint64_t nQ, uint32_t L,
                               uint32_t ls, uint32_t k, int threads, uint32_t** out) {
    uint32_t* mem = nullptr;
    *out = nullptr;
    if (k < 1) return -1;
    const int64_t n = oracle_mems(Rs, nR, Qs, nQ, L, ls, 0, 0, nQ, threads, &mem);
    if (n < 0) return n;
    std::string R, Q;
    normalise(Rs, nR, R);
    normalise(Qs, nQ, Q);
    auto at_most_k = [k](const std::string& T, const std::string& S) {
        uint32_t c = 0;
        for (size_t pos = T.find(S); pos != std::string::npos; pos = T.find(S, pos + 1))
            if (++c > k) return false;
        return true;
    };
    std::vector<Triple> keep;
    for (int64_t i = 0; i < n; ++i) {
        const Triple t{mem[3 * i], mem[3 * i + 1], mem[3 * i + 2]};
        const std::string S = R.substr(t.r, t.len);
        if (at_most_k(R, S) && at_most_k(Q, S)) keep.push_back(t);
    }
    std::free(mem);
    *out = export_triples(keep);
    return *out ? int64_t(keep.size()) : -3;
}
