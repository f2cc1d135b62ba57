/* gen_common.h — seeded, counter-based synthetic INPUT generators (test/bench infrastructure).
 *
 * This module produces the records that both sides consume: the CPU oracle (oracle/) reads
 * them from the host implementation (gen_host.cpp), the CUDA path reads them from the device
 * implementation (gen_dev.cu). Both implementations include THIS header, so record i is the
 * same pure function of (seed, i) on either side. The module holds none of the method's
 * arithmetic: no table hash, no bucket mapping, no grouping — only record synthesis and the
 * closed-form "by construction" counts of the exact-count families (DESIGN.md §Input recipe).
 *
 * Families (SURVEY.md §8(d) "Generators", with the integer-only readings listed in DESIGN.md):
 *   WORDS  — key = spelling of a Zipf-ranked word (C1, C2, C4);     PAPER.md L217 (Word Count)
 *   URLS   — key = a synthetic URL of a Zipf-ranked page (C3);       PAPER.md L213 (Page View Count)
 *   PAIRS  — key = 8-byte splitmix64(rank), value = 8-byte u64 (C5)
 * Rank of record j: idx = perm(j) (seeded Feistel bijection of [0,n)), rank = the r with
 * cum[r-1] <= idx < cum[r], where cum[r] = sum_{s<=r} c_s and c_s is the exact count of rank s
 * (c_s = floor(C / s^alpha), computed once on the host; UNIFORM: c_s = m for all s).
 */
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD static inline
#endif

enum { GEN_WORDS = 0, GEN_URLS = 1, GEN_PAIRS = 2 };

/* Parameters of one synthetic stream. Pointers are host or device as the call states. */
typedef struct gen_params {
    int32_t  family;        /* GEN_WORDS / GEN_URLS / GEN_PAIRS */
    int32_t  with_doc_vals; /* WORDS only: value = u32 doc id of the record (C4 inverted index) */
    uint64_t seed;
    uint64_t n;             /* records in the whole (global) stream */
    uint64_t n_ranks;       /* ranks with c_r >= 1 (ranks are 1..n_ranks) */
    uint64_t uniform_m;     /* if > 0: c_r = uniform_m for every rank, cum unused */
    const uint64_t* cum;    /* cum[0..n_ranks], cum[0] = 0, cum[n_ranks] = n */
    uint64_t n_docs;        /* with_doc_vals: number of documents */
    const uint64_t* doc_start; /* doc_start[0..n_docs], doc d = records [doc_start[d], doc_start[d+1]) */
} gen_params;

/* ---- counter-based randomness (SplitMix64 finalizer) ---- */
GEN_HD uint64_t gen_mix64(uint64_t z) {
    z ^= z >> 30; z *= 0xbf58476d1ce4e5b9ULL;
    z ^= z >> 27; z *= 0x94d049bb133111ebULL;
    z ^= z >> 31; return z;
}
GEN_HD uint64_t gen_rnd(uint64_t seed, uint64_t stream, uint64_t i) {
    return gen_mix64(gen_mix64(seed * 0x9E3779B97F4A7C15ULL + stream) ^ (i * 0xD1B54A32D192ED03ULL + 0x632BE59BD9B4E019ULL));
}
enum { GEN_S_PERM = 0x5045524dULL, GEN_S_URL = 0x55524cULL, GEN_S_VAL = 0x56414cULL, GEN_S_DOC = 0x444f43ULL,
       GEN_S_KEY = 0x4b4559ULL };

/* ---- seeded bijection of [0, n): balanced 4-round Feistel on 2k bits + cycle walking ---- */
GEN_HD int gen_perm_half_bits(uint64_t n) {
    int bits = 2;
    while (bits < 64 && (1ULL << bits) < n) bits += 2;
    return bits / 2;
}
GEN_HD uint64_t gen_feistel(uint64_t x, int half, uint64_t seed) {
    uint64_t mask = (half >= 32) ? 0xffffffffULL : ((1ULL << half) - 1);
    uint64_t L = x >> half, R = x & mask;
    for (int r = 0; r < 4; ++r) {
        uint64_t k = gen_rnd(seed, GEN_S_PERM, (uint64_t)r);
        uint64_t nL = R, nR = L ^ (gen_mix64(R ^ k) & mask);
        L = nL; R = nR;
    }
    return (L << half) | R;
}
GEN_HD uint64_t gen_feistel_inv(uint64_t y, int half, uint64_t seed) {
    uint64_t mask = (half >= 32) ? 0xffffffffULL : ((1ULL << half) - 1);
    uint64_t L = y >> half, R = y & mask;
    for (int r = 3; r >= 0; --r) {
        uint64_t k = gen_rnd(seed, GEN_S_PERM, (uint64_t)r);
        uint64_t pR = L, pL = R ^ (gen_mix64(L ^ k) & mask);
        L = pL; R = pR;
    }
    return (L << half) | R;
}
GEN_HD uint64_t gen_perm(uint64_t j, uint64_t n, uint64_t seed) {
    int half = gen_perm_half_bits(n);
    uint64_t y = gen_feistel(j, half, seed);
    while (y >= n) y = gen_feistel(y, half, seed);
    return y;
}
GEN_HD uint64_t gen_perm_inv(uint64_t idx, uint64_t n, uint64_t seed) {
    int half = gen_perm_half_bits(n);
    uint64_t y = gen_feistel_inv(idx, half, seed);
    while (y >= n) y = gen_feistel_inv(y, half, seed);
    return y;
}

/* rank (1-based) of multiset position idx: smallest r with cum[r] > idx */
GEN_HD uint64_t gen_rank_of(const gen_params* p, uint64_t idx) {
    if (p->uniform_m) return idx / p->uniform_m + 1;
    uint64_t lo = 1, hi = p->n_ranks;
    while (lo < hi) {
        uint64_t mid = lo + ((hi - lo) >> 1);
        if (p->cum[mid] > idx) hi = mid; else lo = mid + 1;
    }
    return lo;
}
GEN_HD uint64_t gen_rank(const gen_params* p, uint64_t j) {
    return gen_rank_of(p, gen_perm(j, p->n, p->seed));
}

/* ---- WORDS: spelling of rank r >= 1 ----
 * L(r) = min(16, max(#base-26 digits of r, 2 + floor(log2 r / 2))); letters = base-26 digits
 * of r, most significant first, left-padded with 'a'. Injective: equal lengths => distinct
 * numerals. */
GEN_HD uint32_t gen_word_len(uint64_t r) {
    uint32_t d = 1; uint64_t p = 26;
    while (d < 16 && p <= r) { p *= 26; ++d; }
    int lg = 63; while (lg > 0 && !((r >> lg) & 1)) --lg;
    uint32_t b = 2 + (uint32_t)(lg / 2);
    uint32_t L = d > b ? d : b;
    return L < 16 ? L : 16;
}
GEN_HD void gen_word_spell(uint64_t r, uint32_t L, uint8_t* out) {
    for (int i = (int)L - 1; i >= 0; --i) { out[i] = (uint8_t)('a' + (r % 26)); r /= 26; }
}

/* ---- URLS: "https://h" + hex4 + ".example/" + base36(r) + "/" + base36 padding to L(r) ----
 * L(r) = 24 + a%32 + b%32 + (c%8==0 ? d%161 : 0), clamped to [prefix_len, 256] (mean ~65 B). */
GEN_HD uint32_t gen_b36_len(uint64_t r) { uint32_t k = 1; while (r >= 36) { r /= 36; ++k; } return k; }
GEN_HD uint32_t gen_url_len(const gen_params* p, uint64_t r) {
    uint64_t h = gen_rnd(p->seed, GEN_S_URL, r);
    uint32_t L = 24 + (uint32_t)(h & 31) + (uint32_t)((h >> 5) & 31) + ((((h >> 10) & 7) == 0) ? (uint32_t)((h >> 13) % 161) : 0);
    uint32_t pre = 23 + gen_b36_len(r);
    if (L < pre) L = pre;
    if (L > 256) L = 256;
    return L;
}
GEN_HD void gen_url_spell(const gen_params* p, uint64_t r, uint32_t L, uint8_t* out) {
    const char* b36 = "0123456789abcdefghijklmnopqrstuvwxyz";
    const char* hx = "0123456789abcdef";
    uint64_t h = gen_rnd(p->seed, GEN_S_URL, r);
    uint32_t host = (uint32_t)(h >> 48);
    const char* a = "https://h"; uint32_t q = 0;
    for (int i = 0; i < 9; ++i) out[q++] = (uint8_t)a[i];
    for (int i = 3; i >= 0; --i) out[q++] = (uint8_t)hx[(host >> (4 * i)) & 15];
    const char* e = ".example/";
    for (int i = 0; i < 9; ++i) out[q++] = (uint8_t)e[i];
    uint32_t k = gen_b36_len(r); uint64_t t = r;
    for (int i = (int)k - 1; i >= 0; --i) { out[q + i] = (uint8_t)b36[t % 36]; t /= 36; }
    q += k; out[q++] = '/';
    for (; q < L; ++q) out[q] = (uint8_t)b36[gen_mix64(h ^ (uint64_t)q) % 36];
}

/* ---- raw text (word streams): the separator written after word j — '\n' with p = 1/10, else
 * ' ' (SURVEY §8(d) C1 recipe) — so record j's word starts at text byte offs[j] + j ---- */
GEN_HD uint8_t gen_text_sep(const gen_params* p, uint64_t j) {
    return (gen_rnd(p->seed, 0x7e47ULL, j) % 10 == 0) ? (uint8_t)'\n' : (uint8_t)' ';
}

/* ---- PAIRS: key = splitmix64 finalizer of rank (bijective on u64), value = lo32 random ---- */
GEN_HD uint64_t gen_pair_key(uint64_t r) { return gen_mix64(r); }
GEN_HD uint64_t gen_pair_val(const gen_params* p, uint64_t j) { return gen_rnd(p->seed, GEN_S_VAL, j) & 0xffffffffULL; }

/* key length of record j (bytes) */
GEN_HD uint32_t gen_key_len_of_rank(const gen_params* p, uint64_t r) {
    if (p->family == GEN_WORDS) return gen_word_len(r);
    if (p->family == GEN_URLS) return gen_url_len(p, r);
    return 8;
}
GEN_HD void gen_key_spell(const gen_params* p, uint64_t r, uint32_t L, uint8_t* out) {
    if (p->family == GEN_WORDS) gen_word_spell(r, L, out);
    else if (p->family == GEN_URLS) gen_url_spell(p, r, L, out);
    else { uint64_t k = gen_pair_key(r); for (int i = 0; i < 8; ++i) out[i] = (uint8_t)(k >> (8 * i)); }
}
/* doc id of record j (with_doc_vals): largest d with doc_start[d] <= j */
GEN_HD uint64_t gen_doc_of(const gen_params* p, uint64_t j) {
    uint64_t lo = 0, hi = p->n_docs - 1;
    while (lo < hi) {
        uint64_t mid = lo + ((hi - lo + 1) >> 1);
        if (p->doc_start[mid] <= j) lo = mid; else hi = mid - 1;
    }
    return lo;
}
/* document length in words (C4): 512 + rnd % 1025 */
GEN_HD uint64_t gen_doc_len(uint64_t seed, uint64_t d) { return 512 + gen_rnd(seed, GEN_S_DOC, d) % 1025; }
