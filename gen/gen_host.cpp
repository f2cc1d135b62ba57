// gen_host.cpp — host implementation of the synthetic input generators (gen_common.h).
// Test/bench infrastructure shared by the oracle side and the CUDA side; no method arithmetic.
#include "gen_common.h"
#include <string.h>
#include <omp.h>

extern "C" {

// out_lens[i] = key length of rank r0 + i (used to size workloads on the host).
void gen_key_lens_of_ranks_host(const gen_params* p, uint64_t r0, uint64_t cnt, uint32_t* out_lens) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) out_lens[i] = gen_key_len_of_rank(p, r0 + (uint64_t)i);
}

// Key bytes of rank r (caller buffer >= 256 B); returns its length.
uint32_t gen_spell_rank_host(const gen_params* p, uint64_t r, uint8_t* out) {
    uint32_t L = gen_key_len_of_rank(p, r);
    gen_key_spell(p, r, L, out);
    return L;
}

// ranks[i] = rank of record j0 + i.
void gen_ranks_host(const gen_params* p, uint64_t j0, uint64_t cnt, uint64_t* ranks) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) ranks[i] = gen_rank(p, j0 + (uint64_t)i);
}

// out[i] = perm^{-1}(idx[i]) : the record holding multiset position idx[i].
void gen_perm_inv_host(const gen_params* p, const uint64_t* idx, uint64_t cnt, uint64_t* out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) out[i] = gen_perm_inv(idx[i], p->n, p->seed);
}
void gen_perm_host(const gen_params* p, const uint64_t* j, uint64_t cnt, uint64_t* out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) out[i] = gen_perm(j[i], p->n, p->seed);
}

// Record values for records j[i] (PAIRS: u64 value; WORDS+docs: doc id) — closed-form helpers.
void gen_vals_of_records_host(const gen_params* p, const uint64_t* j, uint64_t cnt, uint64_t* out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i)
        out[i] = (p->family == GEN_PAIRS) ? gen_pair_val(p, j[i]) : gen_doc_of(p, j[i]);
}

// offs[0..cnt]: offs[0] = 0, offs[i+1] = offs[i] + len(key of record j0+i). Returns offs[cnt].
uint64_t gen_offsets_host(const gen_params* p, uint64_t j0, uint64_t cnt, uint64_t* offs) {
    offs[0] = 0;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) offs[i + 1] = gen_key_len_of_rank(p, gen_rank(p, j0 + (uint64_t)i));
    for (uint64_t i = 0; i < cnt; ++i) offs[i + 1] += offs[i];
    return offs[cnt];
}

// Key bytes (CSR with offs from gen_offsets_host) and values: PAIRS -> 8 B LE u64 per record,
// WORDS with_doc_vals -> 4 B LE u32 doc id per record; vals may be NULL.
void gen_keys_host(const gen_params* p, uint64_t j0, uint64_t cnt, const uint64_t* offs, uint8_t* keys, uint8_t* vals) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) {
        uint64_t j = j0 + (uint64_t)i;
        uint64_t r = gen_rank(p, j);
        gen_key_spell(p, r, (uint32_t)(offs[i + 1] - offs[i]), keys + offs[i]);
        if (vals) {
            if (p->family == GEN_PAIRS) { uint64_t v = gen_pair_val(p, j); memcpy(vals + 8 * i, &v, 8); }
            else if (p->with_doc_vals) { uint32_t d = (uint32_t)gen_doc_of(p, j); memcpy(vals + 4 * i, &d, 4); }
        }
    }
}

int gen_num_threads(void) { return omp_get_max_threads(); }
}

// raw text of records [j0, j0+cnt) from their CSR (see gen_text_sep)
extern "C" void gen_text_host(const gen_params* p, uint64_t j0, uint64_t cnt, const uint64_t* offs, const uint8_t* keys,
                              uint8_t* text) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) {
        const uint64_t o = offs[i] - offs[0], e = offs[i + 1] - offs[0];
        for (uint64_t q = o; q < e; ++q) text[q + (uint64_t)i] = keys[q];
        text[e + (uint64_t)i] = gen_text_sep(p, j0 + (uint64_t)i);
    }
}
extern "C" void gen_doc_lens_host(uint64_t seed, uint64_t d0, uint64_t cnt, uint64_t* out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) out[i] = gen_doc_len(seed, d0 + (uint64_t)i);
}

// ---------------------------------------------------------------- closed-form checks (tests only)
// These evaluate the generators' construction backwards — which rank a key spells, and what the
// records of a rank carry — so a full-size result (10^8-10^9 records) can be checked key by key
// without a CPU group-by. Nothing here hashes or groups records.
namespace {
// gen_perm_inv with the four round keys computed once (same arithmetic as gen_feistel_inv)
struct PermInv {
    int half;
    uint64_t mask, k[4], n, seed;
    PermInv(uint64_t n_, uint64_t seed_) : n(n_), seed(seed_) {
        half = gen_perm_half_bits(n);
        mask = (half >= 32) ? 0xffffffffULL : ((1ULL << half) - 1);
        for (int r = 0; r < 4; ++r) k[r] = gen_rnd(seed, GEN_S_PERM, (uint64_t)r);
    }
    uint64_t once(uint64_t y) const {
        uint64_t L = y >> half, R = y & mask;
        for (int r = 3; r >= 0; --r) {
            uint64_t pR = L, pL = R ^ (gen_mix64(L ^ k[r]) & mask);
            L = pL; R = pR;
        }
        return (L << half) | R;
    }
    uint64_t operator()(uint64_t idx) const {
        uint64_t y = once(idx);
        while (y >= n) y = once(y);
        return y;
    }
};
uint64_t unxorshift(uint64_t z, int s) {  // inverse of z ^= z >> s
    uint64_t y = z;
    for (int i = 0; i < 64 / s + 1; ++i) y = z ^ (y >> s);
    return y;
}
uint64_t inv_odd(uint64_t a) {  // a^-1 mod 2^64 (Newton)
    uint64_t x = a;
    for (int i = 0; i < 6; ++i) x *= 2 - a * x;
    return x;
}
uint64_t unmix64(uint64_t z) {  // inverse of gen_mix64
    z = unxorshift(z, 31);
    z *= inv_odd(0x94d049bb133111ebULL);
    z = unxorshift(z, 27);
    z *= inv_odd(0xbf58476d1ce4e5b9ULL);
    return unxorshift(z, 30);
}
uint64_t digest_mix(uint64_t v) { return gen_mix64(v ^ 0x6a09e667f3bcc909ULL); }
}  // namespace

extern "C" {
// out[i] = the rank r in [1, n_ranks] whose key spelling is key i (keys[offs[i]..offs[i+1])), or 0
// if no rank spells it (verified by re-spelling r).
void gen_key_ranks_host(const gen_params* p, const uint8_t* keys, const uint64_t* offs, uint64_t n_keys, uint64_t* out) {
#pragma omp parallel for schedule(static, 4096)
    for (int64_t i = 0; i < (int64_t)n_keys; ++i) {
        const uint8_t* k = keys + offs[i];
        const uint64_t L = offs[i + 1] - offs[i];
        uint64_t r = 0;
        bool ok = true;
        if (p->family == GEN_WORDS) {
            ok = L >= 1 && L <= 16;
            for (uint64_t q = 0; ok && q < L; ++q) {
                if (k[q] < 'a' || k[q] > 'z') ok = false;
                else { r = r * 26 + (uint64_t)(k[q] - 'a'); if (r > p->n_ranks) ok = false; }
            }
        } else if (p->family == GEN_URLS) {
            ok = L > 23 && L <= 256 && memcmp(k, "https://h", 9) == 0 && memcmp(k + 13, ".example/", 9) == 0;
            uint64_t q = 22;
            for (; ok && q < L && k[q] != '/'; ++q) {
                const uint8_t c = k[q];
                uint64_t dgt = (c >= '0' && c <= '9') ? (uint64_t)(c - '0') : (c >= 'a' && c <= 'z') ? (uint64_t)(c - 'a' + 10) : 99;
                if (dgt >= 36) ok = false;
                else { r = r * 36 + dgt; if (r > p->n_ranks) ok = false; }
            }
            if (q == 22 || q >= L) ok = false;
        } else {
            ok = L == 8;
            if (ok) { uint64_t kv; memcpy(&kv, k, 8); r = unmix64(kv); }
        }
        if (ok && (r < 1 || r > p->n_ranks)) ok = false;
        if (ok) {
            uint8_t buf[256];
            const uint32_t L2 = gen_key_len_of_rank(p, r);
            ok = L2 == L;
            if (ok) { gen_key_spell(p, r, L2, buf); ok = memcmp(buf, k, L) == 0; }
        }
        out[i] = ok ? r : 0;
    }
}

// For ranks r0 .. r0+cnt-1: the records holding rank r are perm^{-1} of its multiset block
// [cum[r-1], cum[r]) (uniform: [(r-1) m, r m)). count[i] = block size, sum[i] = sum of the
// records' values mod 2^64, mixsum[i] = sum of digest_mix(value) mod 2^64 (a multiset digest:
// a sum, not a xor, so duplicate values do not cancel). Values: PAIRS u64 value, docs doc id.
void gen_rank_digest_host(const gen_params* p, uint64_t r0, uint64_t cnt, uint64_t* count, uint64_t* sum, uint64_t* mixsum) {
    const PermInv pinv(p->n, p->seed);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < (int64_t)cnt; ++i) {
        const uint64_t r = r0 + (uint64_t)i;
        const uint64_t lo = p->uniform_m ? (r - 1) * p->uniform_m : p->cum[r - 1];
        const uint64_t hi = p->uniform_m ? r * p->uniform_m : p->cum[r];
        uint64_t s = 0, m = 0;
        for (uint64_t idx = lo; idx < hi; ++idx) {
            const uint64_t j = pinv(idx);
            const uint64_t v = (p->family == GEN_PAIRS) ? gen_pair_val(p, j) : gen_doc_of(p, j);
            s += v;
            m += digest_mix(v);
        }
        count[i] = hi - lo;
        sum[i] = s;
        mixsum[i] = m;
    }
}

// The same digest of exported value lists: key i owns values [lo[i], lo[i+1]), value q is the
// little-endian integer of bytes vals[vo[q] .. vo[q+1]) (at most 8 bytes).
void gen_list_digest_host(const uint8_t* vals, const uint64_t* vo, const uint64_t* lo, uint64_t n_keys, uint64_t* count,
                          uint64_t* sum, uint64_t* mixsum) {
#pragma omp parallel for schedule(static, 4096)
    for (int64_t i = 0; i < (int64_t)n_keys; ++i) {
        uint64_t s = 0, m = 0;
        for (uint64_t q = lo[i]; q < lo[i + 1]; ++q) {
            uint64_t v = 0;
            const uint64_t w = vo[q + 1] - vo[q];
            for (uint64_t b = 0; b < w && b < 8; ++b) v |= (uint64_t)vals[vo[q] + b] << (8 * b);
            s += v;
            m += digest_mix(v);
        }
        count[i] = lo[i + 1] - lo[i];
        sum[i] = s;
        mixsum[i] = m;
    }
}
}
