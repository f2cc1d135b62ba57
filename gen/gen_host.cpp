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
