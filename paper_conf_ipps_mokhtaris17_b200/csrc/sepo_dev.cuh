// sepo_dev.cuh — device data structures and primitives of the SEPO hash table (sm_100a).
//
// PAPER.md cited as P:L<line>. Layout of the budget region (one cudaMalloc, host side carves it):
//   dir[n_buckets]      u32 entry refs, "a simple array of null pointers"
//   ctrl                counters (pool_taken, postponed, dead bytes, ...)
//   cursors[G][2]       per-CTA allocation cursors {page<<32 | offset} (key/combine, value)
//   stack[P]            free-page stack (pages handed out by pool_taken)
//   page_state[P]       0 free, 1 entry/key page, 2 value page
//   retain[P]           GROUP: key page kept resident at the pass end
//   evict_list[P]       pages evicted at the last pass boundary
//   pool                P pages of page_bytes (the paper's heap)
//
// Entry refs are u32: ref = pool_offset/8 + 1 (0 = null). A value-list ref (GROUP) is u64:
// generation << 40 | (pool_offset/8 + 1), so a list can point into an evicted generation — the
// relocatable stand-in for the paper's "two pointers ... GPU ... and eventual location in CPU
// memory". Device code never follows a value-list ref, it only CASes the list head.
//
// Every record in a page is 16-byte aligned and starts with a u32 header = size | kind, so an
// evicted page image is parsed linearly on the host (a filler covers every unused tail). The
// first 32 bytes of an entry (header + first 16 key bytes) are fetched with two 16-B vector loads:
//   COMBINE entry       : hdr | next u32 | tag u32 | klen u32 | key[pad8] | value u64
//   GROUP key entry     : hdr | next u32 | tag u32 | klen u32 | key[pad8] | list_head u64 |
//                                      birth_gen u32 | pad u32
//   GROUP value chunk: hdr | fill u32 | owner u64 | values  (16-byte header; the
//                                      capacity follows from the size, the value format from the kind:
//                                      K_VCHUNK fixed-width slots, K_VCHUNKV {u32 length, bytes} items)
//   filler                            : hdr (size of the gap)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sepo {

constexpr uint32_t FULLMASK = 0xffffffffu;
enum : uint32_t { K_FREE = 0, K_COMBINE = 1, K_FILL = 2, K_DEAD = 3, K_GKEY = 4, K_VCHUNK = 5, K_BASIC = 6,
                  K_VCHUNKV = 7 };
constexpr uint32_t KIND_MASK = 7u;
constexpr uint32_t KEY_OFF = 16;     // key bytes start here in combine and group key entries
constexpr uint32_t CHUNK_HDR = 16;   // value chunk header: size | kind, fill, owner
constexpr uint32_t CHUNK_PRIVATE = 0x80000000u;  // fill flag: slots handed out by one CTA (hot key) — a
                                                 // reserving thread sees the chunk as full
constexpr uint32_t NOPAGE = 0xfffffffeu, FULLPAGE = 0xffffffffu;
constexpr uint32_t PAGE_ENTRY = 1, PAGE_VALUE = 2;

// result codes of a slot / record
enum : uint32_t { R_OK = 0, R_POST = 1, R_TOOLARGE = 2 };

struct Ctrl {
    unsigned long long pool_taken;     // pages handed out from the free stack this generation
    unsigned long long postponed;      // per-call accumulator
    unsigned long long toolarge;
    unsigned long long dead_bytes;
    unsigned long long kept_key_bytes; // reprobe: bytes of the still-postponed records
    unsigned long long kept_val_bytes;
    unsigned long long n_evict;        // evict: pages in evict_list
    unsigned long long n_free;         // evict: pages in the new free stack
    unsigned long long n_resident;     // evict: pages that stay resident (retained)
    unsigned long long full;           // 1 once the pool ran out this generation: every later allocation fails
    unsigned long long n_safe;         // evict: free pages that need no copy (never used last generation)
    unsigned int copied;               // evicted pages whose D2H copy finished (written by the copy stream)
    unsigned int failed_slots;         // BASIC: allocator slots whose allocation failed this generation
    unsigned long long text_words;     // sepo_run_text: words tokenized by the last insert call
    unsigned long long next_group;     // GROUP insert: next 32-record group to hand out (dynamic schedule)
    unsigned long long pad[2];
};

struct Dev {
    uint32_t* dir;
    uint64_t n_buckets;
    uint8_t* pool;
    uint32_t page_bytes;
    uint32_t page_shift;
    uint32_t n_pages;
    uint32_t n_free;          // pages available in `stack` this generation
    // Eviction overlapped with the next pass (a10): stack[0, n_safe) are pages the last generation
    // did not use; stack[n_safe + j] is the j-th evicted page, reusable once ctrl->copied > j.
    uint32_t n_safe;
    uint32_t* stack;
    uint8_t* page_state;
    uint8_t* retain;
    uint32_t* evict_list;
    unsigned long long* cursors;  // [grid][2]
    Ctrl* ctrl;
    // per-allocator-slot announcement words (128 B apart): bit 63 = pool full, low bits = warps of
    // that CTA between announcing an allocation and linking its entries (certified declines, R15)
    unsigned long long* ann;
    uint32_t n_slots;
    uint64_t seed;
    uint32_t gen;             // generation (= pass index) of resident data
    uint32_t fail_ppm, fail_mode, fail_until;
    uint32_t batch_seq;
    // Overlapped eviction through the gather kernel (GROUP): warp w of the kernel copies evict-list
    // positions w, w + eprog_n, ... in order and publishes how many it finished in eprog[w], so
    // position j is copied once eprog[j % eprog_n] > j / eprog_n. nullptr: progress is ctrl->copied.
    unsigned int* eprog;
    uint32_t eprog_n;
};

// ---------------------------------------------------------------- memory access helpers
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// Publishing CAS / add with release semantics: the entry (or chunk) written before is visible to
// any thread that reads the new link. Unlike __threadfence() (MEMBAR.SC + CCTL.IVALL on sm_100),
// a release RMW does not invalidate L1, which holds the streamed input keys.
__device__ __forceinline__ uint32_t cas_release(uint32_t* p, uint32_t cmp, uint32_t val) {
    uint32_t old;
    asm volatile("atom.release.gpu.global.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "l"(p), "r"(cmp), "r"(val) : "memory");
    return old;
}
__device__ __forceinline__ unsigned long long cas_release64(unsigned long long* p, unsigned long long cmp,
                                                            unsigned long long val) {
    unsigned long long old;
    asm volatile("atom.release.gpu.global.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
__device__ __forceinline__ void add_release64(unsigned long long* p, unsigned long long v) {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
constexpr unsigned long long ANN_FULL = 1ull << 63;
constexpr uint32_t ANN_STRIDE = 16;  // u64 words between announcement words (128 B)
// ---------------------------------------------------------------- L2 residency policy
// The streamed input (16 GB for C2) would otherwise push table lines out of L2: on B200 a 55 MB
// table next to an evict_normal input stream missed L2 on 58 % of its sectors (ncu, pass 1 of the
// C2 4x job: 71 GB DRAM read for 16 GB of input). Input loads therefore carry an L2 evict_first
// policy (and skip L1 allocation); table accesses keep the default policy.
// createpolicy with a constant fraction folds into the load's memory descriptor (no extra SASS).
__device__ __forceinline__ uint64_t pol_in() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_tab() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// immutable input (keys, offsets, values, re-issue indices): read-only path, L2 evict_first
__device__ __forceinline__ uint64_t ld_in64(const void* p) {
    uint64_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol_in()));
    return v;
}
__device__ __forceinline__ uint32_t ld_in32(const void* p) {
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol_in()));
    return v;
}
__device__ __forceinline__ uint32_t ld_in16(const void* p) {
    unsigned short v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol_in()));
    return v;
}
__device__ __forceinline__ uint32_t ld_in8(const void* p) {
    unsigned short v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol_in()));
    return v & 0xffu;
}
__device__ __forceinline__ uint4 ld_in128(const void* p) {
    uint4 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol_in()));
    return v;
}

// L2-coherent loads of published entry fields (never stale L1 lines)
__device__ __forceinline__ uint64_t ldcg64(const void* p) { return __ldcg(reinterpret_cast<const unsigned long long*>(p)); }
__device__ __forceinline__ uint32_t ldcg32(const void* p) { return __ldcg(reinterpret_cast<const unsigned int*>(p)); }

// input words read lane by lane (key tails beyond the first 16 bytes): L1-allocating, so the
// group's neighbouring keys (one 128-byte line holds two 64-byte URLs) are read from L1 after the
// first lane's miss (L1::no_allocate sent every 8-byte tail load to L2: C3 pass 1 load-bound)
__device__ __forceinline__ uint64_t ld_tail64(const void* p) {
    uint64_t v;
    asm("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol_in()));
    return v;
}
// Bytes [p, p+nb) (1 <= nb <= 8) of immutable INPUT as a little-endian word, zero-extended.
// Only the aligned words that contain requested bytes are read.
__device__ __forceinline__ uint64_t load_in_word(const uint8_t* p, uint32_t nb) {
    uintptr_t a = reinterpret_cast<uintptr_t>(p);
    uint32_t sh = (uint32_t)(a & 7u);
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(a - sh);
    uint64_t v = ld_tail64(q) >> (8 * sh);
    if (sh + nb > 8) v |= ld_tail64(q + 1) << (64 - 8 * sh);
    if (nb < 8) v &= (1ull << (8 * nb)) - 1ull;
    return v;
}

// x << n with the PTX semantics for n >= 64 (result 0), unlike C++ where it is undefined
__device__ __forceinline__ uint64_t shl64_clamp(uint64_t x, uint32_t n) {
    uint64_t r;
    asm("shl.b64 %0, %1, %2;" : "=l"(r) : "l"(x), "r"(n));
    return r;
}

// key word from the aligned words x (holding its first byte) and y (the next): 32-bit halves
// selected by bit 2 of the key's address, then two funnel shifts by 8 x (address & 3)
__device__ __forceinline__ uint64_t key_word(uint64_t x, uint64_t y, bool o, uint32_t s) {
    const uint32_t xl = (uint32_t)x, xh = (uint32_t)(x >> 32), yl = (uint32_t)y, yh = (uint32_t)(y >> 32);
    const uint32_t b0 = o ? xh : xl, b1 = o ? yl : xh, b2 = o ? yh : yl;
    return ((uint64_t)__funnelshift_r(b1, b2, s) << 32) | __funnelshift_r(b0, b1, s);
}
// mask of the key's last word (bytes 1..8 of it are key bytes)
__device__ __forceinline__ uint64_t last_word_mask(uint32_t n) {
    return ~shl64_clamp(~0ull, 8u * (n - 8u * ((n - 1u) >> 3)));
}
// Input bytes [p, p+n) (n >= 1, immutable) as zero-padded 8-byte LE words, U words per round: a
// round's aligned words are loaded together and shifted into key words, so a key tail costs
// ceil(words / U) load round trips instead of one (two loads) per word — the per-word loop held
// 48 % of C3 pass 1's stall samples (ncu source page, profiles/r02_summary.md). f(k, w) receives key
// words k .. k + U - 1 (beyond the key: unspecified, callers test k + u < words) and returns false
// to stop. Used by the long-key kernel instantiations (U > 1); U = 1 keeps the per-word loop.
template <int U, typename F>
__device__ __forceinline__ void tail_rounds(const uint8_t* p, uint32_t n, F&& f) {
    const uintptr_t a = reinterpret_cast<uintptr_t>(p);
    const bool o = (a >> 2) & 1u;
    const uint32_t s = 8u * (uint32_t)(a & 3u);
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(a & ~(uintptr_t)7);
    const uint32_t naw = ((uint32_t)(a & 7u) + n + 7u) >> 3, nw = (n + 7u) >> 3;  // aligned words touched, key words
    const uint64_t lm = last_word_mask(n);
    uint64_t cur = ld_tail64(q);
    for (uint32_t k = 0; k < nw; k += U) {
        uint64_t x[U + 1];
        x[0] = cur;
#pragma unroll
        for (int u = 1; u <= U; ++u) x[u] = k + u < naw ? ld_tail64(q + k + u) : 0ull;
        uint64_t w[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            w[u] = key_word(x[u], x[u + 1], o, s);
            if (k + u == nw - 1) w[u] &= lm;
        }
        if (!f(k, w)) return;
        cur = x[U];
    }
}

// ---------------------------------------------------------------- key hash (the paper leaves it open)
__device__ __forceinline__ uint64_t fmix64(uint64_t k) {
    k ^= k >> 33; k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33; return k;
}
// h = fmix64(head + tail): head = a multiply-xor fold of the length, seed and the first 16 key bytes
// (w0, w1: 8-byte LE words, zero padded); tail = the sum mod 2^64 of mix_word(word k, k) over the
// key's remaining 8-byte words (zero padded). A sum, not a fold, so one key's tail can be hashed by
// one lane or by a whole warp (lanes take words, the warp adds) with the same result (R32).
// Keys of at most 16 bytes hash without branches.
__device__ __forceinline__ uint64_t hash_init(uint32_t len, uint64_t seed) { return seed ^ ((uint64_t)len * 0x87c37b91114253d5ull); }
__device__ __forceinline__ uint64_t hash_word(uint64_t h, uint64_t w) {
    return (h ^ w) * 0x9e3779b97f4a7c15ull;  // odd multiplier: a bijection per word
}
__device__ __forceinline__ uint64_t hash_head(uint32_t len, uint64_t seed, uint64_t w0, uint64_t w1) {
    return hash_word(hash_word(hash_init(len, seed), w0), w1);
}
__device__ __forceinline__ uint64_t mix_word(uint64_t w, uint32_t k) {
    uint64_t t = (w ^ ((uint64_t)(k + 1) * 0x9e3779b97f4a7c15ull)) * 0xbf58476d1ce4e5b9ull;
    return t ^ (t >> 31);
}
// tail sum of the key bytes [p, p+n) (p = key + 16), by one lane
template <int U = 1>
__device__ __forceinline__ uint64_t tail_sum(const uint8_t* p, uint32_t n) {
    uint64_t x = 0;
    if (U == 1) {
        for (uint32_t o = 0, k = 0; o < n; o += 8, ++k) x += mix_word(load_in_word(p + o, n - o < 8 ? n - o : 8), k);
    } else if (n > 0) {
        const uint32_t nw = (n + 7) >> 3;
        tail_rounds<U>(p, n, [&](uint32_t k, const uint64_t (&w)[U]) {
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (k + u < nw) x += mix_word(w[u], k + u);
            return true;
        });
    }
    return x;
}
// hash of a key given its first 16 bytes (w0, w1) and, for longer keys, its bytes at p
template <int U = 1>
__device__ __forceinline__ uint64_t hash_key16(uint32_t len, uint64_t seed, uint64_t w0, uint64_t w1, const uint8_t* p) {
    uint64_t x = hash_head(len, seed, w0, w1);
    if (len > 16) x += tail_sum<U>(p + 16, len - 16);
    return fmix64(x);
}
// Warp-cooperative pieces for one long key (all 32 lanes call with the same p, n; n >= 1): lane l
// takes the key words l, l + 32, ... of the input bytes [p, p+n) — one coalesced load per lane and
// a shuffle for the neighbouring aligned word — instead of one lane walking the whole key.
__device__ __forceinline__ uint64_t shfl_down64(uint64_t v, uint32_t d) {
    const uint32_t lo = __shfl_down_sync(0xffffffffu, (uint32_t)v, d), hi = __shfl_down_sync(0xffffffffu, (uint32_t)(v >> 32), d);
    return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl_xor64(uint64_t v, uint32_t m) {
    const uint32_t lo = __shfl_xor_sync(0xffffffffu, (uint32_t)v, m), hi = __shfl_xor_sync(0xffffffffu, (uint32_t)(v >> 32), m);
    return ((uint64_t)hi << 32) | lo;
}
template <typename F>
__device__ __forceinline__ void warp_tail_words(const uint8_t* p, uint32_t n, F&& f) {
    const uint32_t lane = threadIdx.x & 31u;
    const uintptr_t a = reinterpret_cast<uintptr_t>(p);
    const bool o = (a >> 2) & 1u;
    const uint32_t s = 8u * (uint32_t)(a & 3u);
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(a & ~(uintptr_t)7);
    const uint32_t naw = ((uint32_t)(a & 7u) + n + 7u) >> 3, nw = (n + 7u) >> 3;
    const uint64_t lm = last_word_mask(n);
    for (uint32_t k0 = 0; k0 < nw; k0 += 32) {
        const uint32_t k = k0 + lane;
        const uint64_t x = k < naw ? ld_tail64(q + k) : 0ull;
        uint64_t y = shfl_down64(x, 1);
        if (lane == 31 && k + 1 < naw) y = ld_tail64(q + k + 1);
        uint64_t w = key_word(x, y, o, s);
        if (k == nw - 1) w &= lm;
        if (!f(k, k < nw, w)) return;
    }
}
// the tail sum of hash_key16 for the key bytes [p, p+n) (p = key + 16), in every lane
__device__ __forceinline__ uint64_t warp_tail_sum(const uint8_t* p, uint32_t n) {
    uint64_t acc = 0;
    warp_tail_words(p, n, [&](uint32_t k, bool in, uint64_t w) {
        if (in) acc += mix_word(w, k);
        return true;
    });
#pragma unroll
    for (uint32_t o = 16; o; o >>= 1) acc += shfl_xor64(acc, o);
    return acc;
}
// input bytes [p, p+n) == the zero-padded entry words at ek (8-aligned), in every lane
__device__ __forceinline__ bool warp_tail_eq(const uint8_t* ek, const uint8_t* p, uint32_t n) {
    bool eq = true;
    warp_tail_words(p, n, [&](uint32_t k, bool in, uint64_t w) {
        eq = !__any_sync(0xffffffffu, in && ldcg64(ek + 8 * k) != w);
        return eq;
    });
    return eq;
}
__device__ __forceinline__ void load_key16(const uint8_t* p, uint32_t len, uint64_t& w0, uint64_t& w1);
__device__ __forceinline__ uint64_t hash_key(const uint8_t* p, uint32_t len, uint64_t seed) {
    uint64_t w0, w1;
    load_key16(p, len, w0, w1);
    return hash_key16(len, seed, w0, w1, p);
}
__device__ __forceinline__ uint32_t bucket_of(uint64_t h, uint64_t n_buckets) {
    return (uint32_t)(((h >> 32) * n_buckets) >> 32);
}
__device__ __forceinline__ uint32_t tag_of(uint64_t h) { return (uint32_t)h; }

__device__ __forceinline__ uint32_t align8(uint32_t x) { return (x + 7u) & ~7u; }
__device__ __forceinline__ uint32_t align16(uint32_t x) { return (x + 15u) & ~15u; }
// entry sizes (16-byte aligned records)
__device__ __forceinline__ uint32_t centry_size(uint32_t klen) { return align16(KEY_OFF + align8(klen) + 8u); }
__device__ __forceinline__ uint32_t gkey_size(uint32_t klen) { return align16(KEY_OFF + align8(klen) + 16u); }
// value (COMBINE) / list head (GROUP) of an entry with key length klen
__device__ __forceinline__ uint8_t* entry_val(uint8_t* e, uint32_t klen) { return e + KEY_OFF + align8(klen); }
__device__ __forceinline__ uint8_t* ref_ptr(const Dev& d, uint32_t ref) { return d.pool + ((uint64_t)(ref - 1) << 3); }
__device__ __forceinline__ uint32_t off_ref(uint64_t off) { return (uint32_t)(off >> 3) + 1u; }

// Key equality: entry key at e + koff (8-aligned, zero padded) vs input key [p, p+len).
// U > 1: the entry words of a round are loaded with the input words (no dependency between them).
template <int U = 1>
__device__ __forceinline__ bool entry_key_eq(const uint8_t* ek, const uint8_t* p, uint32_t len) {
    if (U == 1) {
        for (uint32_t o = 0; o < len; o += 8) {
            uint32_t nb = len - o < 8 ? len - o : 8;
            if (ldcg64(ek + o) != load_in_word(p + o, nb)) return false;
        }
        return true;
    }
    if (len == 0) return true;
    const uint32_t nw = (len + 7) >> 3;
    bool eq = true;
    tail_rounds<U>(p, len, [&](uint32_t k, const uint64_t (&w)[U]) {
#pragma unroll
        for (int u = 0; u < U; ++u)
            if (k + u < nw) eq = eq && ldcg64(ek + 8 * (k + u)) == w[u];
        return eq;
    });
    return eq;
}
// Input-vs-input key equality (both immutable input bytes)
__device__ __forceinline__ bool in_key_eq(const uint8_t* a, const uint8_t* b, uint32_t len) {
    for (uint32_t o = 0; o < len; o += 8) {
        uint32_t nb = len - o < 8 ? len - o : 8;
        if (load_in_word(a + o, nb) != load_in_word(b + o, nb)) return false;
    }
    return true;
}
// Copy an input key into an entry (8-aligned destination, zero padded tail)
template <int U = 1>
__device__ __forceinline__ void store_key(uint8_t* ek, const uint8_t* p, uint32_t len) {
    if (U == 1) {
        for (uint32_t o = 0; o < len; o += 8) {
            uint32_t nb = len - o < 8 ? len - o : 8;
            *reinterpret_cast<unsigned long long*>(ek + o) = load_in_word(p + o, nb);
        }
        return;
    }
    if (len == 0) return;
    const uint32_t nw = (len + 7) >> 3;
    tail_rounds<U>(p, len, [&](uint32_t k, const uint64_t (&w)[U]) {
#pragma unroll
        for (int u = 0; u < U; ++u)
            if (k + u < nw) *reinterpret_cast<unsigned long long*>(ek + 8 * (k + u)) = w[u];
        return true;
    });
}

__device__ __forceinline__ uint4 ldcg128(const void* p) { return __ldcg(reinterpret_cast<const uint4*>(p)); }
__device__ __forceinline__ ulonglong2 ldcg128u(const void* p) { return __ldcg(reinterpret_cast<const ulonglong2*>(p)); }
__device__ __forceinline__ uint32_t ld_dir(const uint32_t* p) { return ld_relaxed_u32(p); }

// Walk the chain [ref .. stop) for an entry with (tag, len, key) — key given by its INPUT bytes.
// Only entries of the resident generation are reachable (head insertion; the directory
// is reset at every pass boundary).
__device__ __forceinline__ uint8_t* chain_find(const Dev& d, uint32_t ref, uint32_t stop, uint32_t tag, uint32_t len,
                                               const uint8_t* key) {
    while (ref != 0 && ref != stop) {
        uint8_t* e = ref_ptr(d, ref);
        const uint4 hd = ldcg128(e);  // hdr | next | tag | klen
        if (hd.z == tag && hd.w == len && entry_key_eq(e + KEY_OFF, key, len)) return e;
        ref = hd.y;
    }
    return nullptr;
}
// Same, with the key's first 16 bytes in registers (w0, w1 zero padded); bytes >= 16 of a long
// key are compared against `tail` (the input key + 16).
template <int U = 1>
__device__ __forceinline__ uint8_t* chain_find_w(const Dev& d, uint32_t ref, uint32_t stop, uint32_t tag, uint32_t len,
                                                 uint64_t w0, uint64_t w1, const uint8_t* tail) {
    const uint64_t m0 = len ? ~0ull : 0ull, m1 = len > 8 ? ~0ull : 0ull;  // words that hold key bytes
    while (ref != 0 && ref != stop) {
        uint8_t* e = ref_ptr(d, ref);
        const uint4 hd = ldcg128(e);
        const ulonglong2 kw = ldcg128u(e + KEY_OFF);
        bool eq = hd.z == tag && hd.w == len && !((kw.x ^ w0) & m0) && !((kw.y ^ w1) & m1);
        if (len > 16) eq = eq && entry_key_eq<U>(e + KEY_OFF + 16, tail, len - 16);
        if (eq) return e;
        ref = hd.y;
    }
    return nullptr;
}
// First 16 bytes of an input key as two zero-padded LE words (at most 3 aligned loads).
__device__ __forceinline__ void load_key16(const uint8_t* p, uint32_t len, uint64_t& w0, uint64_t& w1) {
    w0 = 0; w1 = 0;
    if (len == 0) return;
    const uintptr_t a = reinterpret_cast<uintptr_t>(p);
    const uint32_t sh = (uint32_t)(a & 7u);
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(a - sh);
    const uint32_t nb = len < 16 ? len : 16;
    const uint32_t nw = (sh + nb + 7) >> 3;  // aligned words touched (1..3)
    const uint64_t x0 = ld_in64(q);
    const uint64_t x1 = nw > 1 ? ld_in64(q + 1) : 0ull;
    const uint64_t x2 = nw > 2 ? ld_in64(q + 2) : 0ull;
    if (sh == 0) { w0 = x0; w1 = x1; }
    else {
        w0 = (x0 >> (8 * sh)) | (x1 << (64 - 8 * sh));
        w1 = (x1 >> (8 * sh)) | (x2 << (64 - 8 * sh));
    }
    if (nb < 8) { w0 &= (1ull << (8 * nb)) - 1ull; w1 = 0; }
    else if (nb < 16) w1 &= (1ull << (8 * (nb - 8))) - 1ull;
}

// ---------------------------------------------------------------- fault injection (tests only)
__device__ __forceinline__ bool inject_fail(const Dev& d, uint64_t h, uint64_t rec) {
    if (d.fail_ppm == 0 || d.gen >= d.fail_until) return false;
    uint64_t x = d.fail_mode == 0 ? fmix64(h ^ (0x9e37ull * (d.gen + 1)))
                                  : fmix64(rec * 0x100000001b3ull ^ ((uint64_t)d.batch_seq << 40) ^ (d.gen + 7));
    return (x % 1000000ull) < d.fail_ppm;
}

// ---------------------------------------------------------------- page-pool allocator
// Warp-collective bump allocation from this CTA's current page (cursor in shared memory, packed
// {page << 32 | offset}). Lanes with `need` get `size` bytes (multiple of 8, <= page_bytes) and
// the pool offset back, or ~0 when the page is full and the pool has no free page (POSTPONE).
// The first lane whose range crosses the page end writes a filler over the tail, takes a page
// from the free stack (one global atomic per page) and installs it; lanes of other warps that
// overshot wait for the install and retry. Must be called by all 32 lanes.
__device__ __forceinline__ uint64_t warp_alloc(const Dev& d, unsigned long long* scur, bool need, uint32_t size,
                                               uint8_t page_kind, bool monotone = true) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t PB = d.page_bytes;
    uint64_t result = ~0ull;
    bool pending = need;
    // failure is monotone for the whole generation: once the pool ran out, nobody allocates
    // (BASIC passes monotone = false: a slot keeps filling its open page)
    if (monotone && __any_sync(FULLMASK, pending)) {
        unsigned long long full = 0;
        if (lane == 0) full = ld_relaxed_u64(&d.ctrl->full);
        if (__shfl_sync(FULLMASK, full, 0) != 0ull) return ~0ull;  // warp-uniform decision
    }
    while (true) {
        unsigned pm = __ballot_sync(FULLMASK, pending);
        if (!pm) break;
        uint32_t s = pending ? size : 0u;
        uint32_t incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(FULLMASK, incl, o);
            if (lane >= (uint32_t)o) incl += y;
        }
        uint32_t total = __shfl_sync(FULLMASK, incl, 31);
        uint32_t excl = incl - s;
        unsigned long long cur = 0;
        if (lane == 0) cur = atomicAdd(scur, (unsigned long long)total);
        cur = __shfl_sync(FULLMASK, cur, 0);
        const uint32_t page = (uint32_t)(cur >> 32);
        const uint32_t off = (uint32_t)cur;
        if (page == FULLPAGE) break;  // pool exhausted for this CTA: every pending lane POSTPONEs
        bool again = false;
        if (pending) {
            uint64_t start = (uint64_t)off + excl;
            if (page != NOPAGE && start + s <= PB) {
                result = ((uint64_t)page << d.page_shift) + start;
                pending = false;
            } else {
                if (start <= PB) {  // the unique crossing lane: seal the tail, install a new page
                    if (page != NOPAGE && start < PB)
                        *reinterpret_cast<uint32_t*>(d.pool + ((uint64_t)page << d.page_shift) + start) =
                            (uint32_t)(PB - start) | K_FILL;
                    unsigned long long q = atomicAdd(&d.ctrl->pool_taken, 1ull);
                    unsigned long long nw;
                    if (q < d.n_free) {
                        if (q >= d.n_safe) {  // an evicted page: wait until its copy to the host is done
                            const uint32_t jpos = (uint32_t)(q - d.n_safe);
                            const unsigned int* pw = d.eprog ? d.eprog + jpos % d.eprog_n : &d.ctrl->copied;
                            const unsigned int need_copied = d.eprog ? jpos / d.eprog_n + 1u : jpos + 1u;
                            while (true) {
                                unsigned int cp;
                                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(cp) : "l"(pw) : "memory");
                                if (cp >= need_copied) break;
                                __nanosleep(256);
                            }
                        }
                        uint32_t np = d.stack[q];
                        d.page_state[np] = page_kind;
                        nw = (unsigned long long)np << 32;
                    } else {
                        nw = (unsigned long long)FULLPAGE << 32;
                        // the pool ran out: every later allocation of this generation fails. The
                        // bit goes into every slot's announcement word (same-location RMWs order
                        // it against each announcement; see the COMBINE insert kernel).
                        if (atomicExch(&d.ctrl->full, 1ull) == 0ull)
                            for (uint32_t c = 0; c < d.n_slots; ++c) atomicOr(&d.ann[(uint64_t)c * ANN_STRIDE], ANN_FULL);
                    }
                    __threadfence_block();
                    atomicExch(scur, nw);
                }
                again = true;
            }
        }
        if (__any_sync(FULLMASK, again)) {
            if (lane == 0) {
                while ((uint32_t)(*reinterpret_cast<volatile unsigned long long*>(scur) >> 32) == page) __nanosleep(20);
            }
            __syncwarp();
        }
    }
    return result;
}

}  // namespace sepo
