// sepo_kernels.cu — the SEPO hot path on sm_100a (PAPER.md cited as P:L<line>).
//
//   insert_stream_kernel / insert_group_stream_kernel
//                   a1..a7  record ingest + hash, hot-key folding in shared memory, chain walk,
//                           combine / group in place, page-pool allocation, lock-free head link,
//                           certified decline -> postpone bitmap + count
//   reprobe_kernel  a8      end-of-pass re-probe of declined records
//   compact_*       a9      stream compaction of the postponed records (re-issue)
//   seal/classify/relink a10 pass boundary: seal open pages, pick cold pages, rebuild the free
//                           stack and (GROUP) re-link retained key pages
//
// The insert kernels are persistent (one CTA of 1024 threads per SM = one allocator slot); every
// warp streams 32-record groups without CTA barriers (see the kernel comments below).
#include "sepo_dev.cuh"
#include "sepo_kernels.h"
#include <algorithm>
#include <type_traits>
#include <cstring>

namespace sepo {


// lane id (threadIdx.x & 31: measured faster than reading %laneid, C2 4x pass 1 21.6 vs 22.0 ms)
__device__ __forceinline__ uint32_t lane_id() {
    return threadIdx.x & 31u;
}
__device__ __forceinline__ uint32_t lanemask_lt() { return (1u << lane_id()) - 1u; }

// record i of a batch -> its index in keys / key_offsets / vals (re-issue by index, a9)
__device__ __forceinline__ uint64_t rec_index(const Batch& b, uint64_t i) { return b.idx ? ld_in64(b.idx + i) : i; }
// value of record i for COMBINE (vw bytes LE, or 1 when vals == nullptr)
__device__ __forceinline__ uint64_t rec_value(const Batch& b, uint64_t i) {
    if (b.wire) return b.wire[i].v;
    if (b.vals == nullptr) return 1ull;
    i = rec_index(b, i);
    switch (b.vw) {
        case 8: return ld_in64(reinterpret_cast<const unsigned long long*>(b.vals) + i);
        case 4: return ld_in32(reinterpret_cast<const unsigned int*>(b.vals) + i);
        case 2: return ld_in16(reinterpret_cast<const unsigned short*>(b.vals) + i);
        default: return ld_in8(b.vals + i);
    }
}
// ---- raw text (NEXT-2, reading R20): a word is a maximal run of bytes other than ' ', '\n', '\t',
// '\r'; in text batches record i is the word starting at byte i.
__device__ __forceinline__ bool is_sep(uint32_t c) { return c == 0x20u || c == 0x0au || c == 0x09u || c == 0x0du; }
__device__ __forceinline__ uint32_t text_word_len(const uint8_t* t, uint64_t n, uint64_t s) {
    uint64_t e = s;
    while (e < n && !is_sep(ld_in8(t + e))) ++e;
    const uint64_t L = e - s;
    return L > 0xffffffffull ? 0xffffffffu : (uint32_t)L;
}
// first word start at or after byte i (n if none)
__device__ __forceinline__ uint64_t text_next_word(const uint8_t* t, uint64_t n, uint64_t i) {
    if (i > 0 && i < n && !is_sep(ld_in8(t + i - 1)))  // inside a word: skip to its end
        while (i < n && !is_sep(ld_in8(t + i))) ++i;
    while (i < n && is_sep(ld_in8(t + i))) ++i;
    return i;
}
__device__ __forceinline__ void rec_key(const Batch& b, uint64_t i, uint64_t& s, uint32_t& len) {
    if (b.text) { s = i; len = text_word_len(b.keys, b.n, i); return; }
    i = rec_index(b, i);
    if (b.ko) {
        s = ld_in64(b.ko + i);
        len = (uint32_t)(ld_in64(b.ko + i + 1) - s);
    } else {
        s = i * (uint64_t)b.kw;
        len = b.kw;
    }
}
// GROUP value bytes of record i
__device__ __forceinline__ void rec_val_span(const Batch& b, uint64_t i, uint64_t& s, uint32_t& len) {
    i = rec_index(b, i);
    if (b.vo) {
        s = ld_in64(b.vo + i);
        len = (uint32_t)(ld_in64(b.vo + i + 1) - s);
    } else {
        s = i * (uint64_t)b.vw;
        len = b.vw;
    }
}

// ---------------------------------------------------------------- GROUP value-list helpers
// Value chunks hold fixed-width values (vw > 0: capacity and fill count slots) or variable-length
// values (vw == 0: items {u32 length, bytes, pad to 4}; capacity and fill count bytes; an unused
// tail after a reservation that did not fit is closed by a 0xffffffff length).
constexpr uint32_t ITEM_END = 0xffffffffu;
__device__ __forceinline__ uint32_t item_units(uint32_t vw, uint32_t vlen) { return vw ? 1u : ((4u + vlen + 3u) & ~3u); }
// Capacity for `need` units about to be appended: twice the demand (at least 8 slots / 64 bytes).
// Sized by the demand rather than grown from the previous chunk: many CTAs may find a key's head
// chunk full at once and each installs a chunk, so large geometric chunks would mostly stay empty
// (measured: 8x slot over-allocation on C4 with doubling).
__device__ __forceinline__ uint32_t chunk_cap(const Dev& d, uint32_t need, uint32_t vw) {
    const uint32_t unit = vw ? vw : 1u;
    const uint32_t maxcap = (d.page_bytes / 4 - CHUNK_HDR) / unit;
    uint32_t c = max(vw ? 8u : 64u, 2u * need);
    c = min(c, max(maxcap, need));
    return min(c, (d.page_bytes - CHUNK_HDR) / unit);
}
__device__ __forceinline__ uint32_t chunk_bytes(uint32_t cap, uint32_t vw) { return align16(CHUNK_HDR + cap * (vw ? vw : 1u)); }
// capacity (units) of a chunk of `size` bytes: every unit the 16-byte aligned record holds
__device__ __forceinline__ uint32_t chunk_capacity(uint32_t size, uint32_t vw) { return (size - CHUNK_HDR) / (vw ? vw : 1u); }
__device__ __forceinline__ uint64_t vref_of(const Dev& d, uint64_t off) { return ((uint64_t)d.gen << 40) | (uint64_t)off_ref(off); }
__device__ __forceinline__ bool vref_resident(const Dev& d, uint64_t vref) { return vref != 0 && (uint32_t)(vref >> 40) == d.gen; }
__device__ __forceinline__ uint8_t* vref_ptr(const Dev& d, uint64_t vref) { return ref_ptr(d, (uint32_t)vref); }
// owner identity of a key entry: birth generation << 40 | entry ref
__device__ __forceinline__ uint64_t owner_of(const Dev& d, uint8_t* e) {
    uint32_t birth = ldcg32(entry_val(e, ldcg32(e + 12)) + 8);
    return ((uint64_t)birth << 40) | (uint64_t)off_ref((uint64_t)(e - d.pool));
}
__device__ __forceinline__ unsigned long long* list_head(uint8_t* e) {
    return reinterpret_cast<unsigned long long*>(entry_val(e, ldcg32(e + 12)));
}
// a chunk of `cap` units: fill (CHUNK_PRIVATE for a CTA's private chunk) and owner key identity
__device__ __forceinline__ void init_chunk(uint8_t* c, uint32_t cap, uint32_t vwslot, uint32_t fill, uint64_t owner) {
    *reinterpret_cast<uint32_t*>(c) = chunk_bytes(cap, vwslot) | (vwslot ? K_VCHUNK : K_VCHUNKV);
    *reinterpret_cast<uint32_t*>(c + 4) = fill;
    *reinterpret_cast<unsigned long long*>(c + 8) = owner;
}
// push chunk `cref` (header already written) onto the list head of key entry e: one release-
// exchange. The list is never walked (device code only reserves in the head chunk; the host export
// attaches chunks to keys by their owner identity), so chunks keep no `next` link and no CAS retry
// loop serialises the CTAs that push onto a hot key at once.
__device__ __forceinline__ void push_chunk(uint8_t* e, uint64_t cref) {
    unsigned long long* head = list_head(e);
    unsigned long long old;
    asm volatile("atom.release.gpu.global.exch.b64 %0, [%1], %2;" : "=l"(old) : "l"(head), "l"(cref) : "memory");
    (void)old;
}
// Reserve `units` (1 slot, or an item's bytes) in the resident head chunk of key entry e (vw: the
// batch's value format). Returns 1 and the first unit in *base if the whole reservation fits, else 0.
// A reservation that crosses the end of a variable-value chunk closes the chunk's tail with ITEM_END.
__device__ __forceinline__ uint32_t reserve_head(const Dev& d, uint8_t* e, uint32_t units, uint32_t vw, uint64_t* cref,
                                                 uint32_t* base) {
    const uint64_t h = ld_relaxed_u64(list_head(e));
    *cref = 0;
    if (!vref_resident(d, h)) return 0;
    uint8_t* c = vref_ptr(d, h);
    const uint32_t cap = chunk_capacity(ldcg32(c) & ~KIND_MASK, vw);
    if (ldcg32(c + 4) >= cap) return 0;  // full (or private: the fill carries CHUNK_PRIVATE)
    const uint32_t old = atomicAdd(reinterpret_cast<unsigned int*>(c + 4), units);
    if (old + units > cap) {
        if (old + 4 <= cap && vw == 0) *reinterpret_cast<uint32_t*>(c + CHUNK_HDR + old) = ITEM_END;
        return 0;
    }
    *cref = h;
    *base = old;
    return 1;
}

// ================================================================ COMBINE insert (a1..a7): hot set + streaming warps
// Zipf inputs put most records on a few keys (C2: the top 2048 words are 52 % of all words), and
// same-address global atomics serialise (the paper's Word Count contention).
// So a COMBINE batch runs in two steps:
//   (i)  hot-set discovery: a strided sample of the batch is counted in a scratch table; the
//        keys whose sample count clears a threshold (at most HOT_K of them) are looked up or
//        inserted in the table (value 0), giving their resident entry refs;
//   (ii) insert_stream_kernel: one CTA per SM loads the hot set into shared memory (read-only
//        for the whole launch) next to a pending-sum array; every warp then streams 32-record
//        groups with no CTA barrier: key words + hash in registers, __match_any_sync folds equal
//        keys of the warp, the leader adds to the hot key's pending sum in shared memory, or
//        walks the global chain (red.add on a hit; allocate + CAS-link on a miss; POSTPONE if the
//        pool is exhausted), and a __ballot_sync writes the bitmap word. Pending sums are added to
//        the global entries when the CTA finishes (hot entries are resident for the whole
//        generation, so each record's SUCCESS is final).
namespace hot {
#ifndef SEPO_HOT_K
#define SEPO_HOT_K 2048
#endif
constexpr int K = SEPO_HOT_K;    // hot keys at most (a power of two)
constexpr uint32_t EMPTY_LEN = 0xffffffffu;
__device__ __forceinline__ uint32_t fp(uint64_t h) { return (uint32_t)(h >> 32) | 1u; }  // 0 = empty
constexpr int SAMPLE_SLOTS = 1 << 20;  // global scratch table for the sample
struct Entry {                   // one hot key (global list, built by hot_select / hot_resolve)
    uint64_t h, w0, w1;
    uint32_t len, ref;           // ref = resident entry (0: not usable)
    uint64_t src;                // input byte offset of a representative record (tail bytes)
    uint32_t count, pad;         // sample count (placement priority)
};
// Keys claim hot slots in rounds of decreasing sample count (log2 classes): when both of a key's
// buckets are full, the key left out is one of the least frequent ones, never a Zipf head
// (losing a head key sends a few % of all records to one global address).
__device__ __forceinline__ int count_class(uint32_t c) { return 31 - __clz(c | 1u); }
struct SampleSlot { unsigned long long h; unsigned int count, pad; unsigned long long rec; };
}  // namespace hot

__device__ __forceinline__ void red_add_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// hash + first 16 key bytes of record i
__device__ __forceinline__ void rec_hash16(const Dev& d, const Batch& b, uint64_t i, uint64_t& s, uint32_t& len,
                                           uint64_t& w0, uint64_t& w1, uint64_t& h) {
    if (b.wire) {  // a routed record: key words and length in the record
        const WireRec r = b.wire[i];
        s = 0; w0 = r.w0; w1 = r.w1; len = (uint32_t)r.len;
        h = hash_key16(len, d.seed, w0, w1, nullptr);
        return;
    }
    rec_key(b, i, s, len);
    const uint8_t* p = b.keys + s;
    load_key16(p, len, w0, w1);
    h = hash_key16(len, d.seed, w0, w1, p);
}

// (i-a) count a strided sample of the batch: record i = j * stride
__global__ void __launch_bounds__(256) hot_sample_kernel(Dev d, Batch b, uint64_t stride, uint64_t n_sample,
                                                         hot::SampleSlot* tab) {
    for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < n_sample; j += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t i = j * stride;
        if (b.text) {  // the first word starting at or after the sampled byte
            i = text_next_word(b.keys, b.n, i);
            if (i >= b.n) continue;
        }
        uint64_t s, w0, w1, h; uint32_t len;
        rec_hash16(d, b, i, s, len, w0, w1, h);
        const unsigned long long key = h | 1ull;  // 0 marks an empty slot
        uint32_t pos = (uint32_t)(h >> 20) & (hot::SAMPLE_SLOTS - 1);
        for (int probe = 0; probe < 32; ++probe) {
            const unsigned long long cur = atomicCAS(&tab[pos].h, 0ull, key);
            if (cur == 0ull) { tab[pos].rec = i; atomicAdd(&tab[pos].count, 1u); break; }
            if (cur == key) { atomicAdd(&tab[pos].count, 1u); break; }
            pos = (pos + 1) & (hot::SAMPLE_SLOTS - 1);
        }
    }
}

// (i-b) threshold = smallest count such that at most K keys reach it; emit those keys.
// (Hash-identified: two keys with the same 64-bit hash would share a sample slot; the hot set is
// only a cache, so a wrong pick costs speed, never correctness — entries are matched on bytes.)
constexpr int HOT_HIST = 4096;
__global__ void __launch_bounds__(256) hot_hist_kernel(const hot::SampleSlot* tab, unsigned int* hist, uint32_t min_count) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < hot::SAMPLE_SLOTS; i += gridDim.x * blockDim.x) {
        const unsigned c = tab[i].count;
        if (tab[i].h != 0ull && c >= min_count) atomicAdd(&hist[min(c, (unsigned)HOT_HIST - 1)], 1u);
    }
}
// threshold = min { c >= min_count : S(c) <= kmax }, S(c) = keys whose sample count is >= c
// (a suffix sum over the histogram; one CTA, 4 bins per thread)
__global__ void __launch_bounds__(1024) hot_threshold_kernel(unsigned int* hist, uint32_t min_count, uint32_t kmax) {
    __shared__ unsigned int warp_sum[32];
    __shared__ unsigned int s_thr;
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    constexpr int PER = HOT_HIST / 1024;
    // thread t owns bins [HOT_HIST - PER*(t+1), HOT_HIST - PER*t): thread 0 holds the top bins
    unsigned int v[PER], tot = 0;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
        const int c = HOT_HIST - 1 - (int)(PER * tid) - k;
        v[k] = c >= (int)min_count ? hist[c] : 0u;
        tot += v[k];
    }
    unsigned int incl = tot;  // inclusive prefix over threads (top bins first)
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned int y = __shfl_up_sync(FULLMASK, incl, o);
        if (lane >= (uint32_t)o) incl += y;
    }
    if (lane == 31) warp_sum[warp] = incl;
    if (tid == 0) s_thr = 0xffffffffu;
    __syncthreads();
    unsigned int before = 0;
    for (uint32_t w = 0; w < warp; ++w) before += warp_sum[w];
    unsigned int acc = before + incl - tot;  // S of the bin just above this thread's range
#pragma unroll
    for (int k = 0; k < PER; ++k) {
        const int c = HOT_HIST - 1 - (int)(PER * tid) - k;
        acc += v[k];
        if (c >= (int)min_count && acc <= kmax) atomicMin(&s_thr, (unsigned int)c);
    }
    __syncthreads();
    if (tid == 0) hist[HOT_HIST] = s_thr;
}
__global__ void __launch_bounds__(256) hot_emit_kernel(Dev d, Batch b, const hot::SampleSlot* tab, const unsigned int* hist,
                                                       hot::Entry* out, unsigned int* n_out, uint32_t kmax) {
    const unsigned thr = hist[HOT_HIST];
    if (thr == 0xffffffffu) return;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < hot::SAMPLE_SLOTS; i += gridDim.x * blockDim.x) {
        const unsigned c = tab[i].count;
        if (tab[i].h != 0ull && c >= thr) {
            const unsigned j = atomicAdd(n_out, 1u);
            if (j < kmax) {
                uint64_t s, w0, w1, h; uint32_t len;
                rec_hash16(d, b, tab[i].rec, s, len, w0, w1, h);
                hot::Entry e;
                e.h = h; e.w0 = w0; e.w1 = w1; e.len = len; e.ref = 0; e.src = s; e.count = c; e.pad = 0;
                out[j] = e;
            }
        }
    }
}
__global__ void hot_clamp_kernel(unsigned int* n_out, uint32_t kmax) { if (threadIdx.x == 0 && *n_out > kmax) *n_out = kmax; }

// (i-c) one CTA on allocator slot 0: look up / insert (value 0) every hot key
__global__ void __launch_bounds__(1024) hot_resolve_kernel(Dev d, Batch b, hot::Entry* list, const unsigned int* n_list) {
    __shared__ unsigned long long s_cur;
    __shared__ unsigned long long s_dead;
    if (threadIdx.x == 0) { s_cur = d.cursors[0]; s_dead = 0; }
    __syncthreads();
    const unsigned n = *n_list;
    for (unsigned j0 = 0; j0 < n; j0 += blockDim.x) {
        const unsigned j = j0 + threadIdx.x;
        const bool act = j < n;
        hot::Entry e = act ? list[j] : hot::Entry{};
        const uint8_t* tail = b.keys + e.src + 16;
        const uint32_t bkt = act ? bucket_of(e.h, d.n_buckets) : 0;
        const uint32_t tag = tag_of(e.h);
        uint32_t head = 0;
        uint8_t* found = nullptr;
        if (act) {
            head = ld_dir(d.dir + bkt);
            found = chain_find_w(d, head, 0, tag, e.len, e.w0, e.w1, tail);
        }
        const uint32_t esize = centry_size(e.len);
        bool need = act && !found && e.len <= 65535u - 64u && esize <= d.page_bytes && !inject_fail(d, e.h, j);
        uint32_t ref = found ? off_ref((uint64_t)(found - d.pool)) : 0u;
        const uint64_t off = warp_alloc(d, &s_cur, need, esize, (uint8_t)PAGE_ENTRY);
        if (need && off != ~0ull) {
            uint8_t* ne = d.pool + off;
            *reinterpret_cast<uint4*>(ne) = make_uint4(esize | K_COMBINE, head, tag, e.len);
            if (e.len > 0) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF) = e.w0;
            if (e.len > 8) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF + 8) = e.w1;
            if (e.len > 16) store_key(ne + KEY_OFF + 16, tail, e.len - 16);
            *reinterpret_cast<unsigned long long*>(entry_val(ne, e.len)) = 0ull;
            ref = off_ref(off);
            while (true) {
                const uint32_t old = cas_release(d.dir + bkt, head, ref);
                if (old == head) break;
                uint8_t* w = chain_find_w(d, old, head, tag, e.len, e.w0, e.w1, tail);
                if (w) {
                    *reinterpret_cast<uint32_t*>(ne) = esize | K_DEAD;
                    atomicAdd(&s_dead, (unsigned long long)esize);
                    ref = off_ref((uint64_t)(w - d.pool));
                    break;
                }
                head = old;
                *reinterpret_cast<uint32_t*>(ne + 4) = head;
            }
        }
        if (act) list[j].ref = ref;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        d.cursors[0] = s_cur;
        if (s_dead) atomicAdd(&d.ctrl->dead_bytes, s_dead);
    }
}

namespace stream {
#ifndef SEPO_STREAM_THREADS
#define SEPO_STREAM_THREADS 1024  // one persistent CTA per SM (register-bound: 64 regs x 1024)
#endif
#ifndef SEPO_CHUNK_GROUPS
#define SEPO_CHUNK_GROUPS 32      // consecutive 32-record groups a warp streams before it strides
#endif
constexpr int THREADS = SEPO_STREAM_THREADS;
constexpr uint64_t CH = SEPO_CHUNK_GROUPS;
constexpr int QCAP = 64;          // per-warp miss queue (slots): < 32 waiting + one group's 32
struct CtaState {                 // allocator slot (the CTA's active pages) + per-launch counters
    unsigned long long cur[2];
    unsigned long long post, toolarge, dead, pkb;
    unsigned long long wpost[32], wpkb[32];  // per-warp postponed records / key bytes (lane 0 only, no atomics)
};
// Shared memory of the COMBINE stream kernel: the hot set (read-only keys + per-CTA pending sums)
// and one miss queue per warp (records that missed the hot set, resolved 32 at a time).
// slot word of the direct-indexed hot sets: fingerprint (hash bits + the key length saturated at
// 255) | 1 | key index (B bits); 0 marks an empty slot
template <int B>
__device__ __forceinline__ uint32_t dfp_b(uint64_t h, uint32_t len) {
    return ((((uint32_t)(h >> (64 - (23 - B))) << 8) | min(len, 255u)) << (B + 1)) | (1u << B);
}
// Direct-indexed hot set: DS one-word slots (2-choice, one slot per choice); a slot holds the key's
// fingerprint and its index into the dense key arrays, so a probe is two 4-byte loads, two
// compares and one 16-byte key load.
#ifndef SEPO_HOT_DS
#define SEPO_HOT_DS 8192  // 16384 measured slower: the 32 KB it takes from L1 cost C2 0.5x pass 1
#endif                       // 25.5 -> 22.7 ms, C2 4x 19.6 -> 19.3, C3 1x 48.4 -> 47.1 (4096: = 8192)
constexpr int DS = SEPO_HOT_DS;           // slots (2048 hot keys in 8192: load <= 1/4)
constexpr int NKEY = hot::K;
constexpr int IDXB = NKEY <= 2048 ? 11 : (NKEY <= 4096 ? 12 : 13);  // key-index bits of a slot word
__device__ __forceinline__ uint32_t ds1(uint64_t h) { return (uint32_t)(h >> 3) & (DS - 1); }
__device__ __forceinline__ uint32_t ds2(uint64_t h) { return (uint32_t)(h >> 17) & (DS - 1); }
// slot word: fingerprint (12 hash bits + the key length saturated at 255) | 1 | key index (11 bits)
__device__ __forceinline__ uint32_t dfp(uint64_t h, uint32_t len) {
    return dfp_b<IDXB>(h, len);
}
template <bool VALS, int WARPS>
struct Smem {
    uint32_t tags[DS];            // slot words (0: empty)
    ulonglong2 kw[NKEY];          // first 16 key bytes, zero padded (one 16-B load per candidate)
    uint32_t ref[NKEY];           // resident entry (0: empty slot)
    typename std::conditional<VALS, unsigned long long, unsigned int>::type sum[NKEY];  // pending sums
    struct Queue {                // structure of arrays, QCAP slots, ring indexed by a warp counter
        unsigned long long w0[QCAP], w1[QCAP], h[QCAP], s[QCAP];
        typename std::conditional<VALS, unsigned long long, unsigned char>::type v[VALS ? QCAP : 1];
        uint32_t g[QCAP];         // group of the record
        uint32_t ll[QCAP];        // key length << 5 | lane of the record in its group
    } q[WARPS];
    CtaState cs;
};
#if SEPO_HOT_K == 2048  // (experiments with more hot keys only fit the implicit-value kernel)
static_assert(sizeof(Smem<true, SEPO_STREAM_THREADS / 32>) <= 232448, "stream kernel shared memory > 227 KB");
#endif
static_assert(sizeof(Smem<false, SEPO_STREAM_THREADS / 32>) <= 232448, "stream kernel shared memory > 227 KB");
// A warp streams chunks of CH consecutive groups; chunk c belongs to warp c mod nw.
__device__ __forceinline__ uint32_t next_group(uint32_t g, uint32_t nw) {
    return ((g + 1) % (uint32_t)CH) ? g + 1 : g + 1 + (nw - 1) * (uint32_t)CH;
}
}  // namespace stream

__device__ __forceinline__ void smem_add_u64(unsigned int* lo, unsigned int* hi, uint64_t v) {
    const unsigned int vl = (unsigned int)v;
    const unsigned int old = atomicAdd(lo, vl);
    const unsigned int carry = (old + vl < old) ? 1u : 0u;
    const unsigned int vh = (unsigned int)(v >> 32) + carry;
    if (vh) atomicAdd(hi, vh);
}

// Warp-cooperative load of 32 consecutive records (group g): each lane loads one key offset
// (the next lane's offset is its end), then the warp's contiguous key bytes are read as 16-B
// chunks — lane L loads chunk L with one coalesced 128-bit load — and every lane assembles its
// first 16 key bytes from the two chunks that hold them (__shfl_sync + funnel shifts). Falls back
// to per-lane loads when the group's key bytes exceed 512 B (long keys) or the batch is indexed.
__device__ __forceinline__ void warp_load_group(const Batch& b, uint64_t g, uint32_t lane, bool valid, uint64_t& s,
                                                uint32_t& len, uint64_t& w0, uint64_t& w1) {
    const uint64_t i = g * 32 + lane;
    if (b.idx) {  // re-issued records are not contiguous (warp-uniform branch)
        s = 0; len = 0; w0 = 0; w1 = 0;
        if (valid) { rec_key(b, i, s, len); load_key16(b.keys + s, len, w0, w1); }
        return;
    }
    uint64_t e;
    if (b.ko) {
        s = valid ? ld_in64(b.ko + i) : 0ull;
        e = __shfl_down_sync(FULLMASK, s, 1);
        const bool last = valid && (lane == 31 || i + 1 >= b.n);
        if (last) e = ld_in64(b.ko + i + 1);
    } else {
        s = i * (uint64_t)b.kw;
        e = s + b.kw;
    }
    len = valid ? (uint32_t)(e - s) : 0u;
    const uint64_t base = __shfl_sync(FULLMASK, s, 0);
    const unsigned vm = __ballot_sync(FULLMASK, valid);
    const uint32_t lastl = 31 - __clz(vm | 1u);
    const uint64_t end = __shfl_sync(FULLMASK, e, lastl);
    const uint64_t base_al = base & ~15ull;
    const uintptr_t kaddr = reinterpret_cast<uintptr_t>(b.keys);
    if (end - base_al > 512 || (kaddr & 15)) {  // warp-uniform fallback
        w0 = 0; w1 = 0;
        if (valid) load_key16(b.keys + s, len, w0, w1);
        return;
    }
    uint4 ch = make_uint4(0, 0, 0, 0);
    if (base_al + 16ull * lane < end) ch = ld_in128(b.keys + base_al + 16ull * lane);
    const uint32_t off = (uint32_t)(s - base_al);
    const uint32_t c0 = valid ? (off >> 4) : 0u, c1 = min(c0 + 1u, 31u);
    const uint32_t x0 = __shfl_sync(FULLMASK, ch.x, c0), x1 = __shfl_sync(FULLMASK, ch.y, c0);
    const uint32_t x2 = __shfl_sync(FULLMASK, ch.z, c0), x3 = __shfl_sync(FULLMASK, ch.w, c0);
    const uint32_t y0 = __shfl_sync(FULLMASK, ch.x, c1), y1 = __shfl_sync(FULLMASK, ch.y, c1);
    const uint32_t y2 = __shfl_sync(FULLMASK, ch.z, c1), y3 = __shfl_sync(FULLMASK, ch.w, c1);
    const uint64_t X0 = ((uint64_t)x1 << 32) | x0, X1 = ((uint64_t)x3 << 32) | x2;
    const uint64_t Y0 = ((uint64_t)y1 << 32) | y0, Y1 = ((uint64_t)y3 << 32) | y2;
    const uint32_t r = off & 15u, sh = 8u * (r & 7u);
    const uint64_t q0 = r < 8 ? X0 : X1, q1 = r < 8 ? X1 : Y0, q2 = r < 8 ? Y0 : Y1;
    w0 = sh ? (q0 >> sh) | (q1 << (64 - sh)) : q0;
    w1 = sh ? (q1 >> sh) | (q2 << (64 - sh)) : q1;
    if (!valid || len == 0) { w0 = 0; w1 = 0; }
    else if (len < 8) { w0 &= (1ull << (8 * len)) - 1ull; w1 = 0; }
    else if (len < 16) w1 &= (1ull << (8 * (len - 8))) - 1ull;
}

// ---- software-pipelined input of the COMBINE stream (contiguous batches)
// Stage 1 (two groups ahead): the lanes' key offsets (and fixed-width values), plain loads.
// Stage 2 (one group ahead): the group's key bytes as 16-B chunks, chunk `lane` per lane, over the
//   window [start of record 0, start of record 31 + 16) — the first 16 bytes of every key —
//   clamped to the batch's key end. Only the starts are needed, so it is issued as soon as stage 1
//   of that group landed. Groups whose window exceeds 512 B (long keys) load per lane instead.
// Stage 3 (the group itself): ends by shuffle (lane 31: the next group's first start, or one
//   load at a chunk boundary), first 16 key bytes assembled from the chunks (shuffles + funnel).
// Indexed batches (re-issue lists) skip the pipeline and load per lane.
struct InCtx {
    uint32_t ngroups, nw, tail;  // groups, warps in the grid, records in the last group (1..32)
    uint64_t kend;               // key bytes end of the batch (ko[n] or n*kw)
    bool kal;                    // key bytes 16-byte aligned (chunked loads allowed)
    bool dirpf;                  // L2-prefetch a queued miss's directory word (the table exceeds L2)
};
// input forms of a batch (template parameter of the stream kernel): contiguous CSR keys, fixed-
// width keys, or a re-issue index list into the caller's arrays
enum { IN_CSR = 0, IN_FIXED = 1, IN_IDX = 2, IN_WIRE = 3 };  // (IN_WIRE: lean kernel only)
// records in group g (1..32); g < ngroups
__device__ __forceinline__ uint32_t group_cnt(const InCtx& c, uint32_t g) { return g + 1 == c.ngroups ? c.tail : 32u; }
// (CSR: at the last group of a warp's chunk, lane 31 also loads the end of its key — the start of the
// next group, which this warp does not stream — here, two groups ahead, as the low 32 bits in
// `eo`; loaded in stage 3 instead it shared a scoreboard with the loads in flight and stalled)
template <int IN, bool VALS>
__device__ __forceinline__ void in_stage1(const Batch& b, const InCtx& c, uint32_t g, uint32_t lane, uint64_t& s,
                                          uint64_t& v, uint32_t& eo) {
    s = 0;
    v = 1;
    if (IN == IN_IDX || g >= c.ngroups || lane >= group_cnt(c, g)) return;
    const uint64_t i = (uint64_t)g * 32 + lane;
    if (IN == IN_CSR) {
        s = ld_in64(b.ko + i);
        if (lane == 31 && (g + 1) % (uint32_t)stream::CH == 0) eo = ld_in32(b.ko + i + 1);
    }
    if (VALS) v = rec_value(b, i);
}
// Stage 2: the group's key-byte window [base & ~15, min(start of its last record + 16, kend)) —
// the first 16 bytes of every key — as 16-B chunks, chunk `lane` per lane. `win` returns the low
// 32 bits of the aligned window base with bit 0 = the window was loaded (fits 32 x 16 B).
template <int IN, bool PF = false>
__device__ __forceinline__ uint4 in_stage2(const Batch& b, const InCtx& c, uint32_t g, uint32_t lane, uint64_t s,
                                           uint32_t& win) {
    uint4 ch = make_uint4(0, 0, 0, 0);
    win = 0;
    if (IN == IN_IDX || g >= c.ngroups) return ch;
    const uint32_t cnt = group_cnt(c, g);
    uint64_t base, last;
    if (IN == IN_CSR) {
        base = __shfl_sync(FULLMASK, s, 0);
        last = __shfl_sync(FULLMASK, s, (int)cnt - 1);
    } else {
        base = (uint64_t)g * 32 * b.kw;
        last = base + (uint64_t)(cnt - 1) * b.kw;
    }
    const uint64_t base_al = base & ~15ull;
    const uint64_t wend = min(last + 16, c.kend);
    if (PF) {  // long keys: bring the group's bytes (up to 4 KB from its first key) into L2 a group early
        const uint64_t a = (base & ~127ull) + 128ull * lane;
        if (a < min(last + 256, c.kend)) asm volatile("prefetch.global.L2 [%0];" ::"l"(b.keys + a));
    }
    const bool fast = c.kal && wend - base_al <= 512;
    win = (uint32_t)base_al | (fast ? 1u : 0u);
    if (fast && base_al + 16ull * lane < wend) ch = ld_in128(b.keys + base_al + 16ull * lane);
    return ch;
}
// Stage 3: s (in: start from stage 1; out: start), len, first 16 key bytes (zero padded)
template <int IN>
__device__ __forceinline__ void in_stage3(const Batch& b, const InCtx& c, uint32_t g, uint32_t gn, uint32_t lane,
                                          bool valid, uint64_t s_next, uint32_t eo, uint4 ch, uint32_t win, uint64_t& s,
                                          uint32_t& len, uint64_t& w0, uint64_t& w1) {
    w0 = 0; w1 = 0; len = 0;
    if (IN == IN_IDX) {
        s = 0;
        if (valid) { rec_key(b, (uint64_t)g * 32 + lane, s, len); load_key16(b.keys + s, len, w0, w1); }
        return;
    }
    if (IN == IN_CSR) {
        // lengths from the low 32 bits of the offsets (a key is shorter than 2^32 bytes)
        uint32_t e = __shfl_down_sync(FULLMASK, (uint32_t)s, 1);
        const uint32_t first_next = __shfl_sync(FULLMASK, (uint32_t)s_next, 0);
        if (g + 1 == c.ngroups && lane + 1 == c.tail) e = (uint32_t)c.kend;
        else if (lane == 31) e = (gn == g + 1) ? first_next : eo;
        len = valid ? e - (uint32_t)s : 0u;
    } else {
        s = ((uint64_t)g * 32 + lane) * b.kw;
        len = valid ? b.kw : 0u;
    }
    if (!(win & 1u)) {  // warp-uniform: window not loaded (long keys / unaligned key bytes)
        if (valid) load_key16(b.keys + s, len, w0, w1);
        return;
    }
    // every lane takes part in the shuffles (a chunk may sit in a lane past the last record)
    const uint32_t off = valid ? (uint32_t)s - (win & ~1u) : 0u;
    const uint32_t c0 = off >> 4, c1 = min(c0 + 1u, 31u);
    const uint32_t x0 = __shfl_sync(FULLMASK, ch.x, c0), x1 = __shfl_sync(FULLMASK, ch.y, c0);
    const uint32_t x2 = __shfl_sync(FULLMASK, ch.z, c0), x3 = __shfl_sync(FULLMASK, ch.w, c0);
    const uint32_t y0 = __shfl_sync(FULLMASK, ch.x, c1), y1 = __shfl_sync(FULLMASK, ch.y, c1);
    const uint32_t y2 = __shfl_sync(FULLMASK, ch.z, c1), y3 = __shfl_sync(FULLMASK, ch.w, c1);
    const uint64_t X0 = ((uint64_t)x1 << 32) | x0, X1 = ((uint64_t)x3 << 32) | x2;
    const uint64_t Y0 = ((uint64_t)y1 << 32) | y0, Y1 = ((uint64_t)y3 << 32) | y2;
    const uint32_t r = off & 15u, sh = 8u * (r & 7u);
    const uint64_t q0 = r < 8 ? X0 : X1, q1 = r < 8 ? X1 : Y0, q2 = r < 8 ? Y0 : Y1;
    const uint64_t lo = sh ? (q0 >> sh) | (q1 << (64 - sh)) : q0;
    const uint64_t hi = sh ? (q1 >> sh) | (q2 << (64 - sh)) : q1;
    // zero the bytes past the key (len < 16)
    // (PTX shl clamps the shift count at 64: ~(~0 << 64) = all ones)
    const uint32_t nb8 = 8u * min(len, 16u);
    w0 = lo & ~shl64_clamp(~0ull, nb8);
    w1 = hi & ~shl64_clamp(~0ull, nb8 > 64u ? nb8 - 64u : 0u);
}

// Resolve one record per lane (a3..a7) — a lane with act = false only takes part in the warp
// collectives: directory word, chain head entry (header + first 16 key bytes), rest of the chain;
// red.add on a match; otherwise allocate + link a new entry, or decline (certified, R15).
// Declines are OR-ed into their groups' bitmap words (stored as 0 by this warp when the groups
// were streamed, before a __syncwarp) and, in sepo_run, appended to the prepared re-issue list.
// Prepared re-issue list: a warp reserves PREP_CHUNK slots at a time from the global counter (one
// atomic per chunk, not per batch: a single counter hit by every warp serialises in L2); slots a
// warp leaves unused are closed with a sentinel length when it finishes (the reinsert pass skips them).
constexpr uint32_t PREP_CHUNK = 256;
constexpr uint32_t PREP_HOLE = 0xffffffffu;
constexpr unsigned long long PREP_HOLE32 = 0xffffull;  // 32-B records: length field of a hole
struct PrepCursor {
    unsigned long long base = 0;  // first slot of the warp's chunk
    uint32_t used = PREP_CHUNK;   // slots used in it (PREP_CHUNK: no chunk)
};
__device__ __forceinline__ void prep_close(const Batch& b, const PrepCursor& pc) {
    const uint32_t lane = lane_id();
    for (uint32_t k = pc.used + lane; k < PREP_CHUNK; k += 32) {
        const unsigned long long slot = pc.base + k;
        if (slot < b.out_cap) {
            ulonglong2* o = reinterpret_cast<ulonglong2*>(reinterpret_cast<uint8_t*>(b.out) + slot * b.prep_rb);
            if (b.prep_rb == 32) o[1] = make_ulonglong2(0ull, PREP_HOLE32 << 48);
            else o[2] = make_ulonglong2(0ull, (unsigned long long)PREP_HOLE);
        }
    }
}

// Long-key kernels (TU > 1): keys longer than COOP_LEN bytes have their tails hashed and compared by
// the whole warp, one key at a time (warp_tail_sum / warp_tail_eq); shorter tails stay per lane,
// TU words per round trip. Per-lane loops run as long as the warp's longest key, so without the
// split one URL of 200 B kept a warp at 7 of 32 active lanes (r02 C3 ncu source page: 10 of 32
// average over the kernel).
#ifndef SEPO_COOP_LEN
#define SEPO_COOP_LEN 112  // C3 1x pass 1: 80 -> 40.3 ms (est.), 96 39.3, 112 39.1, 144 40.3, no warp path 48.5
#endif
constexpr uint32_t COOP_LEN = SEPO_COOP_LEN;
// verify the tails of the lanes in `cm` (each against its own entry tail) with the whole warp
__device__ __forceinline__ bool coop_verify(unsigned cm, bool eq, const uint8_t* ek, const uint8_t* tail, uint32_t tlen) {
    const uint32_t lane = lane_id();
    while (cm) {
        const int j = __ffs(cm) - 1;
        cm &= cm - 1;
        const uint8_t* ej = reinterpret_cast<const uint8_t*>(__shfl_sync(FULLMASK, reinterpret_cast<uintptr_t>(ek), j));
        const uint8_t* pj = reinterpret_cast<const uint8_t*>(__shfl_sync(FULLMASK, reinterpret_cast<uintptr_t>(tail), j));
        const uint32_t nj = __shfl_sync(FULLMASK, tlen, j);
        const bool r = warp_tail_eq(ej, pj, nj);
        if (lane == (uint32_t)j) eq = r;
    }
    return eq;
}

// RB: bytes of a prepared re-issue record written for a declined record (32: implicit value 1)
template <int RB, int TU = 1>
__device__ __forceinline__ void resolve_core(const Dev& d, const Batch& b, stream::CtaState& S, bool act, uint64_t w0,
                                             uint64_t w1, uint64_t h, uint64_t s, uint64_t v, uint32_t len, uint32_t g,
                                             uint32_t gl, bool inj, bool& w_full, bool& w_quiet, PrepCursor& pc,
                                             bool hinted = false, uint32_t hint = 0) {
    const uint32_t lane = lane_id();
    const uint32_t bkt = bucket_of(h, d.n_buckets);
    const uint32_t tag = tag_of(h);
    const uint8_t* tail = b.keys + s + 16;
    // hinted: the caller read the bucket word earlier (and prefetched its head entry). A stale head
    // is safe: entries are only ever linked at the head, so the chain below an older head is intact;
    // a key linked after the snapshot is found by the CAS re-walk of [current head, stale head) in
    // the allocation path, or by the post-quiescence re-walk of a decline
    uint32_t head = act ? (hinted ? hint : ld_dir(d.dir + bkt)) : 0u;
    uint8_t* found = nullptr;
    const uint8_t* e = ref_ptr(d, head);
    bool eq = false;
    uint32_t nxt = 0;
    if (head) {
        const uint4 e_hd = ldcg128(e);
        const ulonglong2 e_kw = ldcg128u(e + KEY_OFF);
        // entry key words are zero padded to 8 bytes and followed by the value: a key of at most 8
        // bytes compares one word, an empty key none
        const uint64_t m0 = len ? ~0ull : 0ull, m1 = len > 8 ? ~0ull : 0ull;
        eq = e_hd.z == tag && e_hd.w == len && !((e_kw.x ^ w0) & m0) && !((e_kw.y ^ w1) & m1);
        if (TU == 1 || len <= COOP_LEN) {
            if (len > 16) eq = eq && entry_key_eq<TU>(e + KEY_OFF + 16, tail, len - 16);
        }
        nxt = e_hd.y;
    }
    // long keys (TU > 1): the head's tail compared by the whole warp (every lane takes part)
    if (TU > 1) eq = coop_verify(__ballot_sync(FULLMASK, eq && len > COOP_LEN), eq, e + KEY_OFF + 16, tail, len - 16);
    if (head) {
        found = eq ? const_cast<uint8_t*>(e) : chain_find_w<TU>(d, nxt, 0, tag, len, w0, w1, tail);
        if (found) red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(found, len)), v);
    }
    // ---- new keys: allocate + link (a5, a6), decline (a7)
    uint32_t res = R_OK;
    const uint32_t esize = centry_size(len);
    bool need = act && !found;
    if (need && (len > 65535u - 64u || esize > d.page_bytes)) { need = false; res = R_TOOLARGE; }
    if (inj && need && inject_fail(d, h, (uint64_t)g * 32 + gl)) { need = false; res = R_POST; }
    // Certified declines (R15). Allocation failure is monotone for the generation (`full`).
    // A warp announces itself in its CTA's announcement word before it may reserve entries
    // (one RMW; if the word already carries the FULL bit it backs off) and withdraws with a
    // release-add after linking them. The FULL bit is OR-ed into every word when the pool runs
    // out, so per word the RMW order decides: an announcement either precedes the bit (and is
    // counted) or sees it. A declining warp waits (once per launch) until every word shows
    // FULL with no announcement: every entry reserved before the pool ran out is then linked
    // and none can follow, so one re-walk of the chain decides the record for good — absorbed
    // now, or not resident in this generation (the residency guarantee of P:L77/P:L79).
    const bool any_need = __any_sync(FULLMASK, need);
    uint64_t off = ~0ull;
    if (any_need && !w_full) {  // cheap check first: no announcement once the pool is known full
        unsigned long long f0 = 0;
        if (lane == 0) f0 = ld_relaxed_u64(&d.ctrl->full);
        if (__shfl_sync(FULLMASK, f0, 0)) w_full = true;
    }
    if (any_need && !w_full) {
        unsigned long long* my_ann = d.ann + (uint64_t)blockIdx.x * ANN_STRIDE;
        unsigned long long a = 0;
        if (lane == 0) a = atomicAdd(my_ann, 1ull);
        a = __shfl_sync(FULLMASK, a, 0);
        if (a & ANN_FULL) w_full = true;
        else off = warp_alloc(d, &S.cur[0], need, esize, (uint8_t)PAGE_ENTRY);
        if (need && off != ~0ull) {
            uint8_t* e = d.pool + off;
            uint32_t hd = head;
            *reinterpret_cast<uint4*>(e) = make_uint4(esize | K_COMBINE, hd, tag, len);
            if (len > 0) *reinterpret_cast<unsigned long long*>(e + KEY_OFF) = w0;
            if (len > 8) *reinterpret_cast<unsigned long long*>(e + KEY_OFF + 8) = w1;
            if (len > 16) store_key<TU>(e + KEY_OFF + 16, tail, len - 16);
            *reinterpret_cast<unsigned long long*>(entry_val(e, len)) = v;
            const uint32_t me = off_ref(off);
            while (true) {  // lock-free head insertion
                const uint32_t old = cas_release(d.dir + bkt, hd, me);
                if (old == hd) break;
                uint8_t* w = chain_find_w<TU>(d, old, hd, tag, len, w0, w1, tail);
                if (w) {  // linked meanwhile by another warp: combine there, retire ours
                    red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(w, len)), v);
                    *reinterpret_cast<uint32_t*>(e) = esize | K_DEAD;
                    atomicAdd(&S.dead, (unsigned long long)esize);
                    break;
                }
                hd = old;
                *reinterpret_cast<uint32_t*>(e + 4) = hd;
            }
        }
        __syncwarp();
        if (lane == 0) add_release64(my_ann, ~0ull);  // withdraw (-1), after every link above
    }
    const bool declined = need && off == ~0ull;
    if (__any_sync(FULLMASK, declined)) {
        w_full = true;
        if (!w_quiet) {
            if (lane == 0)
                for (uint32_t cs = 0; cs < d.n_slots; ++cs)
                    while (ld_acquire_u64(d.ann + (uint64_t)cs * ANN_STRIDE) != ANN_FULL) __nanosleep(64);
            __syncwarp();
            if (declined) {
                uint8_t* w = chain_find_w<TU>(d, ld_dir(d.dir + bkt), 0, tag, len, w0, w1, tail);
                if (w) red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(w, len)), v);
                else res = R_POST;
            }
            w_quiet = true;
        } else if (declined) {
            res = R_POST;  // walked after quiescence: the miss is final
        }
    }
    // ---- outcomes -> bitmap bits (a7), one atomicOr per group word; counts for the host
    const bool out = act && res != R_OK;
    unsigned pend = __ballot_sync(FULLMASK, out);
    if (pend && b.out) {  // prepared re-issue records (sepo_run), from the warp's reserved chunk
        const unsigned pm = __ballot_sync(FULLMASK, act && res == R_POST);
        const uint32_t k = __popc(pm);
        if (pc.used + k > PREP_CHUNK) {
            prep_close(b, pc);
            unsigned long long nb = 0;
            if (lane == 0) nb = atomicAdd(b.out_n, (unsigned long long)PREP_CHUNK);
            pc.base = __shfl_sync(FULLMASK, nb, 0);
            pc.used = 0;
        }
        const unsigned long long base = pc.base + pc.used + __popc(pm & lanemask_lt());
        pc.used += k;
        if (act && res == R_POST && base >= b.out_cap && b.tbm)  // text: the list is full, mark the word
            atomicOr(b.tbm + (s >> 5), 1u << (s & 31));
        if (act && res == R_POST && base < b.out_cap) {
            constexpr uint32_t RS = RB == 48 ? 48u : 32u;  // record bytes (RB 33: 32-byte records too)
            ulonglong2* o = reinterpret_cast<ulonglong2*>(reinterpret_cast<uint8_t*>(b.out) + base * RS);
            __stcs(o, make_ulonglong2(w0, RB == 33 ? v : w1));
            if (RB == 32 || RB == 33) {
                __stcs(o + 1, make_ulonglong2(h, s | ((unsigned long long)len << 48)));
            } else {
                __stcs(o + 1, make_ulonglong2(h, s));
                __stcs(o + 2, make_ulonglong2(v, (unsigned long long)len));
            }
        }
    }
    if (pend) {
        const unsigned tl = __ballot_sync(FULLMASK, act && res == R_TOOLARGE);
        const unsigned pkb = __reduce_add_sync(FULLMASK, out ? len : 0u);
        if (lane == 0) {  // the warp's own counter slots: plain read-modify-write, no shared atomics
            const uint32_t w = (threadIdx.x >> 5) & 31u;
            S.wpost[w] += (unsigned long long)__popc(pend);
            S.wpkb[w] += (unsigned long long)pkb;
            if (tl) atomicAdd(&S.toolarge, (unsigned long long)__popc(tl));
        }
        // one fire-and-forget red.or per postponed record into its group's bitmap word (the
        // word was stored as 0 when the group was streamed, before a __syncwarp)
        if (out && b.bitmap) atomicOr(b.bitmap + g, 1u << gl);
    }
}

// Resolve up to 32 queued misses of the stream kernel, one per lane.
template <bool VALS, int WARPS, int TU>
__device__ __forceinline__ void resolve_misses(const Dev& d, const Batch& b, stream::Smem<VALS, WARPS>& S,
                                               typename stream::Smem<VALS, WARPS>::Queue& Q, uint32_t qhead,
                                               uint32_t cnt, bool inj, bool& w_full, bool& w_quiet, PrepCursor& pc) {
    const uint32_t lane = lane_id();
    const bool act = lane < cnt;
    const uint32_t k = (qhead + lane) & (stream::QCAP - 1);
    uint64_t w0 = 0, w1 = 0, h = 0, s = 0, v = 1;
    uint32_t g = 0, len = 0, gl = 0;
    if (act) {
        w0 = Q.w0[k]; w1 = Q.w1[k]; h = Q.h[k]; s = Q.s[k];
        if (VALS) v = Q.v[k];
        g = Q.g[k];
        const uint32_t ll = Q.ll[k];
        len = ll >> 5; gl = ll & 31u;
    }
    if (!VALS) resolve_core<32, TU>(d, b, S.cs, act, w0, w1, h, s, v, len, g, gl, inj, w_full, w_quiet, pc);
    else if (b.prep_fmt == 33) resolve_core<33, TU>(d, b, S.cs, act, w0, w1, h, s, v, len, g, gl, inj, w_full, w_quiet, pc);
    else resolve_core<48, TU>(d, b, S.cs, act, w0, w1, h, s, v, len, g, gl, inj, w_full, w_quiet, pc);
}

// Reinsert pass of sepo_run (a9 re-issue): the prepared records of the previous pass, 32 per warp
// step, straight into resolve_core (keys of these passes are the Zipf tail: no hot set).
#ifndef SEPO_REINS_THREADS
#define SEPO_REINS_THREADS 1024
#endif
template <int RB, int TU = 1>
__global__ void __launch_bounds__(SEPO_REINS_THREADS, 1) reinsert_kernel(Dev d, Batch b) {
    __shared__ stream::CtaState S;
    const uint32_t tid = threadIdx.x, lane = lane_id();
    if (tid == 0) {
        S.cur[0] = d.cursors[2 * blockIdx.x];
        S.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.post = 0; S.toolarge = 0; S.dead = 0; S.pkb = 0;
    }
    if (tid < 32) { S.wpost[tid] = 0; S.wpkb[tid] = 0; }
    __syncthreads();
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    bool w_full = false, w_quiet = false;
    PrepCursor pc;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    // the next step's prepared records are loaded while this step's are resolved (RB == 32 only)
    ulonglong2 n0 = make_ulonglong2(0, 0), n1 = make_ulonglong2(0, 0);
    {
        const uint64_t i0 = ((uint64_t)blockIdx.x * (blockDim.x / 32) + (tid >> 5)) * 32 + lane;
        if ((RB == 32 || RB == 33) && i0 < b.n) {
            const ulonglong2* p = reinterpret_cast<const ulonglong2*>(reinterpret_cast<const uint8_t*>(b.prep) + i0 * 32);
            n0 = __ldcs(p); n1 = __ldcs(p + 1);
        }
    }
    for (uint64_t base = ((uint64_t)blockIdx.x * (blockDim.x / 32) + (tid >> 5)) * 32; base < b.n; base += nw * 32) {
        const uint64_t i = base + lane;
        ulonglong2 r0 = make_ulonglong2(0, 0), r1 = make_ulonglong2(0, 0), r2 = make_ulonglong2(1, 0);
        if (RB == 32 || RB == 33) {
            r0 = n0; r1 = n1;
            const uint64_t inx = i + nw * 32;
            if (inx < b.n) {
                const ulonglong2* p = reinterpret_cast<const ulonglong2*>(reinterpret_cast<const uint8_t*>(b.prep) + inx * 32);
                n0 = __ldcs(p); n1 = __ldcs(p + 1);
            }
        } else
        if (i < b.n) {
            const ulonglong2* p = reinterpret_cast<const ulonglong2*>(reinterpret_cast<const uint8_t*>(b.prep) + i * (RB == 48 ? 48 : 32));
            r0 = __ldcs(p); r1 = __ldcs(p + 1);
            if (RB == 48) r2 = __ldcs(p + 2);
        }
        uint64_t s = r1.y, v = r2.x;
        uint32_t len = (uint32_t)r2.y;
        bool act;
        uint64_t kw1 = r0.y;
        if (RB == 32 || RB == 33) {  // {w0, w1 | value, h, s | len << 48}
            len = (uint32_t)(r1.y >> 48);
            s = r1.y & 0xffffffffffffull;
            v = RB == 33 ? r0.y : 1ull;
            if (RB == 33) kw1 = 0;  // keys of at most 8 bytes
            act = i < b.n && len != (uint32_t)PREP_HOLE32;
        } else {
            act = i < b.n && len != PREP_HOLE;
        }
        resolve_core<RB, TU>(d, b, S, act, r0.x, kw1, r1.x, s, v, act ? len : 0u, (uint32_t)(i >> 5), (uint32_t)(i & 31),
                             inj, w_full, w_quiet, pc);
    }
    if (b.out && pc.used < PREP_CHUNK) prep_close(b, pc);
    __syncthreads();
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cur[1];
        for (uint32_t w = 0; w < blockDim.x / 32; ++w) { S.post += S.wpost[w]; S.pkb += S.wpkb[w]; }
        if (S.post) atomicAdd(&d.ctrl->postponed, S.post);
        if (S.toolarge) atomicAdd(&d.ctrl->toolarge, S.toolarge);
        if (S.dead) atomicAdd(&d.ctrl->dead_bytes, S.dead);
        if (S.pkb) atomicAdd(&d.ctrl->kept_key_bytes, S.pkb);
    }
}

// ================================================================ BASIC insert (NEXT-3)
// The paper's basic organization: every pair is its own entry — no key compare, no
// combining; duplicates stay separate entries of the bucket's chain. A pair is POSTPONED when its
// allocator slot's open page is full and the pool has no free page (the slots play the
// paper's bucket groups, R7, and fail independently here: warp_alloc non-monotone). The pass HALTS
// once `halt_slots` slots have failed (50 % of the bucket groups): every later record of the
// pass is postponed without an attempt, and the host evicts the whole heap and restarts from the
// postponed records (R11). No race needs certifying: a postponed pair leaves nothing
// in the table, and a key may legitimately appear in several generations.
__global__ void __launch_bounds__(1024, 1) insert_basic_kernel(Dev d, Batch b, uint32_t halt_slots) {
    __shared__ unsigned long long s_cur;
    __shared__ int s_failed;
    __shared__ unsigned long long s_post[32], s_pkb[32];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    if (tid == 0) { s_cur = d.cursors[2 * blockIdx.x]; s_failed = 0; }
    if (tid < 32) { s_post[tid] = 0; s_pkb[tid] = 0; }
    __syncthreads();
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    const uint64_t ngroups = (b.n + 31) / 32;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    bool halted = false;  // warp-uniform
    for (uint64_t g = (uint64_t)blockIdx.x * (blockDim.x / 32) + warp; g < ngroups; g += nw) {
        const uint64_t i = g * 32 + lane;
        const bool valid = i < b.n;
        if (!halted) {
            unsigned int fs = 0;
            if (lane == 0) fs = ld_relaxed_u32(&d.ctrl->failed_slots);
            halted = __shfl_sync(FULLMASK, fs, 0) >= halt_slots;
        }
        uint64_t s = 0;
        uint32_t len = 0, res = R_POST;
        if (valid) rec_key(b, i, s, len);
        if (!halted) {
            uint64_t w0 = 0, w1 = 0;
            if (valid) load_key16(b.keys + s, len, w0, w1);
            const uint64_t h = hash_key16(len, d.seed, w0, w1, b.keys + s);
            const uint64_t v = valid ? rec_value(b, i) : 0ull;
            const uint32_t esize = centry_size(len);
            bool need = valid;
            res = R_OK;
            if (need && (len > 65535u - 64u || esize > d.page_bytes)) { need = false; res = R_TOOLARGE; }
            if (inj && need && inject_fail(d, h, i)) { need = false; res = R_POST; }
            const uint64_t off = warp_alloc(d, &s_cur, need, esize, (uint8_t)PAGE_ENTRY, false);
            const bool declined = need && off == ~0ull;
            if (declined) res = R_POST;
            if (__any_sync(FULLMASK, declined) && lane == 0 && atomicExch(&s_failed, 1) == 0)
                atomicAdd(&d.ctrl->failed_slots, 1u);  // this slot (bucket group) failed
            // link: the warp's new entries of one bucket form a sub-chain (lane order) that one
            // CAS puts at the head — duplicates of a Zipf head key would otherwise serialise on
            // one directory word, one CAS each
            const bool linking = need && off != ~0ull;
            const uint32_t bkt = bucket_of(h, d.n_buckets);
            const unsigned grp = __match_any_sync(FULLMASK, linking ? (unsigned long long)bkt : (1ull << 32) | lane);
            uint8_t* e = d.pool + (linking ? off : 0ull);
            const uint32_t me = linking ? off_ref(off) : 0u;
            const unsigned above = grp & ~((2u << lane) - 1u);           // group lanes after me
            const uint32_t nxt_lane = above ? (uint32_t)(__ffs(above) - 1) : lane;
            const uint32_t nxt_ref = __shfl_sync(FULLMASK, me, nxt_lane);
            const uint32_t leader = (uint32_t)(__ffs(grp) - 1), tail_lane = 31u - __clz(grp);
            if (linking) {
                *reinterpret_cast<uint4*>(e) = make_uint4(esize | K_BASIC, above ? nxt_ref : 0u, tag_of(h), len);
                if (len > 0) *reinterpret_cast<unsigned long long*>(e + KEY_OFF) = w0;
                if (len > 8) *reinterpret_cast<unsigned long long*>(e + KEY_OFF + 8) = w1;
                if (len > 16) store_key(e + KEY_OFF + 16, b.keys + s + 16, len - 16);
                *reinterpret_cast<unsigned long long*>(entry_val(e, len)) = v;
                __threadfence();
            }
            const unsigned long long tail_e = __shfl_sync(FULLMASK, (unsigned long long)(uintptr_t)e, tail_lane);
            __syncwarp();
            if (linking && lane == leader) {
                // head insertion by exchange: nothing reads a BASIC chain while the batch
                // is inserted (no key is looked up; export parses pages), so the tail's link may
                // follow the exchange — one atomic per sub-chain, no CAS retries on a hot bucket
                const uint32_t old = atomicExch(d.dir + bkt, me);
                *reinterpret_cast<uint32_t*>((uint8_t*)(uintptr_t)tail_e + 4) = old;
            }
        }
        // outcomes -> the group's bitmap word (this warp owns it) + counts (a7)
        const bool out = valid && res != R_OK;
        const unsigned pm = __ballot_sync(FULLMASK, out);
        if (lane == 0 && b.bitmap) b.bitmap[g] = pm;
        if (pm) {
            const unsigned tl = __ballot_sync(FULLMASK, valid && res == R_TOOLARGE);
            const unsigned pkb = __reduce_add_sync(FULLMASK, out ? len : 0u);
            if (lane == 0) {
                s_post[warp] += __popc(pm);
                s_pkb[warp] += pkb;
                if (tl) atomicAdd(&d.ctrl->toolarge, (unsigned long long)__popc(tl));
            }
        }
    }
    __syncthreads();
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = s_cur;
        unsigned long long post = 0, pkb = 0;
        for (uint32_t w = 0; w < blockDim.x / 32; ++w) { post += s_post[w]; pkb += s_pkb[w]; }
        if (post) atomicAdd(&d.ctrl->postponed, post);
        if (pkb) atomicAdd(&d.ctrl->kept_key_bytes, pkb);
    }
}

// The input context (groups, last group's size, warps, key bytes end, alignment) comes from the
// host as a kernel parameter: in the constant bank a loop-invariant costs one load when the
// register-bound loop (64 registers x 1024 threads) rematerialises it, not its whole computation
// (measured ~30 warp instructions per group before).
#ifndef SEPO_LONG_PF
#define SEPO_LONG_PF 1
#endif
template <bool VALS, int THREADS, int IN, int TU = 1>
__global__ void __launch_bounds__(THREADS, 1) insert_stream_kernel(Dev d, Batch b, const hot::Entry* hl,
                                                                   const unsigned int* n_hot, const InCtx c) {
    constexpr int WARPS = THREADS / 32;
    using SM = stream::Smem<VALS, WARPS>;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    SM& S = *reinterpret_cast<SM*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id();
    for (int p = tid; p < stream::NKEY; p += THREADS) { S.ref[p] = 0; S.sum[p] = 0; }
    for (int p = tid; p < stream::DS; p += THREADS) S.tags[p] = 0u;
    if (tid == 0) {
        S.cs.cur[0] = d.cursors[2 * blockIdx.x];
        S.cs.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.cs.post = 0; S.cs.toolarge = 0; S.cs.dead = 0; S.cs.pkb = 0;
    }
    if (tid < 32) { S.cs.wpost[tid] = 0; S.cs.wpkb[tid] = 0; }
    __syncthreads();
    // load the hot set (read-only during the main loop)
    const unsigned nh = hl ? *n_hot : 0u;
    for (int cls = 31; cls >= 0 && nh; --cls) {
        for (unsigned j = tid; j < nh; j += THREADS) {
            const hot::Entry e = hl[j];
            if (e.ref == 0 || hot::count_class(e.count) != cls) continue;
            if (j < (unsigned)stream::NKEY) {  // claim slot ds1, else ds2, else leave the key out
                const uint32_t f = stream::dfp(e.h, e.len) | j;
                if (atomicCAS(&S.tags[stream::ds1(e.h)], 0u, f) == 0u || atomicCAS(&S.tags[stream::ds2(e.h)], 0u, f) == 0u) {
                    S.kw[j] = make_ulonglong2(e.w0, e.w1);
                    S.ref[j] = e.ref;
                }
            }
        }
        __syncthreads();
    }
    __syncthreads();
    const bool have_hot = nh > 0;
    const bool big = b.n >= (1ull << 32);
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    typename SM::Queue& Q = S.q[tid >> 5];
    uint32_t qhead = 0, qtail = 0;  // warp-uniform ring counters
    PrepCursor pc;

    bool w_full = false, w_quiet = false;  // warp-uniform: pool ran out / quiescence observed

    // pipeline prologue: group g (stages 1+2 done), group gn (stage 1 in flight)
    uint32_t g = (blockIdx.x * WARPS + (tid >> 5)) * (uint32_t)stream::CH;
    uint64_t s_c = 0, v_c = 1, s_n = 0, v_n = 1;
    uint32_t win_c, eo_c = 0, eo_n = 0;
    in_stage1<IN, VALS>(b, c, g, lane, s_c, v_c, eo_c);
    uint4 ch_c = in_stage2<IN>(b, c, g, lane, s_c, win_c);
    uint32_t gn = stream::next_group(g, c.nw);
    in_stage1<IN, VALS>(b, c, gn, lane, s_n, v_n, eo_n);

    while (g < c.ngroups) {
        // ---- issue ahead: key chunks of gn, offsets (values) of the group after it
        uint32_t win_n;
        const uint4 ch_n = in_stage2<IN, (TU > 1 && SEPO_LONG_PF)>(b, c, gn, lane, s_n, win_n);
        const uint32_t gnn = stream::next_group(gn, c.nw);
        uint64_t s_nn, v_nn;
        uint32_t eo_nn = 0;
        in_stage1<IN, VALS>(b, c, gnn, lane, s_nn, v_nn, eo_nn);

        // ---- group g: key words + hash (a1)
        const bool valid = lane < group_cnt(c, g);
        uint64_t s = s_c, w0, w1;
        uint32_t len;
        in_stage3<IN>(b, c, g, gn, lane, valid, s_n, eo_c, ch_c, win_c, s, len, w0, w1);
        const uint64_t v = VALS ? (IN == IN_IDX ? (valid ? rec_value(b, (uint64_t)g * 32 + lane) : 0ull) : v_c) : 1ull;
        uint64_t h;
        if (TU == 1) {
            h = hash_key16<TU>(len, d.seed, w0, w1, b.keys + s);
        } else {  // long-key kernel: tails up to COOP_LEN per lane, longer ones by the whole warp
            uint64_t x = hash_head(len, d.seed, w0, w1);
            if (len > 16 && len <= COOP_LEN) x += tail_sum<TU>(b.keys + s + 16, len - 16);
            unsigned cm = __ballot_sync(FULLMASK, len > COOP_LEN);
            while (cm) {
                const int j = __ffs(cm) - 1;
                cm &= cm - 1;
                const uint64_t sj = __shfl_sync(FULLMASK, s, j);
                const uint32_t nj = __shfl_sync(FULLMASK, len, j) - 16u;
                const uint64_t r = warp_tail_sum(b.keys + sj + 16, nj);
                if (lane == (uint32_t)j) x += r;
            }
            h = fmix64(x);
        }
        // ---- hot set (a2): both 4-way fingerprint buckets, then one 16-byte key compare
        int pos = -1;
        if (have_hot) {
            const uint32_t f = stream::dfp(h, len);
            const uint32_t t1 = S.tags[stream::ds1(h)], t2 = S.tags[stream::ds2(h)];
            constexpr uint32_t IM = (1u << stream::IDXB) - 1u;
            const bool m1 = (t1 & ~IM) == f, m2 = (t2 & ~IM) == f;
            const uint32_t p = (m1 ? t1 : t2) & IM;
            const uint8_t* he = nullptr;
            if (valid && (m1 || m2)) {
                const ulonglong2 kk = S.kw[p];
                bool eq = kk.x == w0 && kk.y == w1;
                if (len > 16) {  // long key: exact length (the fingerprint saturates at 255) + tail bytes
                    he = ref_ptr(d, S.ref[p]);
                    if (TU == 1) {
                        eq = eq && ldcg32(he + 12) == len && entry_key_eq<TU>(he + KEY_OFF + 16, b.keys + s + 16, len - 16);
                    } else {
                        eq = eq && (len < 255u || ldcg32(he + 12) == len);
                        if (len <= COOP_LEN) eq = eq && entry_key_eq<TU>(he + KEY_OFF + 16, b.keys + s + 16, len - 16);
                    }
                }
                if (eq) pos = (int)p;
            }
            if (TU > 1) {
                const bool ok = coop_verify(__ballot_sync(FULLMASK, pos >= 0 && len > COOP_LEN), pos >= 0, he + KEY_OFF + 16,
                                            b.keys + s + 16, len - 16);
                if (!ok) pos = -1;
            }
        }
        // ---- fold the hits of the warp per hot slot (a2): one shared atomic per distinct key
        const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
        if (hm) {
            const unsigned grp = __match_any_sync(FULLMASK, pos >= 0 ? (unsigned)pos : (0x10000u | lane)) & hm;
            const bool leader = pos >= 0 && lane == (uint32_t)(__ffs(grp) - 1);
            if (!VALS) {
                if (leader) {
                    const unsigned add = (unsigned)__popc(grp);
                    if (!big) {  // fewer than 2^32 records: a CTA-local count cannot wrap
                        atomicAdd(reinterpret_cast<unsigned int*>(&S.sum[pos]), add);
                    } else {
                        const unsigned old = atomicAdd(reinterpret_cast<unsigned int*>(&S.sum[pos]), add);
                        if (old + add < old)  // 2^32 wrap of the CTA-local count: carry into the entry
                            red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(ref_ptr(d, S.ref[pos]), len)),
                                        1ull << 32);
                    }
                }
            } else {
                uint64_t acc = v;
                if (__any_sync(FULLMASK, __popc(grp) > 1)) {
                    acc = 0;
                    for (int xl = 0; xl < 32; ++xl) {
                        const uint64_t vx = __shfl_sync(FULLMASK, v, xl);
                        if ((grp >> xl) & 1u) acc += vx;
                    }
                }
                if (leader) atomicAdd(reinterpret_cast<unsigned long long*>(&S.sum[pos]), (unsigned long long)acc);
            }
        }
        // ---- misses: queue them (resolved 32 at a time); the group's bitmap word starts at 0
        const bool miss = valid && pos < 0;
        const unsigned mm = __ballot_sync(FULLMASK, miss);
        if (lane == 0) b.bitmap[g] = 0u;
        if (miss) {
            // the directory word is read when the queue is resolved (a few groups later): when the
            // table does not fit L2 (host decision, c.dirpf) start bringing its line in now
            if (c.dirpf)
                asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(d.dir + bucket_of(h, d.n_buckets)));
            const uint32_t k = (qtail + __popc(mm & lanemask_lt())) & (stream::QCAP - 1);
            Q.w0[k] = w0; Q.w1[k] = w1; Q.h[k] = h; Q.s[k] = s;
            if (VALS) Q.v[k] = v;
            Q.g[k] = g;
            Q.ll[k] = (len << 5) | lane;
        }
        qtail += __popc(mm);
        __syncwarp();
        if (qtail - qhead >= 32) {
            resolve_misses<VALS, WARPS, TU>(d, b, S, Q, qhead, 32, inj, w_full, w_quiet, pc);
            qhead += 32;
            __syncwarp();
        }

        // ---- rotate the pipeline
        g = gn; gn = gnn;
        s_c = s_n; v_c = v_n; ch_c = ch_n; win_c = win_n;
        s_n = s_nn; v_n = v_nn;
        eo_c = eo_n; eo_n = eo_nn;
    }
    if (qtail != qhead) resolve_misses<VALS, WARPS, TU>(d, b, S, Q, qhead, qtail - qhead, inj, w_full, w_quiet, pc);
    if (b.out && pc.used < PREP_CHUNK) prep_close(b, pc);
    __syncthreads();
    // flush the hot keys' pending sums into their resident entries
    for (int p = tid; p < stream::NKEY; p += THREADS) {
        if (S.ref[p] == 0 || S.sum[p] == 0) continue;
        uint8_t* e = ref_ptr(d, S.ref[p]);
        red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(e, ldcg32(e + 12))), (unsigned long long)S.sum[p]);
    }
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cs.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cs.cur[1];
        for (uint32_t w = 0; w < (uint32_t)WARPS; ++w) { S.cs.post += S.cs.wpost[w]; S.cs.pkb += S.cs.wpkb[w]; }
        if (S.cs.post) atomicAdd(&d.ctrl->postponed, S.cs.post);
        if (S.cs.toolarge) atomicAdd(&d.ctrl->toolarge, S.cs.toolarge);
        if (S.cs.dead) atomicAdd(&d.ctrl->dead_bytes, S.cs.dead);
        if (S.cs.pkb) atomicAdd(&d.ctrl->kept_key_bytes, S.cs.pkb);
    }
}

#ifndef SEPO_LONG_THREADS
#define SEPO_LONG_THREADS 1024
#endif
#ifndef SEPO_LONG_U
#define SEPO_LONG_U 2  // words per round trip: 2 -> C3 1x pass 1 39.1 ms; 3 40.8; 4 50.5 (spills at 64 registers)
#endif

// ================================================================ COMBINE insert, lean input path (a1..a7)
// Pass-1 COMBINE kernel for contiguous batches (CSR keys or fixed-width keys) whose keys are mostly
// short (words, u64 keys). Same method as insert_stream_kernel — the sampled hot set in shared
// memory with warp folding (a2), a per-warp miss queue resolved 32 misses at a time by resolve_core
// (a3..a7) — with an input path that costs a fraction of the instructions:
//   * every warp streams ONE contiguous range of 32-record groups (the next group is g + 1: no
//     chunk striding, no per-group stage bookkeeping);
//   * each lane loads its own key offsets ko[i] and ko[i + 1] two groups ahead (the second load is
//     an L1 hit: offsets are read L1-allocating with an L2 evict_first policy), and the aligned
//     8-byte words that hold its first 16 key bytes one group ahead (up to three predicated loads;
//     a group's ~220 key bytes sit in 2-4 L1 lines) — no window shuffles;
//   * the first 16 key bytes are assembled from 32-bit pieces with four funnel shifts.
// Keys longer than 16 bytes still work (their tail is hashed and compared from global memory) but
// the host picks insert_stream_kernel for long-key batches (mean key length > 24 B).
// A queued miss is {w0, w1}, {h, s | len << 40 | lane << 59} and its group.
namespace lean {
#ifndef SEPO_LEAN_THREADS
#define SEPO_LEAN_THREADS 1024
#endif
constexpr int THREADS = SEPO_LEAN_THREADS, WARPS = THREADS / 32, QCAP = 64;
constexpr uint64_t S_MASK = (1ull << 40) - 1;
constexpr uint32_t LEN_MAX = (1u << 19) - 1;
template <bool VALS>
struct Smem {
    uint32_t tags[stream::DS];  // direct-indexed hot slots (as insert_stream_kernel)
    ulonglong2 kw[stream::NKEY];
    uint32_t ref[stream::NKEY];
    typename std::conditional<VALS, unsigned long long, unsigned int>::type sum[stream::NKEY];
    struct Queue {
        ulonglong2 k[QCAP];   // first 16 key bytes (zero padded)
        ulonglong2 hs[QCAP];  // hash, key offset | length << 40 | lane << 59
        uint32_t g[QCAP];     // group of the record
        unsigned long long v[VALS ? QCAP : 1];
    } q[WARPS];
    stream::CtaState cs;
};
static_assert(sizeof(Smem<true>) <= 232448, "lean kernel shared memory > 227 KB");

// key offset and length of record i (CSR: two L1-allocating loads; fixed width: arithmetic)
template <int IN>
__device__ __forceinline__ void offsets(const Batch& b, uint64_t i, bool ok, uint64_t& s, uint64_t& e) {
    if (IN == IN_CSR) {
        s = ok ? ld_tail64(b.ko + i) : 0ull;
        e = ok ? ld_tail64(b.ko + i + 1) : 0ull;
    } else {
        s = i * b.kw;
        e = ok ? s + b.kw : s;
    }
}
// the aligned words holding the first min(len, 16) key bytes at keys + s (only words that hold a
// key byte are read)
__device__ __forceinline__ void key_words(const uint8_t* keys, uint64_t s, uint32_t len, uint64_t& x0, uint64_t& x1,
                                          uint64_t& x2) {
    const uintptr_t a = reinterpret_cast<uintptr_t>(keys + s);
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(a & ~(uintptr_t)7);
    const uint32_t need = len ? (uint32_t)(a & 7u) + min(len, 16u) : 0u;  // bytes from q on
    x0 = need > 0 ? ld_tail64(q) : 0ull;
    x1 = need > 8 ? ld_tail64(q + 1) : 0ull;
    x2 = need > 16 ? ld_tail64(q + 2) : 0ull;
}
// first 16 key bytes (zero padded) from the words x0..x2 that start o = (address & 7) bytes early
__device__ __forceinline__ void assemble16(uint64_t x0, uint64_t x1, uint64_t x2, uint32_t o, uint32_t len, uint64_t& w0,
                                           uint64_t& w1) {
    const bool hi = o >= 4u;
    const uint32_t t = 8u * (o & 3u);
    const uint32_t u0 = (uint32_t)x0, u1 = (uint32_t)(x0 >> 32), u2 = (uint32_t)x1, u3 = (uint32_t)(x1 >> 32);
    const uint32_t u4 = (uint32_t)x2, u5 = (uint32_t)(x2 >> 32);
    const uint32_t q0 = hi ? u1 : u0, q1 = hi ? u2 : u1, q2 = hi ? u3 : u2, q3 = hi ? u4 : u3, q4 = hi ? u5 : u4;
    const uint32_t r0 = __funnelshift_r(q0, q1, t), r1 = __funnelshift_r(q1, q2, t);
    const uint32_t r2 = __funnelshift_r(q2, q3, t), r3 = __funnelshift_r(q3, q4, t);
    const uint32_t nb8 = 8u * min(len, 16u);  // (PTX shl clamps the count at 64)
    w0 = (((uint64_t)r1 << 32) | r0) & ~shl64_clamp(~0ull, nb8);
    w1 = (((uint64_t)r3 << 32) | r2) & ~shl64_clamp(~0ull, nb8 > 64u ? nb8 - 64u : 0u);
}
}  // namespace lean

// hot set of a launch into shared memory: keys claim slot ds1, else ds2, in decreasing sample
// count (a Zipf head is never left out); read-only afterwards
template <int DSN, int NK, typename SumT>
__device__ __forceinline__ void load_hot_direct(uint32_t* tags, ulonglong2* kw, uint32_t* ref, SumT* sum,
                                                const hot::Entry* hl, const unsigned int* n_hot) {
    constexpr uint32_t M = DSN - 1;
    const uint32_t tid = threadIdx.x, nt = blockDim.x;
    for (uint32_t p = tid; p < (uint32_t)NK; p += nt) { ref[p] = 0; sum[p] = 0; }
    for (uint32_t p = tid; p < (uint32_t)DSN; p += nt) tags[p] = 0u;
    __syncthreads();
    const unsigned nh = hl ? *n_hot : 0u;
    for (int cls = 31; cls >= 0 && nh; --cls) {
        for (unsigned j = tid; j < nh && j < (unsigned)NK; j += nt) {
            const hot::Entry e = hl[j];
            if (e.ref == 0 || hot::count_class(e.count) != cls) continue;
            const uint32_t f = stream::dfp(e.h, e.len) | j;
            if (atomicCAS(&tags[(uint32_t)(e.h >> 3) & M], 0u, f) == 0u || atomicCAS(&tags[(uint32_t)(e.h >> 17) & M], 0u, f) == 0u) {
                kw[j] = make_ulonglong2(e.w0, e.w1);
                ref[j] = e.ref;
            }
        }
        __syncthreads();
    }
}

template <bool VALS, int RB>
__device__ __forceinline__ void lean_resolve(const Dev& d, const Batch& b, lean::Smem<VALS>& S,
                                             typename lean::Smem<VALS>::Queue& Q, uint32_t qhead, uint32_t cnt, bool inj,
                                             bool& w_full, bool& w_quiet, PrepCursor& pc) {
    const uint32_t lane = lane_id();
    const bool act = lane < cnt;
    const uint32_t k = (qhead + lane) & (lean::QCAP - 1);
    uint64_t w0 = 0, w1 = 0, h = 0, s = 0, v = 1;
    uint32_t g = 0, len = 0, gl = 0;
    if (act) {
        const ulonglong2 kk = Q.k[k], hs = Q.hs[k];
        w0 = kk.x; w1 = kk.y; h = hs.x;
        s = hs.y & lean::S_MASK;
        len = (uint32_t)(hs.y >> 40) & lean::LEN_MAX;
        gl = (uint32_t)(hs.y >> 59);
        g = Q.g[k];
        if (VALS) v = Q.v[k];
    }
    resolve_core<RB>(d, b, S.cs, act, w0, w1, h, s, v, len, g, gl, inj, w_full, w_quiet, pc);
}

// RB: prepared re-issue record format (32: implicit values; 33: <= 8-byte keys with values; 48)
template <bool VALS, int IN, int RB>
__global__ void __launch_bounds__(lean::THREADS, 1) insert_lean_kernel(Dev d, Batch b, const hot::Entry* hl,
                                                                       const unsigned int* n_hot, const InCtx c) {
    using SM = lean::Smem<VALS>;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    SM& S = *reinterpret_cast<SM*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id(), wid = tid >> 5;
    if (tid == 0) {
        S.cs.cur[0] = d.cursors[2 * blockIdx.x];
        S.cs.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.cs.post = 0; S.cs.toolarge = 0; S.cs.dead = 0; S.cs.pkb = 0;
    }
    if (tid < 32) { S.cs.wpost[tid] = 0; S.cs.wpkb[tid] = 0; }
    load_hot_direct<stream::DS, stream::NKEY>(S.tags, S.kw, S.ref, S.sum, hl, n_hot);
    __syncthreads();
    const bool have_hot = hl != nullptr && *n_hot > 0;
    const bool big = b.n >= (1ull << 32);
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    typename SM::Queue& Q = S.q[wid];
    uint32_t qhead = 0, qtail = 0;
    PrepCursor pc;
    bool w_full = false, w_quiet = false;
    // this warp's groups [g, gend): an equal share of the batch, streamed in order
    const uint64_t gw = (uint64_t)blockIdx.x * lean::WARPS + wid;
    uint32_t g = (uint32_t)((uint64_t)c.ngroups * gw / c.nw);
    const uint32_t gend = (uint32_t)((uint64_t)c.ngroups * (gw + 1) / c.nw);
    // pipeline: key words of group g and offsets of g + 1 in flight before group g is processed
    auto cnt_of = [&](uint32_t x) -> uint32_t { return x < gend ? (x + 1 == c.ngroups ? c.tail : 32u) : 0u; };
    // (IN_WIRE: s = 0, e = the key length, x0 / x1 = the record's key words, v = its value)
    auto wire_rec = [&](uint32_t x, uint64_t& s, uint64_t& e, uint64_t& k0, uint64_t& k1, uint64_t& v) {
        s = 0; e = 0; k0 = 0; k1 = 0; v = 0;
        if (lane < cnt_of(x)) {
            const ulonglong2* r = reinterpret_cast<const ulonglong2*>(b.wire + (uint64_t)x * 32 + lane);
            const ulonglong2 a = __ldcs(r), c2 = __ldcs(r + 1);
            k0 = a.x; k1 = a.y; v = c2.x; e = c2.y;
        }
    };
    uint64_t s_c, e_c, s_n = 0, e_n = 0, v_c = 1, x0, x1, x2 = 0;
    if (IN == IN_WIRE) {
        wire_rec(g, s_c, e_c, x0, x1, v_c);
    } else {
        const bool ok = lane < cnt_of(g);
        lean::offsets<IN>(b, (uint64_t)g * 32 + lane, ok, s_c, e_c);
        if (VALS && ok) v_c = rec_value(b, (uint64_t)g * 32 + lane);
        lean::key_words(b.keys, s_c, (uint32_t)(e_c - s_c), x0, x1, x2);
        lean::offsets<IN>(b, (uint64_t)(g + 1) * 32 + lane, lane < cnt_of(g + 1), s_n, e_n);
    }
    for (; g < gend; ++g) {
        // ---- issue ahead: key words (values) of g + 1, offsets of g + 2
        uint64_t y0, y1, y2 = 0, v_n = 1, s_nn = 0, e_nn = 0, s_w = 0, e_w = 0;
        if (IN == IN_WIRE) {
            wire_rec(g + 1, s_w, e_w, y0, y1, v_n);
        } else {
            lean::key_words(b.keys, s_n, (uint32_t)(e_n - s_n), y0, y1, y2);
            if (VALS && lane < cnt_of(g + 1)) v_n = rec_value(b, (uint64_t)(g + 1) * 32 + lane);
            lean::offsets<IN>(b, (uint64_t)(g + 2) * 32 + lane, lane < cnt_of(g + 2), s_nn, e_nn);
        }
        // ---- group g: first 16 key bytes + hash (a1)
        const bool valid = lane < cnt_of(g);
        const uint64_t s = s_c;
        const uint32_t len = (uint32_t)(e_c - s_c);  // 0 for lanes past the end
        uint64_t w0, w1;
        if (IN == IN_WIRE) { w0 = x0; w1 = x1; }
        else lean::assemble16(x0, x1, x2, (uint32_t)(reinterpret_cast<uintptr_t>(b.keys + s) & 7u), len, w0, w1);
        const uint64_t v = VALS ? v_c : 1ull;
        const uint64_t h = hash_key16(len, d.seed, w0, w1, b.keys + s);
        // ---- hot set (a2): two one-word slots, then one 16-byte key compare
        int pos = -1;
        if (have_hot) {
            const uint32_t f = stream::dfp(h, len);
            const uint32_t t1 = S.tags[stream::ds1(h)], t2 = S.tags[stream::ds2(h)];
            constexpr uint32_t IM = (1u << stream::IDXB) - 1u;
            const bool m1 = (t1 & ~IM) == f, m2 = (t2 & ~IM) == f;
            const uint32_t p = (m1 ? t1 : t2) & IM;
            if (valid && (m1 || m2)) {
                const ulonglong2 kk = S.kw[p];
                bool eq = kk.x == w0 && kk.y == w1;
                if (len > 16) {  // long key: exact length (the fingerprint saturates at 255) + tail bytes
                    const uint8_t* e = ref_ptr(d, S.ref[p]);
                    eq = eq && ldcg32(e + 12) == len && entry_key_eq(e + KEY_OFF + 16, b.keys + s + 16, len - 16);
                }
                if (eq) pos = (int)p;
            }
        }
        // ---- fold the warp's hits per hot key: one shared atomic per distinct key (a2)
        const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
        if (hm) {
            const unsigned grp = __match_any_sync(FULLMASK, pos >= 0 ? (unsigned)pos : (0x10000u | lane)) & hm;
            const bool leader = pos >= 0 && lane == (uint32_t)(__ffs(grp) - 1);
            if (!VALS) {
                if (leader) {
                    const unsigned add = (unsigned)__popc(grp);
                    if (!big) {  // fewer than 2^32 records: a CTA-local count cannot wrap (no returned value to wait for)
                        atomicAdd(reinterpret_cast<unsigned int*>(&S.sum[pos]), add);
                    } else {
                        const unsigned old = atomicAdd(reinterpret_cast<unsigned int*>(&S.sum[pos]), add);
                        if (old + add < old)  // 2^32 wrap of the CTA-local count: carry into the entry
                            red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(ref_ptr(d, S.ref[pos]), len)), 1ull << 32);
                    }
                }
            } else {
                uint64_t acc = v;
                if (__any_sync(FULLMASK, __popc(grp) > 1)) {
                    acc = 0;
                    for (int xl = 0; xl < 32; ++xl) {
                        const uint64_t vx = __shfl_sync(FULLMASK, v, xl);
                        if ((grp >> xl) & 1u) acc += vx;
                    }
                }
                if (leader) atomicAdd(reinterpret_cast<unsigned long long*>(&S.sum[pos]), (unsigned long long)acc);
            }
        }
        // ---- misses: the warp's queue, resolved 32 at a time (a3..a7); the bitmap word starts at 0
        const bool miss = valid && pos < 0;
        const unsigned mm = __ballot_sync(FULLMASK, miss);
        if (lane == 0 && b.bitmap) b.bitmap[g] = 0u;
        if (miss) {
            if (c.dirpf) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(d.dir + bucket_of(h, d.n_buckets)));
            const uint32_t k = (qtail + __popc(mm & lanemask_lt())) & (lean::QCAP - 1);
            Q.k[k] = make_ulonglong2(w0, w1);
            Q.hs[k] = make_ulonglong2(h, s | ((uint64_t)min(len, lean::LEN_MAX) << 40) | ((uint64_t)lane << 59));
            Q.g[k] = g;
            if (VALS) Q.v[k] = v;
        }
        qtail += __popc(mm);
        __syncwarp();
        if (qtail - qhead >= 32) {
            lean_resolve<VALS, RB>(d, b, S, Q, qhead, 32, inj, w_full, w_quiet, pc);
            qhead += 32;
            __syncwarp();
        }
        // ---- rotate the pipeline
        if (IN == IN_WIRE) { s_c = s_w; e_c = e_w; }
        else { s_c = s_n; e_c = e_n; }
        v_c = v_n; x0 = y0; x1 = y1; x2 = y2;
        s_n = s_nn; e_n = e_nn;
    }
    if (qtail != qhead) lean_resolve<VALS, RB>(d, b, S, Q, qhead, qtail - qhead, inj, w_full, w_quiet, pc);
    if (b.out && pc.used < PREP_CHUNK) prep_close(b, pc);
    __syncthreads();
    for (int p = tid; p < stream::NKEY; p += lean::THREADS) {  // pending hot sums -> resident entries
        if (S.ref[p] == 0 || S.sum[p] == 0) continue;
        uint8_t* e = ref_ptr(d, S.ref[p]);
        red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(e, ldcg32(e + 12))), (unsigned long long)S.sum[p]);
    }
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cs.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cs.cur[1];
        for (uint32_t w = 0; w < (uint32_t)lean::WARPS; ++w) { S.cs.post += S.cs.wpost[w]; S.cs.pkb += S.cs.wpkb[w]; }
        if (S.cs.post) atomicAdd(&d.ctrl->postponed, S.cs.post);
        if (S.cs.toolarge) atomicAdd(&d.ctrl->toolarge, S.cs.toolarge);
        if (S.cs.dead) atomicAdd(&d.ctrl->dead_bytes, S.cs.dead);
        if (S.cs.pkb) atomicAdd(&d.ctrl->kept_key_bytes, S.cs.pkb);
    }
}

// ================================================================ GROUP insert (a1..a7): hot set + streaming warps
// Multi-valued method. Same structure as the COMBINE kernel: a sampled hot set lives
// in shared memory; each hot key also owns a CTA-PRIVATE value chunk whose slots are handed out by
// a shared-memory word {chunk ref, fill} (a whole warp's values of that key reserved with one
// shared atomic); when it fills, the warp that crosses the end installs the next private chunk.
// Other keys append through the key's shared head chunk (one global atomic per record) or a new
// demand-sized chunk pushed onto the list head (release-CAS). A record whose value cannot get a
// slot while its key is resident is postponed and marks the key's page retained (pending key,
// P:L165); new-key declines are certified as in the COMBINE kernel (R15), so a GROUP pass needs no
// separate re-probe.
namespace gst {
#ifndef SEPO_GROUP_THREADS
#define SEPO_GROUP_THREADS 1024
#endif
constexpr int THREADS = SEPO_GROUP_THREADS;
constexpr int NB = 512, NH = 4 * NB;  // hot slots (2-choice 4-way buckets)
constexpr int K = 1024;               // hot keys at most
constexpr uint32_t PC_CAP = 256;      // slots of a private chunk
struct Smem {
    uint4 tags[NB];
    uint64_t h[NH], w0[NH], w1[NH];
    uint32_t len[NH], ref[NH];
    unsigned long long pw[NH];  // private chunk word: chunk ref << 32 | fill (ref 0: none)
    unsigned long long cur[2];
    unsigned long long post, toolarge, dead;
};
__device__ __forceinline__ uint32_t b1(uint64_t h) { return (uint32_t)(h >> 3) & (NB - 1); }
__device__ __forceinline__ uint32_t b2(uint64_t h) { return (uint32_t)(h >> 13) & (NB - 1); }
}  // namespace gst

// write record i's value into chunk c at unit `at` (slot index, or byte offset of the item)
__device__ __forceinline__ void put_value(const Batch& b, uint64_t i, uint8_t* c, uint32_t at) {
    if (b.vo == nullptr) {
        const uint64_t src = rec_index(b, i) * (uint64_t)b.vw;
        uint8_t* dst = c + CHUNK_HDR + (uint64_t)at * b.vw;
        if (b.vw == 4) *reinterpret_cast<uint32_t*>(dst) = ld_in32(b.vals + src);
        else if (b.vw == 8) *reinterpret_cast<unsigned long long*>(dst) = ld_in64(b.vals + src);
        else for (uint32_t x = 0; x < b.vw; ++x) dst[x] = (uint8_t)ld_in8(b.vals + src + x);
    } else {
        uint64_t vs; uint32_t vl;
        rec_val_span(b, i, vs, vl);
        uint8_t* dst = c + CHUNK_HDR + at;
        *reinterpret_cast<uint32_t*>(dst) = vl;
        for (uint32_t x = 0; x < vl; ++x) dst[4 + x] = (uint8_t)ld_in8(b.vals + vs + x);
    }
}

// GROUP hot keys: look up / insert the key entry (empty list) on allocator slot 0
__global__ void __launch_bounds__(1024) hot_resolve_group_kernel(Dev d, Batch b, hot::Entry* list, const unsigned int* n_list) {
    __shared__ unsigned long long s_cur;
    if (threadIdx.x == 0) s_cur = d.cursors[0];
    __syncthreads();
    const unsigned n = *n_list;
    for (unsigned j0 = 0; j0 < n; j0 += blockDim.x) {
        const unsigned j = j0 + threadIdx.x;
        const bool act = j < n;
        hot::Entry e = act ? list[j] : hot::Entry{};
        const uint8_t* tail = b.keys + e.src + 16;
        const uint32_t bkt = act ? bucket_of(e.h, d.n_buckets) : 0;
        const uint32_t tag = tag_of(e.h);
        uint32_t head = 0;
        uint8_t* found = nullptr;
        if (act) {
            head = ld_dir(d.dir + bkt);
            found = chain_find_w(d, head, 0, tag, e.len, e.w0, e.w1, tail);
        }
        const uint32_t esize = gkey_size(e.len);
        bool need = act && !found && e.len <= 65535u - 64u && esize <= d.page_bytes && !inject_fail(d, e.h, j);
        uint32_t ref = found ? off_ref((uint64_t)(found - d.pool)) : 0u;
        const uint64_t off = warp_alloc(d, &s_cur, need, esize, (uint8_t)PAGE_ENTRY);
        if (need && off != ~0ull) {
            uint8_t* ne = d.pool + off;
            *reinterpret_cast<uint4*>(ne) = make_uint4(esize | K_GKEY, head, tag, e.len);
            if (e.len > 0) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF) = e.w0;
            if (e.len > 8) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF + 8) = e.w1;
            if (e.len > 16) store_key(ne + KEY_OFF + 16, tail, e.len - 16);
            *reinterpret_cast<unsigned long long*>(entry_val(ne, e.len)) = 0ull;
            *reinterpret_cast<uint32_t*>(entry_val(ne, e.len) + 8) = d.gen;
            *reinterpret_cast<uint32_t*>(entry_val(ne, e.len) + 12) = 0u;
            ref = off_ref(off);
            while (true) {
                const uint32_t old = cas_release(d.dir + bkt, head, ref);
                if (old == head) break;
                uint8_t* w = chain_find_w(d, old, head, tag, e.len, e.w0, e.w1, tail);
                if (w) {
                    *reinterpret_cast<uint32_t*>(ne) = esize | K_DEAD;
                    ref = off_ref((uint64_t)(w - d.pool));
                    break;
                }
                head = old;
                *reinterpret_cast<uint32_t*>(ne + 4) = head;
            }
        }
        if (act) list[j].ref = ref;
    }
    __syncthreads();
    if (threadIdx.x == 0) d.cursors[0] = s_cur;
}

__global__ void __launch_bounds__(gst::THREADS, 1) insert_group_stream_kernel(Dev d, Batch b, const hot::Entry* hl,
                                                                              const unsigned int* n_hot) {
    using gst::THREADS; using gst::NB; using gst::NH; using gst::b1; using gst::b2;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    gst::Smem& S = *reinterpret_cast<gst::Smem*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id();
    const uint32_t PB = d.page_bytes;
    const uint32_t vw = b.vo ? 0u : b.vw;  // chunk format: fixed slots, or variable items (vw 0)
    const uint32_t PC_CAP = vw ? gst::PC_CAP : 2048u;  // private chunk capacity (slots / bytes)
    for (int p = tid; p < NH; p += THREADS) { S.len[p] = hot::EMPTY_LEN; S.pw[p] = PC_CAP; }
    for (int p = tid; p < NB; p += THREADS) S.tags[p] = make_uint4(0, 0, 0, 0);
    if (tid == 0) {
        S.cur[0] = d.cursors[2 * blockIdx.x];
        S.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.post = 0; S.toolarge = 0; S.dead = 0;
    }
    __syncthreads();
    const unsigned nh = hl ? *n_hot : 0u;
    for (int cls = 31; cls >= 0 && nh; --cls) {
        for (unsigned j = tid; j < nh; j += THREADS) {
            const hot::Entry e = hl[j];
            if (e.ref == 0 || hot::count_class(e.count) != cls) continue;
            const uint32_t f = hot::fp(e.h);
            int pos = -1;
            for (int c = 0; c < 2 && pos < 0; ++c) {
                const uint32_t bk = c == 0 ? b1(e.h) : b2(e.h);
                uint32_t* t = reinterpret_cast<uint32_t*>(&S.tags[bk]);
                for (int w = 0; w < 4 && pos < 0; ++w)
                    if (atomicCAS(&t[w], 0u, f) == 0u) pos = (int)(bk * 4 + w);
            }
            if (pos < 0) continue;
            S.h[pos] = e.h; S.w0[pos] = e.w0; S.w1[pos] = e.w1; S.ref[pos] = e.ref; S.len[pos] = e.len;
        }
        __syncthreads();
    }
    __syncthreads();
    const bool have_hot = nh > 0;
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    const uint32_t pc_bytes = chunk_bytes(PC_CAP, vw);

    // groups are handed out GS at a time from a global counter (zeroed by the host before the launch):
    // a CTA that starts late — its SM still busy with an overlapped eviction's gather — takes less work
    const uint64_t ngroups = (b.n + 31) / 32;
#ifndef SEPO_GROUP_GS
#define SEPO_GROUP_GS 16
#endif
    constexpr uint64_t GS = SEPO_GROUP_GS;  // groups per grab
    unsigned long long c_post = 0, c_tl = 0, c_dead = 0, c_pkb = 0;
    bool w_full = false, w_quiet = false;
    uint64_t g_lim = 0;
    auto next_g = [&](uint64_t cur) -> uint64_t {
        if (cur + 1 < g_lim) return cur + 1;
        unsigned long long x = 0;
        if (lane == 0) x = atomicAdd(&d.ctrl->next_group, (unsigned long long)GS);
        x = __shfl_sync(FULLMASK, x, 0);
        g_lim = min((uint64_t)x + GS, ngroups);
        return x;
    };
    for (uint64_t g = next_g(~0ull); g < ngroups; g = next_g(g)) {
        const uint64_t i = g * 32 + lane;
        const bool valid = i < b.n;
        uint64_t s, w0, w1;
        uint32_t len;
        warp_load_group(b, g, lane, valid, s, len, w0, w1);
        const uint64_t h = hash_key16(len, d.seed, w0, w1, b.keys + s);
        uint32_t units = 0;  // this record's value size in chunk units
        if (valid) {
            uint32_t vlen = vw;
            if (b.vo) { uint64_t vs; rec_val_span(b, i, vs, vlen); }
            units = item_units(vw, vlen);
        }
        const uint8_t* tail = b.keys + s + 16;
        const uint32_t tag = tag_of(h), bkt = bucket_of(h, d.n_buckets);
        // ---- hot set probe
        int pos = -1;
        if (valid && have_hot) {
            const uint32_t f = hot::fp(h);
            const uint32_t k1 = b1(h), k2 = b2(h);
            const uint4 t1 = S.tags[k1];
            int p = -1;
            if (t1.x == f) p = 4 * k1; else if (t1.y == f) p = 4 * k1 + 1;
            else if (t1.z == f) p = 4 * k1 + 2; else if (t1.w == f) p = 4 * k1 + 3;
            else {
                const uint4 t2 = S.tags[k2];
                if (t2.x == f) p = 4 * k2; else if (t2.y == f) p = 4 * k2 + 1;
                else if (t2.z == f) p = 4 * k2 + 2; else if (t2.w == f) p = 4 * k2 + 3;
            }
            if (p >= 0 && S.h[p] == h && S.len[p] == len && S.w0[p] == w0 && S.w1[p] == w1 &&
                (len <= 16 || entry_key_eq(ref_ptr(d, S.ref[p]) + KEY_OFF + 16, tail, len - 16)))
                pos = p;
        }
        uint32_t head = 0;
        if (valid && pos < 0) head = ld_dir(d.dir + bkt);
        // ---- hot keys: reserve the warp's values of a key in its private chunk (one shared atomic)
        bool done = false;
        uint8_t* e = nullptr;  // resident key entry for the global path
        {
            const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
            if (hm) {
                const unsigned key = pos >= 0 ? (unsigned)pos : (0x10000u | lane);
                const unsigned grp = __match_any_sync(FULLMASK, key) & hm;
                const uint32_t leader = grp ? (uint32_t)(__ffs(grp) - 1) : lane;
                // units of the group before this lane (excl) and in total (tot)
                uint32_t excl = __popc(grp & ((1u << lane) - 1u)), tot = __popc(grp);
                if (!vw && __any_sync(FULLMASK, pos >= 0)) {
                    excl = 0; tot = 0;
                    for (int x2 = 0; x2 < 32; ++x2) {
                        const uint32_t ux = __shfl_sync(FULLMASK, units, x2);
                        if ((grp >> x2) & 1u) { tot += ux; if ((uint32_t)x2 < lane) excl += ux; }
                    }
                }
                unsigned long long old = 0;
                if (pos >= 0 && lane == leader) old = atomicAdd(&S.pw[pos], (unsigned long long)tot);
                old = __shfl_sync(FULLMASK, old, leader);
                const uint32_t cref = (uint32_t)(old >> 32), f0 = (uint32_t)old;
                // the warp that crosses the end of the private chunk installs the next one
                const bool cross = pos >= 0 && f0 <= PC_CAP && f0 + tot > PC_CAP;
                const bool fits_old = pos >= 0 && cref && f0 + excl + units <= PC_CAP;
                // variable items: the old chunk's used extent = the prefix of the group that fits
                uint32_t used = PC_CAP;
                if (!vw) {
                    const unsigned fm = __ballot_sync(FULLMASK, fits_old) & grp;
                    const uint32_t fu = __reduce_add_sync(FULLMASK, ((fm >> lane) & 1u) ? units : 0u);
                    used = f0 + fu;
                }
                const bool want = cross && lane == leader && !w_full;
                unsigned long long ann = 0;
                const bool anyw = __any_sync(FULLMASK, want);
                uint64_t coff = ~0ull;
                if (anyw) {  // announcement protocol (R15) around the allocation
                    if (lane == 0) ann = atomicAdd(d.ann + (uint64_t)blockIdx.x * ANN_STRIDE, 1ull);
                    ann = __shfl_sync(FULLMASK, ann, 0);
                    if (ann & ANN_FULL) w_full = true;
                    else coff = warp_alloc(d, &S.cur[1], want, pc_bytes, (uint8_t)PAGE_VALUE);
                }
                uint32_t nref = 0;
                if (want) {
                    if (cref) *reinterpret_cast<uint32_t*>(ref_ptr(d, cref) + 4) = used;  // old chunk is closed
                    if (coff != ~0ull) {
                        uint8_t* c = d.pool + coff;
                        uint8_t* ke = ref_ptr(d, S.ref[pos]);
                        init_chunk(c, PC_CAP, vw, CHUNK_PRIVATE, owner_of(d, ke));
                        push_chunk(ke, vref_of(d, coff));
                        nref = off_ref(coff);
                        const uint32_t rest = vw ? f0 + tot - PC_CAP : 0u;  // fixed: the overflow goes here
                        atomicExch(&S.pw[pos], ((unsigned long long)nref << 32) | rest);
                    } else {
                        atomicExch(&S.pw[pos], (unsigned long long)PC_CAP << 1);  // no chunk: hits go global
                    }
                }
                if (anyw) {
                    __syncwarp();
                    if (lane == 0) add_release64(d.ann + (uint64_t)blockIdx.x * ANN_STRIDE, ~0ull);
                }
                nref = __shfl_sync(FULLMASK, nref, leader);
                if (pos >= 0) {
                    const uint32_t at = f0 + excl;
                    if (fits_old) { put_value(b, i, ref_ptr(d, cref), at); done = true; }
                    else if (vw && cross && nref) { put_value(b, i, ref_ptr(d, nref), at - PC_CAP); done = true; }
                    else e = ref_ptr(d, S.ref[pos]);  // overflow: this record takes the global path
                }
            }
        }
        // ---- global path: chain walk (non-hot), reserve one slot in the key's shared head chunk
        if (valid && !done && pos < 0) e = chain_find_w(d, head, 0, tag, len, w0, w1, tail);
        bool need_key = valid && !done && e == nullptr;
        bool need_chunk = valid && !done;
        if (valid && !done && e) {
            uint64_t cr = 0;
            uint32_t base = 0;
            if (reserve_head(d, e, units, vw, &cr, &base)) {
                put_value(b, i, vref_ptr(d, cr), base);
                done = true;
                need_chunk = false;
            }
        }
        uint32_t res = R_OK;
        const uint32_t ksize = gkey_size(len);
        const uint32_t ccap = chunk_cap(d, units, vw);
        const uint32_t csize = chunk_bytes(ccap, vw);
        if ((need_key && (len > 65535u - 64u || ksize > PB)) || (need_chunk && CHUNK_HDR + units * (vw ? vw : 1u) > PB)) {
            need_key = false; need_chunk = false; res = R_TOOLARGE;
        }
        if (inj && need_key && inject_fail(d, h, i)) { need_key = false; need_chunk = false; res = R_POST; }
        const bool any_need = __any_sync(FULLMASK, need_chunk);
        uint64_t koff = ~0ull, coff = ~0ull;
        if (any_need && !w_full) {
            unsigned long long f0 = 0;
            if (lane == 0) f0 = ld_relaxed_u64(&d.ctrl->full);
            if (__shfl_sync(FULLMASK, f0, 0)) w_full = true;
        }
        if (any_need && !w_full) {
            unsigned long long* my_ann = d.ann + (uint64_t)blockIdx.x * ANN_STRIDE;
            unsigned long long a = 0;
            if (lane == 0) a = atomicAdd(my_ann, 1ull);
            a = __shfl_sync(FULLMASK, a, 0);
            if (a & ANN_FULL) w_full = true;
            else {
                koff = warp_alloc(d, &S.cur[0], need_key, ksize, (uint8_t)PAGE_ENTRY);
                const bool wc = need_chunk && (!need_key || koff != ~0ull);
                coff = warp_alloc(d, &S.cur[1], wc, csize, (uint8_t)PAGE_VALUE);
            }
            if (need_key && koff != ~0ull) {  // new key entry, linked even if its chunk failed (pending)
                uint8_t* ne = d.pool + koff;
                *reinterpret_cast<uint4*>(ne) = make_uint4(ksize | K_GKEY, head, tag, len);
                if (len > 0) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF) = w0;
                if (len > 8) *reinterpret_cast<unsigned long long*>(ne + KEY_OFF + 8) = w1;
                if (len > 16) store_key(ne + KEY_OFF + 16, tail, len - 16);
                *reinterpret_cast<unsigned long long*>(entry_val(ne, len)) = 0ull;
                *reinterpret_cast<uint32_t*>(entry_val(ne, len) + 8) = d.gen;
                *reinterpret_cast<uint32_t*>(entry_val(ne, len) + 12) = 0u;
                const uint32_t me = off_ref(koff);
                e = ne;
                uint32_t hd = head;
                while (true) {
                    const uint32_t old = cas_release(d.dir + bkt, hd, me);
                    if (old == hd) break;
                    uint8_t* w = chain_find_w(d, old, hd, tag, len, w0, w1, tail);
                    if (w) {
                        *reinterpret_cast<uint32_t*>(ne) = ksize | K_DEAD;
                        c_dead += ksize;
                        e = w;
                        break;
                    }
                    hd = old;
                    *reinterpret_cast<uint32_t*>(ne + 4) = hd;
                }
            }
            if (need_chunk && coff != ~0ull && e) {
                uint8_t* c = d.pool + coff;
                init_chunk(c, ccap, vw, units, owner_of(d, e));
                put_value(b, i, c, 0);
                push_chunk(e, vref_of(d, coff));
                done = true;
            }
            __syncwarp();
            if (lane == 0) add_release64(my_ann, ~0ull);
        }
        // ---- declines: certified for new keys; a resident key with a value left over is pending
        const bool declined = valid && !done && res == R_OK;
        if (__any_sync(FULLMASK, declined)) {
            w_full = true;
            if (!w_quiet) {
                if (lane == 0)
                    for (uint32_t c = 0; c < d.n_slots; ++c)
                        while (ld_acquire_u64(d.ann + (uint64_t)c * ANN_STRIDE) != ANN_FULL) __nanosleep(64);
                __syncwarp();
                w_quiet = true;
                if (declined && !e) e = chain_find_w(d, ld_dir(d.dir + bkt), 0, tag, len, w0, w1, tail);
            }
            if (declined) {
                res = R_POST;
                if (e) {  // resident key: its value may still fit a shared head chunk
                    uint64_t cr = 0;
                    uint32_t base = 0;
                    if (reserve_head(d, e, units, vw, &cr, &base)) {
                        put_value(b, i, vref_ptr(d, cr), base);
                        res = R_OK;
                    } else {
                        d.retain[(uint32_t)((uint64_t)(e - d.pool) >> d.page_shift)] = 1;  // pending key
                    }
                }
            }
        }
        const unsigned bits = __ballot_sync(FULLMASK, valid && res != R_OK);
        if (bits) {
            const unsigned tl = __ballot_sync(FULLMASK, valid && res == R_TOOLARGE);
            const unsigned pkb = __reduce_add_sync(FULLMASK, (valid && res != R_OK) ? len : 0u);
            if (lane == 0) { c_post += __popc(bits); c_tl += __popc(tl); c_pkb += pkb; }
        }
        if (lane == 0) b.bitmap[g] = bits;
    }
    if (lane == 0) {
        if (c_post) atomicAdd(&S.post, c_post);
        if (c_tl) atomicAdd(&S.toolarge, c_tl);
        if (c_pkb) atomicAdd(&d.ctrl->kept_key_bytes, c_pkb);
    }
    if (c_dead) atomicAdd(&S.dead, c_dead);
    __syncthreads();
    // final fill of every private chunk still open
    for (int p = tid; p < NH; p += THREADS) {
        const unsigned long long w = S.pw[p];
        const uint32_t cref = (uint32_t)(w >> 32);
        if (cref) *reinterpret_cast<uint32_t*>(ref_ptr(d, cref) + 4) = min((uint32_t)w, PC_CAP);
    }
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cur[1];
        if (S.post) atomicAdd(&d.ctrl->postponed, S.post);
        if (S.toolarge) atomicAdd(&d.ctrl->toolarge, S.toolarge);
        if (S.dead) atomicAdd(&d.ctrl->dead_bytes, S.dead);
    }
}

// ================================================================ re-probe (a8)
// One warp per bitmap word. Declined records whose key is now resident are combined / appended
// and their bit cleared; per tile of RP_TILE records the remaining count and bytes are written
// for the compaction scan.
constexpr int RP_THREADS = 256;
constexpr int RP_TILE = 2048;  // 64 words, 8 per warp

template <int MODE, bool PROBE>
__global__ void __launch_bounds__(RP_THREADS) reprobe_kernel(Dev d, Batch b, unsigned long long* tile_counts) {
    __shared__ unsigned long long s_cur[2];
    __shared__ unsigned long long s_cnt[3];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    if (PROBE && tid == 0) {
        s_cur[0] = d.cursors[2 * blockIdx.x];
        s_cur[1] = d.cursors[2 * blockIdx.x + 1];
    }
    __syncthreads();
    constexpr int WPW = RP_TILE / 32 / (RP_THREADS / 32);  // bitmap words per warp per tile
    const uint64_t ntiles = (b.n + RP_TILE - 1) / RP_TILE;
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        if (tid < 3) s_cnt[tid] = 0;
        __syncthreads();
        unsigned long long c_rec = 0, c_kb = 0, c_vb = 0;
        for (int wq = 0; wq < WPW; ++wq) {
            const uint64_t w = tile * (RP_TILE / 32) + warp * WPW + wq;
            const uint64_t i = w * 32 + lane;
            if (w * 32 >= b.n) break;  // warp-uniform
            const uint32_t bits = b.bitmap[w];
            if (bits == 0) continue;  // warp-uniform
            const bool mine = (bits >> lane) & 1u;
            bool still = mine;
            uint64_t s = 0;
            uint32_t len = 0;
            if (mine) rec_key(b, i, s, len);
            if (PROBE) {
                uint8_t* e = nullptr;
                uint32_t want_cap = 0, units = 0;
                if (mine) {
                    const uint64_t h = hash_key(b.keys + s, len, d.seed);
                    const uint32_t head = ld_dir(d.dir + bucket_of(h, d.n_buckets));
                    e = chain_find(d, head, 0, tag_of(h), len, b.keys + s);
                    if (MODE == 0 && e) {  // resident: combine now
                        atomicAdd(reinterpret_cast<unsigned long long*>(entry_val(e, len)), (unsigned long long)rec_value(b, i));
                        still = false;
                    }
                    if (MODE == 1 && e) {  // resident key: append the value if its head chunk has room
                        uint64_t vs; uint32_t vl;
                        rec_val_span(b, i, vs, vl);
                        const uint32_t cvw = b.vo ? 0u : b.vw;
                        units = item_units(cvw, vl);
                        uint64_t cref = 0;
                        uint32_t base = 0;
                        if (reserve_head(d, e, units, cvw, &cref, &base)) {
                            put_value(b, i, vref_ptr(d, cref), base);
                            still = false;
                        } else {
                            want_cap = chunk_cap(d, units, cvw);
                        }
                    }
                }
                if (MODE == 1) {
                    const uint32_t cvw = b.vo ? 0u : b.vw;
                    const bool want = mine && still && e != nullptr;
                    const uint64_t coff = warp_alloc(d, &s_cur[1], want, chunk_bytes(want ? want_cap : 0, cvw),
                                                     (uint8_t)PAGE_VALUE);
                    if (want) {
                        if (coff != ~0ull) {
                            uint8_t* c = d.pool + coff;
                            init_chunk(c, want_cap, cvw, units, owner_of(d, e));
                            put_value(b, i, c, 0);
                            push_chunk(e, vref_of(d, coff));
                            still = false;
                        } else {
                            // resident key with values still pending: keep its key page
                            d.retain[(uint32_t)((uint64_t)(e - d.pool) >> d.page_shift)] = 1;
                        }
                    }
                }
                const unsigned nb = __ballot_sync(FULLMASK, still);
                if (lane == 0) b.bitmap[w] = nb;
            }
            if (still) {
                c_rec += 1;
                c_kb += len;
                if (b.vals) {
                    if (b.vo) c_vb += __ldg(reinterpret_cast<const unsigned long long*>(b.vo) + i + 1) -
                                      __ldg(reinterpret_cast<const unsigned long long*>(b.vo) + i);
                    else c_vb += b.vw;
                }
            }
        }
        for (int o = 16; o; o >>= 1) {
            c_rec += __shfl_xor_sync(FULLMASK, c_rec, o);
            c_kb += __shfl_xor_sync(FULLMASK, c_kb, o);
            c_vb += __shfl_xor_sync(FULLMASK, c_vb, o);
        }
        if (lane == 0) {
            atomicAdd(&s_cnt[0], c_rec);
            atomicAdd(&s_cnt[1], c_kb);
            atomicAdd(&s_cnt[2], c_vb);
        }
        __syncthreads();
        if (tid == 0) {
            tile_counts[3 * tile] = s_cnt[0];
            tile_counts[3 * tile + 1] = s_cnt[1];
            tile_counts[3 * tile + 2] = s_cnt[2];
            if (s_cnt[0]) atomicAdd(&d.ctrl->postponed, s_cnt[0]);
            if (s_cnt[1]) atomicAdd(&d.ctrl->kept_key_bytes, s_cnt[1]);
            if (s_cnt[2]) atomicAdd(&d.ctrl->kept_val_bytes, s_cnt[2]);
        }
        __syncthreads();
    }
    __syncthreads();
    if (PROBE && tid == 0) {
        d.cursors[2 * blockIdx.x] = s_cur[0];
        d.cursors[2 * blockIdx.x + 1] = s_cur[1];
    }
}

// ================================================================ compaction (a9)
// exclusive scan of the per-tile (records, key bytes, value bytes) triples, one CTA
__global__ void __launch_bounds__(1024) scan_tiles_kernel(unsigned long long* tc, uint64_t ntiles) {
    __shared__ unsigned long long s_w[32][3];
    __shared__ unsigned long long s_carry[3];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    if (tid < 3) s_carry[tid] = 0;
    __syncthreads();
    for (uint64_t base = 0; base < ntiles; base += 1024) {
        const uint64_t t = base + tid;
        unsigned long long v[3] = {0, 0, 0};
        if (t < ntiles) { v[0] = tc[3 * t]; v[1] = tc[3 * t + 1]; v[2] = tc[3 * t + 2]; }
        unsigned long long inc[3] = {v[0], v[1], v[2]};
        for (int o = 1; o < 32; o <<= 1)
            for (int c = 0; c < 3; ++c) {
                unsigned long long y = __shfl_up_sync(FULLMASK, inc[c], o);
                if (lane >= (uint32_t)o) inc[c] += y;
            }
        if (lane == 31) for (int c = 0; c < 3; ++c) s_w[warp][c] = inc[c];
        __syncthreads();
        if (warp == 0) {
            unsigned long long x[3];
            for (int c = 0; c < 3; ++c) x[c] = s_w[lane][c];
            for (int o = 1; o < 32; o <<= 1)
                for (int c = 0; c < 3; ++c) {
                    unsigned long long y = __shfl_up_sync(FULLMASK, x[c], o);
                    if (lane >= (uint32_t)o) x[c] += y;
                }
            for (int c = 0; c < 3; ++c) s_w[lane][c] = x[c];
        }
        __syncthreads();
        for (int c = 0; c < 3; ++c) {
            unsigned long long before = s_carry[c] + (warp ? s_w[warp - 1][c] : 0ull) + inc[c] - v[c];
            if (t < ntiles) tc[3 * t + c] = before;
        }
        __syncthreads();
        if (tid < 3) s_carry[tid] += s_w[31][tid];
        __syncthreads();
    }
}

// Key bytes [src, src + len) -> [dst, dst + len) at any alignment: byte stores up to dst's first 8-byte
// boundary, then aligned 8-byte stores each assembled from the two aligned source words that hold it
// (funnel shift), then the last bytes. A lane only writes bytes of its own record, so neighbouring
// records (adjacent within a part) never overlap a wide store. (URLs of ~74 bytes: ~17 stores instead
// of 74 byte stores.)
__device__ __forceinline__ void copy_key_bytes(uint8_t* dst, const uint8_t* src, uint32_t len) {
    uint32_t x = min(len, (uint32_t)((8u - (reinterpret_cast<uintptr_t>(dst) & 7u)) & 7u));
    for (uint32_t y = 0; y < x; ++y) dst[y] = (uint8_t)ld_in8(src + y);
    const uint32_t nfull = (len - x) / 8;  // whole 8-byte words of dst from dst + x (8-aligned)
    if (nfull) {
        const uintptr_t sa = reinterpret_cast<uintptr_t>(src + x);
        const uint32_t sh = (uint32_t)(sa & 7u) * 8u;
        const uint64_t* sw = reinterpret_cast<const uint64_t*>(sa & ~(uintptr_t)7);
        uint64_t* dw = reinterpret_cast<uint64_t*>(dst + x);
        if (sh == 0) {
            for (uint32_t k = 0; k < nfull; ++k) dw[k] = ld_in64(sw + k);
        } else {  // (every aligned source word read holds a key byte)
            uint64_t lo = ld_in64(sw);
            for (uint32_t k = 0; k < nfull; ++k) {
                const uint64_t hi = ld_in64(sw + k + 1);
                dw[k] = (lo >> sh) | (hi << (64u - sh));
                lo = hi;
            }
        }
        x += 8 * nfull;
    }
    for (; x < len; ++x) dst[x] = (uint8_t)ld_in8(src + x);
}

// gather: per tile, block scan of (kept, key bytes, value bytes) then copy
constexpr int CP_THREADS = 256;
__global__ void __launch_bounds__(CP_THREADS) compact_kernel(Batch b, const unsigned long long* tile_base, uint8_t* ok,
                                                             uint64_t* oko, uint8_t* ov, uint64_t* ovo) {
    __shared__ unsigned long long s_w[CP_THREADS / 32][3];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    constexpr int PER = RP_TILE / CP_THREADS;  // 8 consecutive records per thread
    const uint64_t ntiles = (b.n + RP_TILE - 1) / RP_TILE;
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const uint64_t i0 = tile * RP_TILE + (uint64_t)tid * PER;
        uint32_t keep = 0;
        unsigned long long kb = 0, vb = 0;
        for (int q = 0; q < PER; ++q) {
            const uint64_t i = i0 + q;
            if (i < b.n && ((b.bitmap[i >> 5] >> (i & 31)) & 1u)) {
                keep |= 1u << q;
                uint64_t s; uint32_t len;
                rec_key(b, i, s, len);
                kb += len;
                if (b.vals) {
                    if (b.vo) { uint64_t vs; uint32_t vl; rec_val_span(b, i, vs, vl); vb += vl; }
                    else vb += b.vw;
                }
            }
        }
        unsigned long long inc[3] = {(unsigned long long)__popc(keep), kb, vb};
        const unsigned long long own[3] = {inc[0], inc[1], inc[2]};
        for (int o = 1; o < 32; o <<= 1)
            for (int c = 0; c < 3; ++c) {
                unsigned long long y = __shfl_up_sync(FULLMASK, inc[c], o);
                if (lane >= (uint32_t)o) inc[c] += y;
            }
        if (lane == 31) for (int c = 0; c < 3; ++c) s_w[warp][c] = inc[c];
        __syncthreads();
        unsigned long long pos[3];
        for (int c = 0; c < 3; ++c) {
            unsigned long long wb = 0;
            for (uint32_t w2 = 0; w2 < warp; ++w2) wb += s_w[w2][c];
            pos[c] = tile_base[3 * tile + c] + wb + inc[c] - own[c];
        }
        __syncthreads();
        for (int q = 0; q < PER; ++q) {
            if (!((keep >> q) & 1u)) continue;
            const uint64_t i = i0 + q;
            uint64_t s; uint32_t len;
            rec_key(b, i, s, len);
            if (b.ko) oko[pos[0]] = pos[1];
            copy_key_bytes(ok + pos[1], b.keys + s, len);
            if (b.vals) {
                uint64_t vs; uint32_t vl;
                if (b.vo) { rec_val_span(b, i, vs, vl); ovo[pos[0]] = pos[2]; }
                else { vs = rec_index(b, i) * (uint64_t)b.vw; vl = b.vw; }
                for (uint32_t x = 0; x < vl; ++x) ov[pos[2] + x] = __ldg(b.vals + vs + x);
                pos[2] += vl;
            }
            pos[0] += 1;
            pos[1] += len;
        }
    }
}

__global__ void finish_offsets_kernel(uint64_t* oko, uint64_t m, uint64_t kb, uint64_t* ovo, uint64_t vb) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        if (oko) oko[m] = kb;
        if (ovo) ovo[m] = vb;
    }
}

// per-tile counts of set bits (COMBINE re-issue: the insert's count is exact, R15)
__global__ void __launch_bounds__(64) tile_popc_kernel(Batch b, unsigned long long* tile_counts) {
    const uint64_t ntiles = (b.n + RP_TILE - 1) / RP_TILE;
    const uint64_t nwords = (b.n + 31) / 32;
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const uint64_t w = tile * (RP_TILE / 32) + threadIdx.x;
        unsigned c = w < nwords ? __popc(b.bitmap[w]) : 0u;
        c = __reduce_add_sync(FULLMASK, c);
        __shared__ unsigned s2[2];
        if ((threadIdx.x & 31) == 0) s2[threadIdx.x >> 5] = c;
        __syncthreads();
        if (threadIdx.x == 0) {
            tile_counts[3 * tile] = s2[0] + s2[1];
            tile_counts[3 * tile + 1] = 0;
            tile_counts[3 * tile + 2] = 0;
        }
        __syncthreads();
    }
}

// index stream compaction (a9): positions of set bits, mapped through the batch's own index
// list, written in order: out[k] = rec_index(b, i) for the k-th postponed record i.
__global__ void __launch_bounds__(256) compact_index_kernel(Batch b, const unsigned long long* tile_base, uint64_t* out) {
    __shared__ unsigned int s_w[8];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    const uint64_t ntiles = (b.n + RP_TILE - 1) / RP_TILE;
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        // thread t owns bits [8t, 8t+8) of the tile = one byte of the tile's 64 bitmap words
        const uint64_t i0 = tile * RP_TILE + (uint64_t)tid * 8;
        uint32_t byte = 0;
        if (i0 < b.n) {
            byte = (b.bitmap[i0 >> 5] >> (i0 & 31)) & 0xffu;
            const uint64_t rem = b.n - i0;
            if (rem < 8) byte &= (1u << rem) - 1u;
        }
        const uint32_t c = __popc(byte);
        uint32_t inc = c;
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULLMASK, inc, o);
            if (lane >= (uint32_t)o) inc += y;
        }
        if (lane == 31) s_w[warp] = inc;
        __syncthreads();
        uint64_t pos = tile_base[3 * tile];
        for (uint32_t w2 = 0; w2 < warp; ++w2) pos += s_w[w2];
        pos += inc - c;
        while (byte) {
            const int q = __ffs(byte) - 1;
            byte &= byte - 1;
            out[pos++] = rec_index(b, i0 + q);
        }
        __syncthreads();
    }
}

// ================================================================ key-hash router (a12, multi-GPU)
// owner(k) = hi32(H(route_seed, k)) * P >> 32 — a hash independent of the table's bucket hash
// (different seed), so a rank's keys spread over all of its buckets. A stable partition of the
// batch by owner: per tile per part counts -> one exclusive scan in part-major order -> scatter,
// so part p's records are contiguous, in input order, with offsets rebased to the part.
constexpr int PT_THREADS = 1024, PT_TILE = 2048, PT_MAXP = 32;

__device__ __forceinline__ uint32_t route_owner(const Batch& b, uint64_t i, uint64_t seed, uint32_t P, uint64_t& s,
                                                uint32_t& len, uint64_t& w0, uint64_t& w1) {
    rec_key(b, i, s, len);
    load_key16(b.keys + s, len, w0, w1);
    const uint64_t h = hash_key16(len, seed, w0, w1, b.keys + s);
    return (uint32_t)(((h >> 32) * (uint64_t)P) >> 32);
}

// Per tile of PT_TILE records, the lanes of a warp with the same owner (one __match_any_sync) reserve
// their slots in their part with ONE shared-memory atomic on a packed per-part cursor {records << 32 |
// key bytes} issued by the group's first lane; a lane's rank is the popcount of the group below it and
// its byte offset the sum of the group's lengths below it, taken bit by bit (one ballot per bit of the
// warp's longest key). Rank and byte offset come from the same atomic, so key bytes and offsets stay a
// CSR. (The order of records within a part follows the atomics; the method is order independent.)
// Pass count: the tile's per-part totals; pass scatter: base of (part, tile) from the scan + the rank.
__device__ __forceinline__ void pt_reserve(unsigned long long* cur, bool valid, uint32_t p, uint32_t len, uint32_t& rank,
                                           uint32_t& boff, unsigned long long& slot) {
    const uint32_t lane = lane_id();
    const unsigned gm = __match_any_sync(FULLMASK, valid ? p : (0x100u | lane));
    const unsigned lt = lanemask_lt();
    const uint32_t nbits = 32u - __clz(__reduce_max_sync(FULLMASK, valid ? len : 0u));
    uint32_t pre = 0, tot = 0;
    for (uint32_t bit = 0; bit < nbits; ++bit) {
        const unsigned m = __ballot_sync(FULLMASK, valid && ((len >> bit) & 1u)) & gm;
        pre += (uint32_t)__popc(m & lt) << bit;
        tot += (uint32_t)__popc(m) << bit;
    }
    const uint32_t leader = (uint32_t)(__ffs(gm) - 1);
    unsigned long long r = 0;
    if (valid && lane == leader) r = atomicAdd(&cur[p], ((unsigned long long)__popc(gm) << 32) | (unsigned long long)tot);
    slot = __shfl_sync(FULLMASK, r, leader);
    rank = (uint32_t)__popc(gm & lt);
    boff = pre;
}
__global__ void __launch_bounds__(PT_THREADS) part_count_kernel(Batch b, uint32_t P, uint64_t seed,
                                                                unsigned long long* counts, uint64_t ntiles) {
    __shared__ unsigned long long cur[PT_MAXP];
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        if (threadIdx.x < PT_MAXP) cur[threadIdx.x] = 0ull;
        __syncthreads();
        for (int k = 0; k < PT_TILE / PT_THREADS; ++k) {
            const uint64_t i = tile * PT_TILE + k * PT_THREADS + threadIdx.x;
            const bool valid = i < b.n;
            uint64_t s = 0, w0, w1; uint32_t len = 0, o = 0;
            if (valid) o = route_owner(b, i, seed, P, s, len, w0, w1);
            uint32_t rank, boff;
            unsigned long long slot;
            pt_reserve(cur, valid, o, len, rank, boff, slot);
        }
        __syncthreads();
        if (threadIdx.x < P) {
            const unsigned long long c = cur[threadIdx.x];
            unsigned long long* dst = counts + ((uint64_t)threadIdx.x * ntiles + tile) * 3;
            dst[0] = c >> 32;
            dst[1] = c & 0xffffffffull;
            dst[2] = b.vals ? (c >> 32) * b.vw : 0ull;
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(PT_THREADS) part_scatter_kernel(Batch b, uint32_t P, uint64_t seed,
                                                                  const unsigned long long* base, uint64_t ntiles,
                                                                  uint8_t* ok, uint64_t* oko, uint8_t* ov) {
    __shared__ unsigned long long cur[PT_MAXP];
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        if (threadIdx.x < PT_MAXP) cur[threadIdx.x] = 0ull;
        __syncthreads();
        for (int k = 0; k < PT_TILE / PT_THREADS; ++k) {
            const uint64_t i = tile * PT_TILE + k * PT_THREADS + threadIdx.x;
            const bool valid = i < b.n;
            uint64_t src = 0, kw0 = 0, kw1 = 0; uint32_t len = 0, p = 0;
            if (valid) p = route_owner(b, i, seed, P, src, len, kw0, kw1);
            uint32_t rank, boff;
            unsigned long long r;
            pt_reserve(cur, valid, p, len, rank, boff, r);
            if (!valid) continue;
            const unsigned long long* bp = base + ((uint64_t)p * ntiles + tile) * 3;
            const unsigned long long* b0 = base + ((uint64_t)p * ntiles) * 3;  // start of part p
            const uint64_t orec = bp[0] + (r >> 32) + rank;
            const uint64_t obyte = bp[1] + (r & 0xffffffffull) + boff;
            if (oko) oko[orec] = obyte - b0[1];  // rebased to the part's segment
            copy_key_bytes(ok + obyte, b.keys + src, len);
            if (b.vals) {
                const uint64_t vs = rec_index(b, i) * (uint64_t)b.vw;
                uint8_t* vd = ov + orec * b.vw;
                if (b.vw == 8) *reinterpret_cast<unsigned long long*>(vd) = ld_in64(b.vals + vs);
                else for (uint32_t x = 0; x < b.vw; ++x) vd[x] = (uint8_t)ld_in8(b.vals + vs + x);
            }
        }
        __syncthreads();
    }
}

// received segments: offsets of segment s are relative to its own bytes; shift them by the bytes
// of the segments before it and close the CSR with the total
__global__ void shift_offsets_kernel(uint64_t* ko, uint64_t n, const uint64_t* seg_rec, const uint64_t* seg_base,
                                     uint32_t n_segs, uint64_t total) {
    for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < n; j += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t sgi = 0;
        while (sgi + 1 < n_segs && seg_rec[sgi + 1] <= j) ++sgi;
        ko[j] += seg_base[sgi];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) ko[n] = total;
}

// longest key of a CSR batch (the pipelined sharded job picks wire records when every rank's keys
// are at most 16 bytes): warp max, one atomicMax per warp
__global__ void __launch_bounds__(256) max_key_len_kernel(const uint64_t* ko, uint64_t n, unsigned long long* out) {
    unsigned long long m = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        m = max(m, (unsigned long long)(ld_in64(ko + i + 1) - ld_in64(ko + i)));
    m = __reduce_max_sync(FULLMASK, (unsigned)min(m, 0xffffffffull));
    if (lane_id() == 0 && m) atomicMax(out, m);
}

// ---- router with hot-key pre-combine (COMBINE mode, keys of at most 16 bytes)
// Records of one rank go to their owners as 32-byte WireRecs {key words, value, length}. The keys of
// the batch's sampled hot set (the same discovery as the insert kernels, on the route hash) never
// leave as records: every CTA folds their records into pending sums in shared memory (warp
// __match_any_sync fold + one shared atomic per distinct key), the CTAs' sums meet in a global array,
// and each hot key leaves the rank ONCE, as one wire record carrying its total (C5-Zipf's top key,
// 18 % of the records, would otherwise overload its owner and the links into it). Other records leave
// one wire record each (a tile of uniform keys holds almost no duplicates to combine).
// Two passes over the batch with the same static split of 32-record groups over the warps (the
// hot / not-hot decision reads a fixed hot set): pass 0 counts each CTA's non-hot records per part,
// the host scans them into per-(part, CTA) bases, pass 1 writes the records through per-CTA cursors
// and flushes the hot sums; rh_emit_hot then appends each part's hot keys after its other records.
// (The order of records within a part is immaterial: the method is order independent.)
namespace rh {
constexpr int THREADS = 1024, WARPS = THREADS / 32;
constexpr int DS = stream::DS, NK = hot::K;  // hot slots (2-choice, direct indexed) / hot keys at most
constexpr int IDXB = stream::IDXB;
struct Smem {
    uint32_t tags[DS];               // slot words: fingerprint | key index
    ulonglong2 kw[NK];               // hot keys' words (zero padded)
    unsigned long long sum[NK];      // the CTA's pending sums
    unsigned int cnt[PT_MAXP];       // pass 0: non-hot records per part; pass 1: cursors
    unsigned long long base[PT_MAXP];
    WireRec* dst[PT_MAXP];           // pass 1: where part p's records go
};
static_assert(sizeof(Smem) <= 232448, "route kernel shared memory > 227 KB");
}  // namespace rh

// out: part p's records at out[bases...] — or, with dstp (the fused route + exchange over peer memory,
// sepo_run_sharded), at dstp[p][bases...]: rank p's receive window, written through NVLink
template <int PASS, int IN>
__global__ void __launch_bounds__(rh::THREADS, 1) route_hot_kernel(Batch b, uint32_t P, uint64_t seed, const hot::Entry* hl,
                                                                  const unsigned int* n_hot, unsigned long long* counts,
                                                                  const unsigned long long* bases, unsigned long long* hot_sum,
                                                                  unsigned long long* long_keys, WireRec* out,
                                                                  WireRec* const* dstp) {
    using namespace rh;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    Smem& S = *reinterpret_cast<Smem*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id(), G = gridDim.x;
    constexpr uint32_t IM = (1u << IDXB) - 1u;
    for (uint32_t x = tid; x < (uint32_t)DS; x += THREADS) S.tags[x] = 0u;
    for (uint32_t x = tid; x < (uint32_t)NK; x += THREADS) S.sum[x] = 0ull;
    if (tid < PT_MAXP) {
        S.cnt[tid] = 0u;
        S.base[tid] = (PASS == 1 && tid < P) ? bases[(uint64_t)tid * G + blockIdx.x] : 0ull;
        S.dst[tid] = (PASS == 1 && tid < P) ? (dstp ? dstp[tid] : out) : nullptr;
    }
    __syncthreads();
    // Slot placement must be the same in both passes and every CTA (pass 0 counts what pass 1 writes),
    // so it is decided by priorities, not by the order of atomics: a key's priority is its sample-count
    // class, then its index in the (hash-sorted, rh_sort_hot) list; round 1 gives slot ds1 to its
    // highest-priority claimant, round 2 gives each slot still empty to the best key that lost round 1.
    const unsigned nh = hl ? min(*n_hot, (unsigned)NK) : 0u;
    if (nh) {
        constexpr uint32_t JB = 12;  // index bits of a priority (NK <= 4096)
        static_assert(NK <= (1 << JB), "hot keys");
        uint32_t prio[(NK + THREADS - 1) / THREADS], d1[(NK + THREADS - 1) / THREADS], d2[(NK + THREADS - 1) / THREADS];
        bool won[(NK + THREADS - 1) / THREADS], try2[(NK + THREADS - 1) / THREADS];
#pragma unroll
        for (int r = 0; r < (NK + THREADS - 1) / THREADS; ++r) {
            const unsigned j = tid + r * THREADS;
            prio[r] = 0; won[r] = false; try2[r] = false; d1[r] = 0; d2[r] = 0;
            if (j < nh) {
                const hot::Entry e = hl[j];
                if (e.len <= 16u) {
                    prio[r] = ((uint32_t)(hot::count_class(e.count) + 1) << JB) | ((1u << JB) - 1u - j);
                    d1[r] = stream::ds1(e.h); d2[r] = stream::ds2(e.h);
                    atomicMax(&S.tags[d1[r]], prio[r]);
                }
            }
        }
        __syncthreads();
#pragma unroll
        for (int r = 0; r < (NK + THREADS - 1) / THREADS; ++r) {
            won[r] = prio[r] && S.tags[d1[r]] == prio[r];
            try2[r] = prio[r] && !won[r] && S.tags[d2[r]] == 0u;  // (read before any round-2 write)
        }
        __syncthreads();
#pragma unroll
        for (int r = 0; r < (NK + THREADS - 1) / THREADS; ++r)
            if (try2[r]) atomicMax(&S.tags[d2[r]], prio[r]);
        __syncthreads();
        uint32_t slot[(NK + THREADS - 1) / THREADS];
#pragma unroll
        for (int r = 0; r < (NK + THREADS - 1) / THREADS; ++r) {
            slot[r] = won[r] ? d1[r] : ((try2[r] && S.tags[d2[r]] == prio[r]) ? d2[r] : ~0u);
        }
        __syncthreads();
        for (uint32_t x = tid; x < (uint32_t)DS; x += THREADS) S.tags[x] = 0u;  // (slots nobody won stay empty)
        __syncthreads();
#pragma unroll
        for (int r = 0; r < (NK + THREADS - 1) / THREADS; ++r) {
            const unsigned j = tid + r * THREADS;
            if (slot[r] != ~0u) {
                const hot::Entry e = hl[j];
                S.tags[slot[r]] = stream::dfp(e.h, e.len) | j;
                S.kw[j] = make_ulonglong2(e.w0, e.w1);
            }
        }
        __syncthreads();
    }
    const uint64_t ngroups = (b.n + 31) / 32, nw = (uint64_t)G * WARPS, gw = (uint64_t)blockIdx.x * WARPS + (tid >> 5);
    unsigned long long nlong = 0;
    for (uint64_t g = ngroups * gw / nw, gend = ngroups * (gw + 1) / nw; g < gend; ++g) {
        const uint64_t i = g * 32 + lane;
        const bool valid = i < b.n;
        uint64_t s = 0, e = 0, w0 = 0, w1 = 0;
        lean::offsets<IN>(b, i, valid, s, e);
        const uint32_t len = (uint32_t)(e - s);
        const bool ok = valid && len <= 16u;
        if (valid && !ok) ++nlong;
        if (ok) {
            uint64_t x0, x1, x2;
            lean::key_words(b.keys, s, len, x0, x1, x2);
            lean::assemble16(x0, x1, x2, (uint32_t)(reinterpret_cast<uintptr_t>(b.keys + s) & 7u), len, w0, w1);
        }
        const uint64_t h = hash_key16(ok ? len : 0u, seed, w0, w1, nullptr);
        int pos = -1;
        if (nh) {
            const uint32_t f = stream::dfp(h, len);
            const uint32_t t1 = S.tags[stream::ds1(h)], t2 = S.tags[stream::ds2(h)];
            const bool m1 = (t1 & ~IM) == f, m2 = (t2 & ~IM) == f;
            const uint32_t p = (m1 ? t1 : t2) & IM;
            if (ok && (m1 || m2)) {
                const ulonglong2 kk = S.kw[p];
                if (kk.x == w0 && kk.y == w1) pos = (int)p;
            }
        }
        if (PASS == 1) {  // hot records: one shared atomic per distinct key of the warp
            const uint64_t v = ok ? rec_value(b, i) : 0ull;
            const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
            if (hm) {
                const unsigned grp = __match_any_sync(FULLMASK, pos >= 0 ? (unsigned)pos : (0x10000u | lane)) & hm;
                uint64_t acc = v;
                if (__any_sync(FULLMASK, __popc(grp) > 1)) {
                    acc = 0;
                    for (int xl = 0; xl < 32; ++xl) {
                        const uint64_t vx = __shfl_sync(FULLMASK, v, xl);
                        if ((grp >> xl) & 1u) acc += vx;
                    }
                }
                if (pos >= 0 && lane == (uint32_t)(__ffs(grp) - 1)) atomicAdd(&S.sum[pos], (unsigned long long)acc);
            }
            // other records: one wire record each, slots reserved per owner group of the warp
            const bool cold = ok && pos < 0;
            const uint32_t owner = (uint32_t)(((h >> 32) * (uint64_t)P) >> 32);
            const unsigned cm = __ballot_sync(FULLMASK, cold);
            if (cm) {
                const unsigned gm = __match_any_sync(FULLMASK, cold ? owner : (0x100u | lane)) & cm;
                const uint32_t leader = (uint32_t)(__ffs(gm | (1u << lane)) - 1);
                unsigned r = 0;
                if (cold && lane == leader) r = atomicAdd(&S.cnt[owner], (unsigned)__popc(gm));
                r = __shfl_sync(FULLMASK, r, leader);
                if (cold) {
                    const uint64_t at = S.base[owner] + r + __popc(gm & lanemask_lt());
                    ulonglong2* o = reinterpret_cast<ulonglong2*>(S.dst[owner] + at);
                    __stcs(o, make_ulonglong2(w0, w1));
                    __stcs(o + 1, make_ulonglong2(v, (unsigned long long)len));
                }
            }
        } else {
            const bool cold = ok && pos < 0;
            const uint32_t owner = (uint32_t)(((h >> 32) * (uint64_t)P) >> 32);
            const unsigned cm = __ballot_sync(FULLMASK, cold);
            if (cm) {
                const unsigned gm = __match_any_sync(FULLMASK, cold ? owner : (0x100u | lane)) & cm;
                if (cold && lane == (uint32_t)(__ffs(gm) - 1)) atomicAdd(&S.cnt[owner], (unsigned)__popc(gm));
            }
        }
    }
    if (nlong && long_keys) atomicAdd(long_keys, nlong);
    __syncthreads();
    if (PASS == 0) {
        if (tid < P) counts[(uint64_t)tid * G + blockIdx.x] = S.cnt[tid];
    } else {
        for (uint32_t j = tid; j < nh; j += THREADS)
            if (S.sum[j]) red_add_u64(&hot_sum[j], S.sum[j]);
        if (dstp) __threadfence_system();  // (peer stores performed before the exchange's barrier)
    }
}
// the emitted hot list in hash order (the emit kernel's order follows its atomics): one CTA, bitonic
// sort of (hash, index) in shared memory, then the entries permuted into `out`
__global__ void __launch_bounds__(1024) rh_sort_hot(const hot::Entry* in, const unsigned int* n_hot, hot::Entry* out) {
    __shared__ unsigned long long kh[hot::K];
    __shared__ uint32_t ki[hot::K];
    const unsigned nh = min(*n_hot, (unsigned)hot::K);
    for (unsigned j = threadIdx.x; j < (unsigned)hot::K; j += blockDim.x) {
        kh[j] = j < nh ? in[j].h : ~0ull;
        ki[j] = j;
    }
    __syncthreads();
    for (unsigned k = 2; k <= (unsigned)hot::K; k <<= 1) {
        for (unsigned jj = k >> 1; jj > 0; jj >>= 1) {
            for (unsigned i = threadIdx.x; i < (unsigned)hot::K; i += blockDim.x) {
                const unsigned l = i ^ jj;
                if (l > i) {
                    const bool up = (i & k) == 0;
                    const bool gt = kh[i] > kh[l] || (kh[i] == kh[l] && ki[i] > ki[l]);
                    if (gt == up) {
                        const unsigned long long th = kh[i]; kh[i] = kh[l]; kh[l] = th;
                        const uint32_t ti = ki[i]; ki[i] = ki[l]; ki[l] = ti;
                    }
                }
            }
            __syncthreads();
        }
    }
    for (unsigned j = threadIdx.x; j < nh; j += blockDim.x) out[j] = in[ki[j]];
}

// per part: hot keys owned (pass 0), then each hot key's wire record after the part's other records
__global__ void rh_count_hot(const hot::Entry* hl, const unsigned int* n_hot, uint32_t P, unsigned long long* hot_pp) {
    const unsigned nh = hl ? min(*n_hot, (unsigned)rh::NK) : 0u;
    for (unsigned j = blockIdx.x * blockDim.x + threadIdx.x; j < nh; j += gridDim.x * blockDim.x)
        if (hl[j].len <= 16u) atomicAdd(&hot_pp[(uint32_t)(((hl[j].h >> 32) * (uint64_t)P) >> 32)], 1ull);
}
__global__ void rh_emit_hot(const hot::Entry* hl, const unsigned int* n_hot, uint32_t P, const unsigned long long* hot_sum,
                            const unsigned long long* hot_base, unsigned long long* hot_cur, WireRec* out,
                            WireRec* const* dstp) {
    const unsigned nh = hl ? min(*n_hot, (unsigned)rh::NK) : 0u;
    for (unsigned j = blockIdx.x * blockDim.x + threadIdx.x; j < nh; j += gridDim.x * blockDim.x) {
        const hot::Entry e = hl[j];
        if (e.len > 16u) continue;
        const uint32_t p = (uint32_t)(((e.h >> 32) * (uint64_t)P) >> 32);
        const unsigned long long at = hot_base[p] + atomicAdd(&hot_cur[p], 1ull);
        WireRec r;
        r.w0 = e.w0; r.w1 = e.w1; r.v = hot_sum[j]; r.len = e.len;
        (dstp ? dstp[p] : out)[at] = r;
    }
    if (dstp) __threadfence_system();
}


// ================================================================ pass boundary (a10)
// Seal every open page (filler over its unused tail) and reset the CTA cursors.
__global__ void seal_kernel(Dev d, uint32_t n_slots) {
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= 2 * n_slots) return;
    const unsigned long long cur = d.cursors[c];
    const uint32_t page = (uint32_t)(cur >> 32), off = (uint32_t)cur;
    if (page < d.n_pages && off < d.page_bytes)
        *reinterpret_cast<uint32_t*>(d.pool + ((uint64_t)page << d.page_shift) + off) = (d.page_bytes - off) | K_FILL;
    d.cursors[c] = ((unsigned long long)NOPAGE << 32) | d.page_bytes;
}

// Choose cold pages: every resident page that is not retained (COMBINE: all of them, P:L171;
// GROUP: value pages + key pages without pending keys). Builds the sorted evict list and
// the new free stack (retained pages excluded). keep_all_retained = 0 forces a full eviction.
__global__ void __launch_bounds__(1024) classify_kernel(Dev d, int honor_retain) {
    __shared__ uint32_t s_w[32][2];
    __shared__ uint32_t s_base[2];
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    if (tid == 0) { s_base[0] = 0; s_base[1] = 0; }
    __syncthreads();
    uint32_t n_res = 0;
    for (uint32_t p0 = 0; p0 < d.n_pages; p0 += 1024) {
        const uint32_t p = p0 + tid;
        uint32_t ev = 0, fr = 0;
        if (p < d.n_pages) {
            const uint8_t st = d.page_state[p];
            const bool keep = honor_retain && st == PAGE_ENTRY && d.retain[p];
            if (st != 0 && !keep) ev = 1;
            if (!keep) fr = 1;
            if (keep) ++n_res;
            if (!keep) d.page_state[p] = 0;
            d.retain[p] = 0;
        }
        // free pages that need no copy first (stack order), the evicted ones follow in copy order
        fr = fr && !ev;
        uint32_t ie = ev, ifr = fr;
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y0 = __shfl_up_sync(FULLMASK, ie, o), y1 = __shfl_up_sync(FULLMASK, ifr, o);
            if (lane >= (uint32_t)o) { ie += y0; ifr += y1; }
        }
        if (lane == 31) { s_w[warp][0] = ie; s_w[warp][1] = ifr; }
        __syncthreads();
        uint32_t be = s_base[0], bf = s_base[1];
        for (uint32_t w2 = 0; w2 < warp; ++w2) { be += s_w[w2][0]; bf += s_w[w2][1]; }
        if (ev) d.evict_list[be + ie - 1] = p;
        if (fr) d.stack[bf + ifr - 1] = p;
        __syncthreads();
        if (tid == 0) {
            for (int w2 = 0; w2 < 32; ++w2) { s_base[0] += s_w[w2][0]; s_base[1] += s_w[w2][1]; }
        }
        __syncthreads();
    }
    for (int o = 16; o; o >>= 1) n_res += __shfl_xor_sync(FULLMASK, n_res, o);
    __shared__ uint32_t s_res;
    if (tid == 0) s_res = 0;
    __syncthreads();
    if (lane == 0) atomicAdd(&s_res, n_res);
    __syncthreads();
    // evicted pages go back to the stack behind the safe ones, in evict-list (= copy) order
    const uint32_t n_ev = s_base[0], n_sf = s_base[1];
    for (uint32_t j = tid; j < n_ev; j += blockDim.x) d.stack[n_sf + j] = d.evict_list[j];
    if (tid == 0) {
        d.ctrl->n_evict = n_ev;
        d.ctrl->n_free = n_sf + n_ev;
        d.ctrl->n_safe = n_sf;
        d.ctrl->n_resident = s_res;
        d.ctrl->pool_taken = 0;
    }
}

// GROUP: re-link the live key entries of retained key pages into the fresh directory, so the
// keys with pending values are found in the next pass. One thread per page.
__global__ void relink_kernel(Dev d) {
    for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < d.n_pages; p += gridDim.x * blockDim.x) {
        if (d.page_state[p] != PAGE_ENTRY) continue;
        uint8_t* base = d.pool + ((uint64_t)p << d.page_shift);
        uint32_t off = 0;
        while (off < d.page_bytes) {
            const uint32_t hdr = *reinterpret_cast<uint32_t*>(base + off);
            const uint32_t size = hdr & ~KIND_MASK;
            if (size == 0) break;
            if ((hdr & KIND_MASK) == K_GKEY) {
                uint8_t* e = base + off;
                const uint32_t tag = *reinterpret_cast<uint32_t*>(e + 8);
                const uint32_t len = *reinterpret_cast<uint32_t*>(e + 12);
                (void)len;
                // recompute the bucket from the stored key
                const uint64_t h = hash_key(e + KEY_OFF, len, d.seed);
                (void)tag;
                const uint32_t bkt = bucket_of(h, d.n_buckets);
                const uint32_t me = off_ref((uint64_t)(e - d.pool));
                uint32_t head = ld_dir(d.dir + bkt);
                while (true) {
                    *reinterpret_cast<uint32_t*>(e + 4) = head;
                    const uint32_t old = cas_release(d.dir + bkt, head, me);
                    if (old == head) break;
                    head = old;
                }
            }
            off += size;
        }
    }
}

__global__ void init_state_kernel(Dev d, uint32_t n_slots) {
    const uint64_t gt = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t gs = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t p = gt; p < d.n_pages; p += gs) {
        d.stack[p] = (uint32_t)p;
        d.page_state[p] = 0;
        d.retain[p] = 0;
    }
    for (uint64_t c = gt; c < 2ull * n_slots; c += gs) d.cursors[c] = ((unsigned long long)NOPAGE << 32) | d.page_bytes;
    if (gt == 0) {
        Ctrl z = {};
        *d.ctrl = z;
    }
}

// ================================================================ fused tokenizer + COMBINE insert (NEXT-2)
// Word count on raw text (reading R20): the text is read once, in 512-byte
// windows (a 16-byte chunk per lane), instead of text -> CSR -> insert. Per window a warp computes the
// separator bits of its bytes, the word starts (a non-separator byte after a separator), their
// warp-wide prefix count and a list of start offsets in shared memory; then it takes the window's
// words 32 at a time, one per lane: the end is the first separator bit at or after the start in
// the [window | next window] bitmap, the first 16 key bytes come from the two-window text ring in
// shared memory, and from there on the word is a record of the COMBINE stream kernel (hash, hot
// set, warp fold, miss queue, resolve_core with value 1). A word belongs to the window it starts
// in; one that runs past the next window (> 512 B) is measured in global memory. Declined words
// go to the prepared re-issue list (key offset = the word's text offset), or — if the list is
// full — set their start bit in b.tbm for the host to convert into prepared records.
namespace textk {
constexpr int THREADS = 1024, WARPS = THREADS / 32;
constexpr int WB = 512;    // window bytes: 32 lanes x 16 B
constexpr int CHW = 64;    // consecutive windows a warp streams before it strides
constexpr int DSZ = 8192;  // hot slots (the text ring takes the room of half the CSR kernel's slots)
constexpr int TK = 2048;   // hot keys at most
__device__ __forceinline__ uint32_t ds1(uint64_t h) { return (uint32_t)(h >> 3) & (DSZ - 1); }
__device__ __forceinline__ uint32_t ds2(uint64_t h) { return (uint32_t)(h >> 17) & (DSZ - 1); }
struct WarpText {
    uint4 t[2][32];         // text ring: two consecutive windows
    uint32_t sep[2][16];    // separator bits, bit j of word k = byte 32k + j of the window
    uint16_t wp[WB / 2];    // word start offsets of the current window
};
struct Smem {
    uint32_t tags[DSZ];
    ulonglong2 kw[TK];
    uint32_t ref[TK];
    unsigned int sum[TK];
    stream::Smem<false, WARPS>::Queue q[WARPS];
    WarpText w[WARPS];
    stream::CtaState cs;
};
// 16 separator bits of a 16-byte chunk (bytes past `valid` count as separators)
__device__ __forceinline__ uint32_t sep16(uint4 c, uint32_t valid) {
    const uint32_t wv[4] = {c.x, c.y, c.z, c.w};
    uint32_t out = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint32_t w = wv[k];
        uint32_t m = __vcmpeq4(w, 0x20202020u) | __vcmpeq4(w, 0x0a0a0a0au) | __vcmpeq4(w, 0x09090909u) |
                     __vcmpeq4(w, 0x0d0d0d0du);
        m &= 0x01010101u;
        out |= ((m * 0x10204080u) >> 28) << (4 * k);  // byte k -> bit k (distinct partial products)
    }
    if (valid < 16) out |= (0xffffu << valid) & 0xffffu;
    return out;
}
// the lane's 16-byte chunk of window `win` (zeros past the end of the text)
__device__ __forceinline__ uint4 load_chunk(const uint8_t* T, uint64_t n, uint64_t win, uint32_t lane, uint32_t& valid) {
    const uint64_t a = win * WB + 16ull * lane;
    if (a + 16 <= n) { valid = 16; return ld_in128(T + a); }
    valid = a < n ? (uint32_t)(n - a) : 0u;
    uint32_t by[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) by[j] = (uint32_t)j < valid ? ld_in8(T + a + j) : 0u;
    return make_uint4(by[0] | by[1] << 8 | by[2] << 16 | by[3] << 24, by[4] | by[5] << 8 | by[6] << 16 | by[7] << 24,
                      by[8] | by[9] << 8 | by[10] << 16 | by[11] << 24, by[12] | by[13] << 8 | by[14] << 16 | by[15] << 24);
}
// stage a chunk into ring slot `slot`: text bytes + the window's separator bits
__device__ __forceinline__ void stage(WarpText& W, uint32_t slot, uint32_t lane, uint4 ch, uint32_t valid) {
    W.t[slot][lane] = ch;
    const uint32_t sp = sep16(ch, valid);
    const uint32_t other = __shfl_down_sync(FULLMASK, sp, 1);
    if (!(lane & 1)) W.sep[slot][lane >> 1] = sp | (other << 16);
}
}  // namespace textk

__global__ void __launch_bounds__(textk::THREADS, 1) insert_text_kernel(Dev d, Batch b, const hot::Entry* hl,
                                                                         const unsigned int* n_hot) {
    using namespace textk;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    textk::Smem& S = *reinterpret_cast<textk::Smem*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id(), wid = tid >> 5;
    for (int p = tid; p < TK; p += THREADS) { S.ref[p] = 0; S.sum[p] = 0; }
    for (int p = tid; p < DSZ; p += THREADS) S.tags[p] = 0u;
    if (tid == 0) {
        S.cs.cur[0] = d.cursors[2 * blockIdx.x];
        S.cs.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.cs.post = 0; S.cs.toolarge = 0; S.cs.dead = 0; S.cs.pkb = 0;
    }
    if (tid < 32) { S.cs.wpost[tid] = 0; S.cs.wpkb[tid] = 0; }
    __syncthreads();
    const unsigned nh = hl ? *n_hot : 0u;
    for (int cls = 31; cls >= 0 && nh; --cls) {  // hot set, most frequent keys first (as the CSR kernel)
        for (unsigned j = tid; j < nh && j < (unsigned)TK; j += THREADS) {
            const hot::Entry e = hl[j];
            if (e.ref == 0 || hot::count_class(e.count) != cls) continue;
            const uint32_t f = stream::dfp_b<11>(e.h, e.len) | j;
            if (atomicCAS(&S.tags[ds1(e.h)], 0u, f) == 0u || atomicCAS(&S.tags[ds2(e.h)], 0u, f) == 0u) {
                S.kw[j] = make_ulonglong2(e.w0, e.w1);
                S.ref[j] = e.ref;
            }
        }
        __syncthreads();
    }
    __syncthreads();
    const bool have_hot = nh > 0;
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    const uint8_t* T = b.keys;
    const uint64_t n = b.n;
    const uint64_t nwin_all = (n + WB - 1) / WB;
    const uint64_t wbeg = b.w_begin, nwin = b.w_end < nwin_all ? b.w_end : nwin_all;  // this launch's windows
    const bool big = n / 2 >= (1ull << 32);  // words < 2^32: a CTA-local count cannot wrap
    WarpText& W = S.w[wid];
    auto& Q = S.q[wid];
    uint32_t qhead = 0, qtail = 0;
    PrepCursor pc;
    bool w_full = false, w_quiet = false;
    unsigned long long words = 0;  // lane 0
    const uint8_t* ring = reinterpret_cast<const uint8_t*>(&W.t[0][0]);
    const uint64_t nwarps = (uint64_t)gridDim.x * WARPS;
    for (uint64_t c0 = wbeg + ((uint64_t)blockIdx.x * WARPS + wid) * CHW; c0 < nwin; c0 += nwarps * CHW) {
        const uint64_t c1 = (c0 + CHW < nwin) ? c0 + CHW : nwin;
        uint32_t prev = 1u;  // is the byte before the window a separator (text start: yes)
        if (c0 > 0) prev = is_sep(ld_in8(T + c0 * WB - 1)) ? 1u : 0u;
        uint32_t vl;
        uint4 ch = load_chunk(T, n, c0, lane, vl);
        stage(W, 0, lane, ch, vl);
        uint32_t vl_n;
        uint4 ch_n = load_chunk(T, n, c0 + 1, lane, vl_n);
        uint32_t slot = 0;
        for (uint64_t w = c0; w < c1; ++w) {
            // window w+1 into the other slot (the words of w may run into it); load w+2 if ours
            stage(W, slot ^ 1u, lane, ch_n, vl_n);
            if (w + 2 < c1 + 1) ch_n = load_chunk(T, n, w + 2, lane, vl_n);
            __syncwarp();
            // ---- word starts of window w (a1): separator bits -> starts -> offsets in smem
            const uint32_t sw = W.sep[slot][lane >> 1];
            const uint32_t sp = (lane & 1) ? (sw >> 16) : (sw & 0xffffu);
            const uint32_t up = __shfl_up_sync(FULLMASK, sp, 1);
            const uint32_t pbit = lane == 0 ? prev : ((up >> 15) & 1u);
            const uint32_t st = ~sp & ((sp << 1) | pbit) & 0xffffu;
            prev = (__shfl_sync(FULLMASK, sp, 31) >> 15) & 1u;
            const uint32_t cnt = __popc(st);
            uint32_t incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(FULLMASK, incl, o);
                if (lane >= (uint32_t)o) incl += y;
            }
            const uint32_t total = __shfl_sync(FULLMASK, incl, 31);
            for (uint32_t m = st, k = incl - cnt; m; m &= m - 1) W.wp[k++] = (uint16_t)(lane * 16 + __ffs(m) - 1);
            words += total;
            __syncwarp();
            for (uint32_t r = 0; r < total; r += 32) {
                const uint32_t k = r + lane;
                const bool valid = k < total;
                const uint32_t p = valid ? W.wp[k] : 0u;
                const uint64_t s = w * WB + p;
                uint32_t len = 0;
                uint64_t w0 = 0, w1 = 0;
                if (valid) {
                    // end: the first separator at or after p in [window w | window w+1]
                    uint32_t wi = p >> 5;
                    uint32_t m2 = W.sep[slot][wi] & (~0u << (p & 31));
                    while (m2 == 0 && wi < 31) {
                        ++wi;
                        m2 = wi < 16 ? W.sep[slot][wi] : W.sep[slot ^ 1u][wi - 16];
                    }
                    len = m2 ? wi * 32 + __ffs(m2) - 1 - p : text_word_len(T, n, s);
                    // first 16 key bytes from the ring (aligned 8-byte words, wrapping at 1 KB)
                    const uint32_t base = slot * WB + p;
                    const uint32_t a0 = (base & ~7u) & 1023u;
                    const uint64_t x0 = *reinterpret_cast<const uint64_t*>(ring + a0);
                    const uint64_t x1 = *reinterpret_cast<const uint64_t*>(ring + ((a0 + 8) & 1023u));
                    const uint64_t x2 = *reinterpret_cast<const uint64_t*>(ring + ((a0 + 16) & 1023u));
                    const uint32_t sh = 8u * (base & 7u);
                    const uint64_t lo = sh ? (x0 >> sh) | (x1 << (64 - sh)) : x0;
                    const uint64_t hi = sh ? (x1 >> sh) | (x2 << (64 - sh)) : x1;
                    const uint32_t nb8 = 8u * min(len, 16u);
                    w0 = lo & ~shl64_clamp(~0ull, nb8);
                    w1 = hi & ~shl64_clamp(~0ull, nb8 > 64u ? nb8 - 64u : 0u);
                }
                const uint64_t h = hash_key16(len, d.seed, w0, w1, T + s);
                // ---- hot set (a2)
                int pos = -1;
                if (have_hot) {
                    const uint32_t f = stream::dfp_b<11>(h, len);
                    const uint32_t t1 = S.tags[ds1(h)], t2 = S.tags[ds2(h)];
                    const bool m1 = (t1 & 0xfffff800u) == f, m2 = (t2 & 0xfffff800u) == f;
                    const uint32_t q = (m1 ? t1 : t2) & 0x7ffu;
                    if (valid && (m1 || m2)) {
                        const ulonglong2 kk = S.kw[q];
                        bool eq = kk.x == w0 && kk.y == w1;
                        if (len > 16) {
                            const uint8_t* e = ref_ptr(d, S.ref[q]);
                            eq = eq && ldcg32(e + 12) == len && entry_key_eq(e + KEY_OFF + 16, T + s + 16, len - 16);
                        }
                        if (eq) pos = (int)q;
                    }
                }
                const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
                if (hm) {
                    const unsigned grp = __match_any_sync(FULLMASK, pos >= 0 ? (unsigned)pos : (0x10000u | lane)) & hm;
                    if (pos >= 0 && lane == (uint32_t)(__ffs(grp) - 1)) {
                        const unsigned add = (unsigned)__popc(grp);
                        const unsigned old = atomicAdd(&S.sum[pos], add);
                        if (big && old + add < old)
                            red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(ref_ptr(d, S.ref[pos]), len)), 1ull << 32);
                    }
                }
                // ---- misses: the warp's queue, resolved 32 at a time (a3..a7)
                const bool miss = valid && pos < 0;
                const unsigned mm = __ballot_sync(FULLMASK, miss);
                if (miss) {
                    if (b.dirpf)  // (tables larger than L2: see the CSR kernel)
                        asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(d.dir + bucket_of(h, d.n_buckets)));
                    const uint32_t kq = (qtail + __popc(mm & lanemask_lt())) & (stream::QCAP - 1);
                    Q.w0[kq] = w0; Q.w1[kq] = w1; Q.h[kq] = h; Q.s[kq] = s;
                    Q.g[kq] = 0;
                    Q.ll[kq] = (min(len, 1u << 26) << 5) | lane;
                }
                qtail += __popc(mm);
                __syncwarp();
                if (qtail - qhead >= 32) {
                    const uint32_t kq = (qhead + lane) & (stream::QCAP - 1);
                    const uint32_t ll = Q.ll[kq];
                    resolve_core<32>(d, b, S.cs, true, Q.w0[kq], Q.w1[kq], Q.h[kq], Q.s[kq], 1ull, ll >> 5, 0u, ll & 31u,
                                     inj, w_full, w_quiet, pc);
                    qhead += 32;
                    __syncwarp();
                }
            }
            slot ^= 1u;
        }
    }
    if (qtail != qhead) {
        const bool act = lane < qtail - qhead;
        const uint32_t kq = (qhead + lane) & (stream::QCAP - 1);
        const uint32_t ll = act ? Q.ll[kq] : 0u;
        resolve_core<32>(d, b, S.cs, act, act ? Q.w0[kq] : 0ull, act ? Q.w1[kq] : 0ull, act ? Q.h[kq] : 0ull,
                         act ? Q.s[kq] : 0ull, 1ull, ll >> 5, 0u, ll & 31u, inj, w_full, w_quiet, pc);
    }
    if (b.out && pc.used < PREP_CHUNK) prep_close(b, pc);
    if (lane == 0 && words) atomicAdd(&d.ctrl->text_words, words);
    __syncthreads();
    for (int p = tid; p < TK; p += THREADS) {
        if (S.ref[p] == 0 || S.sum[p] == 0) continue;
        uint8_t* e = ref_ptr(d, S.ref[p]);
        red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(e, ldcg32(e + 12))), (unsigned long long)S.sum[p]);
    }
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cs.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cs.cur[1];
        for (uint32_t w = 0; w < (uint32_t)WARPS; ++w) { S.cs.post += S.cs.wpost[w]; S.cs.pkb += S.cs.wpkb[w]; }
        if (S.cs.post) atomicAdd(&d.ctrl->postponed, S.cs.post);
        if (S.cs.toolarge) atomicAdd(&d.ctrl->toolarge, S.cs.toolarge);
        if (S.cs.dead) atomicAdd(&d.ctrl->dead_bytes, S.cs.dead);
        if (S.cs.pkb) atomicAdd(&d.ctrl->kept_key_bytes, S.cs.pkb);
    }
}

// ---- fused tokenizer, version 2: full 32-word rounds, three-window ring, cheaper separators
// Same method as insert_text_kernel (a word is a record with value 1; its identity is its text
// offset), restructured so that almost every round hands one word to each of the 32 lanes:
//   * a warp streams ONE contiguous range of 512-byte windows; the ring holds three consecutive
//     windows (text bytes + separator bits), so words of a window that do not fill a round are
//     carried into the next window's first round (their bytes are still in the ring);
//   * separator bits: per 32-bit word, one masked add per separator byte value and one combined
//     test (a byte b is a separator iff b is one of ' ', '\n', '\t', '\r', reading R20);
//   * a word's end: the first separator bit at or after its start in a 64-bit window of the ring's
//     separator bits (words longer than 32 bytes continue the scan, longer than the ring: global);
//   * queue slots as the lean CSR kernel (32 bytes: first 16 key bytes, hash, offset | length).
namespace text2 {
#ifndef SEPO_TEXT_THREADS
#define SEPO_TEXT_THREADS 768  // 24 warps, 80 registers: C2 text 4x pass 1 26.1 -> 25.3 ms, in budget 45.0 -> 28.9 ms
#endif                         // (896: 26.7 / 45.1, 640: 28.9 / 33.2, 512: 34.7 / 39.8; profiles/r02)
constexpr int THREADS = SEPO_TEXT_THREADS, WARPS = THREADS / 32;
constexpr int WB = 512, NSLOT = 3, RINGB = NSLOT * WB, SEPW = RINGB / 32;
#ifndef SEPO_TEXT_DS
#define SEPO_TEXT_DS 8192
#endif
constexpr int DSZ = SEPO_TEXT_DS, TK = 2048;
constexpr int WLCAP = 288;  // carried words (< 32) + one window's word starts (<= 256)
constexpr int QCAP = 64;
struct WarpText {
    // text ring: three consecutive windows, then a ghost copy of the first 32 bytes of slot 0 (so
    // reads of up to 24 bytes past a position never wrap)
    uint4 t[NSLOT * 32 + 2];
    uint32_t sep[SEPW + 2];  // separator bits: bit j of word k = ring byte 32k + j (+ ghost of words 0, 1)
    uint16_t wl[WLCAP];      // ring positions of the word starts waiting for a round
};
struct Smem {
    uint32_t tags[DSZ];
    ulonglong2 kw[TK];
    uint32_t ref[TK];
    unsigned int sum[TK];
    struct Queue {
        ulonglong2 k[QCAP];   // first 16 key bytes
        ulonglong2 hs[QCAP];  // hash, text offset | length << 40 | lane << 59
    } q[WARPS];
    WarpText w[WARPS];
    stream::CtaState cs;
};
static_assert(sizeof(Smem) <= 232448, "text2 kernel shared memory > 227 KB");
// 4 separator bits of the 4 bytes of w (bit k = byte k). Exact per-byte equality with c: for
// x = (w & 0x7f7f7f7f) ^ c7, bit 7 of x + 0x7f7f7f7f is 0 iff the low 7 bits of the byte equal c's;
// bit 7 of the byte itself must be 0 too (every separator is < 0x80).
__device__ __forceinline__ uint32_t sep4(uint32_t w) {
    const uint32_t w7 = w & 0x7f7f7f7fu;
    const uint32_t t1 = (w7 ^ 0x20202020u) + 0x7f7f7f7fu, t2 = (w7 ^ 0x0a0a0a0au) + 0x7f7f7f7fu;
    const uint32_t t3 = (w7 ^ 0x09090909u) + 0x7f7f7f7fu, t4 = (w7 ^ 0x0d0d0d0du) + 0x7f7f7f7fu;
    const uint32_t m = ~((t1 & t2 & t3 & t4) | w) & 0x80808080u;  // 0x80 in every separator byte
    return ((m >> 7) * 0x10204080u) >> 28;                          // byte k -> bit k
}
__device__ __forceinline__ uint32_t sep16(uint4 c, uint32_t valid) {
    uint32_t out = sep4(c.x) | (sep4(c.y) << 4) | (sep4(c.z) << 8) | (sep4(c.w) << 12);
    if (valid < 16) out |= (0xffffu << valid) & 0xffffu;  // bytes past the text end separate
    return out;
}
// stage window chunk `ch` (lane's 16 bytes) into ring slot `slot`: bytes + separator bits
__device__ __forceinline__ void stage(WarpText& W, uint32_t slot, uint32_t lane, uint4 ch, uint32_t valid) {
    W.t[slot * 32 + lane] = ch;
    const uint32_t sp = sep16(ch, valid);
    const uint32_t other = __shfl_down_sync(FULLMASK, sp, 1);
    if (!(lane & 1)) W.sep[slot * 16 + (lane >> 1)] = sp | (other << 16);
    if (slot == 0 && lane < 4) {  // the ghost after slot 2: its first 32 bytes and 2 separator words
        if (lane < 2) W.t[NSLOT * 32 + lane] = ch;
        if (!(lane & 1)) W.sep[SEPW + (lane >> 1)] = sp | (other << 16);
    }
}
}  // namespace text2

__global__ void __launch_bounds__(text2::THREADS, 1) insert_text2_kernel(Dev d, Batch b, const hot::Entry* hl,
                                                                           const unsigned int* n_hot) {
    using namespace text2;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    text2::Smem& S = *reinterpret_cast<text2::Smem*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id(), wid = tid >> 5;
    if (tid == 0) {
        S.cs.cur[0] = d.cursors[2 * blockIdx.x];
        S.cs.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.cs.post = 0; S.cs.toolarge = 0; S.cs.dead = 0; S.cs.pkb = 0;
    }
    if (tid < 32) { S.cs.wpost[tid] = 0; S.cs.wpkb[tid] = 0; }
    load_hot_direct<DSZ, TK>(S.tags, S.kw, S.ref, S.sum, hl, n_hot);
    __syncthreads();
    const bool have_hot = hl != nullptr && *n_hot > 0;
    const bool inj = d.fail_ppm != 0 && d.gen < d.fail_until;
    const uint8_t* T = b.keys;
    const uint64_t n = b.n;
    const uint64_t nwin_all = (n + WB - 1) / WB;
    const uint64_t lw0 = b.w_begin, lw1 = b.w_end < nwin_all ? b.w_end : nwin_all;  // this launch's windows
    const bool big = n / 2 >= (1ull << 32);  // words < 2^32: a CTA-local count cannot wrap
    WarpText& W = S.w[wid];
    auto& Q = S.q[wid];
    const uint64_t* R = reinterpret_cast<const uint64_t*>(&W.t[0]);  // the ring as 192 words (+ ghost)
    uint32_t qhead = 0, qtail = 0;
    PrepCursor pc;
    bool w_full = false, w_quiet = false;
    unsigned long long words = 0;  // lane 0
    // this warp's windows [wa, wz): an equal share of the launch's windows
    const uint64_t nlw = lw1 > lw0 ? lw1 - lw0 : 0;
    const uint64_t gw = (uint64_t)blockIdx.x * WARPS + wid, nwp = (uint64_t)gridDim.x * WARPS;
    const uint64_t wa = lw0 + nlw * gw / nwp, wz = lw0 + nlw * (gw + 1) / nwp;

    if (wa < wz) {
        uint32_t prev = 1u;  // is the byte before window wa a separator (text start: yes)
        if (wa > 0) prev = is_sep(ld_in8(T + wa * WB - 1)) ? 1u : 0u;
        uint32_t vl;
        uint4 ch = textk::load_chunk(T, n, wa, lane, vl);
        stage(W, 0, lane, ch, vl);
        ch = textk::load_chunk(T, n, wa + 1, lane, vl);  // (zeros past the text end)
        stage(W, 1, lane, ch, vl);
        uint32_t vl_n;
        uint4 ch_n = textk::load_chunk(T, n, wa + 2, lane, vl_n);
        uint32_t cslot = 0, nl = 0;  // ring slot of window w; words waiting in the list
        for (uint64_t w = wa; w < wz; ++w) {
            __syncwarp();
            // ---- word starts of window w (a1): a non-separator byte after a separator
            const uint32_t sw = W.sep[cslot * 16 + (lane >> 1)];
            const uint32_t sp = (lane & 1) ? (sw >> 16) : (sw & 0xffffu);
            const uint32_t up = __shfl_up_sync(FULLMASK, sp, 1);
            const uint32_t pbit = lane == 0 ? prev : ((up >> 15) & 1u);
            const uint32_t st = ~sp & ((sp << 1) | pbit) & 0xffffu;
            prev = (__shfl_sync(FULLMASK, sp, 31) >> 15) & 1u;
            const uint32_t cnt = __popc(st);
            uint32_t incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(FULLMASK, incl, o);
                if (lane >= (uint32_t)o) incl += y;
            }
            const uint32_t total = __shfl_sync(FULLMASK, incl, 31);
            const uint32_t rbase = cslot * WB + lane * 16;
            for (uint32_t m = st, k = nl + incl - cnt; m; m &= m - 1) W.wl[k++] = (uint16_t)(rbase + __ffs(m) - 1);
            nl += total;
            words += total;
            __syncwarp();
            // ---- rounds of 32 words (one per lane); a partial round only for carried words of the
            // window before (its ring slot is restaged next) and at the end of the warp's range
            uint32_t h = 0;
            while (true) {
                bool go = nl >= 32;
                if (!go && nl > 0) go = (w + 1 == wz) || ((W.wl[h] >> 9) != cslot);
                if (!go) break;
                const uint32_t nr = min(nl, 32u);
                const bool valid = lane < nr;
                const uint32_t p = valid ? W.wl[h + lane] : 0u;  // ring byte of the word start
                h += nr;
                nl -= nr;
                const uint32_t slot = p >> 9;
                // the word's window: the current one, or (a carried word) the one before it
                const uint64_t s = ((w - (slot != cslot ? 1u : 0u)) << 9) | (p & (WB - 1));
                uint32_t len = 0;
                uint64_t w0 = 0, w1 = 0;
                if (valid) {
                    // end: the first separator bit in the 32 bits from p on (funnel of two map words)
                    uint32_t wi = p >> 5;
                    const uint32_t m32 = __funnelshift_r(W.sep[wi], W.sep[wi + 1], p & 31u);
                    if (m32) {
                        len = (uint32_t)__ffs(m32) - 1;
                    } else {  // 32 bytes or longer: scan on through its window and the next, then global memory
                        const uint32_t wend = ((slot + 2) % NSLOT) * 16;
                        uint32_t m2 = 0;
                        wi = (wi + 1) % SEPW;
                        while (wi != wend && (m2 = W.sep[wi]) == 0) wi = (wi + 1) % SEPW;
                        len = (wi != wend && m2) ? (uint32_t)((wi * 32 + RINGB - p) % RINGB) + __ffs(m2) - 1
                                                 : text_word_len(T, n, s);
                    }
                    // first 16 key bytes from the ring (aligned 8-byte words; the ghost covers the wrap)
                    const uint32_t a = p >> 3;
                    lean::assemble16(R[a], R[a + 1], R[a + 2], p & 7u, len, w0, w1);
                }
                const uint64_t hh = hash_key16(len, d.seed, w0, w1, T + s);
                // ---- hot set (a2)
                int pos = -1;
                if (have_hot) {
                    const uint32_t f = stream::dfp_b<11>(hh, len);
                    const uint32_t t1 = S.tags[(uint32_t)(hh >> 3) & (DSZ - 1)], t2 = S.tags[(uint32_t)(hh >> 17) & (DSZ - 1)];
                    const bool m1 = (t1 & 0xfffff800u) == f, m2 = (t2 & 0xfffff800u) == f;
                    const uint32_t q = (m1 ? t1 : t2) & 0x7ffu;
                    if (valid && (m1 || m2)) {
                        const ulonglong2 kk = S.kw[q];
                        bool eq = kk.x == w0 && kk.y == w1;
                        if (len > 16) {
                            const uint8_t* e = ref_ptr(d, S.ref[q]);
                            eq = eq && ldcg32(e + 12) == len && entry_key_eq(e + KEY_OFF + 16, T + s + 16, len - 16);
                        }
                        if (eq) pos = (int)q;
                    }
                }
                const unsigned hm = __ballot_sync(FULLMASK, pos >= 0);
                if (hm) {
                    const unsigned grp = __match_any_sync(FULLMASK, pos >= 0 ? (unsigned)pos : (0x10000u | lane)) & hm;
                    if (pos >= 0 && lane == (uint32_t)(__ffs(grp) - 1)) {
                        const unsigned add = (unsigned)__popc(grp);
                        const unsigned old = atomicAdd(&S.sum[pos], add);
                        if (big && old + add < old)
                            red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(ref_ptr(d, S.ref[pos]), len)), 1ull << 32);
                    }
                }
                // ---- misses: the warp's queue, resolved 32 at a time (a3..a7)
                const bool miss = valid && pos < 0;
                const unsigned mm = __ballot_sync(FULLMASK, miss);
                if (miss) {
                    if (b.dirpf) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(d.dir + bucket_of(hh, d.n_buckets)));
                    const uint32_t kq = (qtail + __popc(mm & lanemask_lt())) & (QCAP - 1);
                    Q.k[kq] = make_ulonglong2(w0, w1);
                    Q.hs[kq] = make_ulonglong2(hh, s | ((uint64_t)min(len, lean::LEN_MAX) << 40) | ((uint64_t)lane << 59));
                }
                qtail += __popc(mm);
                __syncwarp();
                if (qtail - qhead >= 32) {
                    const uint32_t kq = (qhead + lane) & (QCAP - 1);
                    const ulonglong2 kk = Q.k[kq], hs = Q.hs[kq];
                    resolve_core<32>(d, b, S.cs, true, kk.x, kk.y, hs.x, hs.y & lean::S_MASK, 1ull,
                                     (uint32_t)(hs.y >> 40) & lean::LEN_MAX, 0u, (uint32_t)(hs.y >> 59), inj, w_full, w_quiet,
                                     pc);
                    qhead += 32;
                    __syncwarp();
                }
            }
            // the (< 32) carried words to the front of the list
            if (h && nl) {
                const uint16_t x = lane < nl ? W.wl[h + lane] : (uint16_t)0;
                __syncwarp();
                if (lane < nl) W.wl[lane] = x;
            }
            __syncwarp();
            // ---- window w + 2 into the slot of w - 1 (no carried word is from w - 1 now), load w + 3
            stage(W, (cslot + 2) % NSLOT, lane, ch_n, vl_n);
            if (w + 3 < wz + 2) ch_n = textk::load_chunk(T, n, w + 3, lane, vl_n);
            cslot = (cslot + 1) % NSLOT;
        }
    }
    if (qtail != qhead) {
        const bool act = lane < qtail - qhead;
        const uint32_t kq = (qhead + lane) & (QCAP - 1);
        ulonglong2 kk = make_ulonglong2(0, 0), hs = make_ulonglong2(0, 0);
        if (act) { kk = Q.k[kq]; hs = Q.hs[kq]; }
        resolve_core<32>(d, b, S.cs, act, kk.x, kk.y, hs.x, hs.y & lean::S_MASK, 1ull, (uint32_t)(hs.y >> 40) & lean::LEN_MAX,
                         0u, (uint32_t)(hs.y >> 59), inj, w_full, w_quiet, pc);
    }
    if (b.out && pc.used < PREP_CHUNK) prep_close(b, pc);
    if (lane == 0 && words) atomicAdd(&d.ctrl->text_words, words);
    __syncthreads();
    for (int p = tid; p < TK; p += THREADS) {
        if (S.ref[p] == 0 || S.sum[p] == 0) continue;
        uint8_t* e = ref_ptr(d, S.ref[p]);
        red_add_u64(reinterpret_cast<unsigned long long*>(entry_val(e, ldcg32(e + 12))), (unsigned long long)S.sum[p]);
    }
    if (tid == 0) {
        d.cursors[2 * blockIdx.x] = S.cs.cur[0];
        d.cursors[2 * blockIdx.x + 1] = S.cs.cur[1];
        for (uint32_t w = 0; w < (uint32_t)WARPS; ++w) { S.cs.post += S.cs.wpost[w]; S.cs.pkb += S.cs.wpkb[w]; }
        if (S.cs.post) atomicAdd(&d.ctrl->postponed, S.cs.post);
        if (S.cs.toolarge) atomicAdd(&d.ctrl->toolarge, S.cs.toolarge);
        if (S.cs.dead) atomicAdd(&d.ctrl->dead_bytes, S.cs.dead);
        if (S.cs.pkb) atomicAdd(&d.ctrl->kept_key_bytes, S.cs.pkb);
    }
}

// Words whose start bit is set in b.tbm (declined when the prepared list was full) -> 32-byte
// prepared records appended at out[*counter++]; the bits are cleared for the next use.
__global__ void __launch_bounds__(256) text_bits_kernel(Dev d, Batch b, unsigned long long* counter) {
    const uint64_t nw = (b.n + 31) / 32;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t bits = b.tbm[i];
        if (!bits) continue;
        b.tbm[i] = 0u;
        for (; bits; bits &= bits - 1) {
            const uint64_t s = i * 32 + __ffs(bits) - 1;
            const uint32_t len = text_word_len(b.keys, b.n, s);
            uint64_t w0, w1;
            load_key16(b.keys + s, len, w0, w1);
            const uint64_t h = hash_key16(len, d.seed, w0, w1, b.keys + s);
            const unsigned long long k = atomicAdd(counter, 1ull);
            ulonglong2* o = reinterpret_cast<ulonglong2*>(reinterpret_cast<uint8_t*>(b.out) + k * 32);
            o[0] = make_ulonglong2(w0, w1);
            o[1] = make_ulonglong2(h, s | ((unsigned long long)min(len, 0xfffeu) << 48));
        }
    }
}

// ================================================================ map runtime (NEXT-4): built-in mappers
// The paper's MapReduce library runs map tasks that emit key/value pairs straight into
// the table (MAP_REDUCE -> combining organization, MAP_GROUP -> multi-valued). Map callbacks cannot
// cross a C ABI as device code, so the runtime ships the mappers of the paper's applications as
// kernels: every record of a text chunk becomes a (key, value) pair in a compacted CSR batch that
// the SEPO job then consumes.
//   MAP_LINES     : key = a line (maximal run of bytes other than '\n'), value 1 (Page View Count)
//   MAP_WORD_DOCS : key = a word (reading R20), value = u32 id of the document holding it (Inverted
//                   Index; documents given as byte offsets)
// (MAP_WORDS, Word Count, is the fused tokenizer: sepo_run_text.) Two passes over chunks of MC bytes:
// count the records starting in each chunk and their key bytes, scan, write.
constexpr uint32_t MC = 256;
__device__ __forceinline__ bool map_sep(uint32_t c, int lines) { return lines ? c == 0x0au : is_sep(c); }
// records starting in chunk ch: a non-separator byte at the chunk start preceded by a separator (or
// the text start), or after a separator inside the chunk
__global__ void __launch_bounds__(256) map_count_kernel(const uint8_t* T, uint64_t n, int lines, unsigned long long* tc) {
    const uint64_t nch = (n + MC - 1) / MC;
    for (uint64_t ch = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; ch < nch; ch += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t a = ch * MC, z = min(a + MC, n);
        unsigned long long cnt = 0, bytes = 0;
        bool prev_sep = a == 0 || map_sep(T[a - 1], lines);
        uint64_t i = a;
        while (i < z) {
            const bool sp = map_sep(T[i], lines);
            if (!sp && prev_sep) {  // a record starts at i: measure it (it may run past the chunk)
                uint64_t e = i;
                while (e < n && !map_sep(T[e], lines)) ++e;
                ++cnt;
                bytes += e - i;
                i = e;
                prev_sep = false;
                continue;
            }
            prev_sep = sp;
            ++i;
        }
        tc[3 * ch] = cnt;
        tc[3 * ch + 1] = bytes;
        tc[3 * ch + 2] = 0;
    }
}
__global__ void __launch_bounds__(256) map_write_kernel(const uint8_t* T, uint64_t n, int lines, const unsigned long long* tc,
                                                        const uint64_t* doc_offsets, uint64_t n_docs, uint8_t* okeys,
                                                        uint64_t* oko, uint32_t* odoc) {
    const uint64_t nch = (n + MC - 1) / MC;
    for (uint64_t ch = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; ch < nch; ch += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t a = ch * MC, z = min(a + MC, n);
        uint64_t r = tc[3 * ch], kb = tc[3 * ch + 1];
        bool prev_sep = a == 0 || map_sep(T[a - 1], lines);
        uint64_t i = a;
        while (i < z) {
            const bool sp = map_sep(T[i], lines);
            if (!sp && prev_sep) {
                uint64_t e = i;
                while (e < n && !map_sep(T[e], lines)) { okeys[kb + (e - i)] = T[e]; ++e; }
                oko[r] = kb;
                if (odoc) {  // the document holding byte i: the last d with doc_offsets[d] <= i
                    uint64_t lo = 0, hi = n_docs - 1;
                    while (lo < hi) {
                        const uint64_t mid = lo + ((hi - lo + 1) >> 1);
                        if (doc_offsets[mid] <= i) lo = mid; else hi = mid - 1;
                    }
                    odoc[r] = (uint32_t)lo;
                }
                ++r;
                kb += e - i;
                i = e;
                prev_sep = false;
                continue;
            }
            prev_sep = sp;
            ++i;
        }
    }
}

// ================================================================ SEPO lookups (NEXT-4)
// Lookups on the larger-than-memory table ("The SEPO model can also be used for lookup
// operations on larger-than-memory hash tables"): the host streams the evicted generations back
// through the device pool one at a time (each page to the slot it was evicted from, so refs stay
// valid); the directory is rebuilt from the restored pages and every still-unresolved query is
// probed; queries whose key is not in this generation are POSTPONED to the next one.
__global__ void lookup_link_kernel(Dev d, const uint32_t* pages, uint32_t np) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < np; i += gridDim.x * blockDim.x) {
        uint8_t* base = d.pool + ((uint64_t)pages[i] << d.page_shift);
        for (uint32_t off = 0; off < d.page_bytes;) {
            const uint32_t hdr = *reinterpret_cast<uint32_t*>(base + off);
            const uint32_t size = hdr & ~KIND_MASK;
            if (size == 0) break;
            if ((hdr & KIND_MASK) == K_COMBINE) {
                uint8_t* e = base + off;
                const uint32_t len = *reinterpret_cast<uint32_t*>(e + 12);
                const uint32_t bkt = bucket_of(hash_key(e + KEY_OFF, len, d.seed), d.n_buckets);
                const uint32_t me = off_ref((uint64_t)(e - d.pool));
                uint32_t head = ld_dir(d.dir + bkt);
                while (true) {
                    *reinterpret_cast<uint32_t*>(e + 4) = head;
                    const uint32_t old = cas_release(d.dir + bkt, head, me);
                    if (old == head) break;
                    head = old;
                }
            }
            off += size;
        }
    }
}
// a warp per 32 consecutive queries: the group's found word decides which lanes still probe; keys
// are read with the warp-cooperative 16-byte loads of the insert path; the found word is rewritten
// once per group (this warp owns it)
__global__ void __launch_bounds__(256) lookup_kernel(Dev d, Batch b, unsigned long long* vals_out, uint32_t* found) {
    const uint32_t lane = lane_id();
    const uint64_t ngroups = (b.n + 31) / 32;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    unsigned long long hits = 0;
    for (uint64_t g = (uint64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); g < ngroups; g += nw) {
        const uint32_t fw = found[g];
        const uint64_t i = g * 32 + lane;
        const bool valid = i < b.n;
        const bool todo = valid && !((fw >> lane) & 1u);
        if (!__any_sync(FULLMASK, todo)) continue;
        uint64_t s, w0, w1;
        uint32_t len;
        warp_load_group(b, g, lane, valid, s, len, w0, w1);
        const uint64_t h = hash_key16(len, d.seed, w0, w1, b.keys + s);
        const uint8_t* e = nullptr;
        if (todo)
            e = chain_find_w(d, ld_dir(d.dir + bucket_of(h, d.n_buckets)), 0, tag_of(h), len, w0, w1, b.keys + s + 16);
        if (e) vals_out[i] = ldcg64(entry_val(const_cast<uint8_t*>(e), len));
        const unsigned hm = __ballot_sync(FULLMASK, e != nullptr);
        if (lane == 0 && hm) {
            found[g] = fw | hm;
            hits += __popc(hm);
        }
    }
    if (lane == 0 && hits) atomicAdd(&d.ctrl->postponed, hits);
}

// Eviction gather copy (a10): evicted pages -> one contiguous pinned host region, page k of the
// evict list at dst + k * page_bytes. The host arena is page-locked and mapped (UVA), so SM stores
// cross the host link directly: one launch per eviction however fragmented the evict list is (a
// cudaMemcpyAsync per run of consecutive pages costs microseconds per run: GROUP generations with
// retained key pages evict 10^5 short runs). A warp copies a page with 16-byte loads/stores.
__global__ void __launch_bounds__(512) evict_copy_kernel(const uint8_t* __restrict__ pool, const uint32_t* __restrict__ list,
                                                      uint32_t n, uint8_t* __restrict__ dst, uint32_t page_shift) {
    const uint32_t lane = lane_id();
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
    const uint32_t per_page = (1u << page_shift) / 16;  // 16-byte units
    for (uint64_t k = (uint64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); k < n; k += nw) {
        const uint4* src = reinterpret_cast<const uint4*>(pool + ((uint64_t)list[k] << page_shift));
        uint4* out = reinterpret_cast<uint4*>(dst + (k << page_shift));
        uint32_t u = lane;
        for (; u + 96 < per_page; u += 128) {
            const uint4 a = __ldcg(src + u), b = __ldcg(src + u + 32), c = __ldcg(src + u + 64), e = __ldcg(src + u + 96);
            __stcs(out + u, a); __stcs(out + u + 32, b); __stcs(out + u + 64, c); __stcs(out + u + 96, e);
        }
        for (; u < per_page; u += 32) __stcs(out + u, __ldcg(src + u));
    }
}

// The same gather, overlapped with the next pass (GROUP): warp w copies positions w, w + W, ... in
// order and after each page publishes its count in eprog[w] (release, after __syncwarp: every lane's
// loads of the page are done), so the allocator can reuse a page as soon as its own warp copied it.
__global__ void __launch_bounds__(512) evict_copy_prog_kernel(const uint8_t* __restrict__ pool, const uint32_t* __restrict__ list,
                                                           uint32_t n, uint8_t* __restrict__ dst, uint32_t page_shift,
                                                           unsigned int* eprog) {
    const uint32_t lane = lane_id();
    const uint32_t W = gridDim.x * (blockDim.x / 32), w = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
    const uint32_t per_page = (1u << page_shift) / 16;
    unsigned int done = 0;
    for (uint64_t k = w; k < n; k += W) {
        const uint4* src = reinterpret_cast<const uint4*>(pool + ((uint64_t)list[k] << page_shift));
        uint4* out = reinterpret_cast<uint4*>(dst + (k << page_shift));
        uint32_t u = lane;
        for (; u + 96 < per_page; u += 128) {
            const uint4 a = __ldcg(src + u), b = __ldcg(src + u + 32), c = __ldcg(src + u + 64), e = __ldcg(src + u + 96);
            __stcs(out + u, a); __stcs(out + u + 32, b); __stcs(out + u + 64, c); __stcs(out + u + 96, e);
        }
        for (; u < per_page; u += 32) __stcs(out + u, __ldcg(src + u));
        __syncwarp();
        ++done;
        if (lane == 0) asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(eprog + w), "r"(done) : "memory");
    }
}

}  // namespace sepo

// ================================================================ launchers
using namespace sepo;

// Smallest batch (records; text: bytes) that gets a sampled hot set. Tests move the threshold:
// SEPO_NO_HOT=1 switches the hot set off, SEPO_HOT_MIN=<n> sets the threshold (re-read per launch).
static uint64_t hot_min_records(uint64_t dflt) {
    const char* off = getenv("SEPO_NO_HOT");
    if (off && off[0] == '1') return ~0ull;
    const char* m = getenv("SEPO_HOT_MIN");
    return m ? strtoull(m, nullptr, 10) : dflt;
}

int sepo_launch_insert_text(const Dev& d, const Batch& b0, int grid, cudaStream_t s, void* hot_scratch,
                            uint64_t sample_bytes, bool* hot_built) {
    const hot::Entry* hl = nullptr;
    const unsigned int* nh = nullptr;
    const uint64_t n_sample = 1ull << 18;
    const Batch& b = b0;
    Batch bs = b0;  // bs.n: the prefix the sample positions come from (its words are read whole:
    bs.n = sample_bytes < b0.n ? sample_bytes : b0.n;  // the caller has copied past the prefix)
    const bool reuse = sample_bytes == 0 && *hot_built;
    if (sample_bytes) *hot_built = false;
    if (hot_scratch && reuse) {  // reuse the hot set an earlier launch of this job built
        uint8_t* p = reinterpret_cast<uint8_t*>(hot_scratch);
        hot::Entry* list = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS);
        hl = list;
        nh = reinterpret_cast<unsigned int*>(list + hot::K);
    } else if (hot_scratch && sample_bytes && bs.n >= hot_min_records(64 * n_sample)) {  // discovery on sampled words
        uint8_t* p = reinterpret_cast<uint8_t*>(hot_scratch);
        hot::SampleSlot* tab = reinterpret_cast<hot::SampleSlot*>(p);
        hot::Entry* list = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS);
        unsigned int* n_out = reinterpret_cast<unsigned int*>(list + hot::K);
        unsigned int* hist = n_out + 1;
        cudaMemsetAsync(tab, 0, sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS, s);
        cudaMemsetAsync(n_out, 0, (HOT_HIST + 2) * sizeof(unsigned int), s);
        hot_sample_kernel<<<4 * 148, 256, 0, s>>>(d, b, std::max<uint64_t>(1, bs.n / n_sample), std::min(n_sample, bs.n), tab);  // positions in the prefix
        hot_hist_kernel<<<2 * 148, 256, 0, s>>>(tab, hist, 4u);
        hot_threshold_kernel<<<1, 1024, 0, s>>>(hist, 4u, (uint32_t)textk::TK);
        hot_emit_kernel<<<2 * 148, 256, 0, s>>>(d, b, tab, hist, list, n_out, (uint32_t)textk::TK);
        hot_clamp_kernel<<<1, 32, 0, s>>>(n_out, (uint32_t)textk::TK);
        hot_resolve_kernel<<<1, 1024, 0, s>>>(d, b, list, n_out);
        hl = list;
        nh = n_out;
        *hot_built = true;
    }
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(insert_text_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(textk::Smem));
        cudaFuncSetAttribute(insert_text2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(text2::Smem));
        attr = true;
    }
    const char* v = getenv("SEPO_TEXT2");  // 0: the first fused tokenizer (insert_text_kernel)
    if (v && v[0] == '0') insert_text_kernel<<<grid, textk::THREADS, sizeof(textk::Smem), s>>>(d, b, hl, nh);
    else insert_text2_kernel<<<grid, text2::THREADS, sizeof(text2::Smem), s>>>(d, b, hl, nh);
    return cudaGetLastError();
}
int sepo_launch_lookup_gen(const Dev& d, const Batch& b, const uint32_t* pages, uint32_t np, unsigned long long* vals,
                           uint32_t* found, cudaStream_t s) {
    if (np) lookup_link_kernel<<<(np + 127) / 128, 128, 0, s>>>(d, pages, np);
    if (b.n) lookup_kernel<<<8 * 148, 256, 0, s>>>(d, b, vals, found);
    return cudaGetLastError();
}
int sepo_launch_text_bits(const Dev& d, const Batch& b, unsigned long long* counter, cudaStream_t s) {
    text_bits_kernel<<<4 * 148, 256, 0, s>>>(d, b, counter);
    return cudaGetLastError();
}

int sepo_launch_evict_copy_prog(const Dev& d, uint32_t n, uint8_t* dst, int grid, unsigned int* eprog,
                                const uint32_t* list, cudaStream_t s) {
    if (n) evict_copy_prog_kernel<<<grid, 512, 0, s>>>(d.pool, list, n, dst, d.page_shift, eprog);
    return cudaGetLastError();
}
int sepo_launch_evict_copy(const Dev& d, uint32_t n, uint8_t* dst, int grid, cudaStream_t s) {
    if (n) evict_copy_kernel<<<grid, 512, 0, s>>>(d.pool, d.evict_list, n, dst, d.page_shift);
    return cudaGetLastError();
}

int sepo_launch_insert(const Dev& d, const Batch& b, int mode, int grid, cudaStream_t s, void* hot_scratch,
                       uint32_t halt_slots, uint64_t key_end, bool dir_prefetch, bool* hot_built, bool lean_in,
                       bool long_keys) {
    if (hot_built) *hot_built = false;
    if (mode == 2) {
        insert_basic_kernel<<<grid, 1024, 0, s>>>(d, b, halt_slots);
        return cudaGetLastError();
    }
    if (mode == 0) {
        // hot-set discovery on a strided sample (skipped for small batches)
        const hot::Entry* hl = nullptr;
        const unsigned int* nh = nullptr;
        const uint64_t n_sample = 1ull << 18;
        if (hot_scratch && b.n >= hot_min_records(8 * n_sample)) {
            uint8_t* p = reinterpret_cast<uint8_t*>(hot_scratch);
            hot::SampleSlot* tab = reinterpret_cast<hot::SampleSlot*>(p);
            hot::Entry* list = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS);
            unsigned int* n_out = reinterpret_cast<unsigned int*>(list + hot::K);
            cudaMemsetAsync(tab, 0, sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS, s);
            hot_sample_kernel<<<4 * 148, 256, 0, s>>>(d, b, std::max<uint64_t>(1, b.n / n_sample), std::min(n_sample, b.n), tab);
            unsigned int* hist = n_out + 1;
            cudaMemsetAsync(n_out, 0, (HOT_HIST + 2) * sizeof(unsigned int), s);
            hot_hist_kernel<<<2 * 148, 256, 0, s>>>(tab, hist, 4u);
            const uint32_t kmax = (uint32_t)hot::K;
            hot_threshold_kernel<<<1, 1024, 0, s>>>(hist, 4u, kmax);
            hot_emit_kernel<<<2 * 148, 256, 0, s>>>(d, b, tab, hist, list, n_out, kmax);
            hot_clamp_kernel<<<1, 32, 0, s>>>(n_out, kmax);
            hot_resolve_kernel<<<1, 1024, 0, s>>>(d, b, list, n_out);
            hl = list;
            nh = n_out;
            if (hot_built) *hot_built = true;
        }
        constexpr int T = stream::THREADS;
        const size_t sm = b.vals ? sizeof(stream::Smem<true, T / 32>) : sizeof(stream::Smem<false, T / 32>);
        static bool attr = false;
        if (!attr) {
            const int s0 = (int)sizeof(stream::Smem<false, T / 32>), s1 = (int)sizeof(stream::Smem<true, T / 32>);
            cudaFuncSetAttribute(insert_stream_kernel<false, T, IN_CSR>, cudaFuncAttributeMaxDynamicSharedMemorySize, s0);
            cudaFuncSetAttribute(insert_stream_kernel<false, T, IN_FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, s0);
            cudaFuncSetAttribute(insert_stream_kernel<false, T, IN_IDX>, cudaFuncAttributeMaxDynamicSharedMemorySize, s0);
            cudaFuncSetAttribute(insert_stream_kernel<true, T, IN_CSR>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
            cudaFuncSetAttribute(insert_stream_kernel<true, T, IN_FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
            cudaFuncSetAttribute(insert_stream_kernel<true, T, IN_IDX>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
            attr = true;
        }
        const int in = b.wire ? IN_WIRE : (b.idx ? IN_IDX : (b.ko ? IN_CSR : IN_FIXED));
        InCtx c;
        c.ngroups = (uint32_t)((b.n + 31) / 32);
        c.tail = (uint32_t)(b.n - (uint64_t)(c.ngroups ? c.ngroups - 1 : 0) * 32);
        c.nw = (uint32_t)grid * (T / 32);
        c.kend = in == IN_IDX ? 0ull : (in == IN_CSR ? key_end : b.n * (uint64_t)b.kw);
        c.kal = !(reinterpret_cast<uintptr_t>(b.keys) & 15);
        c.dirpf = dir_prefetch;
        if ((lean_in && in != IN_IDX) || in == IN_WIRE) {  // contiguous batch of mostly short keys: the lean input path
            static bool attr_l = false;
            if (!attr_l) {
                const int s0 = (int)sizeof(lean::Smem<false>), s1 = (int)sizeof(lean::Smem<true>);
                cudaFuncSetAttribute(insert_lean_kernel<false, IN_CSR, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, s0);
                cudaFuncSetAttribute(insert_lean_kernel<false, IN_FIXED, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, s0);
                cudaFuncSetAttribute(insert_lean_kernel<true, IN_CSR, 33>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
                cudaFuncSetAttribute(insert_lean_kernel<true, IN_FIXED, 33>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
                cudaFuncSetAttribute(insert_lean_kernel<true, IN_CSR, 48>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
                cudaFuncSetAttribute(insert_lean_kernel<true, IN_FIXED, 48>, cudaFuncAttributeMaxDynamicSharedMemorySize, s1);
                attr_l = true;
            }
            c.nw = (uint32_t)grid * lean::WARPS;
            const size_t sml = b.vals ? sizeof(lean::Smem<true>) : sizeof(lean::Smem<false>);
            const dim3 G(grid), B(lean::THREADS);
            if (b.wire) {
                static bool attr_w = false;
                if (!attr_w) {
                    cudaFuncSetAttribute(insert_lean_kernel<true, IN_WIRE, 48>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(lean::Smem<true>));
                    cudaFuncSetAttribute(insert_lean_kernel<true, IN_WIRE, 33>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(lean::Smem<true>));
                    attr_w = true;
                }
                // (33: every key of the batch is at most 8 bytes — routed fixed-width keys — so a
                // declined record fits a 32-byte prepared record {key, value, hash, length})
                if (b.prep_fmt == 33) insert_lean_kernel<true, IN_WIRE, 33><<<G, B, sizeof(lean::Smem<true>), s>>>(d, b, hl, nh, c);
                else insert_lean_kernel<true, IN_WIRE, 48><<<G, B, sizeof(lean::Smem<true>), s>>>(d, b, hl, nh, c);
            } else if (!b.vals) {
                if (in == IN_CSR) insert_lean_kernel<false, IN_CSR, 32><<<G, B, sml, s>>>(d, b, hl, nh, c);
                else insert_lean_kernel<false, IN_FIXED, 32><<<G, B, sml, s>>>(d, b, hl, nh, c);
            } else if (b.prep_fmt == 33) {
                if (in == IN_CSR) insert_lean_kernel<true, IN_CSR, 33><<<G, B, sml, s>>>(d, b, hl, nh, c);
                else insert_lean_kernel<true, IN_FIXED, 33><<<G, B, sml, s>>>(d, b, hl, nh, c);
            } else {
                if (in == IN_CSR) insert_lean_kernel<true, IN_CSR, 48><<<G, B, sml, s>>>(d, b, hl, nh, c);
                else insert_lean_kernel<true, IN_FIXED, 48><<<G, B, sml, s>>>(d, b, hl, nh, c);
            }
            return cudaGetLastError();
        }
        if (b.vals && in != IN_CSR) {
            // fixed-width keys with values (C5), and index re-issue batches with values: 24 warps per
            // CTA, 80 registers — C5u 4x pass 1 20.6 -> 12.8 ms, index re-issue passes 18.9 / 15.3 ->
            // 13.2 / 10.0 ms (CSR batches keep 32 warps: C2 in budget 25.5 vs 27.9 ms, C3 48.9 vs 55.7 ms at 24)
            constexpr int T2 = 768;
            static bool attr2 = false;
            if (!attr2) {
                cudaFuncSetAttribute(insert_stream_kernel<true, T2, IN_FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(stream::Smem<true, T2 / 32>));
                cudaFuncSetAttribute(insert_stream_kernel<true, T2, IN_IDX>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(stream::Smem<true, T2 / 32>));
                attr2 = true;
            }
            c.nw = (uint32_t)grid * (T2 / 32);
            const size_t sm2 = sizeof(stream::Smem<true, T2 / 32>);
            if (in == IN_FIXED) insert_stream_kernel<true, T2, IN_FIXED><<<grid, T2, sm2, s>>>(d, b, hl, nh, c);
            else insert_stream_kernel<true, T2, IN_IDX><<<grid, T2, sm2, s>>>(d, b, hl, nh, c);
        } else if (b.vals) {
            if (in == IN_CSR) insert_stream_kernel<true, T, IN_CSR><<<grid, T, sm, s>>>(d, b, hl, nh, c);
            else if (in == IN_FIXED) insert_stream_kernel<true, T, IN_FIXED><<<grid, T, sm, s>>>(d, b, hl, nh, c);
            else insert_stream_kernel<true, T, IN_IDX><<<grid, T, sm, s>>>(d, b, hl, nh, c);
        } else if (in == IN_CSR && long_keys) {
            // long keys: tails read SEPO_LONG_U words per round trip (tail_rounds)
            constexpr int TL = SEPO_LONG_THREADS;
            static bool attr3 = false;
            if (!attr3) {
                cudaFuncSetAttribute(insert_stream_kernel<false, TL, IN_CSR, SEPO_LONG_U>,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(stream::Smem<false, TL / 32>));
                attr3 = true;
            }
            c.nw = (uint32_t)grid * (TL / 32);
            insert_stream_kernel<false, TL, IN_CSR, SEPO_LONG_U>
                <<<grid, TL, sizeof(stream::Smem<false, TL / 32>), s>>>(d, b, hl, nh, c);
        } else {
            if (in == IN_CSR) insert_stream_kernel<false, T, IN_CSR><<<grid, T, sm, s>>>(d, b, hl, nh, c);
            else if (in == IN_FIXED) insert_stream_kernel<false, T, IN_FIXED><<<grid, T, sm, s>>>(d, b, hl, nh, c);
            else insert_stream_kernel<false, T, IN_IDX><<<grid, T, sm, s>>>(d, b, hl, nh, c);
        }
    } else {
        const hot::Entry* hl = nullptr;
        const unsigned int* nh = nullptr;
        const uint64_t n_sample = 1ull << 18;
        if (hot_scratch && b.n >= hot_min_records(8 * n_sample)) {
            uint8_t* p = reinterpret_cast<uint8_t*>(hot_scratch);
            hot::SampleSlot* tab = reinterpret_cast<hot::SampleSlot*>(p);
            hot::Entry* list = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS);
            unsigned int* n_out = reinterpret_cast<unsigned int*>(list + hot::K);
            unsigned int* hist = n_out + 1;
            cudaMemsetAsync(tab, 0, sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS, s);
            cudaMemsetAsync(n_out, 0, (HOT_HIST + 2) * sizeof(unsigned int), s);
            hot_sample_kernel<<<4 * 148, 256, 0, s>>>(d, b, std::max<uint64_t>(1, b.n / n_sample), std::min(n_sample, b.n), tab);
            hot_hist_kernel<<<2 * 148, 256, 0, s>>>(tab, hist, 4u);
            hot_threshold_kernel<<<1, 1024, 0, s>>>(hist, 4u, (uint32_t)gst::K);
            hot_emit_kernel<<<2 * 148, 256, 0, s>>>(d, b, tab, hist, list, n_out, (uint32_t)gst::K);
            hot_clamp_kernel<<<1, 32, 0, s>>>(n_out, (uint32_t)gst::K);
            hot_resolve_group_kernel<<<1, 1024, 0, s>>>(d, b, list, n_out);
            hl = list;
            nh = n_out;
            if (hot_built) *hot_built = true;
        }
        const size_t sm = sizeof(gst::Smem);
        static bool attrg = false;
        if (!attrg) {
            cudaFuncSetAttribute(insert_group_stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            attrg = true;
        }
        insert_group_stream_kernel<<<grid, gst::THREADS, sm, s>>>(d, b, hl, nh);
    }
    return cudaGetLastError();
}
int sepo_launch_reinsert(const Dev& d, const Batch& b, int grid, cudaStream_t s, bool long_keys) {
    if (b.n == 0) return cudaGetLastError();
    if (long_keys && b.prep_rb == 32 && b.prep_fmt != 33) reinsert_kernel<32, SEPO_LONG_U><<<grid, SEPO_REINS_THREADS, 0, s>>>(d, b);
    else if (b.prep_fmt == 33) reinsert_kernel<33><<<grid, SEPO_REINS_THREADS, 0, s>>>(d, b);
    else if (b.prep_rb == 32) reinsert_kernel<32><<<grid, SEPO_REINS_THREADS, 0, s>>>(d, b);
    else reinsert_kernel<48><<<grid, SEPO_REINS_THREADS, 0, s>>>(d, b);
    return cudaGetLastError();
}
size_t sepo_hot_count_offset() { return sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS + sizeof(hot::Entry) * hot::K; }
size_t sepo_hot_scratch_bytes() {
    return sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS + sizeof(hot::Entry) * hot::K + (HOT_HIST + 16) * 4;
}
int sepo_default_grid(int mode, int n_sms) { (void)mode; return n_sms; }

int sepo_launch_reprobe(const Dev& d, const Batch& b, int mode, int probe, int grid, unsigned long long* tile_counts,
                        cudaStream_t s) {
    if (mode == 0) {
        if (probe) reprobe_kernel<0, true><<<grid, RP_THREADS, 0, s>>>(d, b, tile_counts);
        else reprobe_kernel<0, false><<<grid, RP_THREADS, 0, s>>>(d, b, tile_counts);
    } else {
        if (probe) reprobe_kernel<1, true><<<grid, RP_THREADS, 0, s>>>(d, b, tile_counts);
        else reprobe_kernel<1, false><<<grid, RP_THREADS, 0, s>>>(d, b, tile_counts);
    }
    return cudaGetLastError();
}
uint64_t sepo_reprobe_tiles(uint64_t n) { return (n + RP_TILE - 1) / RP_TILE; }

int sepo_launch_compact(const Batch& b, unsigned long long* tile_counts, uint8_t* ok, uint64_t* oko, uint8_t* ov,
                        uint64_t* ovo, uint64_t m, uint64_t kb, uint64_t vb, int grid, cudaStream_t s) {
    const uint64_t nt = sepo_reprobe_tiles(b.n);
    if (nt) {
        scan_tiles_kernel<<<1, 1024, 0, s>>>(tile_counts, nt);
        compact_kernel<<<grid, CP_THREADS, 0, s>>>(b, tile_counts, ok, oko, ov, ovo);
    }
    finish_offsets_kernel<<<1, 32, 0, s>>>(b.ko ? oko : nullptr, m, kb, b.vo ? ovo : nullptr, vb);
    return cudaGetLastError();
}

int sepo_launch_tile_popc(const Batch& b, unsigned long long* tile_counts, int grid, cudaStream_t s) {
    if (b.n) tile_popc_kernel<<<grid, 64, 0, s>>>(b, tile_counts);
    return cudaGetLastError();
}
int sepo_launch_compact_index(const Batch& b, unsigned long long* tile_counts, uint64_t* idx_out, int grid, cudaStream_t s) {
    const uint64_t nt = sepo_reprobe_tiles(b.n);
    if (nt) {
        scan_tiles_kernel<<<1, 1024, 0, s>>>(tile_counts, nt);
        compact_index_kernel<<<grid, 256, 0, s>>>(b, tile_counts, idx_out);
    }
    return cudaGetLastError();
}
int sepo_launch_partition(const Batch& b, uint32_t P, uint64_t seed, unsigned long long* counts, uint8_t* ok,
                          uint64_t* oko, uint8_t* ov, unsigned long long* h_counts, int grid, cudaStream_t s) {
    const uint64_t ntiles = (b.n + PT_TILE - 1) / PT_TILE;
    if (ntiles == 0) { memset(h_counts, 0, sizeof(unsigned long long) * 3 * P); return 0; }
    part_count_kernel<<<grid, PT_THREADS, 0, s>>>(b, P, seed, counts, ntiles);
    // per-part totals (before the scan turns counts into bases): copy the last base later instead
    scan_tiles_kernel<<<1, 1024, 0, s>>>(counts, (uint64_t)P * ntiles);
    part_scatter_kernel<<<grid, PT_THREADS, 0, s>>>(b, P, seed, counts, ntiles, ok, oko, ov);
    // part starts (the bases of tile 0 of every part) to the host: totals follow by difference
    for (uint32_t p = 0; p < P; ++p)
        cudaMemcpyAsync(h_counts + 3 * p, counts + (uint64_t)p * ntiles * 3, 3 * sizeof(unsigned long long),
                        cudaMemcpyDeviceToHost, s);
    return cudaGetLastError();
}
uint64_t sepo_partition_tiles(uint64_t n) { return (n + PT_TILE - 1) / PT_TILE; }
uint64_t sepo_map_chunks(uint64_t n) { return (n + MC - 1) / MC; }
int sepo_launch_map(const uint8_t* text, uint64_t n, int lines, int pass, unsigned long long* tc, const uint64_t* doc_offsets,
                    uint64_t n_docs, uint8_t* okeys, uint64_t* oko, uint32_t* odoc, cudaStream_t s) {
    const uint64_t nch = (n + MC - 1) / MC;
    if (!nch) return 0;
    const int grid = (int)std::min<uint64_t>((nch + 255) / 256, 8 * 148);
    if (pass == 0) {  // (tc has nch + 1 entries: after the scan the last one holds the totals)
        cudaMemsetAsync(tc + 3 * nch, 0, 24, s);
        map_count_kernel<<<grid, 256, 0, s>>>(text, n, lines, tc);
        scan_tiles_kernel<<<1, 1024, 0, s>>>(tc, nch + 1);
    } else {
        map_write_kernel<<<grid, 256, 0, s>>>(text, n, lines, tc, doc_offsets, n_docs, okeys, oko, odoc);
    }
    return cudaGetLastError();
}
// Router scratch (device): hot-set discovery scratch, then counts [P][grid], bases [P][grid], the hot
// keys' sums [K], per-part hot counts / bases / cursors [3][32] and the long-key counter.
static size_t rh_off_counts() { return (sepo_hot_scratch_bytes() + 255) & ~(size_t)255; }
size_t sepo_route_scratch_bytes(uint32_t P, int grid) {
    return rh_off_counts() + 8 * (2 * (size_t)P * grid + hot::K + 3 * 32 + 8);
}
void sepo_route_layout(uint32_t P, int grid, size_t* counts_off, size_t* hot_pp_off) {
    *counts_off = rh_off_counts();
    *hot_pp_off = rh_off_counts() + 8 * (2 * (size_t)P * grid + hot::K);
}
int sepo_launch_route_hot(const Batch& b, uint32_t P, uint64_t seed, int pass, void* scratch, int grid, WireRec* out,
                          cudaStream_t s, WireRec* const* dstp) {
    static bool attr = false;
    if (!attr) {
        const int sm = (int)sizeof(rh::Smem);
        cudaFuncSetAttribute(route_hot_kernel<0, IN_CSR>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        cudaFuncSetAttribute(route_hot_kernel<0, IN_FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        cudaFuncSetAttribute(route_hot_kernel<1, IN_CSR>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        cudaFuncSetAttribute(route_hot_kernel<1, IN_FIXED>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
        attr = true;
    }
    uint8_t* p = reinterpret_cast<uint8_t*>(scratch);
    hot::SampleSlot* tab = reinterpret_cast<hot::SampleSlot*>(p);
    hot::Entry* list = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS);
    unsigned int* n_out = reinterpret_cast<unsigned int*>(list + hot::K);
    unsigned long long* counts = reinterpret_cast<unsigned long long*>(p + rh_off_counts());
    unsigned long long* bases = counts + (size_t)P * grid;
    unsigned long long* hot_sum = bases + (size_t)P * grid;
    unsigned long long* hot_pp = hot_sum + hot::K;   // [32] hot keys per part
    unsigned long long* hot_base = hot_pp + 32;      // [32]
    unsigned long long* hot_cur = hot_base + 32;     // [32]
    unsigned long long* longk = hot_cur + 32;
    const bool have = b.n >= hot_min_records(8ull << 18);
    // the sorted hot list lives in the sample table's space (free once the list is emitted)
    hot::Entry* sorted = reinterpret_cast<hot::Entry*>(p + sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS -
                                                       sizeof(hot::Entry) * hot::K);
    const hot::Entry* hl = have ? sorted : nullptr;
    const size_t sm = sizeof(rh::Smem);
    if (pass == 0) {
        cudaMemsetAsync(hot_pp, 0, 8 * (3 * 32 + 8), s);
        cudaMemsetAsync(n_out, 0, (HOT_HIST + 2) * sizeof(unsigned int), s);
        if (have) {  // hot-set discovery on the route hash (no table entries: nothing to resolve)
            Dev d{};
            d.seed = seed;
            const uint64_t n_sample = 1ull << 18;
            unsigned int* hist = n_out + 1;
            cudaMemsetAsync(tab, 0, sizeof(hot::SampleSlot) * hot::SAMPLE_SLOTS, s);
            hot_sample_kernel<<<4 * 148, 256, 0, s>>>(d, b, std::max<uint64_t>(1, b.n / n_sample), std::min(n_sample, b.n), tab);
            hot_hist_kernel<<<2 * 148, 256, 0, s>>>(tab, hist, 4u);
            hot_threshold_kernel<<<1, 1024, 0, s>>>(hist, 4u, (uint32_t)hot::K);
            hot_emit_kernel<<<2 * 148, 256, 0, s>>>(d, b, tab, hist, list, n_out, (uint32_t)hot::K);
            hot_clamp_kernel<<<1, 32, 0, s>>>(n_out, (uint32_t)hot::K);
            rh_sort_hot<<<1, 1024, 0, s>>>(list, n_out, sorted);
            rh_count_hot<<<8, 256, 0, s>>>(hl, n_out, P, hot_pp);
        }
        if (b.n) {
            if (b.ko) route_hot_kernel<0, IN_CSR><<<grid, rh::THREADS, sm, s>>>(b, P, seed, hl, n_out, counts, nullptr, nullptr, longk, nullptr, nullptr);
            else route_hot_kernel<0, IN_FIXED><<<grid, rh::THREADS, sm, s>>>(b, P, seed, hl, n_out, counts, nullptr, nullptr, longk, nullptr, nullptr);
        } else {
            cudaMemsetAsync(counts, 0, 8 * (size_t)P * grid, s);
        }
    } else {
        cudaMemsetAsync(hot_sum, 0, 8 * hot::K, s);
        if (b.n) {
            if (b.ko) route_hot_kernel<1, IN_CSR><<<grid, rh::THREADS, sm, s>>>(b, P, seed, hl, n_out, nullptr, bases, hot_sum, nullptr, out, dstp);
            else route_hot_kernel<1, IN_FIXED><<<grid, rh::THREADS, sm, s>>>(b, P, seed, hl, n_out, nullptr, bases, hot_sum, nullptr, out, dstp);
        }
        if (have) rh_emit_hot<<<8, 256, 0, s>>>(hl, n_out, P, hot_sum, hot_base, hot_cur, out, dstp);
    }
    return cudaGetLastError();
}
int sepo_launch_max_key_len(const uint64_t* ko, uint64_t n, unsigned long long* out, cudaStream_t s) {
    cudaMemsetAsync(out, 0, 8, s);
    if (n) max_key_len_kernel<<<(unsigned)std::min<uint64_t>((n + 255) / 256, 4 * 148), 256, 0, s>>>(ko, n, out);
    return cudaGetLastError();
}
int sepo_launch_shift_offsets(uint64_t* ko, uint64_t n, const uint64_t* seg_rec, const uint64_t* seg_base, uint32_t n_segs,
                              uint64_t total, cudaStream_t s) {
    shift_offsets_kernel<<<(unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 4096)), 256, 0, s>>>(
        ko, n, seg_rec, seg_base, n_segs, total);
    return cudaGetLastError();
}
int sepo_launch_seal(const Dev& d, uint32_t n_slots, cudaStream_t s) {
    seal_kernel<<<(2 * n_slots + 255) / 256, 256, 0, s>>>(d, n_slots);
    return cudaGetLastError();
}
int sepo_launch_classify(const Dev& d, int honor_retain, cudaStream_t s) {
    classify_kernel<<<1, 1024, 0, s>>>(d, honor_retain);
    return cudaGetLastError();
}
int sepo_launch_relink(const Dev& d, cudaStream_t s) {
    relink_kernel<<<148, 128, 0, s>>>(d);
    return cudaGetLastError();
}
int sepo_launch_init(const Dev& d, uint32_t n_slots, cudaStream_t s) {
    init_state_kernel<<<296, 256, 0, s>>>(d, n_slots);
    return cudaGetLastError();
}
