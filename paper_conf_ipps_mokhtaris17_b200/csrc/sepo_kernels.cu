// sepo_kernels.cu — the SEPO hot path on sm_100a (PAPER.md cited as P:L<line>).
//
//   insert_kernel   a1..a7  record ingest + hash, tile pre-aggregation of equal keys, chain walk,
//                           combine / group in place, page-pool allocation, lock-free head link,
//                           decline -> postpone bitmap + count
//   reprobe_kernel  a8      end-of-pass re-probe of declined records
//   compact_*       a9      stream compaction of the postponed records (re-issue)
//   seal/classify/relink a10 pass boundary: seal open pages, pick cold pages, rebuild the free
//                           stack and (GROUP) re-link retained key pages
//
// The insert kernel is persistent: gridDim.x CTAs (the allocator slots) stride over tiles of TILE
// records; per tile it stages offsets/hashes in shared memory, folds equal keys into one slot of
// a shared open-addressing table (warp __match_any_sync first, so a hot Zipf key costs one shared
// atomic per warp and one global op per tile), then resolves each distinct key against the global
// table with one thread per key.
#include "sepo_dev.cuh"
#include "sepo_kernels.h"

namespace sepo {

constexpr uint32_t EMPTY = 0xffffffffu;

template <int MODE> struct Cfg;
template <> struct Cfg<0> { static constexpr int THREADS = 512, TILE = 2048, NSLOT = 4096; };  // COMBINE
template <> struct Cfg<1> { static constexpr int THREADS = 512, TILE = 1024, NSLOT = 2048; };  // GROUP

template <int MODE>
struct Smem {
    static constexpr int TILE = Cfg<MODE>::TILE, NSLOT = Cfg<MODE>::NSLOT;
    uint64_t rec_off[TILE];
    uint64_t rec_hash[TILE];
    uint32_t rec_len[TILE];
    uint32_t slot_rep[NSLOT];
    unsigned long long slot_sum[NSLOT];  // COMBINE: value sum; GROUP: record count (rank source)
    uint16_t dlist[NSLOT];
    uint8_t slot_res[NSLOT];
    // GROUP: where the slot's values go: chunk A (base slot a, `granted` values), then chunk B
    uint64_t g_a[MODE == 1 ? NSLOT : 1];
    uint64_t g_b[MODE == 1 ? NSLOT : 1];
    uint32_t g_abase[MODE == 1 ? NSLOT : 1];
    uint32_t g_granted[MODE == 1 ? NSLOT : 1];
    unsigned long long cur[2];  // allocation cursors (entry/key pages, value pages)
    uint32_t ndist;
    unsigned long long post, toolarge, dead;
};

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ uint32_t lanemask_lt() { return (1u << lane_id()) - 1u; }

// value of record i for COMBINE (vw bytes LE, or 1 when vals == nullptr)
__device__ __forceinline__ uint64_t rec_value(const Batch& b, uint64_t i) {
    if (b.vals == nullptr) return 1ull;
    switch (b.vw) {
        case 8: return __ldg(reinterpret_cast<const unsigned long long*>(b.vals) + i);
        case 4: return __ldg(reinterpret_cast<const unsigned int*>(b.vals) + i);
        case 2: return __ldg(reinterpret_cast<const unsigned short*>(b.vals) + i);
        default: return b.vals[i];
    }
}
__device__ __forceinline__ void rec_key(const Batch& b, uint64_t i, uint64_t& s, uint32_t& len) {
    if (b.ko) {
        s = __ldg(reinterpret_cast<const unsigned long long*>(b.ko) + i);
        len = (uint32_t)(__ldg(reinterpret_cast<const unsigned long long*>(b.ko) + i + 1) - s);
    } else {
        s = i * (uint64_t)b.kw;
        len = b.kw;
    }
}
// GROUP value bytes of record i
__device__ __forceinline__ void rec_val_span(const Batch& b, uint64_t i, uint64_t& s, uint32_t& len) {
    if (b.vo) {
        s = __ldg(reinterpret_cast<const unsigned long long*>(b.vo) + i);
        len = (uint32_t)(__ldg(reinterpret_cast<const unsigned long long*>(b.vo) + i + 1) - s);
    } else {
        s = i * (uint64_t)b.vw;
        len = b.vw;
    }
}

// ---------------------------------------------------------------- GROUP value-list helpers
// Value chunk capacity for k values when the key's head chunk has capacity `prev` (0: none in
// this generation): geometric growth so a hot key's list is a few large chunks.
__device__ __forceinline__ uint32_t chunk_cap(const Dev& d, uint32_t k, uint32_t prev, uint32_t slot_bytes) {
    uint32_t maxcap = (d.page_bytes / 4 - CHUNK_HDR) / slot_bytes;
    uint32_t c = prev ? min(prev * 2u, maxcap) : 4u;
    c = max(c, k);
    return min(c, (d.page_bytes - CHUNK_HDR) / slot_bytes);
}
__device__ __forceinline__ uint32_t chunk_bytes(uint32_t cap, uint32_t slot_bytes) { return CHUNK_HDR + align8(cap * slot_bytes); }
__device__ __forceinline__ uint64_t vref_of(const Dev& d, uint64_t off) { return ((uint64_t)d.gen << 40) | (uint64_t)off_ref(off); }
__device__ __forceinline__ bool vref_resident(const Dev& d, uint64_t vref) { return vref != 0 && (uint32_t)(vref >> 40) == d.gen; }
__device__ __forceinline__ uint8_t* vref_ptr(const Dev& d, uint64_t vref) { return ref_ptr(d, (uint32_t)vref); }
// owner identity of a key entry: birth generation << 40 | entry ref
__device__ __forceinline__ uint64_t owner_of(const Dev& d, uint8_t* e) {
    uint32_t birth = ldcg32(e + 24);
    return ((uint64_t)birth << 40) | (uint64_t)off_ref((uint64_t)(e - d.pool));
}
__device__ __forceinline__ void init_chunk(uint8_t* c, uint32_t cap, uint32_t vwslot, uint32_t fill, uint64_t owner,
                                           uint64_t next) {
    *reinterpret_cast<uint32_t*>(c) = chunk_bytes(cap, vwslot) | K_VCHUNK;
    *reinterpret_cast<uint32_t*>(c + 4) = fill;
    *reinterpret_cast<unsigned long long*>(c + 8) = owner;
    *reinterpret_cast<unsigned long long*>(c + 16) = next;
    *reinterpret_cast<uint32_t*>(c + 24) = cap;
    *reinterpret_cast<uint32_t*>(c + 28) = vwslot;
}
// push chunk `cref` (already holding its values' slots) onto the list head of key entry e
__device__ __forceinline__ void push_chunk(uint8_t* e, uint8_t* c, uint64_t cref, uint64_t observed) {
    unsigned long long* head = reinterpret_cast<unsigned long long*>(e + 16);
    while (true) {
        *reinterpret_cast<unsigned long long*>(c + 16) = observed;
        __threadfence();
        unsigned long long old = atomicCAS(head, observed, cref);
        if (old == observed) return;
        observed = old;
    }
}
// Reserve k slots in the resident head chunk of key entry e. Returns granted count (0..k),
// the chunk ref in *cref and the first slot in *base; *head_out = observed head, *prev_cap.
__device__ __forceinline__ uint32_t reserve_head(const Dev& d, uint8_t* e, uint32_t k, uint64_t* cref, uint32_t* base,
                                                 uint64_t* head_out, uint32_t* prev_cap) {
    uint64_t h = ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(e + 16));
    *head_out = h;
    *prev_cap = 0;
    *cref = 0;
    if (!vref_resident(d, h)) return 0;
    uint8_t* c = vref_ptr(d, h);
    uint32_t cap = ldcg32(c + 24);
    *prev_cap = cap;
    if (ldcg32(c + 4) >= cap) return 0;
    uint32_t old = atomicAdd(reinterpret_cast<unsigned int*>(c + 4), k);
    if (old >= cap) return 0;
    *cref = h;
    *base = old;
    return min(k, cap - old);
}

// ================================================================ insert kernel (a1..a7)
template <int MODE>
__global__ void __launch_bounds__(Cfg<MODE>::THREADS, 2) insert_kernel(Dev d, Batch b) {
    constexpr int THREADS = Cfg<MODE>::THREADS, TILE = Cfg<MODE>::TILE, NSLOT = Cfg<MODE>::NSLOT;
    constexpr int R = TILE / THREADS;
    extern __shared__ __align__(16) uint8_t smem_raw[];
    Smem<MODE>& S = *reinterpret_cast<Smem<MODE>*>(smem_raw);
    const uint32_t tid = threadIdx.x, lane = lane_id(), warp = tid >> 5;
    const uint32_t PB = d.page_bytes;

    for (int p = tid; p < NSLOT; p += THREADS) { S.slot_rep[p] = EMPTY; S.slot_sum[p] = 0; }
    if (tid == 0) {
        S.cur[0] = d.cursors[2 * blockIdx.x];
        S.cur[1] = d.cursors[2 * blockIdx.x + 1];
        S.post = 0; S.toolarge = 0; S.dead = 0;
    }
    __syncthreads();

    const uint64_t ntiles = (b.n + TILE - 1) / TILE;
    for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const uint64_t t0 = tile * TILE;
        // ---- phase 1: ingest + hash (a1)
        uint64_t my_s[R], my_h[R];
        uint32_t my_len[R];
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const uint32_t r = k * THREADS + tid;
            const uint64_t i = t0 + r;
            my_len[k] = 0; my_s[k] = 0; my_h[k] = 0;
            if (i < b.n) {
                rec_key(b, i, my_s[k], my_len[k]);
                my_h[k] = hash_key(b.keys + my_s[k], my_len[k], d.seed);
                S.rec_off[r] = my_s[k];
                S.rec_len[r] = my_len[k];
                S.rec_hash[r] = my_h[k];
            }
        }
        if (tid == 0) S.ndist = 0;
        __syncthreads();
        // ---- phase 2: fold equal keys of the tile into shared slots (a2)
        uint32_t my_slot[R], my_rank[R];
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const uint32_t r = k * THREADS + tid;
            const bool valid = t0 + r < b.n;
            const unsigned vm = __ballot_sync(FULLMASK, valid);
            const unsigned long long hh = valid ? my_h[k] : (0xffffffff00000000ull | lane);
            unsigned grp = __match_any_sync(FULLMASK, hh) & vm;
            const uint32_t leader = grp ? (uint32_t)(__ffs(grp) - 1) : lane;
            const uint64_t ls = __shfl_sync(FULLMASK, my_s[k], leader);
            const uint32_t llen = __shfl_sync(FULLMASK, my_len[k], leader);
            bool eq = valid && (lane == leader || (llen == my_len[k] && in_key_eq(b.keys + my_s[k], b.keys + ls, llen)));
            const unsigned eqm = __ballot_sync(FULLMASK, eq);
            const unsigned joined = grp & eqm;           // lanes folded into the leader
            const bool inserter = valid && (lane == leader || !eq);
            uint64_t contrib = 0;
            if (MODE == 0) {
                const uint64_t v = valid ? rec_value(b, t0 + r) : 0;
                if (b.vals == nullptr) {
                    contrib = (lane == leader) ? (uint64_t)__popc(joined) : 1ull;
                } else {
                    uint64_t acc = 0;
                    if (__any_sync(FULLMASK, __popc(joined) > 1)) {
                        for (int q = 0; q < 32; ++q) {
                            uint64_t vq = __shfl_sync(FULLMASK, v, q);
                            if ((joined >> q) & 1u) acc += vq;
                        }
                    } else {
                        acc = v;
                    }
                    contrib = (lane == leader) ? acc : v;
                }
            } else {
                contrib = (lane == leader) ? (uint64_t)__popc(joined) : 1ull;
            }
            uint32_t pos = EMPTY, rank0 = 0;
            if (inserter) {
                pos = (uint32_t)(my_h[k] >> 7) & (NSLOT - 1);
                while (true) {
                    uint32_t cur = *reinterpret_cast<volatile uint32_t*>(&S.slot_rep[pos]);
                    if (cur == EMPTY) {
                        cur = atomicCAS(&S.slot_rep[pos], EMPTY, r);
                        if (cur == EMPTY) break;
                    }
                    if (S.rec_hash[cur] == my_h[k] && S.rec_len[cur] == my_len[k] &&
                        in_key_eq(b.keys + S.rec_off[cur], b.keys + my_s[k], my_len[k]))
                        break;
                    pos = (pos + 1) & (NSLOT - 1);
                }
                rank0 = (uint32_t)atomicAdd(&S.slot_sum[pos], (unsigned long long)contrib);
            }
            // followers take the leader's slot; rank of a record among its key's records in the tile
            const uint32_t lpos = __shfl_sync(FULLMASK, pos, leader);
            const uint32_t lrank = __shfl_sync(FULLMASK, rank0, leader);
            if (valid && eq && lane != leader) {
                my_slot[k] = lpos;
                my_rank[k] = lrank + __popc(joined & lanemask_lt());
            } else {
                my_slot[k] = pos;
                my_rank[k] = rank0;
            }
        }
        __syncthreads();
        // ---- phase 3: dense list of the tile's distinct keys
        for (int p0 = 0; p0 < NSLOT; p0 += THREADS) {
            const int p = p0 + tid;
            const bool occ = S.slot_rep[p] != EMPTY;
            const unsigned bal = __ballot_sync(FULLMASK, occ);
            uint32_t base = 0;
            if (lane == 0 && bal) base = atomicAdd(&S.ndist, (uint32_t)__popc(bal));
            base = __shfl_sync(FULLMASK, base, 0);
            if (occ) S.dlist[base + __popc(bal & lanemask_lt())] = (uint16_t)p;
        }
        __syncthreads();
        // ---- phase 4: one thread per distinct key against the global table (a3..a6)
        const uint32_t nd = S.ndist;
        for (uint32_t j0 = 0; j0 < nd; j0 += THREADS) {
            const uint32_t j = j0 + tid;
            const bool act = j < nd;
            uint32_t pos = 0, r = 0, len = 0;
            uint64_t s = 0, h = 0, sum = 0;
            if (act) {
                pos = S.dlist[j];
                r = S.slot_rep[pos];
                s = S.rec_off[r]; len = S.rec_len[r]; h = S.rec_hash[r];
                sum = S.slot_sum[pos];
            }
            const uint8_t* key = b.keys + s;
            const uint32_t bkt = act ? bucket_of(h, d.n_buckets) : 0;
            const uint32_t tag = tag_of(h);
            const uint32_t koff = MODE == 0 ? CENTRY_HDR : GKEY_HDR;
            uint32_t head = 0;
            uint8_t* found = nullptr;
            if (act) {
                head = ld_relaxed_u32(d.dir + bkt);
                found = chain_find(d, head, 0, tag, len, key, koff);
            }
            uint32_t res = R_OK;
            const uint32_t esize = koff + align8(len);
            bool need = act && !found;
            if (need && (len > 65535u - 64u || esize > PB)) { need = false; res = R_TOOLARGE; }
            if (need && inject_fail(d, h, t0 + r)) { need = false; res = R_POST; }

            if (MODE == 0) {
                if (act && found) atomicAdd(reinterpret_cast<unsigned long long*>(found + 16), (unsigned long long)sum);
                const uint64_t off = warp_alloc(d, &S.cur[0], need, esize, (uint8_t)PAGE_ENTRY);
                if (need) {
                    if (off == ~0ull) {
                        res = R_POST;
                    } else {
                        uint8_t* e = d.pool + off;
                        *reinterpret_cast<uint32_t*>(e) = esize | K_COMBINE;
                        *reinterpret_cast<uint32_t*>(e + 4) = head;
                        *reinterpret_cast<uint32_t*>(e + 8) = tag;
                        *reinterpret_cast<uint32_t*>(e + 12) = len;
                        *reinterpret_cast<unsigned long long*>(e + 16) = sum;
                        store_key(e + CENTRY_HDR, key, len);
                        __threadfence();
                        const uint32_t me = off_ref(off);
                        while (true) {  // lock-free head insertion
                            const uint32_t old = atomicCAS(d.dir + bkt, head, me);
                            if (old == head) break;
                            uint8_t* w = chain_find(d, old, head, tag, len, key, CENTRY_HDR);
                            if (w) {  // the key was linked meanwhile: combine there, retire ours
                                atomicAdd(reinterpret_cast<unsigned long long*>(w + 16), (unsigned long long)sum);
                                *reinterpret_cast<uint32_t*>(e) = esize | K_DEAD;
                                atomicAdd(&S.dead, (unsigned long long)esize);
                                break;
                            }
                            head = old;
                            *reinterpret_cast<uint32_t*>(e + 4) = head;
                            __threadfence();
                        }
                    }
                }
                if (act) {
                    S.slot_res[pos] = (uint8_t)res;
                    S.slot_rep[pos] = EMPTY;
                    S.slot_sum[pos] = 0;
                }
            } else {
                // ---------------- GROUP (multi-valued): key entry + value chunks
                const uint32_t k = (uint32_t)sum;
                const uint32_t vws = b.vo ? 0u : b.vw;  // fixed-width slot bytes (variable: see host)
                uint64_t a_ref = 0, b_ref = 0;
                uint32_t abase = 0, granted = 0, prev_cap = 0;
                uint64_t lhead = 0;
                if (act && found) granted = reserve_head(d, found, k, &a_ref, &abase, &lhead, &prev_cap);
                // values that still need a chunk
                const bool need_chunk = act && res == R_OK && granted < k;
                const uint32_t rest = k - granted;
                const uint32_t ccap = need_chunk ? chunk_cap(d, rest, prev_cap, vws) : 0;
                const uint32_t csize = chunk_bytes(ccap, vws);
                // allocate the key entry (new keys), then the chunk (value pages)
                const uint64_t koffp = warp_alloc(d, &S.cur[0], need, esize, (uint8_t)PAGE_ENTRY);
                if (need && koffp == ~0ull) res = R_POST;
                const bool want_chunk = need_chunk && res == R_OK;
                const uint64_t coff = warp_alloc(d, &S.cur[1], want_chunk, csize, (uint8_t)PAGE_VALUE);
                uint8_t* e = found;
                if (need && res == R_OK) {
                    // new key entry; linked even if its chunk allocation failed (then all its
                    // values are pending and its page is retained at the pass end)
                    uint8_t* ne = d.pool + koffp;
                    *reinterpret_cast<uint32_t*>(ne) = esize | K_GKEY;
                    *reinterpret_cast<uint32_t*>(ne + 4) = head;
                    *reinterpret_cast<uint32_t*>(ne + 8) = tag;
                    *reinterpret_cast<uint32_t*>(ne + 12) = len;
                    *reinterpret_cast<unsigned long long*>(ne + 16) = 0ull;
                    *reinterpret_cast<uint32_t*>(ne + 24) = d.gen;
                    *reinterpret_cast<uint32_t*>(ne + 28) = 0u;
                    store_key(ne + GKEY_HDR, key, len);
                    __threadfence();
                    const uint32_t me = off_ref(koffp);
                    e = ne;
                    while (true) {
                        const uint32_t old = atomicCAS(d.dir + bkt, head, me);
                        if (old == head) break;
                        uint8_t* w = chain_find(d, old, head, tag, len, key, GKEY_HDR);
                        if (w) {
                            *reinterpret_cast<uint32_t*>(ne) = esize | K_DEAD;
                            atomicAdd(&S.dead, (unsigned long long)esize);
                            e = w;
                            break;
                        }
                        head = old;
                        *reinterpret_cast<uint32_t*>(ne + 4) = head;
                        __threadfence();
                    }
                }
                if (want_chunk && coff != ~0ull) {
                    uint8_t* c = d.pool + coff;
                    const uint64_t cref = vref_of(d, coff);
                    init_chunk(c, ccap, vws, rest, owner_of(d, e), 0ull);
                    push_chunk(e, c, cref, ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(e + 16)));
                    b_ref = cref;
                } else if (want_chunk) {
                    b_ref = 0;  // rest of the values are postponed (key stays resident: pending)
                }
                if (act) {
                    if (res == R_OK && granted == 0 && b_ref == 0) res = R_POST;
                    S.slot_res[pos] = (uint8_t)res;
                    S.g_a[pos] = a_ref;
                    S.g_b[pos] = b_ref;
                    S.g_abase[pos] = abase;
                    S.g_granted[pos] = granted;
                    S.slot_rep[pos] = EMPTY;
                    S.slot_sum[pos] = 0;
                }
            }
        }
        __syncthreads();
        // ---- phase 5: per-record outcome -> bitmap word (a7); GROUP: write values into slots
#pragma unroll
        for (int k = 0; k < R; ++k) {
            const uint32_t r = k * THREADS + tid;
            const uint64_t i = t0 + r;
            const bool valid = i < b.n;
            bool post = false;
            if (valid) {
                const uint32_t res = S.slot_res[my_slot[k]];
                if (MODE == 0) {
                    post = res != R_OK;
                } else {
                    post = res != R_OK;
                    if (!post) {
                        const uint32_t g = S.g_granted[my_slot[k]];
                        const uint32_t rk = my_rank[k];
                        uint8_t* c = nullptr;
                        uint32_t slot = 0;
                        if (rk < g) { c = vref_ptr(d, S.g_a[my_slot[k]]); slot = S.g_abase[my_slot[k]] + rk; }
                        else if (S.g_b[my_slot[k]]) { c = vref_ptr(d, S.g_b[my_slot[k]]); slot = rk - g; }
                        else post = true;
                        if (c) {
                            uint64_t vs; uint32_t vl;
                            rec_val_span(b, i, vs, vl);
                            uint8_t* dst = c + CHUNK_HDR + (uint64_t)slot * vl;
                            for (uint32_t q = 0; q < vl; ++q) dst[q] = __ldg(b.vals + vs + q);
                        }
                    }
                }
            }
            const unsigned bits = __ballot_sync(FULLMASK, post);
            const unsigned tl = __ballot_sync(FULLMASK, valid && S.slot_res[valid ? my_slot[k] : 0] == R_TOOLARGE);
            const uint64_t wstart = t0 + k * THREADS + warp * 32;
            if (lane == 0 && wstart < b.n) {
                b.bitmap[wstart >> 5] = bits;
                if (bits) atomicAdd(&S.post, (unsigned long long)__popc(bits));
                if (tl) atomicAdd(&S.toolarge, (unsigned long long)__popc(tl));
            }
        }
        __syncthreads();
    }
    __syncthreads();
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
                uint32_t want_cap = 0;
                if (mine) {
                    const uint64_t h = hash_key(b.keys + s, len, d.seed);
                    const uint32_t koff = MODE == 0 ? CENTRY_HDR : GKEY_HDR;
                    const uint32_t head = ld_relaxed_u32(d.dir + bucket_of(h, d.n_buckets));
                    e = chain_find(d, head, 0, tag_of(h), len, b.keys + s, koff);
                    if (MODE == 0 && e) {  // resident: combine now
                        atomicAdd(reinterpret_cast<unsigned long long*>(e + 16), (unsigned long long)rec_value(b, i));
                        still = false;
                    }
                    if (MODE == 1 && e) {  // resident key: append the value if its head chunk has room
                        uint64_t cref = 0, lhead = 0;
                        uint32_t base = 0, pcap = 0;
                        const uint32_t g = reserve_head(d, e, 1, &cref, &base, &lhead, &pcap);
                        if (g) {
                            uint64_t vs; uint32_t vl;
                            rec_val_span(b, i, vs, vl);
                            uint8_t* dst = vref_ptr(d, cref) + CHUNK_HDR + (uint64_t)base * vl;
                            for (uint32_t q = 0; q < vl; ++q) dst[q] = __ldg(b.vals + vs + q);
                            still = false;
                        } else {
                            want_cap = chunk_cap(d, 1, pcap, b.vw);
                        }
                    }
                }
                if (MODE == 1) {
                    const bool want = mine && still && e != nullptr;
                    const uint64_t coff = warp_alloc(d, &s_cur[1], want, chunk_bytes(want ? want_cap : 0, b.vw),
                                                     (uint8_t)PAGE_VALUE);
                    if (want) {
                        if (coff != ~0ull) {
                            uint8_t* c = d.pool + coff;
                            init_chunk(c, want_cap, b.vw, 1, owner_of(d, e), 0ull);
                            uint64_t vs; uint32_t vl;
                            rec_val_span(b, i, vs, vl);
                            for (uint32_t q = 0; q < vl; ++q) c[CHUNK_HDR + q] = __ldg(b.vals + vs + q);
                            push_chunk(e, c, vref_of(d, coff),
                                       ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(e + 16)));
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
            for (uint32_t x = 0; x < len; ++x) ok[pos[1] + x] = __ldg(b.keys + s + x);
            if (b.vals) {
                uint64_t vs; uint32_t vl;
                if (b.vo) { rec_val_span(b, i, vs, vl); ovo[pos[0]] = pos[2]; }
                else { vs = i * (uint64_t)b.vw; vl = b.vw; }
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
    if (tid == 0) {
        d.ctrl->n_evict = s_base[0];
        d.ctrl->n_free = s_base[1];
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
                const uint64_t h = hash_key(e + GKEY_HDR, len, d.seed);
                (void)tag;
                const uint32_t bkt = bucket_of(h, d.n_buckets);
                const uint32_t me = off_ref((uint64_t)(e - d.pool));
                uint32_t head = ld_relaxed_u32(d.dir + bkt);
                while (true) {
                    *reinterpret_cast<uint32_t*>(e + 4) = head;
                    __threadfence();
                    const uint32_t old = atomicCAS(d.dir + bkt, head, me);
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

}  // namespace sepo

// ================================================================ launchers
using namespace sepo;

int sepo_launch_insert(const Dev& d, const Batch& b, int mode, int grid, cudaStream_t s) {
    if (mode == 0) {
        size_t sm = sizeof(Smem<0>);
        static bool attr0 = false;
        if (!attr0) { cudaFuncSetAttribute(insert_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm); attr0 = true; }
        insert_kernel<0><<<grid, Cfg<0>::THREADS, sm, s>>>(d, b);
    } else {
        size_t sm = sizeof(Smem<1>);
        static bool attr1 = false;
        if (!attr1) { cudaFuncSetAttribute(insert_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm); attr1 = true; }
        insert_kernel<1><<<grid, Cfg<1>::THREADS, sm, s>>>(d, b);
    }
    return cudaGetLastError();
}
size_t sepo_insert_smem(int mode) { return mode == 0 ? sizeof(Smem<0>) : sizeof(Smem<1>); }
int sepo_insert_threads(int mode) { return mode == 0 ? Cfg<0>::THREADS : Cfg<1>::THREADS; }

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
