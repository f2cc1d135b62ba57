// sepo_capi.cu — host engine + C ABI of the SEPO hash table (include/sepo.h).
//
// The engine owns: the device budget region (one cudaMalloc, carved into directory, allocator
// state and page pool), a pinned host arena that receives evicted pages, the
// generation images used to assemble the result, streams/events, and device scratch for
// sepo_run's re-issue buffers. All record processing runs in sepo_kernels.cu; the host only
// sequences kernels, copies pages and parses page images into the exported arrays.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <functional>
#include <atomic>
#include <string>
#include <string_view>
#include <thread>
#include <unordered_map>
#include <vector>

#include "sepo.h"
#include "sepo_dev.cuh"
#include "sepo_kernels.h"
#if SEPO_WITH_NCCL
#include <nccl.h>
#endif

using namespace sepo;

namespace {
thread_local std::string g_err;

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}

struct PinChunk {
    uint8_t* p = nullptr;
    size_t cap = 0, used = 0;
};

struct Run {  // consecutive evicted pages [first, first+count) at host address p
    uint32_t first, count;
    uint8_t* p;
};
struct GenImage {
    uint32_t gen;
    std::vector<Run> runs;
};

struct DevBuf {
    void* p = nullptr;
    size_t cap = 0;
    int grow(size_t bytes) {
        if (bytes <= cap) return 0;
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
        // 25 % headroom, 2 MiB granules: re-issue sizes fluctuate from run to run (the order in
        // which warps race for the last pages), and a cudaFree + cudaMalloc of a GiB-sized buffer
        // inside a job costs tens of milliseconds
        size_t want = std::max<size_t>(bytes + bytes / 4, 1 << 20);
        want = (want + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
        if (cudaMalloc(&p, want) != cudaSuccess) {
            cudaGetLastError();
            return -1;
        }
        cap = want;
        return 0;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
    }
};

enum State { ST_ACTIVE = 0, ST_EXPORTED = 1, ST_BROKEN = 2 };
const size_t kMaxGrid = 1024;  // cursor slots reserved in the budget region
const uint64_t kPrepChunk = 256;  // = PREP_CHUNK (sepo_kernels.cu): prepared slots a warp reserves at once
}  // namespace

struct sepo_table {
    int device = 0;
    size_t budget = 0;
    uint64_t n_buckets = 0;
    uint32_t page_bytes = 0, page_shift = 0, n_pages = 0;
    int grid = 0, n_sms = 0;
    uint8_t* region = nullptr;
    int placement = SEPO_POOL_DEVICE;  // where the page pool lives (residency ablations, NEXT-1)
    uint8_t* pool_alloc = nullptr;     // non-device pool: the host pinned / managed allocation
    uint8_t* pool_dev = nullptr;       // its device-visible address
    Dev d{};
    sepo_options opts{};
    cudaStream_t stream = nullptr, copy_stream = nullptr;
    bool own_stream = false;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev_copy = nullptr, ev_comp = nullptr, evc0 = nullptr, evc1 = nullptr;
    Ctrl* h_ctrl = nullptr;        // pinned mirror of the device control block
    uint32_t* h_evict = nullptr;   // pinned evict list
    uint64_t* h_ko = nullptr;      // pinned: first/last key offset of the last insert batch
    State state = ST_ACTIVE;
    bool dirty = false;            // resident generation holds data not yet evicted
    bool configured_once = false;
    bool inserted = false;
    uint32_t batch_seq = 0;
    uint64_t pages_resident_retained = 0;
    uint64_t pending_idx_key_bytes = 0;  // key bytes of the next indexed re-issue batch (stats)
    uint64_t last_job_pages = 0;         // most pages resident at once in the previous job (0: none yet)
    std::vector<PinChunk> arena;
    std::vector<GenImage> gens;
    sepo_stats st{};
    double last_insert_ms = 0;
    // scratch
    DevBuf tile_counts, bm, buf[2][4];  // ping-pong: keys, key offsets, vals, val offsets
    DevBuf in_stage[4];
    DevBuf hot;  // hot-set discovery scratch (COMBINE)
    DevBuf idxb[2];  // sepo_run re-issue index lists (ping-pong)
    DevBuf prep[2];  // sepo_run COMBINE: prepared re-issue records (ping-pong)
    DevBuf prep_n;   // their device counters
    DevBuf lk_pages; // sepo_lookup: page ids of the generation being probed
    // multi-GPU data plane (sepo_attach_nccl / sepo_insert_batch_sharded / sepo_drain)
    void* nccl = nullptr;     // ncclComm_t
    int nranks = 1, rank = 0;
    int shard_fmt = 0;        // records held: 0 none yet, 1 wire records, 2 CSR (keys, offsets[, values])
    DevBuf sh_send[3], sh_held[3], sh_tmp[3], sh_cnt;  // route output; records held; exchange scratch; counts
    uint64_t sh_n = 0, sh_kb = 0, sh_vb = 0;          // records / key bytes / value bytes held
    cudaStream_t route_stream = nullptr;  // sepo_run_sharded: route + exchange of chunk c+1 beside chunk c's insert
    DevBuf sh_recv[2];                    // sepo_run_sharded: wire records received (ping-pong per chunk)
    // sepo_run_sharded over peer memory: a symmetric NCCL window of 2 x win_cap wire records per rank
    void* win_buf = nullptr;              // ncclMemAlloc
    void* win = nullptr;                  // ncclWindow_t (device-side handle)
    uint64_t win_cap = 0;                 // records per slot
    bool win_failed = false;              // registration failed once: NCCL send/recv from then on
    bool lookup_done = false;
    std::vector<cudaEvent_t>* h2d_chunks = nullptr;  // sepo_run on host input: copy events of pass-1 chunks
    uint64_t h2d_chunk_records = 0;  // sepo_lookup restored old generations into the pool: no inserts until reset
    DevBuf tbm;      // sepo_run_text: start bits of declined words that did not fit the prepared list
    DevBuf eprog;    // overlapped gather eviction: per-warp progress of evict_copy_prog_kernel
    DevBuf evl;      // overlapped gather eviction: its own copy of the evict list (the next eviction's
                     // classify rewrites d.evict_list while the gather may still be reading it)
    // cuStreamWriteValue32 (driver entry point): the copy stream publishes eviction progress
    int (*write_value32)(cudaStream_t, unsigned long long, unsigned int, unsigned int) = nullptr;

    // export storage
    std::vector<uint8_t> x_keys, x_vals;
    std::vector<uint64_t> x_koffs, x_values, x_loffs, x_voffs;
    uint64_t x_nkeys = 0, x_nvals = 0;
};

namespace {
int cuda_check(sepo_table* t, cudaError_t e, const char* what) {
    if (e == cudaSuccess) return 0;
    t->state = ST_BROKEN;
    return fail(SEPO_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
#define CK(t, expr)                                              \
    do {                                                         \
        int _rc = cuda_check((t), (cudaError_t)(expr), #expr);   \
        if (_rc) return _rc;                                     \
    } while (0)

uint8_t* arena_alloc(sepo_table* t, size_t bytes) {
    for (auto& c : t->arena)
        if (c.cap - c.used >= bytes) {
            uint8_t* p = c.p + c.used;
            c.used += (bytes + 255) & ~(size_t)255;
            if (c.used > c.cap) c.used = c.cap;
            return p;
        }
    PinChunk c;
    c.cap = std::max<size_t>(bytes, (size_t)256 << 20);
    if (cudaHostAlloc((void**)&c.p, c.cap, cudaHostAllocDefault) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    c.used = (bytes + 255) & ~(size_t)255;
    if (c.used > c.cap) c.used = c.cap;
    t->arena.push_back(c);
    return c.p;
}

int check_active(sepo_table* t) {
    if (!t) return fail(SEPO_E_INVAL, "null table");
    if (t->state == ST_BROKEN) return fail(SEPO_E_CUDA, "table is broken by an earlier CUDA error");
    if (t->state == ST_EXPORTED) return fail(SEPO_E_STATE, "table already exported (sepo_reset to reuse)");
    if (t->lookup_done) return fail(SEPO_E_STATE, "table was probed by sepo_lookup (sepo_reset to insert again)");
    return 0;
}

int make_batch(sepo_table* t, Batch& b, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals, const uint64_t* vo,
               uint64_t n, uint32_t* bitmap) {
    b.keys = keys;
    b.ko = ko;
    b.kw = t->opts.fixed_key_width;
    b.vals = vals;
    b.vo = vo;
    b.vw = t->opts.fixed_val_width;
    b.n = n;
    b.bitmap = bitmap;
    b.idx = nullptr;
    if (n == 0) return 0;
    if (n > (1ull << 36)) return fail(SEPO_E_INVAL, "more than 2^36 records in one batch");
    if (!keys && !(ko == nullptr && b.kw == 0)) return fail(SEPO_E_INVAL, "keys is NULL");
    if (!ko && b.kw == 0) return fail(SEPO_E_INVAL, "key_offsets is NULL and fixed_key_width is 0");
    if (t->opts.mode != SEPO_GROUP) {
        if (vo) return fail(SEPO_E_INVAL, "COMBINE/BASIC mode takes fixed-width values (val_offsets must be NULL)");
        if (vals && !(b.vw == 1 || b.vw == 2 || b.vw == 4 || b.vw == 8))
            return fail(SEPO_E_INVAL, "COMBINE fixed_val_width must be 1, 2, 4 or 8");
        if (vals && ((uintptr_t)vals % b.vw)) return fail(SEPO_E_INVAL, "vals not aligned to fixed_val_width");
    } else {
        if (!vals) return fail(SEPO_E_INVAL, "GROUP mode needs values");
        if (!vo && (b.vw == 0 || b.vw > 256)) return fail(SEPO_E_INVAL, "GROUP fixed_val_width must be in 1..256");
    }
    return 0;
}

void sync_dev(sepo_table* t) { t->d.batch_seq = t->batch_seq; }

int read_ctrl(sepo_table* t) {
    CK(t, cudaMemcpyAsync(t->h_ctrl, t->d.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, t->stream));
    CK(t, cudaStreamSynchronize(t->stream));
    return 0;
}
int zero_ctrl_counters(sepo_table* t) {
    // postponed, toolarge, dead_bytes, kept_key_bytes, kept_val_bytes (fields 1..5)
    CK(t, cudaMemsetAsync(&t->d.ctrl->postponed, 0, 5 * sizeof(unsigned long long), t->stream));
    CK(t, cudaMemsetAsync(&t->d.ctrl->next_group, 0, sizeof(unsigned long long), t->stream));  // (GROUP schedule)
    return 0;
}

double elapsed_ms(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
}

int init_device_state(sepo_table* t) {
    CK(t, cudaMemsetAsync(t->d.dir, 0, t->n_buckets * 4, t->stream));
    CK(t, cudaMemsetAsync(t->d.ann, 0, kMaxGrid * ANN_STRIDE * 8, t->stream));
    int rc = sepo_launch_init(t->d, (uint32_t)kMaxGrid, t->stream);  // every cursor slot, whatever the grid
    if (rc) return cuda_check(t, (cudaError_t)rc, "init kernel");
    t->st.kernel_launches += 1;
    t->d.n_free = t->n_pages;
    t->d.n_safe = t->n_pages;
    t->d.eprog = nullptr;
    t->d.gen = 0;
    CK(t, cudaStreamSynchronize(t->stream));
    return 0;
}
}  // namespace

// (exported functions get C linkage from their declarations in sepo.h)

const char* sepo_last_error(void) { return g_err.c_str(); }
const char* sepo_version(void) { return "sepo-b200 0.1 (sm_100a)"; }

static size_t al256(size_t x) { return (x + 255) & ~(size_t)255; }
static size_t fixed_bytes(uint64_t n_buckets) {
    return al256(n_buckets * 4) + al256(sizeof(Ctrl)) + al256(kMaxGrid * 2 * 8) + al256(kMaxGrid * ANN_STRIDE * 8);
}
static const size_t kPerPageMeta = 4 + 1 + 1 + 4;  // stack, page_state, retain, evict_list

size_t sepo_budget_for(uint64_t n_buckets, uint32_t page_bytes, uint64_t pool_pages) {
    return fixed_bytes(n_buckets) + 4 * 256 + (size_t)page_bytes + pool_pages * ((size_t)page_bytes + kPerPageMeta) + 4096;
}

sepo_table* sepo_create(size_t budget, uint64_t n_buckets, uint32_t page_bytes) {
    return sepo_create_placed(budget, n_buckets, page_bytes, SEPO_POOL_DEVICE);
}

sepo_table* sepo_create_placed(size_t budget, uint64_t n_buckets, uint32_t page_bytes, int placement) {
    if (placement != SEPO_POOL_DEVICE && placement != SEPO_POOL_HOST_PINNED && placement != SEPO_POOL_MANAGED) {
        fail(SEPO_E_INVAL, "unknown pool placement");
        return nullptr;
    }
    if (n_buckets == 0 || n_buckets > 0xffffffffull) { fail(SEPO_E_INVAL, "n_buckets must be in [1, 2^32-1]"); return nullptr; }
    if (page_bytes < 4096 || page_bytes > (4u << 20) || (page_bytes & (page_bytes - 1))) {
        fail(SEPO_E_INVAL, "page_bytes must be a power of two in [4 KiB, 4 MiB]");
        return nullptr;
    }
    auto* t = new sepo_table();
    cudaGetDevice(&t->device);
    cudaDeviceGetAttribute(&t->n_sms, cudaDevAttrMultiProcessorCount, t->device);
    t->budget = budget;
    t->n_buckets = n_buckets;
    t->page_bytes = page_bytes;
    t->page_shift = 0;
    while ((1u << t->page_shift) < page_bytes) ++t->page_shift;
    t->grid = sepo_default_grid(SEPO_COMBINE_SUM_U64, t->n_sms);
    t->opts.mode = SEPO_COMBINE_SUM_U64;
    t->opts.fixed_val_width = 8;
    t->opts.fail_until_pass = 16;
    // carve: dir | ctrl | cursors | stack | page_state | retain | evict_list | (align) pool
    auto al = al256;
    const size_t max_grid = kMaxGrid;
    size_t fixed = fixed_bytes(n_buckets);
    if (budget <= fixed + 4 * (size_t)page_bytes) {
        fail(SEPO_E_NOMEM, "device budget too small for the directory + 4 pages");
        delete t;
        return nullptr;
    }
    size_t per_page = (size_t)page_bytes + kPerPageMeta;
    size_t np = (budget - fixed - 4 * 256 - page_bytes) / per_page;
    if (np > ((size_t)32 << 30) / page_bytes) np = ((size_t)32 << 30) / page_bytes;  // 32 GiB pool limit (u32 refs)
    if (np < 4) {
        fail(SEPO_E_NOMEM, "device budget too small for 4 pages");
        delete t;
        return nullptr;
    }
    t->n_pages = (uint32_t)np;
    t->placement = placement;
    // DEVICE: one allocation of exactly the budget. HOST_PINNED / MANAGED (residency ablations,
    // P:L263-303): directory, control words and page metadata stay in HBM (the paper keeps "everything
    // else" on the GPU); only the page pool moves to pinned host memory mapped into the
    // device address space (every table access crosses the host link) or to managed memory
    // (pages migrate on demand by the hardware paging mechanism).
    const size_t meta_end = fixed + al256(np * 4) + 2 * al256(np) + al256(np * 4) + 4 * 256;
    const size_t dev_bytes = placement == SEPO_POOL_DEVICE ? budget : meta_end;
    if (cudaMalloc((void**)&t->region, dev_bytes) != cudaSuccess) {
        cudaGetLastError();
        fail(SEPO_E_NOMEM, "cudaMalloc of the device budget failed");
        delete t;
        return nullptr;
    }
    uint8_t* pool_base = nullptr;  // non-device pool: page_bytes-aligned start inside t->pool_alloc
    if (placement != SEPO_POOL_DEVICE) {
        const size_t pool_bytes = np * (size_t)page_bytes + page_bytes;
        cudaError_t e;
        if (placement == SEPO_POOL_HOST_PINNED) {
            e = cudaHostAlloc((void**)&t->pool_alloc, pool_bytes, cudaHostAllocMapped);
            uint8_t* dp = nullptr;
            if (e == cudaSuccess) e = cudaHostGetDevicePointer((void**)&dp, t->pool_alloc, 0);
            if (e == cudaSuccess) t->pool_dev = dp;
        } else {
            e = cudaMallocManaged((void**)&t->pool_alloc, pool_bytes, cudaMemAttachGlobal);
            t->pool_dev = t->pool_alloc;
        }
        if (e != cudaSuccess) {
            cudaGetLastError();
            fail(SEPO_E_NOMEM, "pool allocation (host pinned / managed) failed");
            sepo_destroy(t);
            return nullptr;
        }
        pool_base = (uint8_t*)(((uintptr_t)t->pool_dev + page_bytes - 1) & ~(uintptr_t)(page_bytes - 1));
    }
    uint8_t* p = t->region;
    Dev& d = t->d;
    d.dir = (uint32_t*)p; p += al(n_buckets * 4);
    d.ctrl = (Ctrl*)p; p += al(sizeof(Ctrl));
    d.cursors = (unsigned long long*)p; p += al(max_grid * 2 * 8);
    d.ann = (unsigned long long*)p; p += al(max_grid * ANN_STRIDE * 8);
    d.stack = (uint32_t*)p; p += al(np * 4);
    d.page_state = p; p += al(np);
    d.retain = p; p += al(np);
    d.evict_list = (uint32_t*)p; p += al(np * 4);
    uintptr_t pa = ((uintptr_t)p + page_bytes - 1) & ~(uintptr_t)(page_bytes - 1);
    if (pool_base) pa = (uintptr_t)pool_base;
    else if (pa + np * (size_t)page_bytes > (uintptr_t)t->region + budget) {
        // alignment ate a page
        --np;
        t->n_pages = (uint32_t)np;
    }
    d.pool = (uint8_t*)pa;
    d.n_slots = (uint32_t)t->grid;
    d.n_buckets = n_buckets;
    d.page_bytes = page_bytes;
    d.page_shift = t->page_shift;
    d.n_pages = t->n_pages;
    d.seed = 0x5e9053eedull;
    d.fail_until = 16;
    cudaStreamCreateWithFlags(&t->stream, cudaStreamNonBlocking);
    t->own_stream = true;
    cudaStreamCreateWithFlags(&t->copy_stream, cudaStreamNonBlocking);
    cudaEventCreate(&t->ev0);
    cudaEventCreate(&t->ev1);
    cudaEventCreate(&t->evc0);
    cudaEventCreate(&t->evc1);
    cudaEventCreateWithFlags(&t->ev_copy, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&t->ev_comp, cudaEventDisableTiming);
    cudaHostAlloc((void**)&t->h_ctrl, sizeof(Ctrl), cudaHostAllocDefault);
    cudaHostAlloc((void**)&t->h_evict, (size_t)t->n_pages * 4, cudaHostAllocDefault);
    cudaHostAlloc((void**)&t->h_ko, 64, cudaHostAllocDefault);
    if (cudaGetLastError() != cudaSuccess || !t->h_ctrl || !t->h_evict) {
        fail(SEPO_E_CUDA, "stream/event/pinned allocation failed");
        sepo_destroy(t);
        return nullptr;
    }
    t->st.n_buckets = n_buckets;
    t->st.page_bytes = page_bytes;
    t->st.pool_pages = t->n_pages;
    t->st.grid_ctas = t->grid;
    if (init_device_state(t)) {
        sepo_destroy(t);
        return nullptr;
    }
    // stream memory operations for the eviction/next-pass overlap (a10); probed once on the
    // table's own control block — without them every eviction is waited for
    {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q{};
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &fn, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess && fn) {
            auto wv = reinterpret_cast<int (*)(cudaStream_t, unsigned long long, unsigned int, unsigned int)>(fn);
            if (wv(t->copy_stream, (unsigned long long)(uintptr_t)&t->d.ctrl->copied, 0u, 0u) == 0 &&
                cudaStreamSynchronize(t->copy_stream) == cudaSuccess)
                t->write_value32 = wv;
        }
        cudaGetLastError();
    }
    return t;
}

int sepo_configure(sepo_table* t, const sepo_options* o) {
    int rc = check_active(t);
    if (rc) return rc;
    if (!o) return fail(SEPO_E_INVAL, "null options");
    if (t->inserted) return fail(SEPO_E_STATE, "configure only before the first insert (or after sepo_reset)");
    if (o->mode != SEPO_COMBINE_SUM_U64 && o->mode != SEPO_GROUP && o->mode != SEPO_BASIC)
        return fail(SEPO_E_INVAL, "unknown mode");
    if (o->basic_halt_pct > 100) return fail(SEPO_E_INVAL, "basic_halt_pct must be <= 100");
    if (o->fixed_key_width > 65535u - 64u) return fail(SEPO_E_INVAL, "fixed_key_width too large");
    if (o->grid_ctas > 1024) return fail(SEPO_E_INVAL, "grid_ctas must be <= 1024");
    sepo_options n = *o;
    if (n.mode != SEPO_GROUP && n.fixed_val_width == 0) n.fixed_val_width = 8;
    if (n.basic_halt_pct == 0) n.basic_halt_pct = 50;
    if (n.fail_until_pass == 0) n.fail_until_pass = 16;
    if (n.grid_ctas == 0) n.grid_ctas = (uint32_t)sepo_default_grid(n.mode, t->n_sms);
    t->grid = (int)n.grid_ctas;
    t->d.n_slots = (uint32_t)t->grid;
    t->st.grid_ctas = t->grid;
    if (n.stream) {
        if (t->own_stream && t->stream) cudaStreamDestroy(t->stream);
        t->stream = (cudaStream_t)n.stream;
        t->own_stream = false;
    }
    t->opts = n;
    t->d.seed = n.hash_seed ^ 0x5e9053eedull;
    t->d.fail_ppm = n.fail_alloc_ppm;
    t->d.fail_mode = n.fail_mode;
    t->d.fail_until = n.fail_until_pass;
    if (n.host_arena_bytes) {
        size_t have = 0;
        for (auto& c : t->arena) have += c.cap;
        if (have < n.host_arena_bytes) {
            PinChunk c;
            c.cap = n.host_arena_bytes - have;
            if (cudaHostAlloc((void**)&c.p, c.cap, cudaHostAllocDefault) != cudaSuccess) {
                cudaGetLastError();
                return fail(SEPO_E_NOMEM, "pinned host arena allocation failed");
            }
            t->arena.push_back(c);
        }
    }
    t->configured_once = true;
    return 0;
}

// SEPO_TRACE=1: host timestamps of the engine's phases on stderr (diagnostics only)
static void trace(const char* what, uint64_t x = 0) {
    static const bool on = [] { const char* e = getenv("SEPO_TRACE"); return e && e[0] == '1'; }();
    if (!on) return;
    static auto t0 = std::chrono::steady_clock::now();
    const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    fprintf(stderr, "[sepo %10.3f ms] %s %llu\n", ms, what, (unsigned long long)x);
}

// Tables whose resident generation exceeds L2: queued misses' directory lines are prefetched into
// L2 while they wait (measured: helps when directory + entries live in HBM, hurts when a generation
// fits L2). The resident footprint is the directory plus the pages the generation can hold —
// min(pool, pages the previous job used at most) — not the budget, which may be all free HBM
// (P:L101). SEPO_DIR_PF=0/1 forces the choice (read on every call).
static bool dir_prefetch(sepo_table* t) {
    const char* e = getenv("SEPO_DIR_PF");
    if (e && (e[0] == '0' || e[0] == '1')) return e[0] == '1';
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device);
    uint64_t pages = t->n_pages;
    if (t->last_job_pages) pages = std::min<uint64_t>(pages, t->last_job_pages);
    return (uint64_t)t->n_buckets * 4 + pages * (uint64_t)t->page_bytes > (uint64_t)l2;
}

// An insert pass over one batch, split so a caller can overlap other work with the kernel:
// insert_begin enqueues it on t->stream without a host sync (key_begin / key_end = ko[0], ko[n]
// for contiguous CSR batches, known to the caller), insert_end waits for it and reads the counters.
struct InsertLaunch {
    bool hot_built = false;
    uint64_t key_bytes = 0;
};
static int insert_begin(sepo_table* t, const Batch& b, uint64_t key_begin, uint64_t key_end, InsertLaunch& L);
static int64_t insert_end(sepo_table* t, const Batch& b, const InsertLaunch& L);

static int64_t insert_impl(sepo_table* t, const Batch& b) {
    if (b.n == 0) return 0;
    uint64_t key_end = 0, key_begin = 0;
    if (b.ko && !b.idx) {  // the end of the batch's key bytes, a kernel parameter (see the kernel)
        CK(t, cudaMemcpyAsync(&t->h_ko[0], b.ko, 8, cudaMemcpyDeviceToHost, t->stream));
        CK(t, cudaMemcpyAsync(&t->h_ko[1], b.ko + b.n, 8, cudaMemcpyDeviceToHost, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
        key_begin = t->h_ko[0];
        key_end = t->h_ko[1];
    }
    InsertLaunch L;
    int rc = insert_begin(t, b, key_begin, key_end, L);
    if (rc) return rc;
    return insert_end(t, b, L);
}

static int insert_begin(sepo_table* t, const Batch& b, uint64_t key_begin, uint64_t key_end, InsertLaunch& L) {
    int rc;
    const uint64_t n = b.n;
    trace("insert begin", n);
    if (!b.bitmap) return fail(SEPO_E_INVAL, "postponed_bitmap is NULL");
    t->inserted = true;
    t->dirty = true;
    ++t->batch_seq;
    sync_dev(t);
    if ((rc = zero_ctrl_counters(t))) return rc;
    CK(t, cudaEventRecord(t->ev0, t->stream));
    if (t->hot.grow(sepo_hot_scratch_bytes())) return fail(SEPO_E_NOMEM, "hot-set scratch");
    // BASIC halt rule: the pass stops once this many allocator slots failed
    const uint32_t halt_slots = (uint32_t)std::max<uint64_t>(1, ((uint64_t)t->grid * t->opts.basic_halt_pct + 99) / 100);
    if (b.idx) L.key_bytes = t->pending_idx_key_bytes;
    else L.key_bytes = b.ko ? key_end - key_begin : n * (uint64_t)t->opts.fixed_key_width;
    // COMBINE pass 1 on contiguous input: the lean kernel unless the keys are long on average (URLs:
    // insert_stream_kernel's warp-window loads suit them better); SEPO_LEAN=0/1 forces the choice
    bool lean_in = false, long_keys = false;
    if (t->opts.mode == SEPO_COMBINE_SUM_U64 && !b.idx) {
        const char* e = getenv("SEPO_LEAN");
        const uint64_t mean = b.ko ? (key_end - key_begin) / n : t->opts.fixed_key_width;
        // (measured: the lean path wins when the generation is L2-resident and the kernel is
        // issue-bound — C2 4x pass 1 21.2 -> 19.6 ms — and loses ~1.4 % when table accesses go to
        // HBM, where insert_stream_kernel's chunk-interleaved stream keeps fewer L1/L2 lines busy)
        // (in budget, CSR words: lean 21.5 vs stream 21.9 ms with the 4x directory; fixed-width pairs in
        // HBM-resident tables keep the stream kernel: C5u 4x pass 1 147 vs 156 ms, profiles/r02/var_r5.jsonl)
        lean_in = (e && (e[0] == '0' || e[0] == '1')) ? e[0] == '1' : (mean <= 24 && (b.ko || !dir_prefetch(t)));
        const char* el = getenv("SEPO_LONG");
        long_keys = b.ko && ((el && (el[0] == '0' || el[0] == '1')) ? el[0] == '1' : mean > 24);
    }
    rc = sepo_launch_insert(t->d, b, t->opts.mode, t->grid, t->stream, t->hot.p, halt_slots, key_end, dir_prefetch(t),
                            &L.hot_built, lean_in, long_keys);
    if (rc) return cuda_check(t, (cudaError_t)rc, "insert kernel launch");
    CK(t, cudaEventRecord(t->ev1, t->stream));
    t->h_ko[2] = 0;
    if (L.hot_built)
        CK(t, cudaMemcpyAsync(&t->h_ko[2], (uint8_t*)t->hot.p + sepo_hot_count_offset(), 4, cudaMemcpyDeviceToHost,
                              t->stream));
    t->st.kernel_launches += (n >= (8ull << 18)) ? 7 : 1;
    return 0;
}

static int64_t insert_end(sepo_table* t, const Batch& b, const InsertLaunch& L) {
    int rc;
    const uint64_t n = b.n;
    if ((rc = read_ctrl(t))) return rc;
    t->st.hot_keys = std::max<uint64_t>(t->st.hot_keys, t->h_ko[2]);
    t->last_insert_ms = elapsed_ms(t->ev0, t->ev1);
    trace("insert end", t->h_ctrl->postponed);
    t->st.t_insert_ms += t->last_insert_ms;
    if (t->st.passes < SEPO_MAX_PASS_STATS) t->st.t_insert_ms_per_pass[t->st.passes] += t->last_insert_ms;
    t->st.insert_calls++;
    t->st.records_inserted += n;
    t->st.key_bytes_inserted += L.key_bytes;
    t->st.val_bytes_inserted += b.vals ? n * (uint64_t)t->opts.fixed_val_width : 0;
    t->st.dead_bytes += t->h_ctrl->dead_bytes;
    const uint64_t used = std::min<uint64_t>(t->h_ctrl->pool_taken, t->d.n_free) + t->pages_resident_retained;
    t->st.pages_used_max = std::max<uint64_t>(t->st.pages_used_max, used);
    if (t->h_ctrl->toolarge) {
        t->st.toolarge += t->h_ctrl->toolarge;
        return fail(SEPO_E_TOOLARGE, std::to_string(t->h_ctrl->toolarge) + " record(s) cannot fit in one page");
    }
    return (int64_t)t->h_ctrl->postponed;
}

// A reinsert pass of sepo_run (COMBINE): the prepared records of the previous pass (a9).
static int64_t reinsert_impl(sepo_table* t, const Batch& b, uint64_t key_bytes, uint64_t records) {
    int rc;
    if (b.n == 0) return 0;
    trace("reinsert begin", records);
    t->inserted = true;
    t->dirty = true;
    ++t->batch_seq;
    sync_dev(t);
    if ((rc = zero_ctrl_counters(t))) return rc;
    CK(t, cudaEventRecord(t->ev0, t->stream));
    const char* el = getenv("SEPO_LONG");
    const bool long_keys = (el && (el[0] == '0' || el[0] == '1')) ? el[0] == '1' : key_bytes > 24 * records;
    rc = sepo_launch_reinsert(t->d, b, t->grid, t->stream, long_keys);
    if (rc) return cuda_check(t, (cudaError_t)rc, "reinsert kernel launch");
    CK(t, cudaEventRecord(t->ev1, t->stream));
    t->st.kernel_launches += 1;
    if ((rc = read_ctrl(t))) return rc;
    t->last_insert_ms = elapsed_ms(t->ev0, t->ev1);
    t->st.t_insert_ms += t->last_insert_ms;
    if (t->st.passes < SEPO_MAX_PASS_STATS) t->st.t_insert_ms_per_pass[t->st.passes] += t->last_insert_ms;
    t->st.insert_calls++;
    trace("reinsert end", t->h_ctrl->postponed);
    t->st.records_inserted += records;
    t->st.key_bytes_inserted += key_bytes;
    t->st.dead_bytes += t->h_ctrl->dead_bytes;
    const uint64_t used = std::min<uint64_t>(t->h_ctrl->pool_taken, t->d.n_free) + t->pages_resident_retained;
    t->st.pages_used_max = std::max<uint64_t>(t->st.pages_used_max, used);
    return (int64_t)t->h_ctrl->postponed;
}

int64_t sepo_insert_batch(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals, const uint64_t* vo,
                          uint64_t n, uint32_t* bitmap) {
    int rc = check_active(t);
    if (rc) return rc;
    Batch b;
    rc = make_batch(t, b, keys, ko, vals, vo, n, bitmap);
    if (rc) return rc;
    return insert_impl(t, b);
}

static int64_t count_or_probe(sepo_table* t, const Batch& b, int probe, uint64_t* kb, uint64_t* vb) {
    int rc;
    if (kb) *kb = 0;
    if (vb) *vb = 0;
    const uint64_t n = b.n;
    if (n == 0) return 0;
    if (!b.bitmap) return fail(SEPO_E_INVAL, "bitmap is NULL");
    const uint64_t nt = sepo_reprobe_tiles(n);
    if (t->tile_counts.grow(nt * 3 * 8)) return fail(SEPO_E_NOMEM, "tile count scratch");
    sync_dev(t);
    if ((rc = zero_ctrl_counters(t))) return rc;
    // COMBINE re-probe and every count-only pass never allocate: use a full-occupancy grid.
    // GROUP re-probe allocates value chunks, so it runs on the allocator slots (one per CTA).
    const int rgrid = (probe && t->opts.mode == SEPO_GROUP) ? t->grid : 8 * t->n_sms;
    // BASIC: nothing to re-probe (a postponed pair left nothing in the table): count only
    rc = sepo_launch_reprobe(t->d, b, t->opts.mode == SEPO_BASIC ? SEPO_COMBINE_SUM_U64 : t->opts.mode,
                             t->opts.mode == SEPO_BASIC ? 0 : probe, rgrid, (unsigned long long*)t->tile_counts.p,
                             t->stream);
    t->st.kernel_launches += 1;
    if (rc) return cuda_check(t, (cudaError_t)rc, "reprobe kernel launch");
    if ((rc = read_ctrl(t))) return rc;
    if (kb) *kb = t->h_ctrl->kept_key_bytes;
    if (vb) *vb = t->h_ctrl->kept_val_bytes;
    return (int64_t)t->h_ctrl->postponed;
}

// a8 for one batch. COMBINE declines are certified inside the insert kernel (R15), so this is a
// recount — except under record-mode fault injection, whose declines are not monotone per key.
// GROUP re-probes every postponed record (its value may fit now; pending keys).
static int64_t reprobe_impl(sepo_table* t, const Batch& b, uint64_t* kb, uint64_t* vb) {
    CK(t, cudaEventRecord(t->ev0, t->stream));
    const bool record_injection = t->opts.fail_alloc_ppm && t->opts.fail_mode == 1;
    const int probe = (t->opts.mode == SEPO_GROUP || record_injection) ? 1 : 0;
    int64_t r = count_or_probe(t, b, probe, kb, vb);
    if (r < 0) return r;
    CK(t, cudaEventRecord(t->ev1, t->stream));
    CK(t, cudaEventSynchronize(t->ev1));
    t->st.t_reprobe_ms += elapsed_ms(t->ev0, t->ev1);
    const uint64_t pass = t->st.passes;
    if (pass < SEPO_MAX_PASS_STATS) t->st.postponed_per_pass[pass] += (uint64_t)r;
    return r;
}

int64_t sepo_reprobe(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals, const uint64_t* vo,
                     uint64_t n, uint32_t* bitmap, uint64_t* kb, uint64_t* vb) {
    int rc = check_active(t);
    if (rc) return rc;
    Batch b;
    rc = make_batch(t, b, keys, ko, vals, vo, n, bitmap);
    if (rc) return rc;
    return reprobe_impl(t, b, kb, vb);
}

int64_t sepo_compact(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals, const uint64_t* vo,
                     uint64_t n, const uint32_t* bitmap, uint8_t* ok, uint64_t* oko, uint8_t* ov, uint64_t* ovo) {
    int rc = check_active(t);
    if (rc) return rc;
    Batch b;
    rc = make_batch(t, b, keys, ko, vals, vo, n, const_cast<uint32_t*>(bitmap));
    if (rc) return rc;
    CK(t, cudaEventRecord(t->ev0, t->stream));
    uint64_t kb = 0, vb = 0;
    int64_t m = count_or_probe(t, b, 0, &kb, &vb);
    if (m < 0) return m;
    if (m > 0 && (!ok || (ko && !oko) || (vals && !ov) || (vo && !ovo)))
        return fail(SEPO_E_INVAL, "compaction output buffer is NULL");
    rc = sepo_launch_compact(b, (unsigned long long*)t->tile_counts.p, ok, oko, ov, ovo, (uint64_t)m, kb, vb,
                             8 * t->n_sms, t->stream);
    if (rc) return cuda_check(t, (cudaError_t)rc, "compact kernel launch");
    t->st.kernel_launches += sepo_reprobe_tiles(n) ? 3 : 1;
    CK(t, cudaEventRecord(t->ev1, t->stream));
    CK(t, cudaEventSynchronize(t->ev1));
    t->st.t_compact_ms += elapsed_ms(t->ev0, t->ev1);
    return m;
}

// a9 by index (sepo_run): the postponed records of batch b as indices into the original arrays
static int64_t compact_index_impl(sepo_table* t, const Batch& b, uint64_t m, uint64_t* idx_out) {
    int rc;
    CK(t, cudaEventRecord(t->evc0, t->stream));
    rc = sepo_launch_compact_index(b, (unsigned long long*)t->tile_counts.p, idx_out, 8 * t->n_sms, t->stream);
    if (rc) return cuda_check(t, (cudaError_t)rc, "compact_index kernel launch");
    t->st.kernel_launches += 2;
    CK(t, cudaEventRecord(t->evc1, t->stream));
    CK(t, cudaEventSynchronize(t->evc1));
    t->st.t_compact_ms += elapsed_ms(t->evc0, t->evc1);
    return (int64_t)m;
}

// Pass boundary. honor_retain = 0 evicts every resident page (final export / forced).
// `overlap` (optional) enqueues compute-stream work that does not touch the pool (the re-issue
// compaction): it runs while the evicted pages stream to host memory on the copy stream (a10).
static int64_t evict_impl(sepo_table* t, int honor_retain, const std::function<int()>& overlap = nullptr) {
    trace("evict begin", t->st.passes);
    CK(t, cudaEventRecord(t->ev0, t->stream));
    sync_dev(t);
    int rc = sepo_launch_seal(t->d, (uint32_t)t->grid, t->stream);
    if (rc) return cuda_check(t, (cudaError_t)rc, "seal kernel");
    rc = sepo_launch_classify(t->d, honor_retain, t->stream);
    if (rc) return cuda_check(t, (cudaError_t)rc, "classify kernel");
    CK(t, cudaMemsetAsync(&t->d.ctrl->full, 0, sizeof(unsigned long long), t->stream));
    CK(t, cudaMemsetAsync(&t->d.ctrl->failed_slots, 0, sizeof(unsigned int), t->stream));
    CK(t, cudaMemsetAsync(t->d.ann, 0, kMaxGrid * ANN_STRIDE * 8, t->stream));
    t->st.kernel_launches += 2;
    // the previous eviction's copies (and its writes of ctrl->copied) are done before the reset
    CK(t, cudaStreamWaitEvent(t->stream, t->ev_copy, 0));
    CK(t, cudaMemsetAsync(&t->d.ctrl->copied, 0, sizeof(unsigned int), t->stream));
    constexpr int kGatherCtas = 16;  // overlapped gather: a few SMs saturate the host link
    const uint32_t gather_warps = kGatherCtas * 512 / 32;
    if (t->eprog.grow(gather_warps * 4)) return fail(SEPO_E_NOMEM, "eviction progress");
    CK(t, cudaMemsetAsync(t->eprog.p, 0, gather_warps * 4, t->stream));
    t->d.eprog = nullptr;
    if ((rc = read_ctrl(t))) return rc;
    const uint64_t ne = t->h_ctrl->n_evict;
    if (ne) {
        CK(t, cudaMemcpyAsync(t->h_evict, t->d.evict_list, ne * 4, cudaMemcpyDeviceToHost, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
    }
    // page copies on the copy stream, ordered after the compute stream (event). With stream
    // memory operations available, the copy stream publishes its progress (pages copied, in
    // evict-list order) in ctrl->copied after every chunk and the next pass starts at once: its
    // allocator takes the never-used pages first and waits for an evicted page's copy before
    // reusing it ("pages are copied to CPU memory" — overlapped with the next pass).
    if (ne) {  // the gather kernel's own copy of the list, taken in stream order before the next
               // eviction's classify can rewrite d.evict_list (an overlapped gather may outlive a short pass)
        if (t->evl.grow(ne * 4)) return fail(SEPO_E_NOMEM, "evict list copy");
        CK(t, cudaMemcpyAsync(t->evl.p, t->d.evict_list, ne * 4, cudaMemcpyDeviceToDevice, t->stream));
    }
    CK(t, cudaEventRecord(t->ev_comp, t->stream));
    CK(t, cudaStreamWaitEvent(t->copy_stream, t->ev_comp, 0));
    // eviction overlapped with the next pass (the allocator waits per evicted page): measured
    // worth it when a generation is large (C5u 4x job 86 -> 78 ms with a 192 MB pool), not for a
    // pool inside L2 (C2 4x: 30.5 -> 31.8 ms). Fragmented evict lists (GROUP generations with
    // retained key pages between the evicted ones) overlap through the gather kernel on a few SMs,
    // which publishes per-warp progress (one cudaMemcpyAsync per run with progress: C4 3x 496 ->
    // 708 ms). SEPO_EVICT_OVERLAP=0/1 forces the choice.
    bool want_overlap;
    {
        const char* ov = getenv("SEPO_EVICT_OVERLAP");
        int l2 = 0;
        cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device);
        want_overlap = (ov && (ov[0] == '0' || ov[0] == '1'))
                           ? ov[0] == '1'
                           : (t->opts.mode == SEPO_COMBINE_SUM_U64 || t->opts.mode == SEPO_GROUP) &&
                                 (uint64_t)t->n_pages * t->page_bytes > (uint64_t)l2;
    }
    // Fragmented evict lists (many short runs of consecutive pages) go through one gather-copy
    // kernel into a contiguous host region; long runs through cudaMemcpyAsync (copy engine).
    // SEPO_EVICT_KERNEL=0/1 forces either.
    uint64_t n_runs = 0;
    for (uint64_t i = 0; i < ne; ++i) n_runs += (i == 0 || t->h_evict[i] != t->h_evict[i - 1] + 1);
    const char* eks = getenv("SEPO_EVICT_KERNEL");
    const int ek = eks ? atoi(eks) : -1;
    const bool use_kernel = ne > 0 && (ek == 1 || (ek < 0 && n_runs * 64 > ne));
    const bool gather_ov = use_kernel && want_overlap;
    const bool overlapped = gather_ov || (!use_kernel && t->write_value32 != nullptr && want_overlap);
    GenImage img;
    img.gen = t->d.gen;
    uint64_t bytes = 0, done = 0;
    const uint64_t chunk_pages = overlapped ? std::max<uint64_t>(std::max<uint64_t>(1, (1u << 20) >> t->page_shift), ne / 48)
                                            : ~0ull;  // progress granularity (overlap only)
    if (use_kernel) {
        const size_t nbytes = (size_t)ne << t->page_shift;
        uint8_t* hp = arena_alloc(t, nbytes);
        if (!hp) return fail(SEPO_E_NOMEM, "pinned host arena exhausted");
        uint8_t* dp = nullptr;
        CK(t, cudaHostGetDevicePointer((void**)&dp, hp, 0));
        if (gather_ov) {
            rc = sepo_launch_evict_copy_prog(t->d, (uint32_t)ne, dp, kGatherCtas, (unsigned int*)t->eprog.p,
                                             (const uint32_t*)t->evl.p, t->copy_stream);
            t->d.eprog = (unsigned int*)t->eprog.p;  // (the next pass's allocator waits on it)
            t->d.eprog_n = gather_warps;
        } else {
            rc = sepo_launch_evict_copy(t->d, (uint32_t)ne, dp, 2 * t->n_sms, t->copy_stream);
        }
        if (rc) return cuda_check(t, (cudaError_t)rc, "evict copy kernel");
        t->st.kernel_launches += 1;
        for (uint64_t i = 0; i < ne;) {
            uint64_t j = i + 1;
            while (j < ne && t->h_evict[j] == t->h_evict[j - 1] + 1) ++j;
            img.runs.push_back({t->h_evict[i], (uint32_t)(j - i), hp + (i << t->page_shift)});
            i = j;
        }
        bytes = nbytes;
        done = ne;
    }
    for (uint64_t i = use_kernel ? ne : 0; i < ne;) {
        uint64_t j = i + 1;
        while (j < ne && t->h_evict[j] == t->h_evict[j - 1] + 1) ++j;
        const uint32_t first = t->h_evict[i], cnt = (uint32_t)(j - i);
        const size_t nbytes = (size_t)cnt * t->page_bytes;
        uint8_t* hp = arena_alloc(t, nbytes);
        if (!hp) return fail(SEPO_E_NOMEM, "pinned host arena exhausted");
        for (uint64_t c0 = 0; c0 < cnt; c0 += chunk_pages) {
            const uint64_t cc = std::min<uint64_t>(chunk_pages, cnt - c0);
            CK(t, cudaMemcpyAsync(hp + (c0 << t->page_shift), t->d.pool + ((size_t)(first + c0) << t->page_shift),
                                  (size_t)cc << t->page_shift, cudaMemcpyDefault, t->copy_stream));
            done += cc;
            if (overlapped) {
                const int wr = t->write_value32(t->copy_stream, (unsigned long long)(uintptr_t)&t->d.ctrl->copied,
                                                (unsigned int)done, 0);
                if (wr) return fail(SEPO_E_CUDA, "cuStreamWriteValue32 failed");
            }
        }
        img.runs.push_back({first, cnt, hp});
        bytes += nbytes;
        i = j;
    }
    CK(t, cudaEventRecord(t->ev_copy, t->copy_stream));
    if (overlap) {
        int orc = overlap();
        if (orc) return orc;
    }
    if (overlapped) {
        t->d.n_safe = (uint32_t)t->h_ctrl->n_safe;
    } else {  // the freed pages are reused only after their copy finished
        CK(t, cudaStreamWaitEvent(t->stream, t->ev_copy, 0));
        t->d.n_safe = (uint32_t)t->h_ctrl->n_free;
    }
    CK(t, cudaMemsetAsync(t->d.dir, 0, t->n_buckets * 4, t->stream));
    t->d.n_free = (uint32_t)t->h_ctrl->n_free;
    t->pages_resident_retained = t->h_ctrl->n_resident;
    t->d.gen += 1;
    if (t->opts.mode == SEPO_GROUP && t->pages_resident_retained) {
        rc = sepo_launch_relink(t->d, t->stream);
        if (rc) return cuda_check(t, (cudaError_t)rc, "relink kernel");
        t->st.kernel_launches += 1;
    }
    CK(t, cudaEventRecord(t->ev1, t->stream));
    CK(t, cudaEventSynchronize(t->ev1));
    t->st.t_evict_ms += elapsed_ms(t->ev0, t->ev1);
    trace("evict end", bytes);
    if (!img.runs.empty()) t->gens.push_back(std::move(img));
    t->st.bytes_evicted += bytes;
    t->st.passes += 1;
    t->dirty = t->pages_resident_retained > 0;
    return (int64_t)bytes;
}

int64_t sepo_evict(sepo_table* t) {
    int rc = check_active(t);
    if (rc) return rc;
    return evict_impl(t, 1);
}

// ---------------------------------------------------------------- export (host assembly, a11)
namespace {
struct PageRef {
    const uint8_t* p;
    uint32_t page;
    uint32_t gen;
};

void collect_pages(sepo_table* t, std::vector<PageRef>& pages) {
    for (auto& g : t->gens)
        for (auto& r : g.runs)
            for (uint32_t k = 0; k < r.count; ++k) pages.push_back({r.p + (size_t)k * t->page_bytes, r.first + k, g.gen});
}

template <class F>
void parallel_for(size_t n, F f) {
    unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
    if (n < 64) nt = 1;
    std::vector<std::thread> th;
    for (unsigned w = 0; w < nt; ++w)
        th.emplace_back([&, w] {
            size_t lo = n * w / nt, hi = n * (w + 1) / nt;
            f(w, lo, hi);
        });
    for (auto& x : th) x.join();
}

// COMBINE: one entry per key (merge of cross-generation duplicates as a backstop); BASIC: one
// entry per pair (K_BASIC), duplicates are the result, never merged
int export_combine(sepo_table* t) {
    const uint32_t kind = t->opts.mode == SEPO_BASIC ? K_BASIC : K_COMBINE;
    std::vector<PageRef> pages;
    collect_pages(t, pages);
    const uint32_t PB = t->page_bytes;
    const size_t np = pages.size();
    std::vector<uint64_t> pk(np + 1, 0), pb(np + 1, 0);
    std::atomic<int> bad{0};
    parallel_for(np, [&](unsigned, size_t lo, size_t hi) {
        for (size_t i = lo; i < hi; ++i) {
            uint64_t k = 0, kb = 0;
            uint32_t off = 0;
            const uint8_t* base = pages[i].p;
            while (off < PB) {
                uint32_t hdr;
                memcpy(&hdr, base + off, 4);
                uint32_t sz = hdr & ~KIND_MASK;
                if (sz == 0 || off + sz > PB) { bad = 1; break; }
                if ((hdr & KIND_MASK) == kind) {
                    uint32_t klen;
                    memcpy(&klen, base + off + 12, 4);
                    ++k;
                    kb += klen;
                }
                off += sz;
            }
            pk[i + 1] = k;
            pb[i + 1] = kb;
        }
    });
    if (bad) return fail(SEPO_E_STATE, "corrupt page image during export");
    for (size_t i = 0; i < np; ++i) { pk[i + 1] += pk[i]; pb[i + 1] += pb[i]; }
    const uint64_t nk = pk[np], nkb = pb[np];
    t->x_keys.resize(nkb);
    t->x_koffs.resize(nk + 1);
    t->x_values.resize(nk);
    parallel_for(np, [&](unsigned, size_t lo, size_t hi) {
        for (size_t i = lo; i < hi; ++i) {
            uint64_t k = pk[i], kb = pb[i];
            uint32_t off = 0;
            const uint8_t* base = pages[i].p;
            while (off < PB) {
                uint32_t hdr;
                memcpy(&hdr, base + off, 4);
                uint32_t sz = hdr & ~KIND_MASK;
                if ((hdr & KIND_MASK) == kind) {
                    uint32_t klen;
                    memcpy(&klen, base + off + 12, 4);
                    t->x_koffs[k] = kb;
                    memcpy(&t->x_values[k], base + off + KEY_OFF + ((klen + 7) & ~7u), 8);
                    memcpy(t->x_keys.data() + kb, base + off + KEY_OFF, klen);
                    ++k;
                    kb += klen;
                }
                off += sz;
            }
        }
    });
    t->x_koffs[nk] = nkb;
    t->x_nkeys = nk;
    // keys found in more than one generation (only possible under record-mode fault injection)
    const bool merge = kind == K_COMBINE && (t->opts.check_dups || (t->opts.fail_alloc_ppm && t->opts.fail_mode == 1));
    if (merge && nk) {
        std::unordered_map<std::string_view, uint64_t> idx;
        idx.reserve(nk * 2);
        std::vector<uint8_t> keys2;
        std::vector<uint64_t> offs2, vals2;
        offs2.push_back(0);
        uint64_t dups = 0;
        std::vector<uint64_t> order;
        for (uint64_t k = 0; k < nk; ++k) {
            std::string_view sv((const char*)t->x_keys.data() + t->x_koffs[k], t->x_koffs[k + 1] - t->x_koffs[k]);
            auto it = idx.find(sv);
            if (it == idx.end()) {
                idx.emplace(sv, vals2.size());
                vals2.push_back(t->x_values[k]);
                order.push_back(k);
            } else {
                ++dups;
                vals2[it->second] += t->x_values[k];
            }
        }
        if (dups) {
            for (uint64_t k : order) {
                keys2.insert(keys2.end(), t->x_keys.begin() + t->x_koffs[k], t->x_keys.begin() + t->x_koffs[k + 1]);
                offs2.push_back(keys2.size());
            }
            t->x_keys.swap(keys2);
            t->x_koffs.swap(offs2);
            t->x_values.swap(vals2);
            t->x_nkeys = t->x_values.size();
        }
        t->st.cross_gen_dups = dups;
    }
    return 0;
}

int export_group(sepo_table* t) {
    std::vector<PageRef> pages;
    collect_pages(t, pages);
    const uint32_t PB = t->page_bytes;
    const size_t np = pages.size();
    // pass A: key entries (identity = birth gen << 40 | entry ref) and value chunks
    struct KeyRec { const uint8_t* key; uint32_t len; uint64_t id; };
    // units = used slots (fixed-width values, vw > 0) or used bytes (variable items, vw == 0)
    struct ChunkRec { const uint8_t* vals; uint32_t units; uint64_t owner; uint32_t vw; uint32_t nitems; uint64_t nbytes; };
    std::vector<uint64_t> slots(16, 0);
    std::vector<std::vector<KeyRec>> tk(16);
    std::vector<std::vector<ChunkRec>> tc(16);
    std::atomic<int> bad{0};
    parallel_for(np, [&](unsigned w, size_t lo, size_t hi) {
        for (size_t i = lo; i < hi; ++i) {
            uint32_t off = 0;
            const uint8_t* base = pages[i].p;
            while (off < PB) {
                uint32_t hdr;
                memcpy(&hdr, base + off, 4);
                uint32_t sz = hdr & ~KIND_MASK;
                if (sz == 0 || off + sz > PB) { bad = 1; break; }
                uint32_t kind = hdr & KIND_MASK;
                if (kind == K_GKEY) {
                    uint32_t klen, birth;
                    memcpy(&klen, base + off + 12, 4);
                    memcpy(&birth, base + off + KEY_OFF + ((klen + 7) & ~7u) + 8, 4);
                    uint64_t poolo = ((uint64_t)pages[i].page << t->page_shift) + off;
                    tk[w].push_back({base + off + KEY_OFF, klen, ((uint64_t)birth << 40) | ((poolo >> 3) + 1)});
                } else if (kind == K_VCHUNK || kind == K_VCHUNKV) {
                    // 16-byte header: size | kind, fill, owner; the capacity follows from the size
                    // (fixed-width slots of the table's fixed_val_width, or bytes of variable items)
                    uint32_t fill;
                    uint64_t owner;
                    memcpy(&fill, base + off + 4, 4);
                    memcpy(&owner, base + off + 8, 8);
                    const uint32_t cvw = kind == K_VCHUNK ? t->opts.fixed_val_width : 0u;
                    const uint32_t cap = (sz - CHUNK_HDR) / (cvw ? cvw : 1u);
                    fill &= ~CHUNK_PRIVATE;
                    ChunkRec cr{base + off + CHUNK_HDR, std::min(fill, cap), owner, cvw, 0, 0};
                    if (cvw) {
                        cr.nitems = cr.units;
                        cr.nbytes = (uint64_t)cr.units * cvw;
                    } else {  // variable items {u32 len, bytes, pad4} up to the fill or an end mark
                        uint32_t o = 0;
                        while (o + 4 <= cr.units) {
                            uint32_t l;
                            memcpy(&l, cr.vals + o, 4);
                            if (l == 0xffffffffu || o + 4 + l > cr.units) break;
                            ++cr.nitems;
                            cr.nbytes += l;
                            o += (4 + l + 3) & ~3u;
                        }
                    }
                    tc[w].push_back(cr);
                    slots[w] += cap;
                }
                off += sz;
            }
        }
    });
    if (bad) return fail(SEPO_E_STATE, "corrupt page image during export");
    // key index; keys that appear under several identities (forced full evictions / injection) merge
    std::unordered_map<uint64_t, uint64_t> id2k;
    std::unordered_map<std::string_view, uint64_t> name2k;
    std::vector<const KeyRec*> keys;
    uint64_t dups = 0;
    size_t total = 0;
    for (auto& v : tk) total += v.size();
    id2k.reserve(total * 2);
    name2k.reserve(total * 2);
    for (auto& v : tk)
        for (auto& kr : v) {
            std::string_view sv((const char*)kr.key, kr.len);
            auto it = name2k.find(sv);
            uint64_t k;
            if (it == name2k.end()) { k = keys.size(); name2k.emplace(sv, k); keys.push_back(&kr); }
            else { k = it->second; ++dups; }
            id2k[kr.id] = k;
        }
    t->st.cross_gen_dups = dups;
    t->st.value_chunks = 0;
    t->st.value_slots = 0;
    for (auto& v : tc) t->st.value_chunks += v.size();
    for (auto x : slots) t->st.value_slots += x;
    const uint64_t nk = keys.size();
    std::vector<uint64_t> cnt(nk + 1, 0), byt(nk + 1, 0);
    for (auto& v : tc)
        for (auto& c : v) {
            auto it = id2k.find(c.owner);
            if (it == id2k.end()) return fail(SEPO_E_STATE, "value chunk with unknown owner");
            cnt[it->second + 1] += c.nitems;
            byt[it->second + 1] += c.nbytes;
        }
    for (uint64_t k = 0; k < nk; ++k) { cnt[k + 1] += cnt[k]; byt[k + 1] += byt[k]; }
    const uint64_t nv = cnt[nk];
    t->x_loffs.assign(cnt.begin(), cnt.end());
    t->x_vals.resize(byt[nk]);
    t->x_voffs.resize(nv + 1);
    t->x_voffs[nv] = byt[nk];
    std::vector<uint64_t> cur(cnt.begin(), cnt.end() - 1), curb(byt.begin(), byt.end() - 1);
    for (auto& v : tc)
        for (auto& c : v) {
            const uint64_t k = id2k[c.owner];
            if (c.vw) {
                memcpy(t->x_vals.data() + curb[k], c.vals, (size_t)c.nbytes);
                for (uint32_t j = 0; j < c.nitems; ++j) t->x_voffs[cur[k] + j] = curb[k] + (uint64_t)j * c.vw;
                cur[k] += c.nitems;
                curb[k] += c.nbytes;
            } else {
                uint32_t o = 0;
                for (uint32_t j = 0; j < c.nitems; ++j) {
                    uint32_t l;
                    memcpy(&l, c.vals + o, 4);
                    t->x_voffs[cur[k]++] = curb[k];
                    memcpy(t->x_vals.data() + curb[k], c.vals + o + 4, l);
                    curb[k] += l;
                    o += (4 + l + 3) & ~3u;
                }
            }
        }
    uint64_t kb = 0;
    for (auto* kr : keys) kb += kr->len;
    t->x_keys.resize(kb);
    t->x_koffs.resize(nk + 1);
    kb = 0;
    for (uint64_t k = 0; k < nk; ++k) {
        t->x_koffs[k] = kb;
        memcpy(t->x_keys.data() + kb, keys[k]->key, keys[k]->len);
        kb += keys[k]->len;
    }
    t->x_koffs[nk] = kb;
    t->x_nkeys = nk;
    t->x_nvals = nv;
    return 0;
}
}  // namespace

int sepo_export(sepo_table* t, sepo_result* out) {
    if (!t) return fail(SEPO_E_INVAL, "null table");
    if (t->state == ST_BROKEN) return fail(SEPO_E_CUDA, "table is broken by an earlier CUDA error");
    if (t->state == ST_EXPORTED) return fail(SEPO_E_STATE, "table already exported (sepo_reset to reuse)");
    int rc = 0;  // (allowed after sepo_lookup: export reads the host page images)
    if (!out) return fail(SEPO_E_INVAL, "null result");
    if (t->dirty) {
        int64_t e = evict_impl(t, 0);
        if (e < 0) return (int)e;
    }
    CK(t, cudaStreamSynchronize(t->copy_stream));
    auto t0 = std::chrono::steady_clock::now();
    rc = t->opts.mode == SEPO_GROUP ? export_group(t) : export_combine(t);
    if (rc) return rc;
    t->st.t_export_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    memset(out, 0, sizeof(*out));
    out->n_keys = t->x_nkeys;
    out->keys = t->x_keys.data();
    out->key_offsets = t->x_koffs.data();
    if (t->opts.mode != SEPO_GROUP) {  // COMBINE: one (key, sum) per key; BASIC: one (key, value) per pair
        out->values = t->x_values.data();
    } else {
        out->list_offsets = t->x_loffs.data();
        out->n_vals = t->x_nvals;
        out->vals = t->x_vals.data();
        out->val_offsets = t->x_voffs.data();
    }
    t->state = ST_EXPORTED;
    return 0;
}

// ---------------------------------------------------------------- the whole job
static bool is_device_ptr(const void* p) {
    if (!p) return true;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Prepared re-issue passes (a9) of a COMBINE job: evict, then reinsert the `reserved` slots of
// prep[ps] (m postponed records, kb key bytes) until nothing is postponed. <0 on error.
static int64_t prep_passes(sepo_table* t, const Batch& cur, int ps, uint64_t reserved, uint64_t m, uint64_t kb,
                           uint64_t prb, int64_t passes_start) {
    const uint64_t slack = (uint64_t)t->grid * 32 * kPrepChunk;  // holes: < one chunk per warp
    while (m > 0) {
        const uint64_t pass = t->st.passes;
        if (pass < SEPO_MAX_PASS_STATS) t->st.postponed_per_pass[pass] += m;
        const uint64_t ocap = reserved + slack;  // every record may decline again
        if (t->prep[ps ^ 1].grow(ocap * prb)) return fail(SEPO_E_NOMEM, "prepared re-issue list");
        int64_t e = evict_impl(t, 1);
        if (e < 0) return e;
        Batch pb = cur;
        pb.keys = cur.keys; pb.ko = nullptr; pb.vals = nullptr; pb.vo = nullptr; pb.idx = nullptr;
        pb.bitmap = nullptr;
        pb.text = 0; pb.tbm = nullptr;
        pb.wire = nullptr;
        pb.prep = (const PRec*)t->prep[ps].p;
        pb.n = reserved;
        pb.out = (PRec*)t->prep[ps ^ 1].p;
        pb.out_n = (unsigned long long*)t->prep_n.p + (ps ^ 1);
        pb.out_cap = ocap;
        CK(t, cudaMemsetAsync(pb.out_n, 0, 8, t->stream));
        const int64_t m2 = reinsert_impl(t, pb, kb, m);
        if (m2 < 0) return m2;
        if (t->h_ctrl->toolarge) return fail(SEPO_E_TOOLARGE, "record cannot fit in one page");
        kb = t->h_ctrl->kept_key_bytes;
        m = (uint64_t)m2;
        if (m) {
            CK(t, cudaMemcpyAsync(&t->h_ko[0], pb.out_n, 8, cudaMemcpyDeviceToHost, t->stream));
            CK(t, cudaStreamSynchronize(t->stream));
            reserved = t->h_ko[0];
        }
        if (reserved > ocap) return fail(SEPO_E_STATE, "prepared re-issue list overflow");
        ps ^= 1;
        if (t->st.passes - passes_start > 100000) return fail(SEPO_E_STATE, "no progress");
    }
    return 0;
}

static int64_t run_device(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals,
                          const uint64_t* vo, uint64_t n, const WireRec* wire = nullptr);

int64_t sepo_run(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals, const uint64_t* vo,
                 uint64_t n) {
    trace("run begin", n);
    int rc = check_active(t);
    if (rc) return rc;
    const bool dev = is_device_ptr(keys) && is_device_ptr(ko) && is_device_ptr(vals) && is_device_ptr(vo);
    const uint32_t kw = t->opts.fixed_key_width, vw = t->opts.fixed_val_width;
    // (tests shrink the thresholds: SEPO_H2D_PIPE_MIN records, SEPO_H2D_CHUNK records per chunk)
    const char* pmin = getenv("SEPO_H2D_PIPE_MIN");
    const uint64_t pipe_min = pmin ? strtoull(pmin, nullptr, 10) : (64ull << 20);
    if (!dev && n && t->opts.mode == SEPO_COMBINE_SUM_U64 && ko && !vo && n >= pipe_min && !getenv("SEPO_NO_H2D_PIPE")) {
        // host input, COMBINE: the H2D copy (P:L227 counts this transfer) is pipelined with pass 1 —
        // chunks of records go over the host link on the copy stream while the previous chunk is
        // inserted; the staged copy keeps the caller's absolute offsets
        uint64_t kbytes = 0, vbytes = 0, k0 = 0;
        if (ko) { k0 = ko[0]; kbytes = ko[n] - ko[0]; } else kbytes = n * (uint64_t)kw;
        if (vals) vbytes = n * (uint64_t)vw;
        if (t->in_stage[0].grow(kbytes + 16) || (ko && t->in_stage[1].grow((n + 1) * 8)) ||
            (vals && t->in_stage[2].grow(vbytes + 16)))
            return fail(SEPO_E_NOMEM, "device staging for host input");
        const char* pch = getenv("SEPO_H2D_CHUNK");
        uint64_t per = pch ? strtoull(pch, nullptr, 10) : (32ull << 20);  // records per chunk
        per = std::max<uint64_t>(32, per & ~31ull);                       // a multiple of 32: bitmap words
        const uint64_t nch = (n + per - 1) / per;
        std::vector<cudaEvent_t> evs(nch);
        for (auto& e : evs) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
        cudaEvent_t h0, h1;
        cudaEventCreate(&h0);
        cudaEventCreate(&h1);
        CK(t, cudaEventRecord(h0, t->copy_stream));
        uint8_t* kst = (uint8_t*)t->in_stage[0].p;
        uint64_t* ost = (uint64_t*)t->in_stage[1].p;
        for (uint64_t c = 0; c < nch; ++c) {
            const uint64_t r0 = c * per, r1 = std::min(n, r0 + per);
            const uint64_t b0 = ko ? ko[r0] - k0 : r0 * kw, b1 = ko ? ko[r1] - k0 : r1 * kw;
            CK(t, cudaMemcpyAsync(kst + b0, keys + k0 + b0, b1 - b0, cudaMemcpyHostToDevice, t->copy_stream));
            // r1 - r0 + 1 offsets: the chunk's last key ends at ko[r1] (the next chunk copies it again)
            if (ko) CK(t, cudaMemcpyAsync(ost + r0, ko + r0, (r1 - r0 + 1) * 8, cudaMemcpyHostToDevice, t->copy_stream));
            if (vals) CK(t, cudaMemcpyAsync((uint8_t*)t->in_stage[2].p + r0 * vw, vals + r0 * vw, (r1 - r0) * vw,
                                            cudaMemcpyHostToDevice, t->copy_stream));
            CK(t, cudaEventRecord(evs[c], t->copy_stream));
        }
        CK(t, cudaEventRecord(h1, t->copy_stream));
        t->h2d_chunks = &evs;
        t->h2d_chunk_records = per;
        // (the staged copy is device memory: no second pointer classification — a rebased key base
        // kst - k0 may lie outside every allocation)
        const int64_t r = run_device(t, kst - k0, ko ? ost : nullptr, vals ? (const uint8_t*)t->in_stage[2].p : nullptr,
                                     nullptr, n);
        t->h2d_chunks = nullptr;
        cudaEventSynchronize(h1);
        t->st.t_h2d_ms += elapsed_ms(h0, h1);
        for (auto& e : evs) cudaEventDestroy(e);
        cudaEventDestroy(h0);
        cudaEventDestroy(h1);
        return r;
    }
    if (!dev && n) {
        // host input: stage it in device memory (one H2D per array, P:L227 counts this transfer)
        auto t0 = std::chrono::steady_clock::now();
        uint64_t kbytes = 0, vbytes = 0;
        uint64_t k0 = 0, v0 = 0;
        if (ko) { k0 = ko[0]; kbytes = ko[n] - ko[0]; } else kbytes = n * (uint64_t)kw;
        if (vals) { if (vo) { v0 = vo[0]; vbytes = vo[n] - vo[0]; } else vbytes = n * (uint64_t)vw; }
        if (t->in_stage[0].grow(kbytes + 16) || (ko && t->in_stage[1].grow((n + 1) * 8)) ||
            (vals && t->in_stage[2].grow(vbytes + 16)) || (vo && t->in_stage[3].grow((n + 1) * 8)))
            return fail(SEPO_E_NOMEM, "device staging for host input");
        CK(t, cudaMemcpyAsync(t->in_stage[0].p, keys + k0, kbytes, cudaMemcpyHostToDevice, t->stream));
        if (ko) CK(t, cudaMemcpyAsync(t->in_stage[1].p, ko, (n + 1) * 8, cudaMemcpyHostToDevice, t->stream));
        if (vals) CK(t, cudaMemcpyAsync(t->in_stage[2].p, vals + v0, vbytes, cudaMemcpyHostToDevice, t->stream));
        if (vo) CK(t, cudaMemcpyAsync(t->in_stage[3].p, vo, (n + 1) * 8, cudaMemcpyHostToDevice, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
        t->st.t_h2d_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        // offsets stay absolute: shift the key base so keys[ko[i]] addresses the staged copy
        const uint8_t* kdev = (const uint8_t*)t->in_stage[0].p - k0;
        const uint8_t* vdev = vals ? (const uint8_t*)t->in_stage[2].p - v0 : nullptr;
        return run_device(t, kdev, ko ? (const uint64_t*)t->in_stage[1].p : nullptr, vdev,
                          vo ? (const uint64_t*)t->in_stage[3].p : nullptr, n);
    }
    return run_device(t, keys, ko, vals, vo, n);
}

// sepo_run on device-resident input (the caller's arrays, or the staged copy of host input)
static int64_t run_device(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals,
                          const uint64_t* vo, uint64_t n, const WireRec* wire) {
    trace("run: inputs on device");
    const uint32_t kw = wire ? 0u : t->opts.fixed_key_width;
    Batch cur;
    if (wire) {  // routed records (a12): keys <= 16 bytes with pre-combined u64 values
        cur = Batch{};
        cur.wire = wire;
        cur.n = n;
        cur.vw = 8;
        cur.vals = reinterpret_cast<const uint8_t*>(wire);  // (values present: 48-byte prepared records)
    } else {
        int rc2 = make_batch(t, cur, keys, ko, vals, vo, n, nullptr);
        if (rc2) return rc2;
    }
    int side = 0;
    int64_t passes_start = (int64_t)t->st.passes;
    uint64_t prev = ~0ull;
    // both streaming kernels certify their declines (R15) and mark pending GROUP keys' pages
    // themselves, so the insert's count is exact — except under record-mode injection
    const bool combine_exact = t->opts.mode == SEPO_BASIC || !(t->opts.fail_alloc_ppm && t->opts.fail_mode == 1);
    // COMBINE re-issue in prepared form (a9): the first pass appends each declined record as
    // {hash, first 16 key bytes, key offset, value, length}; later passes read those records
    // densely (no gather through an index list, no re-hash). The first pass's list is sized
    // n/4 (SEPO_PREP_CAP overrides); on overflow the job continues on the index path.
    const char* no_prep = getenv("SEPO_NO_PREP");
    bool use_prep = t->opts.mode == SEPO_COMBINE_SUM_U64 && combine_exact && !(no_prep && no_prep[0] == '1') && n > 0;
    // prepared record bytes: 32 for implicit values, 32 for values with fixed keys of <= 8 bytes
    // (the key is one word: {key, value, hash, offset | length}), else 48
    // (routed wire records carry values: 48-byte records, the format the wire kernel writes)
    const bool short_keys = !wire && !ko && kw > 0 && kw <= 8;
    const bool has_vals = vals != nullptr || wire != nullptr;
    const uint64_t prb = (has_vals && !short_keys) ? sizeof(PRec) : 32;
    cur.prep_rb = (uint32_t)prb;
    cur.prep_fmt = (has_vals && short_keys) ? 33u : 0u;
    if (wire && !use_prep) return fail(SEPO_E_INVAL, "routed records need the prepared re-issue path (COMBINE)");
    if (use_prep) {
        uint64_t cap = std::max<uint64_t>(1ull << 16, n / 4);
        if (const char* pc = getenv("SEPO_PREP_CAP")) cap = strtoull(pc, nullptr, 10);
        if (wire) cap = std::max<uint64_t>(1ull << 16, n);  // (no index re-issue for routed records: never overflow)
        if ((uint64_t)t->prep[0].cap < cap * prb) {  // first use / larger input: bound by free memory
            size_t fr = 0, tot = 0;
            if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) cap = std::min<uint64_t>(cap, (fr + t->prep[0].cap) / 3 / prb);
        }
        if (t->prep_n.grow(64) || t->prep[0].grow(std::max<uint64_t>(cap, 1) * prb)) {
            if (wire) return fail(SEPO_E_NOMEM, "prepared re-issue list for routed records");
            use_prep = false;
        } else {
            CK(t, cudaMemsetAsync(t->prep_n.p, 0, 16, t->stream));
            cur.out = (PRec*)t->prep[0].p;
            cur.out_n = (unsigned long long*)t->prep_n.p;
            cur.out_cap = cap;
        }
    }
    std::vector<cudaEvent_t>* chunks = t->h2d_chunks;  // pass 1 of pipelined host input
    t->h2d_chunks = nullptr;
    while (cur.n > 0) {
        if (t->bm.grow(((cur.n + 31) / 32) * 4)) return fail(SEPO_E_NOMEM, "bitmap scratch");
        cur.bitmap = (uint32_t*)t->bm.p;
        int64_t c = 0;
        uint64_t kb = 0, vb = 0;
        if (chunks) {  // insert each chunk as soon as its copy landed
            const uint64_t per = t->h2d_chunk_records;
            for (size_t k = 0; k < chunks->size(); ++k) {
                CK(t, cudaStreamWaitEvent(t->stream, (*chunks)[k], 0));
                Batch bc = cur;
                const uint64_t r0 = k * per, r1 = std::min(cur.n, r0 + per);
                if (cur.ko) bc.ko = cur.ko + r0;
                else bc.keys = cur.keys + r0 * (uint64_t)cur.kw;
                if (cur.vals) bc.vals = cur.vals + r0 * (uint64_t)cur.vw;
                bc.n = r1 - r0;
                bc.bitmap = cur.bitmap + r0 / 32;
                const int64_t cc = insert_impl(t, bc);
                if (cc < 0) return cc;
                c += cc;
                kb += t->h_ctrl->kept_key_bytes;
            }
            chunks = nullptr;
        } else {
            c = insert_impl(t, cur);
            if (c < 0) return c;
            kb = t->h_ctrl->kept_key_bytes;
        }
        if (c > 0 && !combine_exact) c = reprobe_impl(t, cur, &kb, &vb);
        if (c < 0) return c;
        if (c == 0) break;
        uint64_t reserved = 0;  // prepared slots the pass reserved (records + closed holes)
        if (cur.out) {
            CK(t, cudaMemcpyAsync(&t->h_ko[0], cur.out_n, 8, cudaMemcpyDeviceToHost, t->stream));
            CK(t, cudaStreamSynchronize(t->stream));
            reserved = t->h_ko[0];
        }
        if (cur.out && reserved <= cur.out_cap) {
            // prepared re-issue: reinsert passes until nothing is postponed
            const int64_t r = prep_passes(t, cur, 0, reserved, (uint64_t)c, kb, prb, passes_start);
            if (r < 0) return r;
            break;
        }
        if (wire) return fail(SEPO_E_STATE, "prepared re-issue list overflow (routed records)");
        cur.out = nullptr;  // index re-issue from here on
        if (combine_exact) {
            // the insert's count is exact (certified declines, R15): only the per-tile counts
            const uint64_t pass = t->st.passes;
            if (pass < SEPO_MAX_PASS_STATS) t->st.postponed_per_pass[pass] += (uint64_t)c;
            if (t->tile_counts.grow(sepo_reprobe_tiles(cur.n) * 3 * 8)) return fail(SEPO_E_NOMEM, "tile count scratch");
            int rc3 = sepo_launch_tile_popc(cur, (unsigned long long*)t->tile_counts.p, 8 * t->n_sms, t->stream);
            if (rc3) return cuda_check(t, (cudaError_t)rc3, "tile_popc kernel");
            t->st.kernel_launches += 1;
        }
        // re-issue by index: the postponed records stay where they are in the caller's arrays
        if (t->idxb[side].grow((uint64_t)c * 8)) return fail(SEPO_E_NOMEM, "re-issue index list");
        uint64_t* nidx = (uint64_t*)t->idxb[side].p;
        const int64_t m = c;
        // GROUP: a pass without progress (retained key pages starve the pool) evicts everything
        // (the paper is silent; reading R14)
        int honor = 1;
        if (t->opts.mode == SEPO_GROUP && (uint64_t)m >= prev) {
            honor = 0;
            t->st.forced_full_evictions++;
        }
        prev = (uint64_t)m;
        // the compaction only reads the bitmap: it overlaps the eviction's D2H copies
        int64_t e = evict_impl(t, honor, [&]() -> int {
            const int64_t mm = compact_index_impl(t, cur, (uint64_t)c, nidx);
            return mm < 0 ? (int)mm : 0;
        });
        if (e < 0) return e;
        cur.idx = nidx;
        cur.n = (uint64_t)m;
        t->pending_idx_key_bytes = kb;
        side ^= 1;
        if (t->st.passes - passes_start > 100000) return fail(SEPO_E_STATE, "no progress");
    }
    // final generation to host (P:L227 timing scope includes the table transfer)
    if (t->dirty) {
        int64_t e = evict_impl(t, 0);
        if (e < 0) return e;
    }
    CK(t, cudaStreamSynchronize(t->copy_stream));
    trace("run end", t->st.passes - passes_start);
    return (int64_t)t->st.passes - passes_start;
}

// ---------------------------------------------------------------- raw-text word count (NEXT-2)
// The whole SEPO job on raw text (COMBINE, value 1 per word): pass 1 tokenizes and inserts in one
// kernel (insert_text_kernel); declined words become prepared records (their text offsets); later
// passes are the ordinary reinsert passes. Words declined after the prepared list filled up set
// their start bit in a text bitmap and are converted to prepared records after pass 1.
int64_t sepo_run_text(sepo_table* t, const uint8_t* text, uint64_t n_bytes) {
    trace("run_text begin", n_bytes);
    int rc = check_active(t);
    if (rc) return rc;
    if (t->opts.mode != SEPO_COMBINE_SUM_U64) return fail(SEPO_E_INVAL, "sepo_run_text needs COMBINE mode");
    if (n_bytes && !text) return fail(SEPO_E_INVAL, "text is NULL");
    if (n_bytes == 0) {
        if (t->dirty) { int64_t e = evict_impl(t, 0); if (e < 0) return e; }
        return 0;
    }
    if (!is_device_ptr(text)) {
        // host text: the H2D copy (P:L227 counts this transfer) is pipelined with pass 1 — 1 GiB
        // chunks (whole 512-byte windows) go over the host link on the copy stream, each with
        // max(64 KiB, page_bytes) of the next so the words that cross its end are complete when its
        // windows are inserted (a longer word cannot be stored anyway: SEPO_E_TOOLARGE)
        if (t->in_stage[0].grow(n_bytes + 16)) return fail(SEPO_E_NOMEM, "device staging for host text");
        const char* pch = getenv("SEPO_H2D_TEXT_CHUNK");
        uint64_t cb = pch ? strtoull(pch, nullptr, 10) : (1ull << 30);
        cb = std::max<uint64_t>(512, cb & ~511ull);
        const uint64_t nch = (n_bytes + cb - 1) / cb;
        std::vector<cudaEvent_t> evs(nch);
        for (auto& e : evs) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
        cudaEvent_t h0, h1;
        cudaEventCreate(&h0);
        cudaEventCreate(&h1);
        uint8_t* dst = (uint8_t*)t->in_stage[0].p;
        CK(t, cudaEventRecord(h0, t->copy_stream));
        uint64_t copied = 0;  // bytes [0, copied) are enqueued
        for (uint64_t c = 0; c < nch; ++c) {
            // the overlap covers any word that can be stored (an entry fits one page)
            const uint64_t want = std::min<uint64_t>(n_bytes, (c + 1) * cb + std::max<uint64_t>(64ull << 10, t->page_bytes));
            if (want > copied) {
                CK(t, cudaMemcpyAsync(dst + copied, text + copied, want - copied, cudaMemcpyHostToDevice, t->copy_stream));
                copied = want;
            }
            CK(t, cudaEventRecord(evs[c], t->copy_stream));
        }
        CK(t, cudaEventRecord(h1, t->copy_stream));
        t->h2d_chunks = &evs;
        t->h2d_chunk_records = cb;  // (bytes per chunk for text)
        const int64_t r = sepo_run_text(t, dst, n_bytes);
        t->h2d_chunks = nullptr;
        cudaEventSynchronize(h1);
        t->st.t_h2d_ms += elapsed_ms(h0, h1);
        for (auto& e : evs) cudaEventDestroy(e);
        cudaEventDestroy(h0);
        cudaEventDestroy(h1);
        return r;
    }
    std::vector<cudaEvent_t>* chunks = t->h2d_chunks;  // pipelined host text: per-chunk copy events
    t->h2d_chunks = nullptr;
    if ((uintptr_t)text & 15) return fail(SEPO_E_INVAL, "device text must be 16-byte aligned");
    const int64_t passes_start = (int64_t)t->st.passes;
    Batch cur{};
    cur.keys = text;
    cur.n = n_bytes;
    cur.text = 1;
    cur.prep_rb = 32;
    cur.dirpf = dir_prefetch(t) ? 1u : 0u;
    // prepared list for pass 1 (a word is >= 2 bytes with its separator; ~n/32 slots = a quarter of
    // 8-byte words), the overflow bitmap over the text bytes (zero between uses)
    uint64_t cap = std::max<uint64_t>(1ull << 16, n_bytes / 32);
    if (const char* pc = getenv("SEPO_PREP_CAP")) cap = strtoull(pc, nullptr, 10);
    const uint64_t tbm_bytes = ((n_bytes + 31) / 32) * 4;
    if (t->prep_n.grow(64) || t->prep[0].grow(std::max<uint64_t>(cap, 1) * 32)) return fail(SEPO_E_NOMEM, "prepared list");
    if ((size_t)t->tbm.cap < tbm_bytes) {
        if (t->tbm.grow(tbm_bytes)) return fail(SEPO_E_NOMEM, "text overflow bitmap");
        CK(t, cudaMemsetAsync(t->tbm.p, 0, t->tbm.cap, t->stream));
    }
    CK(t, cudaMemsetAsync(t->prep_n.p, 0, 16, t->stream));
    cur.out = (PRec*)t->prep[0].p;
    cur.out_n = (unsigned long long*)t->prep_n.p;
    cur.out_cap = cap;
    cur.tbm = (uint32_t*)t->tbm.p;
    // ---- pass 1: fused tokenize + insert
    t->inserted = true;
    t->dirty = true;
    ++t->batch_seq;
    sync_dev(t);
    if ((rc = zero_ctrl_counters(t))) return rc;
    CK(t, cudaMemsetAsync(&t->d.ctrl->text_words, 0, 8, t->stream));
    CK(t, cudaEventRecord(t->ev0, t->stream));
    if (t->hot.grow(sepo_hot_scratch_bytes())) return fail(SEPO_E_NOMEM, "hot-set scratch");
    bool hot_built = false;  // this job's hot set (chunks >= 1 reuse the one chunk 0 sampled, if any)
    if (chunks) {  // each chunk's windows as soon as its copy landed; the hot set from the first
        const uint64_t cb = t->h2d_chunk_records;
        for (size_t k = 0; k < chunks->size(); ++k) {
            CK(t, cudaStreamWaitEvent(t->stream, (*chunks)[k], 0));
            Batch bc = cur;
            bc.w_begin = (k * cb) / 512;
            bc.w_end = std::min<uint64_t>((k + 1) * cb, n_bytes + 511) / 512;
            if (k + 1 == chunks->size()) bc.w_end = ~0ull;
            rc = sepo_launch_insert_text(t->d, bc, t->grid, t->stream, t->hot.p, k == 0 ? std::min<uint64_t>(cb, n_bytes) : 0,
                                         &hot_built);
            if (rc) return cuda_check(t, (cudaError_t)rc, "text insert kernel launch");
        }
    } else {
        rc = sepo_launch_insert_text(t->d, cur, t->grid, t->stream, t->hot.p, n_bytes, &hot_built);
        if (rc) return cuda_check(t, (cudaError_t)rc, "text insert kernel launch");
    }
    CK(t, cudaEventRecord(t->ev1, t->stream));
    t->st.kernel_launches += (n_bytes >= (64ull << 18)) ? 7 : 1;
    CK(t, cudaMemcpyAsync(&t->h_ko[0], cur.out_n, 8, cudaMemcpyDeviceToHost, t->stream));
    t->h_ko[2] = 0;
    if (hot_built)
        CK(t, cudaMemcpyAsync(&t->h_ko[2], (uint8_t*)t->hot.p + sepo_hot_count_offset(), 4, cudaMemcpyDeviceToHost,
                              t->stream));
    if ((rc = read_ctrl(t))) return rc;
    t->st.hot_keys = std::max<uint64_t>(t->st.hot_keys, t->h_ko[2]);
    t->last_insert_ms = elapsed_ms(t->ev0, t->ev1);
    t->st.t_insert_ms += t->last_insert_ms;
    if (t->st.passes < SEPO_MAX_PASS_STATS) t->st.t_insert_ms_per_pass[t->st.passes] += t->last_insert_ms;
    t->st.insert_calls++;
    t->st.records_inserted += t->h_ctrl->text_words;
    t->st.key_bytes_inserted += n_bytes;
    t->st.dead_bytes += t->h_ctrl->dead_bytes;
    {
        const uint64_t used = std::min<uint64_t>(t->h_ctrl->pool_taken, t->d.n_free) + t->pages_resident_retained;
        t->st.pages_used_max = std::max<uint64_t>(t->st.pages_used_max, used);
    }
    if (t->h_ctrl->toolarge) {
        t->st.toolarge += t->h_ctrl->toolarge;
        // pass 1 may have set overflow bits that are never converted: the bitmap must be all zero
        // for the next job (text_bits_kernel clears the bits it converts on the normal path)
        CK(t, cudaMemsetAsync(t->tbm.p, 0, t->tbm.cap, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
        return fail(SEPO_E_TOOLARGE, std::to_string(t->h_ctrl->toolarge) + " word(s) cannot fit in one page");
    }
    const uint64_t c = t->h_ctrl->postponed;
    uint64_t kb = t->h_ctrl->kept_key_bytes;
    uint64_t reserved = t->h_ko[0];
    int ps = 0;
    if (c > 0 && reserved > cap) {
        // overflow: the first `cap` slots hold prepared records, the other declined words are
        // bits of tbm -> copy the list to prep[1] and append one record per bit behind it
        const uint64_t slack = (uint64_t)t->grid * 32 * kPrepChunk;
        if (t->prep[1].grow((cap + c + slack) * 32)) return fail(SEPO_E_NOMEM, "prepared list (overflow)");
        CK(t, cudaMemcpyAsync(t->prep[1].p, t->prep[0].p, cap * 32, cudaMemcpyDeviceToDevice, t->stream));
        unsigned long long* counter = (unsigned long long*)t->prep_n.p + 2;
        t->h_ko[0] = cap;
        CK(t, cudaMemcpyAsync(counter, &t->h_ko[0], 8, cudaMemcpyHostToDevice, t->stream));
        Batch bb = cur;
        bb.out = (PRec*)t->prep[1].p;
        rc = sepo_launch_text_bits(t->d, bb, counter, t->stream);
        if (rc) return cuda_check(t, (cudaError_t)rc, "text bits kernel");
        t->st.kernel_launches += 1;
        CK(t, cudaMemcpyAsync(&t->h_ko[0], counter, 8, cudaMemcpyDeviceToHost, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
        reserved = t->h_ko[0];
        ps = 1;
    }
    if (c > 0) {
        const int64_t r = prep_passes(t, cur, ps, reserved, c, kb, 32, passes_start);
        if (r < 0) return r;
    }
    if (t->dirty) {
        int64_t e = evict_impl(t, 0);
        if (e < 0) return e;
    }
    CK(t, cudaStreamSynchronize(t->copy_stream));
    trace("run_text end", t->st.passes - passes_start);
    return (int64_t)t->st.passes - passes_start;
}

// ---------------------------------------------------------------- SEPO lookups (NEXT-4)
int64_t sepo_lookup(sepo_table* t, const uint8_t* keys, const uint64_t* ko, uint64_t n, uint64_t* values_out,
                    uint32_t* found_bitmap) {
    if (!t) return fail(SEPO_E_INVAL, "null table");
    if (t->state == ST_BROKEN) return fail(SEPO_E_CUDA, "table is broken by an earlier CUDA error");
    if (t->opts.mode != SEPO_COMBINE_SUM_U64) return fail(SEPO_E_INVAL, "sepo_lookup supports COMBINE tables");
    if (n == 0) return 0;
    if (!values_out || !found_bitmap) return fail(SEPO_E_INVAL, "values_out / found_bitmap is NULL");
    if (!is_device_ptr(keys) || !is_device_ptr(ko) || !is_device_ptr(values_out) || !is_device_ptr(found_bitmap))
        return fail(SEPO_E_INVAL, "sepo_lookup takes device arrays");
    Batch b;
    int rc = make_batch(t, b, keys, ko, nullptr, nullptr, n, nullptr);
    if (rc) return rc;
    if (t->state == ST_ACTIVE && t->dirty) {  // the resident generation joins the host images first
        int64_t e = evict_impl(t, 0);
        if (e < 0) return e;
    }
    CK(t, cudaStreamSynchronize(t->copy_stream));
    CK(t, cudaMemsetAsync(found_bitmap, 0, ((n + 31) / 32) * 4, t->stream));
    CK(t, cudaMemsetAsync(values_out, 0, n * 8, t->stream));
    t->lookup_done = true;  // the pool now holds restored images: inserts need sepo_reset
    uint64_t found = 0;
    std::vector<uint32_t> ids;
    for (auto& g : t->gens) {
        // restore the generation's pages to their slots (one H2D per run), then link + probe
        ids.clear();
        for (auto& r : g.runs) {
            CK(t, cudaMemcpyAsync(t->d.pool + ((size_t)r.first << t->page_shift), r.p, (size_t)r.count << t->page_shift,
                                  cudaMemcpyDefault, t->stream));
            for (uint32_t k = 0; k < r.count; ++k) ids.push_back(r.first + k);
        }
        if (t->lk_pages.grow(ids.size() * 4 + 4)) return fail(SEPO_E_NOMEM, "lookup page list");
        CK(t, cudaMemcpyAsync(t->lk_pages.p, ids.data(), ids.size() * 4, cudaMemcpyHostToDevice, t->stream));
        CK(t, cudaMemsetAsync(t->d.dir, 0, t->n_buckets * 4, t->stream));
        if ((rc = zero_ctrl_counters(t))) return rc;
        rc = sepo_launch_lookup_gen(t->d, b, (const uint32_t*)t->lk_pages.p, (uint32_t)ids.size(),
                                    (unsigned long long*)values_out, found_bitmap, t->stream);
        if (rc) return cuda_check(t, (cudaError_t)rc, "lookup kernels");
        t->st.kernel_launches += 2;
        if ((rc = read_ctrl(t))) return rc;  // (also orders the host vector reuse after the copy)
        found += t->h_ctrl->postponed;
        if (found == n) break;  // every query resolved: later generations are not needed
    }
    return (int64_t)found;
}

int sepo_reset(sepo_table* t) {
    trace("reset");
    if (!t) return fail(SEPO_E_INVAL, "null table");
    if (t->state == ST_BROKEN) return fail(SEPO_E_CUDA, "table is broken");
    cudaStreamSynchronize(t->copy_stream);
    for (auto& c : t->arena) c.used = 0;
    t->gens.clear();
    t->state = ST_ACTIVE;
    t->dirty = false;
    t->inserted = false;
    t->batch_seq = 0;
    t->pages_resident_retained = 0;
    t->lookup_done = false;
    trace("reset: copy stream idle");
    if (t->st.pages_used_max) t->last_job_pages = t->st.pages_used_max;
    sepo_stats z{};
    z.n_buckets = t->n_buckets;
    z.page_bytes = t->page_bytes;
    z.pool_pages = t->n_pages;
    z.grid_ctas = t->grid;
    t->st = z;
    if (t->placement == SEPO_POOL_MANAGED) {
        // residency ablation: between jobs a managed pool's pages go back to host memory, so every
        // job pays the hardware demand paging of its table
        CK(t, cudaMemPrefetchAsync(t->pool_alloc, (size_t)t->n_pages * t->page_bytes + t->page_bytes, cudaCpuDeviceId,
                                   t->stream));
    }
    return init_device_state(t);
}

int sepo_stats_get(const sepo_table* t, sepo_stats* out) {
    if (!t || !out) return fail(SEPO_E_INVAL, "null argument");
    *out = t->st;
    return 0;
}

double sepo_last_insert_ms(const sepo_table* t) { return t ? t->last_insert_ms : 0.0; }

void sepo_destroy(sepo_table* t) {
    if (!t) return;
    if (t->stream) cudaStreamSynchronize(t->stream);
    if (t->copy_stream) cudaStreamSynchronize(t->copy_stream);
    t->tile_counts.release();
    t->hot.release();
    t->idxb[0].release();
    t->idxb[1].release();
    t->prep[0].release();
    t->prep[1].release();
    t->prep_n.release();
    t->tbm.release();
    t->eprog.release();
    t->evl.release();
    t->lk_pages.release();
    t->bm.release();
    for (int i = 0; i < 3; ++i) { t->sh_send[i].release(); t->sh_held[i].release(); t->sh_tmp[i].release(); }
    t->sh_cnt.release();
#if SEPO_WITH_NCCL
    if (t->route_stream) cudaStreamSynchronize(t->route_stream);
    if (t->nccl && t->win) ncclCommWindowDeregister((ncclComm_t)t->nccl, (ncclWindow_t)t->win);
    if (t->win_buf) ncclMemFree(t->win_buf);
    if (t->nccl) ncclCommDestroy((ncclComm_t)t->nccl);
#endif
    for (auto& s : t->buf)
        for (auto& b : s) b.release();
    for (auto& b : t->in_stage) b.release();
    for (auto& c : t->arena) cudaFreeHost(c.p);
    if (t->h_ctrl) cudaFreeHost(t->h_ctrl);
    if (t->h_evict) cudaFreeHost(t->h_evict);
    if (t->h_ko) cudaFreeHost(t->h_ko);
    if (t->region) cudaFree(t->region);
    if (t->pool_alloc) {
        if (t->placement == SEPO_POOL_HOST_PINNED) cudaFreeHost(t->pool_alloc);
        else cudaFree(t->pool_alloc);
    }
    if (t->ev0) cudaEventDestroy(t->ev0);
    if (t->ev1) cudaEventDestroy(t->ev1);
    if (t->evc0) cudaEventDestroy(t->evc0);
    if (t->evc1) cudaEventDestroy(t->evc1);
    if (t->ev_copy) cudaEventDestroy(t->ev_copy);
    if (t->ev_comp) cudaEventDestroy(t->ev_comp);
    if (t->own_stream && t->stream) cudaStreamDestroy(t->stream);
    if (t->copy_stream) cudaStreamDestroy(t->copy_stream);
    if (t->route_stream) cudaStreamDestroy(t->route_stream);
    for (auto& b : t->sh_recv) b.release();
    delete t;
}

// ---------------------------------------------------------------- key-hash router (a12)
int64_t sepo_run_wire(sepo_table* t, const void* wire, uint64_t n) {
    trace("run_wire begin", n);
    int rc = check_active(t);
    if (rc) return rc;
    if (t->opts.mode != SEPO_COMBINE_SUM_U64) return fail(SEPO_E_INVAL, "sepo_run_wire needs COMBINE mode");
    if (n && !is_device_ptr(wire)) return fail(SEPO_E_INVAL, "wire records must be device memory");
    if (n == 0) {
        if (t->dirty) { int64_t e = evict_impl(t, 0); if (e < 0) return e; }
        return 0;
    }
    return run_device(t, nullptr, nullptr, nullptr, nullptr, n, reinterpret_cast<const WireRec*>(wire));
}

static int cur_sms() {
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    return nsm;
}
size_t sepo_route_scratch(uint32_t n_parts) { return sepo_route_scratch_bytes(std::max<uint32_t>(n_parts, 1), cur_sms()); }

namespace {
// The router's two passes, split so sepo_run_sharded can place the parts itself (peer windows).
// route_pass0: hot-set discovery + counts; hc = [P][G] non-hot records per (part, CTA), then per part
// the hot keys it owns [32], (unused) [64], the long-key count. Synchronizes s.
int route_pass0(const Batch& b, uint32_t P, uint64_t seed, void* scratch, int G, cudaStream_t s,
                std::vector<unsigned long long>& hc) {
    int rc = sepo_launch_route_hot(b, P, seed, 0, scratch, G, nullptr, s);
    if (rc) return fail(SEPO_E_CUDA, std::string("route: ") + cudaGetErrorString((cudaError_t)rc));
    size_t co = 0, ho = 0;
    sepo_route_layout(P, G, &co, &ho);
    hc.assign((size_t)P * G + 3 * 32 + 8, 0);
    if (cudaMemcpyAsync(hc.data(), (uint8_t*)scratch + co, 8 * (size_t)P * G, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaMemcpyAsync(hc.data() + (size_t)P * G, (uint8_t*)scratch + ho, 8 * (3 * 32 + 8), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
        return fail(SEPO_E_CUDA, "route counts");
    if (hc[(size_t)P * G + 3 * 32]) return fail(SEPO_E_TOOLARGE, "route combine: keys longer than 16 bytes (route them as CSR)");
    return 0;
}
// records this rank sends to each part (non-hot + hot keys owned)
void route_part_totals(const std::vector<unsigned long long>& hc, uint32_t P, int G, std::vector<uint64_t>& tot) {
    tot.assign(P, 0);
    for (uint32_t p = 0; p < P; ++p) {
        for (int c = 0; c < G; ++c) tot[p] += hc[(size_t)p * G + c];
        tot[p] += hc[(size_t)P * G + p];
    }
}
// route_pass1: part p's records from record index start[p] of its destination (out, or dstp[p]):
// CTA by CTA, then its hot keys. Enqueued on s (no sync).
int route_pass1(const Batch& b, uint32_t P, uint64_t seed, void* scratch, int G, cudaStream_t s,
                const std::vector<unsigned long long>& hc, const std::vector<uint64_t>& start, WireRec* out,
                WireRec* const* dstp) {
    std::vector<unsigned long long> hb((size_t)P * G + 32, 0);
    for (uint32_t p = 0; p < P; ++p) {
        uint64_t at = start[p];
        for (int c = 0; c < G; ++c) { hb[(size_t)p * G + c] = at; at += hc[(size_t)p * G + c]; }
        hb[(size_t)P * G + p] = at;  // hot base of part p
    }
    size_t co = 0, ho = 0;
    sepo_route_layout(P, G, &co, &ho);
    unsigned long long* bases = (unsigned long long*)((uint8_t*)scratch + co) + (size_t)P * G;
    unsigned long long* hot_base = (unsigned long long*)((uint8_t*)scratch + ho) + 32;
    // (hb is pageable host memory: these copies complete before cudaMemcpyAsync returns)
    if (cudaMemcpyAsync(bases, hb.data(), 8 * (size_t)P * G, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        cudaMemcpyAsync(hot_base, hb.data() + (size_t)P * G, 8 * P, cudaMemcpyHostToDevice, s) != cudaSuccess)
        return fail(SEPO_E_CUDA, "route bases");
    int rc = sepo_launch_route_hot(b, P, seed, 1, scratch, G, out, s, dstp);
    if (rc) return fail(SEPO_E_CUDA, std::string("route: ") + cudaGetErrorString((cudaError_t)rc));
    return 0;
}
}  // namespace

int64_t sepo_route_combine(const uint8_t* keys, const uint64_t* ko, uint32_t kw, const uint8_t* vals, uint32_t vw,
                           uint64_t n, uint32_t n_parts, uint64_t route_seed, void* out_wire, uint64_t out_cap,
                           uint64_t* part_counts, void* scratch, size_t scratch_bytes, void* stream) {
    if (n_parts < 1 || n_parts > 32) return fail(SEPO_E_INVAL, "n_parts must be in 1..32");
    if (!ko && kw == 0) return fail(SEPO_E_INVAL, "key_offsets is NULL and fixed_key_width is 0");
    if (vals && !(vw == 1 || vw == 2 || vw == 4 || vw == 8)) return fail(SEPO_E_INVAL, "fixed_val_width must be 1, 2, 4 or 8");
    if (!part_counts || !scratch || scratch_bytes < sepo_route_scratch(n_parts)) return fail(SEPO_E_INVAL, "scratch / part_counts");
    const uint32_t P = n_parts;
    const int G = cur_sms();
    cudaStream_t s = (cudaStream_t)stream;
    Batch b{};
    b.keys = keys; b.ko = ko; b.kw = kw; b.vals = vals; b.vw = vw; b.n = n;
    // the same route hash as sepo_partition (seed decorrelated from a table seed of equal value)
    route_seed ^= 0x6a09e667f3bcc909ull;
    std::vector<unsigned long long> hc;
    int rc = route_pass0(b, P, route_seed, scratch, G, s, hc);
    if (rc) return rc;
    std::vector<uint64_t> tot, start(P, 0);
    route_part_totals(hc, P, G, tot);
    uint64_t all = 0;
    for (uint32_t p = 0; p < P; ++p) { part_counts[p] = start[p] = all; all += tot[p]; }
    part_counts[P] = all;
    if (!out_wire) return (int64_t)all;  // sizing call
    if (out_cap < all) return fail(SEPO_E_NOMEM, "route combine: out_cap < " + std::to_string(all) + " records");
    rc = route_pass1(b, P, route_seed, scratch, G, s, hc, start, (WireRec*)out_wire, nullptr);
    if (rc) return rc;
    if (cudaStreamSynchronize(s) != cudaSuccess) return fail(SEPO_E_CUDA, "route");
    return (int64_t)all;
}

size_t sepo_partition_scratch(uint64_t n, uint32_t n_parts) {
    return (size_t)sepo_partition_tiles(n) * n_parts * 3 * 8 + 256;
}

int sepo_partition(const uint8_t* keys, const uint64_t* ko, uint32_t kw, const uint8_t* vals, uint32_t vw, uint64_t n,
                   uint32_t P, uint64_t route_seed, uint8_t* ok, uint64_t* oko, uint8_t* ov, uint64_t* part_starts,
                   void* scratch, size_t scratch_bytes, void* stream) {
    if (P < 1 || P > 32) return fail(SEPO_E_INVAL, "n_parts must be in [1, 32]");
    if (!part_starts) return fail(SEPO_E_INVAL, "part_starts is NULL");
    if (!ko && kw == 0) return fail(SEPO_E_INVAL, "key_offsets is NULL and fixed_key_width is 0");
    if (vals && vw == 0) return fail(SEPO_E_INVAL, "fixed_val_width is 0");
    if (scratch_bytes < sepo_partition_scratch(n, P)) return fail(SEPO_E_INVAL, "partition scratch too small");
    if (n && (!keys || !ok || (ko && !oko) || (vals && !ov))) return fail(SEPO_E_INVAL, "NULL buffer");
    Batch b;
    b.keys = keys; b.ko = ko; b.kw = kw; b.vals = vals; b.vo = nullptr; b.vw = vw; b.n = n; b.bitmap = nullptr; b.idx = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<unsigned long long> h(3 * P, 0);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int rc = sepo_launch_partition(b, P, route_seed ^ 0x6a09e667f3bcc909ull, (unsigned long long*)scratch, ok, oko, ov,
                                   h.data(), sms, s);
    if (rc) return fail(SEPO_E_CUDA, std::string("partition: ") + cudaGetErrorString((cudaError_t)rc));
    cudaError_t e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(SEPO_E_CUDA, std::string("partition: ") + cudaGetErrorString(e));
    for (uint32_t p = 0; p < 3 * P; ++p) part_starts[p] = h[p];
    part_starts[3 * P] = n;
    part_starts[3 * P + 1] = ko ? 0 : n * (uint64_t)kw;
    part_starts[3 * P + 2] = vals ? n * (uint64_t)vw : 0;
    if (ko && n) {
        uint64_t first = 0, last = 0;
        cudaMemcpy(&first, ko, 8, cudaMemcpyDeviceToHost);
        cudaMemcpy(&last, ko + n, 8, cudaMemcpyDeviceToHost);
        part_starts[3 * P + 1] = last - first;
    }
    return 0;
}

int sepo_shift_offsets(uint64_t* ko, uint64_t n, const uint64_t* seg_rec, const uint64_t* seg_base, uint32_t n_segs,
                       uint64_t total, void* stream) {
    if (!ko || (n && (!seg_rec || !seg_base || n_segs == 0))) return fail(SEPO_E_INVAL, "NULL argument");
    int rc = sepo_launch_shift_offsets(ko, n, seg_rec, seg_base, n_segs, total, (cudaStream_t)stream);
    if (rc) return fail(SEPO_E_CUDA, std::string("shift_offsets: ") + cudaGetErrorString((cudaError_t)rc));
    return 0;
}

// ---------------------------------------------------------------- map runtime (NEXT-4)
int64_t sepo_map_run(sepo_table* t, int mapper, const uint8_t* text, uint64_t n_bytes, const uint64_t* doc_offsets,
                     uint64_t n_docs) {
    int rc = check_active(t);
    if (rc) return rc;
    if (mapper == SEPO_MAP_WORDS) return sepo_run_text(t, text, n_bytes);
    if (mapper != SEPO_MAP_LINES && mapper != SEPO_MAP_WORD_DOCS) return fail(SEPO_E_INVAL, "unknown mapper");
    if (mapper == SEPO_MAP_LINES && t->opts.mode != SEPO_COMBINE_SUM_U64) return fail(SEPO_E_INVAL, "MAP_LINES needs COMBINE");
    if (mapper == SEPO_MAP_WORD_DOCS) {
        if (t->opts.mode != SEPO_GROUP || t->opts.fixed_val_width != 4) return fail(SEPO_E_INVAL, "MAP_WORD_DOCS needs GROUP, fixed_val_width 4");
        if (!doc_offsets || n_docs == 0 || n_docs > 0xffffffffull) return fail(SEPO_E_INVAL, "doc_offsets / n_docs");
        if (!is_device_ptr(doc_offsets)) return fail(SEPO_E_INVAL, "doc_offsets must be device memory");
    }
    if (n_bytes && (!text || !is_device_ptr(text))) return fail(SEPO_E_INVAL, "text must be device memory");
    if (t->opts.fixed_key_width) return fail(SEPO_E_INVAL, "map runs produce CSR keys (fixed_key_width must be 0)");
    const int lines = mapper == SEPO_MAP_LINES;
    const uint64_t nch = sepo_map_chunks(n_bytes);
    if (t->tile_counts.grow((nch + 1) * 24)) return fail(SEPO_E_NOMEM, "map counts");
    unsigned long long* tc = (unsigned long long*)t->tile_counts.p;
    uint64_t tot[3] = {0, 0, 0};
    if (nch) {
        rc = sepo_launch_map(text, n_bytes, lines, 0, tc, nullptr, 0, nullptr, nullptr, nullptr, t->stream);
        if (rc) return cuda_check(t, (cudaError_t)rc, "map count");
        CK(t, cudaMemcpyAsync(tot, tc + 3 * nch, 24, cudaMemcpyDeviceToHost, t->stream));
        CK(t, cudaStreamSynchronize(t->stream));
    }
    const uint64_t m = tot[0], kbytes = tot[1];
    // the mapped batch (table-owned scratch): key bytes, offsets, doc ids
    if (t->buf[0][0].grow(kbytes + 16) || t->buf[0][1].grow((m + 1) * 8) ||
        (mapper == SEPO_MAP_WORD_DOCS && t->buf[0][2].grow(m * 4 + 16)))
        return fail(SEPO_E_NOMEM, "mapped batch");
    uint8_t* okeys = (uint8_t*)t->buf[0][0].p;
    uint64_t* oko = (uint64_t*)t->buf[0][1].p;
    uint32_t* odoc = mapper == SEPO_MAP_WORD_DOCS ? (uint32_t*)t->buf[0][2].p : nullptr;
    if (m) {
        rc = sepo_launch_map(text, n_bytes, lines, 1, tc, doc_offsets, n_docs, okeys, oko, odoc, t->stream);
        if (rc) return cuda_check(t, (cudaError_t)rc, "map write");
    }
    t->h_ko[3] = kbytes;
    CK(t, cudaMemcpyAsync(oko + m, &t->h_ko[3], 8, cudaMemcpyHostToDevice, t->stream));
    CK(t, cudaStreamSynchronize(t->stream));
    return run_device(t, okeys, oko, (const uint8_t*)odoc, nullptr, m);
}

// ---------------------------------------------------------------- multi-GPU data plane (a12)
// One process per GPU. sepo_insert_batch_sharded routes a batch by key owner (pre-combined wire
// records for COMBINE batches of keys <= 16 bytes, else a CSR partition), exchanges the parts with
// NCCL point-to-point sends over NVLink (one ncclGroup: counts, then payloads), and appends what
// this rank owns to a table-owned buffer; sepo_drain runs the SEPO job on it (insert, postpone,
// evict, re-issue until nothing is postponed). Postponed records are never re-routed: a key's
// records all live on its owner, so every rank's export is final (no merge).
#if SEPO_WITH_NCCL
#include <nccl_device.h>
namespace {
// destination of part p in chunk slot `off` of the window: rank p's copy, through its LSA (NVLink) mapping
__global__ void p2p_ptrs_kernel(ncclWindow_t w, size_t off, int P, sepo::WireRec** out) {
    const int p = threadIdx.x;
    if (p < P) out[p] = reinterpret_cast<sepo::WireRec*>(ncclGetPeerPointer(w, off, p));
}
const uint64_t kRouteSeed = 0x5eedull;  // owner hash seed (the library decorrelates it from table seeds)
int nccl_check(sepo_table* t, ncclResult_t r, const char* what) {
    if (r == ncclSuccess) return 0;
    t->state = ST_BROKEN;
    return fail(SEPO_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}
#define NK(t, expr)                                                  \
    do {                                                             \
        int _rc = nccl_check((t), (expr), #expr);                    \
        if (_rc) return _rc;                                         \
    } while (0)
// append device bytes [src, src + bytes) to buffer b (holding `have` bytes)
int append_dev(sepo_table* t, DevBuf& b, uint64_t have, const void* src, uint64_t bytes, DevBuf& tmp) {
    if (!bytes) return 0;
    if ((uint64_t)b.cap < have + bytes) {  // grow, keeping the contents
        if (tmp.grow(have + bytes)) return fail(SEPO_E_NOMEM, "sharded buffer");
        if (have) CK(t, cudaMemcpyAsync(tmp.p, b.p, have, cudaMemcpyDeviceToDevice, t->stream));
        std::swap(b.p, tmp.p);
        std::swap(b.cap, tmp.cap);
    }
    CK(t, cudaMemcpyAsync((uint8_t*)b.p + have, src, bytes, cudaMemcpyDeviceToDevice, t->stream));
    return 0;
}
}  // namespace
#endif

int sepo_nccl_unique_id(void* out_id) {
#if SEPO_WITH_NCCL
    if (!out_id) return fail(SEPO_E_INVAL, "out_id is NULL");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return fail(SEPO_E_NCCL, ncclGetErrorString(r));
    memcpy(out_id, &id, sizeof(id));
    return 0;
#else
    (void)out_id;
    return fail(SEPO_E_NCCL, "built without NCCL");
#endif
}

int sepo_attach_nccl(sepo_table* t, const void* nccl_unique_id, int nranks, int rank) {
    int rc = check_active(t);
    if (rc) return rc;
    if (!nccl_unique_id || nranks < 1 || nranks > 32 || rank < 0 || rank >= nranks)
        return fail(SEPO_E_INVAL, "attach: id / nranks in 1..32 / rank");
#if SEPO_WITH_NCCL
    if (t->nccl) return fail(SEPO_E_STATE, "a communicator is attached already");
    CK(t, cudaSetDevice(t->device));
    ncclUniqueId id;
    memcpy(&id, nccl_unique_id, sizeof(id));
    ncclComm_t comm;
    NK(t, ncclCommInitRank(&comm, nranks, id, rank));
    t->nccl = comm;
    t->nranks = nranks;
    t->rank = rank;
    return 0;
#else
    return fail(SEPO_E_NCCL, "built without NCCL");
#endif
}

int64_t sepo_insert_batch_sharded(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals,
                                  const uint64_t* vo, uint64_t n) {
    int rc = check_active(t);
    if (rc) return rc;
#if SEPO_WITH_NCCL
    if (!t->nccl) return fail(SEPO_E_STATE, "no communicator (sepo_attach_nccl)");
    if (vo) return fail(SEPO_E_INVAL, "sharded batches take fixed-width values");
    if (n && !(is_device_ptr(keys) && is_device_ptr(ko) && is_device_ptr(vals))) return fail(SEPO_E_INVAL, "device inputs only");
    const uint32_t P = (uint32_t)t->nranks;
    const uint32_t kw = t->opts.fixed_key_width, vw = vals ? t->opts.fixed_val_width : 0u;
    ncclComm_t comm = (ncclComm_t)t->nccl;
    cudaStream_t s = t->stream;
    if (t->sh_cnt.grow(8 * (6 * (size_t)P + 64))) return fail(SEPO_E_NOMEM, "count scratch");
    uint64_t* dsend = (uint64_t*)t->sh_cnt.p;   // [P][3]: records, key bytes, value bytes per destination
    uint64_t* drecv = dsend + 3 * P;             // [P][3] from each source
    std::vector<uint64_t> send(3 * P, 0), recv(3 * P, 0);
    // ---- route: pre-combined wire records (COMBINE, keys <= 16 bytes), else a CSR partition
    int fmt = 0;
    int64_t m = -1;
    std::vector<uint64_t> pc(P + 1, 0);
    if (t->opts.mode == SEPO_COMBINE_SUM_U64 && t->shard_fmt != 2 && n) {
        void* scr = nullptr;
        if (t->sh_tmp[2].grow(sepo_route_scratch(P))) return fail(SEPO_E_NOMEM, "route scratch");
        scr = t->sh_tmp[2].p;
        // (one call: a batch leaves at most one wire record per record)
        if (t->sh_send[0].grow((size_t)std::max<uint64_t>(n, 1) * sizeof(WireRec))) return fail(SEPO_E_NOMEM, "wire send buffer");
        m = sepo_route_combine(keys, ko, kw, vals, vw, n, P, kRouteSeed, t->sh_send[0].p, n, pc.data(), scr,
                               sepo_route_scratch(P), s);
        if (m >= 0) {
            fmt = 1;
            for (uint32_t p = 0; p < P; ++p) send[3 * p] = pc[p + 1] - pc[p];
        } else if (m != SEPO_E_TOOLARGE) {
            return m;
        }
    }
    if (!fmt && n) {
        if (t->shard_fmt == 1) return fail(SEPO_E_INVAL, "a batch with keys longer than 16 bytes after wire batches");
        const uint64_t kbytes = ko ? 0 : n * (uint64_t)kw;
        uint64_t k0 = 0, kend = kbytes;
        if (ko) {
            CK(t, cudaMemcpy(&k0, ko, 8, cudaMemcpyDeviceToHost));
            CK(t, cudaMemcpy(&kend, ko + n, 8, cudaMemcpyDeviceToHost));
        }
        if (t->sh_send[0].grow(kend - k0 + 16) || (ko && t->sh_send[1].grow((n + 1) * 8)) ||
            (vals && t->sh_send[2].grow(n * (uint64_t)vw + 16)) || t->sh_tmp[2].grow(sepo_partition_scratch(n, P)))
            return fail(SEPO_E_NOMEM, "partition buffers");
        std::vector<uint64_t> st(3 * (P + 1));
        rc = sepo_partition(keys, ko, kw, vals, vw, n, P, kRouteSeed, (uint8_t*)t->sh_send[0].p,
                            ko ? (uint64_t*)t->sh_send[1].p : nullptr, vals ? (uint8_t*)t->sh_send[2].p : nullptr, st.data(),
                            t->sh_tmp[2].p, sepo_partition_scratch(n, P), s);
        if (rc) return rc;
        fmt = 2;
        for (uint32_t p = 0; p < P; ++p)
            for (int c = 0; c < 3; ++c) send[3 * p + c] = st[3 * (p + 1) + c] - st[3 * p + c];
        for (uint32_t p = 0; p < P; ++p) pc[p] = st[3 * p];
    }
    if (!fmt) fmt = t->shard_fmt ? t->shard_fmt : 1;  // (an empty batch: nothing to send, counts still exchanged)
    // ---- counts (every rank takes part, also with n == 0)
    CK(t, cudaMemcpyAsync(dsend, send.data(), 8 * 3 * P, cudaMemcpyHostToDevice, s));
    NK(t, ncclGroupStart());
    for (uint32_t p = 0; p < P; ++p) {
        NK(t, ncclSend(dsend + 3 * p, 3, ncclUint64, (int)p, comm, s));
        NK(t, ncclRecv(drecv + 3 * p, 3, ncclUint64, (int)p, comm, s));
    }
    NK(t, ncclGroupEnd());
    CK(t, cudaMemcpyAsync(recv.data(), drecv, 8 * 3 * P, cudaMemcpyDeviceToHost, s));
    CK(t, cudaStreamSynchronize(s));
    // (a rank whose batch was empty learns the format from its peers' counts: wire batches send no key bytes)
    uint64_t rn = 0, rk = 0, rv = 0;
    for (uint32_t p = 0; p < P; ++p) { rn += recv[3 * p]; rk += recv[3 * p + 1]; rv += recv[3 * p + 2]; }
    if (rk && fmt == 1 && !n) fmt = 2;
    if (t->shard_fmt && t->shard_fmt != fmt && rn) return fail(SEPO_E_INVAL, "mixed wire / CSR sharded batches");
    // ---- payloads into receive scratch, then appended to the records held
    const uint64_t rb0 = fmt == 1 ? rn * sizeof(WireRec) : rk;
    if (t->sh_tmp[0].grow(rb0 + 16) || (fmt == 2 && t->sh_tmp[1].grow((rn + 1) * 8)) || (fmt == 2 && t->sh_tmp[2].grow(rv + 16)))
        return fail(SEPO_E_NOMEM, "receive buffers");
    NK(t, ncclGroupStart());
    uint64_t so = 0, ro = 0, sko = 0, rko = 0, svo = 0, rvo = 0;
    for (uint32_t p = 0; p < P; ++p) {
        if (fmt == 1) {
            const uint64_t sb = send[3 * p] * sizeof(WireRec), rbb = recv[3 * p] * sizeof(WireRec);
            if (sb) NK(t, ncclSend((uint8_t*)t->sh_send[0].p + pc[p] * sizeof(WireRec), sb, ncclUint8, (int)p, comm, s));
            if (rbb) NK(t, ncclRecv((uint8_t*)t->sh_tmp[0].p + ro, rbb, ncclUint8, (int)p, comm, s));
            ro += rbb;
        } else {
            if (send[3 * p + 1]) NK(t, ncclSend((uint8_t*)t->sh_send[0].p + so, send[3 * p + 1], ncclUint8, (int)p, comm, s));
            if (recv[3 * p + 1]) NK(t, ncclRecv((uint8_t*)t->sh_tmp[0].p + ro, recv[3 * p + 1], ncclUint8, (int)p, comm, s));
            if (ko && send[3 * p]) NK(t, ncclSend((uint64_t*)t->sh_send[1].p + sko, send[3 * p], ncclUint64, (int)p, comm, s));
            if (recv[3 * p] && (ko || t->opts.fixed_key_width == 0))
                NK(t, ncclRecv((uint64_t*)t->sh_tmp[1].p + rko, recv[3 * p], ncclUint64, (int)p, comm, s));
            if (vals && send[3 * p + 2]) NK(t, ncclSend((uint8_t*)t->sh_send[2].p + svo, send[3 * p + 2], ncclUint8, (int)p, comm, s));
            if (recv[3 * p + 2]) NK(t, ncclRecv((uint8_t*)t->sh_tmp[2].p + rvo, recv[3 * p + 2], ncclUint8, (int)p, comm, s));
            so += send[3 * p + 1]; ro += recv[3 * p + 1]; sko += send[3 * p]; rko += recv[3 * p];
            svo += send[3 * p + 2]; rvo += recv[3 * p + 2];
        }
    }
    NK(t, ncclGroupEnd());
    DevBuf scratch;
    if (fmt == 1) {
        rc = append_dev(t, t->sh_held[0], t->sh_n * sizeof(WireRec), t->sh_tmp[0].p, rn * sizeof(WireRec), scratch);
        if (rc) { scratch.release(); return rc; }
    } else if (rn) {
        // received offsets are relative to each sender's segment: rebase them onto the key bytes held
        const bool csr = ko || t->opts.fixed_key_width == 0;
        if (csr) {
            std::vector<uint64_t> seg_rec(P), seg_base(P);
            uint64_t r = 0, kb = 0;
            for (uint32_t p = 0; p < P; ++p) { seg_rec[p] = r; seg_base[p] = t->sh_kb + kb; r += recv[3 * p]; kb += recv[3 * p + 1]; }
            uint64_t* dseg = drecv + 3 * P;  // (2P words after the counts)
            CK(t, cudaMemcpyAsync(dseg, seg_rec.data(), 8 * P, cudaMemcpyHostToDevice, s));
            CK(t, cudaMemcpyAsync(dseg + P, seg_base.data(), 8 * P, cudaMemcpyHostToDevice, s));
            rc = sepo_launch_shift_offsets((uint64_t*)t->sh_tmp[1].p, rn, dseg, dseg + P, P, t->sh_kb + rk, s);
            if (rc) { scratch.release(); return cuda_check(t, (cudaError_t)rc, "shift offsets"); }
            // held offsets: n + 1 entries (the last one is rewritten by each append)
            const uint64_t have = t->sh_n ? t->sh_n * 8 : 0;
            rc = append_dev(t, t->sh_held[1], have, t->sh_tmp[1].p, (rn + 1) * 8, scratch);
            if (rc) { scratch.release(); return rc; }
        }
        rc = append_dev(t, t->sh_held[0], t->sh_kb, t->sh_tmp[0].p, rk, scratch);
        if (!rc) rc = append_dev(t, t->sh_held[2], t->sh_vb, t->sh_tmp[2].p, rv, scratch);
        if (rc) { scratch.release(); return rc; }
    }
    CK(t, cudaStreamSynchronize(s));
    scratch.release();
    if (rn) t->shard_fmt = fmt;
    t->sh_n += rn;
    t->sh_kb += fmt == 2 ? rk : 0;
    t->sh_vb += fmt == 2 ? rv : 0;
    return (int64_t)t->sh_n;
#else
    (void)keys; (void)ko; (void)vals; (void)vo; (void)n;
    return fail(SEPO_E_NCCL, "built without NCCL");
#endif
}

int64_t sepo_drain(sepo_table* t) {
    int rc = check_active(t);
    if (rc) return rc;
    int64_t r = 0;
    const uint64_t n = t->sh_n;
    if (t->shard_fmt == 1) {
        r = run_device(t, nullptr, nullptr, nullptr, nullptr, n, (const WireRec*)t->sh_held[0].p);
    } else if (t->shard_fmt == 2) {
        const bool csr = t->opts.fixed_key_width == 0;
        r = run_device(t, (const uint8_t*)t->sh_held[0].p, csr ? (const uint64_t*)t->sh_held[1].p : nullptr,
                       t->sh_vb ? (const uint8_t*)t->sh_held[2].p : nullptr, nullptr, n);
    } else if (t->dirty) {
        int64_t e = evict_impl(t, 0);
        if (e < 0) return e;
    }
    if (r < 0) return r;
    t->sh_n = t->sh_kb = t->sh_vb = 0;
    t->shard_fmt = 0;
    return r;
}

// ---------------------------------------------------------------- pipelined sharded job (a12)
// sepo_run_sharded: the whole SEPO job over a batch sharded by key owner, with pass 1 pipelined
// against the exchange. The batch is cut into chunks (SEPO_SHARD_CHUNK records, a multiple of the
// router's 2048-record tile); for chunk c the route stream runs the router and the two NCCL groups
// (counts, payload) while t->stream inserts chunk c-1 — each insert waits only for its own chunk's
// receive event, and the host reads an insert's counters only after the next chunk's exchange is
// enqueued. Declined records become prepared re-issue records (a9; the list is kept large enough for
// every record received so far, so pass 1 never needs an index re-issue), then the ordinary re-issue
// passes and evictions run locally (no communication: a key's records all live on its owner).
//   wire format (every rank's keys <= 16 bytes): pre-combined 32-byte records, received into a
//     ping-pong pair of buffers (the prepared records carry the whole key);
//   CSR (some key > 16 bytes): partitioned key bytes / offsets [/ values] appended to the records
//     held (prepared records of long keys point into them), offsets rebased on the device.
#if SEPO_WITH_NCCL
namespace {
// grow b to hold `need` bytes keeping its first `have` bytes (stream s is synchronised)
int grow_keep(sepo_table* t, DevBuf& b, size_t have, size_t need, cudaStream_t s) {
    if (need <= b.cap) return 0;
    DevBuf nb;
    if (nb.grow(std::max(need, b.cap + b.cap / 2))) return fail(SEPO_E_NOMEM, "sharded job buffer");
    if (have) CK(t, cudaMemcpyAsync(nb.p, b.p, have, cudaMemcpyDeviceToDevice, s));
    CK(t, cudaStreamSynchronize(s));
    b.release();
    b = nb;
    return 0;
}
// The receive window of the peer-memory exchange: 2 slots of `need` (+25 %) wire records, symmetric
// (ncclMemAlloc + ncclCommWindowRegister, COLLECTIVE — every rank calls this with the same `need`, which
// comes from the all-gathered count matrix). Returns 0, or 1 if some rank could not register one (the
// ranks agree through an all-reduce; the job then uses NCCL send/recv).
int ensure_window(sepo_table* t, ncclComm_t comm, uint64_t need, uint64_t* dflag) {
    if (need <= t->win_cap && t->win) return 0;
    CK(t, cudaStreamSynchronize(t->stream));  // (an insert may still read the old window)
    CK(t, cudaStreamSynchronize(t->route_stream));
    if (t->win) ncclCommWindowDeregister(comm, (ncclWindow_t)t->win);
    if (t->win_buf) ncclMemFree(t->win_buf);
    t->win = nullptr; t->win_buf = nullptr; t->win_cap = 0;
    const uint64_t cap = std::max<uint64_t>(need + need / 4, 1ull << 16);
    const size_t bytes = ((2 * cap * sizeof(WireRec)) + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
    void* buf = nullptr;
    ncclWindow_t w = nullptr;
    uint64_t ok = ncclMemAlloc(&buf, bytes) == ncclSuccess && ncclCommWindowRegister(comm, buf, bytes, &w, NCCL_WIN_COLL_SYMMETRIC) == ncclSuccess;
    CK(t, cudaMemcpyAsync(dflag, &ok, 8, cudaMemcpyHostToDevice, t->route_stream));
    NK(t, ncclAllReduce(dflag, dflag, 1, ncclUint64, ncclMin, comm, t->route_stream));
    CK(t, cudaMemcpyAsync(&ok, dflag, 8, cudaMemcpyDeviceToHost, t->route_stream));
    CK(t, cudaStreamSynchronize(t->route_stream));
    if (!ok) {
        if (w) ncclCommWindowDeregister(comm, w);
        if (buf) ncclMemFree(buf);
        t->win_failed = true;
        trace("run_sharded: peer window unavailable, NCCL send/recv");
        return 1;
    }
    t->win = w; t->win_buf = buf; t->win_cap = cap;
    return 0;
}
}  // namespace
#endif

int64_t sepo_run_sharded(sepo_table* t, const uint8_t* keys, const uint64_t* ko, const uint8_t* vals,
                         const uint64_t* vo, uint64_t n) {
    trace("run_sharded begin", n);
    int rc = check_active(t);
    if (rc) return rc;
#if SEPO_WITH_NCCL
    if (!t->nccl) return fail(SEPO_E_STATE, "no communicator (sepo_attach_nccl)");
    if (t->opts.mode != SEPO_COMBINE_SUM_U64) return fail(SEPO_E_INVAL, "sepo_run_sharded needs COMBINE mode");
    if (t->opts.fail_alloc_ppm && t->opts.fail_mode == 1) return fail(SEPO_E_INVAL, "record-mode fault injection");
    if (vo) return fail(SEPO_E_INVAL, "sharded batches take fixed-width values");
    if (t->sh_n) return fail(SEPO_E_STATE, "records held by sepo_insert_batch_sharded (sepo_drain first)");
    const uint32_t kw = t->opts.fixed_key_width, vw = vals ? t->opts.fixed_val_width : 0u;
    if (n && (!keys || (!ko && kw == 0))) return fail(SEPO_E_INVAL, "keys / key_offsets");
    if (n && !(is_device_ptr(keys) && is_device_ptr(ko) && is_device_ptr(vals))) return fail(SEPO_E_INVAL, "device inputs only");
    if (vals && !(vw == 1 || vw == 2 || vw == 4 || vw == 8)) return fail(SEPO_E_INVAL, "fixed_val_width must be 1, 2, 4 or 8");
    const uint32_t P = (uint32_t)t->nranks;
    ncclComm_t comm = (ncclComm_t)t->nccl;
    cudaStream_t s = t->stream;
    if (!t->route_stream) CK(t, cudaStreamCreateWithFlags(&t->route_stream, cudaStreamNonBlocking));
    cudaStream_t rs = t->route_stream;
    // (the caller's inputs may have been written on t->stream or on the legacy default stream)
    CK(t, cudaStreamSynchronize(s));
    CK(t, cudaStreamSynchronize(cudaStreamLegacy));
    if (t->sh_cnt.grow(8 * ((size_t)P * P + 10 * (size_t)P + 64))) return fail(SEPO_E_NOMEM, "count scratch");
    uint64_t* dsend = (uint64_t*)t->sh_cnt.p;  // [P][3] records, key bytes, value bytes per destination
    uint64_t* drecv = dsend + 3 * P;            // [P][3] from each source
    uint64_t* dseg = drecv + 3 * P;             // [2P] segment starts / byte bases of a received chunk
    uint64_t* dagree = dseg + 2 * P;            // [2] longest key, chunks
    uint64_t* dflag = dagree + 2;               // [2] window agreement / barrier word
    uint64_t* dmat = dflag + 2;                 // [P][P] records rank s sends to rank d (peer-memory path)
    WireRec** dptr = (WireRec**)(dmat + (size_t)P * P);  // [P] destination of each part
    // ---- agree on the format and the number of chunks: one all-reduce (max)
    uint64_t per = 256ull << 20;  // (each chunk pays two hot-set discoveries and ~6 host syncs)
    if (const char* e = getenv("SEPO_SHARD_CHUNK")) per = strtoull(e, nullptr, 10);
    per = std::max<uint64_t>(2048, per / 2048 * 2048);
    // CSR batches whose keys are all <= 16 bytes (words) travel as wire records too: with the hot keys
    // folded out, C2 at N = 1 takes 76.9 ms per routed job as wire records vs 116.5 ms as a CSR partition
    // (profiles/r02/routed_n1.jsonl); SEPO_SHARD_WIRE=0 keeps CSR batches CSR
    const char* ew = getenv("SEPO_SHARD_WIRE");
    const bool wire_csr = !(ew && ew[0] == '0');
    uint64_t agree[2] = {ko ? 0ull : (uint64_t)kw, (n + per - 1) / per};
    if (ko && !wire_csr) agree[0] = 1ull << 20;  // (never wire)
    if (ko && wire_csr) {
        rc = sepo_launch_max_key_len(ko, n, (unsigned long long*)dagree, rs);
        if (rc) return cuda_check(t, (cudaError_t)rc, "max key length");
        t->st.kernel_launches += 1;
    } else {
        CK(t, cudaMemcpyAsync(dagree, &agree[0], 8, cudaMemcpyHostToDevice, rs));
    }
    CK(t, cudaMemcpyAsync(dagree + 1, &agree[1], 8, cudaMemcpyHostToDevice, rs));
    CK(t, cudaStreamSynchronize(rs));  // (agree is pageable host memory)
    NK(t, ncclAllReduce(dagree, dagree, 2, ncclUint64, ncclMax, comm, rs));
    CK(t, cudaMemcpyAsync(agree, dagree, 16, cudaMemcpyDeviceToHost, rs));
    CK(t, cudaStreamSynchronize(rs));
    const bool wire = agree[0] <= 16;
    const uint64_t nch = agree[1];
    const bool csr_keys = !wire && (ko != nullptr || kw == 0);  // received keys carry offsets
    // wire chunks go straight into the owners' receive windows over peer memory (the route kernel's
    // stores are the exchange, NEXT-2 ii) unless SEPO_SHARD_P2P=0 or a window cannot be registered
    const char* ep = getenv("SEPO_SHARD_P2P");
    bool p2p = wire && !(ep && ep[0] == '0') && !t->win_failed;
    const uint64_t seed_x = kRouteSeed ^ 0x6a09e667f3bcc909ull;  // (as sepo_route_combine)
    // ---- job state (as run_device): prepared re-issue records sized for what was received
    Batch cur{};
    cur.kw = wire ? 0u : kw;
    cur.vw = wire ? 8u : vw;
    // (fixed-width keys of at most 8 bytes, routed as wire records or not: 32-byte prepared records)
    const bool short_keys = !csr_keys && kw > 0 && kw <= 8;
    const bool has_vals = wire || vals != nullptr;
    const uint64_t prb = (has_vals && !short_keys) ? sizeof(PRec) : 32;
    cur.prep_rb = (uint32_t)prb;
    cur.prep_fmt = (has_vals && short_keys) ? 33u : 0u;
    const uint64_t slack = (uint64_t)t->grid * 32 * kPrepChunk;
    if (t->prep_n.grow(64)) return fail(SEPO_E_NOMEM, "prepared list counter");
    {   // the prepared list: room for a quarter of the records this rank sends (hash routing balances
        // the parts), at most a quarter of the free memory; it grows by half (one copy) when a chunk
        // could overflow it (a table far over budget declines most records)
        size_t fr = 0, tot = 0;
        uint64_t want = n / 4 + slack * std::max<uint64_t>(nch, 1);
        if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) want = std::min<uint64_t>(want, (fr + t->prep[0].cap) / 4 / prb);
        if ((uint64_t)t->prep[0].cap < want * prb) {
            t->prep[0].release();
            if (t->prep[0].grow(want * prb)) return fail(SEPO_E_NOMEM, "prepared re-issue list");
        }
    }
    if (!wire && n) {  // CSR: room for about as many records / bytes as this rank sends (grown if needed)
        uint64_t kb = n * (uint64_t)kw;
        if (ko) {
            CK(t, cudaMemcpyAsync(&t->h_ko[4], ko, 8, cudaMemcpyDeviceToHost, rs));
            CK(t, cudaMemcpyAsync(&t->h_ko[5], ko + n, 8, cudaMemcpyDeviceToHost, rs));
            CK(t, cudaStreamSynchronize(rs));
            kb = t->h_ko[5] - t->h_ko[4];
        }
        const uint64_t m = n + n / 16;
        if (t->sh_held[0].grow(kb + kb / 16 + 16) || (csr_keys && t->sh_held[1].grow((m + 1) * 8)) ||
            (vals && t->sh_held[2].grow(m * (uint64_t)vw + 16)))
            return fail(SEPO_E_NOMEM, "sharded job: records held");
    }
    CK(t, cudaMemsetAsync(t->prep_n.p, 0, 16, s));
    int64_t passes_start = (int64_t)t->st.passes;
    std::vector<cudaEvent_t> evs(std::max<uint64_t>(nch, 1));
    for (auto& e : evs) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    struct Guard {
        std::vector<cudaEvent_t>& e;
        ~Guard() { for (auto& x : e) cudaEventDestroy(x); }
    } guard{evs};
    // records / key bytes / value bytes held (CSR) and the previous chunk's insert
    uint64_t hn = 0, hkb = 0, hvb = 0;
    uint64_t post = 0, kept_kb = 0, reserved = 0;
    bool prev_live = false;
    Batch prev{};
    InsertLaunch prevL;
    auto finish_prev = [&]() -> int {
        if (!prev_live) return 0;
        prev_live = false;
        const int64_t c = insert_end(t, prev, prevL);
        if (c < 0) return (int)c;
        post += (uint64_t)c;
        kept_kb += t->h_ctrl->kept_key_bytes;
        CK(t, cudaMemcpyAsync(&t->h_ko[0], t->prep_n.p, 8, cudaMemcpyDeviceToHost, s));
        CK(t, cudaStreamSynchronize(s));
        reserved = t->h_ko[0];
        return 0;
    };
    const uint64_t scr_bytes = wire ? sepo_route_scratch(P) : sepo_partition_scratch(std::min(n, per), P);
    if (t->sh_tmp[2].grow(scr_bytes)) return fail(SEPO_E_NOMEM, "route scratch");
    for (uint64_t c = 0; c < nch; ++c) {
        const uint64_t r0 = std::min(n, c * per), r1 = std::min(n, r0 + per), cn = r1 - r0;
        std::vector<uint64_t> send(3 * P, 0), recv(3 * P, 0), pc(P + 1, 0);
        const WireRec* p2p_in = nullptr;  // this rank's window slot holding chunk c (peer-memory path)
        uint64_t rn = 0, rk = 0, rv = 0;
        if (p2p) {
            // ---- route pass 0, all-gather of the count matrix, pass 1 storing into the owners' windows
            Batch bc{};
            bc.keys = keys + (ko ? 0 : r0 * (uint64_t)kw); bc.ko = ko ? ko + r0 : nullptr; bc.kw = kw;
            bc.vals = vals ? vals + r0 * (uint64_t)vw : nullptr; bc.vw = vw; bc.n = cn;
            std::vector<unsigned long long> hc;
            std::vector<uint64_t> tot, mat((size_t)P * P), start(P, 0);
            rc = route_pass0(bc, P, seed_x, t->sh_tmp[2].p, cur_sms(), rs, hc);
            if (rc) return rc;
            route_part_totals(hc, P, cur_sms(), tot);
            CK(t, cudaMemcpyAsync(dsend, tot.data(), 8 * P, cudaMemcpyHostToDevice, rs));
            NK(t, ncclAllGather(dsend, dmat, P, ncclUint64, comm, rs));
            CK(t, cudaMemcpyAsync(mat.data(), dmat, 8 * (size_t)P * P, cudaMemcpyDeviceToHost, rs));
            CK(t, cudaStreamSynchronize(rs));
            uint64_t need = 0;
            for (uint32_t d = 0; d < P; ++d) {
                uint64_t in = 0;
                for (uint32_t sr = 0; sr < P; ++sr) {
                    in += mat[(size_t)sr * P + d];
                    if (sr < (uint32_t)t->rank) start[d] += mat[(size_t)sr * P + d];
                }
                need = std::max(need, in);
                if (d == (uint32_t)t->rank) rn = in;
            }
            t->st.kernel_launches += 2;
            trace("run_sharded: counts gathered", rn);
            rc = ensure_window(t, comm, need, dflag);
            if (rc < 0) return rc;
            if (rc == 0) {
                const size_t off = (size_t)(c & 1) * t->win_cap * sizeof(WireRec);
                p2p_ptrs_kernel<<<1, 32, 0, rs>>>((ncclWindow_t)t->win, off, (int)P, dptr);
                rc = route_pass1(bc, P, seed_x, t->sh_tmp[2].p, cur_sms(), rs, hc, start, nullptr, dptr);
                if (rc) return rc;
                // every rank's stores into every window are done before any rank reads its own
                NK(t, ncclAllReduce(dflag + 1, dflag + 1, 1, ncclUint64, ncclSum, comm, rs));
                CK(t, cudaEventRecord(evs[c], rs));
                p2p_in = reinterpret_cast<const WireRec*>((const uint8_t*)t->win_buf + off);
                t->st.kernel_launches += 3;
                t->st.p2p_chunks++;
            } else {
                p2p = false;  // (all ranks: the agreement above) — this chunk and the rest via send/recv
            }
        }
        if (p2p_in) {
            // (received already: skip the send/recv exchange)
        } else if (cn && wire) {
            if (t->sh_send[0].grow(cn * sizeof(WireRec))) return fail(SEPO_E_NOMEM, "wire send buffer");
            const int64_t m = sepo_route_combine(keys + (ko ? 0 : r0 * (uint64_t)kw), ko ? ko + r0 : nullptr, kw,
                                                 vals ? vals + r0 * (uint64_t)vw : nullptr, vw, cn, P, kRouteSeed,
                                                 t->sh_send[0].p, cn, pc.data(), t->sh_tmp[2].p, scr_bytes, rs);
            if (m < 0) return m;
            for (uint32_t p = 0; p < P; ++p) send[3 * p] = pc[p + 1] - pc[p];
            t->st.kernel_launches += 2;
        } else if (cn) {
            uint64_t kb0 = r0 * (uint64_t)kw, kb1 = r1 * (uint64_t)kw;
            if (ko) {
                CK(t, cudaMemcpyAsync(&t->h_ko[4], ko + r0, 8, cudaMemcpyDeviceToHost, rs));
                CK(t, cudaMemcpyAsync(&t->h_ko[5], ko + r1, 8, cudaMemcpyDeviceToHost, rs));
                CK(t, cudaStreamSynchronize(rs));
                kb0 = t->h_ko[4];
                kb1 = t->h_ko[5];
            }
            if (t->sh_send[0].grow(kb1 - kb0 + 16) || (csr_keys && t->sh_send[1].grow((cn + 1) * 8)) ||
                (vals && t->sh_send[2].grow(cn * (uint64_t)vw + 16)))
                return fail(SEPO_E_NOMEM, "partition buffers");
            std::vector<uint64_t> st(3 * (P + 1));
            rc = sepo_partition(ko ? keys : keys + kb0, ko ? ko + r0 : nullptr, kw, vals ? vals + r0 * (uint64_t)vw : nullptr,
                                vw, cn, P, kRouteSeed, (uint8_t*)t->sh_send[0].p, csr_keys ? (uint64_t*)t->sh_send[1].p : nullptr,
                                vals ? (uint8_t*)t->sh_send[2].p : nullptr, st.data(), t->sh_tmp[2].p, scr_bytes, rs);
            if (rc) return rc;
            for (uint32_t p = 0; p < P; ++p)
                for (int x = 0; x < 3; ++x) send[3 * p + x] = st[3 * (p + 1) + x] - st[3 * p + x];
            t->st.kernel_launches += 3;
        }
        if (!p2p_in) {
            trace("run_sharded: chunk routed", c);
            // ---- counts
            CK(t, cudaMemcpyAsync(dsend, send.data(), 8 * 3 * P, cudaMemcpyHostToDevice, rs));
            NK(t, ncclGroupStart());
            for (uint32_t p = 0; p < P; ++p) {
                NK(t, ncclSend(dsend + 3 * p, 3, ncclUint64, (int)p, comm, rs));
                NK(t, ncclRecv(drecv + 3 * p, 3, ncclUint64, (int)p, comm, rs));
            }
            NK(t, ncclGroupEnd());
            CK(t, cudaMemcpyAsync(recv.data(), drecv, 8 * 3 * P, cudaMemcpyDeviceToHost, rs));
            CK(t, cudaStreamSynchronize(rs));
            for (uint32_t p = 0; p < P; ++p) { rn += recv[3 * p]; rk += recv[3 * p + 1]; rv += recv[3 * p + 2]; }
            trace("run_sharded: counts exchanged", rn);
            // ---- receive space (wire: slot c & 1, last read by chunk c-2's insert, finished already;
            // CSR: appended to the records held — growing them waits for the running insert)
            if (wire) {
                if (t->sh_recv[c & 1].grow(std::max<uint64_t>(rn, 1) * sizeof(WireRec))) return fail(SEPO_E_NOMEM, "wire receive buffer");
            } else {
                const bool fit = hkb + rk + 16 <= t->sh_held[0].cap && (!csr_keys || (hn + rn + 1) * 8 <= t->sh_held[1].cap) &&
                                 (!vals || hvb + rv + 16 <= t->sh_held[2].cap);
                if (!fit) {
                    CK(t, cudaStreamSynchronize(s));
                    if ((rc = grow_keep(t, t->sh_held[0], hkb, hkb + rk + 16, rs))) return rc;
                    if (csr_keys && (rc = grow_keep(t, t->sh_held[1], hn * 8, (hn + rn + 1) * 8, rs))) return rc;
                    if (vals && (rc = grow_keep(t, t->sh_held[2], hvb, hvb + rv + 16, rs))) return rc;
                }
            }
            // ---- payload (one NCCL group), then rebase the received offsets onto the bytes held
            NK(t, ncclGroupStart());
            uint64_t so = 0, ro = 0, sko = 0, rko = 0, svo = 0, rvo = 0;
            for (uint32_t p = 0; p < P; ++p) {
                if (wire) {
                    const uint64_t sb = send[3 * p] * sizeof(WireRec), rbb = recv[3 * p] * sizeof(WireRec);
                    if (sb) NK(t, ncclSend((uint8_t*)t->sh_send[0].p + pc[p] * sizeof(WireRec), sb, ncclUint8, (int)p, comm, rs));
                    if (rbb) NK(t, ncclRecv((uint8_t*)t->sh_recv[c & 1].p + ro, rbb, ncclUint8, (int)p, comm, rs));
                    ro += rbb;
                    continue;
                }
                uint8_t* hk = (uint8_t*)t->sh_held[0].p + hkb;
                uint64_t* hko = (uint64_t*)t->sh_held[1].p + hn;
                uint8_t* hv = (uint8_t*)t->sh_held[2].p + hvb;
                if (send[3 * p + 1]) NK(t, ncclSend((uint8_t*)t->sh_send[0].p + so, send[3 * p + 1], ncclUint8, (int)p, comm, rs));
                if (recv[3 * p + 1]) NK(t, ncclRecv(hk + ro, recv[3 * p + 1], ncclUint8, (int)p, comm, rs));
                if (csr_keys && send[3 * p]) NK(t, ncclSend((uint64_t*)t->sh_send[1].p + sko, send[3 * p], ncclUint64, (int)p, comm, rs));
                if (csr_keys && recv[3 * p]) NK(t, ncclRecv(hko + rko, recv[3 * p], ncclUint64, (int)p, comm, rs));
                if (vals && send[3 * p + 2]) NK(t, ncclSend((uint8_t*)t->sh_send[2].p + svo, send[3 * p + 2], ncclUint8, (int)p, comm, rs));
                if (vals && recv[3 * p + 2]) NK(t, ncclRecv(hv + rvo, recv[3 * p + 2], ncclUint8, (int)p, comm, rs));
                so += send[3 * p + 1]; ro += recv[3 * p + 1]; sko += send[3 * p]; rko += recv[3 * p];
                svo += send[3 * p + 2]; rvo += recv[3 * p + 2];
            }
            NK(t, ncclGroupEnd());
            if (!wire && csr_keys && rn) {
                std::vector<uint64_t> seg(2 * P);
                uint64_t r = 0, kb = 0;
                for (uint32_t p = 0; p < P; ++p) { seg[p] = r; seg[P + p] = hkb + kb; r += recv[3 * p]; kb += recv[3 * p + 1]; }
                CK(t, cudaMemcpyAsync(dseg, seg.data(), 16 * P, cudaMemcpyHostToDevice, rs));
                rc = sepo_launch_shift_offsets((uint64_t*)t->sh_held[1].p + hn, rn, dseg, dseg + P, P, hkb + rk, rs);
                if (rc) return cuda_check(t, (cudaError_t)rc, "shift offsets");
                t->st.kernel_launches += 1;
                CK(t, cudaStreamSynchronize(rs));  // (seg is pageable host memory read by the copy above)
            }
            CK(t, cudaEventRecord(evs[c], rs));
        }
        // ---- the previous chunk's counters, room in the prepared list, then this chunk's insert
        if ((rc = finish_prev())) return rc;
        if (rn) {
            const uint64_t need = (reserved + rn + slack) * prb;
            if ((uint64_t)t->prep[0].cap < need && (rc = grow_keep(t, t->prep[0], reserved * prb, need, s))) return rc;
            if (t->bm.grow(((rn + 31) / 32) * 4)) return fail(SEPO_E_NOMEM, "bitmap scratch");
            CK(t, cudaStreamWaitEvent(s, evs[c], 0));
            Batch bc = cur;
            if (wire) {
                bc.wire = p2p_in ? p2p_in : (const WireRec*)t->sh_recv[c & 1].p;
                bc.vals = (const uint8_t*)bc.wire;
            } else {
                bc.keys = (const uint8_t*)t->sh_held[0].p + (csr_keys ? 0 : hkb);
                bc.ko = csr_keys ? (const uint64_t*)t->sh_held[1].p + hn : nullptr;
                bc.vals = vals ? (const uint8_t*)t->sh_held[2].p + hvb : nullptr;
            }
            bc.n = rn;
            bc.bitmap = (uint32_t*)t->bm.p;
            bc.out = (PRec*)t->prep[0].p;
            bc.out_n = (unsigned long long*)t->prep_n.p;
            bc.out_cap = t->prep[0].cap / prb;
            rc = insert_begin(t, bc, csr_keys ? hkb : 0, csr_keys ? hkb + rk : 0, prevL);
            if (rc) return rc;
            prev = bc;
            prev_live = true;
        }
        if (!wire) { hn += rn; hkb += rk; hvb += rv; }
    }
    if ((rc = finish_prev())) return rc;
    if (reserved > t->prep[0].cap / prb) return fail(SEPO_E_STATE, "prepared re-issue list overflow (sharded job)");
    trace("run_sharded pass 1 end", post);
    if (post) {
        cur.keys = wire ? nullptr : (const uint8_t*)t->sh_held[0].p;
        const int64_t r = prep_passes(t, cur, 0, reserved, post, kept_kb, prb, passes_start);
        if (r < 0) return r;
    }
    if (t->dirty) {
        int64_t e = evict_impl(t, 0);
        if (e < 0) return e;
    }
    CK(t, cudaStreamSynchronize(t->copy_stream));
    trace("run_sharded end", t->st.passes - passes_start);
    return (int64_t)t->st.passes - passes_start;
#else
    (void)keys; (void)ko; (void)vals; (void)vo; (void)n;
    return fail(SEPO_E_NCCL, "built without NCCL");
#endif
}
