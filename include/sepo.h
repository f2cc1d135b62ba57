/* sepo.h — C ABI of the B200-native SEPO hash table (Mokhtari & Stumm, IPDPS 2017).
 *
 * PAPER.md (= /root/reference/PAPER.md) is cited as P:L<line>. The calls follow the paper's
 * statement of the problem:
 *   * an insert either succeeds or returns POSTPONE, "like EAGAIN";
 *   * the requestor tracks declined records in a bitmap with one bit per input record (P:L75,
 *     P:L149) and re-issues only those later;
 *   * at the end of each pass the table is told it no longer needs its resident pairs and copies
 *     them to CPU memory, freeing the GPU heap;
 *   * the final table is accessible from the CPU.
 *
 * Conventions for every call:
 *   - "device" pointers are CUDA device memory (e.g. torch tensors' data_ptr()) and are
 *     CALLER-OWNED: they must stay valid until the call returns; the library never frees them.
 *   - Bitmap convention: bit (i & 31) of word (i >> 5) is 1 <=> record i was POSTPONED.
 *     A bitmap for n records has ceil(n / 32) uint32 words.
 *   - Key i of a batch is the byte string keys[ko[i] .. ko[i+1]) (ko = key_offsets, absolute
 *     offsets into keys, ko[0] need not be 0); ko == NULL means fixed-width keys of
 *     opts.fixed_key_width bytes (key i at keys + i * width).
 *   - Errors: a negative return is an error code (sepo_status); sepo_last_error() describes the
 *     last one on the calling thread. Argument errors leave the table unchanged. CUDA errors are
 *     sticky: the table then only accepts sepo_stats / sepo_destroy.
 *   - A table is bound to the CUDA device current at sepo_create and is NOT thread-safe.
 *   - Every hot-path step runs in this library's sm_100a kernels; there is no CPU fallback.
 */
#ifndef SEPO_H
#define SEPO_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sepo_table sepo_table; /* opaque; one per GPU */

enum sepo_status {
    SEPO_OK = 0,
    SEPO_E_INVAL = -1,    /* bad argument / unsupported combination */
    SEPO_E_NOMEM = -2,    /* budget too small, or a host/device allocation failed */
    SEPO_E_TOOLARGE = -3, /* a record's entry can never fit in one page (its bit is set) */
    SEPO_E_CUDA = -4,     /* CUDA error (sticky) */
    SEPO_E_STATE = -5,    /* call not allowed in the table's current state */
    SEPO_E_NCCL = -6      /* NCCL error (sticky) */
};

/* Bucket organizations. */
typedef enum {
    SEPO_COMBINE_SUM_U64 = 0, /* "combining": one entry per key, value = u64 wrapping sum */
    SEPO_GROUP = 1,           /* "multi-valued": key entries + per-key value lists */
    SEPO_BASIC = 2            /* "basic": every pair its own entry, duplicates kept;
                                 a pass halts once basic_halt_pct % of the allocator slots failed
                                 (P:L153-161). Values as COMBINE (fixed width <= 8 B LE, or 1). */
} sepo_mode;

typedef struct sepo_options {
    int32_t mode;             /* sepo_mode; default SEPO_COMBINE_SUM_U64 */
    uint32_t fixed_key_width; /* key bytes when key_offsets == NULL (1..page_bytes-32) */
    uint32_t fixed_val_width; /* COMBINE: bytes of each LE unsigned value when vals != NULL
                                 (1, 2, 4 or 8; default 8). GROUP: bytes per value when
                                 val_offsets == NULL (1..256). */
    uint32_t grid_ctas;       /* persistent CTAs = allocator slots (0 = 2 per SM) */
    uint64_t hash_seed;       /* seed of the table's key hash (result is independent of it) */
    uint32_t fail_alloc_ppm;  /* TEST ONLY: decline this many allocations per million */
    uint32_t fail_mode;       /* 0: by hash(key, pass) (monotone per key); 1: by (record, pass) */
    uint32_t fail_until_pass; /* injection is off from this pass on (default 16) */
    uint32_t check_dups;      /* sepo_export merges + counts keys found in >1 generation */
    void* stream;             /* cudaStream_t for all device work (NULL: a table-owned stream) */
    uint64_t host_arena_bytes;/* pinned host memory to pre-allocate for evicted pages */
    uint32_t basic_halt_pct;  /* BASIC: halt the pass once this % of allocator slots (the paper's
                                 bucket groups) failed to allocate (1..100; 0 = 50) */
    uint32_t pad_;
} sepo_options;

/* Host-side result, owned by the table (valid until the next sepo_reset / sepo_destroy).
 * Order of keys is unspecified (canonicalise by sorting to compare). */
typedef struct sepo_result {
    uint64_t n_keys;
    const uint8_t* keys;          /* key bytes, CSR */
    const uint64_t* key_offsets;  /* n_keys + 1 */
    const uint64_t* values;       /* COMBINE: n_keys u64 sums */
    const uint64_t* list_offsets; /* GROUP: n_keys + 1, key k owns values [lo[k], lo[k+1]) */
    uint64_t n_vals;              /* GROUP */
    const uint8_t* vals;          /* GROUP: value bytes, CSR */
    const uint64_t* val_offsets;  /* GROUP: n_vals + 1 */
} sepo_result;

#define SEPO_MAX_PASS_STATS 64
typedef struct sepo_stats {
    uint64_t passes;               /* evictions so far, the final one included (P:L237 counts) */
    uint64_t insert_calls;
    uint64_t records_inserted;     /* records handed to sepo_insert_batch (re-issues included) */
    uint64_t postponed_per_pass[SEPO_MAX_PASS_STATS]; /* after re-probe, per pass */
    uint64_t n_buckets, page_bytes, pool_pages, grid_ctas;
    uint64_t pages_used_max;       /* most pages resident at once */
    uint64_t bytes_evicted;        /* D2H bytes of evicted pages (final export included) */
    uint64_t dead_bytes;           /* bytes of entries that lost a link race */
    uint64_t cross_gen_dups;       /* keys merged across generations at export (check_dups) */
    uint64_t forced_full_evictions;/* GROUP: passes that evicted retained key pages */
    uint64_t toolarge;             /* records whose entry cannot fit a page */
    uint64_t key_bytes_inserted;   /* key bytes handed to sepo_insert_batch */
    uint64_t val_bytes_inserted;   /* value bytes handed to sepo_insert_batch */
    uint64_t kernel_launches;      /* this library's kernels launched since create/reset */
    uint64_t value_chunks;         /* GROUP export: value chunks parsed */
    uint64_t value_slots;          /* GROUP export: value slots in those chunks (capacity) */
    double t_insert_ms, t_reprobe_ms, t_compact_ms, t_evict_ms, t_export_ms, t_h2d_ms;
    double t_insert_ms_per_pass[SEPO_MAX_PASS_STATS]; /* insert-kernel time of each pass */
    uint64_t hot_keys;             /* most keys a sampled hot set held in one insert call (a2; 0: none) */
    uint64_t p2p_chunks;           /* sepo_run_sharded: chunks routed straight into the owners' windows
                                      over peer memory (0: NCCL send/recv) */
} sepo_stats;

/* Create a table on the current CUDA device.
 * device_budget_bytes: ONE device allocation of exactly this size holds the bucket directory
 *   (4 B x n_buckets), the allocator state and the page pool ("a heap
 *   pre-allocated in GPU memory ... partitioned into pages"). The paper sizes the heap as "the
 *   remaining free space"; here the caller caps it, which is how tables larger than the
 *   budget are produced. Must leave room for at least 4 pages; the pool is limited to 32 GiB.
 * n_buckets: >= 1, <= 2^32 - 1.   page_bytes: power of two in [4096, 16 MiB].
 * Returns NULL on error (sepo_last_error()). */
sepo_table* sepo_create(size_t device_budget_bytes, uint64_t n_buckets, uint32_t page_bytes);

/* Residency ablations: the same table and kernels with the
 * page pool placed elsewhere. Directory, control words and page metadata stay in device memory
 * (the paper's pinned experiment keeps "everything else" on the GPU); `device_budget_bytes`
 * still fixes the pool size (pool pages as for sepo_create), but only the directory + metadata part
 * is allocated on the device.
 *   SEPO_POOL_DEVICE      = sepo_create (the SEPO table: the pool is the device budget)
 *   SEPO_POOL_HOST_PINNED = pool in pinned host memory mapped into the device address space: every
 *                           entry read, combine atomic and allocation touches host memory over the link
 *   SEPO_POOL_MANAGED     = pool in cudaMallocManaged memory: pages migrate on demand (hardware paging);
 *                           sepo_reset prefetches the pool back to host memory, so every job pays it
 * Returns NULL on error (sepo_last_error): unknown placement -> INVAL; allocation failure -> NOMEM. */
enum { SEPO_POOL_DEVICE = 0, SEPO_POOL_HOST_PINNED = 1, SEPO_POOL_MANAGED = 2 };
sepo_table* sepo_create_placed(size_t device_budget_bytes, uint64_t n_buckets, uint32_t page_bytes, int placement);

/* Budget (bytes) that sepo_create needs so that the pool holds exactly `pool_pages` pages.
 * Pure arithmetic on the host (no CUDA call). */
size_t sepo_budget_for(uint64_t n_buckets, uint32_t page_bytes, uint64_t pool_pages);

/* Set options (only before the first insert, or right after sepo_reset). */
int sepo_configure(sepo_table* t, const sepo_options* opts);

/* Insert n records (the SEPO "insert"). Each key is hashed to a bucket, the
 * bucket chain is walked; a key already resident in this pass is combined/grouped in place
 * (P:L77); a new key gets an entry allocated from the page pool and linked at the
 * chain head. If allocation fails the record is POSTPONED: its bitmap bit is set.
 * keys/key_offsets/vals/val_offsets: device; see conventions above.
 *   COMBINE: vals == NULL => every value is 1 (Word Count / PVC); else fixed-width LE
 *            unsigned values (opts.fixed_val_width bytes each); val_offsets must be NULL.
 *   GROUP:   vals required; val_offsets != NULL => value i = vals[vo[i] .. vo[i+1]) (variable
 *            length, stored as {u32 length, bytes} items; at most page_bytes - 40 bytes), else
 *            opts.fixed_val_width bytes each (1..256).
 * postponed_bitmap: device, ceil(n/32) words, fully written (bits >= n are 0).
 * Returns the number of postponed records (>= 0; POSTPONE is not an error), or < 0.
 * The count is an upper bound of what must be re-issued: a declined record whose key another
 * thread linked concurrently is absorbed by sepo_reprobe at the end of the pass.
 * Stream-ordered on the table's stream; synchronizes once to read the count. */
int64_t sepo_insert_batch(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                          const uint64_t* val_offsets, uint64_t n, uint32_t* postponed_bitmap);

/* End-of-pass re-probe (restores the residency guarantee P:L77, P:L79 under
 * lock-free insertion). For every record whose bit is set, look its key up in the resident
 * generation: if present, combine/append it now and clear the bit; in GROUP mode a resident key
 * that still cannot take its value marks its key page as retained. Call after the last
 * insert of a pass and before sepo_evict, with each batch of the pass.
 * bitmap: device, updated in place. *key_bytes / *val_bytes (may be NULL) receive the bytes the
 * remaining records occupy (to size sepo_compact's outputs). Returns the remaining count. */
int64_t sepo_reprobe(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                     const uint64_t* val_offsets, uint64_t n, uint32_t* bitmap, uint64_t* key_bytes,
                     uint64_t* val_bytes);

/* Stream-compaction re-issue (a9; replaces the paper's restart "from the point where a request
 * was postponed for the first time"): gather the records whose bit is set, in
 * input order, into out_* (device, caller-owned, sized from sepo_reprobe's byte counts; out_ko
 * and out_vo need m + 1 entries). Output offsets are rebased to 0. Fixed-width keys/values stay
 * fixed-width (out_ko / out_vo unused then and may be NULL). Returns m. */
int64_t sepo_compact(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                     const uint64_t* val_offsets, uint64_t n, const uint32_t* bitmap, uint8_t* out_keys,
                     uint64_t* out_key_offsets, uint8_t* out_vals, uint64_t* out_val_offsets);

/* Pass boundary (a10): copy the cold pages — COMBINE: every page of the generation;
 * GROUP: value pages + key pages without pending keys — to pinned host memory and
 * return them to the pool; reset the bucket directory. Returns bytes copied (>= 0) or < 0. */
int64_t sepo_evict(sepo_table* t);

/* Finish the job (a11): evict the resident generation, wait for all copies, and assemble the
 * result on the host from every generation's page images. After this only
 * sepo_stats / sepo_reset / sepo_destroy are allowed. */
int sepo_export(sepo_table* t, sepo_result* out);

/* The whole SEPO job in one call: insert all n records, then re-probe / compact / evict and
 * re-issue until nothing is postponed, then evict the final generation (the table is then on the
 * host; call sepo_export for the assembled result). keys/key_offsets/vals/val_offsets may be
 * HOST or DEVICE memory (all four alike); host input is streamed to the device in chunks.
 * Returns the number of passes (>= 1) or < 0. */
int64_t sepo_run(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                 const uint64_t* val_offsets, uint64_t n);

/* Word count on RAW TEXT (the paper's WC): the whole SEPO job like
 * sepo_run, with the tokenizer fused into the insert kernel (text is read once; no CSR). A word is
 * a maximal run of bytes other than ' ', '\n', '\t', '\r' (reading R20); every word is a record
 * with value 1, combined by u64 sum (COMBINE mode only, else SEPO_E_INVAL). `text` is device
 * memory (16-byte aligned, else SEPO_E_INVAL) or host memory (staged to the device first).
 * Returns the number of passes (evictions, the final one included) or < 0; stats.records_inserted
 * counts the words of pass 1 plus every re-issue. A word longer than page_bytes - 32 fails the job
 * with SEPO_E_TOOLARGE. */
int64_t sepo_run_text(sepo_table* t, const uint8_t* text, uint64_t n_bytes);

/* SEPO LOOKUPS on the larger-than-memory table ("The SEPO model can also
 * be used for lookup operations on larger-than-memory hash tables"). COMBINE tables only (else
 * SEPO_E_INVAL). keys/key_offsets (CSR, or fixed_key_width when key_offsets is NULL), values_out
 * (n u64) and found_bitmap (ceil(n/32) u32) are DEVICE arrays (else SEPO_E_INVAL). The resident
 * generation is evicted first; then every generation's page images go back into the device pool
 * (each page to the slot it left, so entry refs stay valid), the directory is rebuilt from them
 * and every query not yet found is probed — a query whose key is not in this generation is
 * postponed to the next one. Query i: bit (i&31) of found_bitmap[i>>5] = 1 and values_out[i] =
 * the key's value if the key is in the table, else bit 0 and value 0. Returns the number found
 * (or < 0). Allowed before or after sepo_export; afterwards only sepo_lookup, sepo_export,
 * sepo_stats, sepo_reset and sepo_destroy (inserts: SEPO_E_STATE until sepo_reset). */
int64_t sepo_lookup(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, uint64_t n, uint64_t* values_out,
                    uint32_t* found_bitmap);

/* Drop all generations and results and start a new job with the same budget and options;
 * pinned host memory and device scratch are kept for reuse. */
int sepo_reset(sepo_table* t);

int sepo_stats_get(const sepo_table* t, sepo_stats* out);

/* Milliseconds of device time of the most recent sepo_insert_batch kernel(s), measured with CUDA
 * events on the table's stream (bench roofline). */
double sepo_last_insert_ms(const sepo_table* t);

void sepo_destroy(sepo_table* t);

/* ---------------------------------------------------------------- multi-GPU key-hash router (a12)
 * The method shards naturally: a key's result depends only on its own records, so the table is
 * split across GPUs by owner(k) = hi32(H(route_seed, k)) * n_parts >> 32 (H = the table's key hash
 * with another seed, so owner and bucket are independent). Each rank partitions its slice of the
 * input, exchanges the parts with an all-to-all (NCCL over NVLink, driven by the caller's process
 * group), then runs its own SEPO job; the union of the ranks' exports is the result (no merge). */

/* Device scratch bytes sepo_partition needs for n records and n_parts parts. */
size_t sepo_partition_scratch(uint64_t n, uint32_t n_parts);

/* Stable partition of n records by owner (1 <= n_parts <= 32). Inputs as in sepo_insert_batch
 * (key_offsets == NULL => fixed_key_width; vals == NULL => no values, else fixed_val_width bytes
 * each). Outputs (device, caller-owned, same sizes as the inputs): out_keys, out_key_offsets
 * (n entries: record j's offset relative to the first byte of ITS part; NULL for fixed-width
 * keys), out_vals. part_starts (HOST, 3 * (n_parts + 1) u64): for part p, (first record, first key
 * byte, first value byte) in the outputs; entry n_parts holds the totals. The order of records within a
 * part is unspecified (each record takes its slot with one shared-memory atomic). Synchronizes the stream. */
int sepo_partition(const uint8_t* keys, const uint64_t* key_offsets, uint32_t fixed_key_width, const uint8_t* vals,
                   uint32_t fixed_val_width, uint64_t n, uint32_t n_parts, uint64_t route_seed, uint8_t* out_keys,
                   uint64_t* out_key_offsets, uint8_t* out_vals, uint64_t* part_starts, void* scratch,
                   size_t scratch_bytes, void* stream);

/* After an exchange, key_offsets[0..n) holds n_segs received segments whose offsets are relative
 * to their own key bytes. Adds seg_byte_base[s] to segment s (records [seg_rec_start[s],
 * seg_rec_start[s+1]); device arrays of n_segs entries) and writes key_offsets[n] = total_bytes. */
int sepo_shift_offsets(uint64_t* key_offsets, uint64_t n, const uint64_t* seg_rec_start, const uint64_t* seg_byte_base,
                       uint32_t n_segs, uint64_t total_bytes, void* stream);
/* Router with pre-combine (COMBINE mode; "CTA-level pre-combine of duplicate keys
 * into (key, partial sum)"). Partitions n records by owner like sepo_partition, but the keys of the
 * batch's sampled hot set (batches of >= 2^21 records; the insert kernels' discovery on the route hash)
 * are combined over the whole batch first — each leaves as ONE record carrying its sum (u64 wrapping sum
 * of the values, implicit 1 when vals == NULL); every other record leaves as its own record.
 * Every output record is a 32-byte wire record
 *     struct { uint64_t w0, w1;  // key bytes 0..15, little endian, zero padded
 *              uint64_t value;   // the combined value
 *              uint64_t len; }   // key length (0..16)
 * Keys must be at most 16 bytes (words, u64 keys); a longer key fails the call with SEPO_E_TOOLARGE and
 * nothing is written (route such batches with sepo_partition). Inputs (device) as sepo_partition.
 * out_wire (device, caller-owned, out_cap records) receives part p's records at [part_counts[p],
 * part_counts[p + 1]); part_counts (HOST, n_parts + 1) is the exclusive prefix of the per-part counts
 * with the total last. out_wire == NULL is a sizing call (counts only). The order of records within a
 * part is unspecified. scratch: device, sepo_route_scratch(n_parts) bytes (for the current device).
 * Synchronizes the stream.
 * Returns the number of wire records, or < 0 (SEPO_E_NOMEM: out_cap too small; part_counts valid). */
size_t sepo_route_scratch(uint32_t n_parts);
int64_t sepo_route_combine(const uint8_t* keys, const uint64_t* key_offsets, uint32_t fixed_key_width, const uint8_t* vals,
                           uint32_t fixed_val_width, uint64_t n, uint32_t n_parts, uint64_t route_seed, void* out_wire,
                           uint64_t out_cap, uint64_t* part_counts, void* scratch, size_t scratch_bytes, void* stream);

/* The whole SEPO job (as sepo_run) on n wire records (device; the records a rank received after
 * sepo_route_combine + the exchange): key = the record's first len bytes, value = its u64. COMBINE
 * mode only. Returns the number of passes or < 0. */
int64_t sepo_run_wire(sepo_table* t, const void* wire, uint64_t n);

/* ---- map runtime (the paper's MapReduce library): the map tasks of the
 * paper's applications as built-in kernels that turn raw text into the records of one SEPO job (map
 * callbacks cannot cross a C ABI as device code).
 *   SEPO_MAP_WORDS     MAP_REDUCE, COMBINE table: every word -> (word, 1)   (Word Count)
 *                      = sepo_run_text (tokenizer fused into the insert kernel)
 *   SEPO_MAP_LINES     MAP_REDUCE, COMBINE table: every non-empty line (bytes other than '\n') -> (line, 1)
 *                      (Page View Count on a log of URLs, one per line)
 *   SEPO_MAP_WORD_DOCS MAP_GROUP, GROUP table with fixed_val_width 4: every word -> (word, u32 doc id),
 *                      doc d = text bytes [doc_offsets[d], doc_offsets[d+1]) (Inverted Index)
 * text, doc_offsets (n_docs entries, ascending, doc_offsets[0] = 0): device memory. Words follow reading
 * R20. The mapped batch lives in table-owned scratch; the whole SEPO job runs as sepo_run (all passes, final
 * eviction). Returns the number of passes or < 0. */
enum { SEPO_MAP_WORDS = 0, SEPO_MAP_LINES = 1, SEPO_MAP_WORD_DOCS = 2 };
int64_t sepo_map_run(sepo_table* t, int mapper, const uint8_t* text, uint64_t n_bytes, const uint64_t* doc_offsets,
                     uint64_t n_docs);

/* ---- the multi-GPU data plane inside the library (one process per GPU; NCCL over NVLink / NVSwitch)
 * sepo_nccl_unique_id: 128 bytes for out_id (ncclGetUniqueId) — rank 0 creates it, the caller
 *   broadcasts it (e.g. torch.distributed) to every rank.
 * sepo_attach_nccl: joins the table to a communicator of nranks (1..32) ranks (ncclCommInitRank on the
 *   table's device; collective). SEPO_E_NCCL on NCCL errors (sticky), SEPO_E_STATE if one is attached.
 * sepo_insert_batch_sharded: COLLECTIVE over the attached ranks (every rank calls it, n may be 0).
 *   The batch (device arrays as sepo_insert_batch; fixed-width values only) is routed by key owner
 *   owner(k) = hi32(H(route seed, k)) * nranks >> 32 — COMBINE batches of keys <= 16 bytes as
 *   pre-combined wire records (sepo_route_combine), others as a CSR partition (sepo_partition) —
 *   the parts are exchanged with NCCL send/recv (counts, then payloads, each one NCCL group on the
 *   table's stream), and the records this rank owns are appended to a table-owned buffer. A table
 *   holds one format at a time (wire or CSR: SEPO_E_INVAL on a mix). Returns the records held.
 * sepo_drain: the SEPO job on the records held (as sepo_run: insert, postpone, evict, re-issue until
 *   nothing is postponed; the final generation goes to host memory), then the buffer is emptied.
 *   No communication: postponed records are never re-routed, a key's records all live on its owner,
 *   so each rank's sepo_export is final and the union over ranks is the result (no merge).
 *   Returns the number of passes or < 0. */
int sepo_nccl_unique_id(void* out_id);
int sepo_attach_nccl(sepo_table* t, const void* nccl_unique_id, int nranks, int rank);
int64_t sepo_insert_batch_sharded(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                                  const uint64_t* val_offsets, uint64_t n);
int64_t sepo_drain(sepo_table* t);
/* sepo_run_sharded: COLLECTIVE; the whole SEPO job over a batch sharded by key
 *   owner, with the exchange pipelined against pass 1 (chunk c+1 is routed and exchanged
 *   on a second stream while chunk c is inserted). COMBINE mode only; device inputs as sepo_insert_batch
 *   (fixed-width values, val_offsets NULL; n may be 0 on some ranks). The ranks agree (one NCCL
 *   all-reduce) on the number of chunks (SEPO_SHARD_CHUNK records each, default 2^28, a multiple of
 *   2048) and on the format: pre-combined wire records when every rank's keys are <= 16 bytes, else a
 *   CSR partition. Records declined in pass 1 become prepared re-issue records; the re-issue passes,
 *   evictions and the final transfer to host run locally. Afterwards sepo_export gives this rank's
 *   keys; the union over ranks is the result. Returns the number of passes or < 0 (SEPO_E_STATE if
 *   records from sepo_insert_batch_sharded are held, SEPO_E_INVAL for GROUP / BASIC tables). */
int64_t sepo_run_sharded(sepo_table* t, const uint8_t* keys, const uint64_t* key_offsets, const uint8_t* vals,
                         const uint64_t* val_offsets, uint64_t n);

const char* sepo_last_error(void);
const char* sepo_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SEPO_H */
