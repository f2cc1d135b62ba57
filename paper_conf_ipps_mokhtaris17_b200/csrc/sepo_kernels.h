// sepo_kernels.h — launcher interface between the host engine (sepo_capi.cu) and the kernels.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "sepo_dev.cuh"

namespace sepo {
struct WireRec;
// A postponed COMBINE record, re-issued by sepo_run in "prepared" form (a9): its hash, first 16
// key bytes (zero padded), key offset in the caller's key bytes (tail of keys longer than 16 B),
// value and key length — the next pass needs neither the input gather nor the hash again.
struct PRec {
    uint64_t w0, w1, h, s, v;
    uint32_t len, pad;
};
static_assert(sizeof(PRec) == 48, "PRec layout");
// One batch of records as passed to sepo_insert_batch / sepo_reprobe / sepo_compact.
struct Batch {
    const uint8_t* keys;
    const uint64_t* ko;   // nullptr => fixed width kw
    uint32_t kw;
    uint32_t vw;          // COMBINE: value bytes (vals != nullptr); GROUP: fixed value bytes
    const uint8_t* vals;  // COMBINE: nullptr => 1
    const uint64_t* vo;   // GROUP variable-length values (not supported yet: must be nullptr)
    uint64_t n;
    uint32_t* bitmap;
    const uint64_t* idx;  // nullptr, or: record i of the batch is record idx[i] of keys/ko/vals (re-issue)
    // COMBINE, sepo_run only: declined records are also appended to out[] (capacity out_cap; the
    // counter *out_n may exceed it, then the host falls back to the bitmap), and a prepared batch
    // (prep != nullptr) replaces keys/ko/vals as the input of reinsert passes.
    PRec* out = nullptr;
    unsigned long long* out_n = nullptr;
    uint64_t out_cap = 0;
    const PRec* prep = nullptr;
    uint32_t prep_rb = 48;  // bytes per prepared record: 48 (PRec), or 32 when every value is 1:
                            // {w0, w1, h, s | len << 48} (a third less re-issue traffic)
    uint32_t prep_fmt = 0;  // 33: 32-byte records {key, value, h, s | len << 48} (keys of <= 8 bytes)
    uint32_t dirpf = 0;     // text kernel: L2-prefetch queued misses' directory lines (table > L2)
    // raw-text input (sepo_run_text, NEXT-2): keys = text bytes, n = text bytes; records are the
    // words (maximal runs of non-separator bytes), identified by their start offset. Declined
    // words that do not fit the prepared list set bit (start) in tbm (u32 words over the text).
    uint32_t text = 0;
    uint32_t* tbm = nullptr;
    uint64_t w_begin = 0, w_end = ~0ull;  // text: the 512-byte windows this launch tokenizes
    // wire input (a12, the routed path): record i is the 32-byte WireRec wire[i] (keys of at most
    // 16 bytes, pre-combined values); keys / ko / vals are unused then
    const struct WireRec* wire = nullptr;
};
// A routed record (a12): a key of at most 16 bytes (zero padded) and its pre-combined u64 value.
struct WireRec {
    uint64_t w0, w1, v, len;
};
static_assert(sizeof(WireRec) == 32, "WireRec layout");
}  // namespace sepo

// key_end: key_offsets[n] of a CSR batch (the end of its key bytes), read by the host
// lean_in: COMBINE contiguous batches take insert_lean_kernel (mostly short keys; the host decides)
// long_keys: a CSR COMBINE batch of long keys (URLs): the stream kernel instantiation that reads key
// tails several words per round trip
// *hot_built (optional): whether this launch selected a sampled hot set (its size is the u32 at
// hot_scratch + sepo_hot_count_offset(), clamped to the kernel's capacity)
int sepo_launch_insert(const sepo::Dev& d, const sepo::Batch& b, int mode, int grid, cudaStream_t s, void* hot_scratch,
                       uint32_t halt_slots = 0, uint64_t key_end = 0, bool dir_prefetch = false,
                       bool* hot_built = nullptr, bool lean_in = false, bool long_keys = false);
size_t sepo_hot_count_offset();
int sepo_launch_reinsert(const sepo::Dev& d, const sepo::Batch& b, int grid, cudaStream_t s, bool long_keys = false);
// Router with hot-key pre-combine (a12). Scratch (device, sepo_route_scratch_bytes): hot-set
// discovery scratch, counts [P][grid] at counts_off, bases [P][grid], hot sums [K], then at
// hot_pp_off: hot keys per part [32], hot bases [32], hot cursors [32], long-key counter.
// Pass 0 (discovery + counts; the host scans counts / hot_pp into bases / hot bases), pass 1 (write).
size_t sepo_route_scratch_bytes(uint32_t P, int grid);
void sepo_route_layout(uint32_t P, int grid, size_t* counts_off, size_t* hot_pp_off);
int sepo_launch_route_hot(const sepo::Batch& b, uint32_t P, uint64_t seed, int pass, void* scratch, int grid,
                          sepo::WireRec* out, cudaStream_t s, sepo::WireRec* const* dstp = nullptr);
size_t sepo_hot_scratch_bytes();
int sepo_default_grid(int mode, int n_sms);
int sepo_launch_reprobe(const sepo::Dev& d, const sepo::Batch& b, int mode, int probe, int grid,
                        unsigned long long* tile_counts, cudaStream_t s);
uint64_t sepo_reprobe_tiles(uint64_t n);
int sepo_launch_compact(const sepo::Batch& b, unsigned long long* tile_counts, uint8_t* ok, uint64_t* oko, uint8_t* ov,
                        uint64_t* ovo, uint64_t m, uint64_t kb, uint64_t vb, int grid, cudaStream_t s);
int sepo_launch_tile_popc(const sepo::Batch& b, unsigned long long* tile_counts, int grid, cudaStream_t s);
int sepo_launch_compact_index(const sepo::Batch& b, unsigned long long* tile_counts, uint64_t* idx_out, int grid,
                              cudaStream_t s);
int sepo_launch_partition(const sepo::Batch& b, uint32_t P, uint64_t seed, unsigned long long* counts, uint8_t* ok,
                          uint64_t* oko, uint8_t* ov, unsigned long long* h_counts, int grid, cudaStream_t s);
uint64_t sepo_partition_tiles(uint64_t n);
// map runtime (NEXT-4): pass 0 counts records / key bytes per chunk of text into tc (3 u64 per chunk)
// and scans them; pass 1 writes the compacted CSR (okeys, oko) and, with doc_offsets, u32 doc ids
uint64_t sepo_map_chunks(uint64_t n);
int sepo_launch_map(const uint8_t* text, uint64_t n, int lines, int pass, unsigned long long* tc, const uint64_t* doc_offsets,
                    uint64_t n_docs, uint8_t* okeys, uint64_t* oko, uint32_t* odoc, cudaStream_t s);
int sepo_launch_max_key_len(const uint64_t* ko, uint64_t n, unsigned long long* out, cudaStream_t s);
int sepo_launch_shift_offsets(uint64_t* ko, uint64_t n, const uint64_t* seg_rec, const uint64_t* seg_base, uint32_t n_segs,
                              uint64_t total, cudaStream_t s);
int sepo_launch_seal(const sepo::Dev& d, uint32_t n_slots, cudaStream_t s);
int sepo_launch_evict_copy(const sepo::Dev& d, uint32_t n, uint8_t* dst, int grid, cudaStream_t s);
// (list: a snapshot of the evict list — the overlapped gather may still run when the next eviction's
// classify rewrites d.evict_list)
int sepo_launch_evict_copy_prog(const sepo::Dev& d, uint32_t n, uint8_t* dst, int grid, unsigned int* eprog,
                                const uint32_t* list, cudaStream_t s);
// sample_bytes: tokenize a hot-set sample from the first sample_bytes of the text; 0: reuse the hot
// set an earlier launch of the same job built, if *hot_built says it did (else no hot set).
// *hot_built (in/out, host): set when this launch builds a hot set, cleared when it samples none.
int sepo_launch_insert_text(const sepo::Dev& d, const sepo::Batch& b, int grid, cudaStream_t s, void* hot_scratch,
                            uint64_t sample_bytes, bool* hot_built);
int sepo_launch_lookup_gen(const sepo::Dev& d, const sepo::Batch& b, const uint32_t* pages, uint32_t np,
                           unsigned long long* vals, uint32_t* found, cudaStream_t s);
int sepo_launch_text_bits(const sepo::Dev& d, const sepo::Batch& b, unsigned long long* counter, cudaStream_t s);
int sepo_launch_classify(const sepo::Dev& d, int honor_retain, cudaStream_t s);
int sepo_launch_relink(const sepo::Dev& d, cudaStream_t s);
int sepo_launch_init(const sepo::Dev& d, uint32_t n_slots, cudaStream_t s);
