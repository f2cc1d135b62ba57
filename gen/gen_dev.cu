// gen_dev.cu — device implementation of the synthetic input generators (same gen_common.h as
// gen_host.cpp, so record j is byte-identical on both sides). Test/bench infrastructure only:
// the product library (libsepo.so) neither links nor includes this.
#include "gen_common.h"
#include <cuda_runtime.h>
#include <cub/device/device_scan.cuh>

namespace {
__global__ void k_lens(gen_params p, uint64_t j0, uint64_t cnt, uint64_t* offs) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x) {
        offs[i + 1] = gen_key_len_of_rank(&p, gen_rank(&p, j0 + i));
        if (i == 0) offs[0] = 0;
    }
}
__global__ void k_keys(gen_params p, uint64_t j0, uint64_t cnt, const uint64_t* offs, uint8_t* keys, uint8_t* vals) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t j = j0 + i;
        uint64_t r = gen_rank(&p, j);
        uint64_t o = offs[i];
        uint32_t L = (uint32_t)(offs[i + 1] - o);
        uint8_t buf[256];
        gen_key_spell(&p, r, L, buf);
        for (uint32_t q = 0; q < L; ++q) keys[o + q] = buf[q];
        if (vals) {
            if (p.family == GEN_PAIRS) reinterpret_cast<uint64_t*>(vals)[i] = gen_pair_val(&p, j);
            else if (p.with_doc_vals) reinterpret_cast<uint32_t*>(vals)[i] = (uint32_t)gen_doc_of(&p, j);
        }
    }
}
__global__ void k_ranks(gen_params p, uint64_t j0, uint64_t cnt, uint64_t* ranks) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x)
        ranks[i] = gen_rank(&p, j0 + i);
}
// raw text of records [j0, j0+cnt): word j (CSR keys/offs) at text[offs[i] - offs[0] + i], then its separator
__global__ void k_text(gen_params p, uint64_t j0, uint64_t cnt, const uint64_t* offs, const uint8_t* keys, uint8_t* text) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t o = offs[i] - offs[0], e = offs[i + 1] - offs[0];
        for (uint64_t q = o; q < e; ++q) text[q + i] = keys[q];
        text[e + i] = gen_text_sep(&p, j0 + i);
    }
}
int grid_for(uint64_t cnt) {
    uint64_t g = (cnt + 255) / 256;
    return (int)(g < 148 * 64 ? (g ? g : 1) : 148 * 64);
}
}  // namespace

extern "C" {
// p: host struct whose cum/doc_start pointers are DEVICE pointers. offs: device, cnt+1 u64.
// temp: device scratch of temp_bytes (query with temp == NULL: returns required bytes).
int64_t gen_offsets_dev(const gen_params* p, uint64_t j0, uint64_t cnt, uint64_t* offs, void* temp, uint64_t temp_bytes, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    size_t need = 0;
    cub::DeviceScan::InclusiveSum(nullptr, need, offs + 1, offs + 1, (int64_t)cnt, s);
    if (temp == nullptr) return (int64_t)need;
    if (temp_bytes < need) return -1;
    if (cnt == 0) { cudaMemsetAsync(offs, 0, 8, s); return 0; }
    k_lens<<<grid_for(cnt), 256, 0, s>>>(*p, j0, cnt, offs);
    cub::DeviceScan::InclusiveSum(temp, need, offs + 1, offs + 1, (int64_t)cnt, s);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
int gen_keys_dev(const gen_params* p, uint64_t j0, uint64_t cnt, const uint64_t* offs, uint8_t* keys, uint8_t* vals, void* stream) {
    if (cnt == 0) return 0;
    k_keys<<<grid_for(cnt), 256, 0, (cudaStream_t)stream>>>(*p, j0, cnt, offs, keys, vals);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
int gen_text_dev(const gen_params* p, uint64_t j0, uint64_t cnt, const uint64_t* offs, const uint8_t* keys, uint8_t* text,
                 void* stream) {
    if (cnt == 0) return 0;
    k_text<<<grid_for(cnt), 256, 0, (cudaStream_t)stream>>>(*p, j0, cnt, offs, keys, text);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
int gen_ranks_dev(const gen_params* p, uint64_t j0, uint64_t cnt, uint64_t* ranks, void* stream) {
    if (cnt == 0) return 0;
    k_ranks<<<grid_for(cnt), 256, 0, (cudaStream_t)stream>>>(*p, j0, cnt, ranks);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
}
