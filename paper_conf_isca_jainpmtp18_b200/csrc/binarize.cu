// binarize.cu — a1: Binarize encode of a ReLU output (§III-A, §IV-A).
//
// mask bit i = (y[i] > 0): one bit per fp32 (32x).  HBM-bound: reads 4n bytes,
// writes n/8.  Each warp streams a 1024-element chunk (8 coalesced 512-byte LDG.128 waves
// in flight), turns every float4 into a nibble, ORs 8 lanes' nibbles into a 32-bit word
// with three xor-shuffles and stores 32 words (128 B) with one coalesced STG.32 per lane.
#include "common.cuh"
#include "kernels.h"

#ifndef GIST_BIN_CTAS
#define GIST_BIN_CTAS 8
#endif

namespace gist {

namespace {

constexpr int kBinThreads = 256;
constexpr int kChunk = 1024;  // elements per warp iteration = 32 mask words

__device__ __forceinline__ uint32_t nib4(float4 v) {
    return (uint32_t)(v.x > 0.0f) | ((uint32_t)(v.y > 0.0f) << 1) | ((uint32_t)(v.z > 0.0f) << 2) |
           ((uint32_t)(v.w > 0.0f) << 3);
}

__global__ void __launch_bounds__(kBinThreads)
binarize_kernel(const float *__restrict__ y, int64_t n, uint32_t *__restrict__ mask) {
    pdl_enter();
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * kBinThreads + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * kBinThreads) >> 5;
    const int64_t full_chunks = n / kChunk;
    const float4 *y4 = reinterpret_cast<const float4 *>(y);

    for (int64_t c = warp; c < full_chunks; c += nwarps) {
        float4 v[8];
        const float4 *src = y4 + c * (kChunk / 4) + lane;
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = ld_stream_f4(src + 32 * j);
        uint32_t mine = 0;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            // lane l holds elements 128j + 4l .. +3 -> word 4j + (l>>3), nibble (l&7)
            uint32_t w = nib4(v[j]) << (4 * (lane & 7));
            w |= __shfl_xor_sync(kFull, w, 1);
            w |= __shfl_xor_sync(kFull, w, 2);
            w |= __shfl_xor_sync(kFull, w, 4);
            if (j == (lane & 7)) mine = w;
        }
        // lane l owns word 4*(l&7) + (l>>3): a permutation of the chunk's 32 words
        mask[c * 32 + 4 * (lane & 7) + (lane >> 3)] = mine;
    }

    // Ragged tail (< 1024 elements): the last warp of the grid, one word per lane.
    if (warp == nwarps - 1) {
        const int64_t base = full_chunks * kChunk;
        const int64_t words = (n - base + 31) / 32;
        if (lane < words) {
            uint32_t w = 0;
            for (int b = 0; b < 32; ++b) {
                int64_t i = base + 32 * lane + b;
                if (i < n && y[i] > 0.0f) w |= 1u << b;
            }
            mask[base / 32 + lane] = w;
        }
    }
}

}  // namespace

cudaError_t launch_binarize(const float *y, int64_t n, uint32_t *mask, cudaStream_t stream) {
    const int64_t chunks = n / kChunk + 1;
    const int64_t per_block = kBinThreads / 32;
    int64_t blocks = ceil_div(chunks, per_block);
    const int64_t cap = (int64_t)num_sms() * GIST_BIN_CTAS;  // resident 256-thread CTAs per SM
    if (blocks > cap) blocks = cap;
    launch_k(binarize_kernel, (unsigned)blocks, kBinThreads, 0, stream, y, n, mask);
    return cudaPeekAtLastError();
}

}  // namespace gist
