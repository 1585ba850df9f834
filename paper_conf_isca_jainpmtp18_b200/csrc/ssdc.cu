// ssdc.cu — a4/a5: Sparse Storage, Dense Compute (PAPER.md P:158-P:164 §IV-A).
//
// Encode: dense fp32 -> CSR with 256-column rows and uint8 column indices (Narrow Value
// Optimization).  One pass over x (4n bytes read, 5*nnz + 4*rows written):
//   * a CTA owns a tile of 32 rows (8192 elements); tiles are claimed in order through an
//     atomic ticket so every predecessor is already running (forward progress);
//   * each warp holds 4 rows in registers (8 LDG.128 per lane), counts nonzero bit
//     patterns per half-row and scans 4 rows at once with one packed 8-bit-lane
//     shuffle scan; warp 0 scans the tile's 32 row counts;
//   * the tile's global offset comes from a decoupled look-back over the predecessors'
//     {aggregate, inclusive-prefix} descriptors (one 64-bit word each: 2-bit status +
//     value), read 32 at a time by warp 0;
//   * rows are then written straight from registers: row_end, and each lane's nonzeros
//     at consecutive offsets (stores of a warp fall in one contiguous output range).
// Decode: a warp expands 4 consecutive rows (whose entries are one contiguous range)
//   through a 4 KB shared-memory row buffer and writes them back with float4 stores.
#include "common.cuh"
#include "kernels.h"

namespace gist {

namespace {

constexpr int kRow = 256;
constexpr int kEncThreads = 256;
constexpr int kRowsPerWarp = 4;
constexpr int kTileRows = (kEncThreads / 32) * kRowsPerWarp;  // 32
constexpr uint64_t kStatusA = 1ull << 62;                    // aggregate available
constexpr uint64_t kStatusP = 2ull << 62;                    // inclusive prefix available
constexpr uint64_t kValueMask = (1ull << 62) - 1;

struct Workspace {
    uint32_t ticket;
    uint32_t pad;
    uint64_t desc[1];  // [tiles]
};

__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint32_t nz(float v) { return __float_as_uint(v) != 0u; }

__global__ void ssdc_ws_init(uint64_t *ws, int64_t words) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += (int64_t)gridDim.x * blockDim.x)
        ws[i] = 0ull;
}

__global__ void __launch_bounds__(kEncThreads)
ssdc_encode_kernel(const float *__restrict__ x, int64_t n, int64_t rows, int64_t tiles,
                   int32_t *__restrict__ row_end, uint8_t *__restrict__ col, float *__restrict__ val,
                   int64_t capacity, int64_t *__restrict__ nnz_out, Workspace *__restrict__ ws) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_row_cnt[kTileRows];
    __shared__ uint32_t s_row_excl[kTileRows];
    __shared__ int64_t s_prefix;

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_tile = atomicAdd(&ws->ticket, 1u);
    __syncthreads();
    const int64_t tile = s_tile;
    if (tile >= tiles) return;

    // ---- load 4 rows per warp: lane holds cols [4l, 4l+4) and [128+4l, 128+4l+4)
    const int64_t row0 = tile * kTileRows + warp * kRowsPerWarp;
    float4 lo[kRowsPerWarp], hi[kRowsPerWarp];
#pragma unroll
    for (int r = 0; r < kRowsPerWarp; ++r) {
        const int64_t base = (row0 + r) * kRow;
        if (base + kRow <= n) {
            lo[r] = ld_stream_f4(reinterpret_cast<const float4 *>(x + base) + lane);
            hi[r] = ld_stream_f4(reinterpret_cast<const float4 *>(x + base + 128) + lane);
        } else {  // ragged last row (or beyond the end): scalar, zero-filled
            float t[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int64_t i = base + (j < 4 ? 4 * lane + j : 128 + 4 * lane + j - 4);
                t[j] = (i < n) ? x[i] : 0.0f;
            }
            lo[r] = make_float4(t[0], t[1], t[2], t[3]);
            hi[r] = make_float4(t[4], t[5], t[6], t[7]);
        }
    }

    // ---- per-lane counts, 4 rows x {lo, hi} packed into two 4x8-bit words, warp scan
    uint32_t m_lo[kRowsPerWarp], m_hi[kRowsPerWarp];
    uint32_t pk_lo = 0, pk_hi = 0;
#pragma unroll
    for (int r = 0; r < kRowsPerWarp; ++r) {
        m_lo[r] = nz(lo[r].x) | (nz(lo[r].y) << 1) | (nz(lo[r].z) << 2) | (nz(lo[r].w) << 3);
        m_hi[r] = nz(hi[r].x) | (nz(hi[r].y) << 1) | (nz(hi[r].z) << 2) | (nz(hi[r].w) << 3);
        pk_lo |= (uint32_t)__popc(m_lo[r]) << (8 * r);
        pk_hi |= (uint32_t)__popc(m_hi[r]) << (8 * r);
    }
    uint32_t in_lo = pk_lo, in_hi = pk_hi;  // inclusive scans (each 8-bit lane <= 128)
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t a = __shfl_up_sync(kFull, in_lo, d);
        const uint32_t b = __shfl_up_sync(kFull, in_hi, d);
        if (lane >= d) {
            in_lo += a;
            in_hi += b;
        }
    }
    const uint32_t tot_lo = __shfl_sync(kFull, in_lo, 31);
    const uint32_t tot_hi = __shfl_sync(kFull, in_hi, 31);
    if (lane < kRowsPerWarp)
        s_row_cnt[warp * kRowsPerWarp + lane] = ((tot_lo >> (8 * lane)) & 0xffu) + ((tot_hi >> (8 * lane)) & 0xffu);
    __syncthreads();

    // ---- warp 0: tile-level row scan + decoupled look-back for the tile's offset
    if (warp == 0) {
        const uint32_t c = s_row_cnt[lane];
        uint32_t inc = c;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t t = __shfl_up_sync(kFull, inc, d);
            if (lane >= d) inc += t;
        }
        s_row_excl[lane] = inc - c;
        const uint64_t total = __shfl_sync(kFull, inc, 31);
        int64_t excl = 0;
        if (tile == 0) {
            if (lane == 0) st_relaxed(&ws->desc[0], kStatusP | total);
        } else {
            if (lane == 0) st_relaxed(&ws->desc[tile], kStatusA | total);
            // Look back over predecessors base, base-1, ... 32 at a time (lane i reads
            // tile base-i).  Sum aggregates up to and including the nearest inclusive
            // prefix; spin only on descriptors that are still unpublished and needed.
            int64_t base = tile - 1;
            while (true) {
                const int64_t idx = base - lane;
                uint64_t d = (idx >= 0) ? ld_relaxed(&ws->desc[idx]) : kStatusP;  // virtual P(0)
                uint32_t pmask, need;
                while (true) {
                    pmask = __ballot_sync(kFull, (d >> 62) == 2);
                    const uint32_t xmask = __ballot_sync(kFull, (d >> 62) == 0);
                    need = pmask ? (((pmask & (0u - pmask)) << 1) - 1u) : kFull;
                    if (!(xmask & need)) break;
                    if ((d >> 62) == 0) d = ld_relaxed(&ws->desc[idx]);
                }
                uint64_t v = ((need >> lane) & 1u) ? (d & kValueMask) : 0ull;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
                excl += (int64_t)v;
                if (pmask) break;
                base -= 32;
            }
            if (lane == 0) st_relaxed(&ws->desc[tile], kStatusP | (uint64_t)(excl + (int64_t)total));
        }
        if (lane == 0) {
            s_prefix = excl;
            if (tile == tiles - 1) *nnz_out = excl + (int64_t)total;
        }
        // row ends for the tile
        const int64_t r = tile * kTileRows + lane;
        if (r < rows) row_end[r] = (int32_t)(excl + inc);
    }
    __syncthreads();

    // ---- scatter this warp's nonzeros (ascending column order within each row)
    const int64_t prefix = s_prefix;
#pragma unroll
    for (int r = 0; r < kRowsPerWarp; ++r) {
        const int rr = warp * kRowsPerWarp + r;
        const int64_t row_base = prefix + s_row_excl[rr];
        const uint32_t ex_lo = ((in_lo >> (8 * r)) & 0xffu) - __popc(m_lo[r]);
        const uint32_t ex_hi = ((in_hi >> (8 * r)) & 0xffu) - __popc(m_hi[r]);
        const uint32_t t_lo = (tot_lo >> (8 * r)) & 0xffu;
        int64_t o = row_base + ex_lo;
        const float vl[4] = {lo[r].x, lo[r].y, lo[r].z, lo[r].w};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            if ((m_lo[r] >> j) & 1u) {
                if (o < capacity) {
                    col[o] = (uint8_t)(4 * lane + j);
                    val[o] = vl[j];
                }
                ++o;
            }
        }
        o = row_base + t_lo + ex_hi;
        const float vh[4] = {hi[r].x, hi[r].y, hi[r].z, hi[r].w};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            if ((m_hi[r] >> j) & 1u) {
                if (o < capacity) {
                    col[o] = (uint8_t)(128 + 4 * lane + j);
                    val[o] = vh[j];
                }
                ++o;
            }
        }
    }
}

constexpr int kDecThreads = 256;
constexpr int kDecRows = 4;  // rows per warp iteration

__global__ void __launch_bounds__(kDecThreads)
ssdc_decode_kernel(const int32_t *__restrict__ row_end, const uint8_t *__restrict__ col,
                   const float *__restrict__ val, int64_t n, int64_t rows, float *__restrict__ x) {
    __shared__ __align__(16) float s_buf[kDecThreads / 32][kDecRows * kRow];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    float *buf = s_buf[warp];
    const int64_t groups = (rows + kDecRows - 1) / kDecRows;
    const int64_t gwarp = ((int64_t)blockIdx.x * kDecThreads + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * kDecThreads) >> 5;

    for (int64_t g = gwarp; g < groups; g += nwarps) {
        const int64_t r0 = g * kDecRows;
        // lanes 0..4 fetch the row boundaries: bound[j] = end of row r0-1+j
        int32_t bnd = 0;
        if (lane <= kDecRows) {
            const int64_t r = r0 - 1 + lane;
            bnd = (r < 0) ? 0 : (r < rows ? row_end[r] : row_end[rows - 1]);
        }
        const int32_t b0 = __shfl_sync(kFull, bnd, 0), b1 = __shfl_sync(kFull, bnd, 1);
        const int32_t b2 = __shfl_sync(kFull, bnd, 2), b3 = __shfl_sync(kFull, bnd, 3);
        const int32_t b4 = __shfl_sync(kFull, bnd, 4);
        // zero the 4-row buffer
        float4 *b4p = reinterpret_cast<float4 *>(buf);
#pragma unroll
        for (int j = 0; j < kDecRows * kRow / 4 / 32; ++j) b4p[lane + 32 * j] = make_float4(0.f, 0.f, 0.f, 0.f);
        __syncwarp();
        for (int32_t k = b0 + lane; k < b4; k += 32) {
            const int rr = (k >= b1) + (k >= b2) + (k >= b3);
            buf[rr * kRow + col[k]] = val[k];
        }
        __syncwarp();
        const int64_t base = r0 * kRow;
        if (base + kDecRows * kRow <= n) {
            float4 *dst = reinterpret_cast<float4 *>(x + base);
#pragma unroll
            for (int j = 0; j < kDecRows * kRow / 4 / 32; ++j) dst[lane + 32 * j] = b4p[lane + 32 * j];
        } else {
            for (int j = lane; j < kDecRows * kRow; j += 32)
                if (base + j < n) x[base + j] = buf[j];
        }
        __syncwarp();
    }
}

}  // namespace

size_t ssdc_workspace_bytes(int64_t n) {
    const int64_t rows = (n + kRow - 1) / kRow;
    const int64_t tiles = (rows + kTileRows - 1) / kTileRows;
    return 8 + 8 * (size_t)(tiles > 0 ? tiles : 1);
}

cudaError_t launch_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val,
                               int64_t capacity, int64_t *nnz, void *workspace, cudaStream_t s) {
    const int64_t rows = (n + kRow - 1) / kRow;
    const int64_t tiles = (rows + kTileRows - 1) / kTileRows;
    const int64_t ws_words = (int64_t)ssdc_workspace_bytes(n) / 8;
    int64_t iblocks = ceil_div(ws_words, 256);
    if (iblocks > 1024) iblocks = 1024;
    ssdc_ws_init<<<(unsigned)iblocks, 256, 0, s>>>(reinterpret_cast<uint64_t *>(workspace), ws_words);
    ssdc_encode_kernel<<<(unsigned)tiles, kEncThreads, 0, s>>>(x, n, rows, tiles, row_end, col, val, capacity,
                                                               nnz, reinterpret_cast<Workspace *>(workspace));
    return cudaPeekAtLastError();
}

cudaError_t launch_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n, float *x,
                               cudaStream_t s) {
    const int64_t rows = (n + kRow - 1) / kRow;
    const int64_t groups = (rows + kDecRows - 1) / kDecRows;
    int64_t blocks = ceil_div(groups, kDecThreads / 32);
    const int64_t cap = (int64_t)num_sms() * 6;
    if (blocks > cap) blocks = cap;
    ssdc_decode_kernel<<<(unsigned)blocks, kDecThreads, 0, s>>>(row_end, col, val, n, rows, x);
    return cudaPeekAtLastError();
}

}  // namespace gist
