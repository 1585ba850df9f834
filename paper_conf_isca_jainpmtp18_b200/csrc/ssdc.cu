// ssdc.cu — a4/a5: Sparse Storage, Dense Compute (PAPER.md P:158-P:164 §IV-A).
//
// Encode: dense fp32 -> CSR with 256-column rows and uint8 column indices (Narrow Value
// Optimization).  One pass over x (4n bytes read, 5*nnz + 4*rows written).
// Persistent, warp-specialized CTAs (3 per SM) stream 16-row tiles (4096 elements, 16 KB)
// through a 4-stage shared-memory ring filled by 1-D TMA bulk copies (cp.async.bulk +
// mbarrier).  Tiles are claimed in order through an atomic ticket, so every predecessor of a
// tile is held by a running CTA (forward progress).  Roles, linked only by mbarriers:
//   * counter warp: as soon as a tile lands, counts the nonzero bit patterns of its rows
//     (R8), scans the 16 row counts and publishes the tile aggregate — aggregates appear one
//     TMA latency after the ticket, independent of how far the writers are;
//   * look-back warp: decoupled look-back (32 predecessors' 64-bit {status, value}
//     descriptors per round) -> the tile's global offset; publishes the inclusive prefix and
//     the tile's row_end entries;
//   * 4 writer warps: each holds 4 rows in registers (lane: cols [4l,4l+4) and
//     [128+4l,128+4l+4)), takes ranks from warp ballots, compacts the whole tile in place,
//     shifted to the global 16-byte phase, and lane 0 of warp 0 writes the aligned bodies of
//     val/col with TMA bulk stores (cp.async.bulk.global.shared::cta); ragged ends by lanes.
// Decode: a warp expands 4 consecutive rows (whose entries are one contiguous range)
//   through a 4 KB shared-memory row buffer and writes them back with float4 stores.
#include "common.cuh"
#include "kernels.h"
#include "tma.cuh"

#include <mutex>

namespace gist {

namespace {

constexpr int kRow = 256;
constexpr int kEncThreads = 128;  // worker threads (4 warps x 4 rows)
constexpr int kRowsPerWarp = 4;
constexpr int kTileRows = (kEncThreads / 32) * kRowsPerWarp;  // 16
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


__global__ void ssdc_ws_init(uint64_t *ws, int64_t words) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += (int64_t)gridDim.x * blockDim.x)
        ws[i] = 0ull;
}

constexpr int kStages = 4;                       // TMA ring depth per CTA
constexpr int kCtasPerSm = 3;                    // smem/register-limited residency
constexpr int kTileElems = kTileRows * kRow;     // 4096 elements
constexpr uint32_t kTileBytes = kTileElems * 4;  // 16 KB
constexpr int kWarps = kEncThreads / 32;         // writer warps (4 rows each)
constexpr int kCountWarp = kWarps;               // counts every tile as soon as it lands
constexpr int kLbWarp = kWarps + 1;              // first of kLbWarps look-back warps
constexpr int kLbWarps = 1;                      // (more take alternate tiles)
constexpr int kCtaThreads = kEncThreads + 32 + 32 * kLbWarps;

struct __align__(128) EncSmem {
    float tile[kStages][kTileElems + 4];    // TMA destinations; the written tile is compacted in place
    uint8_t colbuf[kTileElems + 16];        // compacted column bytes of the tile being written
    uint64_t full[kStages];                 // TMA landed (or no tile: arrive without bytes)
    uint64_t counted[kStages];              // counter warp -> look-back warp
    uint64_t resolved[kStages];             // look-back warp -> writers
    int64_t ticket[kStages];                // tile index held by each stage
    uint32_t row_cnt[kStages][kTileRows];   // per-row nonzeros
    uint32_t row_excl[kStages][kTileRows];  // tile-local exclusive row offsets
    int64_t excl[kStages];                  // global offset of each stage's tile
    int32_t last_j;                         // CTA-local index of the first "no tile" ticket
};

// Start the TMA bulk load of tile t (a ticket claimed earlier, in order, so every predecessor
// is held by a running CTA) into stage s.  Always completes one arrival on full[s], so the
// counter warp also learns about "no more tiles".  One thread.
__device__ __forceinline__ void load_tile(EncSmem &S, int s, int64_t t, const float *x, int64_t n, int64_t tiles) {
    S.ticket[s] = t;
    uint32_t bytes = 0;
    if (t < tiles) {
        const int64_t avail = n - t * kTileElems;
        bytes = avail >= kTileElems ? kTileBytes : (uint32_t)((avail * 4) & ~15ll);
    }
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&S.full[s], bytes);
    if (bytes) tma_load_1d(S.tile[s], x + t * kTileElems, bytes, &S.full[s]);
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Decoupled look-back by one warp: lane i reads tile base-i.  Sums aggregates up to and
// including the nearest inclusive prefix, re-polling only needed unpublished descriptors.
__device__ __forceinline__ int64_t look_back(const Workspace *ws, int64_t tile, int lane) {
    int64_t excl = 0;
    for (int64_t base = tile - 1;; base -= 32) {
        const int64_t idx = base - lane;
        uint64_t d = (idx >= 0) ? ld_relaxed(&ws->desc[idx]) : kStatusP;  // virtual P(0)
        uint32_t pm, need;
        for (;;) {
            pm = __ballot_sync(kFull, (d >> 62) == 2);
            const uint32_t xm = __ballot_sync(kFull, (d >> 62) == 0);
            need = pm ? (((pm & (0u - pm)) << 1) - 1u) : kFull;
            if (!(xm & need)) break;
            if ((d >> 62) == 0) d = ld_relaxed(&ws->desc[idx]);
        }
        uint64_t v = ((need >> lane) & 1u) ? (d & kValueMask) : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
        excl += (int64_t)v;
        if (pm) return excl;
    }
}

__device__ __forceinline__ void writers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kEncThreads) : "memory"); }

__global__ void __launch_bounds__(kCtaThreads, kCtasPerSm)
ssdc_encode_kernel(const float *__restrict__ x, int64_t n, int64_t rows, int64_t tiles,
                   int32_t *__restrict__ row_end, uint8_t *__restrict__ col, float *__restrict__ val,
                   int64_t capacity, int64_t *__restrict__ nnz_out, Workspace *__restrict__ ws) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    EncSmem &S = *reinterpret_cast<EncSmem *>(smem_raw);
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&S.full[s], 1);
            mbar_init(&S.counted[s], 1);
            mbar_init(&S.resolved[s], 1);
        }
        fence_mbar_init();
        S.last_j = 0x7fffffff;
        for (int s = 0; s < kStages; ++s) load_tile(S, s, atomicAdd(&ws->ticket, 1u), x, n, tiles);
    }
    __syncthreads();

    if (warp == kCountWarp) {
        // ---- counter: nonzero bit patterns (R8) of every row, tile scan, publish aggregate
        for (int j = 0;; ++j) {
            const int s = j % kStages;
            mbar_wait(&S.full[s], (uint32_t)(j / kStages) & 1u);
            const int64_t tile = S.ticket[s];
            if (tile < tiles) {
                float *T = S.tile[s];
                if (tile == tiles - 1) {  // ragged last tile: tail the TMA could not copy, zeros
                    const int64_t avail = n - tile * kTileElems;
                    const int from = avail >= kTileElems ? kTileElems : (int)(((avail * 4) & ~15ll) / 4);
                    for (int i = from + lane; i < kTileElems; i += 32)
                        T[i] = (i < avail) ? x[tile * kTileElems + i] : 0.0f;
                    __syncwarp();
                }
                uint32_t mine = 0;  // lane r ends up with row r's count
#pragma unroll 4
                for (int r = 0; r < kTileRows; ++r) {
                    const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                    const uint4 a = row4[lane], b = row4[32 + lane];
                    const uint32_t c = (a.x != 0u) + (a.y != 0u) + (a.z != 0u) + (a.w != 0u) + (b.x != 0u) +
                                       (b.y != 0u) + (b.z != 0u) + (b.w != 0u);
                    const uint32_t t = __reduce_add_sync(kFull, c);
                    if (lane == r) mine = t;
                }
                uint32_t inc = mine;
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t t = __shfl_up_sync(kFull, inc, d);
                    if (lane >= d) inc += t;
                }
                if (lane < kTileRows) {
                    S.row_cnt[s][lane] = mine;
                    S.row_excl[s][lane] = inc - mine;
                }
                if (lane == 31) st_relaxed(&ws->desc[tile], (tile == 0 ? kStatusP : kStatusA) | (uint64_t)inc);
            }
            __syncwarp();
            if (lane == 0) {
                if (tile >= tiles) *(volatile int32_t *)&S.last_j = j;  // before the arrival
                mbar_arrive(&S.counted[s]);
            }
            if (tile >= tiles) break;
        }
    } else if (warp >= kLbWarp) {
        // ---- look-back: global offset of each counted tile; publish prefix, row ends, nnz.
        // Warp kLbWarp + i resolves the CTA's tiles j = i, i + kLbWarps, ...
        for (int j = warp - kLbWarp;; j += kLbWarps) {
            const int s = j % kStages;
            // poll: past the CTA's last tile no arrival will ever come for this j
            bool ready = false;
            while (!(ready = mbar_test(&S.counted[s], (uint32_t)(j / kStages) & 1u)))
                if (*(volatile int32_t *)&S.last_j < j) break;
            if (!ready) break;
            const int64_t tile = S.ticket[s];
            if (tile < tiles) {
                const int64_t excl = (tile == 0) ? 0 : look_back(ws, tile, lane);
                const uint32_t total = S.row_excl[s][kTileRows - 1] + S.row_cnt[s][kTileRows - 1];
                if (lane == 0) {
                    S.excl[s] = excl;
                    if (tile > 0) st_relaxed(&ws->desc[tile], kStatusP | (uint64_t)(excl + total));
                    if (tile == tiles - 1) *nnz_out = excl + total;
                }
                const int64_t r = tile * kTileRows + lane;
                if (lane < kTileRows && r < rows)
                    row_end[r] = (int32_t)(excl + S.row_excl[s][lane] + S.row_cnt[s][lane]);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&S.resolved[s]);
            if (tile >= tiles) break;
        }
    } else {
        // ---- writers: compact the tile contiguously in place, shifted so smem and global share
        // their 16-byte phase (value k -> T[sv + k] = val[excl + k], column -> colbuf[sc + k]),
        // then TMA bulk-store the aligned bodies; ranks from ballots (lane l holds cols 4l+j
        // "lo" and 128+4l+j "hi", j = 0..3).
        const uint32_t lt = (1u << lane) - 1u;
        for (int j = 0;; ++j) {
            const int s = j % kStages;
            mbar_wait(&S.resolved[s], (uint32_t)(j / kStages) & 1u);
            const int64_t tile = S.ticket[s];
            if (tile >= tiles) break;
            float *T = S.tile[s];
            const int64_t excl = S.excl[s];
            const uint32_t sv = (uint32_t)excl & 3u, sc = (uint32_t)excl & 15u;
            float v[kRowsPerWarp][8];
            uint32_t bal[kRowsPerWarp][8];
#pragma unroll
            for (int r = 0; r < kRowsPerWarp; ++r) {
                const float4 *row4 = reinterpret_cast<const float4 *>(T + (warp * kRowsPerWarp + r) * kRow);
                const float4 a = row4[lane], b = row4[32 + lane];
                v[r][0] = a.x; v[r][1] = a.y; v[r][2] = a.z; v[r][3] = a.w;
                v[r][4] = b.x; v[r][5] = b.y; v[r][6] = b.z; v[r][7] = b.w;
#pragma unroll
                for (int k = 0; k < 8; ++k) bal[r][k] = __ballot_sync(kFull, __float_as_uint(v[r][k]) != 0u);
            }
            writers_sync();  // whole tile in registers (and the previous bulk store read out)
#pragma unroll
            for (int r = 0; r < kRowsPerWarp; ++r) {
                const uint32_t q0 = sv + S.row_excl[s][warp * kRowsPerWarp + r];
                uint32_t p_lo = q0 + __popc(bal[r][0] & lt) + __popc(bal[r][1] & lt) + __popc(bal[r][2] & lt) +
                                __popc(bal[r][3] & lt);
                uint32_t p_hi = q0 + __popc(bal[r][0]) + __popc(bal[r][1]) + __popc(bal[r][2]) + __popc(bal[r][3]) +
                                __popc(bal[r][4] & lt) + __popc(bal[r][5] & lt) + __popc(bal[r][6] & lt) +
                                __popc(bal[r][7] & lt);
                uint8_t *cb = S.colbuf + sc - sv;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t on = (bal[r][k] >> lane) & 1u;
                    if (on) {
                        T[p_lo] = v[r][k];
                        cb[p_lo] = (uint8_t)(4 * lane + k);
                    }
                    p_lo += on;
                }
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t on = (bal[r][4 + k] >> lane) & 1u;
                    if (on) {
                        T[p_hi] = v[r][4 + k];
                        cb[p_hi] = (uint8_t)(128 + 4 * lane + k);
                    }
                    p_hi += on;
                }
            }
            fence_proxy_async_smem();  // generic smem writes before the async-proxy bulk store
            writers_sync();
            if (warp == 0) {
                const int64_t total = S.row_excl[s][kTileRows - 1] + S.row_cnt[s][kTileRows - 1];
                int64_t lim = total;
                if (excl + lim > capacity) lim = capacity > excl ? capacity - excl : 0;
                const int64_t hv = (4 - sv) & 3, hc = (16 - sc) & 15;  // heads up to 16-B alignment
                const int64_t bv = lim > hv ? (lim - hv) & ~3ll : 0, bc = lim > hc ? (lim - hc) & ~15ll : 0;
                // ragged ends: < 4 values and < 16 columns at each end
                const int64_t k0 = lane, k1 = hv + bv + lane, k2 = hc + bc + lane;
                if (k0 < hv && k0 < lim) val[excl + k0] = T[sv + k0];
                if (lane < 4 && k1 < lim) val[excl + k1] = T[sv + k1];
                if (k0 < hc && k0 < lim) col[excl + k0] = S.colbuf[sc + k0];
                if (lane < 16 && k2 < lim) col[excl + k2] = S.colbuf[sc + k2];
                __syncwarp();
                if (lane == 0) {
                    if (bv) tma_store_1d(val + excl + hv, T + sv + hv, (uint32_t)(4 * bv));
                    if (bc) tma_store_1d(col + excl + hc, S.colbuf + sc + hc, (uint32_t)bc);
                    bulk_commit();
                    bulk_wait_read();  // stage + colbuf read out
                    load_tile(S, s, atomicAdd(&ws->ticket, 1u), x, n, tiles);  // refill this stage
                }
                __syncwarp();
            }
        }
        if (threadIdx.x == 0) bulk_wait_all();
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
    static std::once_flag attr_once;
    std::call_once(attr_once, [] {
        cudaFuncSetAttribute(ssdc_encode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(EncSmem));
    });
    int64_t grid = (int64_t)num_sms() * kCtasPerSm;  // persistent, smem-limited residency
    if (grid > tiles) grid = tiles;
    ssdc_encode_kernel<<<(unsigned)grid, kCtaThreads, sizeof(EncSmem), s>>>(
        x, n, rows, tiles, row_end, col, val, capacity, nnz, reinterpret_cast<Workspace *>(workspace));
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
