// ssdc.cu — a4/a5: Sparse Storage, Dense Compute (PAPER.md P:158-P:164 §IV-A).
//
// Encode: dense fp32 -> CSR with 256-column rows and uint8 column indices (Narrow Value
// Optimization).  One pass over x (4n bytes read, 5*nnz + 4*rows written).
// Persistent, warp-specialized CTAs (2 per SM, 9 warps), all roles linked by mbarriers:
//   * producer warp: claims tiles (16 rows = 4096 elements = 16 KB) in ticket order — so every
//     predecessor of a tile is held by a running CTA (forward progress) — and keeps a 4-stage
//     raw ring full with 1-D TMA bulk copies (cp.async.bulk + mbarrier complete_tx);
//   * counter warp: as soon as a tile lands, counts the nonzero bit patterns of its rows (R8),
//     scans the 16 row counts and publishes the tile aggregate (so aggregates appear one TMA
//     latency after the ticket);
//   * look-back warp: decoupled look-back over 64-bit {status, value} descriptors, 32 per
//     round -> the tile's global offset; publishes the inclusive prefix and row_end;
//   * 4 compactor warps (4 rows each): rank nonzeros with warp ballots (lane l holds cols [4l,4l+4) and
//     [128+4l,128+4l+4)), move them into a variable-size (wrapping) pending ring in smem and
//     release the raw stage at once — the raw ring turns over at TMA speed while compacted
//     tiles (~1/5 of the raw bytes at 80% sparsity) wait for their offsets;
//   * 2 store warps: copy each resolved tile from the pending ring to val/col with coalesced
//     stores, then release its ring space and queue slot, in order.
// Decode: a warp expands 4 consecutive rows (whose entries are one contiguous range)
//   through a 4 KB shared-memory row buffer and writes them back with float4 stores.
#include "common.cuh"
#include "kernels.h"
#include "tma.cuh"

#include <mutex>

namespace gist {

namespace {

constexpr int kRow = 256;
constexpr int kEncThreads = 128;  // compactor threads (4 warps x 4 rows)
constexpr int kRowsPerWarp = 4;
constexpr int kTileRows = (kEncThreads / 32) * kRowsPerWarp;  // 16
constexpr uint64_t kStatusA = 1ull << 62;                    // aggregate available
constexpr uint64_t kStatusP = 2ull << 62;                    // inclusive prefix available
constexpr uint64_t kValueMask = (1ull << 62) - 1;

struct Workspace {
    uint32_t ticket;
    uint32_t pad;
    uint64_t desc[1];  // [tiles * kDescStride]
};

#ifndef GIST_SSDC_DESC_STRIDE
#define GIST_SSDC_DESC_STRIDE 1
#endif
// Descriptor spacing in 64-bit words (1: 16 tiles per 128-B L2 line).
constexpr int kDescStride = GIST_SSDC_DESC_STRIDE;
__device__ __forceinline__ uint64_t *desc_at(Workspace *ws, int64_t tile) { return &ws->desc[tile * kDescStride]; }

__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}


#ifdef GIST_SSDC_TRACE
// Timing experiment only: per-tile hand-off timestamps (%globaltimer, ns) for the first
// kTraceCtas CTAs: [cta][j][event], events 0 claim, 1 landed, 2 counted, 3 resolved,
// 4 compacted, 5 stored.
constexpr int kTraceCtas = 4, kTraceTiles = 256;
__device__ uint64_t *g_trace = nullptr;
__device__ __forceinline__ void trace(int j, int ev) {
    if (g_trace && blockIdx.x < kTraceCtas && j < kTraceTiles) {
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_trace[((int64_t)blockIdx.x * kTraceTiles + j) * 8 + ev] = t;
    }
}
#define TRACE(j, ev) trace(j, ev)
#else
#define TRACE(j, ev)
#endif

__global__ void ssdc_ws_init(uint64_t *ws, int64_t words) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += (int64_t)gridDim.x * blockDim.x)
        ws[i] = 0ull;
}

#ifndef GIST_SSDC_STAGES
#define GIST_SSDC_STAGES 4
#endif
#ifndef GIST_SSDC_RING
#define GIST_SSDC_RING 8192
#endif
#ifndef GIST_SSDC_CTAS
#define GIST_SSDC_CTAS 2
#endif
#ifndef GIST_SSDC_COUNTERS
#define GIST_SSDC_COUNTERS 2
#endif
#ifndef GIST_SSDC_LBS
#define GIST_SSDC_LBS 2
#endif
constexpr int kStages = GIST_SSDC_STAGES;         // raw TMA ring (16 KB tiles)
constexpr int kRing = GIST_SSDC_RING;            // pending ring entries (compacted, awaiting offset)
#ifndef GIST_SSDC_QUEUE
#define GIST_SSDC_QUEUE 16
#endif
constexpr int kQ = GIST_SSDC_QUEUE;              // per-CTA tile queue slots (counted .. stored)
constexpr int kCtasPerSm = GIST_SSDC_CTAS;
constexpr int kTileElems = kTileRows * kRow;     // 4096 elements
constexpr uint32_t kTileBytes = kTileElems * 4;  // 16 KB
constexpr int kWarps = kEncThreads / 32;         // compactor warps (kRowsPerWarp rows each)
constexpr int kCountWarp = kWarps;               // first of kCountWarps counters (alternate tiles)
constexpr int kCountWarps = GIST_SSDC_COUNTERS;
constexpr int kLbWarp = kCountWarp + kCountWarps;  // first of kLbWarps look-back warps (alternate tiles)
constexpr int kLbWarps = GIST_SSDC_LBS;
constexpr int kProdWarp = kLbWarp + kLbWarps;    // claims tickets, issues TMA loads
constexpr int kStoreWarp = kProdWarp + 1;        // first of kStoreWarps store warps
constexpr int kStoreWarps = 2;
constexpr int kCtaThreads = 32 * (kStoreWarp + kStoreWarps);
static_assert((kRing & (kRing - 1)) == 0 && kRing >= kTileRows * kRow, "pending ring: power of two >= one tile");
// Each mbarrier phase must be awaited by one warp only (test_wait.parity on a phase that has not
// started would alias the previous one), so role warps that alternate tiles must own disjoint
// stages / queue slots.
static_assert(kStages % kCountWarps == 0, "counter warps must own disjoint raw stages");
static_assert(kQ % kLbWarps == 0, "look-back warps must own disjoint queue slots");

struct __align__(128) EncSmem {
    float tile[kStages][kTileElems];  // raw tiles (TMA destinations)
    float vring[kRing];               // compacted values, tile-local order
    uint8_t cring[kRing];             // compacted column bytes
    uint64_t full[kStages];           // TMA landed (or "no tile" arrival)
    uint64_t empty[kStages];          // compactors done with the raw tile
    uint64_t counted[kQ];             // counter -> look-back, compactors
    uint64_t resolved[kQ];            // look-back -> storers
    uint64_t compacted[kQ];           // compactors -> storers
    int64_t st_ticket[kStages];       // tile index per raw stage
    int64_t q_ticket[kQ];             // tile index per queue slot
    uint32_t row_cnt[kQ][kTileRows];  // per-row nonzeros
    uint32_t row_excl[kQ][kTileRows]; // tile-local exclusive row offsets
    uint32_t total[kQ];               // tile nonzeros
    int64_t excl[kQ];                 // global offset of the tile
    uint32_t pos[kQ];                 // ring offset of the tile's compacted entries
    int64_t ring_end[kQ];             // monotonic ring position after the tile
    int64_t alloc_pos;                // monotonic ring allocation cursor (compactor leader)
    unsigned long long free_pos;      // monotonic ring release cursor (storers; atomic access)
    int32_t stored;                   // tiles fully stored by this CTA (atomic access)
    int32_t last_j;                   // CTA-local index of the "no more tiles" ticket (atomic access)
};

// Start the TMA bulk load of tile t (claimed in ticket order) into stage s; always one arrival
// on full[s] (zero bytes when there is no tile), so consumers also learn about the end.
__device__ __forceinline__ void load_tile(EncSmem &S, int s, int64_t t, const float *x, int64_t n, int64_t tiles) {
    S.st_ticket[s] = t;
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
// On reaching that prefix the warp also publishes the inclusive prefixes of the aggregate-only
// tiles it summed over in that round (their values follow from it; every writer writes the same
// value), so the prefix frontier advances by up to 31 tiles per look-back.
__device__ __forceinline__ int64_t look_back(Workspace *ws, int64_t tile, int lane, int *rounds = nullptr,
                                             int *polls = nullptr) {
    int64_t excl = 0;
    for (int64_t base = tile - 1;; base -= 32) {
        if (rounds) ++*rounds;
        const int64_t idx = base - lane;
        uint64_t d = (idx >= 0) ? ld_relaxed(desc_at(ws, idx)) : kStatusP;  // virtual P(0)
        uint32_t pm, need;
        for (;;) {
            pm = __ballot_sync(kFull, (d >> 62) == 2);
            const uint32_t xm = __ballot_sync(kFull, (d >> 62) == 0);
            need = pm ? (((pm & (0u - pm)) << 1) - 1u) : kFull;
            if (!(xm & need)) break;
            if (polls) ++*polls;
            if ((d >> 62) == 0) d = ld_relaxed(desc_at(ws, idx));
        }
        const uint64_t v = ((need >> lane) & 1u) ? (d & kValueMask) : 0ull;
        if (pm) {
            uint64_t suf = v;  // suffix sum over lanes [lane, first P]: inclusive prefix of tile base-lane
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t t = __shfl_down_sync(kFull, suf, o);
                if (lane + o < 32) suf += t;
            }
            const int first_p = __ffs(pm) - 1;
            if (lane < first_p && idx >= 0) st_relaxed(desc_at(ws, idx), kStatusP | suf);
            return excl + (int64_t)__shfl_sync(kFull, suf, 0);
        }
        uint64_t w = v;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) w += __shfl_xor_sync(kFull, w, o);
        excl += (int64_t)w;
    }
}

// Cross-role flags in shared memory: release (fence, then atomic store) / acquire (atomic load,
// then fence), so the hand-offs that are not mbarrier phases are ordered like them.
__device__ __forceinline__ int32_t flag_ld(int32_t *p) {
    const int32_t v = atomicAdd(p, 0);
    __threadfence_block();
    return v;
}
__device__ __forceinline__ void flag_st(int32_t *p, int32_t v) {
    __threadfence_block();
    atomicExch(p, v);
}
__device__ __forceinline__ int64_t flag_ld64(unsigned long long *p) {
    const unsigned long long v = atomicAdd(p, 0ull);
    __threadfence_block();
    return (int64_t)v;
}
__device__ __forceinline__ void flag_st64(unsigned long long *p, int64_t v) {
    __threadfence_block();
    atomicExch(p, (unsigned long long)v);
}

__device__ __forceinline__ void compactors_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kEncThreads) : "memory"); }
__device__ __forceinline__ void storers_sync() { asm volatile("bar.sync 2, %0;" ::"n"(32 * kStoreWarps) : "memory"); }

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
            mbar_init(&S.empty[s], kWarps);
        }
        for (int q = 0; q < kQ; ++q) {
            mbar_init(&S.counted[q], 1);
            mbar_init(&S.resolved[q], 1);
            mbar_init(&S.compacted[q], kWarps);
        }
        S.alloc_pos = 0;
        S.free_pos = 0;
        S.stored = 0;
        S.last_j = 0x7fffffff;
        fence_mbar_init();
    }
    __syncthreads();

    if (warp == kProdWarp) {
        // ---- producer: keep the raw ring full, in ticket order.  The next ticket is claimed
        // while waiting for a free stage, so the atomic's round trip is off the refill path.
        if (lane == 0) {
            int64_t t = atomicAdd(&ws->ticket, 1u);
            for (int j = 0;; ++j) {
                const int s = j % kStages;
                if (j >= kStages) mbar_wait(&S.empty[s], (uint32_t)(j / kStages - 1) & 1u);
                TRACE(j, 0);
                load_tile(S, s, t, x, n, tiles);
                if (t >= tiles) break;
                t = atomicAdd(&ws->ticket, 1u);
            }
        }
    } else if (warp >= kCountWarp && warp < kCountWarp + kCountWarps) {
        // ---- counters (alternate tiles): nonzero bit patterns (R8) of every row, tile scan,
        // publish the aggregate as soon as the tile lands
        for (int j = warp - kCountWarp;; j += kCountWarps) {
            const int s = j % kStages, q = j % kQ;
            bool ready;  // sleep-wait; past the CTA's last tile no arrival ever comes for this j
            while (!(ready = mbar_try(&S.full[s], (uint32_t)(j / kStages) & 1u, 1000)))
                if (flag_ld(&S.last_j) < j) break;
            if (!ready) break;
            if (lane == 0) TRACE(j, 1);
            while (j - flag_ld(&S.stored) >= kQ) __nanosleep(64);  // queue slot still held by an unstored tile
            const int64_t tile = S.st_ticket[s];
            if (lane == 0) S.q_ticket[q] = tile;

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
#pragma unroll
                for (int r = 0; r < kTileRows; r += 2) {  // two rows per reduction (16-bit fields)
                    const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                    const uint4 a = row4[lane], b = row4[32 + lane], c = row4[64 + lane], d = row4[96 + lane];
                    const uint32_t c0 = (a.x != 0u) + (a.y != 0u) + (a.z != 0u) + (a.w != 0u) + (b.x != 0u) +
                                        (b.y != 0u) + (b.z != 0u) + (b.w != 0u);
                    const uint32_t c1 = (c.x != 0u) + (c.y != 0u) + (c.z != 0u) + (c.w != 0u) + (d.x != 0u) +
                                        (d.y != 0u) + (d.z != 0u) + (d.w != 0u);
                    const uint32_t t = __reduce_add_sync(kFull, c0 | (c1 << 16));
                    if (lane == r) mine = t & 0xffffu;
                    if (lane == r + 1) mine = t >> 16;
                }
                uint32_t inc = mine;
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t t = __shfl_up_sync(kFull, inc, d);
                    if (lane >= d) inc += t;
                }
                if (lane < kTileRows) {
                    S.row_cnt[q][lane] = mine;
                    S.row_excl[q][lane] = inc - mine;
                }
                if (lane == 31) {
                    S.total[q] = inc;
                    st_relaxed(desc_at(ws, tile), (tile == 0 ? kStatusP : kStatusA) | (uint64_t)inc);
                }
            }
            __syncwarp();
            if (lane == 0) {
                if (tile >= tiles) flag_st(&S.last_j, j);  // before the arrival
                TRACE(j, 2);
                mbar_arrive(&S.counted[q]);
            }
            if (tile >= tiles) break;
        }
    } else if (warp >= kLbWarp && warp < kLbWarp + kLbWarps) {
        // ---- look-back (alternate tiles): global offset of each counted tile; publish the
        // inclusive prefix, row ends and, for the last tile, nnz
        for (int j = warp - kLbWarp;; j += kLbWarps) {
            const int q = j % kQ;
            bool ready;  // sleep-wait; past the CTA's last tile no arrival ever comes for this j
            while (!(ready = mbar_try(&S.counted[q], (uint32_t)(j / kQ) & 1u, 1000)))
                if (flag_ld(&S.last_j) < j) break;
            if (!ready) break;
            const int64_t tile = S.q_ticket[q];
            if (tile < tiles) {
#ifdef GIST_SSDC_ABLATE_LOOKBACK  // timing experiment only: no look-back (wrong output)
                const int64_t excl = 0;
#else
#ifdef GIST_SSDC_TRACE
                int rounds = 0, polls = 0;
                if (lane == 0) TRACE(j, 6);
                const int64_t excl = (tile == 0) ? 0 : look_back(ws, tile, lane, &rounds, &polls);
                if (lane == 0 && g_trace && blockIdx.x < kTraceCtas && j < kTraceTiles)
                    g_trace[((int64_t)blockIdx.x * kTraceTiles + j) * 8 + 7] = (uint64_t)rounds * 1000000 + polls;
#else
                const int64_t excl = (tile == 0) ? 0 : look_back(ws, tile, lane);
#endif
#endif
                const uint32_t total = S.total[q];
                if (lane == 0) {
                    S.excl[q] = excl;
                    if (tile > 0) st_relaxed(desc_at(ws, tile), kStatusP | (uint64_t)(excl + total));
                    if (tile == tiles - 1) *nnz_out = excl + total;
                }
                const int64_t r = tile * kTileRows + lane;
                if (lane < kTileRows && r < rows) row_end[r] = (int32_t)(excl + S.row_excl[q][lane] + S.row_cnt[q][lane]);
            }
            __syncwarp();
            if (lane == 0) {
                TRACE(j, 3);
                mbar_arrive(&S.resolved[q]);
            }
            if (tile >= tiles) break;
        }
    } else if (warp < kWarps) {
        // ---- compactors: move the tile's nonzeros into the pending ring (tile-local order),
        // then release the raw stage at once.  Ranks from ballots: lane l holds cols 4l+k
        // ("lo") and 128+4l+k ("hi"), k = 0..3.
        const uint32_t lt = (1u << lane) - 1u;
        for (int j = 0;; ++j) {
            const int s = j % kStages, q = j % kQ;
            mbar_wait(&S.counted[q], (uint32_t)(j / kQ) & 1u);
            const int64_t tile = S.q_ticket[q];
            if (tile >= tiles) break;
            if (threadIdx.x == 0) {  // allocate T ring entries (indices wrap modulo kRing)
                const uint32_t T = S.total[q];
                const int64_t p = S.alloc_pos;
                while (p + T - flag_ld64(&S.free_pos) > kRing) __nanosleep(64);
                S.pos[q] = (uint32_t)(p & (kRing - 1));
                S.ring_end[q] = p + T;
                S.alloc_pos = p + T;
            }
            compactors_sync();
#ifdef GIST_SSDC_ABLATE_COMPACT  // timing experiment only: skip compaction (wrong output)
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&S.empty[s]);
                mbar_arrive(&S.compacted[q]);
            }
            continue;
#endif
            const float *Tr = S.tile[s];
            const uint32_t rp = S.pos[q];
            float *vr = S.vring;
            uint8_t *cr = S.cring;
#pragma unroll
            for (int r = 0; r < kRowsPerWarp; ++r) {
                const int rr = warp * kRowsPerWarp + r;
                const float4 *row4 = reinterpret_cast<const float4 *>(Tr + rr * kRow);
                const float4 a = row4[lane], b = row4[32 + lane];
                const float v[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
                uint32_t bal[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) bal[k] = __ballot_sync(kFull, __float_as_uint(v[k]) != 0u);
                const uint32_t q0 = S.row_excl[q][rr];
                uint32_t p_lo = q0 + __popc(bal[0] & lt) + __popc(bal[1] & lt) + __popc(bal[2] & lt) + __popc(bal[3] & lt);
                uint32_t p_hi = q0 + __popc(bal[0]) + __popc(bal[1]) + __popc(bal[2]) + __popc(bal[3]) +
                                __popc(bal[4] & lt) + __popc(bal[5] & lt) + __popc(bal[6] & lt) + __popc(bal[7] & lt);
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t on = (bal[k] >> lane) & 1u;
                    if (on) {
                        const uint32_t m = (rp + p_lo) & (kRing - 1);
                        vr[m] = v[k];
                        cr[m] = (uint8_t)(4 * lane + k);
                    }
                    p_lo += on;
                }
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t on = (bal[4 + k] >> lane) & 1u;
                    if (on) {
                        const uint32_t m = (rp + p_hi) & (kRing - 1);
                        vr[m] = v[4 + k];
                        cr[m] = (uint8_t)(128 + 4 * lane + k);
                    }
                    p_hi += on;
                }
            }
            fence_proxy_async_smem();  // our reads of the raw stage precede the next TMA write
            __syncwarp();
            if (lane == 0) {
                if (warp == 0) TRACE(j, 4);
                mbar_arrive(&S.empty[s]);
                mbar_arrive(&S.compacted[q]);
            }
        }
    } else {
        // ---- storers: once a tile is compacted and resolved, copy its entries to val/col
        // (coalesced), then release its ring space and queue slot, in order.
        const int sl = threadIdx.x - 32 * kStoreWarp;
        for (int j = 0;; ++j) {
            const int q = j % kQ;
            const uint32_t par = (uint32_t)(j / kQ) & 1u;
            mbar_wait(&S.resolved[q], par);
            const int64_t tile = S.q_ticket[q];
            if (tile >= tiles) break;
            mbar_wait(&S.compacted[q], par);
            const int64_t excl = S.excl[q];
            int64_t lim = S.total[q];
            if (excl + lim > capacity) lim = capacity > excl ? capacity - excl : 0;
            const uint32_t rp = S.pos[q];
            float *vo = val + excl;
            uint8_t *co = col + excl;
#ifdef GIST_SSDC_ABLATE_STORE  // timing experiment only: skip the global stores (wrong output)
            lim = 0;
#endif
#pragma unroll 4
            for (int k = sl; k < (int)lim; k += 32 * kStoreWarps) {
                const uint32_t m = (rp + (uint32_t)k) & (kRing - 1);
                vo[k] = S.vring[m];
                co[k] = S.cring[m];
            }
            storers_sync();
            if (sl == 0) {
                TRACE(j, 5);
                flag_st64(&S.free_pos, S.ring_end[q]);
                flag_st(&S.stored, j + 1);
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

#ifdef GIST_SSDC_TRACE
extern "C" int gist_debug_ssdc_trace(void *buf) {
    return (int)cudaMemcpyToSymbol(g_trace, &buf, sizeof(void *));
}
#endif

size_t ssdc_workspace_bytes(int64_t n) {
    const int64_t rows = (n + kRow - 1) / kRow;
    const int64_t tiles = (rows + kTileRows - 1) / kTileRows;
    return 8 + 8 * (size_t)kDescStride * (size_t)(tiles > 0 ? tiles : 1);
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
