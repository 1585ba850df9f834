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

// WAR between generic-proxy reads of a TMA stage and the next TMA write into it: the
// consumer's mbarrier arrive -> producer's wait already orders them (as in CUTLASS pipelines);
// fence.proxy.async there stalls until the CTA's in-flight bulk copies land, so it is a
// measured variant only (GIST_PROXY_FENCE=1).
#ifndef GIST_PROXY_FENCE
#define GIST_PROXY_FENCE 0
#endif
__device__ __forceinline__ void ring_release_fence() {
#if GIST_PROXY_FENCE
    fence_proxy_async_smem();
#endif
}

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
    ring_release_fence();
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
                    fence_proxy_async_smem();  // generic writes into a TMA stage (once per call)
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
            ring_release_fence();  // (variant knob; the mbarrier hand-off orders the reads)
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

// ---------------------------------------------------------------------------------------------
// Encode v3: count, then compact from a second read served by L2; every CTA keeps its own
// running prefix over ALL tile totals, so there is no serial look-back chain.
//
// Tiles are slices of kSliceRows = 32 rows (32 KB), claimed in ticket order by persistent CTAs
// (one per SM).  The global offset of tile t is sum(tot[0..t)); a CTA's gatherer sums the
// published totals from where it stopped for its previous tile up to t-1 — about one grid's
// worth of totals per tile, loaded in one coalesced round trip — so offsets never wait on
// another CTA's look-back, only on the (recent) predecessors' counts.  Warp roles per CTA,
// linked by mbarriers:
//   * producer (1 lane): claims tiles (pre-claiming the next ticket) and streams each tile's
//     four 8 KB parts into a kStages3-deep shared-memory ring with 1-D TMA bulk copies
//     (HBM -> smem; the lines stay in L2 for the second read);
//   * 4 counter warps (one per part): per-row nonzero bit-pattern counts (R8), stage released;
//   * publisher warp: tile-local row scan -> rinc[], tile total published (flag | count in one
//     word) to tot[tile];
//   * gatherer warp: running prefix over tot[] -> the tile's global offset;
//   * 8 writer warps (4 rows each): re-read their rows with 128-bit loads (L2 hits; issued one
//     tile ahead for memory-level parallelism), rank nonzeros with warp ballots, stage them in
//     shared memory congruent to the output mod 4 and store val/col with 128-/32-bit stores,
//     plus row_end.
// A CTA holds at most kQ3 tiles between claim and write-out (bounded L2 footprint).  HBM sees
// the algorithmic traffic: 4n read once, 5*nnz + 4*rows written.
#ifndef GIST_SSDC_ALGO
#define GIST_SSDC_ALGO 4
#endif
#ifndef GIST_SSDC3_STAGES
#define GIST_SSDC3_STAGES 16
#endif
#ifndef GIST_SSDC3_Q
#define GIST_SSDC3_Q 8
#endif
#ifndef GIST_SSDC3_KEEP
#define GIST_SSDC3_KEEP 0
#endif
#ifndef GIST_SSDC3_PARTS
#define GIST_SSDC3_PARTS 4
#endif
constexpr int k3Writers = 8;
constexpr int k2RowsPerWarp = 4;
constexpr int kSliceRows = k3Writers * k2RowsPerWarp;  // 32 rows = 8192 elements = 32 KB
constexpr int kParts = GIST_SSDC3_PARTS;               // counter warps = TMA stages per tile
constexpr int kPartRows = kSliceRows / kParts;
constexpr int kPartElems = kPartRows * kRow;           // 8 KB per TMA stage (4 parts)
constexpr int kStages3 = GIST_SSDC3_STAGES;
constexpr int kQ3 = GIST_SSDC3_Q;
constexpr int k3Prod = 0, k3Count = 1, k3Pub = k3Count + kParts, k3Gather = k3Pub + 1, k3Writer0 = k3Gather + 1;
constexpr int k3Threads = 32 * (k3Writer0 + k3Writers);  // 480
constexpr uint32_t kTotFlag = 0x80000000u;
constexpr int kStage = k2RowsPerWarp * kRow + 4;  // staged entries per writer warp (+ alignment pad)
constexpr int kGatherPer = 8;                     // totals per lane per gather round (256 per warp)
constexpr int kTotOffset = 32;                    // tot[] after the ticket, one 128-B line apart
static_assert(kStages3 % kParts == 0, "each counter warp owns the stages of its part");
static_assert(kPartRows % 2 == 0, "counters reduce two rows at a time");

struct __align__(128) Enc3Smem {
    float raw[kStages3][kPartElems];  // TMA ring (parts of tiles)
    float vst[k3Writers][kStage];     // per-writer compacted values (congruent to the output mod 4)
    uint8_t cst[k3Writers][kStage];   // per-writer compacted column bytes
    uint32_t rcnt[kQ3][kSliceRows];   // per-row nonzero counts
    uint32_t rinc[kQ3][kSliceRows];   // tile-local inclusive row ends
    int64_t base[kQ3];                // global offset of the tile
    int64_t tile[kQ3];                // tile claimed in this slot (>= tiles: no more work)
    uint64_t full[kStages3], empty[kStages3];
    uint64_t counted[kQ3], published[kQ3], resolved[kQ3], freed[kQ3];
};

// The tile totals are self-contained words (flag | count) and nothing else is published with
// them, so relaxed gpu-scope accesses suffice (no fences, no L1 invalidation).
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(uint32_t *p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void mbar_arrive1(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Rows [4w, 4w+4) of tile t: lane l gets cols [4l, 4l+4) in lo[r] and [128+4l, 128+4l+4) in
// hi[r].  Last use of the data: L2 evict-first.  Elements past n read as zeros (never counted).
__device__ __forceinline__ void load_rows(const float *__restrict__ x, int64_t n, int64_t t, int w, int lane,
                                          uint4 (&lo)[k2RowsPerWarp], uint4 (&hi)[k2RowsPerWarp]) {
#pragma unroll
    for (int r = 0; r < k2RowsPerWarp; ++r) {
        const int64_t e0 = (t * kSliceRows + w * k2RowsPerWarp + r) * kRow;
        const uint4 *p = reinterpret_cast<const uint4 *>(x + e0);
        if (e0 + kRow <= n) {
            lo[r] = __ldcs(p + lane);
            hi[r] = __ldcs(p + 32 + lane);
        } else {
            uint32_t v[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const int64_t e = e0 + (k < 4 ? 4 * lane + k : 128 + 4 * lane + k - 4);
                v[k] = e < n ? __float_as_uint(x[e]) : 0u;
            }
            lo[r] = make_uint4(v[0], v[1], v[2], v[3]);
            hi[r] = make_uint4(v[4], v[5], v[6], v[7]);
        }
    }
}

__device__ __forceinline__ uint32_t nz4(const uint4 &a) {  // nonzero bit patterns among 4 words
    return umin(a.x, 1u) + umin(a.y, 1u) + umin(a.z, 1u) + umin(a.w, 1u);
}

// Writer: compact the 4 rows held in lo/hi (tile t, queue slot q) to val/col, and row_end.
__device__ __forceinline__ void write_rows(Enc3Smem &S, int q, int64_t t, int64_t rows, int w, int lane,
                                           const uint4 (&lo)[k2RowsPerWarp], const uint4 (&hi)[k2RowsPerWarp],
                                           int32_t *__restrict__ row_end, uint8_t *__restrict__ col,
                                           float *__restrict__ val, int64_t capacity) {
    const uint32_t lt = (1u << lane) - 1u;
    const int rw = w * k2RowsPerWarp;
    const int64_t tile_base = S.base[q];
    const uint32_t w_excl = rw ? S.rinc[q][rw - 1] : 0u;
    const uint32_t w_cnt = S.rinc[q][rw + k2RowsPerWarp - 1] - w_excl;
    const int64_t off = tile_base + w_excl;  // global index of the warp's first entry
    if (w_cnt) {
        const int a = (int)(off & 3);  // staging index = a + local index
        float *vs = S.vst[w];
        uint8_t *cs = S.cst[w];
#pragma unroll
        for (int r = 0; r < k2RowsPerWarp; ++r) {
            const uint32_t v[8] = {lo[r].x, lo[r].y, lo[r].z, lo[r].w, hi[r].x, hi[r].y, hi[r].z, hi[r].w};
            uint32_t bal[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) bal[k] = __ballot_sync(kFull, v[k] != 0u);
            const uint32_t q0 = a + (rw + r ? S.rinc[q][rw + r - 1] : 0u) - w_excl;
            uint32_t p_lo = q0 + __popc(bal[0] & lt) + __popc(bal[1] & lt) + __popc(bal[2] & lt) + __popc(bal[3] & lt);
            uint32_t p_hi = q0 + __popc(bal[0]) + __popc(bal[1]) + __popc(bal[2]) + __popc(bal[3]) +
                            __popc(bal[4] & lt) + __popc(bal[5] & lt) + __popc(bal[6] & lt) + __popc(bal[7] & lt);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                if (v[k]) {
                    vs[p_lo] = __uint_as_float(v[k]);
                    cs[p_lo] = (uint8_t)(4 * lane + k);
                    ++p_lo;
                }
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                if (v[4 + k]) {
                    vs[p_hi] = __uint_as_float(v[4 + k]);
                    cs[p_hi] = (uint8_t)(128 + 4 * lane + k);
                    ++p_hi;
                }
            }
        }
        __syncwarp();
        // global entries [off, lim) in 4-entry groups g = [4g, 4g+4); staging index 4g - (off & ~3)
        const int64_t lim = (off + w_cnt < capacity) ? off + w_cnt : capacity;
        const int64_t g_lo = off >> 2, g_hi = (lim + 3) >> 2;
        for (int64_t g = g_lo + lane; g < g_hi; g += 32) {
            const int si = (int)(4 * (g - g_lo));
            const int64_t e = 4 * g;
            if (e >= off && e + 4 <= lim) {
                *reinterpret_cast<float4 *>(val + e) = *reinterpret_cast<const float4 *>(vs + si);
                *reinterpret_cast<uint32_t *>(col + e) = *reinterpret_cast<const uint32_t *>(cs + si);
            } else {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    if (e + j >= off && e + j < lim) {
                        val[e + j] = vs[si + j];
                        col[e + j] = cs[si + j];
                    }
                }
            }
        }
        __syncwarp();
    }
    if (lane < k2RowsPerWarp) {
        const int64_t r = t * kSliceRows + rw + lane;
        if (r < rows) row_end[r] = (int32_t)(tile_base + S.rinc[q][rw + lane]);
    }
}

#ifdef GIST_SSDC3_TRACE
// Timing experiment only: per (CTA, local tile j) timestamps (%globaltimer, ns): 0 producer
// issues the tile, 1 tile total published, 2 tile offset resolved, 3 writer 0 done.
constexpr int kTrace3Tiles = 256;
__device__ uint64_t *g_trace3 = nullptr;
__device__ __forceinline__ void trace3(int64_t j, int ev) {
    if (g_trace3 && j < kTrace3Tiles - 1) {
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_trace3[((int64_t)blockIdx.x * kTrace3Tiles + j) * 4 + ev] = t;
    }
}
#define TRACE3(j, ev) trace3(j, ev)
#else
#define TRACE3(j, ev)
#endif

__global__ void __launch_bounds__(k3Threads, 1)
ssdc_encode3_kernel(const float *__restrict__ x, int64_t n, int64_t rows, int64_t tiles,
                    int32_t *__restrict__ row_end, uint8_t *__restrict__ col, float *__restrict__ val,
                    int64_t capacity, int64_t *__restrict__ nnz_out, uint32_t *__restrict__ ws) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Enc3Smem &S = *reinterpret_cast<Enc3Smem *>(smem_raw);
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    uint32_t *ticket = ws;
    uint32_t *tot = ws + kTotOffset;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages3; ++s) {
            mbar_init(&S.full[s], 1);
            mbar_init(&S.empty[s], 1);
        }
        for (int q = 0; q < kQ3; ++q) {
            mbar_init(&S.counted[q], kParts);
            mbar_init(&S.published[q], 1);
            mbar_init(&S.resolved[q], 1);
            mbar_init(&S.freed[q], k3Writers);
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (warp == k3Prod) {
        // ---- producer: claim tiles in ticket order (next one pre-claimed), stream their parts.
        // The end ("no more tiles") is a slot whose tile is >= tiles; its parts arrive with 0 bytes.
        if (lane == 0) {
#ifdef GIST_SSDC3_TRACE
            if (g_trace3) {
                uint32_t smid;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                g_trace3[((int64_t)blockIdx.x * kTrace3Tiles + kTrace3Tiles - 1) * 4 + 3] = smid;
            }
#endif
            int64_t t = atomicAdd(ticket, 1u);
            for (int64_t j = 0;; ++j) {
                const int q = (int)(j % kQ3);
                if (j >= kQ3) mbar_wait(&S.freed[q], (uint32_t)(j / kQ3 - 1) & 1u);
                S.tile[q] = t;
                TRACE3(j, 0);
                const int64_t e_tile = t * (int64_t)(kSliceRows * kRow);
                for (int h = 0; h < kParts; ++h) {
                    const int64_t js = kParts * j + h;
                    const int s = (int)(js % kStages3);
                    if (js >= kStages3) mbar_wait(&S.empty[s], (uint32_t)(js / kStages3 - 1) & 1u);
                    const int64_t e0 = e_tile + h * kPartElems;
                    const int64_t avail = t < tiles ? n - e0 : 0;
                    const uint32_t bytes =
                        avail >= kPartElems ? kPartElems * 4u : (avail > 0 ? (uint32_t)((avail * 4) & ~15ll) : 0u);
                    ring_release_fence();
                    mbar_arrive_expect_tx(&S.full[s], bytes);  // also publishes S.tile[q] to the counter
                    if (bytes) {
#if GIST_SSDC3_KEEP
                        tma_load_1d_keep(S.raw[s], x + e0, bytes, &S.full[s]);
#else
                        tma_load_1d_normal(S.raw[s], x + e0, bytes, &S.full[s]);
#endif
                    }
                }
                if (t >= tiles) break;
                t = atomicAdd(ticket, 1u);
            }
        }
    } else if (warp >= k3Count && warp < k3Count + kParts) {
        // ---- counters: part h of every tile; lane r ends up with row r's count
        const int h = warp - k3Count;
        for (int64_t j = 0;; ++j) {
            const int64_t js = kParts * j + h;
            const int s = (int)(js % kStages3);
            const int q = (int)(j % kQ3);
            mbar_wait(&S.full[s], (uint32_t)(js / kStages3) & 1u);
            const int64_t t = S.tile[q];
            if (t < tiles) {
                float *T = S.raw[s];
                const int64_t e0 = t * (int64_t)(kSliceRows * kRow) + h * kPartElems;
                const int64_t avail = n - e0;
                if (avail < kPartElems) {  // ragged end of the map: the part the TMA could not copy, zeros
                    const int from = avail > 0 ? (int)(((avail * 4) & ~15ll) / 4) : 0;
                    for (int i = from + lane; i < kPartElems; i += 32) T[i] = (i < avail) ? x[e0 + i] : 0.0f;
                    fence_proxy_async_smem();  // generic writes into a TMA stage (once per call)
                    __syncwarp();
                }
                uint32_t mine = 0;
#pragma unroll
                for (int r = 0; r < kPartRows; r += 2) {  // two rows per reduction (16-bit fields)
                    const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                    const uint4 a0 = row4[lane], b0 = row4[32 + lane], c0 = row4[64 + lane], d0 = row4[96 + lane];
                    const uint32_t u = __reduce_add_sync(kFull, (nz4(a0) + nz4(b0)) | ((nz4(c0) + nz4(d0)) << 16));
                    if (lane == r) mine = u & 0xffffu;
                    if (lane == r + 1) mine = u >> 16;
                }
                if (lane < kPartRows) S.rcnt[q][h * kPartRows + lane] = mine;
            }
            ring_release_fence();  // (variant knob; the mbarrier hand-off orders the reads)
            __syncwarp();
            if (lane == 0) {
                mbar_arrive1(&S.empty[s]);
                mbar_arrive1(&S.counted[q]);
            }
            if (t >= tiles) break;
        }
    } else if (warp == k3Pub) {
        // ---- publisher: tile-local row scan, tile total -> tot[tile]
        for (int64_t j = 0;; ++j) {
            const int q = (int)(j % kQ3);
            mbar_wait(&S.counted[q], (uint32_t)(j / kQ3) & 1u);
            const int64_t t = S.tile[q];
            if (t < tiles) {
                uint32_t inc = S.rcnt[q][lane];
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t u = __shfl_up_sync(kFull, inc, d);
                    if (lane >= d) inc += u;
                }
                S.rinc[q][lane] = inc;
                if (lane == 31) st_relaxed_u32(&tot[t], kTotFlag | inc);
            }
            __syncwarp();
            if (lane == 0) {
                TRACE3(j, 1);
                mbar_arrive1(&S.published[q]);
            }
            if (t >= tiles) break;
        }
    } else if (warp == k3Gather) {
        // ---- gatherer: running prefix over all tile totals, in tile order.  For each of this
        // CTA's tiles t: sum tot[pos .. t) (up to 256 totals per coalesced round trip; re-poll
        // until all are published), base(t) = sum.
        int64_t pos = 0, sum = 0;
        for (int64_t j = 0;; ++j) {
            const int q = (int)(j % kQ3);
            mbar_wait(&S.published[q], (uint32_t)(j / kQ3) & 1u);
            const int64_t t = S.tile[q];
            const int64_t upto = t < tiles ? t : 0;
            while (pos < upto) {
                uint32_t v[kGatherPer];
#pragma unroll
                for (int i = 0; i < kGatherPer; ++i) {
                    const int64_t idx = pos + 32 * i + lane;
                    v[i] = idx < upto ? ld_relaxed_u32(&tot[idx]) : kTotFlag;  // past upto: ready, 0
                }
                // the longest fully published prefix of the window
                int64_t ready = 32 * kGatherPer;
#pragma unroll
                for (int i = kGatherPer - 1; i >= 0; --i) {
                    const uint32_t miss = __ballot_sync(kFull, !(v[i] & kTotFlag));
                    if (miss) ready = 32 * i + __ffs(miss) - 1;
                }
                uint32_t add = 0;
#pragma unroll
                for (int i = 0; i < kGatherPer; ++i)
                    if (32 * i + lane < ready) add += v[i] & ~kTotFlag;
                sum += (int64_t)__reduce_add_sync(kFull, add);
                pos += ready;
                if (pos > upto) pos = upto;
                if (ready < 32 * kGatherPer && pos < upto) __nanosleep(32);
            }
            if (t < tiles) {
                if (lane == 0) S.base[q] = sum;
                if (t == tiles - 1 && lane == 0) *nnz_out = sum + S.rinc[q][kSliceRows - 1];
            }
            __syncwarp();
            if (lane == 0) {
                TRACE3(j, 2);
                mbar_arrive1(&S.resolved[q]);
            }
            if (t >= tiles) break;
        }
    } else {
        // ---- writers: rows [4w, 4w+4) of each tile; the next tile's loads are in flight while
        // the current one is compacted (two register sets, manual 2x unroll)
        const int w = warp - k3Writer0;
        uint4 lo0[k2RowsPerWarp], hi0[k2RowsPerWarp], lo1[k2RowsPerWarp], hi1[k2RowsPerWarp];
        mbar_wait(&S.published[0], 0u);
        int64_t t0 = S.tile[0], t1 = tiles;
        if (t0 < tiles) load_rows(x, n, t0, w, lane, lo0, hi0);
        for (int64_t j = 0; t0 < tiles; j += 2) {
            // even j: data in set 0, prefetch j+1 into set 1
            mbar_wait(&S.published[(j + 1) % kQ3], (uint32_t)((j + 1) / kQ3) & 1u);
            t1 = S.tile[(j + 1) % kQ3];
            if (t1 < tiles) load_rows(x, n, t1, w, lane, lo1, hi1);
            {
                const int q = (int)(j % kQ3);
                mbar_wait(&S.resolved[q], (uint32_t)(j / kQ3) & 1u);
                write_rows(S, q, t0, rows, w, lane, lo0, hi0, row_end, col, val, capacity);
                __syncwarp();
                if (lane == 0) {
                    if (w == 0) TRACE3(j, 3);
                    mbar_arrive1(&S.freed[q]);
                }
            }
            if (t1 >= tiles) break;
            // odd j+1: data in set 1, prefetch j+2 into set 0
            mbar_wait(&S.published[(j + 2) % kQ3], (uint32_t)((j + 2) / kQ3) & 1u);
            t0 = S.tile[(j + 2) % kQ3];
            if (t0 < tiles) load_rows(x, n, t0, w, lane, lo0, hi0);
            {
                const int q = (int)((j + 1) % kQ3);
                mbar_wait(&S.resolved[q], (uint32_t)((j + 1) / kQ3) & 1u);
                write_rows(S, q, t1, rows, w, lane, lo1, hi1, row_end, col, val, capacity);
                __syncwarp();
                if (lane == 0) {
                    if (w == 0) TRACE3(j + 1, 3);
                    mbar_arrive1(&S.freed[q]);
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------
// Encode v4: one pass — compact straight from the TMA stage into a pending ring, publish the
// tile count at once, and resolve offsets with a per-CTA running prefix over all tile totals.
//
// Tiles are kTile4Rows = 16 rows (16 KB); tickets hand out groups of kGroup4 consecutive tiles
// (32 KB) to persistent CTAs (one per SM) in ticket order.  The global offset of tile t is
// sum(tot[0..t)).  Warp roles per CTA, linked by mbarriers:
//   * producer (1 lane): claims groups (next one pre-claimed) and streams each tile into a
//     kStages4-deep shared-memory ring with one 1-D TMA bulk copy (cp.async.bulk);
//   * kComp4 compactor warps (tile j goes to warp j % kComp4): warp ballots rank the nonzero bit
//     patterns (R8) of each row; the tile total is published to tot[tile] (flag | count, one
//     word) before anything else, then the tile's (value, column) pairs are scattered in
//     tile-local order into a wrapping pending ring (one 64-bit store per entry) and the stage
//     is released;
//   * gatherer warp: running prefix over tot[] (up to 512 totals per coalesced round trip) ->
//     each of the CTA's tiles gets its global offset as soon as all earlier tiles are counted;
//   * kStore4 storer warps: copy each resolved tile from the ring to val/col (coalesced) and
//     write its row_end, in order, then free its ring space and slot.
// No tile waits on another CTA's look-back; HBM sees the algorithmic traffic only (4n read
// once, 5*nnz + 4*rows written).
#ifndef GIST_SSDC4_STAGES
#define GIST_SSDC4_STAGES 8
#endif
#ifndef GIST_SSDC4_COMP
#define GIST_SSDC4_COMP 4
#endif
#ifndef GIST_SSDC4_STORE
#define GIST_SSDC4_STORE 2
#endif
#ifndef GIST_SSDC4_RING
#define GIST_SSDC4_RING 8192
#endif
constexpr int kTile4Rows = 16;
constexpr int kTile4Elems = kTile4Rows * kRow;    // 4096 elements = 16 KB
constexpr int kGroup4 = 2;                        // tiles per ticket (32 KB)
constexpr int kStages4 = GIST_SSDC4_STAGES;
constexpr int kComp4 = GIST_SSDC4_COMP;
constexpr int kStore4 = GIST_SSDC4_STORE;
constexpr int kRing4 = GIST_SSDC4_RING;           // pending (value, column) pairs
constexpr int kQ4 = 32;                           // tiles in flight per CTA (claim .. stored)
constexpr int k4Prod = 0, k4Comp = 1, k4Gather = k4Comp + kComp4, k4Store = k4Gather + 1;
constexpr int k4Threads = 32 * (k4Store + kStore4);
constexpr uint32_t kTot4Flag = 0x80000000u;
constexpr int kGather4Per = 16;                   // totals per lane per gather round (512 per warp)
constexpr int kTot4Offset = 32;                   // tot[] after the ticket, one 128-B line apart
static_assert(kStages4 % kComp4 == 0, "each compactor owns the stages of its tiles");
static_assert((kRing4 & (kRing4 - 1)) == 0 && kRing4 >= kTile4Elems, "ring: power of two >= one tile");

struct __align__(128) Enc4Smem {
    float raw[kStages4][kTile4Elems];   // TMA ring
    uint2 pend[kRing4];                 // pending (value bits, column) pairs, tile-local order
    int64_t tile[kQ4];                  // tile of each slot (>= tiles: no more work)
    int64_t base[kQ4];                  // global offset of the tile (gatherer)
    int64_t ring_end[kQ4];              // monotonic ring position after the tile
    uint32_t rinc[kQ4][kTile4Rows];     // tile-local inclusive row ends
    uint32_t pos[kQ4];                  // ring start of the tile (masked)
    uint64_t full[kStages4], empty[kStages4];
    uint64_t counted[kQ4], compacted[kQ4], resolved[kQ4], freed[kQ4];
    int64_t alloc_pos;                  // monotonic ring allocation cursor (compactors, in tile order)
    unsigned long long free_pos;        // monotonic ring release cursor (storers; atomic access)
    int32_t alloc_turn;                 // local tile index allowed to allocate next (atomic access)
    int32_t last_j;                     // local index of the end marker (atomic access)
};

#ifdef GIST_SSDC4_TRACE
// Timing experiment only: per (CTA, local tile j) timestamps (%globaltimer, ns): 0 issued,
// 1 landed, 2 counted, 3 allocated, 4 compacted, 5 resolved, 6 stored.
constexpr int kTrace4Tiles = 512;
__device__ uint64_t *g_trace4 = nullptr;
__device__ __forceinline__ void trace4(int64_t j, int ev) {
    if (g_trace4 && j < kTrace4Tiles) {
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_trace4[((int64_t)blockIdx.x * kTrace4Tiles + j) * 8 + ev] = t;
    }
}
#define TRACE4(j, ev) trace4(j, ev)
#else
#define TRACE4(j, ev)
#endif

__global__ void __launch_bounds__(k4Threads, 1)
ssdc_encode4_kernel(const float *__restrict__ x, int64_t n, int64_t rows, int64_t tiles,
                    int32_t *__restrict__ row_end, uint8_t *__restrict__ col, float *__restrict__ val,
                    int64_t capacity, int64_t *__restrict__ nnz_out, uint32_t *__restrict__ ws) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Enc4Smem &S = *reinterpret_cast<Enc4Smem *>(smem_raw);
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    uint32_t *ticket = ws;
    uint32_t *tot = ws + kTot4Offset;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages4; ++s) {
            mbar_init(&S.full[s], 1);
            mbar_init(&S.empty[s], 1);
        }
        for (int q = 0; q < kQ4; ++q) {
            mbar_init(&S.counted[q], 1);
            mbar_init(&S.compacted[q], 1);
            mbar_init(&S.resolved[q], 1);
            mbar_init(&S.freed[q], 1);
        }
        S.alloc_pos = 0;
        S.free_pos = 0;
        S.alloc_turn = 0;
        S.last_j = 0x7fffffff;
        fence_mbar_init();
    }
    __syncthreads();

    if (warp == k4Prod) {
        // ---- producer: claim groups of tiles in ticket order (next group pre-claimed) and
        // stream each tile.  The end is a slot whose tile is >= tiles (0-byte arrival).
        if (lane == 0) {
            int64_t g = atomicAdd(ticket, 1u);
            for (int64_t j = 0;; ++j) {
                const int64_t t = (g < (tiles + kGroup4 - 1) / kGroup4) ? g * kGroup4 + j % kGroup4 : tiles;
                const int q = (int)(j % kQ4);
                const int s = (int)(j % kStages4);
                if (j >= kQ4) mbar_wait_sleep(&S.freed[q], (uint32_t)(j / kQ4 - 1) & 1u);
                if (j >= kStages4) mbar_wait_sleep(&S.empty[s], (uint32_t)(j / kStages4 - 1) & 1u);
                const int64_t tt = t < tiles ? t : tiles;
                S.tile[q] = tt;
                const int64_t e0 = tt * (int64_t)kTile4Elems;
                const int64_t avail = tt < tiles ? n - e0 : 0;
                const uint32_t bytes =
                    avail >= kTile4Elems ? kTile4Elems * 4u : (avail > 0 ? (uint32_t)((avail * 4) & ~15ll) : 0u);
                ring_release_fence();
                TRACE4(j, 0);
                mbar_arrive_expect_tx(&S.full[s], bytes);  // also publishes S.tile[q] to the compactor
                if (bytes) tma_load_1d(S.raw[s], x + e0, bytes, &S.full[s]);
                if (tt >= tiles) break;
                if (j % kGroup4 == kGroup4 - 1) g = atomicAdd(ticket, 1u);
            }
        }
    } else if (warp >= k4Comp && warp < k4Comp + kComp4) {
        // ---- compactors: tile j = c, c + kComp4, ... of this CTA.  Lane l holds columns
        // [4l, 4l+4) ("lo") and [128+4l, 128+4l+4) ("hi") of each row.
        const int c = warp - k4Comp;
        const uint32_t lt = (1u << lane) - 1u;
        for (int64_t j = c;; j += kComp4) {
            const int s = (int)(j % kStages4);
            const int q = (int)(j % kQ4);
            bool ready;  // past the end marker no arrival ever comes for this j
            while (!(ready = mbar_try(&S.full[s], (uint32_t)(j / kStages4) & 1u, 1000)))
                if (atomicAdd(&S.last_j, 0) < j) break;
            if (!ready) break;
            if (lane == 0) TRACE4(j, 1);
            const int64_t t = S.tile[q];
            if (t >= tiles) {  // end marker: tell the other compactors, the gatherer and the storers
                if (lane == 0) atomicExch(&S.last_j, (int32_t)j);
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive1(&S.counted[q]);
                    mbar_arrive1(&S.compacted[q]);
                }
                break;
            }
            float *T = S.raw[s];
            const int64_t e0 = t * (int64_t)kTile4Elems;
            const int64_t avail = n - e0;
            if (avail < kTile4Elems) {  // ragged end of the map: the part the TMA could not copy, zeros
                const int from = (int)(((avail * 4) & ~15ll) / 4);
                for (int i = from + lane; i < kTile4Elems; i += 32) T[i] = (i < avail) ? x[e0 + i] : 0.0f;
                fence_proxy_async_smem();  // generic writes into a TMA stage (once per call)
                __syncwarp();
            }
            // pass 1: ballots -> per-row counts -> tile-local row ends; publish the total
            uint32_t mine = 0;  // lane r: row r's count
#pragma unroll
            for (int r = 0; r < kTile4Rows; ++r) {
                const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                const uint4 a = row4[lane], b2 = row4[32 + lane];
                const uint32_t cnt = __reduce_add_sync(kFull, nz4(a) + nz4(b2));
                if (lane == r) mine = cnt;
            }
            uint32_t inc = mine;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t u = __shfl_up_sync(kFull, inc, d);
                if (lane >= d) inc += u;
            }
            const uint32_t total = __shfl_sync(kFull, inc, kTile4Rows - 1);
            if (lane == 0) st_relaxed_u32(&tot[t], kTot4Flag | total);
            if (lane < kTile4Rows) S.rinc[q][lane] = inc;
            __syncwarp();
            if (lane == 0) {
                TRACE4(j, 2);
                mbar_arrive1(&S.counted[q]);
            }
            // ring space, allocated in local tile order
            if (lane == 0) {
                while (atomicAdd(&S.alloc_turn, 0) != (int32_t)j) __nanosleep(32);
                const int64_t p = S.alloc_pos;
                while (p + total - (int64_t)atomicAdd(&S.free_pos, 0ull) > kRing4) __nanosleep(64);
                S.pos[q] = (uint32_t)(p & (kRing4 - 1));
                S.ring_end[q] = p + total;
                S.alloc_pos = p + total;
                __threadfence_block();
                atomicExch(&S.alloc_turn, (int32_t)(j + 1));
                TRACE4(j, 3);
            }
            __syncwarp();
            // pass 2: scatter (value, column) pairs in tile-local order
            const uint32_t rp = S.pos[q];
            uint2 *ring = S.pend;
#pragma unroll 4
            for (int r = 0; r < kTile4Rows; ++r) {
                const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                const uint4 a = row4[lane], b2 = row4[32 + lane];
                const uint32_t v[8] = {a.x, a.y, a.z, a.w, b2.x, b2.y, b2.z, b2.w};
                uint32_t bal[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) bal[k] = __ballot_sync(kFull, v[k] != 0u);
                const uint32_t q0 = rp + (r ? S.rinc[q][r - 1] : 0u);
                uint32_t p_lo = q0 + __popc(bal[0] & lt) + __popc(bal[1] & lt) + __popc(bal[2] & lt) + __popc(bal[3] & lt);
                uint32_t p_hi = q0 + __popc(bal[0]) + __popc(bal[1]) + __popc(bal[2]) + __popc(bal[3]) +
                                __popc(bal[4] & lt) + __popc(bal[5] & lt) + __popc(bal[6] & lt) + __popc(bal[7] & lt);
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    if (v[k]) ring[p_lo & (kRing4 - 1)] = make_uint2(v[k], 4u * lane + k);
                    p_lo += v[k] != 0u;
                }
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    if (v[4 + k]) ring[p_hi & (kRing4 - 1)] = make_uint2(v[4 + k], 128u + 4u * lane + k);
                    p_hi += v[4 + k] != 0u;
                }
            }
            ring_release_fence();  // (variant knob; the mbarrier hand-off orders the reads)
            __syncwarp();
            if (lane == 0) {
                TRACE4(j, 4);
                mbar_arrive1(&S.empty[s]);
                mbar_arrive1(&S.compacted[q]);
            }
        }
    } else if (warp == k4Gather) {
        // ---- gatherer: running prefix over all tile totals, in tile order.
        int64_t pos = 0, sum = 0;
        for (int64_t j = 0;; ++j) {
            const int q = (int)(j % kQ4);
            mbar_wait_sleep(&S.counted[q], (uint32_t)(j / kQ4) & 1u);
            const int64_t t = S.tile[q];
            const int64_t upto = t < tiles ? t : 0;
            while (pos < upto) {
                uint32_t v[kGather4Per];
#pragma unroll
                for (int i = 0; i < kGather4Per; ++i) {
                    const int64_t idx = pos + 32 * i + lane;
                    v[i] = idx < upto ? ld_relaxed_u32(&tot[idx]) : kTot4Flag;  // past upto: ready, 0
                }
                int64_t ready = 32 * kGather4Per;  // longest fully published prefix of the window
#pragma unroll
                for (int i = kGather4Per - 1; i >= 0; --i) {
                    const uint32_t miss = __ballot_sync(kFull, !(v[i] & kTot4Flag));
                    if (miss) ready = 32 * i + __ffs(miss) - 1;
                }
                uint32_t add = 0;
#pragma unroll
                for (int i = 0; i < kGather4Per; ++i)
                    if (32 * i + lane < ready) add += v[i] & ~kTot4Flag;
                sum += (int64_t)__reduce_add_sync(kFull, add);
                pos += ready;
                if (pos > upto) pos = upto;
                if (ready < 32 * kGather4Per && pos < upto) __nanosleep(32);
            }
            if (t < tiles) {
                if (lane == 0) S.base[q] = sum;
                if (t == tiles - 1 && lane == 0) *nnz_out = sum + S.rinc[q][kTile4Rows - 1];
            }
            __syncwarp();
            if (lane == 0) {
                TRACE4(j, 5);
                mbar_arrive1(&S.resolved[q]);
            }
            if (t >= tiles) break;
        }
    } else {
        // ---- storers: in tile order, copy resolved tiles from the ring to val/col (coalesced)
        // and write row_end; then free ring space and the slot.
        const int sl = threadIdx.x - 32 * k4Store;
        constexpr int kST = 32 * kStore4;
        for (int64_t j = 0;; ++j) {
            const int q = (int)(j % kQ4);
            const uint32_t par = (uint32_t)(j / kQ4) & 1u;
            mbar_wait_sleep(&S.resolved[q], par);
            const int64_t t = S.tile[q];
            if (t >= tiles) break;
            mbar_wait_sleep(&S.compacted[q], par);
            const int64_t base = S.base[q];
            const uint32_t total = S.rinc[q][kTile4Rows - 1];
            const uint32_t rp = S.pos[q];
            if (sl < kTile4Rows) {
                const int64_t r = t * kTile4Rows + sl;
                if (r < rows) row_end[r] = (int32_t)(base + S.rinc[q][sl]);
            }
            int64_t lim = (base + total < capacity) ? base + total : capacity;
            // output entries [base, lim): aligned groups of 4 with 128-bit / 32-bit stores
            const int64_t g_lo = base >> 2, g_hi = (lim + 3) >> 2;
            for (int64_t g = g_lo + sl; g < g_hi; g += kST) {
                const int64_t e = 4 * g;
                uint2 pr[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int64_t ek = e + k;
                    pr[k] = (ek >= base && ek < lim) ? S.pend[(rp + (uint32_t)(ek - base)) & (kRing4 - 1)]
                                                     : make_uint2(0u, 0u);
                }
                if (e >= base && e + 4 <= lim) {
                    *reinterpret_cast<uint4 *>(val + e) = make_uint4(pr[0].x, pr[1].x, pr[2].x, pr[3].x);
                    *reinterpret_cast<uint32_t *>(col + e) =
                        __byte_perm(__byte_perm(pr[0].y, pr[1].y, 0x0040), __byte_perm(pr[2].y, pr[3].y, 0x0040), 0x5410);
                } else {
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        if (e + k >= base && e + k < lim) {
                            val[e + k] = __uint_as_float(pr[k].x);
                            col[e + k] = (uint8_t)pr[k].y;
                        }
                    }
                }
            }
            asm volatile("bar.sync 1, %0;" ::"n"(kST) : "memory");
            if (sl == 0) {
                __threadfence_block();
                atomicExch(&S.free_pos, (unsigned long long)S.ring_end[q]);
                TRACE4(j, 6);
                mbar_arrive1(&S.freed[q]);
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

#ifdef GIST_SSDC4_TRACE
extern "C" int gist_debug_ssdc4_trace(void *buf) {
    return (int)cudaMemcpyToSymbol(g_trace4, &buf, sizeof(void *));
}
#endif
#ifdef GIST_SSDC3_TRACE
extern "C" int gist_debug_ssdc3_trace(void *buf) {
    return (int)cudaMemcpyToSymbol(g_trace3, &buf, sizeof(void *));
}
#endif
#ifdef GIST_SSDC_TRACE
extern "C" int gist_debug_ssdc_trace(void *buf) {
    return (int)cudaMemcpyToSymbol(g_trace, &buf, sizeof(void *));
}
#endif

size_t ssdc_workspace_bytes(int64_t n) {
    const int64_t rows = (n + kRow - 1) / kRow;
#if GIST_SSDC_ALGO == 4
    const int64_t tiles = (rows + kTile4Rows - 1) / kTile4Rows;
    return 4 * (size_t)kTot4Offset + 8 * (size_t)((tiles + 1) / 2);  // ticket line + tot[tiles] uint32
#elif GIST_SSDC_ALGO == 3
    const int64_t tiles = (rows + kSliceRows - 1) / kSliceRows;
    return 4 * (size_t)kTotOffset + 8 * (size_t)((tiles + 1) / 2);  // ticket line + tot[tiles] uint32
#else
    const int64_t tiles = (rows + kTileRows - 1) / kTileRows;
    return 8 + 8 * (size_t)kDescStride * (size_t)(tiles > 0 ? tiles : 1);
#endif
}

cudaError_t launch_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val,
                               int64_t capacity, int64_t *nnz, void *workspace, cudaStream_t s) {
    const int64_t rows = (n + kRow - 1) / kRow;
    const int64_t ws_words = (int64_t)ssdc_workspace_bytes(n) / 8;
    int64_t iblocks = ceil_div(ws_words, 256);
    if (iblocks > 1024) iblocks = 1024;
    ssdc_ws_init<<<(unsigned)iblocks, 256, 0, s>>>(reinterpret_cast<uint64_t *>(workspace), ws_words);
#if GIST_SSDC_ALGO == 4
    static std::once_flag attr_once;
    std::call_once(attr_once, [] {
        cudaFuncSetAttribute(ssdc_encode4_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(Enc4Smem));
    });
    const int64_t tiles = (rows + kTile4Rows - 1) / kTile4Rows;
    const int64_t groups = (tiles + kGroup4 - 1) / kGroup4;
    const int64_t grid = groups < num_sms() ? groups : num_sms();
    ssdc_encode4_kernel<<<(unsigned)grid, k4Threads, sizeof(Enc4Smem), s>>>(
        x, n, rows, tiles, row_end, col, val, capacity, nnz, reinterpret_cast<uint32_t *>(workspace));
#elif GIST_SSDC_ALGO == 3
    // A tile's offset waits for the totals of all earlier tiles, claimed in ticket order by
    // running CTAs: one persistent CTA per SM (the shared-memory ring allows no more).
    static std::once_flag attr_once;
    std::call_once(attr_once, [] {
        cudaFuncSetAttribute(ssdc_encode3_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(Enc3Smem));
    });
    const int64_t tiles = (rows + kSliceRows - 1) / kSliceRows;
    const int64_t grid = tiles < num_sms() ? tiles : num_sms();
    ssdc_encode3_kernel<<<(unsigned)grid, k3Threads, sizeof(Enc3Smem), s>>>(
        x, n, rows, tiles, row_end, col, val, capacity, nnz, reinterpret_cast<uint32_t *>(workspace));
#else
    const int64_t tiles = (rows + kTileRows - 1) / kTileRows;
    static std::once_flag attr_once;
    std::call_once(attr_once, [] {
        cudaFuncSetAttribute(ssdc_encode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(EncSmem));
    });
    int64_t grid = (int64_t)num_sms() * kCtasPerSm;  // persistent, smem-limited residency
    if (grid > tiles) grid = tiles;
    ssdc_encode_kernel<<<(unsigned)grid, kCtaThreads, sizeof(EncSmem), s>>>(
        x, n, rows, tiles, row_end, col, val, capacity, nnz, reinterpret_cast<Workspace *>(workspace));
#endif
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
