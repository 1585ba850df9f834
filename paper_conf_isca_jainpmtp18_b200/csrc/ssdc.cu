// ssdc.cu — a4/a5: Sparse Storage, Dense Compute (PAPER.md P:158-P:164 §IV-A).
//
// Encode: dense fp32 -> CSR with 256-column rows and uint8 column indices (Narrow Value
// Optimization): row_end[rows] (inclusive ends, R10), col[nnz], val[nnz], nnz.
//
// One read of x: count and compact from the same shared-memory ring; every CTA keeps its own
// running prefix over ALL tile totals, so no tile waits on a serial look-back chain.
//
// Tiles are kTileRows = 32 rows (32 KB), claimed in ticket order by persistent CTAs (one per
// SM).  The global offset of tile t is sum(tot[0..t)); a CTA's gatherer sums the published
// totals from where it stopped for its previous tile up to t-1 — about one grid's worth of
// totals per tile, loaded in one coalesced round trip — so offsets only wait on the (recent)
// predecessors' counts.  Warp roles per CTA, linked by mbarriers:
//   * producer (1 lane): claims tiles (pre-claiming the next ticket) and streams each tile's
//     four 8 KB parts into a kStages-deep shared-memory ring with 1-D TMA bulk copies
//     (cp.async.bulk, HBM -> smem);
//   * 4 counter warps (one per part): per-row nonzero bit-pattern counts (R8);
//   * publisher warp: tile-local row scan -> rinc[], tile total published (epoch tag | count
//     in one word) to tot[tile];
//   * gatherer warp: running prefix over tot[] -> the tile's global offset, and row_end;
//   * 8 writer warps (4 rows each): once the tile is published, load their rows from the ring
//     into registers (one tile ahead) and release the stage; rank nonzeros (lane l owns columns
//     l + 32k; one ballot per 32 columns, row starts from the publisher's row scan) and, once the
//     offset is resolved, stage them in shared memory congruent to the output mod 16;
//   * store warp: the whole 16-entry groups of val/col leave with two 1-D bulk copies (shared ->
//     global) per tile, the ragged head and tail with plain stores; the staging buffer then goes
//     back to the writers and the tile slot to the producer.
// HBM sees the algorithmic traffic: 4n read once, 5*nnz + 4*rows written.
// DESIGN.md §6 has the measured history of the alternatives (decoupled look-back, chunked
// all-to-all prefix, single-pass compaction into a pending ring, L2 re-read writers).
//
// Decode: a warp expands 4 consecutive rows (whose entries are one contiguous range)
//   through a 4 KB shared-memory row buffer and writes them back with float4 stores; the next
//   group's row bounds are loaded one group ahead and up to 8 col/val entries per lane are in
//   flight before the scatter.
#include "common.cuh"
#include "kernels.h"
#include "tma.cuh"
#include "tcgen05.cuh"  // named_bar


namespace gist {

namespace {

constexpr int kRow = 256;

#ifndef GIST_SSDC_STAGES
#define GIST_SSDC_STAGES 16
#endif
#ifndef GIST_SSDC_Q
#define GIST_SSDC_Q 8
#endif
#ifndef GIST_SSDC_PARTS
#define GIST_SSDC_PARTS 4
#endif
#ifndef GIST_SSDC_DEC_CTAS
#define GIST_SSDC_DEC_CTAS 3  // decode CTAs per SM (grid cap); 4-6 measured slower in isolation
#endif
#ifndef GIST_SSDC_LPRE
#define GIST_SSDC_LPRE 0  // 1 (with GIST_SSDC_BALLOT=0): the counters also scan the writers' lane counts (writers skip count + scan): 0.228 -> 0.265 ms, the counters then pace the prefix chain
#endif
#ifndef GIST_SSDC_BALLOT
// 1: writer lane l holds columns l + 32k of its rows and one ballot per 32 columns ranks the nonzeros
// (row starts from rinc: no lane counts, no shuffle scan).  With 4 rows per writer (8 writer warps),
// relu1_1 b64 s = .5 / .8 / .9: 0.246 / 0.228 / 0.228 -> 0.226 / 0.224 / 0.222 ms, C3 step a4 70% -> 73%.
// 0: lane l holds columns [8l, 8l+8) and a shuffle scan of the lane counts ranks them (2 rows per writer).
#define GIST_SSDC_BALLOT 1
#endif
#ifndef GIST_SSDC_SPIN_NS
// producer (ring space), counters (data) and publisher (counts) poll with test_wait + __nanosleep:
// their try_wait loops took ~24% of the kernel's issue slots (ncu), which the writers need
#define GIST_SSDC_SPIN_NS 256  // relu1_1 s = .8: 0.2257 (try_wait) vs 0.2298 / 0.2277 / 0.2257 / 0.2245 ms at 32 / 64 / 128 / 256 ns
#endif
#ifndef GIST_SSDC_WROWS
#define GIST_SSDC_WROWS (GIST_SSDC_BALLOT ? 4 : 2)
#endif
constexpr int kWRows = GIST_SSDC_WROWS;        // rows per writer warp per tile
static_assert(!(GIST_SSDC_LPRE && GIST_SSDC_BALLOT), "lane prefixes are for the scan path");
constexpr int kTileRows = 32;                         // rows per tile = 8192 elements = 32 KB
static_assert(kTileRows == 32, "the gatherer writes row_end with one lane per row");
constexpr int kWriters = kTileRows / kWRows;
#ifndef GIST_SSDC_DEPTH
#define GIST_SSDC_DEPTH 2
#endif
constexpr int kDepth = GIST_SSDC_DEPTH;                 // writer register sets (tiles in flight)
static_assert(kDepth >= 2, "the writer loop prefetches at least one tile ahead");
constexpr int kParts = GIST_SSDC_PARTS;               // counter warps = TMA stages per tile
constexpr int kPartRows = kTileRows / kParts;
constexpr int kPartElems = kPartRows * kRow;           // 8 KB per TMA stage (4 parts)
constexpr int kStages = GIST_SSDC_STAGES;
constexpr int kQ = GIST_SSDC_Q;
#ifndef GIST_SSDC_STORER
#define GIST_SSDC_STORER 1  // a store warp issues each tile's bulk copies (the writers never wait on each other)
#endif
constexpr int kProd = 0, kCount = 1, kPub = kCount + kParts, kGather = kPub + 1, kWriter0 = kGather + 1;
constexpr int kStorer = kWriter0 + kWriters;
constexpr int kEncThreads = 32 * (kWriter0 + kWriters + GIST_SSDC_STORER);  // 16 warps = 512 threads (8 writers)
constexpr int kStage = kTileRows * kRow + 16;  // staged entries per tile (+ 16-entry phase)
constexpr int kWriterThreads = 32 * kWriters;
constexpr int kGatherPer = 8;                     // totals per lane per gather round (256 per warp)
constexpr int kMaxEncJobs = 48;                   // maps per encode launch (job table in kernel params)
// Workspace (zeroed once by the caller, left reusable by every call): u32 words ticket [0],
// done [1] (CTAs finished), epoch [2] (calls completed); u64 tot[tiles] from word kTotOffset.
// tot[t] = (epoch + 1) << 32 | count: the tag makes the previous call's totals read as
// unpublished, so no per-call clearing is needed.  The last CTA to finish resets ticket and
// done and advances the epoch.
constexpr int kTotOffset = 32;                    // tot[] one 128-B line after the counters
constexpr uint32_t kWsMagic = 0x47495354u;        // word 3 of an initialised workspace ("GIST")

__global__ void ssdc_ws_init_kernel(uint32_t *ws, int64_t words) {
    pdl_enter();
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += (int64_t)gridDim.x * blockDim.x)
        ws[i] = i == 3 ? kWsMagic : 0u;
}
static_assert(kStages % kParts == 0, "each counter warp owns the stages of its part");
static_assert(kPartRows % 2 == 0, "counters reduce two rows at a time");

// Job table (a kernel parameter, < 4 KB): one launch encodes up to kMaxEncJobs maps.  The tiles of
// all jobs form one ticket space (job j owns global tiles [tile0_j, tile0_{j+1})), so a single
// persistent grid streams every map with one fill and one drain, and each job's running prefix
// restarts at its first tile (no wait on the totals of earlier jobs).
struct EncJob {
    const float *x;
    int32_t *row_end;
    uint8_t *col;
    float *val;
    int64_t *nnz;
    const int64_t *base;  // NULL, or the device offset where this job's entries start (append mode)
    int64_t n, capacity, tile0;
    int32_t head;  // first job of this job's chain (a job whose offset is the previous job's nnz
                   // continues that job's entries; the prefix then runs across both)
};
struct EncJobs {
    EncJob j[kMaxEncJobs];
    int64_t tiles;  // total tiles of all jobs
    int32_t count;
};
static_assert(sizeof(EncJobs) + 16 <= 4096, "kernel parameters must fit 4 KB");

struct __align__(128) EncSmem {
    float raw[kStages][kPartElems];  // TMA ring (parts of tiles)
    uint32_t vst[2][kStage];         // compacted value bits of a tile (congruent to the output mod 16),
    uint8_t cst[2][kStage];          // and its columns (bytes, same index); double-buffered by tile
    uint32_t rcnt[kQ][kTileRows];   // per-row nonzero counts
#if GIST_SSDC_LPRE
    uint32_t lpre[kQ][kWriters][32];  // per writer lane: row-0 | row-1 exclusive offsets (16 bits each)
#endif
    uint32_t rinc[kQ][kTileRows];   // tile-local inclusive row ends
    int64_t base[kQ];                // global offset of the tile
    int64_t tile[kQ];                // tile claimed in this slot (>= tiles: no more work)
    int32_t job[kQ];                 // job of that tile
    uint64_t full[kStages], empty[kStages];
    uint64_t counted[kQ], published[kQ], resolved[kQ], freed[kQ];
    uint64_t staged[kQ], sfree[2];  // writers -> store warp (tile staged), store warp -> writers (buffer read)
};

// The tile totals are self-contained words (tag | count) and nothing else is published with
// them, so relaxed gpu-scope accesses suffice (no fences, no L1 invalidation).
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void mbar_arrive1(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ uint32_t min1(uint32_t v) {  // 1 if the bit pattern is nonzero (one IMNMX)
    uint32_t r;
    asm("min.u32 %0, %1, 1;" : "=r"(r) : "r"(v));
    return r;
}
__device__ __forceinline__ uint32_t nz4(const uint4 &a) {  // nonzero bit patterns among 4 words
    return min1(a.x) + min1(a.y) + min1(a.z) + min1(a.w);
}

// Writer: stage the nonzeros of the rows held in lo/hi (queue slot q) into the tile's staging
// buffer sb.  The lane counts (0..8) of both rows are scanned together (two 16-bit fields, one
// 5-step shuffle scan); then each lane's nonzeros go to consecutive staging slots (value word and
// column byte at the same index).  The staging index of output entry e is e - (tile base & ~15),
// so after all writers have staged, the tile's whole 16-entry groups of val (64 B) and col (16 B)
// leave as ONE pair of 1-D bulk copies (store_tile).
__device__ __forceinline__ void stage_rows(EncSmem &S, int q, int sb, int w, int lane, const uint4 (&lo)[kWRows],
                                           const uint4 (&hi)[kWRows]) {
    const int rw = w * kWRows;
    const uint32_t w_excl = rw ? S.rinc[q][rw - 1] : 0u;
    if (S.rinc[q][rw + kWRows - 1] == w_excl) return;  // no nonzeros in these rows
    const uint32_t p = (uint32_t)(S.base[q] & 15) + w_excl;  // staging index of the writer's first entry
#if GIST_SSDC_BALLOT
    // lane l holds columns l + 32k of each row (k = 0..7: lo.x..w, hi.x..w).  Row r's entries start
    // at rinc[rw + r - 1] (tile-local), so no lane counts or scans: one ballot per 32 columns gives
    // each nonzero its rank, and the entries of columns [32k, 32k + 32) follow those of lower k
    // (ascending column order, O4).
    const uint32_t lt = (1u << lane) - 1u;
    uint32_t *vs = S.vst[sb];
    uint8_t *cs = S.cst[sb];
#pragma unroll
    for (int r = 0; r < kWRows; ++r) {
        const uint32_t v[8] = {lo[r].x, lo[r].y, lo[r].z, lo[r].w, hi[r].x, hi[r].y, hi[r].z, hi[r].w};
        uint32_t base = p + ((r ? S.rinc[q][rw + r - 1] : w_excl) - w_excl);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t b = __ballot_sync(kFull, v[k] != 0u);  // R8: nonzero bit patterns
            if (v[k] != 0u) {
                const uint32_t i = base + __popc(b & lt);
                vs[i] = v[k];
                cs[i] = (uint8_t)(32 * k + lane);
            }
            base += __popc(b);
        }
    }
#else
    static_assert(kWRows == 2, "the packed scan carries two rows");
#if GIST_SSDC_LPRE
    // the counters scanned this writer's lane counts (published with the tile, ordered by published[q])
    const uint32_t pk = S.lpre[q][w][lane];
    const uint32_t excl[2] = {pk & 0xffffu, pk >> 16};
#else
    // lane prefix of both rows' lane counts in one warp scan (16-bit fields: row counts <= 256)
    const uint32_t cnt0 = nz4(lo[0]) + nz4(hi[0]), cnt1 = nz4(lo[1]) + nz4(hi[1]);
    uint32_t inc = cnt0 | (cnt1 << 16);
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t u = __shfl_up_sync(kFull, inc, d);
        if (lane >= d) inc += u;
    }
    const uint32_t row0_tot = __shfl_sync(kFull, inc, 31) & 0xffffu;
    const uint32_t excl[2] = {(inc & 0xffffu) - cnt0, row0_tot + (inc >> 16) - cnt1};
#endif
#pragma unroll
    for (int r = 0; r < kWRows; ++r) {
        const uint32_t v[8] = {lo[r].x, lo[r].y, lo[r].z, lo[r].w, hi[r].x, hi[r].y, hi[r].z, hi[r].w};
        const uint32_t i = p + excl[r];
        uint32_t addr = smem_u32(S.vst[sb] + i), caddr = smem_u32(S.cst[sb] + i);
        const uint32_t c0 = 8u * lane;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            asm volatile(
                "{\n\t.reg .pred p;\n\t"
                "setp.ne.u32 p, %2, 0;\n\t"
                "@p st.shared.u32 [%0], %2;\n\t"
                "@p st.shared.u8 [%1], %3;\n\t"
                "@p add.u32 %0, %0, 4;\n\t"
                "@p add.u32 %1, %1, 1;\n\t}"
                : "+r"(addr), "+r"(caddr)
                : "r"(v[k]), "r"(c0 + k)
                : "memory");
        }
    }
#endif  // GIST_SSDC_BALLOT
}

// Writer warp 0, once every writer has staged the tile: the whole 16-entry groups leave as two
// bulk copies issued by lane 0; the ragged head and tail (< 16 entries each) by lanes 0..15 and
// 16..31.  Entries at or past the job's capacity are not written.
__device__ __forceinline__ void store_tile(EncSmem &S, int q, int sb, int lane, const EncJobs &J) {
    const EncJob &jb = J.j[S.job[q]];
    const int64_t off = S.base[q];
    const int64_t cnt = S.rinc[q][kTileRows - 1];
    const int64_t lim = (off + cnt < jb.capacity) ? off + cnt : jb.capacity;
    if (lim <= off) return;
    const uint32_t *vs = S.vst[sb];
    const uint8_t *cs = S.cst[sb];
    const int64_t base16 = off & ~15ll;                     // staging index of entry e: e - base16
    const int64_t g_lo = (off + 15) >> 4, g_hi = lim >> 4;  // whole 16-entry groups [g_lo, g_hi)
    if (g_hi > g_lo) {
        if (lane == 0) {
            const int s0 = (int)(16 * g_lo - base16);
            const uint32_t ng = (uint32_t)(g_hi - g_lo);
            tma_store_1d(jb.val + 16 * g_lo, vs + s0, 64u * ng);
            tma_store_1d(jb.col + 16 * g_lo, cs + s0, 16u * ng);
            bulk_commit();
        }
        const int64_t e = lane < 16 ? 16 * g_lo - 16 + lane : 16 * g_hi + lane - 16;
        if (e >= off && e < lim) {
            jb.val[e] = __uint_as_float(vs[e - base16]);
            jb.col[e] = cs[e - base16];
        }
    } else {
        // no whole 16-entry group: fewer than 32 entries
        for (int64_t e = off + lane; e < lim; e += 32) {
            jb.val[e] = __uint_as_float(vs[e - base16]);
            jb.col[e] = cs[e - base16];
        }
    }
}

#ifdef GIST_SSDC_TRACE
// Timing experiment only: per (CTA, local tile j) timestamps (%globaltimer, ns): 0 producer
// issues the tile, 1 tile total published, 2 tile offset resolved, 3 writer 0 done.
constexpr int kTraceTiles = 256;
__device__ uint64_t *g_trace = nullptr;
__device__ __forceinline__ void trace(int64_t j, int ev) {
    if (g_trace && j < kTraceTiles - 1) {
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_trace[((int64_t)blockIdx.x * kTraceTiles + j) * 4 + ev] = t;
    }
}
#define TRACE(j, ev) trace(j, ev)
#else
#define TRACE(j, ev)
#endif

__global__ void __launch_bounds__(kEncThreads, 1)
ssdc_encode_kernel(const __grid_constant__ EncJobs J, uint32_t *__restrict__ ws) {
    const int64_t tiles = J.tiles;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    EncSmem &S = *reinterpret_cast<EncSmem *>(smem_raw);
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    uint32_t *ticket = ws;
    uint64_t *tot = reinterpret_cast<uint64_t *>(ws + kTotOffset);
    // Prologue before the programmatic-dependency wait touches shared memory only (the barrier
    // initialisation overlaps the previous kernel's tail); after it, the first ticket claim and
    // the read of the counter line (epoch, magic) are issued together.
#if GIST_PDL && GIST_PDL_EARLY
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&S.full[s], 1);
            mbar_init(&S.empty[s], kPartRows / kWRows);  // released by the part's writers
        }
        for (int q = 0; q < kQ; ++q) {
            mbar_init(&S.counted[q], kParts);
            mbar_init(&S.published[q], 1);
            mbar_init(&S.resolved[q], 1);
            mbar_init(&S.freed[q], GIST_SSDC_STORER ? 1 : kWriters);
            mbar_init(&S.staged[q], kWriters);
        }
        for (int b = 0; b < 2; ++b) mbar_init(&S.sfree[b], 1);
        fence_mbar_init();
    }
#if GIST_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
    // thread 0 is the producer lane: its first ticket is claimed now (on an uninitialised
    // workspace the claim is harmless: the call reports and returns)
    const uint32_t first_ticket = threadIdx.x == 0 ? atomicAdd(ticket, 1u) : 0u;
    uint32_t epoch, magic;
    asm volatile("ld.volatile.global.v2.u32 {%0, %1}, [%2];" : "=r"(epoch), "=r"(magic) : "l"(ws + 2) : "memory");
    if (magic != kWsMagic) {  // never initialised: report, no work
        if (blockIdx.x == 0 && threadIdx.x == 0)
            for (int k = 0; k < J.count; ++k) *J.j[k].nnz = -1;
        return;
    }
    // every CTA reads the epoch before it counts itself done, so all see the same value
    const uint64_t tag = (uint64_t)(epoch + 1u) << 32;
    __syncthreads();

    if (warp == kProd) {
        // ---- producer: claim tiles in ticket order (next one pre-claimed), stream their parts.
        // The end ("no more tiles") is a slot whose tile is >= tiles; its parts arrive with 0 bytes.
        if (lane == 0) {
#ifdef GIST_SSDC_TRACE
            if (g_trace) {
                uint32_t smid;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                g_trace[((int64_t)blockIdx.x * kTraceTiles + kTraceTiles - 1) * 4 + 3] = smid;
            }
#endif
            int64_t t = first_ticket;
            int jc = 0;  // job cursor: tickets rise, so jobs only move forward
            for (uint32_t j = 0;; ++j) {
                const int q = (int)(j % kQ);
                if (j >= kQ) mbar_wait_sleep(&S.freed[q], (uint32_t)(j / kQ - 1) & 1u);
                if (t < tiles)
                    while (jc + 1 < J.count && t >= J.j[jc + 1].tile0) ++jc;
                S.tile[q] = t;
                S.job[q] = jc;
                TRACE(j, 0);
                const EncJob &jb = J.j[jc];
                const int64_t e_tile = (t - jb.tile0) * (int64_t)(kTileRows * kRow);
                for (int h = 0; h < kParts; ++h) {
                    const uint32_t js = kParts * j + h;
                    const int s = (int)(js % kStages);
                    if (js >= kStages) mbar_wait_backoff(&S.empty[s], (uint32_t)(js / kStages - 1) & 1u, GIST_SSDC_SPIN_NS);
                    const int64_t e0 = e_tile + h * kPartElems;
                    const int64_t avail = t < tiles ? jb.n - e0 : 0;
                    const uint32_t bytes =
                        avail >= kPartElems ? kPartElems * 4u : (avail > 0 ? (uint32_t)((avail * 4) & ~15ll) : 0u);
                    mbar_arrive_expect_tx(&S.full[s], bytes);  // also publishes S.tile/job[q] to the counter
                    if (bytes) {
                        tma_load_1d_normal(S.raw[s], jb.x + e0, bytes, &S.full[s]);
                    }
                }
                if (t >= tiles) break;
                t = atomicAdd(ticket, 1u);
            }
        }
    } else if (warp >= kCount && warp < kCount + kParts) {
        // ---- counters: part h of every tile; lane r ends up with row r's count
        const int h = warp - kCount;
        for (uint32_t j = 0;; ++j) {
            const uint32_t js = kParts * j + h;
            const int s = (int)(js % kStages);
            const int q = (int)(j % kQ);
            mbar_wait_backoff(&S.full[s], (uint32_t)(js / kStages) & 1u, GIST_SSDC_SPIN_NS);
            const int64_t t = S.tile[q];
            if (t < tiles) {
                float *T = S.raw[s];
                const EncJob &jb = J.j[S.job[q]];
                const int64_t e0 = (t - jb.tile0) * (int64_t)(kTileRows * kRow) + h * kPartElems;
                const int64_t avail = jb.n - e0;
                // racecheck reports these ring writes against the writers' ring reads (fetch): ordered by
                // counted[q] (counter arrive, release) -> publisher wait (acquire) ... published[q] arrive
                // -> writer wait in fetch, a chain of mbarrier release/acquire pairs racecheck does not model
                if (avail < kPartElems) {  // ragged end of the map: the part the TMA could not copy, zeros
                    const int from = avail > 0 ? (int)(((avail * 4) & ~15ll) / 4) : 0;
                    for (int i = from + lane; i < kPartElems; i += 32) T[i] = (i < avail) ? jb.x[e0 + i] : 0.0f;
                    fence_proxy_async_smem();  // generic writes into a TMA stage (once per call)
                    __syncwarp();
                }
                uint32_t mine = 0;
#if GIST_SSDC_LPRE
                // in the writers' layout (lane l: columns 8l .. 8l+7 of each row): the row pair of writer
                // w = part * 4 + r/2 is scanned here, its per-lane exclusive offsets left in lpre
#pragma unroll
                for (int r = 0; r < kPartRows; r += 2) {
                    const uint4 *r0 = reinterpret_cast<const uint4 *>(T + r * kRow), *r1 = r0 + kRow / 4;
                    const uint32_t cnt0 = nz4(r0[2 * lane]) + nz4(r0[2 * lane + 1]);
                    const uint32_t cnt1 = nz4(r1[2 * lane]) + nz4(r1[2 * lane + 1]);
                    uint32_t inc = cnt0 | (cnt1 << 16);
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
                        const uint32_t u = __shfl_up_sync(kFull, inc, d);
                        if (lane >= d) inc += u;
                    }
                    const uint32_t tot = __shfl_sync(kFull, inc, 31);
                    const uint32_t row0_tot = tot & 0xffffu;
                    S.lpre[q][(h * kPartRows + r) / kWRows][lane] = ((inc & 0xffffu) - cnt0) | ((row0_tot + (inc >> 16) - cnt1) << 16);
                    if (lane == r) mine = row0_tot;
                    if (lane == r + 1) mine = tot >> 16;
                }
#else
#pragma unroll
                for (int r = 0; r < kPartRows; r += 2) {  // two rows per reduction (16-bit fields)
                    const uint4 *row4 = reinterpret_cast<const uint4 *>(T + r * kRow);
                    const uint4 a0 = row4[lane], b0 = row4[32 + lane], c0 = row4[64 + lane], d0 = row4[96 + lane];
                    const uint32_t u = __reduce_add_sync(kFull, (nz4(a0) + nz4(b0)) | ((nz4(c0) + nz4(d0)) << 16));
                    if (lane == r) mine = u & 0xffffu;
                    if (lane == r + 1) mine = u >> 16;
                }
#endif
                // rcnt -> publisher: counted[q] arrive (release) / wait (acquire); the slot is rewritten
                // only after freed[q] (every writer done with tile j - kQ) -- racecheck hazard, ordered
                if (lane < kPartRows) S.rcnt[q][h * kPartRows + lane] = mine;
            }
            __syncwarp();
            if (lane == 0) {
                mbar_arrive1(&S.counted[q]);
            }
            if (t >= tiles) break;
        }
    } else if (warp == kPub) {
        // ---- publisher: tile-local row scan, tile total -> tot[tile]
        for (uint32_t j = 0;; ++j) {
            const int q = (int)(j % kQ);
            mbar_wait_backoff(&S.counted[q], (uint32_t)(j / kQ) & 1u, GIST_SSDC_SPIN_NS);
            const int64_t t = S.tile[q];
            if (t < tiles) {
                uint32_t inc = S.rcnt[q][lane];
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t u = __shfl_up_sync(kFull, inc, d);
                    if (lane >= d) inc += u;
                }
                // rinc -> gatherer / writers: published[q] (and resolved[q]) arrive / wait; rewritten
                // only after freed[q] -- racecheck hazard, ordered by those mbarriers
                S.rinc[q][lane] = inc;
                if (lane == 31) st_relaxed_u64(&tot[t], tag | inc);
            }
            __syncwarp();
            if (lane == 0) {
                TRACE(j, 1);
                mbar_arrive1(&S.published[q]);
            }
            if (t >= tiles) break;
        }
    } else if (GIST_SSDC_STORER && warp == kStorer) {
        // ---- store warp: once the writers have staged tile jj, its whole 16-entry groups leave as two
        // bulk copies (and the ragged head and tail as plain stores); when the copies have read the
        // staging buffer, the buffer goes back to the writers and the slot to the producer
        for (uint32_t jj = 0;; ++jj) {
            const int q = (int)(jj % kQ);
            const int sb = (int)(jj & 1);
            mbar_wait_sleep(&S.published[q], (uint32_t)(jj / kQ) & 1u);
            if (S.tile[q] >= tiles) break;
            mbar_wait_sleep(&S.staged[q], (uint32_t)(jj / kQ) & 1u);
            store_tile(S, q, sb, lane, J);
            if (lane == 0) bulk_wait_read();
            __syncwarp();
            if (lane == 0) {
                TRACE(jj, 3);
                mbar_arrive1(&S.sfree[sb]);
                mbar_arrive1(&S.freed[q]);
            }
        }
        if (lane == 0) bulk_wait_all();
    } else if (warp == kGather) {
        // ---- gatherer: running prefix over all tile totals, in tile order.  For each of this
        // CTA's tiles t: sum tot[pos .. t) (up to 256 totals per coalesced round trip; re-poll
        // until all are published), base(t) = sum.
        int64_t pos = 0, sum = 0;
        int cur = -1;  // chain head of the running prefix
        for (uint32_t j = 0;; ++j) {
            const int q = (int)(j % kQ);
            mbar_wait_sleep(&S.published[q], (uint32_t)(j / kQ) & 1u);
            const int64_t t = S.tile[q];
            const int jj = S.job[q];
            if (t < tiles && J.j[jj].head != cur) {  // first tile of a new chain for this CTA: restart
                cur = J.j[jj].head;
                pos = J.j[cur].tile0;
                sum = J.j[cur].base ? *J.j[cur].base : 0;
            }
            const int64_t upto = t < tiles ? t : pos;
            while (pos < upto) {
                uint64_t v[kGatherPer];
#pragma unroll
                for (int i = 0; i < kGatherPer; ++i) {
                    const int64_t idx = pos + 32 * i + lane;
                    v[i] = idx < upto ? ld_relaxed_u64(&tot[idx]) : tag;  // past upto: ready, 0
                }
                // the longest fully published prefix of the window
                int64_t ready = 32 * kGatherPer;
#pragma unroll
                for (int i = kGatherPer - 1; i >= 0; --i) {
                    const uint32_t miss = __ballot_sync(kFull, (v[i] >> 32) != (tag >> 32));
                    if (miss) ready = 32 * i + __ffs(miss) - 1;
                }
                uint32_t add = 0;
#pragma unroll
                for (int i = 0; i < kGatherPer; ++i)
                    if (32 * i + lane < ready) add += (uint32_t)v[i];
                sum += (int64_t)__reduce_add_sync(kFull, add);
                pos += ready;
                if (pos > upto) pos = upto;
                if (ready < 32 * kGatherPer && pos < upto) __nanosleep(32);
            }
            if (t < tiles) {
                const EncJob &jb = J.j[jj];
                if (lane == 0) S.base[q] = sum;
                const int64_t r = (t - jb.tile0) * kTileRows + lane;  // kTileRows == 32: lane r owns row r
                if (r < (jb.n + kRow - 1) / kRow) jb.row_end[r] = (int32_t)(sum + S.rinc[q][lane]);
                const int64_t last = (jj + 1 < J.count ? J.j[jj + 1].tile0 : tiles) - 1;
                if (t == last && lane == 0) *jb.nnz = sum + S.rinc[q][kTileRows - 1];
            }
            __syncwarp();
            if (lane == 0) {
                TRACE(j, 2);
                mbar_arrive1(&S.resolved[q]);
            }
            if (t >= tiles) break;
        }
    } else {
        // ---- writers: rows [rw, rw + kWRows) of each tile.  kDepth register sets: the
        // loads of the next kDepth - 1 tiles are in flight while the current one is compacted
        // (manual unroll so every set stays in registers).
        const int w = warp - kWriter0;
        uint4 lo[kDepth][kWRows], hi[kDepth][kWRows];
        int64_t tt[kDepth];
        // the tile of local slot jj once published (its count is in rinc[]; its rows still in
        // the ring); lane l gets the 8 consecutive columns [8l, 8l+8) of each of its rows, so a
        // lane's nonzeros are contiguous in the output (elements past n were zero-filled)
        auto fetch = [&](uint32_t jj, uint4 (&l)[kWRows], uint4 (&h)[kWRows]) -> int64_t {
            const int q = (int)(jj % kQ);
            mbar_wait_sleep(&S.published[q], (uint32_t)(jj / kQ) & 1u);
            const int64_t t = S.tile[q];
            // the tile is still in the TMA ring (the counters do not release it): read the rows
            // from shared memory, then release the stage (the part's kPartRows / kWRows writers)
            if (t < tiles) {
                const int part = (w * kWRows) / kPartRows;
                const uint32_t js = kParts * jj + part;
                const int st = (int)(js % kStages);
                const float *rowp = S.raw[st] + (w * kWRows - part * kPartRows) * kRow;
#pragma unroll
                for (int r = 0; r < kWRows; ++r) {
#if GIST_SSDC_BALLOT
                    // columns lane + 32k (conflict-free 32-bit loads)
                    const uint32_t *p1 = reinterpret_cast<const uint32_t *>(rowp + r * kRow) + lane;
                    l[r] = make_uint4(p1[0], p1[32], p1[64], p1[96]);
                    h[r] = make_uint4(p1[128], p1[160], p1[192], p1[224]);
#else
                    const uint4 *p4 = reinterpret_cast<const uint4 *>(rowp + r * kRow);
                    l[r] = p4[2 * lane];
                    h[r] = p4[2 * lane + 1];
#endif
                }
                __syncwarp();
                if (lane == 0) mbar_arrive1(&S.empty[st]);
            }
            return t;
        };
        // tile jj stages into buffer jj & 1.  One named barrier per tile among the writers: after
        // it, the tile is fully staged (writer 0 then stores it), and writer 0's bulk copies of the
        // previous tile, which it waited on just before, have read buffer (jj - 1) & 1, so tile
        // jj + 1 may overwrite it.
        auto retire = [&](uint32_t jj, int64_t t, const uint4 (&l)[kWRows], const uint4 (&h)[kWRows]) {
            const int q = (int)(jj % kQ);
            const int sb = (int)(jj & 1);
            mbar_wait_sleep(&S.resolved[q], (uint32_t)(jj / kQ) & 1u);
#if GIST_SSDC_STORER
            // buffer sb was last staged for tile jj - 2: wait until the store warp's copies have read it
            if (jj >= 2) mbar_wait_sleep(&S.sfree[sb], (uint32_t)((jj - 2) / 2) & 1u);
            stage_rows(S, q, sb, w, lane, l, h);
            fence_proxy_async_smem();  // generic staging writes -> async-proxy bulk reads
            __syncwarp();
            if (lane == 0) mbar_arrive1(&S.staged[q]);
            return;
#endif
            stage_rows(S, q, sb, w, lane, l, h);
            fence_proxy_async_smem();  // generic staging writes -> async-proxy bulk reads
            if (w == 0 && lane == 0) bulk_wait_read();
            named_bar(1, kWriterThreads);
            if (w == 0) {
                store_tile(S, q, sb, lane, J);
                __syncwarp();
            }
            if (lane == 0) {
                if (w == 0) TRACE(jj, 3);
                mbar_arrive1(&S.freed[q]);
            }
        };
#pragma unroll
        for (int d = 0; d < kDepth - 1; ++d) tt[d] = (d == 0 || tt[d - 1] < tiles) ? fetch(d, lo[d], hi[d]) : tiles;
        for (uint32_t j = 0;; j += kDepth) {
#pragma unroll
            for (int d = 0; d < kDepth; ++d) {
                // set d holds tile j+d; prefetch j+d+kDepth-1 into set (d + kDepth - 1) % kDepth
                const int nd = (d + kDepth - 1) % kDepth;
                const int pd = (d + kDepth - 2) % kDepth;  // set of tile j+d+kDepth-2
                if (tt[d] >= tiles) goto writers_done;
                tt[nd] = (tt[pd] < tiles) ? fetch(j + d + kDepth - 1, lo[nd], hi[nd]) : tiles;
                retire(j + d, tt[d], lo[d], hi[d]);
            }
        }
    writers_done:;
        if (lane == 0) bulk_wait_all();
    }
    // the last CTA to finish leaves the workspace ready for the next call
    __syncthreads();
    if (threadIdx.x == 0 && atomicAdd(ws + 1, 1u) == gridDim.x - 1) {
        ws[0] = 0u;
        ws[1] = 0u;
        ws[2] += 1u;
    }
}

constexpr int kDecThreads = 256;
constexpr int kDecRows = 4;  // rows per warp iteration
#ifndef GIST_SSDC_DEC_BATCH
#define GIST_SSDC_DEC_BATCH 8
#endif
constexpr int kDecBatch = GIST_SSDC_DEC_BATCH;  // col/val entries per lane in flight
constexpr int kMaxDecJobs = 64;                 // maps per decode launch (job table in kernel params)

struct DecJob {
    const int32_t *row_end;
    const uint8_t *col;
    const float *val;
    const int64_t *base;  // NULL, or the device offset where the map's entries start (append mode)
    float *x;
    int64_t n;
    int64_t g0;  // first global 4-row group of the map
};
struct DecJobs {
    DecJob j[kMaxDecJobs];
    int64_t groups;
    int32_t count;
};
static_assert(sizeof(DecJobs) + 16 <= 4096, "kernel parameters must fit 4 KB");

// The 4-row groups of all maps form one index space; a warp takes groups g, g + nwarps, ... and
// advances its job cursor monotonically.
__global__ void __launch_bounds__(kDecThreads)
ssdc_decode_kernel(const __grid_constant__ DecJobs J) {
    pdl_enter();
    __shared__ __align__(16) float s_buf[kDecThreads / 32][kDecRows * kRow];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    float *buf = s_buf[warp];
    const int64_t groups = J.groups;
    const int64_t gwarp = ((int64_t)blockIdx.x * kDecThreads + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * kDecThreads) >> 5;
    auto job_of = [&](int64_t g, int jc) {
        while (jc + 1 < J.count && g >= J.j[jc + 1].g0) ++jc;
        return jc;
    };

    // lanes 0..4 hold the row boundaries of the warp's next group: bound[j] = end of row r0-1+j
    // (loaded one group ahead, so only the col/val loads are on each group's critical path)
    auto bounds = [&](int64_t g, int jc) -> int32_t {
        if (g >= groups || lane > kDecRows) return 0;
        const DecJob &jb = J.j[jc];
        const int64_t rows = (jb.n + kRow - 1) / kRow;
        const int64_t r = (g - jb.g0) * kDecRows - 1 + lane;
        if (r < 0) return jb.base ? (int32_t)*jb.base : 0;
        return r < rows ? jb.row_end[r] : jb.row_end[rows - 1];
    };
    int jc = job_of(gwarp < groups ? gwarp : 0, 0);
    int32_t bnd = bounds(gwarp, jc);
    for (int64_t g = gwarp; g < groups; g += nwarps) {
        const DecJob &jb = J.j[jc];
        const int64_t r0 = (g - jb.g0) * kDecRows;
        const int32_t b0 = __shfl_sync(kFull, bnd, 0), b1 = __shfl_sync(kFull, bnd, 1);
        const int32_t b2 = __shfl_sync(kFull, bnd, 2), b3 = __shfl_sync(kFull, bnd, 3);
        const int32_t b4 = __shfl_sync(kFull, bnd, 4);
        const uint8_t *__restrict__ col = jb.col;
        const float *__restrict__ val = jb.val;
        float *__restrict__ x = jb.x;
        const int64_t n = jb.n;
        const int64_t gn = g + nwarps;
        const int jn = gn < groups ? job_of(gn, jc) : jc;
        bnd = bounds(gn, jn);
        // zero the 4-row buffer
        float4 *b4p = reinterpret_cast<float4 *>(buf);
#pragma unroll
        for (int j = 0; j < kDecRows * kRow / 4 / 32; ++j) b4p[lane + 32 * j] = make_float4(0.f, 0.f, 0.f, 0.f);
        __syncwarp();
        // up to kDecBatch entries per lane in flight before any scatter
        for (int32_t kb = b0; kb < b4; kb += 32 * kDecBatch) {
            uint32_t c[kDecBatch];
            float v[kDecBatch];
#pragma unroll
            for (int i = 0; i < kDecBatch; ++i) {
                const int32_t k = kb + 32 * i + lane;
                if (k < b4) {
                    c[i] = col[k];
                    v[i] = val[k];
                }
            }
#pragma unroll
            for (int i = 0; i < kDecBatch; ++i) {
                const int32_t k = kb + 32 * i + lane;
                if (k < b4) buf[((k >= b1) + (k >= b2) + (k >= b3)) * kRow + c[i]] = v[i];
            }
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
        jc = jn;
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
    return 4 * (size_t)kTotOffset + 8 * (size_t)tiles;  // counters line + tot[tiles] uint64
}

cudaError_t launch_ssdc_workspace_init(void *workspace, size_t bytes, cudaStream_t s) {
    const int64_t words = (int64_t)(bytes / 4);
    int64_t blocks = ceil_div(words, 256);
    if (blocks > 1024) blocks = 1024;
    launch_k(ssdc_ws_init_kernel, (unsigned)blocks, 256, 0, s, reinterpret_cast<uint32_t *>(workspace), words);
    return cudaPeekAtLastError();
}

int64_t ssdc_tiles(int64_t n) { return (((n + kRow - 1) / kRow) + kTileRows - 1) / kTileRows; }

size_t ssdc_workspace_bytes_many(const gist_ssdc_job *jobs, int32_t count) {
    int64_t tiles = 0;
    for (int32_t k = 0; k < count; ++k) tiles += ssdc_tiles(jobs[k].n);
    return 4 * (size_t)kTotOffset + 8 * (size_t)tiles;
}

// Every map of the call in one persistent launch per kMaxEncJobs maps (launches share the
// workspace in stream order; each leaves it ready for the next).  Maps with n == 0 only publish
// *nnz (= *offset or 0) through a one-job launch of zero tiles... they are filtered by the caller.
cudaError_t launch_ssdc_encode_many(const gist_ssdc_job *jobs, int32_t count, void *workspace, cudaStream_t s,
                                    int *launches) {
    static PerDeviceAttr attr;
    const cudaError_t ea = attr.ensure(reinterpret_cast<const void *>(ssdc_encode_kernel), (int)sizeof(EncSmem));
    if (ea != cudaSuccess) return ea;
    *launches = 0;
    for (int32_t k0 = 0; k0 < count; k0 += kMaxEncJobs) {
        EncJobs J{};
        J.count = 0;
        int64_t tiles = 0;
        for (int32_t k = k0; k < count && k < k0 + kMaxEncJobs; ++k) {
            EncJob &e = J.j[J.count++];
            e.x = jobs[k].x;
            e.row_end = jobs[k].row_end;
            e.col = jobs[k].col;
            e.val = jobs[k].val;
            e.nnz = jobs[k].nnz;
            e.base = jobs[k].offset;
            e.n = jobs[k].n;
            e.capacity = jobs[k].capacity;
            e.tile0 = tiles;
            // chained: this map's entries follow the previous map's in the same arena
            const bool chained = k > k0 && jobs[k].offset && jobs[k].offset == jobs[k - 1].nnz;
            e.head = chained ? J.j[J.count - 2].head : J.count - 1;
            tiles += ssdc_tiles(jobs[k].n);
        }
        J.tiles = tiles;
        // A tile's offset waits for the totals of all earlier tiles of its map, claimed in ticket
        // order by running CTAs: one persistent CTA per SM (the shared-memory ring allows no more).
        const int64_t grid = tiles < num_sms() ? tiles : num_sms();
        launch_k(ssdc_encode_kernel, (unsigned)grid, kEncThreads, sizeof(EncSmem), s, J,
                 reinterpret_cast<uint32_t *>(workspace));
        const cudaError_t e = cudaPeekAtLastError();
        if (e != cudaSuccess) return e;
        ++*launches;
    }
    return cudaSuccess;
}

cudaError_t launch_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val,
                               int64_t capacity, int64_t *nnz, void *workspace, cudaStream_t s) {
    gist_ssdc_job job{x, n, row_end, col, val, capacity, nnz, nullptr};
    int launches = 0;
    return launch_ssdc_encode_many(&job, 1, workspace, s, &launches);
}

cudaError_t launch_ssdc_decode_many(const gist_ssdc_decode_job *jobs, int32_t count, cudaStream_t s, int *launches) {
    *launches = 0;
    for (int32_t k0 = 0; k0 < count; k0 += kMaxDecJobs) {
        DecJobs J{};
        int64_t groups = 0;
        for (int32_t k = k0; k < count && k < k0 + kMaxDecJobs; ++k) {
            DecJob &e = J.j[J.count++];
            e.row_end = jobs[k].row_end;
            e.col = jobs[k].col;
            e.val = jobs[k].val;
            e.base = jobs[k].offset;
            e.x = jobs[k].x;
            e.n = jobs[k].n;
            e.g0 = groups;
            groups += ((jobs[k].n + kRow - 1) / kRow + kDecRows - 1) / kDecRows;
        }
        J.groups = groups;
        int64_t blocks = ceil_div(groups, kDecThreads / 32);
        const int64_t cap = (int64_t)num_sms() * GIST_SSDC_DEC_CTAS;
        if (blocks > cap) blocks = cap;
        if (blocks < 1) blocks = 1;
        launch_k(ssdc_decode_kernel, (unsigned)blocks, kDecThreads, 0, s, J);
        const cudaError_t e = cudaPeekAtLastError();
        if (e != cudaSuccess) return e;
        ++*launches;
    }
    return cudaSuccess;
}

cudaError_t launch_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n, float *x,
                               cudaStream_t s) {
    gist_ssdc_decode_job job{row_end, col, val, nullptr, n, x};
    int launches = 0;
    return launch_ssdc_decode_many(&job, 1, s, &launches);
}

}  // namespace gist
