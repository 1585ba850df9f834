// wgrad.cu — f4: the conv weight gradient with the SSDC decode inside the GEMM operand producer
// (§IV-A: "the backward pass implementation can be modified to work directly on
// precision-reduced values"; §V-H: "decode only the data that is required in near
// future ... the near-future tile in a tiled matrix multiplication").
//
// For a 3x3 / stride-1 / pad-1 convolution (every VGG16 conv) whose input X was stashed as SSDC
// (ReLU->Conv), the weight gradient
//     dW[co][ci][kh][kw] = sum_{n,oh,ow} dY[n][co][oh][ow] * X[n][ci][oh+kh-1][ow+kw-1]
// is an implicit GEMM  D[M = co][N = (tap, ci)] += A[co][k] * B[(tap, ci)][k]  over
// k = (n, oh, ow).  X is never dense in HBM: for every K-tile (R output rows of one image) the
// producer warps decode the CSR rows covering those rows (+1 halo row each side) for a block of 16
// input channels into a zero-padded shared-memory slab, and build the im2col operand B from it
// directly in the UMMA 128-byte-swizzle layout.  A (dY) streams in by 2-D TMA (UTMALDG).  One
// elected thread issues tcgen05.mma (kind::tf32, M = 128, N = 144, K = 8) into a TMEM
// accumulator; the epilogue reads it back with tcgen05.ld.
//
// Precision: passes = 3 splits both operands into TF32 hi + lo parts and accumulates
// A_hi*B_hi + A_hi*B_lo + A_lo*B_hi in fp32 ("3xTF32", round-to-nearest splits: products within 2^-20 + 2^-22 of the fp32
// products); passes = 1 multiplies in TF32 (hardware truncation of the fp32 operands).
// The fp32 accumulation in registers spans at most one chunk of K-tiles (~8192 products); each
// chunk's partial goes to a workspace slot and a second kernel sums the slots in binary64 in a
// fixed order (deterministic), rounding once.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>

#include "common.cuh"
#include "kernels.h"
#include "tcgen05.cuh"

namespace gist {

namespace {

#ifndef GIST_WG_ATMEM
#define GIST_WG_ATMEM 1  // 3xTF32: A_hi / A_lo in tensor memory (the MMAs read only B from shared memory)
#endif

constexpr int kCiBlk = 16;              // input channels per CTA tile
constexpr int kTaps = 9;                // 3x3 window
constexpr int kN = kCiBlk * kTaps;      // 144 GEMM columns: n = tap * 16 + ci
constexpr int kM = 128;                 // output channels per CTA tile (UMMA M)
constexpr int kKs = 32;                 // K per pipeline stage = one 128-byte swizzle row of fp32
constexpr int kBldWarps = 4;                 // operand builders: B = im2col(X) (hi/lo) and A_lo
constexpr int kBldThreads = 32 * kBldWarps;  // one thread per (ci, 4-position chunk) of a stage
constexpr int kDecWarps = 4;                 // decoders: CSR rows of X -> the next K-tile's slab
constexpr int kDecThreads = 32 * kDecWarps;
constexpr int kBld0 = 2, kDec0 = kBld0 + kBldWarps;
constexpr int kEpiWarps = 8;                 // two per TMEM lane quarter (taps 0-4 / 5-8)
constexpr int kEpi0 = kDec0 + kDecWarps;     // first epilogue warp
// warp 0: TMA + TMEM owner, warp 1: MMA, 2..5: builders, 6..9: decoders, 10..17: accumulator drain
constexpr int kThreads = 32 * (kEpi0 + kEpiWarps);
static_assert(kBldThreads == kCiBlk * (kKs / 4), "one builder thread per (ci, chunk)");
constexpr int kDecU = 8;                     // decoder: CSR entries per lane in flight (16: more spills, slower)
// timing-only knobs (outputs invalid): skip the decode / the B build / the A split
#ifndef GIST_WG_SKIP_DEC
#define GIST_WG_SKIP_DEC 0
#endif
#ifndef GIST_WG_SKIP_B
#define GIST_WG_SKIP_B 0
#endif
#ifndef GIST_WG_SKIP_ASPLIT
#define GIST_WG_SKIP_ASPLIT 0
#endif
constexpr int kTmemCols = 512;               // two accumulators, then (3xTF32) the A stages
constexpr int kAccStride = kN;               // accumulator b at columns [144 b, 144 b + 144)
// 3xTF32 with A in tensor memory: stage s's A_hi at columns [288 + 64 s, +32), A_lo at the next 32
// (lane = output channel, column = k), after the two accumulators: up to 3 stages in 512 columns
__host__ __device__ constexpr uint32_t a_tmem_col(int s) { return 2u * kN + 64u * (uint32_t)s; }
constexpr uint32_t kIdesc = idesc_tf32<kM, kN>();
static_assert(kN % 16 == 0 && kN <= 256, "UMMA M=128 needs N % 16 == 0, N <= 256");

struct WgArgs {
    const int32_t *row_end;
    const uint8_t *col;
    const float *val;
    float *partial;  // [units][Co][Ci*9]: one fp32 partial per chunk of `chunk` K-tiles
    int32_t N, Ci, Co, H, W;
    int32_t R;        // output rows per K-tile
    int32_t spt;      // stages per K-tile
    int32_t ktiles;   // K-tiles per image = ceil(H / R)
    int32_t m_blocks, n_blocks, splits;
    int32_t pp;       // TMEM accumulation periods per K-tile (1 <= pp <= spt)
    int32_t chunk;    // K-tiles per partial (the fp32 register accumulation spans at most this many)
    int32_t units;    // partials per output tile = ceil(T / chunk)
    int64_t T;        // K-tiles in total = N * ktiles
    int32_t SWP;      // slab row pitch (W + 2 halo columns, rounded up to a multiple of 4)
    int32_t rpc;      // CSR rows a K-tile's input rows of one channel can touch (4 channels x rpc <= 32)
    int32_t slab_floats;  // one slab buffer: kCiBlk * (R + 2) * SWP
    FastDiv div_w;
};

// NA dY stages (the TMA ring, deeper: its loads come from L2 with a long latency) and NB operand
// stages (B hi/lo and A_lo, written by the builders); stage g uses A slot g % NA and B slot g % NB.
template <int PASSES, int NA, int NB>
struct __align__(1024) WgSmem {
    float a[NA][kM * kKs];                          // dY tiles (TMA, 128-B swizzle): A_hi after the split
    float alo[PASSES == 3 && !GIST_WG_ATMEM ? NB : 1][PASSES == 3 && !GIST_WG_ATMEM ? kM * kKs : 256];  // A - tf32(A) in shared memory (3xTF32 without ATMEM; 1 KB keeps bhi 1024-aligned)
    float bhi[NB][kN * kKs];                        // im2col(X) tiles, same layout
    float blo[PASSES == 3 ? NB : 1][PASSES == 3 ? kN * kKs : 256];
    uint64_t a_full[NA], b_full[NB], b_empty[NB], acc_full[2], acc_empty[2];
    uint64_t slab_full[2], slab_empty[2];  // decoders -> builders, builders -> decoders (per slab buffer)
    uint32_t tmem_base;
};
// every operand tile must start on a 1024-byte boundary (the 128-byte swizzle atom)
static_assert(sizeof(float) * kM * kKs % 1024 == 0 && sizeof(float) * kN * kKs % 1024 == 0, "tile sizes");

// Long waits (the TMA lane on a free stage, the epilogue on a finished period, the decoders on a
// free slab) back off instead of spinning on the issue slots the builders need.
#ifndef GIST_WG_SKIP_TMA
#define GIST_WG_SKIP_TMA 0
#endif
#ifndef GIST_WG_SPIN
#define GIST_WG_SPIN 0
#endif
#ifndef GIST_WG_SKIP_EPI
#define GIST_WG_SKIP_EPI 0  // timing only: the epilogue releases each period without reading TMEM
#endif
__device__ __forceinline__ void wait_backoff(uint64_t *bar, uint32_t parity) {
#if GIST_WG_SPIN
    mbar_wait(bar, parity);
#else
    while (!mbar_test(bar, parity)) __nanosleep(64);
#endif
}

#ifdef GIST_WG_TRACE
// Timing experiment only: clock64 stamps of CTA 0 for its first kWgTrace stages: 0 MMA thread starts
// waiting for b_full, 1 b_full observed, 2 the stage's MMAs issued, 3 builder warp 0 observed
// b_empty, 4 builder warp 0 arrives b_full, 5 decoder warp 0 finished the K-tile (slab_full arrive)
constexpr int kWgTrace = 256;
__device__ long long *g_wg_trace = nullptr;
#define WG_TRACE(g, ev)                                                                     \
    do {                                                                                    \
        if (g_wg_trace && blockIdx.x == 0 && (g) < kWgTrace) g_wg_trace[(g) * 8 + (ev)] = clock64(); \
    } while (0)
#else
#define WG_TRACE(g, ev)
#endif

template <int PASSES, int NA, int NB, bool VEC>
__global__ void __launch_bounds__(kThreads, 1)
wgrad_ssdc_kernel(const __grid_constant__ CUtensorMap tmap_dy, const WgArgs a) {
    static_assert(NA == NB, "one empty barrier per stage serves the dY ring and the operand stages");
    using Smem = WgSmem<PASSES, NA, NB>;
    extern __shared__ unsigned char smem_raw[];
    // the 128-byte swizzle repeats every 1024 bytes: align the tiles to that
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    Smem &S = *reinterpret_cast<Smem *>(smem_raw + pad);
    float *slabs = reinterpret_cast<float *>(smem_raw + pad + sizeof(Smem));  // two slab buffers
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    const int nb = blockIdx.x % a.n_blocks;
    const int mb = (blockIdx.x / a.n_blocks) % a.m_blocks;
    const int sp = blockIdx.x / (a.n_blocks * a.m_blocks);
    // this CTA's K-tiles: whole chunks [u0, u1) (a chunk's partial has exactly one writer)
    const int64_t u0 = (int64_t)sp * a.units / a.splits, u1 = (int64_t)(sp + 1) * a.units / a.splits;
    const int64_t t0 = u0 * a.chunk, t1 = min(a.T, u1 * (int64_t)a.chunk);
    const int co0 = mb * kM, ci0 = nb * kCiBlk;
    const int64_t nst = (t1 - t0) * a.spt;  // pipeline stages of this CTA
    const int RW = a.R * a.W, SW = a.SWP, SR = a.R + 2;

    if (threadIdx.x == 0) {
        for (int s = 0; s < NA; ++s) mbar_init(&S.a_full[s], 1);
        for (int s = 0; s < NB; ++s) {
            mbar_init(&S.b_full[s], kBldWarps);
            mbar_init(&S.b_empty[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&S.acc_full[b], 1);
            mbar_init(&S.acc_empty[b], kEpiWarps);
            mbar_init(&S.slab_full[b], kDecWarps);
            mbar_init(&S.slab_empty[b], kBldWarps);
        }
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc<kTmemCols>(&S.tmem_base);
#if GIST_PDL
#if GIST_PDL_EARLY
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = S.tmem_base;

    if (warp == 0) {
        // ---- TMA producer: the dY tile [co0, co0+128) x [k, k+32) of each stage
        if (lane == 0) {
            prefetch_tmap(&tmap_dy);
            // (image, K-tile row, stage) advanced incrementally: no division on this thread's path
            int n = (int)(t0 / a.ktiles), ty = (int)(t0 % a.ktiles), j = 0, st = 0;
            uint32_t ph = 0;
            for (int64_t g = 0; g < nst; ++g) {
                if (g >= NA) wait_backoff(&S.b_empty[st], ph ^ 1u);  // NA == NB: one empty barrier per stage
#if GIST_WG_SKIP_TMA
                (void)n, (void)ty, (void)j;
                mbar_arrive_1(&S.a_full[st]);  // timing only: no dY load
#else
                mbar_arrive_expect_tx(&S.a_full[st], kM * kKs * 4);
                tma_load_2d(S.a[st], &tmap_dy, ty * RW + j * kKs, n * a.Co + co0, &S.a_full[st]);
#endif
                if (++st == NA) {
                    st = 0;
                    ph ^= 1u;
                }
                if (++j == a.spt) {
                    j = 0;
                    if (++ty == a.ktiles) {
                        ty = 0;
                        ++n;
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ---- MMA issuer (one thread)
        if (lane == 0) {
            // Each accumulation period (`pp` per K-tile, a run of consecutive stages) accumulates into
            // its own TMEM buffer (period % 2), drained by the epilogue warps into fp32 registers: the
            // tensor core's own accumulation then spans at most ceil(spt/pp) stages, which keeps its
            // rounding error near fp32's (f4).
            // stage / period bookkeeping advanced incrementally (no per-stage division on this thread's
            // path); period q of a K-tile covers stages [floor(q spt / pp), floor((q+1) spt / pp))
            int64_t gp = 0;  // accumulation periods started so far
            int sa = 0, st = 0, j = 0, q = 0;
            uint32_t pha = 0, phb = 0;
            int q_start = 0, q_end = a.spt / a.pp;
            for (int64_t g = 0; g < nst; ++g) {
                const bool first = j == q_start;
                const bool last = j + 1 == q_end;
                const int b = (int)(gp & 1);
                if (first && gp >= 2) mbar_wait(&S.acc_empty[b], (uint32_t)((gp / 2) - 1) & 1u);
                // one wait per stage: the builders arrive on b_full only after the stage's dY tile has
                // landed (a_full), so b_full covers both operands
                WG_TRACE(g, 0);
                mbar_wait(&S.b_full[st], phb);
                WG_TRACE(g, 1);
                tc_fence_after();
                const uint32_t d = tmem + (uint32_t)(b * kAccStride);
                const uint32_t ab = smem_u32(S.a[sa]), bb = smem_u32(S.bhi[st]);
                if constexpr (PASSES == 3 && GIST_WG_ATMEM) {
                    static_assert(2 * kN + 64 * NB <= kTmemCols, "the A stages fit beside the accumulators");
                    const uint32_t at = tmem + a_tmem_col(st);
#pragma unroll
                    for (int kk = 0; kk < kKs / 8; ++kk) {  // K = 8 tf32 per instruction = 8 TMEM columns
                        const uint64_t db = umma_desc_sw128(bb + 32 * kk);
                        umma_tf32_ts(d, at + 8 * kk, db, kIdesc, (!first || kk != 0) ? 1u : 0u);
                        umma_tf32_ts(d, at + 8 * kk, umma_desc_sw128(smem_u32(S.blo[st]) + 32 * kk), kIdesc, 1u);
                        umma_tf32_ts(d, at + 32 + 8 * kk, db, kIdesc, 1u);
                    }
                } else {
#pragma unroll
                for (int kk = 0; kk < kKs / 8; ++kk) {  // K = 8 tf32 (32 bytes) per instruction
                    const uint64_t da = umma_desc_sw128(ab + 32 * kk), db = umma_desc_sw128(bb + 32 * kk);
                    umma_tf32(d, da, db, kIdesc, (!first || kk != 0) ? 1u : 0u);
                    if constexpr (PASSES == 3) {
                        umma_tf32(d, da, umma_desc_sw128(smem_u32(S.blo[st]) + 32 * kk), kIdesc, 1u);
                        umma_tf32(d, umma_desc_sw128(smem_u32(S.alo[st]) + 32 * kk), db, kIdesc, 1u);
                    }
                }
                }
                umma_commit(&S.b_empty[st]);  // the stage's smem (A and B) is free once these MMAs complete
                WG_TRACE(g, 2);
                if (last) {
                    umma_commit(&S.acc_full[b]);
                    ++gp;
                }
                if (++sa == NA) {
                    sa = 0;
                    pha ^= 1u;
                }
                if (++st == NB) {
                    st = 0;
                    phb ^= 1u;
                }
                if (last) {
                    if (++q == a.pp) q = 0;
                    q_start = q == 0 ? 0 : q_end;
                    q_end = ((q + 1) * a.spt) / a.pp;
                }
                if (++j == a.spt) j = 0;
            }
        }
    } else if (warp >= kEpi0) {
        // ---- epilogue: drain each K-tile's accumulator into fp32 registers (round-to-nearest adds),
        // then write this CTA's split-K partial.  Warp e covers TMEM lane quarter warp % 4 and the taps
        // of its half: 0-4 or 5-8 (16 columns per tap: n = tap * 16 + ci).
        const int e = warp - kEpi0;
        const int q = warp & 3, half = e >> 2;
        const int row = 32 * q + lane;
        float acc[5][kCiBlk];
#pragma unroll
        for (int i = 0; i < 5; ++i)
#pragma unroll
            for (int c = 0; c < kCiBlk; ++c) acc[i][c] = 0.0f;
        const int64_t nper = (t1 - t0) * a.pp;
        for (int64_t gp = 0; gp < nper; ++gp) {
            const int b = (int)(gp & 1);
            wait_backoff(&S.acc_full[b], (uint32_t)(gp / 2) & 1u);
            tc_fence_after();
#pragma unroll
            for (int i = 0; i < 5; ++i) {
                const int tap = 5 * half + i;
                if (tap < kTaps && !GIST_WG_SKIP_EPI) {
                    uint32_t v[16];
                    tmem_ld16(tmem + (uint32_t)(b * kAccStride) + ((uint32_t)(32 * q) << 16) + (uint32_t)(tap * kCiBlk), v);
                    tmem_wait_ld();
#pragma unroll
                    for (int c = 0; c < kCiBlk; ++c) acc[i][c] += __uint_as_float(v[c]);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive_1(&S.acc_empty[b]);
            if ((gp + 1) % a.pp != 0) continue;
            const int64_t t = t0 + gp / a.pp;
            if ((t + 1) % a.chunk == 0 || t + 1 == t1) {
                // chunk done: its fp32 partial goes to slot t / chunk; the reduce kernel sums the slots
                // in binary64 (DESIGN.md §6 f4: bounds the fp32 accumulation to `chunk` K-tiles)
                float *dst = a.partial + (((t / a.chunk) * a.Co + co0 + row) * a.Ci + ci0) * kTaps;
#pragma unroll
                for (int i = 0; i < 5; ++i) {
                    const int tap = 5 * half + i;
                    if (tap < kTaps)
#pragma unroll
                        for (int c = 0; c < kCiBlk; ++c) {
                            dst[c * kTaps + tap] = acc[i][c];
                            acc[i][c] = 0.0f;
                        }
                }
            }
        }
    } else if (warp >= kDec0) {
        // ---- decoders: for each K-tile t of this CTA, the input rows [oh0-1, oh0+R] of its image for
        // the 16 channels, zero-filled then scattered from the CSR rows that cover them, into slab
        // buffer (t - t0) % 2 while the builders read the other one
        const int dp = threadIdx.x - 32 * kDec0, dw = warp - kDec0;
        constexpr int kCh = kCiBlk / kDecWarps;
        const int npairs = kCh * a.rpc;
        // lane l's (channel, CSR row) pair of K-tile t: the row's entry range [e0, e1), issued one
        // K-tile ahead so that its latency hides under the previous K-tile's entry loads
        auto pair_range = [&](int64_t t, int32_t &e0, int32_t &e1) {
            e0 = e1 = 0;
            if (t >= t1 || lane >= npairs) return;
            const int n = (int)(t / a.ktiles), oh0 = (int)(t % a.ktiles) * a.R;
            const int ih_lo = max(0, oh0 - 1), ih_hi = min(a.H, oh0 + a.R + 1);
            if (ih_hi <= ih_lo) return;
            const int ci = dw * kCh + lane / a.rpc, rr = lane % a.rpc;
            const int64_t plane0 = ((int64_t)n * a.Ci + ci0 + ci) * a.H * a.W;
            const int64_t F0 = plane0 + (int64_t)ih_lo * a.W, F1 = plane0 + (int64_t)ih_hi * a.W;
            const int64_t r = (F0 >> 8) + rr;
            if (r <= (F1 - 1) >> 8) {
                e0 = r ? a.row_end[r - 1] : 0;
                e1 = a.row_end[r];
            }
        };
        int32_t cur_e0, cur_e1;
        pair_range(t0, cur_e0, cur_e1);
        for (int64_t t = t0; t < t1; ++t) {
            const int64_t tl = t - t0;
            const int sb = (int)(tl & 1);
            if (tl >= 2) wait_backoff(&S.slab_empty[sb], (uint32_t)((tl / 2) - 1) & 1u);
            float *slab = slabs + (size_t)sb * a.slab_floats;
            const int n = (int)(t / a.ktiles), ty = (int)(t % a.ktiles);
            const int oh0 = ty * a.R;
            {
                float4 *s4 = reinterpret_cast<float4 *>(slab);
                for (int i = dp; i < a.slab_floats / 4; i += kDecThreads) s4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
            named_bar(2, kDecThreads);  // the buffer is zero before any scatter
            const int ih_lo = max(0, oh0 - 1), ih_hi = min(a.H, oh0 + a.R + 1);
#if !GIST_WG_SKIP_DEC
            // Each warp decodes its 4 channels: lane l holds the entry range of (channel, CSR row) pair
            // l (<= 32 pairs, loaded one K-tile ahead); a warp scan flattens the pairs into one entry
            // list, and the lanes load kDecU entries each (all in flight) before scattering them.
            {
                const int32_t pe0 = cur_e0, pcnt = cur_e1 - cur_e0;
                int pend = pcnt;  // inclusive end of pair `lane` in the flat list
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const int u = __shfl_up_sync(kFull, pend, d);
                    if (lane >= d) pend += u;
                }
                const int total = __shfl_sync(kFull, pend, 31);
                int p = 0;  // pair of this lane's current entry (entries are visited in increasing order)
                for (int k0 = 0; k0 < total; k0 += 32 * kDecU) {
                    int32_t kk[kDecU];
                    int pr[kDecU];
                    uint8_t cv[kDecU];
                    float vv[kDecU];
#pragma unroll
                    for (int u = 0; u < kDecU; ++u) {
                        const int k = k0 + 32 * u + lane;
                        // advance to the first pair whose end exceeds k (whole-warp shuffles: every
                        // lane takes part in each round, so each source lane is active)
                        for (;;) {
                            const int nxt = __shfl_sync(kFull, pend, p);
                            const bool adv = k < total && k >= nxt;
                            if (!__any_sync(kFull, adv)) break;
                            if (adv) ++p;
                        }
                        pr[u] = k < total ? p : -1;
                    }
#pragma unroll
                    for (int u = 0; u < kDecU; ++u) {
                        // entry index: the pair's first entry + the offset inside the pair
                        const int ps = pr[u] < 0 ? 0 : pr[u];
                        const int32_t e0p = __shfl_sync(kFull, pe0, ps), endp = __shfl_sync(kFull, pend, ps),
                                      cntp = __shfl_sync(kFull, pcnt, ps);
                        const int k = k0 + 32 * u + lane;
                        kk[u] = e0p + (k - (endp - cntp));
                        if (pr[u] >= 0) {
                            cv[u] = a.col[kk[u]];
                            vv[u] = a.val[kk[u]];
                        }
                    }
                    if (k0 == 0) pair_range(t + 1, cur_e0, cur_e1);  // the next K-tile's ranges, in flight now
#pragma unroll
                    for (int u = 0; u < kDecU; ++u) {
                        if (pr[u] < 0) continue;
                        const int ci = dw * kCh + pr[u] / a.rpc, rr = pr[u] % a.rpc;
                        const int64_t plane0 = ((int64_t)n * a.Ci + ci0 + ci) * a.H * a.W;
                        const int64_t F0 = plane0 + (int64_t)ih_lo * a.W, F1 = plane0 + (int64_t)ih_hi * a.W;
                        const int64_t flat = 256 * ((F0 >> 8) + rr) + cv[u];
                        if (flat >= F0 && flat < F1) {
                            uint32_t ih, iw;
                            a.div_w.divmod((uint32_t)(flat - plane0), ih, iw);
                            // racecheck reports these slab writes against the builders' slab reads: they
                            // are ordered by slab_full[sb] (decoder arrive, release -> builder wait,
                            // acquire) and, for the next refill, slab_empty[sb] (builder arrive -> wait)
                            slab[(size_t)ci * SR * SW + ((int)ih - oh0 + 1) * SW + (int)iw + 1] = vv[u];
                        }
                    }
                }
                if (total == 0) pair_range(t + 1, cur_e0, cur_e1);
            }
#else
            pair_range(t + 1, cur_e0, cur_e1);
#endif
            __syncwarp();
            if (dp == 0) WG_TRACE(tl * a.spt, 5);
            if (lane == 0) mbar_arrive_1(&S.slab_full[sb]);
        }
    } else {
        // ---- builders: per stage, B rows (tap, ci) x 32 positions from the slab (hi and lo parts) and
        // A_lo; thread p owns channel ci_b and the 4-position chunk ch of every stage
        const int p = threadIdx.x - 32 * kBld0;
        const int ci_b = p >> 3, ch = p & 7;
        for (int64_t t = t0; t < t1; ++t) {
            const int64_t tl = t - t0;
            const int sb = (int)(tl & 1);
            mbar_wait(&S.slab_full[sb], (uint32_t)(tl / 2) & 1u);
            const float *slab = slabs + (size_t)sb * a.slab_floats;
            const int oh0 = (int)(t % a.ktiles) * a.R;
            for (int j = 0; j < a.spt; ++j) {
                const int64_t g = tl * a.spt + j;
                const int st = (int)(g % NB), sa = (int)(g % NA);
                if (g >= NB) mbar_wait(&S.b_empty[st], (uint32_t)((g / NB) - 1) & 1u);
                if (p == 0) WG_TRACE(g, 3);
                const int pos = j * kKs + 4 * ch;  // the chunk's first position in the K-tile
                uint32_t ohr = 0, ow = 0;
                a.div_w.divmod((uint32_t)pos, ohr, ow);
                unsigned char *bh = reinterpret_cast<unsigned char *>(S.bhi[st]);
                unsigned char *bl = reinterpret_cast<unsigned char *>(S.blo[PASSES == 3 ? st : 0]);
                if (GIST_WG_SKIP_B) {
                } else if constexpr (VEC) {
                    // W % 4 == 0: the chunk lies in one output row at ow % 4 == 0; slab row kh holds the
                    // 6 inputs (cols ow .. ow+5) of its 3 taps: two 16-byte loads
                    const bool valid = pos < RW && oh0 + (int)ohr < a.H;
                    const float *src = slab + ((size_t)ci_b * SR + ohr) * SW + ow;
#pragma unroll
                    for (int kh = 0; kh < 3; ++kh) {
                        float4 l0 = make_float4(0.f, 0.f, 0.f, 0.f), l1 = l0;
                        if (valid) {
                            l0 = *reinterpret_cast<const float4 *>(src + kh * SW);
                            l1 = *reinterpret_cast<const float4 *>(src + kh * SW + 4);
                        }
                        const float v[6] = {l0.x, l0.y, l0.z, l0.w, l1.x, l1.y};
                        float hi[6], lo[6];
#pragma unroll
                        for (int e = 0; e < 6; ++e) {
                            hi[e] = PASSES == 3 ? to_tf32(v[e]) : v[e];
                            lo[e] = v[e] - hi[e];
                        }
#pragma unroll
                        for (int kw = 0; kw < 3; ++kw) {
                            const uint32_t off = sw128_offset((uint32_t)((3 * kh + kw) * kCiBlk + ci_b), (uint32_t)ch);
                            *reinterpret_cast<float4 *>(bh + off) = make_float4(hi[kw], hi[kw + 1], hi[kw + 2], hi[kw + 3]);
                            if constexpr (PASSES == 3)
                                *reinterpret_cast<float4 *>(bl + off) = make_float4(lo[kw], lo[kw + 1], lo[kw + 2], lo[kw + 3]);
                        }
                    }
                } else {
                    // any W: the 4 positions may straddle an output row; slab offset of each for tap (0, 0)
                    int off[4];
                    bool ok[4];
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        ok[e] = pos + e < RW && oh0 + (int)ohr < a.H;
                        off[e] = ((ci_b * SR) + (int)ohr) * SW + (int)ow;
                        if (++ow == (uint32_t)a.W) {
                            ow = 0;
                            ++ohr;
                        }
                    }
#pragma unroll
                    for (int tap = 0; tap < kTaps; ++tap) {
                        const int kh = tap / 3, kw = tap % 3;
                        float v[4], hi[4], lo[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            v[e] = ok[e] ? slab[off[e] + kh * SW + kw] : 0.0f;
                            hi[e] = PASSES == 3 ? to_tf32(v[e]) : v[e];
                            lo[e] = v[e] - hi[e];
                        }
                        const uint32_t o = sw128_offset((uint32_t)(tap * kCiBlk + ci_b), (uint32_t)ch);
                        *reinterpret_cast<float4 *>(bh + o) = make_float4(hi[0], hi[1], hi[2], hi[3]);
                        if constexpr (PASSES == 3)
                            *reinterpret_cast<float4 *>(bl + o) = make_float4(lo[0], lo[1], lo[2], lo[3]);
                    }
                }
                if (PASSES == 3 && GIST_WG_ATMEM) {
                    // A_hi = tf32_rn(A), A_lo = A - A_hi (exact) into tensor memory: builder thread = one row
                    // (output channel) of the dY tile, its lane of the warp's TMEM lane quarter
                    mbar_wait(&S.a_full[sa], (uint32_t)(g / NA) & 1u);
                    const uint32_t r = 32u * (uint32_t)(warp & 3) + (uint32_t)lane;
                    const unsigned char *arow = reinterpret_cast<const unsigned char *>(S.a[sa]);
                    uint32_t hv[32], lv[32];
#pragma unroll
                    for (int c = 0; c < 8; ++c) {  // chunk c (k = 4c .. 4c+3) of row r, 128-byte swizzle
                        const float4 x = *reinterpret_cast<const float4 *>(arow + sw128_offset(r, (uint32_t)c));
                        const float xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            const float h = to_tf32(xs[e]);
                            hv[4 * c + e] = __float_as_uint(h);
                            lv[4 * c + e] = __float_as_uint(xs[e] - h);
                        }
                    }
                    const uint32_t taddr = tmem + ((32u * (uint32_t)(warp & 3)) << 16) + a_tmem_col(st);
                    tmem_st32(taddr, hv);
                    tmem_st32(taddr + 32, lv);
                    tmem_wait_st();
                    tc_fence_before();
                } else if (PASSES == 3 && !GIST_WG_SKIP_ASPLIT) {
                    // A_hi = tf32_rn(A) written back in place, A_lo = A - A_hi (exact in fp32); the layouts
                    // of a[] and alo[] are identical, so chunk by chunk
                    mbar_wait(&S.a_full[sa], (uint32_t)(g / NA) & 1u);
                    float4 *ar = reinterpret_cast<float4 *>(S.a[sa]);
                    float4 *al = reinterpret_cast<float4 *>(S.alo[st]);
#pragma unroll
                    for (int i = 0; i < kM * kKs / 4 / kBldThreads; ++i) {
                        const float4 x = ar[p + i * kBldThreads];
                        const float4 h = make_float4(to_tf32(x.x), to_tf32(x.y), to_tf32(x.z), to_tf32(x.w));
                        ar[p + i * kBldThreads] = h;
                        al[p + i * kBldThreads] = make_float4(x.x - h.x, x.y - h.y, x.z - h.z, x.w - h.w);
                    }
                }
                if constexpr (PASSES == 1) mbar_wait(&S.a_full[sa], (uint32_t)(g / NA) & 1u);  // b_full implies A
                fence_proxy_async_smem();  // generic smem writes -> visible to the tensor core (async proxy)
                __syncwarp();
                if (p == 0) WG_TRACE(g, 4);
                if (lane == 0) mbar_arrive_1(&S.b_full[st]);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive_1(&S.slab_empty[sb]);  // this K-tile's slab is no longer read
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc<kTmemCols>(tmem);
    }
}

// dW = the chunk partials summed in binary64 in slot order (deterministic), rounded once to fp32
__global__ void __launch_bounds__(256) wgrad_reduce_kernel(const float *__restrict__ partial, int32_t units,
                                                           int64_t count, float *__restrict__ dw) {
    pdl_enter();
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        double acc = 0.0;
        for (int u = 0; u < units; ++u) acc += (double)partial[(int64_t)u * count + i];
        dw[i] = (float)acc;
    }
}

struct WgPlan {
    int32_t R, spt, ktiles, m_blocks, n_blocks, splits, pp, chunk, units;
    int64_t T;
};

constexpr int64_t kChunkK = 8192;  // output positions (GEMM K) per fp32 partial

WgPlan wg_plan(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes) {
    WgPlan P{};
    // R output rows per K-tile: about 256 positions, and R*W % 4 == 0 so that every K-tile's dY box
    // starts 16-byte aligned (a TMA requirement); one tile when that covers the whole map
    const int32_t m = W % 4 == 0 ? 1 : W % 2 == 0 ? 2 : 4;
    P.R = std::max(1, 256 / W);
    P.R = (P.R + m - 1) / m * m;
    if (P.R >= H) P.R = H;
    P.spt = (int32_t)ceil_div((int64_t)P.R * W, kKs);
    P.ktiles = (int32_t)ceil_div(H, P.R);
    P.T = (int64_t)N * P.ktiles;
    P.m_blocks = Co / kM;
    P.n_blocks = Ci / kCiBlk;
    P.pp = passes == 3 ? std::min<int32_t>(2, P.spt) : 1;
    P.chunk = (int32_t)std::max<int64_t>(1, kChunkK / ((int64_t)P.R * W));
    P.units = (int32_t)ceil_div(P.T, P.chunk);
    const int64_t tiles = (int64_t)P.m_blocks * P.n_blocks;
    int64_t s = std::max<int64_t>(1, num_sms() / std::max<int64_t>(1, tiles));
    if (s > P.units) s = P.units;
    P.splits = (int32_t)std::max<int64_t>(1, s);
    return P;
}

int32_t slab_pitch(int32_t W) { return (W + 2 + 3) / 4 * 4; }

#ifndef GIST_WG_NS3
#define GIST_WG_NS3 2  // pipeline stages, 3xTF32 (3 with A in TMEM: no faster)
#endif
#ifndef GIST_WG_NS1
#define GIST_WG_NS1 4  // pipeline stages, 1xTF32 (3xTF32: 2; a deeper dY-only ring measured slower)
#endif
constexpr int kNS1 = GIST_WG_NS1, kNS3 = GIST_WG_NS3;
constexpr size_t kMaxSmemW = 227 * 1024;

template <int PASSES, int NA, int NB>
size_t wg_smem_bytes(const WgPlan &P, int32_t W) {
    return sizeof(WgSmem<PASSES, NA, NB>) + 2 * (size_t)kCiBlk * (P.R + 2) * slab_pitch(W) * 4 + 1024;
}

PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }
    return fn;
}

template <int PASSES, int NA, int NB, bool VEC>
cudaError_t launch_wg(const CUtensorMap &tm, const WgArgs &args, const WgPlan &P, int32_t W, cudaStream_t s) {
    static PerDeviceAttr attr;
    const size_t smem = wg_smem_bytes<PASSES, NA, NB>(P, W);
    const cudaError_t ea =
        attr.ensure(reinterpret_cast<const void *>(wgrad_ssdc_kernel<PASSES, NA, NB, VEC>), (int)smem);
    if (ea != cudaSuccess) return ea;
    const unsigned grid = (unsigned)((int64_t)P.m_blocks * P.n_blocks * P.splits);
    launch_k(wgrad_ssdc_kernel<PASSES, NA, NB, VEC>, grid, kThreads, smem, s, tm, args);
    return cudaPeekAtLastError();
}

}  // namespace

#ifdef GIST_WG_TRACE
extern "C" int gist_debug_wg_trace(void *buf) { return (int)cudaMemcpyToSymbol(g_wg_trace, &buf, sizeof(void *)); }
#endif

size_t wgrad_smem_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes);
constexpr size_t kMaxSmem = 227 * 1024;  // sm_100 opt-in dynamic shared memory per CTA

bool wgrad_shape_ok(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W) {
    // H*W % 4: the dY rows are TMA rows, whose stride must be a multiple of 16 bytes; the decode slab
    // of R+2 rows must fit beside the pipeline stages (odd W > 64 needs R = 4: W <= 252 is not enough)
    if (!(N > 0 && H > 0 && W > 0 && Co % kM == 0 && Ci % kCiBlk == 0 && W <= 252 && (int64_t)H * W % 4 == 0))
        return false;
    const WgPlan P = wg_plan(N, Ci, Co, H, W, 3);
    const int64_t rpc = ((int64_t)(P.R + 2) * W + 255) / 256 + 1;  // decoder pairs: 16 * rpc <= 128
    return (kCiBlk / kDecWarps) * rpc <= 32 && wgrad_smem_bytes(N, Ci, Co, H, W, 3) <= kMaxSmem &&
           wgrad_smem_bytes(N, Ci, Co, H, W, 1) <= kMaxSmem;
}

size_t wgrad_workspace_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W) {
    const WgPlan P = wg_plan(N, Ci, Co, H, W, 3);  // units do not depend on passes
    return (size_t)P.units * Co * Ci * kTaps * 4;
}

size_t wgrad_smem_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes) {
    const WgPlan P = wg_plan(N, Ci, Co, H, W, passes);
    return passes == 3 ? wg_smem_bytes<3, 2, 2>(P, W) : wg_smem_bytes<1, 4, 4>(P, W);  // the shallow ring always fits
}

cudaError_t launch_wgrad_ssdc(const float *dy, const int32_t *row_end, const uint8_t *col, const float *val, int32_t N,
                              int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes, float *dw, void *workspace,
                              cudaStream_t s, int *launches) {
    *launches = 0;
    auto encode = tensor_map_encoder();
    if (!encode) return cudaErrorNotSupported;
    const WgPlan P = wg_plan(N, Ci, Co, H, W, passes);
    CUtensorMap tm;
    const cuuint64_t gdim[2] = {(cuuint64_t)H * W, (cuuint64_t)N * Co};
    const cuuint64_t gstride[1] = {(cuuint64_t)H * W * 4};
    const cuuint32_t box[2] = {(cuuint32_t)kKs, (cuuint32_t)kM};
    const cuuint32_t estride[2] = {1, 1};
    const CUresult r = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(dy), gdim, gstride, box,
                              estride, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return cudaErrorInvalidValue;
    WgArgs args{};
    args.row_end = row_end;
    args.col = col;
    args.val = val;
    args.partial = reinterpret_cast<float *>(workspace);
    args.N = N;
    args.Ci = Ci;
    args.Co = Co;
    args.H = H;
    args.W = W;
    args.R = P.R;
    args.spt = P.spt;
    args.ktiles = P.ktiles;
    args.m_blocks = P.m_blocks;
    args.n_blocks = P.n_blocks;
    args.splits = P.splits;
    args.pp = P.pp;
    args.chunk = P.chunk;
    args.units = P.units;
    args.T = P.T;
    args.div_w = FastDiv::make((uint32_t)W);
    args.SWP = slab_pitch(W);
    args.rpc = (int32_t)(((int64_t)(P.R + 2) * W + 255) / 256 + 1);
    args.slab_floats = kCiBlk * (P.R + 2) * args.SWP;
    const bool vec = W % 4 == 0;
    // the deeper dY ring when the slabs leave room for it
    const bool deep1 = wg_smem_bytes<1, kNS1, kNS1>(P, W) <= kMaxSmemW;
    cudaError_t e;
    const bool deep3 = wg_smem_bytes<3, kNS3, kNS3>(P, W) <= kMaxSmemW;
    if (passes == 3) {
        if (deep3) e = vec ? launch_wg<3, kNS3, kNS3, true>(tm, args, P, W, s) : launch_wg<3, kNS3, kNS3, false>(tm, args, P, W, s);
        else e = vec ? launch_wg<3, 2, 2, true>(tm, args, P, W, s) : launch_wg<3, 2, 2, false>(tm, args, P, W, s);
    } else {
        if (deep1) e = vec ? launch_wg<1, kNS1, kNS1, true>(tm, args, P, W, s) : launch_wg<1, kNS1, kNS1, false>(tm, args, P, W, s);
        else e = vec ? launch_wg<1, 4, 4, true>(tm, args, P, W, s) : launch_wg<1, 4, 4, false>(tm, args, P, W, s);
    }
    if (e != cudaSuccess) return e;
    ++*launches;
    const int64_t count = (int64_t)Co * Ci * kTaps;
    int64_t blocks = ceil_div(count, 256);
    if (blocks > (int64_t)num_sms() * 8) blocks = (int64_t)num_sms() * 8;
    launch_k(wgrad_reduce_kernel, (unsigned)blocks, 256, 0, s, (const float *)args.partial, P.units, count, dw);
    const cudaError_t e2 = cudaPeekAtLastError();
    if (e2 != cudaSuccess) return e2;
    ++*launches;
    return cudaSuccess;
}

}  // namespace gist
