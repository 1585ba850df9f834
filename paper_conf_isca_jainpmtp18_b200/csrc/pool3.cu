// pool3.cu — a2 (+a1 fused) and a3 for 3x3 windows, stride 1 or 2, padding 0 or 1, floor or ceil
// mode: the AlexNet / NiN / GoogLeNet pools (§III-A, P:151-P:156 §IV-A).
//
// Plane tiles through a TMA ring.  A tile is G whole planes; their input (forward) or their dY,
// argmax words and mask words (backward) are contiguous ranges of the maps, so one persistent CTA
// per (half) SM streams tile after tile into a 2-4 stage shared-memory ring with 1-D bulk copies
// (cp.async.bulk, issued by one thread) while its 256 threads compute the current tile from shared
// memory: HBM sees each byte once, and the loads of the next tiles are in flight during compute.
//   forward, stride 2: one thread per output (lanes = consecutive outputs); taps outside the input
//     read as -inf (never selected under the strict '>' rule, R3), the argmax starts at the
//     window's first in-bounds position, so an all -inf window gives the oracle's index.  8-lane
//     groups OR their nibbles into one argmax word.
//   forward, stride 1: separable.  One thread per output column of a plane walks down the rows,
//     keeping the row-wise (max, index) of the last three input rows: each input row is scanned
//     once, not three times.  Scanning rows, then combining the row results in row order with the
//     same rule, is the row-major scan of the window (last NaN wins, else first maximum).
//     Nibbles go to shared memory (one byte per output) and are packed into words afterwards.
//   the a1 mask (forward, when requested): one thread per mask word reads its 32 staged floats.
//   backward, stride 2: one thread per 2x2 input block: its 4 candidate windows (A-1,b-1), (A-1,b),
//     (A,b-1), (A,b) route fixed nibbles to fixed block positions, in ascending output order (R6).
//   backward, stride 1: one thread per input element, its 9 candidate windows in ascending output
//     order; both select with the mask bit (R7).
// Word ownership (forward): a tile owns the argmax words whose first output lies in its planes and
// the mask words whose first element does; the tail of its last word may lie in the next plane, so
// the tile also stages the first rows of plane p0+G.  Tiles never share an output word.
#include <math_constants.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "kernels.h"
#include "tma.cuh"

namespace gist {

namespace {

#ifndef GIST_POOL3_THREADS
#define GIST_POOL3_THREADS 512  // 256: 10-40% slower, 1024: 5-25% slower (3x3/s1 maps, GoogLeNet b64)
#endif
constexpr int kRT = GIST_POOL3_THREADS;  // threads per CTA
#ifndef GIST_POOL3_BWD_SEG
#define GIST_POOL3_BWD_SEG 0  // 1: row segments for tiles with few columns (measured slower in the C4 step)
#endif
#ifndef GIST_POOL3_BWD_HITS
#define GIST_POOL3_BWD_HITS 1  // backward through hit masks (0: nibble planes + per-input tests)
#endif
#ifndef GIST_POOL3_BWD_STRIP
#define GIST_POOL3_BWD_STRIP 1  // stride-1 backward: column strips for tiles of >= kRT/2 columns (0: never)
#endif
constexpr int kMaxRS = 4;  // ring stages: a.rs <= kMaxRS stages of a.sf floats (host: ring_for)
constexpr int kNbBytes = 12 * 1024;   // nibble bytes of one tile (nibble-plane backward)
constexpr int kNbFwd = 8 * 1024;      // forward: nibble bytes of one tile, two tiles' worth in the aux area
constexpr int kHitBytes = 16 * 1024;  // hit masks of one tile (backward): 16 bits (S = 1) or 4 bits per input
constexpr int kAuxBytes = kHitBytes;  // the per-CTA area after the ring (>= kNbBytes)

struct P3Args {
    int32_t H, W, Ho, Wo, S, P;
    int32_t HW, HoWo;
    int32_t G;       // planes per tile
    int32_t xrows;   // forward: input rows of plane p0+G a tile may need (0: none)
    int32_t hb, wb;  // stride-2 backward: 2x2 blocks per plane (rows, columns)
    int32_t PR, PC;  // backward: padded nibble-byte plane (rows, columns)
    int32_t a_off, m_off;  // backward stage layout (floats): dY at 0, argmax words, mask words
    int32_t segs, segr;    // stride-2 forward: row segments per plane column, output rows per segment
    int32_t rs, sf;        // ring: stages, floats per stage
    int32_t bands, br;     // stride-2 forward of planes larger than a stage: bands per plane, output rows per band
    int64_t NC, tiles, n_in, n_out;
    FastDiv div_hw, div_w, div_howo, div_wo, div_blk, div_wb, div_seg;
};

__device__ __forceinline__ void take3(float v, int idx, float &best, int &bi) {
    if (v > best || v != v) {  // R3: strict '>' keeps the first maximum; NaN always wins
        best = v;
        bi = idx;
    }
}

template <bool RELU>
__device__ __forceinline__ float act3(float v) {
    return RELU ? (v < 0.0f ? 0.0f : v) : v;  // f3 in-place ReLU (R21)
}

// The bulk copy of floats [lo, hi) of g: from the 16-B aligned sb = lo & ~3, the whole quads; the
// ragged <= 3 elements at the end are loaded by the consumers (tail_fill).
__device__ __forceinline__ uint32_t ring_bytes(int64_t lo, int64_t hi) {
    return (uint32_t)(((hi - (lo & ~3ll)) & ~3ll) * 4);
}

__device__ __forceinline__ void ring_copy(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    constexpr uint32_t kChunk = 16 * 1024;  // several copies in flight per stage
    for (uint32_t off = 0; off < bytes; off += kChunk)
        tma_load_1d(static_cast<char *>(dst) + off, static_cast<const char *>(src) + off,
                    bytes - off < kChunk ? bytes - off : kChunk, bar);
}

// Loads the ragged tail (elements past the bulk-copied quads) of [lo, hi) with threads tid0..tid0+2.
template <typename T>
__device__ __forceinline__ bool tail_fill(T *dst, const T *__restrict__ src, int64_t lo, int64_t hi, int tid0) {
    const int64_t sb = lo & ~3ll, te = sb + ((hi - sb) & ~3ll);
    const int t = (int)threadIdx.x - tid0;
    if (t >= 0 && t < hi - te) {
        dst[te - sb + t] = src[te + t];
        return true;
    }
    return false;
}

struct FwdTile {
    int64_t p0, lo, hi, oa, ob, ia, ib;
    int64_t ce;   // end of the bulk-copied range (>= hi except at the map's ragged end)
    int64_t olo;  // first output of the tile (plane p0, output row oh0)
    int np;
    int oh0, oh1;  // output rows of the tile's planes ([0, Ho) unless banded)
};

__device__ __forceinline__ FwdTile fwd_tile(const P3Args &a, int64_t k) {
    FwdTile t;
    if (a.bands > 1) {
        // one band of output rows [oh0, oh1) of plane p0 (stride 2, P = 0, Wo % 8 == 0 and 2W % 32 ==
        // 0, so a band owns whole argmax words and the mask words of its input rows [2 oh0, 2 oh1),
        // the last band up to H); it stages input rows [2 oh0, min(H, 2 oh1 + 1))
        t.p0 = k / a.bands;
        const int b = (int)(k - t.p0 * a.bands);
        t.np = 1;
        t.oh0 = b * a.br;
        t.oh1 = min(a.Ho, t.oh0 + a.br);
        const int64_t pb = t.p0 * a.HW;
        const int ih_own1 = t.oh1 == a.Ho ? a.H : 2 * t.oh1;
        t.olo = t.p0 * a.HoWo + (int64_t)t.oh0 * a.Wo;
        t.oa = t.olo;
        t.ob = t.p0 * a.HoWo + (int64_t)t.oh1 * a.Wo;
        t.ia = pb + (int64_t)(2 * t.oh0) * a.W;
        t.ib = pb + (int64_t)ih_own1 * a.W;
        t.lo = t.ia;
        t.hi = pb + (int64_t)min(a.H, 2 * t.oh1 + 1) * a.W;
        const int64_t up = (t.hi + 3) & ~3ll;
        t.ce = up <= a.n_in ? up : (t.hi & ~3ll);
        if (t.ce < (t.lo & ~3ll)) t.ce = t.lo & ~3ll;
        return t;
    }
    t.oh0 = 0;
    t.oh1 = a.Ho;
    t.p0 = k * a.G;
    t.np = (int)min((int64_t)a.G, a.NC - t.p0);
    const bool last = t.p0 + t.np == a.NC;
    t.oa = (t.p0 * a.HoWo + 7) & ~7ll;
    t.ob = last ? a.n_out : (((t.p0 + t.np) * a.HoWo + 7) & ~7ll);
    t.ia = (t.p0 * a.HW + 31) & ~31ll;
    t.ib = last ? a.n_in : (((t.p0 + t.np) * a.HW + 31) & ~31ll);
    t.olo = t.p0 * a.HoWo;
    t.lo = t.p0 * a.HW;
    const int64_t end = t.lo + (int64_t)t.np * a.HW;
    t.hi = last ? end : min(a.n_in, end + max((int64_t)a.xrows * a.W, t.ib - end));
    // the copy ends on a 16-byte boundary past hi when the map has the elements (<= 3 more floats,
    // within the stage's slack), so only the map's last tile needs threads to load a ragged tail
    const int64_t up = (t.hi + 3) & ~3ll;
    t.ce = up <= a.n_in ? up : (t.hi & ~3ll);
    if (t.ce < (t.lo & ~3ll)) t.ce = t.lo & ~3ll;
    return t;
}

// Row-wise scan of input row ih over columns iw0 .. iw0+2 (stride 1): (max, column index).
template <bool RELU>
__device__ __forceinline__ void hscan(const float *row, int ih, int iw0, const P3Args &a, float &v, int &x) {
    v = -CUDART_INF_F;
    x = max(0, -iw0);
    if (ih < 0 || ih >= a.H) return;
#pragma unroll
    for (int dx = 0; dx < 3; ++dx) {
        const int iw = iw0 + dx;
        if (iw >= 0 && iw < a.W) take3(act3<RELU>(row[iw]), dx, v, x);
    }
}

template <int S, bool MASK, bool RELU, bool CHECK>
__global__ void __launch_bounds__(kRT)
pool3_fwd_kernel(const float *__restrict__ y, P3Args a, float *__restrict__ out, uint32_t *__restrict__ arg,
                 uint32_t *__restrict__ mask) {
    pdl_enter();
    extern __shared__ __align__(128) unsigned char smp[];
    float *ring = reinterpret_cast<float *>(smp);
    uint8_t *nbs0 = smp + (size_t)a.rs * a.sf * 4;  // nibble bytes of two tiles (one per output), kNbFwd each
    uint64_t *full = reinterpret_cast<uint64_t *>(nbs0 + kAuxBytes);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const float ninf = -CUDART_INF_F;
    if (tid == 0) {
        for (int s = 0; s < a.rs; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    FwdTile *desc = reinterpret_cast<FwdTile *>(full + kMaxRS);  // per stage: the tile it holds
    const int64_t mine = a.tiles > blockIdx.x ? (a.tiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    // one thread computes a tile's ranges when it issues the tile's copy and leaves them with the
    // stage (the full barrier's arrive releases them to the consumers)
    auto issue = [&](int64_t j, int st) {
        const FwdTile t = fwd_tile(a, blockIdx.x + j * gridDim.x);
        desc[st] = t;
        const uint32_t b = (uint32_t)((t.ce - (t.lo & ~3ll)) * 4);
        mbar_arrive_expect_tx(&full[st], b);
        if (b) ring_copy(ring + (size_t)st * a.sf, y + (t.lo & ~3ll), b, &full[st]);
    };
    // argmax words of a finished tile from its nibble bytes (8 per word, one aligned 64-bit load);
    // only the map's last word can be partial (its pad nibbles are 0).  Run one tile later, between
    // the next tile's walk and the barrier that ends it (the bytes are double-buffered).
    auto pack = [&](const FwdTile &t, const uint8_t *nbs) {
        const int64_t olo = t.olo;
        const int64_t olo8 = S == 2 ? (olo & ~7ll) : olo;  // stride 1: tiles hold whole words
        const int w0 = S == 2 ? (int)((t.oa - olo8) >> 3) : 0;
        const int64_t oend = S == 2 ? t.ob : olo + (int64_t)t.np * a.HoWo;
        const int w1 = (int)((oend - olo8 + 7) >> 3);
        const int nvalid = (int)(oend - olo8);  // nibble bytes from olo8 on
        for (int w = w0 + tid; w < w1; w += kRT) {
            const uint2 b = *reinterpret_cast<const uint2 *>(nbs + 8 * w);
            const uint32_t lo4 = (b.x & 0xfu) | ((b.x >> 4) & 0xf0u) | ((b.x >> 8) & 0xf00u) | ((b.x >> 12) & 0xf000u);
            const uint32_t hi4 = (b.y & 0xfu) | ((b.y >> 4) & 0xf0u) | ((b.y >> 8) & 0xf00u) | ((b.y >> 12) & 0xf000u);
            const int valid = nvalid - 8 * w;
            const uint32_t keep = valid >= 8 ? ~0u : ((1u << (4 * valid)) - 1u);
            arg[(olo8 >> 3) + w] = (lo4 | (hi4 << 16)) & keep;
        }
    };
    if (tid == 0)
        for (int64_t j = 0; j < a.rs && j < mine; ++j) issue(j, (int)j);
    int st = 0;
    uint32_t ph = 0;
    FwdTile prev{};
    for (int64_t j = 0; j < mine; ++j) {
        float *R = ring + (size_t)st * a.sf;
        uint8_t *nbs = nbs0 + (j & 1) * kNbFwd;
        mbar_wait(&full[st], ph);
        const FwdTile t = desc[st];
        const int64_t sb = t.lo & ~3ll;  // stage index of element e: e - sb
        if (t.ce < t.hi) {  // the map's ragged end (tile-uniform): threads load the last <= 3 elements
            if (tid < t.hi - t.ce) {
                R[t.ce - sb + tid] = y[t.ce + tid];
                fence_proxy_async_smem();  // generic writes into a TMA stage
            }
            __syncthreads();
        }
        // a1 mask words [ia/32, ib/32) (relu(y) > 0 iff y > 0): lane l of a warp reads element
        // 32 w + l of each of 4 words (conflict-free), one ballot per word; tile-local 32-bit indices
        if (MASK) {
            const int nw = (int)((t.ib - t.ia + 31) >> 5);
            const int lim = (int)(t.hi - t.ia);  // staged elements from ia (the map ends there)
            const float *E = R + (t.ia - sb);
            uint32_t *mw = mask + (t.ia >> 5);
            // every tile but the map's last: whole groups of 4 words without bounds tests
            const int nw4 = lim >= 32 * nw ? (nw & ~3) : 0;
            for (int w0 = warp * 4; w0 < nw4; w0 += kRT / 8) {
                const float *e = E + 32 * w0 + lane;  // O1: y > 0 (NaN, -0.0 -> 0)
                uint32_t word = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t b = __ballot_sync(kFull, e[32 * k] > 0.0f);
                    word = lane == k ? b : word;
                }
                if (lane < 4) mw[w0 + lane] = word;
            }
            for (int w = nw4 + warp; w < nw; w += kRT / 32) {  // the rest, elements past the map read 0
                const int e = 32 * w + lane;
                const uint32_t b = __ballot_sync(kFull, e < lim && E[e] > 0.0f);
                if (lane == 0) mw[w] = b;
            }
        }
        const int64_t olo = t.olo;
        if (S == 2) {
            // one thread per (plane, output column, row segment) walks down the segment's output
            // rows: input row 2 oh - P + 2 of one output is row 2 (oh + 1) - P of the next, so each
            // step scans two new input rows (separable, as for stride 1).  Nibble bytes go to
            // shared memory by output index - olo8 (word boundaries 8-byte aligned).
            const int64_t olo8 = olo & ~7ll;
            // banded tiles: the tile's output rows [t.oh0, t.oh1) of plane p0; P0 addresses row 0 of
            // that plane (rows above the band are not staged and not read)
            uint8_t *nb0 = nbs + (olo - olo8) - (int64_t)t.oh0 * a.Wo;
            const float *P0 = R + (t.p0 * a.HW - sb);  // plane 0 of the tile
            float *otile = out + olo - (int64_t)t.oh0 * a.Wo;
            const int items = t.np * a.segs * a.Wo;
            for (int it = tid; it < items; it += kRT) {
                uint32_t ps, ow, pl, sg;
                a.div_wo.divmod((uint32_t)it, ps, ow);
                a.div_seg.divmod(ps, pl, sg);
                const int oh0 = t.oh0 + (int)sg * a.segr, oh1 = min(t.oh1, oh0 + a.segr);
                const float *pb = P0 + (int)pl * a.HW;
                const int iw0 = 2 * (int)ow - a.P;
                const int dx0 = max(0, -iw0);
                int oo = (int)pl * a.HoWo + (int)ow;  // tile-local output index
                if (!CHECK) {
                    // every window inside the plane: the first tap of a row starts its scan, the
                    // first row starts the window's (equal to the -inf start of R3's scan)
                    const float *r = pb + 2 * oh0 * a.W + iw0;
                    oo += oh0 * a.Wo;
                    float hv0 = act3<RELU>(r[0]);
                    int hx0 = 0;
                    take3(act3<RELU>(r[1]), 1, hv0, hx0);
                    take3(act3<RELU>(r[2]), 2, hv0, hx0);
                    for (int oh = oh0; oh < oh1; ++oh) {
                        r += a.W;
                        float hv1 = act3<RELU>(r[0]), hv2 = act3<RELU>(r[a.W]);
                        int hx1 = 0, hx2 = 0;
                        take3(act3<RELU>(r[1]), 1, hv1, hx1);
                        take3(act3<RELU>(r[a.W + 1]), 1, hv2, hx2);
                        take3(act3<RELU>(r[2]), 2, hv1, hx1);
                        take3(act3<RELU>(r[a.W + 2]), 2, hv2, hx2);
                        float best = hv0;
                        int bi = hx0;
                        take3(hv1, 3 + hx1, best, bi);
                        take3(hv2, 6 + hx2, best, bi);
                        otile[oo] = best;
                        nb0[oo] = (uint8_t)bi;
                        oo += a.Wo;
                        hv0 = hv2, hx0 = hx2;
                        r += a.W;
                    }
                    continue;
                }
                float hv0, hv1, hv2;
                int hx0, hx1, hx2;
                hscan<RELU>(pb + (2 * oh0 - a.P) * a.W, 2 * oh0 - a.P, iw0, a, hv0, hx0);
                for (int oh = oh0; oh < oh1; ++oh) {
                    const int ih1 = 2 * oh - a.P + 1;
                    hscan<RELU>(pb + ih1 * a.W, ih1, iw0, a, hv1, hx1);
                    hscan<RELU>(pb + (ih1 + 1) * a.W, ih1 + 1, iw0, a, hv2, hx2);
                    float best = ninf;
                    int bi = max(0, a.P - 2 * oh) * 3 + dx0;  // first in-bounds position (all -inf)
                    take3(hv0, hx0, best, bi);
                    take3(hv1, 3 + hx1, best, bi);
                    take3(hv2, 6 + hx2, best, bi);
                    otile[oo + oh * a.Wo] = best;
                    nb0[oo + oh * a.Wo] = (uint8_t)bi;
                    hv0 = hv2, hx0 = hx2;
                }
            }
            // the outputs of plane p0 + np in this tile's last argmax word (<= 7, nibbles only)
            const int ext = (int)(t.ob - (t.p0 + t.np) * a.HoWo);
            if (tid < ext) {
                uint32_t oh, ow;
                a.div_wo.divmod((uint32_t)tid, oh, ow);
                const int ih0 = (int)oh * 2 - a.P, iw0 = (int)ow * 2 - a.P;
                const float *pb = P0 + t.np * a.HW;
                int bi = max(0, -ih0) * 3 + max(0, -iw0);
                float best = ninf;
#pragma unroll
                for (int dy = 0; dy < 3; ++dy)
#pragma unroll
                    for (int dx = 0; dx < 3; ++dx) {
                        const int ih = ih0 + dy, iw = iw0 + dx;
                        const bool ok = ih >= 0 && ih < a.H && iw >= 0 && iw < a.W;
                        take3(ok ? act3<RELU>(pb[ok ? ih * a.W + iw : 0]) : ninf, 3 * dy + dx, best, bi);
                    }
                nb0[t.np * a.HoWo + tid] = (uint8_t)bi;
            }
        } else {
            // stride 1 (G * HoWo % 8 == 0: every word whole in the tile): one thread per (plane,
            // output column, row segment) walks down the segment, one new input row per output.
            // Border taps (padding) are masked with selects on clamped addresses, not branches.
            float *otile = out + olo;
            const int items = t.np * a.segs * a.Wo;
            for (int it = tid; it < items; it += kRT) {
                uint32_t ps, ow, pl, sg;
                a.div_wo.divmod((uint32_t)it, ps, ow);
                a.div_seg.divmod(ps, pl, sg);
                const int oh0 = (int)sg * a.segr, oh1 = min(a.Ho, oh0 + a.segr);
                const float *pb = R + ((t.p0 + pl) * a.HW - sb);
                const int iw0 = (int)ow - a.P;
                const bool okL = iw0 >= 0, okR = iw0 + 2 < a.W;
                const int cM = iw0 + 1, cL = okL ? iw0 : cM, cR = okR ? iw0 + 2 : cM;
                const int dx0 = okL ? 0 : 1;  // first in-bounds column of the window (P <= 1)
                // row scan of input row ih: (max, column) in R3's order; an absent row: (-inf, dx0)
                auto hrow = [&](int ih, float &v, int &x) {
                    const float *rp = pb + min(max(ih, 0), a.H - 1) * a.W;
                    const float l = act3<RELU>(rp[cL]), m = act3<RELU>(rp[cM]), r = act3<RELU>(rp[cR]);
                    v = okL ? l : ninf;
                    x = dx0;
                    take3(m, 1, v, x);
                    take3(okR ? r : ninf, 2, v, x);
                    if ((unsigned)ih >= (unsigned)a.H) v = ninf, x = dx0;
                };
                float hv0, hv1, hv2;
                int hx0, hx1, hx2;
                hrow(oh0 - a.P, hv0, hx0);
                hrow(oh0 - a.P + 1, hv1, hx1);
                int oo = (int)pl * a.HoWo + oh0 * a.Wo + (int)ow;  // tile-local output index
                for (int oh = oh0; oh < oh1; ++oh) {
                    hrow(oh - a.P + 2, hv2, hx2);
                    float best = hv0;  // the window's first row (an absent first row: -inf, bi = 3 + dx0)
                    int bi = hx0 + (oh - a.P >= 0 ? 0 : 3);
                    take3(hv1, 3 + hx1, best, bi);
                    take3(hv2, 6 + hx2, best, bi);
                    otile[oo] = best;
                    nbs[oo] = (uint8_t)bi;
                    oo += a.Wo;
                    hv0 = hv1, hx0 = hx1;
                    hv1 = hv2, hx1 = hx2;
                }
            }
        }
        // the previous tile's words, from the other nibble buffer (complete since the last barrier)
        if (j > 0) pack(prev, nbs0 + ((j - 1) & 1) * kNbFwd);
        prev = t;
        // one barrier per tile: stage st and the previous tile's nibble bytes are consumed, this
        // tile's nibble bytes are complete (packed during the next tile's walk)
        __syncthreads();
        if (tid == 0 && j + a.rs < mine) issue(j + a.rs, st);
        if (++st == a.rs) st = 0, ph ^= 1u;
    }
    if (mine > 0) pack(prev, nbs0 + ((mine - 1) & 1) * kNbFwd);
}

// ---------------------------------------------------------------- backward
struct BwdTile {
    int64_t p0, olo, ohi, ilo, ihi, aw_lo, aw_hi, mw_lo, mw_hi;
    int np;
};

__device__ __forceinline__ BwdTile bwd_tile(const P3Args &a, int64_t k) {
    BwdTile t;
    t.p0 = k * a.G;
    t.np = (int)min((int64_t)a.G, a.NC - t.p0);
    t.olo = t.p0 * a.HoWo;
    t.ohi = t.olo + (int64_t)t.np * a.HoWo;
    t.ilo = t.p0 * a.HW;
    t.ihi = t.ilo + (int64_t)t.np * a.HW;
    t.aw_lo = t.olo >> 3;
    t.aw_hi = (t.ohi + 7) >> 3;
    t.mw_lo = t.ilo >> 5;
    t.mw_hi = (t.ihi + 31) >> 5;
    return t;
}

template <int S, bool MASK>
__global__ void __launch_bounds__(kRT)
pool3_bwd_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg, const uint32_t *__restrict__ mask,
                 P3Args a, float *__restrict__ dx) {
    pdl_enter();
    extern __shared__ __align__(128) unsigned char smp[];
    float *ring = reinterpret_cast<float *>(smp);
    uint8_t *nbb = smp + (size_t)a.rs * a.sf * 4;  // padded nibble-byte planes of the tile
    uint64_t *full = reinterpret_cast<uint64_t *>(nbb + kAuxBytes);
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < a.rs; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t mine = a.tiles > blockIdx.x ? (a.tiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    auto issue = [&](int64_t j) {
        const BwdTile t = bwd_tile(a, blockIdx.x + j * gridDim.x);
        const int st = (int)(j % a.rs);
        float *R = ring + (size_t)st * a.sf;
        const uint32_t bd = ring_bytes(t.olo, t.ohi), ba = ring_bytes(t.aw_lo, t.aw_hi);
        const uint32_t bm = MASK ? ring_bytes(t.mw_lo, t.mw_hi) : 0u;
        mbar_arrive_expect_tx(&full[st], bd + ba + bm);
        if (bd) ring_copy(R, dout + (t.olo & ~3ll), bd, &full[st]);
        if (ba) ring_copy(R + a.a_off, arg + (t.aw_lo & ~3ll), ba, &full[st]);
        if (bm) ring_copy(R + a.m_off, mask + (t.mw_lo & ~3ll), bm, &full[st]);
    };
    if (tid == 0)
        for (int64_t j = 0; j < a.rs && j < mine; ++j) issue(j);
    for (int64_t j = 0; j < mine; ++j) {
        const int st = (int)(j % a.rs);
        float *R = ring + (size_t)st * a.sf;
        const BwdTile t = bwd_tile(a, blockIdx.x + j * gridDim.x);
        mbar_wait(&full[st], (uint32_t)(j / a.rs) & 1u);
        {
            uint32_t *RA = reinterpret_cast<uint32_t *>(R + a.a_off), *RM = reinterpret_cast<uint32_t *>(R + a.m_off);
            bool wrote = tail_fill(R, dout, t.olo, t.ohi, 0);
            wrote |= tail_fill(RA, arg, t.aw_lo, t.aw_hi, 4);
            if (MASK) wrote |= tail_fill(RM, mask, t.mw_lo, t.mw_hi, 8);
            if (wrote) fence_proxy_async_smem();
        }
        __syncthreads();
        const float *D = R + (t.olo - (t.olo & ~3ll));  // dY by tile-local output index
        // argmax / mask words by (tile-local index + phase) >> 3 / >> 5
        const uint32_t *Aw = reinterpret_cast<const uint32_t *>(R + a.a_off) + (t.aw_lo - (t.aw_lo & ~3ll));
        const uint32_t *Mw = reinterpret_cast<const uint32_t *>(R + a.m_off) + (t.mw_lo - (t.mw_lo & ~3ll));
        const int aph = (int)(t.olo & 7), mph = (int)(t.ilo & 31);
        // nibbles -> one byte per window in padded planes (window (oh, ow) at (oh + OFF, ow + OFF),
        // OFF = 2 for stride 1, 1 for stride 2); cells holding no window read 0xF (never a hit)
        constexpr int OFF = S == 1 ? 2 : 1;
        const int PP = a.PR * a.PC;
        {
            uint4 *n4 = reinterpret_cast<uint4 *>(nbb);
            const int c16 = (t.np * PP + 15) >> 4;
            for (int i = tid; i < c16; i += kRT) n4[i] = make_uint4(~0u, ~0u, ~0u, ~0u);
        }
        __syncthreads();
        {
            const int no = t.np * a.HoWo;
            const int nw = (aph + no + 7) >> 3;
            for (int w = tid; w < nw; w += kRT) {
                const uint32_t word = Aw[w];
                const int l0 = 8 * w - aph;  // tile-local output of nibble 0
                uint32_t pl, rem, oh, ow;
                a.div_howo.divmod((uint32_t)(l0 > 0 ? l0 : 0), pl, rem);
                a.div_wo.divmod(rem, oh, ow);
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int l = l0 + k;
                    if (l >= 0 && l < no) {
                        nbb[(int)pl * PP + ((int)oh + OFF) * a.PC + (int)ow + OFF] = (uint8_t)((word >> (4 * k)) & 0xfu);
                        if (++ow == (uint32_t)a.Wo) {
                            ow = 0;
                            if (++oh == (uint32_t)a.Ho) {
                                oh = 0;
                                ++pl;
                            }
                        }
                    }
                }
            }
        }
        __syncthreads();
        auto mbit = [&](int il) { return !MASK || ((Mw[(il + mph) >> 5] >> ((il + mph) & 31)) & 1u); };
        float *dxt = dx + t.ilo;
        if (S == 2) {
            const int nblk = t.np * a.hb * a.wb;
            for (int q = tid; q < nblk; q += kRT) {
                uint32_t pl, rem, A, b;
                a.div_blk.divmod((uint32_t)q, pl, rem);
                a.div_wb.divmod(rem, A, b);
                const int c11 = (int)pl * PP + ((int)A + 1) * a.PC + (int)b + 1;  // window (A, b)
                const unsigned n00 = nbb[c11 - a.PC - 1], n01 = nbb[c11 - a.PC], n10 = nbb[c11 - 1], n11 = nbb[c11];
                const int o11 = (int)pl * a.HoWo + (int)A * a.Wo + (int)b;  // dY of window (A, b)
                float a00 = 0.0f, a01 = 0.0f, a10 = 0.0f, a11 = 0.0f;  // +0.0f, then ascending o
                if (n00 == 8u) a00 = a00 + D[o11 - a.Wo - 1];
                if (n01 == 6u) a00 = a00 + D[o11 - a.Wo];
                if (n01 == 7u) a01 = a01 + D[o11 - a.Wo];
                if (n10 == 2u) a00 = a00 + D[o11 - 1];
                if (n10 == 5u) a10 = a10 + D[o11 - 1];
                if (n11 == 0u) a00 = a00 + D[o11];
                if (n11 == 1u) a01 = a01 + D[o11];
                if (n11 == 3u) a10 = a10 + D[o11];
                if (n11 == 4u) a11 = a11 + D[o11];
                // inputs of the block that exist: ih = 2A + r - P, iw = 2b + c - P
                const int ih0 = 2 * (int)A - a.P, iw0 = 2 * (int)b - a.P;
                const bool r0 = ih0 >= 0, r1 = ih0 + 1 < a.H, c0 = iw0 >= 0, c1 = iw0 + 1 < a.W;
                const int il = (int)pl * a.HW + ih0 * a.W + iw0;
                if (r0 && c0) dxt[il] = mbit(il) ? a00 : 0.0f;
                if (r0 && c1) dxt[il + 1] = mbit(il + 1) ? a01 : 0.0f;
                if (r1 && c0) dxt[il + a.W] = mbit(il + a.W) ? a10 : 0.0f;
                if (r1 && c1) dxt[il + a.W + 1] = mbit(il + a.W + 1) ? a11 : 0.0f;
            }
        } else {
            if (GIST_POOL3_BWD_STRIP) {
            // one thread per input column segment (segr rows) of a plane walks down its rows; a tile with
            // few columns (GoogLeNet's 28x28 planes) is cut into row segments so every thread has work.  Input (ih, iw) is position
            // (dy, dx) = (th - oh, tw - ow) of the windows oh in [th-2, th], ow in [tw-2, tw] (th = ih + P):
            // padded nibble rows th, th+1, th+2 (dy = 2, 1, 0) x columns tw, tw+1, tw+2 (dx = 2, 1, 0),
            // visited in that order = ascending output order (R6).  Moving down one row shifts the
            // rows by one, so each window row's three nibbles are loaded once per column, not three times.
            const int cols = t.np * a.W;
            const int nseg = (!GIST_POOL3_BWD_SEG || cols >= kRT / 2) ? 1 : (kRT + cols - 1) / cols;  // row segments
            const int segr = (a.H + nseg - 1) / nseg;
            for (int it = tid; it < cols * nseg; it += kRT) {
                const int sg = it / cols;
                uint32_t pl, iw;
                a.div_w.divmod((uint32_t)(it - sg * cols), pl, iw);
                const int tw = (int)iw + a.P;
                const int ih_beg = sg * segr, ih_end = min(a.H, ih_beg + segr);
                const unsigned char *nb = nbb + (int)pl * PP + tw;  // padded column tw of row 0
                const float *Dp = D + (int)pl * a.HoWo + tw;          // dY of window (0, tw)
                unsigned n0[3], n1[3], n2[3];
#pragma unroll
                for (int c = 0; c < 3; ++c) {
                    n0[c] = nb[(ih_beg + a.P) * a.PC + c];
                    n1[c] = nb[(ih_beg + a.P + 1) * a.PC + c];
                }
                const int il0 = (int)pl * a.HW + (int)iw;
                for (int ih = ih_beg; ih < ih_end; ++ih) {
                    const int th = ih + a.P;
#pragma unroll
                    for (int c = 0; c < 3; ++c) n2[c] = nb[(th + 2) * a.PC + c];
                    const int il = il0 + ih * a.W;
                    const bool on = mbit(il);
                    float acc = 0.0f;  // R6: +0.0f, then ascending output order
                    if (on) {
                        const float *d0 = Dp + (th - 2) * a.Wo;  // window row th-2: dY at column tw - 2 + c
#pragma unroll
                        for (int c = 0; c < 3; ++c)
                            if (n0[c] == 8u - c) acc = acc + d0[c - 2];
#pragma unroll
                        for (int c = 0; c < 3; ++c)
                            if (n1[c] == 5u - c) acc = acc + d0[a.Wo + c - 2];
#pragma unroll
                        for (int c = 0; c < 3; ++c)
                            if (n2[c] == 2u - c) acc = acc + d0[2 * a.Wo + c - 2];
                    }
                    dxt[il] = on ? acc : 0.0f;
#pragma unroll
                    for (int c = 0; c < 3; ++c) {
                        n0[c] = n1[c];
                        n1[c] = n2[c];
                    }
                }
            }
            } else {
            // one thread per input element; windows (oh, ow) = (th - dy, tw - dx), th = ih + P, in
            // ascending output order; the hit nibble is 3 dy + dx
            const int cnt = t.np * a.HW;
            for (int l = tid; l < cnt; l += kRT) {
                const bool on = mbit(l);
                float acc = 0.0f;  // R6: +0.0f, then ascending output order
                if (on) {
                    uint32_t pl, rem, ih, iw;
                    a.div_hw.divmod((uint32_t)l, pl, rem);
                    a.div_w.divmod(rem, ih, iw);
                    const int th = (int)ih + a.P, tw = (int)iw + a.P;
                    const int cell = (int)pl * PP + (th + 2) * a.PC + tw + 2;  // window (th, tw)
                    const int ol = (int)pl * a.HoWo + th * a.Wo + tw;          // its dY (when it exists)
#pragma unroll
                    for (int dy = 2; dy >= 0; --dy)
#pragma unroll
                        for (int dxx = 2; dxx >= 0; --dxx)
                            if (nbb[cell - dy * a.PC - dxx] == (unsigned)(3 * dy + dxx)) acc = acc + D[ol - dy * a.Wo - dxx];
                }
                dxt[l] = on ? acc : 0.0f;
            }
            }
        }
        __syncthreads();  // stage st consumed
        if (tid == 0 && j + a.rs < mine) issue(j + a.rs);
    }
}

// Backward through hit masks.  Pass 1 (one thread per argmax word): every window ORs one bit into
// the hit mask of the input its argmax selects -- bit 3 (2 - dy) + (2 - dx) for stride 1 (9 bits,
// 16 per input), bit 2 r + c for stride 2 (4 bits per input; r = 0 for the upper of two covering
// window rows, c likewise) -- so that a mask's bits in ascending order are its windows in ascending
// output order.  Pass 2 (one thread per input element): +0.0f, then dY of each set bit in that
// order (R6), selected by the a1 mask bit (R7).  OR is order-free, so the result does not depend
// on the atomics' order; the work is one atomic per window and one step per hit instead of 9 (4)
// nibble tests per input.
template <int S, bool MASK, bool SAME>
__global__ void __launch_bounds__(kRT)
pool3_bwd_hits_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                      const uint32_t *__restrict__ mask, P3Args a, float *__restrict__ dx) {
    pdl_enter();
    extern __shared__ __align__(128) unsigned char smp[];
    float *ring = reinterpret_cast<float *>(smp);
    uint32_t *hits = reinterpret_cast<uint32_t *>(smp + (size_t)a.rs * a.sf * 4);
    uint64_t *full = reinterpret_cast<uint64_t *>(smp + (size_t)a.rs * a.sf * 4 + kAuxBytes);
    constexpr int kHB = S == 1 ? 16 : 4;  // hit bits per input
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < a.rs; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t mine = a.tiles > blockIdx.x ? (a.tiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    auto issue = [&](int64_t j, int st) {
        const BwdTile t = bwd_tile(a, blockIdx.x + j * gridDim.x);
        float *R = ring + (size_t)st * a.sf;
        const uint32_t bd = ring_bytes(t.olo, t.ohi), ba = ring_bytes(t.aw_lo, t.aw_hi);
        const uint32_t bm = MASK ? ring_bytes(t.mw_lo, t.mw_hi) : 0u;
        mbar_arrive_expect_tx(&full[st], bd + ba + bm);
        if (bd) ring_copy(R, dout + (t.olo & ~3ll), bd, &full[st]);
        if (ba) ring_copy(R + a.a_off, arg + (t.aw_lo & ~3ll), ba, &full[st]);
        if (bm) ring_copy(R + a.m_off, mask + (t.mw_lo & ~3ll), bm, &full[st]);
    };
    if (tid == 0)
        for (int64_t j = 0; j < a.rs && j < mine; ++j) issue(j, (int)j);
    int st = 0;
    uint32_t ph = 0;
    for (int64_t j = 0; j < mine; ++j) {
        float *R = ring + (size_t)st * a.sf;
        const BwdTile t = bwd_tile(a, blockIdx.x + j * gridDim.x);
        const int cnt = t.np * a.HW;
        {  // clear the tile's hit masks (the previous tile's gather has finished: end-of-tile barrier)
            uint4 *h4 = reinterpret_cast<uint4 *>(hits);
            const int n16 = (cnt * kHB / 8 + 15) >> 4;
            for (int i = tid; i < n16; i += kRT) h4[i] = make_uint4(0u, 0u, 0u, 0u);
        }
        mbar_wait(&full[st], ph);
        {
            uint32_t *RA = reinterpret_cast<uint32_t *>(R + a.a_off), *RM = reinterpret_cast<uint32_t *>(R + a.m_off);
            bool wrote = tail_fill(R, dout, t.olo, t.ohi, 0);
            wrote |= tail_fill(RA, arg, t.aw_lo, t.aw_hi, 4);
            if (MASK) wrote |= tail_fill(RM, mask, t.mw_lo, t.mw_hi, 8);
            if (wrote) fence_proxy_async_smem();
        }
        __syncthreads();
        const float *D = R + (t.olo - (t.olo & ~3ll));  // dY by tile-local output index
        const uint32_t *Aw = reinterpret_cast<const uint32_t *>(R + a.a_off) + (t.aw_lo - (t.aw_lo & ~3ll));
        const uint32_t *Mw = reinterpret_cast<const uint32_t *>(R + a.m_off) + (t.mw_lo - (t.mw_lo & ~3ll));
        const int aph = (int)(t.olo & 7), mph = (int)(t.ilo & 31);
        {  // pass 1: scatter one hit bit per window
            const int no = t.np * a.HoWo;
            const int nw = (aph + no + 7) >> 3;
            for (int w = tid; w < nw; w += kRT) {
                const uint32_t word = Aw[w];
                const int l0 = 8 * w - aph;  // tile-local output of nibble 0
                if (SAME) {  // 3x3/s1/p1 with Ho = H, Wo = W: window l is centred on input l
#pragma unroll
                    for (int k = 0; k < 8; ++k) {
                        const int l = l0 + k;
                        const int jn = (int)((word >> (4 * k)) & 0xfu);
                        const int dy = (jn * 11) >> 5, dxx = jn - 3 * dy;
                        const int tt = l + (dy - 1) * a.W + dxx - 1;
                        if (l >= 0 && l < no && jn <= 8 && (unsigned)tt < (unsigned)cnt)
                            atomicOr(&hits[tt >> 1], (1u << (8 - jn)) << (16 * (tt & 1)));
                    }
                    continue;
                }
                uint32_t pl, rem, oh, ow;
                a.div_howo.divmod((uint32_t)(l0 > 0 ? l0 : 0), pl, rem);
                a.div_wo.divmod(rem, oh, ow);
                int base = (int)pl * a.HW + ((int)oh * S - a.P) * a.W + (int)ow * S - a.P;  // window's (0, 0) tap
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int l = l0 + k;
                    if (l >= 0 && l < no) {
                        const int jn = (int)((word >> (4 * k)) & 0xfu);
                        const int dy = (jn * 11) >> 5, dxx = jn - 3 * dy;  // jn / 3, jn % 3 (jn <= 8)
                        const int tt = base + dy * a.W + dxx;               // the selected input
                        if (jn <= 8 && (unsigned)tt < (unsigned)cnt) {      // (a malformed map cannot write outside)
                            if (S == 1) {
                                atomicOr(&hits[tt >> 1], (1u << (8 - jn)) << (16 * (tt & 1)));
                            } else {
                                const int bit = (dy == 2 ? 0 : 2) + (dxx == 2 ? 0 : 1);
                                atomicOr(&hits[tt >> 3], 1u << (4 * (tt & 7) + bit));
                            }
                        }
                        base += S;
                        if (++ow == (uint32_t)a.Wo) {
                            ow = 0;
                            base += S * a.W - a.Wo * S;
                            if (++oh == (uint32_t)a.Ho) {
                                oh = 0;
                                base += a.HW - a.Ho * S * a.W;
                            }
                        }
                    }
                }
            }
        }
        __syncthreads();
        {  // pass 2: gather per input element
            float *dxt = dx + t.ilo;
            for (int l = tid; l < cnt; l += kRT) {
                uint32_t h = (hits[l * kHB / 32] >> ((l * kHB) & 31)) & ((1u << kHB) - 1u);
                const bool on = !MASK || ((Mw[(l + mph) >> 5] >> ((l + mph) & 31)) & 1u);
                float acc = 0.0f;  // R6: +0.0f, then ascending output order
                if (SAME && on && h) {  // window l - W - 1 is (th - 2, tw - 2)
                    const float *Dp = D + l - a.W - 1;
#pragma unroll
                    for (int k = 0; k < 9; ++k)
                        if (h & (1u << k)) acc = acc + Dp[(k / 3) * a.W + k % 3];
                } else if (on && h) {
                    uint32_t pl, rem, ih, iw;
                    a.div_hw.divmod((uint32_t)l, pl, rem);
                    a.div_w.divmod(rem, ih, iw);
                    const int th = (int)ih + a.P, tw = (int)iw + a.P;
                    // a fixed, predicated walk over the bits (a loop over set bits diverges: the
                    // warp would run as many steps as its most-hit lane)
                    if (S == 1) {
                        const float *Dp = D + (int)pl * a.HoWo + (th - 2) * a.Wo + (tw - 2);  // window (th-2, tw-2)
#pragma unroll
                        for (int k = 0; k < 9; ++k)
                            if (h & (1u << k)) acc = acc + Dp[(k / 3) * a.Wo + k % 3];
                    } else {
                        const float *Dp = D + (int)pl * a.HoWo + ((th >> 1) - 1) * a.Wo + ((tw >> 1) - 1);
                        if (h & 1u) acc = acc + Dp[0];
                        if (h & 2u) acc = acc + Dp[1];
                        if (h & 4u) acc = acc + Dp[a.Wo];
                        if (h & 8u) acc = acc + Dp[a.Wo + 1];
                    }
                }
                dxt[l] = acc;
            }
        }
        __syncthreads();  // stage st and the hit masks consumed
        if (tid == 0 && j + a.rs < mine) issue(j + a.rs, st);
        if (++st == a.rs) st = 0, ph ^= 1u;
    }
}

int gcd_i(int a, int b) {
    while (b) {
        const int t = a % b;
        a = b;
        b = t;
    }
    return a;
}

P3Args p3_args(int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo) {
    P3Args a{};
    a.H = H;
    a.W = W;
    a.Ho = Ho;
    a.Wo = Wo;
    a.S = p.sh;
    a.P = p.ph;
    a.HW = H * W;
    a.HoWo = Ho * Wo;
    a.NC = (int64_t)N * C;
    a.n_in = a.NC * a.HW;
    a.n_out = a.NC * a.HoWo;
    a.div_hw = FastDiv::make((uint32_t)a.HW);
    a.div_w = FastDiv::make((uint32_t)W);
    a.div_howo = FastDiv::make((uint32_t)a.HoWo);
    a.div_wo = FastDiv::make((uint32_t)Wo);
    return a;
}

// Planes per tile: as many as a stage holds (`per_plane` floats each, `fixed` floats of slack),
// a multiple of `unit`, but no more than keeps ~4 tiles per CTA.  0: one unit does not fit.
int32_t choose_g(int64_t NC, int64_t per_plane, int64_t fixed, int32_t unit, int64_t ctas, int64_t stage_floats) {
    const int64_t fit = (stage_floats - fixed) / per_plane;
    if (fit < unit) return 0;
    int64_t g = std::min<int64_t>(fit, std::max<int64_t>(1, NC / (4 * ctas)));
    g = std::max<int64_t>(unit, g / unit * unit);
    return (int32_t)g;
}

// Forward tile plan: planes per tile G (a multiple of `unit`, at most gmax) and output rows per
// walker segment, chosen to minimise the busiest CTA's walk time: tiles per CTA x (rounds of kRT
// items x (segment rows + the item's setup and first rows, `warm`) + a per-tile overhead), in row
// steps.  (The earlier
// rule -- G for ~4 tiles per CTA, then about one item per thread -- left e.g. 336 of 512 threads
// busy on GoogLeNet's 14x14 planes.)
#ifndef GIST_POOL3_PLAN
#define GIST_POOL3_PLAN 1
#endif
struct FwdPlan {
    int32_t G, segr, segs;
};
FwdPlan plan_fwd(int64_t NC, int32_t Ho, int32_t Wo, int32_t unit, int32_t gmax, int64_t ctas, double warm) {
    FwdPlan best{0, 0, 0};
    double best_cost = 1e300;
    for (int32_t g = unit; g <= gmax; g += unit) {
        const int64_t per_cta = ((NC + g - 1) / g + ctas - 1) / ctas;
        for (int32_t segr = 1; segr <= Ho; ++segr) {
            const int32_t segs = (Ho + segr - 1) / segr;
            if (segr > 1 && (Ho + segr - 2) / (segr - 1) == segs) continue;  // same segments, longer rows
            const int64_t rounds = ((int64_t)g * Wo * segs + kRT - 1) / kRT;
            const double cost = (double)per_cta * ((double)rounds * (segr + warm) + 4.0);
            // ties go to the larger G (fewer tiles: GoogLeNet inc4b 14x14, G = 28 vs 36 at equal cost
            // measured 27.4 vs 20.0 us)
            if (cost < best_cost - 1e-9 || (cost < best_cost + 1e-9 && g > best.G))
                best_cost = cost, best = FwdPlan{g, segr, segs};
        }
    }
    return best;
}

// Backward (hit masks) tile plan: planes per tile chosen to minimise the busiest CTA's time, tiles
// per CTA x (rounds of kRT argmax words x 3 + rounds of kRT inputs + a per-tile overhead of 4).
// The caller keeps the earlier G when it is larger (GoogLeNet inc3a: the model's pick, 7 planes
// instead of 8, measured 6% slower).
int32_t plan_bwd_hits(int64_t NC, int64_t HoWo, int64_t HW, int32_t gmax, int64_t ctas) {
    int32_t best = 0;
    double best_cost = 1e300;
    for (int32_t g = 1; g <= gmax; ++g) {
        const int64_t per_cta = ((NC + g - 1) / g + ctas - 1) / ctas;
        const int64_t r1 = ((g * HoWo + 7) / 8 + kRT - 1) / kRT, r2 = (g * HW + kRT - 1) / kRT;
        const double cost = (double)per_cta * (3.0 * r1 + r2 + 4.0);
        if (cost < best_cost + 1e-9) best_cost = std::min(best_cost, cost), best = g;  // ties: the larger G
    }
    return best;
}

// Ring per kernel kind (stages x KB per stage), measured on B200 (AlexNet / NiN / GoogLeNet maps):
// stride-2 forward 2 x 48 KB (was 3 x 32: AlexNet relu1 62 -> 52 us, fewer per-tile overheads),
// the others 3 x 32 KB.  GIST_POOL3_RING="f1=3x32,f2=2x48,b1=3x32,b2=3x32" overrides (tuning).
struct Ring {
    int rs, kb;
};
Ring ring_for(bool fwd, int S) {
    static Ring cfg[2][2] = {{{3, 32}, {3, 32}}, {{3, 32}, {2, 48}}};  // [fwd][S - 1]
    static const bool parsed = [] {
        if (const char *e = getenv("GIST_POOL3_RING")) {
            for (const char *q = e; *q;) {
                char kind = 0;
                int sd = 0, rs = 0, kb = 0, used = 0;
                if (sscanf(q, "%c%d=%dx%d%n", &kind, &sd, &rs, &kb, &used) == 4 && (sd == 1 || sd == 2) &&
                    rs >= 2 && rs <= kMaxRS && kb >= 8 && kb <= 96)
                    cfg[kind == 'f'][sd - 1] = Ring{rs, kb};
                q += used ? used : 1;
                while (*q == ',') ++q;
            }
        }
        return true;
    }();
    (void)parsed;
    return cfg[fwd ? 1 : 0][S - 1];
}
size_t ring_smem(const Ring &r) {
    return (size_t)r.rs * r.kb * 1024 + kAuxBytes + 8 * kMaxRS + kMaxRS * sizeof(FwdTile);
}
int64_t resident_ctas(size_t smem) {
    return std::max<int64_t>(1, std::min<int64_t>(2, (int64_t)(227 * 1024) / (int64_t)(smem + 1024))) * num_sms();
}

}  // namespace

// Used for stride 1 (GoogLeNet's in-module pools): forward 16% -> 28% of HBM, backward 12% -> 21%
// (inc3a b64, isolated), and for the stride-2 forward (column walker, 2 x 48 KB ring): AlexNet relu1
// b128 56 -> 52 us, with the a1 mask 72 (L1 kernel + binarize) -> 68 us; NiN relu_cccp2 b256
// 144 -> 125 us.  The stride-2 backward stays on pool.cu's 2x2-block kernel (82 vs 100 us on
// AlexNet relu1) unless GIST_POOL3_S2_BWD=1.
#ifndef GIST_POOL3_S2
#define GIST_POOL3_S2 1
#endif
#ifndef GIST_POOL3_BAND
#define GIST_POOL3_BAND 1  // stride-2 forward of planes larger than a stage in bands of output rows
#endif
#ifndef GIST_POOL3_S2_BWD
#define GIST_POOL3_S2_BWD 0
#endif
bool pool3_ok(const gist_pool2d &p, bool fwd) {
    const bool s2 = fwd ? GIST_POOL3_S2 : GIST_POOL3_S2_BWD;
    return p.kh == 3 && p.kw == 3 && p.sh == p.sw && (p.sh == 1 || (s2 && p.sh == 2)) && p.ph == p.pw &&
           p.ph <= 1;
}

// Forward (+ the a1 mask when mask != NULL, + relu on load when relu).  Returns cudaErrorNotSupported
// when a plane does not fit a stage (the caller uses the generic kernels).
cudaError_t launch_pool3_fwd(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                             int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, uint32_t *mask, bool relu,
                             cudaStream_t s) {
    P3Args a = p3_args(N, C, H, W, p, Ho, Wo);
    const Ring ring = ring_for(true, a.S);
    a.rs = ring.rs;
    a.sf = ring.kb * 256;
    const size_t smem = ring_smem(ring);
    const int64_t ctas = resident_ctas(smem);
    if (a.S == 1) {
        // whole argmax (and mask) words per tile; the nibble bytes of a tile fit kNbBytes
        int32_t unit = 8 / gcd_i(a.HoWo, 8);
        if (mask) {
            const int32_t mu = 32 / gcd_i(a.HW, 32);
            unit = unit * mu / gcd_i(unit, mu);
        }
        a.G = choose_g(a.NC, a.HW, 64, unit, ctas, a.sf);
        while (a.G > unit && (int64_t)a.G * a.HoWo > kNbFwd) a.G -= unit;
        if (a.G == 0 || (int64_t)a.G * a.HoWo > kNbFwd) return cudaErrorNotSupported;
        const int64_t cols = (int64_t)a.G * Wo;  // row segments: about one item per thread
        const int32_t want = (int32_t)std::max<int64_t>(1, std::min<int64_t>(Ho, kRT / cols));
        a.segr = (Ho + want - 1) / want;
        a.segs = (Ho + a.segr - 1) / a.segr;
        if (GIST_POOL3_PLAN) {
            int32_t gmax = (int32_t)std::min<int64_t>((a.sf - 64) / a.HW, kNbFwd / a.HoWo);
            gmax = gmax / unit * unit;
            const char *fg = getenv("GIST_POOL3_FWD_G");  // tuning only: a fixed G (its segments planned)
            const int32_t gf = fg ? atoi(fg) / unit * unit : 0;
            const FwdPlan pl = gf > 0 && gf <= gmax ? plan_fwd(a.NC, Ho, Wo, gf, gf, ctas, 1.6) : plan_fwd(a.NC, Ho, Wo, unit, gmax, ctas, 1.6);
            if (pl.G > 0) a.G = pl.G, a.segr = pl.segr, a.segs = pl.segs;
        }
        a.div_seg = FastDiv::make((uint32_t)a.segs);
    } else {
        // rows of the next plane a tile may need: the windows of its last argmax word's (<= 7)
        // outputs there, and the (<= 31) elements of its last mask word
        int32_t xr = 0;
        if (a.HoWo % 8) xr = std::min(H, (std::min(6, a.HoWo - 1) / Wo) * a.S - a.P + 3);
        if (mask && a.HW % 32) xr = std::max(xr, std::min(H, (30 + W) / W));
        a.xrows = xr;
        a.G = choose_g(a.NC, a.HW, 64 + (int64_t)xr * W + 32, 1, ctas, a.sf);
        while (a.G > 1 && (int64_t)a.G * a.HoWo + 14 > kNbFwd) --a.G;
        const bool fits = a.G > 0 && (int64_t)a.G * a.HoWo + 14 <= kNbFwd;
        // a plane larger than a stage (GoogLeNet's 112x112 stem): bands of output rows, when every
        // band owns whole argmax and mask words (P = 0, Wo % 8 == 0, W % 16 == 0, HW % 32 == 0)
        const char *fb = getenv("GIST_POOL3_BANDS");  // testing: force this many bands per plane
        const int32_t force = fb ? atoi(fb) : 0;
        if ((!fits || force > 1) && GIST_POOL3_BAND && a.P == 0 && Wo % 8 == 0 && W % 16 == 0 && a.HW % 32 == 0) {
            const int32_t br_max = (int32_t)std::min<int64_t>((((int64_t)a.sf - 64) / W - 1) / 2, kNbFwd / Wo);
            if (br_max < 1) return cudaErrorNotSupported;
            a.bands = force > 1 ? std::min(force, Ho) : (Ho + br_max - 1) / br_max;
            a.br = (Ho + a.bands - 1) / a.bands;
            a.bands = (Ho + a.br - 1) / a.br;
            if (a.br > br_max) return cudaErrorNotSupported;
            a.G = 1;
            a.xrows = 0;
            const int32_t want = (int32_t)std::max<int64_t>(1, std::min<int64_t>(a.br, kRT / Wo));
            a.segr = (a.br + want - 1) / want;
            a.segs = (a.br + a.segr - 1) / a.segr;
            a.div_seg = FastDiv::make((uint32_t)a.segs);
            a.tiles = a.NC * a.bands;
            goto launch;
        }
        if (!fits) return cudaErrorNotSupported;
        // row segments: about one (plane, column, segment) item per thread
        const int64_t cols = (int64_t)a.G * Wo;
        const int32_t want = (int32_t)std::max<int64_t>(1, std::min<int64_t>(Ho, kRT / cols));
        a.segr = (Ho + want - 1) / want;
        a.segs = (Ho + a.segr - 1) / a.segr;
        if (GIST_POOL3_PLAN) {
            int32_t gmax = (int32_t)std::min<int64_t>((a.sf - 64 - (int64_t)xr * W - 32) / a.HW, (kNbFwd - 14) / a.HoWo);
            const FwdPlan pl = plan_fwd(a.NC, Ho, Wo, 1, gmax, ctas, 1.0);
            if (pl.G > 0) a.G = pl.G, a.segr = pl.segr, a.segs = pl.segs;
        }
        a.div_seg = FastDiv::make((uint32_t)a.segs);
    }
    a.tiles = ceil_div(a.NC, a.G);
launch:
    // every window inside the input: no bounds tests (AlexNet's floor-mode 3x3/s2)
    const bool check = !(a.P == 0 && (Ho - 1) * a.S + 3 <= H && (Wo - 1) * a.S + 3 <= W);
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(a.tiles, ctas));
#define P3F(S_, M_, R_, C_)                                                                                 \
    do {                                                                                                    \
        static PerDeviceAttr attr;                                                                          \
        const cudaError_t e =                                                                               \
            attr.ensure(reinterpret_cast<const void *>(pool3_fwd_kernel<S_, M_, R_, C_>), (int)smem);       \
        if (e != cudaSuccess) return e;                                                                     \
        launch_k(pool3_fwd_kernel<S_, M_, R_, C_>, grid, kRT, smem, s, y, a, out, argmax, mask);            \
    } while (0)
    const bool m = mask != nullptr;
    if (a.S == 1) {
        if (m) {
            if (relu) P3F(1, true, true, true); else P3F(1, true, false, true);
        } else {
            if (relu) P3F(1, false, true, true); else P3F(1, false, false, true);
        }
    } else if (check) {
        if (m) {
            if (relu) P3F(2, true, true, true); else P3F(2, true, false, true);
        } else {
            if (relu) P3F(2, false, true, true); else P3F(2, false, false, true);
        }
    } else {
        if (m) {
            if (relu) P3F(2, true, true, false); else P3F(2, true, false, false);
        } else {
            if (relu) P3F(2, false, true, false); else P3F(2, false, false, false);
        }
    }
#undef P3F
    return cudaPeekAtLastError();
}

cudaError_t launch_pool3_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                             int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo, float *dx,
                             cudaStream_t s) {
    P3Args a = p3_args(N, C, H, W, p, Ho, Wo);
    const Ring ring = ring_for(false, a.S);
    a.rs = ring.rs;
    a.sf = ring.kb * 256;
    const size_t smem = ring_smem(ring);
    const int64_t ctas = resident_ctas(smem);
    const bool hitk = GIST_POOL3_BWD_HITS != 0;
    if (a.S == 2) {
        a.hb = (H + a.P + 1) / 2;
        a.wb = (W + a.P + 1) / 2;
        a.div_blk = FastDiv::make((uint32_t)(a.hb * a.wb));
        a.div_wb = FastDiv::make((uint32_t)a.wb);
        a.PR = std::max(Ho, a.hb) + 1;
        a.PC = std::max(Wo, a.wb) + 1;
    } else {
        a.PR = Ho + 4;
        a.PC = Wo + 4;
    }
    // stage floats per plane: dY (HoWo) + argmax words (HoWo/8) + mask words (HW/32), and the
    // phases / round-ups of the three ranges
    const int64_t per_plane = (int64_t)a.HoWo + (a.HoWo + 7) / 8 + (mask ? (a.HW + 31) / 32 : 0) + 1;
    a.G = choose_g(a.NC, per_plane, 64, 1, ctas, a.sf);
    // the tile's hit masks (hits kernel) or padded nibble planes must fit the area after the ring
    const int64_t aux_plane = hitk ? (int64_t)a.HW * (a.S == 1 ? 2 : 1) / 1 : (int64_t)a.PR * a.PC;
    const int64_t aux_cap = hitk ? (a.S == 1 ? kHitBytes : 2 * (int64_t)kHitBytes) : kNbBytes;  // S = 2: half bytes
    while (a.G > 1 && (int64_t)a.G * aux_plane + 32 > aux_cap) --a.G;
    if (a.G == 0 || (int64_t)a.G * aux_plane + 32 > aux_cap) return cudaErrorNotSupported;
    if (hitk && GIST_POOL3_PLAN) {
        const int64_t gfit = std::min<int64_t>((a.sf - 64) / per_plane, (aux_cap - 32) / aux_plane);
        const int32_t g = plan_bwd_hits(a.NC, a.HoWo, a.HW, (int32_t)gfit, ctas);
        if (g > a.G) a.G = g;
    }
    a.tiles = ceil_div(a.NC, a.G);
    const int64_t G = a.G;
    a.a_off = (int32_t)((G * a.HoWo + 8 + 3) & ~3ll);
    a.m_off = (int32_t)((a.a_off + (G * a.HoWo + 7) / 8 + 8 + 3) & ~3ll);
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(a.tiles, ctas));
    if (hitk) {
#define P3H(S_, M_, SM_)                                                                                     \
    do {                                                                                                     \
        static PerDeviceAttr attr;                                                                           \
        const cudaError_t e =                                                                                \
            attr.ensure(reinterpret_cast<const void *>(pool3_bwd_hits_kernel<S_, M_, SM_>), (int)smem);     \
        if (e != cudaSuccess) return e;                                                                      \
        launch_k(pool3_bwd_hits_kernel<S_, M_, SM_>, grid, kRT, smem, s, dout, argmax, mask, a, dx);         \
    } while (0)
        const bool same = a.S == 1 && a.P == 1 && Ho == H && Wo == W;
        if (a.S == 1) {
            if (same) {
                if (mask) P3H(1, true, true); else P3H(1, false, true);
            } else {
                if (mask) P3H(1, true, false); else P3H(1, false, false);
            }
        } else {
            if (mask) P3H(2, true, false); else P3H(2, false, false);
        }
#undef P3H
        return cudaPeekAtLastError();
    }
#define P3B(S_, M_)                                                                                          \
    do {                                                                                                     \
        static PerDeviceAttr attr;                                                                           \
        const cudaError_t e = attr.ensure(reinterpret_cast<const void *>(pool3_bwd_kernel<S_, M_>), (int)smem); \
        if (e != cudaSuccess) return e;                                                                      \
        launch_k(pool3_bwd_kernel<S_, M_>, grid, kRT, smem, s, dout, argmax, mask, a, dx);                   \
    } while (0)
    if (a.S == 1) {
        if (mask) P3B(1, true); else P3B(1, false);
    } else {
        if (mask) P3B(2, true); else P3B(2, false);
    }
#undef P3B
    return cudaPeekAtLastError();
}

}  // namespace gist
