// pool.cu — a2: MaxPool forward + 4-bit Y->X argmax map, a3: fused pool+ReLU backward from
// the encodings (§III-A, P:151-P:156 §IV-A).
//
// Forward: one thread per pool output; a warp covers 32 consecutive outputs (4 argmax
// words), ORs the nibbles of each 8-lane group with three xor-shuffles and lane 8g stores
// word g.  Windows are read through L1 (__ldg): neighbouring outputs share input rows.
// The 2x2/s2 unpadded case (VGG16, OverFeat) reads each window row as one aligned float2.
//
// Backward: gather form — one thread per input element (2 adjacent elements for 2x2/s2)
// walks the covering windows in ascending output order, adds dY of every window whose
// argmax is this element (accumulator starts at +0.0f: reading R6), and selects with the
// ReLU mask bit (R7).  Every dx element is written exactly once with no atomics, so the
// result is deterministic and equal to the oracle's ascending-o scatter.
#include <math_constants.h>

#include <algorithm>
#include <type_traits>

#include "common.cuh"
#include "kernels.h"

namespace gist {

namespace {

constexpr int kPoolThreads = 256;
#ifndef GIST_POOL_FWD_CTAS
#define GIST_POOL_FWD_CTAS 6  // grid cap, CTAs per SM (8, 7, 5, 4 measured slower on VGG16 maps)
#endif
#ifndef GIST_POOL_GEN_CTAS
#define GIST_POOL_GEN_CTAS 32  // generic-geometry kernels: grid cap in CTAs per SM (8 resident); 32-64 measured
                               // 8-14% faster than 8 on the 3x3/s2 maps (AlexNet, NiN), 4 and 1000 slower
#endif
#ifndef GIST_POOL3
#define GIST_POOL3 1  // 3x3 windows through the plane-tiled kernels of pool3.cu (0: the L1 kernels below)
#endif
#ifndef GIST_POOL_BWD_CTAS
#define GIST_POOL_BWD_CTAS 6
#endif

struct PoolArgs {
    int32_t H, W, Ho, Wo;
    int32_t kh, kw, sh, sw, ph, pw;
    int32_t n_out;  // N*C*Ho*Wo
    int32_t n_in;   // N*C*H*W
    FastDiv div_wo, div_ho, div_w, div_h;
};

__device__ __forceinline__ void take(float v, int idx, float &best, int &bi) {
    if (v > best || v != v) {  // R3: strict '>' keeps the first maximum; NaN always wins
        best = v;
        bi = idx;
    }
}

// f3 in-place ReLU: the pre-activation map x is read and relu(v) = (v < 0 ? +0.0 : v)
// (R21: torch's ReLU — -0.0 and NaN pass through) is applied on load, so the ReLU output never
// exists in HBM.  relu(v) > 0 iff v > 0, so the a1 mask is the same either way.
template <bool RELU>
__device__ __forceinline__ float act(float v) {
    return RELU ? (v < 0.0f ? 0.0f : v) : v;
}

// KH/KW > 0: compile-time window; 0: runtime (a.kh, a.kw).  RELU: relu(y) on load (f3).
template <int KH, int KW, bool RELU = false>
__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_kernel(const float *__restrict__ y, PoolArgs a, float *__restrict__ out, uint32_t *__restrict__ arg) {
    pdl_enter();
    const int kh = KH ? KH : a.kh, kw = KW ? KW : a.kw;
    const int lane = threadIdx.x & 31;
    // 32-bit output indices (the API rejects maps of 2^31 elements or more)
    const uint32_t chunks = ((uint32_t)a.n_out + 31) / 32;
    const uint32_t nwarps = (gridDim.x * kPoolThreads) >> 5;
    for (uint32_t c = (blockIdx.x * kPoolThreads + threadIdx.x) >> 5; c < chunks; c += nwarps) {
        const uint32_t o = c * 32 + lane;
        uint32_t nib = 0;
        if (o < (uint32_t)a.n_out) {
            uint32_t q, ow, nc, oh;
            a.div_wo.divmod(o, q, ow);
            a.div_ho.divmod(q, nc, oh);
            const int h0 = (int)oh * a.sh - a.ph, w0 = (int)ow * a.sw - a.pw;
            const float *plane = y + nc * (uint32_t)(a.H * a.W);
            float best = -CUDART_INF_F;
            int bi = -1;
            if (KH && KW) {
                // branch-free: out-of-bounds taps read as -inf (never selected under the strict '>'
                // rule, R3) and the argmax starts at the first in-bounds position, so border and
                // interior windows run the same instructions (no warp divergence).
                // When every active lane's window is interior (warp-uniform vote) the bounds
                // tests are skipped altogether.
                float v[KH ? KH : 1][KW ? KW : 1];
                const bool interior = h0 >= 0 && w0 >= 0 && h0 + kh <= a.H && w0 + kw <= a.W;
                if (__all_sync(__activemask(), interior)) {
#pragma unroll
                    for (int dy = 0; dy < (KH ? KH : 1); ++dy)
#pragma unroll
                        for (int dx = 0; dx < (KW ? KW : 1); ++dx) v[dy][dx] = act<RELU>(ld_ro(plane + (h0 + dy) * a.W + w0 + dx));
                    bi = 0;
                } else {
#pragma unroll
                    for (int dy = 0; dy < (KH ? KH : 1); ++dy)
#pragma unroll
                        for (int dx = 0; dx < (KW ? KW : 1); ++dx) {
                            const int ih = h0 + dy, iw = w0 + dx;
                            const bool in = ih >= 0 && ih < a.H && iw >= 0 && iw < a.W;
                            v[dy][dx] = in ? act<RELU>(ld_ro(plane + ih * a.W + iw)) : -CUDART_INF_F;
                        }
                    bi = max(0, -h0) * kw + max(0, -w0);
                }
#pragma unroll
                for (int dy = 0; dy < (KH ? KH : 1); ++dy)
#pragma unroll
                    for (int dx = 0; dx < (KW ? KW : 1); ++dx) take(v[dy][dx], dy * kw + dx, best, bi);
            } else
            for (int dy = 0; dy < kh; ++dy) {
                const int ih = h0 + dy;
                if (ih < 0 || ih >= a.H) continue;
                for (int dx = 0; dx < kw; ++dx) {
                    const int iw = w0 + dx;
                    if (iw < 0 || iw >= a.W) continue;
                    const float v = act<RELU>(ld_ro(plane + ih * a.W + iw));
                    if (bi < 0) bi = dy * kw + dx;  // first in-bounds position (all -inf case)
                    take(v, dy * kw + dx, best, bi);
                }
            }
            out[o] = best;
            nib = (uint32_t)bi << (4 * (lane & 7));
        }
        nib |= __shfl_xor_sync(kFull, nib, 1);
        nib |= __shfl_xor_sync(kFull, nib, 2);
        nib |= __shfl_xor_sync(kFull, nib, 4);
        if ((lane & 7) == 0 && o < (uint32_t)a.n_out) arg[o >> 3] = nib;
    }
}

// 2x2 stride 2, no padding, every window fully inside (W even): two float2 row loads per
// output.  A warp handles kFwdU chunks of 32 consecutive outputs per iteration with all
// 2*kFwdU loads issued before any compare (memory-level parallelism).
constexpr int kFwdU = 4;

__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_k2s2_kernel(const float *__restrict__ y, PoolArgs a, float *__restrict__ out,
                        uint32_t *__restrict__ arg) {
    pdl_enter();
    const int lane = threadIdx.x & 31;
    const int64_t chunks = ((int64_t)a.n_out + 31) / 32;
    const int64_t nwarps = ((int64_t)gridDim.x * kPoolThreads) >> 5;
    for (int64_t c0 = (((int64_t)blockIdx.x * kPoolThreads + threadIdx.x) >> 5) * kFwdU; c0 < chunks;
         c0 += nwarps * kFwdU) {
        float2 r0[kFwdU], r1[kFwdU];
#pragma unroll
        for (int u = 0; u < kFwdU; ++u) {
            const int64_t o = (c0 + u) * 32 + lane;
            if (o < a.n_out) {
                uint32_t q, ow, nc, oh;
                a.div_wo.divmod((uint32_t)o, q, ow);
                a.div_ho.divmod(q, nc, oh);
                const float *p = y + (int64_t)nc * a.H * a.W + (int64_t)(2 * oh) * a.W + 2 * ow;
                r0[u] = ld_stream_f2(reinterpret_cast<const float2 *>(p));
                r1[u] = ld_stream_f2(reinterpret_cast<const float2 *>(p + a.W));
            }
        }
#pragma unroll
        for (int u = 0; u < kFwdU; ++u) {
            const int64_t o = (c0 + u) * 32 + lane;
            uint32_t nib = 0;
            if (o < a.n_out) {
                float best = -CUDART_INF_F;
                int bi = 0;
                take(r0[u].x, 0, best, bi);
                take(r0[u].y, 1, best, bi);
                take(r1[u].x, 2, best, bi);
                take(r1[u].y, 3, best, bi);
                out[o] = best;
                nib = (uint32_t)bi << (4 * (lane & 7));
            }
            nib |= __shfl_xor_sync(kFull, nib, 1);
            nib |= __shfl_xor_sync(kFull, nib, 2);
            nib |= __shfl_xor_sync(kFull, nib, 4);
            if ((lane & 7) == 0 && o < a.n_out) arg[o >> 3] = nib;
        }
    }
}

// ---- 2x2 stride 2, no padding, W % 4 == 0 (every VGG16 / most OverFeat sites): one thread
// per PAIR of adjacent outputs = one 2x4 input block, so both input rows are single aligned
// float4 accesses.  Flat output row R = o / Wo needs one fast division; when H is even the
// window's top input row is simply 2R.  Four consecutive lanes own one argmax word.
#ifndef GIST_POOL_PAIR_U
#define GIST_POOL_PAIR_U 1
#endif
constexpr int kPairU = GIST_POOL_PAIR_U;  // output pairs in flight per thread

template <bool EVEN_H>
__device__ __forceinline__ int64_t pair_top_left(const PoolArgs &a, uint32_t o, uint32_t &R, uint32_t &ow) {
    a.div_wo.divmod(o, R, ow);
    if (EVEN_H) return (int64_t)(2 * R) * a.W + 2 * ow;
    uint32_t nc, oh;
    a.div_ho.divmod(R, nc, oh);
    return ((int64_t)nc * a.H + 2 * oh) * a.W + 2 * ow;
}

__device__ __forceinline__ void win4(float t0, float t1, float b0, float b1, float &best, uint32_t &bi) {
    float m = -CUDART_INF_F;
    int k = 0;
    take(t0, 0, m, k);
    take(t1, 1, m, k);
    take(b0, 2, m, k);
    take(b1, 3, m, k);
    best = m;
    bi = (uint32_t)k;
}

template <bool EVEN_H>
__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_k2s2_pair_kernel(const float *__restrict__ y, PoolArgs a, float *__restrict__ out,
                             uint32_t *__restrict__ arg) {
    pdl_enter();
    const int lane = threadIdx.x & 31;
    const int64_t pairs = (int64_t)a.n_out / 2;
    const int64_t chunks = (pairs + 31) / 32;
    const int64_t nwarps = ((int64_t)gridDim.x * kPoolThreads) >> 5;
    for (int64_t c0 = (((int64_t)blockIdx.x * kPoolThreads + threadIdx.x) >> 5) * kPairU; c0 < chunks;
         c0 += nwarps * kPairU) {
        float4 t[kPairU], b[kPairU];
#pragma unroll
        for (int u = 0; u < kPairU; ++u) {
            const int64_t q = (c0 + u) * 32 + lane;
            if (q < pairs) {
                uint32_t R, ow;
                const int64_t i0 = pair_top_left<EVEN_H>(a, (uint32_t)(2 * q), R, ow);
                t[u] = ld_stream_f4(reinterpret_cast<const float4 *>(y + i0));
                b[u] = ld_stream_f4(reinterpret_cast<const float4 *>(y + i0 + a.W));
            }
        }
#pragma unroll
        for (int u = 0; u < kPairU; ++u) {
            const int64_t q = (c0 + u) * 32 + lane;
            uint32_t byte = 0;
            if (q < pairs) {
                float m0, m1;
                uint32_t k0, k1;
                win4(t[u].x, t[u].y, b[u].x, b[u].y, m0, k0);
                win4(t[u].z, t[u].w, b[u].z, b[u].w, m1, k1);
                reinterpret_cast<float2 *>(out)[q] = make_float2(m0, m1);
                byte = (k0 | (k1 << 4)) << (8 * (lane & 3));
            }
            byte |= __shfl_xor_sync(kFull, byte, 1);
            byte |= __shfl_xor_sync(kFull, byte, 2);
            if ((lane & 3) == 0 && q < pairs) arg[q >> 2] = byte;
        }
    }
}

// ---- 2x2/s2 forward with the a1 mask fused, any even W, H even: the map is a sequence of
// row blocks (input rows 2R, 2R+1 = output row R) that are contiguous in NCHW, so a run of
// whole blocks is one contiguous range of y, out, argmax nibbles and mask bits.  Runs ("units")
// of BR blocks with BR*W = 0 mod 16 start on argmax-word and mask-word boundaries, so a warp
// owns every word of its unit.  Items: V = 4 columns (an output pair, float4 rows, W % 4 == 0)
// or V = 2 (one output, float2 rows).  Each item's V top and V bottom mask bits go to a per-warp
// byte buffer (one byte per V-bit unit, in memory order: a block's top units, then its bottom
// units), which the warp packs into whole mask words at the end of the unit.  y is read once.
constexpr int kFusedUnitItems = 512;  // items per unit (upper bound; host picks BR)
constexpr int kFusedU = 4;            // items per lane in flight

template <int V, bool RELU = false>
__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_k2s2_fused_kernel(const float *__restrict__ y, PoolArgs a, int64_t blocks, int32_t BR, FastDiv div_ipr,
                              float *__restrict__ out, uint32_t *__restrict__ arg, uint32_t *__restrict__ mask) {
    pdl_enter();
    __shared__ __align__(16) uint8_t s_units[kPoolThreads / 32][2 * kFusedUnitItems + 32];
    using VecT = typename std::conditional<V == 4, float4, float2>::type;
    const int lane = threadIdx.x & 31;
    uint8_t *ub = s_units[threadIdx.x >> 5];
    const int ipr = a.W / V;                      // items per row
    const int64_t units = (blocks + BR - 1) / BR;
    const int64_t nwarps = ((int64_t)gridDim.x * kPoolThreads) >> 5;
    for (int64_t u = ((int64_t)blockIdx.x * kPoolThreads + threadIdx.x) >> 5; u < units; u += nwarps) {
        const int64_t R0 = u * BR;
        const int nb = (int)((R0 + BR <= blocks) ? BR : blocks - R0);
        const int ni = nb * ipr;                  // items in this unit
        const int64_t e0 = R0 * 2 * a.W;          // first input element (word aligned)
        const int64_t o0 = R0 * a.Wo;             // first output (argmax-word aligned)
        for (int jb = 0; jb < ni; jb += 32 * kFusedU) {
            VecT t[kFusedU], bt[kFusedU];
            uint32_t rb[kFusedU], rp[kFusedU];
#pragma unroll
            for (int k = 0; k < kFusedU; ++k) {
                const int j = jb + 32 * k + lane;
                if (j < ni) {
                    div_ipr.divmod((uint32_t)j, rb[k], rp[k]);
                    const float *p = y + e0 + (int64_t)rb[k] * 2 * a.W + V * rp[k];
                    t[k] = *reinterpret_cast<const VecT *>(p);   // (streamed: read once)
                    bt[k] = *reinterpret_cast<const VecT *>(p + a.W);
                }
            }
#pragma unroll
            for (int k = 0; k < kFusedU; ++k) {
                const int j = jb + 32 * k + lane;
                uint32_t part = 0;
                if (j < ni) {
                    uint32_t nt, nbm;
                    if constexpr (V == 4) {
                        float m0, m1;
                        uint32_t k0, k1;
                        // mask bits below compare the raw values: relu(v) > 0 iff v > 0
                        win4(act<RELU>(t[k].x), act<RELU>(t[k].y), act<RELU>(bt[k].x), act<RELU>(bt[k].y), m0, k0);
                        win4(act<RELU>(t[k].z), act<RELU>(t[k].w), act<RELU>(bt[k].z), act<RELU>(bt[k].w), m1, k1);
                        reinterpret_cast<float2 *>(out + o0)[j] = make_float2(m0, m1);
                        part = (k0 | (k1 << 4)) << (8 * (lane & 3));
                        nt = (uint32_t)(t[k].x > 0.0f) | ((uint32_t)(t[k].y > 0.0f) << 1) |
                             ((uint32_t)(t[k].z > 0.0f) << 2) | ((uint32_t)(t[k].w > 0.0f) << 3);
                        nbm = (uint32_t)(bt[k].x > 0.0f) | ((uint32_t)(bt[k].y > 0.0f) << 1) |
                              ((uint32_t)(bt[k].z > 0.0f) << 2) | ((uint32_t)(bt[k].w > 0.0f) << 3);
                    } else {
                        float m;
                        uint32_t kk;
                        win4(act<RELU>(t[k].x), act<RELU>(t[k].y), act<RELU>(bt[k].x), act<RELU>(bt[k].y), m, kk);
                        out[o0 + j] = m;
                        part = kk << (4 * (lane & 7));
                        nt = (uint32_t)(t[k].x > 0.0f) | ((uint32_t)(t[k].y > 0.0f) << 1);
                        nbm = (uint32_t)(bt[k].x > 0.0f) | ((uint32_t)(bt[k].y > 0.0f) << 1);
                    }
                    // R1 bits of the item's top and bottom units, in memory order
                    const int ut = (int)rb[k] * 2 * ipr + (int)rp[k];
                    ub[ut] = (uint8_t)nt;
                    ub[ut + ipr] = (uint8_t)nbm;
                }
                if constexpr (V == 4) {  // 4 items (8 nibbles) per argmax word
                    part |= __shfl_xor_sync(kFull, part, 1);
                    part |= __shfl_xor_sync(kFull, part, 2);
                    if ((lane & 3) == 0 && j < ni) arg[((o0 >> 1) + j) >> 2] = part;
                } else {                 // 8 items per argmax word
                    part |= __shfl_xor_sync(kFull, part, 1);
                    part |= __shfl_xor_sync(kFull, part, 2);
                    part |= __shfl_xor_sync(kFull, part, 4);
                    if ((lane & 7) == 0 && j < ni) arg[(o0 + j) >> 3] = part;
                }
            }
        }
        __syncwarp();
        // pack the unit's mask words: 32 / V units of V bits each
        constexpr int kPer = 32 / V;
        const int nu = 2 * ni;
        const int nw = (nu + kPer - 1) / kPer;
        for (int w = lane; w < nw; w += 32) {
            uint32_t word = 0;
#pragma unroll
            for (int i = 0; i < kPer; ++i) {
                const int x = w * kPer + i;
                if (x < nu) word |= (uint32_t)ub[x] << (V * i);
            }
            mask[(e0 >> 5) + w] = word;
        }
        __syncwarp();
    }
}

template <bool EVEN_H>
__global__ void __launch_bounds__(kPoolThreads)
pool_bwd_k2s2_pair_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                          const uint32_t *__restrict__ mask, PoolArgs a, float *__restrict__ dx) {
    pdl_enter();
    const int64_t pairs = (int64_t)a.n_out / 2;
    const int64_t stride = (int64_t)gridDim.x * kPoolThreads;
    for (int64_t q0 = (int64_t)blockIdx.x * kPoolThreads + threadIdx.x; q0 < pairs; q0 += stride * kPairU) {
        float2 g[kPairU];
        uint32_t nb[kPairU], m0[kPairU], m1[kPairU], R[kPairU], ow[kPairU];
        int64_t i0[kPairU];
#pragma unroll
        for (int u = 0; u < kPairU; ++u) {
            const int64_t q = q0 + u * stride;
            if (q < pairs) {
                i0[u] = pair_top_left<EVEN_H>(a, (uint32_t)(2 * q), R[u], ow[u]);
                g[u] = ld_stream_f2(reinterpret_cast<const float2 *>(dout) + q);
                nb[u] = ld_ro(arg + (q >> 2)) >> (8 * (q & 3));
                if (mask) {
                    m0[u] = ld_ro(mask + (i0[u] >> 5)) >> (i0[u] & 31);
                    m1[u] = ld_ro(mask + ((i0[u] + a.W) >> 5)) >> ((i0[u] + a.W) & 31);
                } else {
                    m0[u] = m1[u] = 0xfu;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kPairU; ++u) {
            const int64_t q = q0 + u * stride;
            if (q >= pairs) break;
            const float v0 = 0.0f + g[u].x, v1 = 0.0f + g[u].y;  // R6: +0.0f + dY
            const uint32_t k0 = nb[u] & 0xfu, k1 = (nb[u] >> 4) & 0xfu;
            float4 top, bot;
            top.x = (k0 == 0 && (m0[u] & 1u)) ? v0 : 0.0f;
            top.y = (k0 == 1 && (m0[u] & 2u)) ? v0 : 0.0f;
            top.z = (k1 == 0 && (m0[u] & 4u)) ? v1 : 0.0f;
            top.w = (k1 == 1 && (m0[u] & 8u)) ? v1 : 0.0f;
            bot.x = (k0 == 2 && (m1[u] & 1u)) ? v0 : 0.0f;
            bot.y = (k0 == 3 && (m1[u] & 2u)) ? v0 : 0.0f;
            bot.z = (k1 == 2 && (m1[u] & 4u)) ? v1 : 0.0f;
            bot.w = (k1 == 3 && (m1[u] & 8u)) ? v1 : 0.0f;
            *reinterpret_cast<float4 *>(dx + i0[u]) = top;
            *reinterpret_cast<float4 *>(dx + i0[u] + a.W) = bot;
            if (!EVEN_H) {  // floor mode, odd H: zero the plane's uncovered last input row
                uint32_t nc, oh;
                a.div_ho.divmod(R[u], nc, oh);
                if ((int)oh == a.Ho - 1)
                    *reinterpret_cast<float4 *>(dx + i0[u] + 2 * (int64_t)a.W) = make_float4(0.f, 0.f, 0.f, 0.f);
            }
        }
    }
}

__device__ __forceinline__ uint32_t nibble(const uint32_t *__restrict__ arg, int64_t o) {
    return (ld_ro(arg + (o >> 3)) >> (4 * (o & 7))) & 0xfu;
}

__device__ __forceinline__ bool mask_bit(const uint32_t *__restrict__ mask, int64_t i) {
    return (ld_ro(mask + (i >> 5)) >> (i & 31)) & 1u;
}

// Generic gather backward: one thread per input element.
template <int KH, int KW, int SH, int SW>
__global__ void __launch_bounds__(kPoolThreads)
pool_bwd_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg, const uint32_t *__restrict__ mask,
                PoolArgs a, float *__restrict__ dx) {
    pdl_enter();
    const int kh = KH ? KH : a.kh, kw = KW ? KW : a.kw;
    const int sh = SH ? SH : a.sh, sw = SW ? SW : a.sw;
    const int64_t stride = (int64_t)gridDim.x * kPoolThreads;
    for (int64_t i = (int64_t)blockIdx.x * kPoolThreads + threadIdx.x; i < a.n_in; i += stride) {
        uint32_t q, iw, nc, ih;
        a.div_w.divmod((uint32_t)i, q, iw);
        a.div_h.divmod(q, nc, ih);
        float acc = 0.0f;
        if (mask == nullptr || mask_bit(mask, i)) {
            const int th = (int)ih + a.ph, tw = (int)iw + a.pw;
            const int oh_lo = th - kh + 1 > 0 ? (th - kh + 1 + sh - 1) / sh : 0;
            const int oh_hi = min(a.Ho - 1, th / sh);
            const int ow_lo = tw - kw + 1 > 0 ? (tw - kw + 1 + sw - 1) / sw : 0;
            const int ow_hi = min(a.Wo - 1, tw / sw);
            const int64_t obase = (int64_t)nc * a.Ho;
            for (int oh = oh_lo; oh <= oh_hi; ++oh) {
                const int ly = th - oh * sh;  // = ih - (oh*sh - ph)
                for (int ow = ow_lo; ow <= ow_hi; ++ow) {
                    const int64_t o = (obase + oh) * a.Wo + ow;
                    if (nibble(arg, o) == (uint32_t)(ly * kw + (tw - ow * sw))) acc = acc + ld_ro(dout + o);
                }
            }
        }
        dx[i] = acc;
    }
}

// 2x2 stride 2, no padding, every window inside: one thread per pool output writes its
// whole 2x2 input block (two float2 rows).  Windows do not overlap, so dx is dY routed to
// the argmax slot (+0.0f + dY, R6) and selected by the mask (R7); inputs in an uncovered
// last row (odd H, floor mode) are zeroed by the owner of the row above.  All loads of
// kBwdU outputs are issued before use.
constexpr int kBwdU = 4;

__global__ void __launch_bounds__(kPoolThreads)
pool_bwd_k2s2_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                     const uint32_t *__restrict__ mask, PoolArgs a, float *__restrict__ dx) {
    pdl_enter();
    const int64_t stride = (int64_t)gridDim.x * kPoolThreads;
    const bool odd_h = (a.H & 1) != 0;
    for (int64_t o0 = (int64_t)blockIdx.x * kPoolThreads + threadIdx.x; o0 < a.n_out; o0 += stride * kBwdU) {
        float g[kBwdU];
        uint32_t nib[kBwdU], m0[kBwdU], m1[kBwdU];
        int64_t i0[kBwdU];
#pragma unroll
        for (int u = 0; u < kBwdU; ++u) {
            const int64_t o = o0 + u * stride;
            if (o < a.n_out) {
                uint32_t q, ow, nc, oh;
                a.div_wo.divmod((uint32_t)o, q, ow);
                a.div_ho.divmod(q, nc, oh);
                i0[u] = ((int64_t)nc * a.H + 2 * oh) * a.W + 2 * ow;  // top-left input
                g[u] = ld_stream_f32(dout + o);
                nib[u] = ld_ro(arg + (o >> 3)) >> (4 * (o & 7));
                if (mask) {
                    m0[u] = ld_ro(mask + (i0[u] >> 5)) >> (i0[u] & 31);
                    m1[u] = ld_ro(mask + ((i0[u] + a.W) >> 5)) >> ((i0[u] + a.W) & 31);
                } else {
                    m0[u] = m1[u] = 3u;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kBwdU; ++u) {
            const int64_t o = o0 + u * stride;
            if (o >= a.n_out) break;
            const float v = 0.0f + g[u];
            const uint32_t k = nib[u] & 0xfu;
            float2 top, bot;
            top.x = (k == 0 && (m0[u] & 1u)) ? v : 0.0f;
            top.y = (k == 1 && (m0[u] & 2u)) ? v : 0.0f;
            bot.x = (k == 2 && (m1[u] & 1u)) ? v : 0.0f;
            bot.y = (k == 3 && (m1[u] & 2u)) ? v : 0.0f;
            *reinterpret_cast<float2 *>(dx + i0[u]) = top;
            *reinterpret_cast<float2 *>(dx + i0[u] + a.W) = bot;
            if (odd_h) {  // zero the uncovered last input row of the plane
                uint32_t q, ow, nc, oh;
                a.div_wo.divmod((uint32_t)o, q, ow);
                a.div_ho.divmod(q, nc, oh);
                if ((int)oh == a.Ho - 1 && 2 * a.Ho < a.H)
                    *reinterpret_cast<float2 *>(dx + i0[u] + 2 * (int64_t)a.W) = make_float2(0.0f, 0.0f);
            }
        }
    }
}

// ---- Generic-geometry backward (any window <= 16 positions, stride, padding, ceil mode):
// shared-memory tiles.  A tile is a band of output rows of one plane ("band") or several whole
// planes ("multi"); its dY rows are one contiguous range, staged once with coalesced float4
// loads, so every covering window is read from shared memory.
constexpr int kTileIn = 8192;   // staged floats per tile (32 KB)
constexpr int kTileThreads = 256;

struct TileSpec {
    int32_t multi;   // 1: G whole planes per tile, 0: TR output rows of one plane
    int32_t G, TR;
    int32_t bands;   // band mode: tiles per plane
    int64_t tiles;
    int32_t NC;
    FastDiv div_bands;
};

struct TileRange {
    int64_t p0, np;    // first plane, planes
    int32_t oh0, oh1;  // output rows [oh0, oh1) (multi: [0, Ho))
};

__device__ __forceinline__ TileRange tile_range(const TileSpec &T, const PoolArgs &a, int64_t tile) {
    TileRange r;
    if (T.multi) {
        r.p0 = tile * T.G;
        r.np = min((int64_t)T.G, (int64_t)T.NC - r.p0);
        r.oh0 = 0;
        r.oh1 = a.Ho;
    } else {
        uint32_t plane, band;
        T.div_bands.divmod((uint32_t)tile, plane, band);
        r.p0 = plane;
        r.np = 1;
        r.oh0 = (int)band * T.TR;
        r.oh1 = min(a.Ho, r.oh0 + T.TR);
    }
    return r;
}

// Stage global floats [g_lo, g_hi) into smem: s[g - base], base = g_lo & ~3 (16-B phase kept).
__device__ __forceinline__ int64_t stage_range(float *s, const float *__restrict__ g, int64_t g_lo, int64_t g_hi,
                                               int64_t n_total) {
    const int64_t base = g_lo & ~3ll;
    const int64_t q_end = (g_hi + 3) >> 2;
    for (int64_t q4 = (base >> 2) + threadIdx.x; q4 < q_end; q4 += blockDim.x) {
        const int64_t e = q4 * 4;
        if (e + 4 <= n_total) {
            reinterpret_cast<float4 *>(s)[q4 - (base >> 2)] = ld_stream_f4(reinterpret_cast<const float4 *>(g) + q4);
        } else {
            for (int k = 0; k < 4; ++k) s[e - base + k] = (e + k < n_total) ? g[e + k] : 0.0f;
        }
    }
    return base;
}

template <int KH, int KW, int SH, int SW>
__global__ void __launch_bounds__(kTileThreads)
pool_bwd_tiled_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                      const uint32_t *__restrict__ mask, PoolArgs a, TileSpec T, float *__restrict__ dx) {
    pdl_enter();
    __shared__ __align__(16) float s_dy[kTileIn + 8];
    __shared__ uint32_t s_arg[kTileIn / 8 + 2];
    const int kh = KH ? KH : a.kh, kw = KW ? KW : a.kw, sh = SH ? SH : a.sh, sw = SW ? SW : a.sw;
    const int64_t HW = (int64_t)a.H * a.W, HoWo = (int64_t)a.Ho * a.Wo;
    for (int64_t tile = blockIdx.x; tile < T.tiles; tile += gridDim.x) {
        const TileRange r = tile_range(T, a, tile);
        // owned input rows: a partition of [0, H) across the plane's bands
        const int r_lo = (T.multi || r.oh0 == 0) ? 0 : min(a.H, max(0, r.oh0 * sh - a.ph));
        const int r_hi = (T.multi || r.oh1 == a.Ho) ? a.H : min(a.H, max(0, r.oh1 * sh - a.ph));
        // output rows whose windows cover them
        const int t_lo = r_lo + a.ph - kh + 1;
        const int os_lo = T.multi ? 0 : max(0, t_lo > 0 ? (t_lo + sh - 1) / sh : 0);
        const int os_hi = T.multi ? a.Ho : min(a.Ho, r_hi > r_lo ? (r_hi - 1 + a.ph) / sh + 1 : os_lo);
        const int64_t od_lo = r.p0 * HoWo + (int64_t)os_lo * a.Wo;
        const int64_t od_hi = (r.p0 + r.np - 1) * HoWo + (int64_t)max(os_hi, os_lo) * a.Wo;
        const int64_t dbase = stage_range(s_dy, dout, od_lo, od_hi, a.n_out);
        const int64_t w_lo = od_lo >> 3;
        for (int64_t w = w_lo + threadIdx.x; w < ((od_hi + 7) >> 3); w += blockDim.x) s_arg[w - w_lo] = ld_ro(arg + w);
        __syncthreads();
        const int64_t i_lo = r.p0 * HW + (int64_t)r_lo * a.W;
        const int64_t i_hi = (r.p0 + r.np - 1) * HW + (int64_t)r_hi * a.W;
        for (int64_t i = i_lo + threadIdx.x; i < i_hi; i += blockDim.x) {
            uint32_t q, iw, nc, ih;
            a.div_w.divmod((uint32_t)i, q, iw);
            a.div_h.divmod(q, nc, ih);
            float acc = 0.0f;  // R6: +0.0f, then ascending output order
            if (mask == nullptr || ((ld_ro(mask + (i >> 5)) >> (i & 31)) & 1u)) {
                const int th = (int)ih + a.ph, tw = (int)iw + a.pw;
                const int oh_lo = th - kh + 1 > 0 ? (th - kh + 1 + sh - 1) / sh : 0;
                const int oh_hi = min(a.Ho - 1, th / sh);
                const int ow_lo = tw - kw + 1 > 0 ? (tw - kw + 1 + sw - 1) / sw : 0;
                const int ow_hi = min(a.Wo - 1, tw / sw);
                const int64_t ob = (int64_t)nc * HoWo;
                for (int oh = oh_lo; oh <= oh_hi; ++oh) {
                    const int ly = th - oh * sh;
                    for (int ow = ow_lo; ow <= ow_hi; ++ow) {
                        const int64_t o = ob + (int64_t)oh * a.Wo + ow;
                        const uint32_t nib = (s_arg[(o >> 3) - w_lo] >> (4 * (o & 7))) & 0xfu;
                        if (nib == (uint32_t)(ly * kw + (tw - ow * sw))) acc = acc + s_dy[o - dbase];
                    }
                }
            }
            dx[i] = acc;
        }
        __syncthreads();
    }
}

// Same 2x2-block formulation without tiles: candidate windows' dY and nibbles come straight
// through L1 (neighbouring blocks share them), all loads issued before use.  For 3x3 stride 2
// each window can only hit block (A, b) = rows 2A..2A+1 x cols 2b..2b+1 through fixed nibbles
// (nibble = 3*dy + dx):  (A-1,b-1): 8 -> (0,0);  (A-1,b): 6 -> (0,0), 7 -> (0,1);
// (A,b-1): 2 -> (0,0), 5 -> (1,0);  (A,b): 0 -> (0,0), 1 -> (0,1), 3 -> (1,0), 4 -> (1,1).
// Windows are visited in ascending output order (R6).
__global__ void __launch_bounds__(kPoolThreads)
pool_bwd_k3s2_block_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                           const uint32_t *__restrict__ mask, PoolArgs a, FastDiv div_wb, FastDiv div_hb,
                           int64_t nblk, float *__restrict__ dx) {
    pdl_enter();
    // 32-bit element indices (the API rejects maps of 2^31 elements or more): one 64-bit address per
    // row of loads or stores, the rest immediate offsets
    const uint32_t HW = (uint32_t)a.H * (uint32_t)a.W, HoWo = (uint32_t)a.Ho * (uint32_t)a.Wo;
    const uint32_t stride = gridDim.x * blockDim.x, nb = (uint32_t)nblk;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < nb; t += stride) {
        uint32_t q, b, plane, A;
        div_wb.divmod(t, q, b);
        div_hb.divmod(q, plane, A);
        const bool up = A >= 1, left = b >= 1;                      // windows (A-1, .) / (., b-1) exist
        const bool here_r = (int)A < a.Ho, here_c = (int)b < a.Wo;  // windows (A, .) / (., b) exist
        // signed offsets: o00 (and o11 - 1) are negative at the map's first windows, where the
        // loads they address are not made
        const int o11 = (int)(plane * HoWo + A * (uint32_t)a.Wo + b);  // window (A, b)
        const int o00 = o11 - a.Wo - 1;                                 // window (A-1, b-1)
        const float *g0 = dout + o00, *g1 = dout + (o11 - 1);          // rows A-1 and A of dY
        float g[4] = {0.f, 0.f, 0.f, 0.f};
        uint32_t nbv[4] = {15u, 15u, 15u, 15u};  // 15: no window / no hit
        const bool ok[4] = {up && left, up && here_c, here_r && left, here_r && here_c};
        const int os[4] = {o00, o00 + 1, o11 - 1, o11};
        const uint32_t i00 = plane * HW + (2 * A) * (uint32_t)a.W + 2 * b;
        const bool r1 = 2 * (int)A + 1 < a.H, c1 = 2 * (int)b + 1 < a.W;
        // every load is issued before any is used (the mask words' latency overlaps the dY and
        // argmax loads'; with the mask read after the nibbles were decoded it was a second round trip)
        const bool hm = mask != nullptr;
        const uint32_t i10 = i00 + (uint32_t)a.W;
        // the right-hand bit is read only when that column exists (c1): in the last column of an
        // odd-W map, element i00 + 1 may be element n, one word past the mask buffer
        const uint32_t w0 = hm ? ld_ro(mask + (i00 >> 5)) : ~0u;
        const uint32_t w0b = hm && c1 ? ld_ro(mask + ((i00 + 1) >> 5)) : ~0u;
        const uint32_t w1 = hm && r1 ? ld_ro(mask + (i10 >> 5)) : ~0u;
        const uint32_t w1b = hm && r1 && c1 ? ld_ro(mask + ((i10 + 1) >> 5)) : ~0u;
        uint32_t aw[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) aw[k] = ok[k] ? ld_ro(arg + (os[k] >> 3)) : 0u;
        if (ok[0]) g[0] = ld_ro(g0);
        if (ok[1]) g[1] = ld_ro(g0 + 1);
        if (ok[2]) g[2] = ld_ro(g1);
        if (ok[3]) g[3] = ld_ro(g1 + 1);
#pragma unroll
        for (int k = 0; k < 4; ++k)
            if (ok[k]) nbv[k] = (aw[k] >> (4 * (os[k] & 7))) & 0xfu;
        const uint32_t m0 = ((w0 >> (i00 & 31)) & 1u) | (((w0b >> ((i00 + 1) & 31)) & 1u) << 1);
        const uint32_t m1 = ((w1 >> (i10 & 31)) & 1u) | (((w1b >> ((i10 + 1) & 31)) & 1u) << 1);
        float a00 = 0.0f, a01 = 0.0f, a10 = 0.0f, a11 = 0.0f;  // +0.0f, then ascending o
        if (nbv[0] == 8u) a00 = a00 + g[0];
        if (nbv[1] == 6u) a00 = a00 + g[1];
        if (nbv[1] == 7u) a01 = a01 + g[1];
        if (nbv[2] == 2u) a00 = a00 + g[2];
        if (nbv[2] == 5u) a10 = a10 + g[2];
        if (nbv[3] == 0u) a00 = a00 + g[3];
        if (nbv[3] == 1u) a01 = a01 + g[3];
        if (nbv[3] == 3u) a10 = a10 + g[3];
        if (nbv[3] == 4u) a11 = a11 + g[3];
        float *d0 = dx + i00, *d1 = d0 + a.W;
        d0[0] = (m0 & 1u) ? a00 : 0.0f;
        if (c1) d0[1] = (m0 & 2u) ? a01 : 0.0f;
        if (r1) {
            d1[0] = (m1 & 1u) ? a10 : 0.0f;
            if (c1) d1[1] = (m1 & 2u) ? a11 : 0.0f;
        }
    }
}

// Host: tiles for the generic kernels.  Forward stages input rows (bounded by kTileIn floats);
// backward stages dY rows (bounded likewise).
TileSpec make_tiles(const PoolArgs &a, int32_t NC, bool backward) {
    TileSpec T{};
    T.NC = NC;
    // forward stages input rows and keeps one nibble byte per output; backward stages dY rows
    const int64_t plane = backward ? (int64_t)a.Ho * a.Wo : std::max((int64_t)a.H * a.W, (int64_t)a.Ho * a.Wo);
    if (plane <= kTileIn) {
        T.multi = 1;
        T.G = (int32_t)(kTileIn / plane);
        T.tiles = ceil_div(NC, T.G);
        T.TR = a.Ho;
        T.bands = 1;
    } else {
        T.multi = 0;
        int64_t tr;
        if (backward) {  // staged output rows = TR + floor((kh-1)/sh) <= kTileIn / Wo
            tr = kTileIn / a.Wo - (a.kh - 1) / a.sh - 1;
        } else {  // staged input rows (TR-1)*sh + kh <= kTileIn / W, and TR*Wo nibbles
            tr = std::min<int64_t>((kTileIn / a.W - a.kh) / a.sh + 1, kTileIn / a.Wo);
        }
        T.TR = (int32_t)std::min<int64_t>(std::max<int64_t>(1, tr), a.Ho);
        T.bands = (int32_t)ceil_div(a.Ho, T.TR);
        T.tiles = (int64_t)NC * T.bands;
        T.G = 1;
    }
    T.div_bands = FastDiv::make((uint32_t)std::max(1, T.bands));
    return T;
}

PoolArgs make_args(int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo) {
    PoolArgs a;
    a.H = H;
    a.W = W;
    a.Ho = Ho;
    a.Wo = Wo;
    a.kh = p.kh;
    a.kw = p.kw;
    a.sh = p.sh;
    a.sw = p.sw;
    a.ph = p.ph;
    a.pw = p.pw;
    a.n_out = (int32_t)((int64_t)N * C * Ho * Wo);
    a.n_in = (int32_t)((int64_t)N * C * H * W);
    a.div_wo = FastDiv::make((uint32_t)Wo);
    a.div_ho = FastDiv::make((uint32_t)Ho);
    a.div_w = FastDiv::make((uint32_t)W);
    a.div_h = FastDiv::make((uint32_t)H);
    return a;
}

// The tiled kernels need a band of at least one output row's windows (fwd) / one staged output
// row (bwd) to fit the tile, and windows of at most 4x4.
bool tiled_ok(const PoolArgs &a) {
    return a.kh <= 4 && a.kw <= 4 && (int64_t)a.kh * a.W <= kTileIn && (int64_t)(a.kh + 2) * a.Wo <= kTileIn;
}

bool is_k2s2_exact(const gist_pool2d &p, int32_t H, int32_t W, int32_t Ho, int32_t Wo) {
    // every window fully inside: 2x2/s2/p0 with 2*Ho <= H and 2*Wo == W (W even)
    return p.kh == 2 && p.kw == 2 && p.sh == 2 && p.sw == 2 && p.ph == 0 && p.pw == 0 && (W % 2 == 0) &&
           2 * Ho <= H && 2 * Wo == W;
}

unsigned grid_for(int64_t work_items, int64_t items_per_block, int per_sm) {
    int64_t blocks = ceil_div(work_items, items_per_block);
    const int64_t cap = (int64_t)num_sms() * per_sm;
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    return (unsigned)blocks;
}

}  // namespace

cudaError_t launch_relu_maxpool_fwd(const float *x, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                                    int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, uint32_t *mask, bool *mask_fused,
                                    cudaStream_t s) {
    // f3: relu on load.  The fused 2x2/s2 kernel writes the mask in the same pass; other
    // geometries use the L1 forward with relu on load and the caller adds binarize(x).
    const PoolArgs a = make_args(N, C, H, W, p, Ho, Wo);
    *mask_fused = false;
    if (GIST_POOL3 && pool3_ok(p, true)) {
        const cudaError_t e = launch_pool3_fwd(x, N, C, H, W, p, Ho, Wo, out, argmax, mask, true, s);
        if (e != cudaErrorNotSupported) {
            *mask_fused = mask != nullptr;
            return e;
        }
    }
    if (is_k2s2_exact(p, H, W, Ho, Wo) && H == 2 * Ho) {
        const int V = (W % 4 == 0) ? 4 : 2;
        const int ipr = W / V;
        int align = 16;
        for (int g = W; g % 2 == 0 && align > 1; g /= 2) align /= 2;
        const int64_t blocks = (int64_t)N * C * Ho;
        const int64_t BR = align * std::max<int64_t>(1, 256 / ((int64_t)align * ipr));
        if (BR * ipr <= kFusedUnitItems) {
            const unsigned g = grid_for(ceil_div(blocks, BR), kPoolThreads / 32, GIST_POOL_FWD_CTAS);
            const FastDiv d = FastDiv::make((uint32_t)ipr);
            if (V == 4)
                launch_k(maxpool_fwd_k2s2_fused_kernel<4, true>, g, kPoolThreads, 0, s, x, a, blocks, (int32_t)BR, d, out, argmax, mask);
            else
                launch_k(maxpool_fwd_k2s2_fused_kernel<2, true>, g, kPoolThreads, 0, s, x, a, blocks, (int32_t)BR, d, out, argmax, mask);
            *mask_fused = true;
            return cudaPeekAtLastError();
        }
    }
    const unsigned grid = grid_for(a.n_out, kPoolThreads, GIST_POOL_GEN_CTAS);
    if (p.kh == 3 && p.kw == 3)
        launch_k(maxpool_fwd_kernel<3, 3, true>, grid, kPoolThreads, 0, s, x, a, out, argmax);
    else
        launch_k(maxpool_fwd_kernel<0, 0, true>, grid, kPoolThreads, 0, s, x, a, out, argmax);
    return cudaPeekAtLastError();
}

cudaError_t launch_maxpool_fwd(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                               int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, cudaStream_t s, uint32_t *mask,
                               bool *mask_fused) {
    const PoolArgs a = make_args(N, C, H, W, p, Ho, Wo);
    if (mask_fused) *mask_fused = false;
    if (GIST_POOL3 && pool3_ok(p, true)) {
        const cudaError_t e = launch_pool3_fwd(y, N, C, H, W, p, Ho, Wo, out, argmax, mask_fused ? mask : nullptr,
                                               false, s);
        if (e != cudaErrorNotSupported) {
            if (mask_fused) *mask_fused = mask != nullptr;
            return e;
        }
    }
    if (mask && is_k2s2_exact(p, H, W, Ho, Wo) && H == 2 * Ho) {
        // units of BR whole row blocks with BR*W = 0 mod 16 (word-aligned), ~256 items each
        const int V = (W % 4 == 0) ? 4 : 2;
        const int ipr = W / V;
        int align = 16;
        for (int g = W; g % 2 == 0 && align > 1; g /= 2) align /= 2;  // 16 / gcd(W, 16)
        const int64_t blocks = (int64_t)N * C * Ho;
        int64_t BR = align * std::max<int64_t>(1, 256 / ((int64_t)align * ipr));
        if (BR * ipr <= kFusedUnitItems) {
            const unsigned g = grid_for(ceil_div(blocks, BR), kPoolThreads / 32, GIST_POOL_FWD_CTAS);
            const FastDiv d = FastDiv::make((uint32_t)ipr);
            if (V == 4)
                launch_k(maxpool_fwd_k2s2_fused_kernel<4>, g, kPoolThreads, 0, s, y, a, blocks, (int32_t)BR, d, out, argmax, mask);
            else
                launch_k(maxpool_fwd_k2s2_fused_kernel<2>, g, kPoolThreads, 0, s, y, a, blocks, (int32_t)BR, d, out, argmax, mask);
            if (mask_fused) *mask_fused = true;
            return cudaPeekAtLastError();
        }
    }
    const unsigned grid = grid_for(a.n_out, kPoolThreads, GIST_POOL_GEN_CTAS);
    if (is_k2s2_exact(p, H, W, Ho, Wo) && W % 4 == 0) {
        const unsigned g2 = grid_for(ceil_div(a.n_out / 2, 32 * kPairU), kPoolThreads / 32, 8);
        if (H == 2 * Ho) launch_k(maxpool_fwd_k2s2_pair_kernel<true>, g2, kPoolThreads, 0, s, y, a, out, argmax);
        else launch_k(maxpool_fwd_k2s2_pair_kernel<false>, g2, kPoolThreads, 0, s, y, a, out, argmax);
    } else if (is_k2s2_exact(p, H, W, Ho, Wo))
        launch_k(maxpool_fwd_k2s2_kernel, grid_for(ceil_div(a.n_out, kFwdU), kPoolThreads, 8), kPoolThreads, 0, s, y, a, out, argmax);
    else if (p.kh == 3 && p.kw == 3)
        launch_k(maxpool_fwd_kernel<3, 3>, grid, kPoolThreads, 0, s, y, a, out, argmax);
    else
        launch_k(maxpool_fwd_kernel<0, 0>, grid, kPoolThreads, 0, s, y, a, out, argmax);
    return cudaPeekAtLastError();
}

cudaError_t launch_pool_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                            int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo, float *dx,
                            cudaStream_t s) {
    const PoolArgs a = make_args(N, C, H, W, p, Ho, Wo);
    if (GIST_POOL3 && pool3_ok(p, false)) {
        const cudaError_t e = launch_pool3_bwd(dout, argmax, mask, N, C, H, W, p, Ho, Wo, dx, s);
        if (e != cudaErrorNotSupported) return e;
    }
    if (is_k2s2_exact(p, H, W, Ho, Wo) && W % 4 == 0) {
        const unsigned g2 = grid_for(ceil_div(a.n_out / 2, kPairU), kPoolThreads, GIST_POOL_BWD_CTAS);
        if (H == 2 * Ho) launch_k(pool_bwd_k2s2_pair_kernel<true>, g2, kPoolThreads, 0, s, dout, argmax, mask, a, dx);
        else launch_k(pool_bwd_k2s2_pair_kernel<false>, g2, kPoolThreads, 0, s, dout, argmax, mask, a, dx);
    } else if (pool_planes_ok(p, H, W, Ho, Wo)) {
        return launch_pool3s1_planes_bwd(dout, argmax, mask, N, C, H, W, p, Ho, Wo, dx, s);
    } else if (is_k2s2_exact(p, H, W, Ho, Wo)) {
        launch_k(pool_bwd_k2s2_kernel, grid_for(ceil_div(a.n_out, kBwdU), kPoolThreads, GIST_POOL_BWD_CTAS), kPoolThreads, 0, s, dout, argmax, mask, a, dx);
    } else if (p.kh == 3 && p.kw == 3 && p.sh == 2 && p.sw == 2 && p.ph == 0 && p.pw == 0) {
        const int32_t hb = (H + 1) / 2, wb = (W + 1) / 2;
        const int64_t nblk = (int64_t)N * C * hb * wb;
        launch_k(pool_bwd_k3s2_block_kernel, grid_for(nblk, kPoolThreads, GIST_POOL_GEN_CTAS), kPoolThreads, 0, s, 
            dout, argmax, mask, a, FastDiv::make(wb), FastDiv::make(hb), nblk, dx);
    } else if (tiled_ok(a)) {
        const TileSpec T = make_tiles(a, N * C, true);
        const unsigned gt = (unsigned)std::min<int64_t>(T.tiles, (int64_t)num_sms() * 6);
        if (p.kh == 3 && p.kw == 3 && p.sh == 2 && p.sw == 2)
            launch_k(pool_bwd_tiled_kernel<3, 3, 2, 2>, gt, kTileThreads, 0, s, dout, argmax, mask, a, T, dx);
        else if (p.kh == 3 && p.kw == 3 && p.sh == 1 && p.sw == 1)
            launch_k(pool_bwd_tiled_kernel<3, 3, 1, 1>, gt, kTileThreads, 0, s, dout, argmax, mask, a, T, dx);
        else
            launch_k(pool_bwd_tiled_kernel<0, 0, 0, 0>, gt, kTileThreads, 0, s, dout, argmax, mask, a, T, dx);
    } else {
        const unsigned grid = grid_for(a.n_in, kPoolThreads, 8);
        if (p.kh == 3 && p.kw == 3 && p.sh == 2 && p.sw == 2)
            launch_k(pool_bwd_kernel<3, 3, 2, 2>, grid, kPoolThreads, 0, s, dout, argmax, mask, a, dx);
        else if (p.kh == 3 && p.kw == 3 && p.sh == 1 && p.sw == 1)
            launch_k(pool_bwd_kernel<3, 3, 1, 1>, grid, kPoolThreads, 0, s, dout, argmax, mask, a, dx);
        else
            launch_k(pool_bwd_kernel<0, 0, 0, 0>, grid, kPoolThreads, 0, s, dout, argmax, mask, a, dx);
    }
    return cudaPeekAtLastError();
}

}  // namespace gist
