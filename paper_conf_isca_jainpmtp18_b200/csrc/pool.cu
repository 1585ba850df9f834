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

#include "common.cuh"
#include "kernels.h"

namespace gist {

namespace {

constexpr int kPoolThreads = 256;

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

// KH/KW > 0: compile-time window; 0: runtime (a.kh, a.kw).
template <int KH, int KW>
__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_kernel(const float *__restrict__ y, PoolArgs a, float *__restrict__ out, uint32_t *__restrict__ arg) {
    const int kh = KH ? KH : a.kh, kw = KW ? KW : a.kw;
    const int lane = threadIdx.x & 31;
    const int64_t chunks = ((int64_t)a.n_out + 31) / 32;
    const int64_t nwarps = ((int64_t)gridDim.x * kPoolThreads) >> 5;
    for (int64_t c = ((int64_t)blockIdx.x * kPoolThreads + threadIdx.x) >> 5; c < chunks; c += nwarps) {
        const int64_t o = c * 32 + lane;
        uint32_t nib = 0;
        if (o < a.n_out) {
            uint32_t q, ow, nc, oh;
            a.div_wo.divmod((uint32_t)o, q, ow);
            a.div_ho.divmod(q, nc, oh);
            const int h0 = (int)oh * a.sh - a.ph, w0 = (int)ow * a.sw - a.pw;
            const float *plane = y + (int64_t)nc * a.H * a.W;
            float best = -CUDART_INF_F;
            int bi = -1;
            for (int dy = 0; dy < kh; ++dy) {
                const int ih = h0 + dy;
                if (ih < 0 || ih >= a.H) continue;
                for (int dx = 0; dx < kw; ++dx) {
                    const int iw = w0 + dx;
                    if (iw < 0 || iw >= a.W) continue;
                    const float v = ld_ro(plane + ih * a.W + iw);
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
        if ((lane & 7) == 0 && o < a.n_out) arg[o >> 3] = nib;
    }
}

// 2x2 stride 2, no padding, every window fully inside (W even): two float2 row loads per
// output.  A warp handles kFwdU chunks of 32 consecutive outputs per iteration with all
// 2*kFwdU loads issued before any compare (memory-level parallelism).
constexpr int kFwdU = 4;

__global__ void __launch_bounds__(kPoolThreads)
maxpool_fwd_k2s2_kernel(const float *__restrict__ y, PoolArgs a, float *__restrict__ out,
                        uint32_t *__restrict__ arg) {
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

template <bool EVEN_H>
__global__ void __launch_bounds__(kPoolThreads)
pool_bwd_k2s2_pair_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                          const uint32_t *__restrict__ mask, PoolArgs a, float *__restrict__ dx) {
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

cudaError_t launch_maxpool_fwd(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                               int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, cudaStream_t s) {
    const PoolArgs a = make_args(N, C, H, W, p, Ho, Wo);
    const unsigned grid = grid_for(a.n_out, kPoolThreads, 8);
    if (is_k2s2_exact(p, H, W, Ho, Wo) && W % 4 == 0) {
        const unsigned g2 = grid_for(ceil_div(a.n_out / 2, 32 * kPairU), kPoolThreads / 32, 8);
        if (H == 2 * Ho) maxpool_fwd_k2s2_pair_kernel<true><<<g2, kPoolThreads, 0, s>>>(y, a, out, argmax);
        else maxpool_fwd_k2s2_pair_kernel<false><<<g2, kPoolThreads, 0, s>>>(y, a, out, argmax);
    } else if (is_k2s2_exact(p, H, W, Ho, Wo))
        maxpool_fwd_k2s2_kernel<<<grid_for(ceil_div(a.n_out, kFwdU), kPoolThreads, 8), kPoolThreads, 0, s>>>(y, a, out, argmax);
    else if (p.kh == 3 && p.kw == 3)
        maxpool_fwd_kernel<3, 3><<<grid, kPoolThreads, 0, s>>>(y, a, out, argmax);
    else if (p.kh == 2 && p.kw == 2)
        maxpool_fwd_kernel<2, 2><<<grid, kPoolThreads, 0, s>>>(y, a, out, argmax);
    else
        maxpool_fwd_kernel<0, 0><<<grid, kPoolThreads, 0, s>>>(y, a, out, argmax);
    return cudaPeekAtLastError();
}

cudaError_t launch_pool_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                            int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo, float *dx,
                            cudaStream_t s) {
    const PoolArgs a = make_args(N, C, H, W, p, Ho, Wo);
    if (is_k2s2_exact(p, H, W, Ho, Wo) && W % 4 == 0) {
        const unsigned g2 = grid_for(ceil_div(a.n_out / 2, kPairU), kPoolThreads, 8);
        if (H == 2 * Ho) pool_bwd_k2s2_pair_kernel<true><<<g2, kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
        else pool_bwd_k2s2_pair_kernel<false><<<g2, kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
    } else if (is_k2s2_exact(p, H, W, Ho, Wo)) {
        pool_bwd_k2s2_kernel<<<grid_for(ceil_div(a.n_out, kBwdU), kPoolThreads, 8), kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
    } else {
        const unsigned grid = grid_for(a.n_in, kPoolThreads, 8);
        if (p.kh == 3 && p.kw == 3 && p.sh == 2 && p.sw == 2)
            pool_bwd_kernel<3, 3, 2, 2><<<grid, kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
        else if (p.kh == 3 && p.kw == 3 && p.sh == 1 && p.sw == 1)
            pool_bwd_kernel<3, 3, 1, 1><<<grid, kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
        else
            pool_bwd_kernel<0, 0, 0, 0><<<grid, kPoolThreads, 0, s>>>(dout, argmax, mask, a, dx);
    }
    return cudaPeekAtLastError();
}

}  // namespace gist
