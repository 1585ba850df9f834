// dpr.cu — a6/a7: Delayed Precision Reduction encode/decode (PAPER.md P:166-P:171 §IV-A).
//
// fp32 -> FP16 (IEEE 1-5-10) / FP10 (1-5-4) / FP8 (1-4-3), 2/3/4 codes per 32-bit word.
// HBM-bound streaming kernels.  Encode: every thread converts whole 16-byte groups (FP16:
// 1 float4 -> 2 words; FP8: 1 float4 -> 1 word; FP10: 3 float4 -> 4 words = one uint4), with
// 8 (FP16/FP8) or 4 (FP10) independent groups in flight per thread.  Decode: FP16/FP8 mirror
// that mapping (both sides of every warp access contiguous); FP10 decodes 128 words per warp
// and transposes the 384 values through shared memory so the float4 stores are coalesced.
//
// FP10/FP8 use branch-free integer rounding on the fp32 bit pattern: adding
// 2^(s-1)-1 + lsb and shifting right by s = 23-M rounds the significand to M bits with ties
// to even, and the carry ripples into the exponent exactly like step 3 of the paper's
// conversion (O6).  Re-biasing, flush-below-min-normal ("we ignore
// denormalized numbers") and saturation ("clamped at maximum/minimum") are one umin and one
// select.  FP16 uses the hardware cvt.rn.f16x2.f32 after a symmetric clamp to +-65504.
#include <cuda_fp16.h>

#include "common.cuh"
#include "kernels.h"

namespace gist {

namespace {

constexpr int kDprThreads = 256;
constexpr int kUnroll = 4;  // groups in flight per thread (FP10: 48 B each)
constexpr int kUnroll4 = 8;  // FP16/FP8: 16-byte groups, so twice as many in flight

template <int E, int M>
__device__ __forceinline__ uint32_t enc_small(float x) {
    constexpr int SH = 23 - M;
    constexpr int BIAS = (1 << (E - 1)) - 1;
    constexpr uint32_t ADJ = (uint32_t)(127 - BIAS) << M;  // fp32 -> target exponent re-bias
    constexpr uint32_t MAXC = (((1u << E) - 1u) << M) | ((1u << M) - 1u);
    constexpr uint32_t LO = ADJ + (1u << M);  // smallest rounded pattern with exponent >= 1
    const uint32_t u = __float_as_uint(x);
    const uint32_t a = u & 0x7fffffffu;
    const uint32_t r = (a + ((1u << (SH - 1)) - 1u) + ((a >> SH) & 1u)) >> SH;  // RNE, Inf/NaN huge
    uint32_t c = min(r, MAXC + ADJ) - ADJ;  // saturate (Inf/NaN included)
    c = (r >= LO) ? c : 0u;                 // flush-to-zero below min normal (and zeros)
    return c | ((u >> 31) << (E + M));
}

template <int E, int M>
__device__ __forceinline__ float dec_small(uint32_t c) {
    constexpr int BIAS = (1 << (E - 1)) - 1;
    const uint32_t mag = c & ((1u << (E + M)) - 1u);
    uint32_t b = (mag << (23 - M)) + ((uint32_t)(127 - BIAS) << 23);
    b = (mag >> M) ? b : 0u;  // exponent field 0 encodes zero (R14)
    return __uint_as_float(b | (((c >> (E + M)) & 1u) << 31));
}

// Two fp32 -> two IEEE halves packed low|high<<16.
__device__ __forceinline__ uint32_t enc_half2(float a, float b) {
    const float ca = fminf(fmaxf(a, -65504.0f), 65504.0f);
    const float cb = fminf(fmaxf(b, -65504.0f), 65504.0f);
    __half2 h = __floats2half2_rn(ca, cb);  // cvt.rn.f16x2.f32: IEEE RNE, subnormals kept
    uint32_t w = *reinterpret_cast<uint32_t *>(&h);
    if (a != a) w = (w & 0xffff0000u) | 0x7e00u | ((__float_as_uint(a) >> 16) & 0x8000u);
    if (b != b) w = (w & 0x0000ffffu) | 0x7e000000u | (__float_as_uint(b) & 0x80000000u);
    return w;
}

__device__ __forceinline__ float dec_half(uint32_t h) {
    if ((h & 0x7c00u) == 0x7c00u && (h & 0x3ffu))  // NaN: IEEE widening keeps the payload
        return __uint_as_float(((h & 0x8000u) << 16) | 0x7f800000u | ((h & 0x3ffu) << 13));
    return __half2float(__ushort_as_half((unsigned short)h));  // exact, subnormals included
}

template <int BITS>
struct Fmt;
template <>
struct Fmt<16> {
    static constexpr int K = 2;
};
template <>
struct Fmt<10> {
    static constexpr int K = 3;
};
template <>
struct Fmt<8> {
    static constexpr int K = 4;
};

template <int BITS>
__device__ __forceinline__ uint32_t code(float x) {
    if constexpr (BITS == 10) return enc_small<5, 4>(x);
    else return enc_small<4, 3>(x);
}

template <int BITS>
__device__ __forceinline__ float value(uint32_t c) {
    if constexpr (BITS == 16) return dec_half(c);
    else if constexpr (BITS == 10) return dec_small<5, 4>(c);
    else return dec_small<4, 3>(c);
}

// Scalar encode of word w (tail path), zero-filled unused fields.
template <int BITS>
__device__ uint32_t encode_word_scalar(const float *x, int64_t n, int64_t w) {
    constexpr int K = Fmt<BITS>::K;
    uint32_t word = 0;
    for (int j = 0; j < K; ++j) {
        int64_t i = w * K + j;
        if (i < n) {
            uint32_t c;
            if constexpr (BITS == 16) c = enc_half2(x[i], 0.0f) & 0xffffu;
            else c = code<BITS>(x[i]);
            word |= c << (BITS * j);
        }
    }
    return word;
}

// Group = 16 input bytes per step for FP16/FP8 (1 float4), 48 for FP10 (3 float4).
// One map, by thread `tid` of `nthreads` (the many-map kernels rotate tid per map so that small
// maps land on different threads).
template <int BITS>
__device__ __forceinline__ void dpr_encode_body(const float *__restrict__ x, int64_t n, uint32_t *__restrict__ packed,
                                                int64_t tid, int64_t nthreads) {
    constexpr int K = Fmt<BITS>::K;
    constexpr int GF = (BITS == 10) ? 12 : 4;  // floats per group
    const int64_t groups = n / GF;
    const float4 *x4 = reinterpret_cast<const float4 *>(x);
    constexpr int U = (BITS == 10) ? kUnroll : kUnroll4;

    for (int64_t g0 = tid; g0 < groups; g0 += nthreads * U) {
        float4 v[U][GF / 4];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t g = g0 + (int64_t)u * nthreads;
            if (g < groups) {
#pragma unroll
                for (int q = 0; q < GF / 4; ++q) v[u][q] = ld_stream_f4(x4 + g * (GF / 4) + q);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t g = g0 + (int64_t)u * nthreads;
            if (g >= groups) break;
            if constexpr (BITS == 16) {
                uint2 o;
                o.x = enc_half2(v[u][0].x, v[u][0].y);
                o.y = enc_half2(v[u][0].z, v[u][0].w);
                reinterpret_cast<uint2 *>(packed)[g] = o;
            } else if constexpr (BITS == 8) {
                const float4 a = v[u][0];
                packed[g] = code<8>(a.x) | (code<8>(a.y) << 8) | (code<8>(a.z) << 16) | (code<8>(a.w) << 24);
            } else {
                const float f[12] = {v[u][0].x, v[u][0].y, v[u][0].z, v[u][0].w, v[u][1].x, v[u][1].y,
                                     v[u][1].z, v[u][1].w, v[u][2].x, v[u][2].y, v[u][2].z, v[u][2].w};
                uint4 o;
                o.x = code<10>(f[0]) | (code<10>(f[1]) << 10) | (code<10>(f[2]) << 20);
                o.y = code<10>(f[3]) | (code<10>(f[4]) << 10) | (code<10>(f[5]) << 20);
                o.z = code<10>(f[6]) | (code<10>(f[7]) << 10) | (code<10>(f[8]) << 20);
                o.w = code<10>(f[9]) | (code<10>(f[10]) << 10) | (code<10>(f[11]) << 20);
                reinterpret_cast<uint4 *>(packed)[g] = o;
            }
        }
    }
    // Tail: the words not produced by whole groups (fewer than GF/K + 1 of them).
    if (tid == nthreads - 1) {
        const int64_t first = groups * GF / K;
        const int64_t words = (n + K - 1) / K;
        for (int64_t w = first; w < words; ++w) packed[w] = encode_word_scalar<BITS>(x, n, w);
    }
}

template <int BITS>
__global__ void __launch_bounds__(kDprThreads)
dpr_encode_kernel(const float *__restrict__ x, int64_t n, uint32_t *__restrict__ packed, const int64_t *__restrict__ n_dev) {
    pdl_enter();
    if (n_dev) n = min(n, *n_dev);  // count known only on the device (DPR over SSDC values)
    dpr_encode_body<BITS>(x, n, packed, (int64_t)blockIdx.x * kDprThreads + threadIdx.x,
                          (int64_t)gridDim.x * kDprThreads);
}

template <int BITS>
__device__ __forceinline__ void dpr_decode_body(const uint32_t *__restrict__ packed, int64_t n, float *__restrict__ x,
                                                int64_t tid, int64_t nthreads) {
    constexpr int K = Fmt<BITS>::K;
    constexpr uint32_t FIELD = (1u << BITS) - 1u;
    float4 *x4 = reinterpret_cast<float4 *>(x);
    if constexpr (BITS != 10) {
        // FP16: one uint2 (2 words) -> one float4; FP8: one word -> one float4.  Both sides of
        // every warp access are contiguous.
        constexpr int GW = 4 / K;  // words per float4 group: 2 / 1
        const int64_t groups = n / 4;
        for (int64_t g0 = tid; g0 < groups; g0 += nthreads * kUnroll4) {
            uint32_t w[kUnroll4][GW];
#pragma unroll
            for (int u = 0; u < kUnroll4; ++u) {
                const int64_t g = g0 + (int64_t)u * nthreads;
                if (g < groups) {
                    if constexpr (GW == 1) {
                        w[u][0] = ld_stream_u32(packed + g);
                    } else {
                        const uint2 t = ld_stream_u2(reinterpret_cast<const uint2 *>(packed) + g);
                        w[u][0] = t.x;
                        w[u][1] = t.y;
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < kUnroll4; ++u) {
                const int64_t g = g0 + (int64_t)u * nthreads;
                if (g >= groups) break;
                float f[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) f[i] = value<BITS>((w[u][i / K] >> (BITS * (i % K))) & FIELD);
                x4[g] = make_float4(f[0], f[1], f[2], f[3]);
            }
        }
        if (tid == nthreads - 1)
            for (int64_t i = groups * 4; i < n; ++i) x[i] = value<BITS>((packed[i / K] >> (BITS * (i % K))) & FIELD);
    } else {
        // FP10: a warp decodes 128 consecutive words (384 values): lane l loads words
        // [4l, 4l+4) as one uint4, writes its 12 values to shared memory, and the warp stores
        // the 384 values back as 96 contiguous float4 (3 coalesced waves), instead of 48-byte
        // strided stores that leave every write sector half-filled.
        __shared__ __align__(16) float s_buf[kDprThreads / 32][384];
        const int lane = threadIdx.x & 31;
        float *buf = s_buf[threadIdx.x >> 5];
        const int64_t chunks = n / 384;
        const int64_t gwarp = tid >> 5, nwarps = nthreads >> 5;
        for (int64_t c = gwarp; c < chunks; c += nwarps) {
            const uint4 t = ld_stream_u4(reinterpret_cast<const uint4 *>(packed + c * 128) + lane);
            const uint32_t w[4] = {t.x, t.y, t.z, t.w};
            float f[12];
#pragma unroll
            for (int i = 0; i < 12; ++i) f[i] = value<10>((w[i / 3] >> (10 * (i % 3))) & FIELD);
            float4 *b4 = reinterpret_cast<float4 *>(buf);
#pragma unroll
            for (int q = 0; q < 3; ++q) b4[3 * lane + q] = make_float4(f[4 * q], f[4 * q + 1], f[4 * q + 2], f[4 * q + 3]);
            __syncwarp();
#pragma unroll
            for (int q = 0; q < 3; ++q) x4[c * 96 + 32 * q + lane] = b4[32 * q + lane];
            __syncwarp();
        }
        // the < 384 values past the last whole chunk: one per thread (not a serial loop)
        for (int64_t i = chunks * 384 + tid; i < n; i += nthreads) x[i] = value<10>((packed[i / 3] >> (10 * (i % 3))) & FIELD);
    }
}

template <int BITS>
__global__ void __launch_bounds__(kDprThreads)
dpr_decode_kernel(const uint32_t *__restrict__ packed, int64_t n, float *__restrict__ x, const int64_t *__restrict__ n_dev) {
    pdl_enter();
    if (n_dev) n = min(n, *n_dev);  // count known only on the device (DPR over SSDC values)
    dpr_decode_body<BITS>(packed, n, x, (int64_t)blockIdx.x * kDprThreads + threadIdx.x,
                          (int64_t)gridDim.x * kDprThreads);
}

// Many maps in one launch ("these conversions can happen in parallel"): the grid walks the
// maps in order, each with the single-map loop; map k's thread index is rotated by the groups of
// the maps before it, so consecutive small maps run on different threads (and SMs) at once.
constexpr int kMaxDprJobs = 96;
struct DprJob {
    const void *in;
    void *out;
    int64_t n;
};
struct DprJobs {
    DprJob j[kMaxDprJobs];
    int32_t count;
};
static_assert(sizeof(DprJobs) + 16 <= 4096, "kernel parameters must fit 4 KB");

template <int BITS, bool ENCODE>
__global__ void __launch_bounds__(kDprThreads)
dpr_many_kernel(const __grid_constant__ DprJobs J) {
    pdl_enter();
    const int64_t nthreads = (int64_t)gridDim.x * kDprThreads;
    const int64_t me = (int64_t)blockIdx.x * kDprThreads + threadIdx.x;
    // FP10 decode is warp-based (384-value chunks): rotate by whole warps
    constexpr bool WARPS = !ENCODE && BITS == 10;
    constexpr int GF = ENCODE ? ((BITS == 10) ? 12 : 4) : (BITS == 10 ? 384 : 4);
    int64_t rot = 0;
    for (int k = 0; k < J.count; ++k) {
        const DprJob &jb = J.j[k];
        int64_t tid = WARPS ? (me + 32 * rot) % nthreads : (me + rot) % nthreads;
        if (ENCODE)
            dpr_encode_body<BITS>(reinterpret_cast<const float *>(jb.in), jb.n, reinterpret_cast<uint32_t *>(jb.out),
                                  tid, nthreads);
        else
            dpr_decode_body<BITS>(reinterpret_cast<const uint32_t *>(jb.in), jb.n, reinterpret_cast<float *>(jb.out),
                                  tid, nthreads);
        rot += jb.n / GF + 1;
    }
}

#ifndef GIST_DPR_CTAS
#define GIST_DPR_CTAS 8  // grid cap, CTAs per SM
#endif
#ifndef GIST_DPR_MANY_CTAS
#define GIST_DPR_MANY_CTAS 4  // many-map grid cap (C3's four DPR sites: 8 -> 4 CTAs/SM took a6 57% -> 62%, a7 64% -> 73%)
#endif
template <int BITS>
int64_t dpr_blocks(int64_t n, int per_sm = GIST_DPR_CTAS) {
    // one group per thread until the grid cap is reached (the unrolled loops then take several
    // per thread): small maps get every SM instead of 1/U of the threads
    constexpr int GF = (BITS == 10) ? 12 : 4;
    int64_t groups = n / GF + 1;
    int64_t blocks = ceil_div(groups, kDprThreads);
    const int64_t cap = (int64_t)num_sms() * per_sm;
    return blocks > cap ? cap : blocks;
}

}  // namespace

cudaError_t launch_dpr_encode(const float *x, int64_t n, int bits, uint32_t *packed, cudaStream_t s,
                              const int64_t *n_dev) {
    switch (bits) {
        case 16: launch_k(dpr_encode_kernel<16>, (unsigned)dpr_blocks<16>(n), kDprThreads, 0, s, x, n, packed, n_dev); break;
        case 10: launch_k(dpr_encode_kernel<10>, (unsigned)dpr_blocks<10>(n), kDprThreads, 0, s, x, n, packed, n_dev); break;
        case 8: launch_k(dpr_encode_kernel<8>, (unsigned)dpr_blocks<8>(n), kDprThreads, 0, s, x, n, packed, n_dev); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaPeekAtLastError();
}

cudaError_t launch_dpr_decode(const uint32_t *packed, int64_t n, int bits, float *x, cudaStream_t s,
                              const int64_t *n_dev) {
    switch (bits) {
        case 16: launch_k(dpr_decode_kernel<16>, (unsigned)dpr_blocks<16>(n), kDprThreads, 0, s, packed, n, x, n_dev); break;
        case 10: launch_k(dpr_decode_kernel<10>, (unsigned)dpr_blocks<10>(n), kDprThreads, 0, s, packed, n, x, n_dev); break;
        case 8: launch_k(dpr_decode_kernel<8>, (unsigned)dpr_blocks<8>(n), kDprThreads, 0, s, packed, n, x, n_dev); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaPeekAtLastError();
}

cudaError_t launch_dpr_many(const gist_dpr_job *jobs, int32_t count, int bits, bool encode, cudaStream_t s,
                            int *launches) {
    *launches = 0;
    for (int32_t k0 = 0; k0 < count; k0 += kMaxDprJobs) {
        DprJobs J{};
        int64_t n_max = 0;
        for (int32_t k = k0; k < count && k < k0 + kMaxDprJobs; ++k) {
            DprJob &e = J.j[J.count++];
            e.in = encode ? (const void *)jobs[k].x : (const void *)jobs[k].packed;
            e.out = encode ? (void *)jobs[k].packed : (void *)jobs[k].x;
            e.n = jobs[k].n;
            n_max = n_max > jobs[k].n ? n_max : jobs[k].n;
        }
        int64_t n_sum = 0;
        for (int k = 0; k < J.count; ++k) n_sum += J.j[k].n;
        unsigned grid = 1;
        switch (bits) {
            case 16: grid = (unsigned)dpr_blocks<16>(n_sum, GIST_DPR_MANY_CTAS); break;
            case 10: grid = (unsigned)dpr_blocks<10>(n_sum, GIST_DPR_MANY_CTAS); break;
            case 8: grid = (unsigned)dpr_blocks<8>(n_sum, GIST_DPR_MANY_CTAS); break;
            default: return cudaErrorInvalidValue;
        }
        (void)n_max;
#define GIST_DPR_MANY(B) \
    (encode ? launch_k(dpr_many_kernel<B, true>, grid, kDprThreads, 0, s, J) \
            : launch_k(dpr_many_kernel<B, false>, grid, kDprThreads, 0, s, J))
        switch (bits) {
            case 16: GIST_DPR_MANY(16); break;
            case 10: GIST_DPR_MANY(10); break;
            case 8: GIST_DPR_MANY(8); break;
        }
#undef GIST_DPR_MANY
        const cudaError_t e = cudaPeekAtLastError();
        if (e != cudaSuccess) return e;
        ++*launches;
    }
    return cudaSuccess;
}

}  // namespace gist
