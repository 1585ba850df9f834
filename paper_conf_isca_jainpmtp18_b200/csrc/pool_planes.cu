// pool_planes.cu — a3 for 3x3 / stride 1 / pad 1 windows (GoogLeNet's in-module pools),
// PAPER.md P:74 §III-A, P:151-P:156 §IV-A.
//
// Every input element is covered by up to 9 windows, so the gather reads each dY and argmax
// nibble ~9 times: through L1 that is LSU-bound (10% of HBM).  Here a persistent CTA (one per
// SM, 1024 threads) streams GROUPS OF WHOLE PLANES — one contiguous range of dY, of the argmax
// words and of the mask words — through a kPStages-deep shared-memory ring filled by 1-D TMA
// bulk copies (cp.async.bulk), and a thread per input element gathers from shared memory: the
// windows whose argmax is this element, in ascending output order (R6: +0.0f first), selected
// by the ReLU mask bit (R7), one coalesced fp32 store.
// (A forward and a stride-2 backward built the same way measured no faster than the L1 kernels
// in pool.cu — they are issue-bound at ~3 warp-instructions per output — see DESIGN.md §6.)
#include <math_constants.h>

#include <algorithm>

#include "common.cuh"
#include "kernels.h"
#include "tma.cuh"

namespace gist {

namespace {

constexpr int kPT = 1024;                // threads per CTA (one CTA per SM)
constexpr int kPStages = 3;              // ring depth
constexpr int kPStageBytes = 64 * 1024;  // bytes per ring stage
constexpr int kChunkBytes = 16 * 1024;   // one stage range as several bulk copies
constexpr int kPStageFloats = kPStageBytes / 4;

struct PlaneArgs {
    int32_t H, W, Ho, Wo, ph, pw;
    int32_t HW, HoWo;
    int64_t NC, n_in, n_out;
    int32_t G;        // planes per group
    int64_t groups;
    int32_t a_off, m_off;  // backward stage layout (floats): dY at 0, argmax words, mask words
    FastDiv div_hw, div_w;
};

// Stage the contiguous float range [lo, hi) of src: TMA for the 16-B aligned body starting at
// base = lo & ~3 (the ragged <= 3 floats at the end are loaded by the consumers).  Returns the
// bytes the TMA delivers.
__device__ __forceinline__ uint32_t stage_bytes(int64_t lo, int64_t hi) {
    const int64_t base = lo & ~3ll;
    return (uint32_t)(((hi - base) & ~3ll) * 4);
}

// One stage range as several bulk copies (the TMA engine streams each copy in order; smaller
// copies keep more of them in flight).
__device__ __forceinline__ void tma_load_chunks(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    for (uint32_t off = 0; off < bytes; off += kChunkBytes)
        tma_load_1d(static_cast<char *>(dst) + off, static_cast<const char *>(src) + off,
                    bytes - off < kChunkBytes ? bytes - off : kChunkBytes, bar);
}

__global__ void __launch_bounds__(kPT, 1)
pool3s1_planes_bwd_kernel(const float *__restrict__ dout, const uint32_t *__restrict__ arg,
                        const uint32_t *__restrict__ mask, PlaneArgs a, float *__restrict__ dx) {
    pdl_enter();
    extern __shared__ __align__(128) unsigned char smem[];
    float *ring = reinterpret_cast<float *>(smem);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + kPStages * kPStageBytes);
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < kPStages; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t mine = a.groups > blockIdx.x ? (a.groups - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    const int64_t a_words = (a.n_out + 7) >> 3, m_words = (a.n_in + 31) >> 5;
    struct Ranges {
        int64_t p0, np, o_lo, o_hi, i_lo, i_hi, aw_lo, aw_hi, mw_lo, mw_hi;
    };
    auto ranges = [&](int64_t k) {
        Ranges r;
        r.p0 = (blockIdx.x + k * gridDim.x) * (int64_t)a.G;
        r.np = min((int64_t)a.G, a.NC - r.p0);
        r.o_lo = r.p0 * a.HoWo;
        r.o_hi = (r.p0 + r.np) * a.HoWo;
        r.i_lo = r.p0 * a.HW;
        r.i_hi = (r.p0 + r.np) * a.HW;
        r.aw_lo = r.o_lo >> 3;
        r.aw_hi = min(a_words, (r.o_hi + 7) >> 3);
        r.mw_lo = r.i_lo >> 5;
        r.mw_hi = min(m_words, (r.i_hi + 31) >> 5);
        return r;
    };
    auto issue = [&](int64_t k) {
        const Ranges r = ranges(k);
        const int st = (int)(k % kPStages);
        float *R = ring + (int64_t)st * kPStageFloats;
        const uint32_t bd = stage_bytes(r.o_lo, r.o_hi);
        const uint32_t ba = stage_bytes(r.aw_lo, r.aw_hi);
        const uint32_t bm = mask ? stage_bytes(r.mw_lo, r.mw_hi) : 0u;
        mbar_arrive_expect_tx(&full[st], bd + ba + bm);
        if (bd) tma_load_chunks(R, dout + (r.o_lo & ~3ll), bd, &full[st]);
        if (ba) tma_load_1d(R + a.a_off, arg + (r.aw_lo & ~3ll), ba, &full[st]);
        if (bm) tma_load_1d(R + a.m_off, mask + (r.mw_lo & ~3ll), bm, &full[st]);
    };
    if (tid == 0)
        for (int64_t k = 0; k < kPStages && k < mine; ++k) issue(k);

    for (int64_t k = 0; k < mine; ++k) {
        const int st = (int)(k % kPStages);
        float *R = ring + (int64_t)st * kPStageFloats;
        const Ranges r = ranges(k);
        mbar_wait(&full[st], (uint32_t)(k / kPStages) & 1u);
        // ragged tails (<= 3 elements each) of the three staged ranges
        {
            const int64_t db = r.o_lo & ~3ll, de = db + ((r.o_hi - db) & ~3ll);
            const int64_t ab = r.aw_lo & ~3ll, ae = ab + ((r.aw_hi - ab) & ~3ll);
            const int64_t mb = r.mw_lo & ~3ll, me = mb + ((r.mw_hi - mb) & ~3ll);
            uint32_t *RA = reinterpret_cast<uint32_t *>(R + a.a_off), *RM = reinterpret_cast<uint32_t *>(R + a.m_off);
            bool wrote = false;
            if (tid < r.o_hi - de) R[de - db + tid] = dout[de + tid], wrote = true;
            if (tid >= 4 && tid - 4 < r.aw_hi - ae) RA[ae - ab + tid - 4] = arg[ae + tid - 4], wrote = true;
            if (mask && tid >= 8 && tid - 8 < r.mw_hi - me) RM[me - mb + tid - 8] = mask[me + tid - 8], wrote = true;
            if (wrote) fence_proxy_async_smem();
        }
        __syncthreads();
        const float *D = R + (r.o_lo - (r.o_lo & ~3ll));  // dY, local output index
        // argmax / mask words indexed by (local index + phase) >> 3 / >> 5
        const uint32_t *A = reinterpret_cast<const uint32_t *>(R + a.a_off) + ((r.o_lo >> 3) - (r.aw_lo & ~3ll));
        const uint32_t *M = reinterpret_cast<const uint32_t *>(R + a.m_off) + ((r.i_lo >> 5) - (r.mw_lo & ~3ll));
        const int aph = (int)(r.o_lo & 7), mph = (int)(r.i_lo & 31);
        float *dxg = dx + r.i_lo;
        auto nibble = [&](int ol) { return (A[(ol + aph) >> 3] >> (4 * ((ol + aph) & 7))) & 0xfu; };
        auto maskbit = [&](int il) { return mask == nullptr || ((M[(il + mph) >> 5] >> ((il + mph) & 31)) & 1u); };
        // thread per input element; windows (oh, ow) with oh in [th-2, th], ow in [tw-2, tw]
        // (th = ih + ph), visited in ascending o; the hit nibble is 3*(th-oh) + (tw-ow)
        const int cnt = (int)r.np * a.HW;
        for (int l = tid; l < cnt; l += kPT) {
            float acc = 0.0f;  // R6: +0.0f, then ascending output order
            const bool on = maskbit(l);
            if (on) {
                uint32_t pl, q, ih, iw;
                a.div_hw.divmod((uint32_t)l, pl, q);
                a.div_w.divmod(q, ih, iw);
                const int th = (int)ih + a.ph, tw = (int)iw + a.pw;
                const int ob = (int)pl * a.HoWo;
#pragma unroll
                for (int dh = 2; dh >= 0; --dh) {
                    const int oh = th - dh;  // stride 1
                    if (oh < 0 || oh >= a.Ho) continue;
#pragma unroll
                    for (int dw = 2; dw >= 0; --dw) {
                        const int ow = tw - dw;
                        if (ow < 0 || ow >= a.Wo) continue;
                        const int ol = ob + oh * a.Wo + ow;
                        if (nibble(ol) == (uint32_t)(3 * dh + dw)) acc = acc + D[ol];
                    }
                }
            }
            dxg[l] = on ? acc : 0.0f;
        }
        __syncthreads();  // stage st consumed
        if (tid == 0 && k + kPStages < mine) issue(k + kPStages);
    }
}

size_t planes_smem() { return (size_t)kPStages * kPStageBytes + 64; }

PlaneArgs plane_args(int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo) {
    PlaneArgs a{};
    a.H = H;
    a.W = W;
    a.Ho = Ho;
    a.Wo = Wo;
    a.ph = p.ph;
    a.pw = p.pw;
    a.HW = H * W;
    a.HoWo = Ho * Wo;
    a.NC = (int64_t)N * C;
    a.n_in = a.NC * a.HW;
    a.n_out = a.NC * a.HoWo;
    a.div_hw = FastDiv::make((uint32_t)a.HW);
    a.div_w = FastDiv::make((uint32_t)W);
    return a;
}

// Planes per group: what one stage holds, but no more than keeps >= 4 groups per CTA.
void choose_groups(PlaneArgs &a, int64_t per_plane_floats) {
    int64_t g = std::max<int64_t>(1, (kPStageFloats - 64) / per_plane_floats);
    const int64_t spread = ceil_div(a.NC, 4 * (int64_t)num_sms());
    g = std::max<int64_t>(1, std::min(g, spread));
    a.G = (int32_t)g;
    a.groups = ceil_div(a.NC, g);
}

}  // namespace

bool pool_planes_ok(const gist_pool2d &p, int32_t H, int32_t W, int32_t Ho, int32_t Wo) {
    if (p.kh != 3 || p.kw != 3 || p.sh != 1 || p.sw != 1 || p.ph > 1 || p.pw > 1) return false;
    // dY, argmax words and mask words of one plane (plus their 16-B phases) fit a stage
    const int64_t HW = (int64_t)H * W, HoWo = (int64_t)Ho * Wo;
    return HoWo + HoWo / 8 + HW / 32 + 64 <= kPStageFloats;
}

cudaError_t launch_pool3s1_planes_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N,
                                      int32_t C, int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo,
                                      float *dx, cudaStream_t s) {
    PlaneArgs a = plane_args(N, C, H, W, p, Ho, Wo);
    // stage floats per plane: dY (HoWo) + argmax words (HoWo/8) + mask words (HW/32), plus
    // the three 16-B phases and word round-ups
    choose_groups(a, (int64_t)a.HoWo + (a.HoWo + 7) / 8 + (mask ? (a.HW + 31) / 32 : 0) + 1);
    const int64_t G = a.G;
    a.a_off = (int32_t)((G * a.HoWo + 8 + 3) & ~3ll);
    a.m_off = (int32_t)((a.a_off + (G * a.HoWo + 7) / 8 + 8 + 3) & ~3ll);
    static PerDeviceAttr attr;
    const cudaError_t ea = attr.ensure(reinterpret_cast<const void *>(pool3s1_planes_bwd_kernel), (int)planes_smem());
    if (ea != cudaSuccess) return ea;
    const unsigned grid = (unsigned)std::min<int64_t>(a.groups, num_sms());
    launch_k(pool3s1_planes_bwd_kernel, grid, kPT, planes_smem(), s, dout, argmax, mask, a, dx);
    return cudaPeekAtLastError();
}

}  // namespace gist
