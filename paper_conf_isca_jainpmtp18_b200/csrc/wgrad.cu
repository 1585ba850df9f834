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

constexpr int kCiBlk = 16;              // input channels per CTA tile
constexpr int kTaps = 9;                // 3x3 window
constexpr int kN = kCiBlk * kTaps;      // 144 GEMM columns: n = tap * 16 + ci
constexpr int kM = 128;                 // output channels per CTA tile (UMMA M)
constexpr int kKs = 32;                 // K per pipeline stage = one 128-byte swizzle row of fp32
constexpr int kProdWarps = 8;
constexpr int kProdThreads = 32 * kProdWarps;
constexpr int kEpiWarps = 8;                 // two per TMEM lane quarter (taps 0-4 / 5-8)
constexpr int kEpi0 = 2 + kProdWarps;        // first epilogue warp
// warp 0: TMA + TMEM owner, warp 1: MMA, 2..9: producers, 10..17: accumulator drain (epilogue)
constexpr int kThreads = 32 * (kEpi0 + kEpiWarps);
constexpr int kTmemCols = 512;               // two accumulators (K-tile t uses columns 256 (t % 2) + n)
constexpr int kAccStride = 256;
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
    FastDiv div_w;
};

template <int PASSES, int STAGES>
struct __align__(1024) WgSmem {
    float a[STAGES][kM * kKs];                      // dY tiles (TMA, 128-B swizzle): A_hi as loaded
    float alo[PASSES == 3 ? STAGES : 1][PASSES == 3 ? kM * kKs : 256];  // A - tf32(A) (3xTF32 only; 1 KB keeps bhi 1024-aligned)
    float bhi[STAGES][kN * kKs];                    // im2col(X) tiles, same layout
    float blo[PASSES == 3 ? STAGES : 1][PASSES == 3 ? kN * kKs : 256];
    uint64_t a_full[STAGES], b_full[STAGES], empty[STAGES], acc_full[2], acc_empty[2];
    uint32_t tmem_base;
};
// every operand tile must start on a 1024-byte boundary (the 128-byte swizzle atom)
static_assert(sizeof(float) * kM * kKs % 1024 == 0 && sizeof(float) * kN * kKs % 1024 == 0, "tile sizes");

template <int PASSES, int STAGES>
__global__ void __launch_bounds__(kThreads, 1)
wgrad_ssdc_kernel(const __grid_constant__ CUtensorMap tmap_dy, const WgArgs a) {
    using Smem = WgSmem<PASSES, STAGES>;
    extern __shared__ unsigned char smem_raw[];
    // the 128-byte swizzle repeats every 1024 bytes: align the tiles to that
    const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
    Smem &S = *reinterpret_cast<Smem *>(smem_raw + pad);
    float *slab = reinterpret_cast<float *>(smem_raw + pad + sizeof(Smem));
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    const int nb = blockIdx.x % a.n_blocks;
    const int mb = (blockIdx.x / a.n_blocks) % a.m_blocks;
    const int sp = blockIdx.x / (a.n_blocks * a.m_blocks);
    // this CTA's K-tiles: whole chunks [u0, u1) (a chunk's partial has exactly one writer)
    const int64_t u0 = (int64_t)sp * a.units / a.splits, u1 = (int64_t)(sp + 1) * a.units / a.splits;
    const int64_t t0 = u0 * a.chunk, t1 = min(a.T, u1 * (int64_t)a.chunk);
    const int co0 = mb * kM, ci0 = nb * kCiBlk;
    const int64_t nst = (t1 - t0) * a.spt;  // pipeline stages of this CTA
    const int RW = a.R * a.W, SW = a.W + 2, SR = a.R + 2;

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&S.a_full[s], 1);
            mbar_init(&S.b_full[s], kProdWarps);
            mbar_init(&S.empty[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&S.acc_full[b], 1);
            mbar_init(&S.acc_empty[b], kEpiWarps);
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
            for (int64_t g = 0; g < nst; ++g) {
                const int st = (int)(g % STAGES);
                if (g >= STAGES) mbar_wait(&S.empty[st], (uint32_t)((g / STAGES) - 1) & 1u);
                const int64_t t = t0 + g / a.spt;
                const int j = (int)(g % a.spt);
                const int n = (int)(t / a.ktiles), ty = (int)(t % a.ktiles);
                mbar_arrive_expect_tx(&S.a_full[st], kM * kKs * 4);
                tma_load_2d(S.a[st], &tmap_dy, ty * RW + j * kKs, n * a.Co + co0, &S.a_full[st]);
            }
        }
    } else if (warp == 1) {
        // ---- MMA issuer (one thread)
        if (lane == 0) {
            // Each accumulation period (`pp` per K-tile, a run of consecutive stages) accumulates into
            // its own TMEM buffer (period % 2), drained by the epilogue warps into fp32 registers: the
            // tensor core's own accumulation then spans at most ceil(spt/pp) stages, which keeps its
            // rounding error near fp32's (f4).
            int64_t gp = 0;  // accumulation periods started so far
            for (int64_t g = 0; g < nst; ++g) {
                const int st = (int)(g % STAGES);
                const uint32_t par = (uint32_t)(g / STAGES) & 1u;
                const int j = (int)(g % a.spt);
                const int q = j * a.pp / a.spt;
                const bool first = j == 0 || (j - 1) * a.pp / a.spt != q;
                const bool last = j == a.spt - 1 || (j + 1) * a.pp / a.spt != q;
                const int b = (int)(gp & 1);
                if (first && gp >= 2) mbar_wait(&S.acc_empty[b], (uint32_t)((gp / 2) - 1) & 1u);
                mbar_wait(&S.a_full[st], par);
                mbar_wait(&S.b_full[st], par);
                tc_fence_after();
                const uint32_t d = tmem + (uint32_t)(b * kAccStride);
                const uint32_t ab = smem_u32(S.a[st]), bb = smem_u32(S.bhi[st]);
#pragma unroll
                for (int kk = 0; kk < kKs / 8; ++kk) {  // K = 8 tf32 (32 bytes) per instruction
                    const uint64_t da = umma_desc_sw128(ab + 32 * kk), db = umma_desc_sw128(bb + 32 * kk);
                    umma_tf32(d, da, db, kIdesc, (!first || kk != 0) ? 1u : 0u);
                    if constexpr (PASSES == 3) {
                        umma_tf32(d, da, umma_desc_sw128(smem_u32(S.blo[st]) + 32 * kk), kIdesc, 1u);
                        umma_tf32(d, umma_desc_sw128(smem_u32(S.alo[st]) + 32 * kk), db, kIdesc, 1u);
                    }
                }
                umma_commit(&S.empty[st]);  // the stage's smem is free once these MMAs complete
                if (last) {
                    umma_commit(&S.acc_full[b]);
                    ++gp;
                }
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
            mbar_wait(&S.acc_full[b], (uint32_t)(gp / 2) & 1u);
            tc_fence_after();
#pragma unroll
            for (int i = 0; i < 5; ++i) {
                const int tap = 5 * half + i;
                if (tap < kTaps) {
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
    } else {
        // ---- producers: decode X (SSDC) into the slab, build B (im2col, hi/lo) and A_lo
        const int p = threadIdx.x - 64;
        const int wp = warp - 2;
        const int ci_b = p >> 4, ch = (p >> 1) & 7, half = p & 1;  // B chunk owned by this thread
        for (int64_t t = t0; t < t1; ++t) {
            const int n = (int)(t / a.ktiles), ty = (int)(t % a.ktiles);
            const int oh0 = ty * a.R;
            named_bar(1, kProdThreads);  // every producer is done reading the previous slab
            {
                float4 *s4 = reinterpret_cast<float4 *>(slab);
                const int n4 = kCiBlk * SR * SW / 4;
                for (int i = p; i < n4; i += kProdThreads) s4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
            named_bar(1, kProdThreads);
            // each warp decodes two channels: the CSR rows covering input rows [oh0-1, oh0+R]
            for (int cc = 0; cc < 2; ++cc) {
                const int ci = 2 * wp + cc;
                const int64_t plane0 = ((int64_t)n * a.Ci + ci0 + ci) * a.H * a.W;
                const int ih_lo = max(0, oh0 - 1), ih_hi = min(a.H, oh0 + a.R + 1);
                const int64_t F0 = plane0 + (int64_t)ih_lo * a.W, F1 = plane0 + (int64_t)ih_hi * a.W;
                if (F1 <= F0) continue;
                float *sl = slab + (size_t)ci * SR * SW;
                for (int64_t r = F0 >> 8; r <= (F1 - 1) >> 8; ++r) {
                    const int32_t e0 = r ? a.row_end[r - 1] : 0, e1 = a.row_end[r];
                    for (int32_t k = e0 + lane; k < e1; k += 32) {
                        const int64_t flat = 256 * r + a.col[k];
                        if (flat >= F0 && flat < F1) {
                            uint32_t ih, iw;
                            a.div_w.divmod((uint32_t)(flat - plane0), ih, iw);
                            sl[((int)ih - oh0 + 1) * SW + (int)iw + 1] = a.val[k];
                        }
                    }
                }
            }
            named_bar(1, kProdThreads);
            for (int j = 0; j < a.spt; ++j) {
                const int64_t g = (t - t0) * a.spt + j;
                const int st = (int)(g % STAGES);
                if (g >= STAGES) mbar_wait(&S.empty[st], (uint32_t)((g / STAGES) - 1) & 1u);
                // B rows (tap, ci_b), chunk ch = output positions pos .. pos+3 of the K-tile (they may
                // straddle an output row when W % 4 != 0); slab offset of each for tap (0, 0)
                const int pos = j * kKs + 4 * ch;
                uint32_t ohr = 0, ow = 0;
                a.div_w.divmod((uint32_t)pos, ohr, ow);
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
                unsigned char *bh = reinterpret_cast<unsigned char *>(S.bhi[st]);
                unsigned char *bl = reinterpret_cast<unsigned char *>(S.blo[PASSES == 3 ? st : 0]);
#pragma unroll
                for (int i = 0; i < 5; ++i) {
                    const int tap = half ? 5 + i : i;
                    if (tap >= kTaps) break;
                    const int kh = tap / 3, kw = tap % 3;
                    float v[4];
#pragma unroll
                    for (int e = 0; e < 4; ++e) v[e] = ok[e] ? slab[off[e] + kh * SW + kw] : 0.0f;
                    const uint32_t off = sw128_offset((uint32_t)(tap * kCiBlk + ci_b), (uint32_t)ch);
                    if constexpr (PASSES == 3) {
                        float hi[4], lo[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            hi[e] = to_tf32(v[e]);
                            lo[e] = v[e] - hi[e];
                        }
                        *reinterpret_cast<float4 *>(bh + off) = make_float4(hi[0], hi[1], hi[2], hi[3]);
                        *reinterpret_cast<float4 *>(bl + off) = make_float4(lo[0], lo[1], lo[2], lo[3]);
                    } else {
                        *reinterpret_cast<float4 *>(bh + off) = make_float4(v[0], v[1], v[2], v[3]);
                    }
                }
                if constexpr (PASSES == 3) {
                    // A_hi = tf32_rn(A) written back in place, A_lo = A - A_hi (exact in fp32); the layouts
                    // of a[] and alo[] are identical, so chunk by chunk
                    mbar_wait(&S.a_full[st], (uint32_t)(g / STAGES) & 1u);
                    float4 *ar = reinterpret_cast<float4 *>(S.a[st]);
                    float4 *al = reinterpret_cast<float4 *>(S.alo[st]);
#pragma unroll
                    for (int i = 0; i < kM * kKs / 4 / kProdThreads; ++i) {
                        const float4 x = ar[p + i * kProdThreads];
                        const float4 h = make_float4(to_tf32(x.x), to_tf32(x.y), to_tf32(x.z), to_tf32(x.w));
                        ar[p + i * kProdThreads] = h;
                        al[p + i * kProdThreads] = make_float4(x.x - h.x, x.y - h.y, x.z - h.z, x.w - h.w);
                    }
                }
                fence_proxy_async_smem();  // generic smem writes -> visible to the tensor core (async proxy)
                __syncwarp();
                if (lane == 0) mbar_arrive_1(&S.b_full[st]);
            }
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

template <int PASSES, int STAGES>
size_t wg_smem_bytes(const WgPlan &P, int32_t W) {
    return sizeof(WgSmem<PASSES, STAGES>) + (size_t)kCiBlk * (P.R + 2) * (W + 2) * 4 + 1024;
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

template <int PASSES, int STAGES>
cudaError_t launch_wg(const CUtensorMap &tm, const WgArgs &args, const WgPlan &P, int32_t W, cudaStream_t s) {
    static PerDeviceAttr attr;
    const size_t smem = wg_smem_bytes<PASSES, STAGES>(P, W);
    const cudaError_t ea = attr.ensure(reinterpret_cast<const void *>(wgrad_ssdc_kernel<PASSES, STAGES>), (int)smem);
    if (ea != cudaSuccess) return ea;
    const unsigned grid = (unsigned)((int64_t)P.m_blocks * P.n_blocks * P.splits);
    launch_k(wgrad_ssdc_kernel<PASSES, STAGES>, grid, kThreads, smem, s, tm, args);
    return cudaPeekAtLastError();
}

}  // namespace

size_t wgrad_smem_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes);
constexpr size_t kMaxSmem = 227 * 1024;  // sm_100 opt-in dynamic shared memory per CTA

bool wgrad_shape_ok(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W) {
    // H*W % 4: the dY rows are TMA rows, whose stride must be a multiple of 16 bytes; the decode slab
    // of R+2 rows must fit beside the pipeline stages (odd W > 64 needs R = 4: W <= 252 is not enough)
    if (!(N > 0 && H > 0 && W > 0 && Co % kM == 0 && Ci % kCiBlk == 0 && W <= 252 && (int64_t)H * W % 4 == 0))
        return false;
    return wgrad_smem_bytes(N, Ci, Co, H, W, 3) <= kMaxSmem && wgrad_smem_bytes(N, Ci, Co, H, W, 1) <= kMaxSmem;
}

size_t wgrad_workspace_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W) {
    const WgPlan P = wg_plan(N, Ci, Co, H, W, 3);  // units do not depend on passes
    return (size_t)P.units * Co * Ci * kTaps * 4;
}

size_t wgrad_smem_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes) {
    const WgPlan P = wg_plan(N, Ci, Co, H, W, passes);
    return passes == 3 ? wg_smem_bytes<3, 2>(P, W) : wg_smem_bytes<1, 4>(P, W);
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
    const cudaError_t e = passes == 3 ? launch_wg<3, 2>(tm, args, P, W, s) : launch_wg<1, 4>(tm, args, P, W, s);
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
