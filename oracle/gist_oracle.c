/*
 * oracle/gist_oracle.c — CPU ORACLE for Gist's stash-time encode/decode hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_isca_jainpmtp18_b200/) never links, imports or calls it, and the two
 * share no code, headers, tables or helpers.
 *
 * Plain, slow, obviously-correct scalar C.  Each function follows the passage of the
 * paper (Jain et al., "Gist", ISCA 2018; /root/reference/PAPER.md, cited as P:<line>
 * §<section>) and the reading recorded in DESIGN.md §3 ("readings").  No blocking, no
 * fusion, no reordering beyond what the definition states.  Build with
 *     gcc -O2 -fno-fast-math -ffp-contract=off -shared -fPIC
 * so every float operation is a single IEEE-754 binary32 operation.
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py against
 * library routines (numpy packbits / float16, torch CPU max_pool2d + autograd,
 * torch to_sparse_csr, torch float8_e4m3fn, ml_dtypes), closed forms, brute force and
 * golden values under tests/golden/.  No function is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------------------
 * O1 — Binarize encode.  P:74 §III-A ("dX is set to dY only if corresponding element in
 * Y is positive, else dX is set to 0"), §IV-A, P:154 ("a 1-bit data structure that
 * replaces the ReLU feature map, storing information whether the stashed feature map
 * value was positive").  Reading R1: element i -> word i>>5, bit i&31 (LSB first),
 * tail bits 0.  NaN and -0.0 are "not positive" -> bit 0.
 * ---------------------------------------------------------------------------------- */
int64_t oracle_binarize_words(int64_t n) { return (n + 31) / 32; }

void oracle_binarize_encode(const float *y, int64_t n, uint32_t *mask)
{
    int64_t words = oracle_binarize_words(n);
    for (int64_t w = 0; w < words; ++w) mask[w] = 0u;
    for (int64_t i = 0; i < n; ++i)
        if (y[i] > 0.0f) mask[i >> 5] |= 1u << (i & 31);
}

/* ------------------------------------------------------------------------------------
 * O2 — MaxPool forward + Y->X argmax map.  P:152 §IV-A ("create a mapping from Y to X in
 * the forward pass that keeps track of these locations"), P:154 ("each element is stored
 * in 4 bits (the largest sliding window in our application suite is 3x3)").
 * Readings R2 (window-local index dy*kw+dx, nibble k -> word k>>3 bits 4(k&7)),
 * R3 (first max in row-major scan; NaN counts as max; update iff v > best || isnan(v)),
 * R4 (padding + ceil mode with torch semantics; padded positions never selected).
 * ---------------------------------------------------------------------------------- */
int32_t oracle_pool_out_dim(int32_t in, int32_t k, int32_t s, int32_t p, int32_t ceil_mode)
{
    /* out = floor((in + 2p - k)/s) + 1, or ceil(...) + 1 in ceil mode, and in ceil mode
       the last window must start inside the (left-)padded input: (out-1)*s < in + p.  */
    int32_t span = in + 2 * p - k;
    if (span < 0) return 0;
    int32_t out = ceil_mode ? (span + s - 1) / s + 1 : span / s + 1;
    if (ceil_mode && (out - 1) * s >= in + p) out -= 1;
    return out;
}

int64_t oracle_argmax_words(int64_t n_out) { return (n_out + 7) / 8; }

void oracle_maxpool_fwd_argmax(const float *y, int32_t N, int32_t C, int32_t H, int32_t W,
                               int32_t kh, int32_t kw, int32_t sh, int32_t sw,
                               int32_t ph, int32_t pw, int32_t ceil_mode,
                               float *out, uint32_t *arg)
{
    int32_t Ho = oracle_pool_out_dim(H, kh, sh, ph, ceil_mode);
    int32_t Wo = oracle_pool_out_dim(W, kw, sw, pw, ceil_mode);
    int64_t n_out = (int64_t)N * C * Ho * Wo;
    for (int64_t w = 0; w < oracle_argmax_words(n_out); ++w) arg[w] = 0u;
    int64_t o = 0;
    for (int64_t nc = 0; nc < (int64_t)N * C; ++nc) {
        const float *plane = y + nc * H * W;
        for (int32_t oh = 0; oh < Ho; ++oh) {
            for (int32_t ow = 0; ow < Wo; ++ow, ++o) {
                int32_t h0 = oh * sh - ph, w0 = ow * sw - pw;
                float best = -INFINITY;
                int32_t best_idx = -1;
                for (int32_t dy = 0; dy < kh; ++dy) {
                    for (int32_t dx = 0; dx < kw; ++dx) {
                        int32_t ih = h0 + dy, iw = w0 + dx;
                        if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
                        float v = plane[(int64_t)ih * W + iw];
                        if (best_idx < 0) best_idx = dy * kw + dx; /* first in-bounds */
                        if (v > best || isnan(v)) { best = v; best_idx = dy * kw + dx; }
                    }
                }
                out[o] = best;
                arg[o >> 3] |= (uint32_t)best_idx << (4 * (o & 7));
            }
        }
    }
}

/* ------------------------------------------------------------------------------------
 * O3 — MaxPool + ReLU backward computed from the encodings only.  P:74 (ReLU backward
 * needs only the sign of Y; MaxPool backward "passes on dY to that location of dX in the
 * window, from where the maximum value of X was chosen"), P:152, P:156 ("Pool and ReLU
 * backward pass have been updated to perform computation on the encoded data structures
 * itself").  Textbook max-pool backward: dx starts at +0.0f; for every output o in
 * ascending flat order, dx[argmax position of o] += dY[o] (one fp32 add each; reading
 * R6).  Then ReLU backward is a select (reading R7): dx = bit(mask,i) ? dx : +0.0f.
 * mask == NULL gives the pool-only backward (GoogLeNet in-module pools).
 * ---------------------------------------------------------------------------------- */
void oracle_pool_relu_bwd(const float *dout, const uint32_t *arg, const uint32_t *mask,
                          int32_t N, int32_t C, int32_t H, int32_t W,
                          int32_t kh, int32_t kw, int32_t sh, int32_t sw,
                          int32_t ph, int32_t pw, int32_t ceil_mode, float *dx)
{
    int32_t Ho = oracle_pool_out_dim(H, kh, sh, ph, ceil_mode);
    int32_t Wo = oracle_pool_out_dim(W, kw, sw, pw, ceil_mode);
    int64_t n = (int64_t)N * C * H * W;
    for (int64_t i = 0; i < n; ++i) dx[i] = +0.0f;
    int64_t o = 0;
    for (int64_t nc = 0; nc < (int64_t)N * C; ++nc) {
        for (int32_t oh = 0; oh < Ho; ++oh) {
            for (int32_t ow = 0; ow < Wo; ++ow, ++o) {
                uint32_t a = (arg[o >> 3] >> (4 * (o & 7))) & 0xFu;
                int32_t ih = oh * sh - ph + (int32_t)a / kw;
                int32_t iw = ow * sw - pw + (int32_t)a % kw;
                int64_t i = nc * H * W + (int64_t)ih * W + iw;
                dx[i] = dx[i] + dout[o];
            }
        }
    }
    if (mask)
        for (int64_t i = 0; i < n; ++i)
            if (!((mask[i >> 5] >> (i & 31)) & 1u)) dx[i] = +0.0f;
}

/* ------------------------------------------------------------------------------------
 * O4/O5 — SSDC: Sparse Storage, Dense Compute.  P:158-P:164 §IV-A.  CSR "stores all the
 * non-zero values, along with a meta array that holds the column indices"; the
 * n-d map is collapsed to 2-D and Narrow Value Optimization "reshape[s] the 2D
 * matrix and restrict[s] the number of columns to 256, requiring only 1 byte per column
 * index".  Readings R8 (nonzero = bit pattern != 0, so -0.0 is kept), R9 (row r
 * = elements [256r, 256r+256) of the flattened NCHW map, last row partial), R10 (the
 * "extra meta array" = int32 inclusive row END offsets, rows entries).
 * Returns nnz.  col/val must hold at least nnz entries (n is always enough).
 * ---------------------------------------------------------------------------------- */
int64_t oracle_ssdc_rows(int64_t n) { return (n + 255) / 256; }

int64_t oracle_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val)
{
    int64_t nnz = 0;
    for (int64_t r = 0; r < oracle_ssdc_rows(n); ++r) {
        for (int64_t j = 0; j < 256 && 256 * r + j < n; ++j) {
            float v = x[256 * r + j];
            uint32_t bits;
            memcpy(&bits, &v, 4);
            if (bits != 0u) {
                col[nnz] = (uint8_t)j;
                val[nnz] = v;
                nnz++;
            }
        }
        row_end[r] = (int32_t)nnz;
    }
    return nnz;
}

void oracle_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n,
                        float *x)
{
    for (int64_t i = 0; i < n; ++i) x[i] = +0.0f;
    for (int64_t r = 0; r < oracle_ssdc_rows(n); ++r) {
        int64_t begin = r ? row_end[r - 1] : 0;
        for (int64_t k = begin; k < row_end[r]; ++k) x[256 * r + col[k]] = val[k];
    }
}

/* ------------------------------------------------------------------------------------
 * O6/O7 — DPR: Delayed Precision Reduction.  P:166-P:171 §IV-A: "three smaller
 * representations of 16, 10 and 8 bits, packing 2, 3 and 4 values, respectively, into 4
 * bytes"; FP16 = IEEE half (1-5-10); FP8 = 1-4-3; FP10 = 1-5-4 ("rendering 2-bits
 * useless"); "We ignore denormalized numbers"; "round-to-nearest"; "clamped at
 * maximum/minimum value if the FP32 value is larger/smaller than the range".
 * Readings R13 (bias 2^(E-1)-1), R14 (no Inf/NaN codes in FP10/FP8: every nonzero
 * exponent is normal, exponent 0 means zero), R15 (ties to even), R16 (FP10/FP8 flush
 * below min normal AFTER rounding; FP16 keeps IEEE subnormals), R17 (symmetric
 * saturation), R18 (NaN: FP16 -> 0x7E00|sign, FP10/FP8 -> +-max), R19 (field j of a word
 * at bits [j*b, (j+1)*b), unused bits and tail fields 0).
 * Arithmetic in double via frexp/ldexp: every intermediate here is exact in binary64.
 * ---------------------------------------------------------------------------------- */

/* Round-half-to-even of a non-negative double, written out (R15). */
static double round_half_even(double v)
{
    double fl = floor(v);
    double frac = v - fl;
    if (frac > 0.5) return fl + 1.0;
    if (frac < 0.5) return fl;
    return fmod(fl, 2.0) == 0.0 ? fl : fl + 1.0;
}

/* FP10 (E=5, M=4) and FP8 (E=4, M=3): the step-by-step conversion of DESIGN.md O6. */
static uint32_t small_float_code(float x, int E, int M)
{
    uint32_t s = signbit(x) ? 1u : 0u;
    uint32_t sign_field = s << (E + M);
    uint32_t maxcode = (((1u << E) - 1u) << M) | ((1u << M) - 1u);
    int bias = (1 << (E - 1)) - 1;
    if (isnan(x) || isinf(x)) return sign_field | maxcode;  /* R18 / clamp */
    if (x == 0.0f) return sign_field;
    int e;
    double m = frexp(fabs((double)x), &e); /* |x| = m * 2^e, m in [0.5, 1) */
    m *= 2.0;                              /* -> m in [1, 2) */
    e -= 1;
    double f = round_half_even(m * (double)(1 << M)); /* P:171 round-to-nearest */
    if (f == (double)(1 << (M + 1))) { f = (double)(1 << M); e += 1; }
    int be = e + bias;
    if (be < 1) return sign_field;                          /* denormals ignored: flush */
    if (be > (1 << E) - 1) return sign_field | maxcode;     /* clamp at maximum */
    return sign_field | ((uint32_t)be << M) | (uint32_t)(f - (double)(1 << M));
}

/* FP16: IEEE binary16 after symmetric clamping to +-65504, subnormals kept. */
static uint32_t half_code(float x)
{
    uint32_t s = signbit(x) ? 1u : 0u;
    if (isnan(x)) return (s << 15) | 0x7E00u;               /* R18 */
    double a = fabs((double)x);
    if (a > 65504.0) a = 65504.0;                           /* clamp, inf too */
    if (a == 0.0) return s << 15;
    int e;
    double m = frexp(a, &e);
    m *= 2.0;
    e -= 1;
    if (e < -14) { /* IEEE subnormal: units of 2^-24 */
        double f = round_half_even(ldexp(a, 24));
        return (s << 15) | (uint32_t)f; /* f == 1024 is exactly the min-normal code */
    }
    double f = round_half_even(m * 1024.0);
    if (f == 2048.0) { f = 1024.0; e += 1; }
    return (s << 15) | ((uint32_t)(e + 15) << 10) | (uint32_t)(f - 1024.0);
}

uint32_t oracle_dpr_code(float x, int32_t bits)
{
    if (bits == 16) return half_code(x);
    if (bits == 10) return small_float_code(x, 5, 4);
    if (bits == 8) return small_float_code(x, 4, 3);
    return 0u;
}

float oracle_dpr_value(uint32_t code, int32_t bits)
{
    if (bits == 16) {
        uint32_t s = (code >> 15) & 1u, e = (code >> 10) & 0x1Fu, m = code & 0x3FFu;
        double mag;
        if (e == 0x1Fu) { /* Inf / NaN: IEEE widening keeps the payload */
            uint32_t b = (s << 31) | 0x7F800000u | (m << 13);
            float f;
            memcpy(&f, &b, 4);
            return f;
        }
        if (e == 0u) mag = ldexp((double)m, -24);
        else mag = ldexp(1.0 + (double)m / 1024.0, (int)e - 15);
        return (float)(s ? -mag : mag);
    }
    int E = bits == 10 ? 5 : 4, M = bits == 10 ? 4 : 3;
    int bias = (1 << (E - 1)) - 1;
    uint32_t s = (code >> (E + M)) & 1u;
    uint32_t e = (code >> M) & ((1u << E) - 1u);
    uint32_t m = code & ((1u << M) - 1u);
    if (e == 0u) return s ? -0.0f : 0.0f;                    /* R14: exponent 0 is zero */
    double mag = ldexp(1.0 + (double)m / (double)(1 << M), (int)e - bias);
    return (float)(s ? -mag : mag);
}

int32_t oracle_dpr_per_word(int32_t bits) { return bits == 16 ? 2 : bits == 10 ? 3 : bits == 8 ? 4 : 0; }

int64_t oracle_dpr_words(int64_t n, int32_t bits)
{
    int32_t k = oracle_dpr_per_word(bits);
    return k ? (n + k - 1) / k : -1;
}

void oracle_dpr_encode(const float *x, int64_t n, int32_t bits, uint32_t *packed)
{
    int32_t k = oracle_dpr_per_word(bits);
    for (int64_t w = 0; w < oracle_dpr_words(n, bits); ++w) packed[w] = 0u;
    for (int64_t i = 0; i < n; ++i)
        packed[i / k] |= oracle_dpr_code(x[i], bits) << (bits * (int32_t)(i % k));
}

void oracle_dpr_decode(const uint32_t *packed, int64_t n, int32_t bits, float *x)
{
    int32_t k = oracle_dpr_per_word(bits);
    uint32_t field = (1u << bits) - 1u;
    for (int64_t i = 0; i < n; ++i)
        x[i] = oracle_dpr_value((packed[i / k] >> (bits * (int32_t)(i % k))) & field, bits);
}

/* Elementwise code helpers used by the pin tests over large value sets. */
void oracle_dpr_codes(const float *x, int64_t n, int32_t bits, uint32_t *codes)
{
    for (int64_t i = 0; i < n; ++i) codes[i] = oracle_dpr_code(x[i], bits);
}

void oracle_dpr_values(const uint32_t *codes, int64_t n, int32_t bits, float *x)
{
    for (int64_t i = 0; i < n; ++i) x[i] = oracle_dpr_value(codes[i], bits);
}

/* ------------------------------------------------------------------------------------
 * O8 — f4 reference: weight gradient of a 3x3 / stride 1 / pad 1 convolution from the upstream
 * gradient dY and the (decoded) stashed input X.  P:128 §III ("the backward pass of the
 * convolution needs the input feature map X to compute the weight gradient"), §IV-A and
 * P:271-272 §V-H (the decode moved into the consumer GEMM: the result is the same weight
 * gradient).  Definition written out, accumulated in binary64:
 *     dW[co][ci][kh][kw] = sum_{n,oh,ow} dY[n][co][oh][ow] * X[n][ci][oh+kh-1][ow+kw-1]
 * with X = 0 outside the map.  dw_abs receives sum |dY * X| (the normwise error scale the f4
 * parity tolerance is stated against).  entries: the (co, ci, tap) triples to evaluate
 * (tap = 3 kh + kw); the full gradient is all Co*Ci*9 of them.
 * ---------------------------------------------------------------------------------- */
void oracle_conv3x3_wgrad_entries(const float *dy, const float *x, int32_t N, int32_t Ci, int32_t Co, int32_t H,
                                  int32_t W, const int32_t *entries, int64_t count, double *dw, double *dw_abs)
{
    for (int64_t e = 0; e < count; ++e) {
        int32_t co = entries[3 * e], ci = entries[3 * e + 1], tap = entries[3 * e + 2];
        int32_t kh = tap / 3, kw = tap % 3;
        double acc = 0.0, mag = 0.0;
        for (int32_t n = 0; n < N; ++n)
            for (int32_t oh = 0; oh < H; ++oh) {
                int32_t ih = oh + kh - 1;
                if (ih < 0 || ih >= H) continue;
                for (int32_t ow = 0; ow < W; ++ow) {
                    int32_t iw = ow + kw - 1;
                    if (iw < 0 || iw >= W) continue;
                    double g = dy[(((int64_t)n * Co + co) * H + oh) * W + ow];
                    double v = x[(((int64_t)n * Ci + ci) * H + ih) * W + iw];
                    acc += g * v;
                    mag += fabs(g * v);
                }
            }
        dw[e] = acc;
        dw_abs[e] = mag;
    }
}
