/*
 * include/gist.h — C ABI of the B200-native Gist stash-time encode/decode hot path.
 *
 * Gist (Jain, Phanishayee, Mars, Tang, Pekhimenko, ISCA 2018) stores each stashed fp32
 * feature map in an encoded form during the long gap between its forward and backward
 * use (§III, §IV-A: "E, the encoded intermediate feature map in
 * the forward pass, and D, the decoded intermediate feature map in the backward pass").
 * This library provides the three encodings of §IV-A:
 *
 *   Binarize (P:151-P:156)  gist_binarize_encode, gist_maxpool_fwd_argmax, gist_pool_relu_bwd
 *   SSDC     (P:158-P:164)  gist_ssdc_encode, gist_ssdc_decode
 *   DPR      (P:166-P:171)  gist_dpr_encode, gist_dpr_decode
 *
 * Conventions for every call:
 *   - All buffer pointers are DEVICE pointers (cudaMalloc / torch CUDA tensors) owned by
 *     the caller.  The library never allocates, frees or synchronizes: each call
 *     validates its arguments on the host, enqueues kernels on `stream` and returns.
 *     Outputs are valid once the stream reaches that point.
 *   - Layout: feature maps are dense, contiguous NCHW fp32 (CNTK and cuDNN use
 *     NCHW).  "Flat index" means the row-major NCHW offset.
 *   - Every buffer base pointer must be 16-byte aligned (GIST_ERR_MISALIGNED otherwise).
 *     Fresh torch / cudaMalloc allocations are.
 *   - n == 0 (or an empty shape) returns GIST_OK without launching anything.
 *   - Host-side argument errors are returned synchronously and nothing is launched.
 *     A launch failure returns GIST_ERR_CUDA.  Device faults surface at the caller's
 *     next synchronization, as for any CUDA kernel.
 *   - Deterministic: all encodings are bit-identical run to run; padding bits, unused
 *     fields and tail fields are always written as 0, so whole buffers compare with
 *     memcmp.  The library is stateless apart from per-device caches (SM count, the
 *     dynamic shared-memory opt-in of the kernels that need it) filled on first use on each device;
 *     calls act on the CURRENT device (cudaSetDevice).  Concurrent calls on different
 *     streams are safe when they use distinct outputs and workspaces.
 *   - Inputs and outputs must not overlap (GIST_ERR_INVALID_ARGUMENT).
 *
 * The readings of the paper taken wherever it is silent (bit orders, tie rules, rounding,
 * denormals, row-pointer form, ...) are listed in DESIGN.md §3 and cited below as R<k>.
 */
#ifndef GIST_H_
#define GIST_H_

#include <stddef.h>
#include <stdint.h>

#ifndef __CUDA_RUNTIME_H__
typedef struct CUstream_st *cudaStream_t; /* ABI-identical to the CUDA runtime's typedef */
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GIST_OK = 0,
    GIST_ERR_INVALID_ARGUMENT = 1, /* NULL buffer with n > 0, negative size, bad geometry, overlap */
    GIST_ERR_MISALIGNED = 2,       /* a buffer base pointer not 16-byte aligned */
    GIST_ERR_UNSUPPORTED = 3,      /* DPR bits not in {8,10,16}; pool window > 16 positions */
    GIST_ERR_TOO_LARGE = 4,        /* size exceeds the format's index range (see each call) */
    GIST_ERR_CUDA = 5              /* kernel launch failed (cudaPeekAtLastError) */
} gist_status;

/* Max-pool geometry (torch semantics): window kh x kw, stride sh x sw, zero-free padding
 * ph x pw (padded positions are never selected), ceil_mode != 0 rounds the output size
 * up (reading R4).  Constraints: k >= 1, s >= 1, 0 <= p <= k/2, kh*kw <= 16 (the argmax
 * is stored in 4 bits), output dims >= 1. */
typedef struct {
    int32_t kh, kw, sh, sw, ph, pw, ceil_mode;
} gist_pool2d;

const char *gist_status_string(gist_status s);

/* ---------------------------------------------------------------- size helpers (host) */
/* ceil(n/32): uint32 words of the 1-bit ReLU mask (32x). */
int64_t gist_binarize_words(int64_t n);
/* ceil(n_out/8): uint32 words of the 4-bit argmax map (8x). */
int64_t gist_argmax_words(int64_t n_out);
/* Output height/width of a pool (torch rules, R4).  Returns INVALID_ARGUMENT /
 * UNSUPPORTED for geometries the kernels refuse. */
gist_status gist_pool2d_out_dims(int32_t H, int32_t W, const gist_pool2d *p, int32_t *Ho, int32_t *Wo);
/* ceil(n/256): SSDC rows (Narrow Value Optimization: 256 columns, 1-byte index). */
int64_t gist_ssdc_rows(int64_t n);
/* 5*nnz + 4*rows: SSDC encoded bytes (fp32 value + uint8 column per nonzero, int32 row end
 * per row; R10). */
int64_t gist_ssdc_bytes(int64_t n, int64_t nnz);
/* Device workspace gist_ssdc_encode needs for n elements: a 128-byte counter line (tile
 * ticket, finished-CTA count, call epoch) plus one epoch-tagged 64-bit total per 32-row tile
 * (128 + 8*ceil(rows/32) bytes).  A workspace sized for n serves every n' <= n. */
size_t gist_ssdc_workspace_bytes(int64_t n);
/* Initialise a workspace on `stream`: zero it and mark it initialised (one small kernel).
 * Required ONCE before the workspace's first gist_ssdc_encode; every encode leaves it ready for
 * the next one.  INVALID_ARGUMENT if bytes < gist_ssdc_workspace_bytes(1) (the counter line). */
gist_status gist_ssdc_workspace_init(void *workspace, size_t bytes, cudaStream_t stream);
/* ceil(n / k), k = 2, 3, 4 values per 32-bit word for bits = 16, 10, 8; -1 for
 * unsupported bits. */
int64_t gist_dpr_words(int64_t n, int32_t bits);

/* ---------------------------------------------------------------- a1: Binarize encode
 * P:74 §III-A, §IV-A.  mask bit i = (y[i] > 0.0f): element i -> word i>>5, bit i&31,
 * LSB first (R1); NaN and -0.0 give 0; tail bits of the last word are 0.
 *   y     [n] fp32, read.          mask  [gist_binarize_words(n)] uint32, written.
 * Any n >= 0 (64-bit). */
gist_status gist_binarize_encode(const float *y, int64_t n, uint32_t *mask, cudaStream_t stream);

/* ---------------------------------------------------------------- a2: MaxPool fwd + argmax
 * P:152 ("create a mapping from Y to X in the forward pass that keeps track of these
 * locations"), P:154 (4 bits per pool output).  For every output o (flat NCHW over
 * [N,C,Ho,Wo]): out[o] = max over the in-bounds window positions (first maximum in
 * row-major window order; NaN counts as maximum, last NaN wins: R3), and nibble o of
 * argmax = window-local index dy*kw + dx of that position (R2): word o>>3, bits 4*(o&7).
 * Padding nibbles of the last word are 0.
 *   y      [N,C,H,W] fp32, read.
 *   out    [N,C,Ho,Wo] fp32, written (the pool output, still consumed in forward).
 *   argmax [gist_argmax_words(N*C*Ho*Wo)] uint32, written.
 *   mask   NULL, or [gist_binarize_words(N*C*H*W)] uint32: if non-NULL the a1 mask of y is
 *          written too — in the same pass (one read of y) for 2x2/s2 unpadded pools with H and
 *          W even whose warp unit of BR whole row pairs fits 512 items: BR*W/V <= 512 with
 *          V = 4 if W % 4 == 0 else 2, a = 16/gcd(W,16), BR = a*max(1, floor(256/(a*W/V)))
 *          (every VGG16 and OverFeat map), and for 3x3 windows of stride 1 or 2 with padding
 *          0 or 1 (AlexNet, NiN, GoogLeNet: whole-plane tiles staged in shared memory) when
 *          the planes of one tile fit a ring stage: stride 1, a multiple of 32/gcd(H*W,32)
 *          and of 8/gcd(Ho*Wo,8) planes in 32 KB with G*Ho*Wo <= 12288; stride 2, one plane
 *          plus the <= 3 rows of the next in 48 KB (H*W up to ~12000: not GoogLeNet's
 *          112x112 stem); otherwise by a second kernel over y.
 * TOO_LARGE if N*C*H*W >= 2^31. */
gist_status gist_maxpool_fwd_argmax(const float *y, int32_t N, int32_t C, int32_t H, int32_t W,
                                    const gist_pool2d *p, float *out, uint32_t *argmax,
                                    uint32_t *mask, cudaStream_t stream);

/* ---------------------------------------------------------------- f3: in-place ReLU + a1 + a2
 * P:139 (inplace ReLU: the ReLU output is never a separate buffer) with P:152-P:156: x is the
 * PRE-activation map (the producing conv's output).  Writes exactly what
 * gist_maxpool_fwd_argmax(relu(x), ..., mask) writes, with relu(v) = (v < 0 ? +0.0f : v)
 * (R21: torch's ReLU; -0.0 and NaN pass through), reading x once: out = the window max of
 * relu(x), argmax = its 4-bit in-window index, mask bit i = (x[i] > 0) (= relu(x)[i] > 0).
 * mask is required.  One kernel for 2x2/s2 with even H and W (VGG16, OverFeat) and for the 3x3
 * pools that gist_maxpool_fwd_argmax fuses; other geometries run the forward with relu
 * on load plus a binarize pass over x.  Errors as
 * gist_maxpool_fwd_argmax; mask == NULL -> INVALID_ARGUMENT. */
gist_status gist_relu_maxpool_fwd_argmax(const float *x, int32_t N, int32_t C, int32_t H, int32_t W,
                                         const gist_pool2d *p, float *out, uint32_t *argmax, uint32_t *mask,
                                         cudaStream_t stream);

/* ---------------------------------------------------------------- a3: fused pool+ReLU bwd
 * P:74 (ReLU bwd: dX = dY where Y > 0, else 0; MaxPool bwd routes dY to the argmax
 * location), P:156 ("Pool and ReLU backward pass ... perform computation on the encoded
 * data structures itself").  For every input element i:
 *   dx[i] = bit(mask, i) ? (+0.0f + sum of dout[o] over outputs o whose argmax is i, added
 *                           in ascending o, one fp32 add each)            : +0.0f
 * (R6, R7).  mask == NULL gives the plain max-pool backward.  Bit-identical to torch CPU
 * autograd of relu -> max_pool2d.
 *   dout [N,C,Ho,Wo] fp32, argmax as written by gist_maxpool_fwd_argmax with the same
 *   geometry, mask NULL or as written by gist_binarize_encode of the pool input,
 *   dx [N,C,H,W] fp32 written (every element).
 * TOO_LARGE if N*C*H*W >= 2^31. */
gist_status gist_pool_relu_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask,
                               int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d *p,
                               float *dx, cudaStream_t stream);

/* ---------------------------------------------------------------- a4: SSDC encode
 * P:158-P:164 §IV-A.  x is flattened and cut into rows of 256 elements (Narrow Value
 * Optimization; the last row may be partial, R9).  Row r keeps, in ascending column
 * order, every element whose BIT PATTERN is nonzero (R8: -0.0 is kept, so the round trip
 * is memcmp-exact):  col[k] = column (uint8), val[k] = value (fp32).
 *   row_end [gist_ssdc_rows(n)] int32 written: inclusive end offset of each row's entries
 *           (R10: the "extra meta array" of P:162, without the leading 0).
 *   col [capacity] uint8, val [capacity] fp32: entries with global offset < capacity are
 *           written; entries beyond are dropped.
 *   nnz     one DEVICE int64, written with the true number of nonzeros.  The encoding is
 *           complete iff *nnz <= capacity (capacity = n is always enough).
 *   workspace [>= gist_ssdc_workspace_bytes(n)] device bytes, zeroed once with
 *           gist_ssdc_workspace_init before its first use; each call leaves it reusable (the
 *           tile totals carry the call's epoch, so nothing is cleared per call).  One workspace
 *           must not serve two calls that may run concurrently (different streams).  A
 *           workspace that was never initialised is detected on the device: the call then writes
 *           *nnz = -1 and nothing else.
 * x is streamed from HBM once through a shared-memory ring (tile counts and compaction); tile
 * offsets come from a running prefix over all tile totals kept by each CTA.  One kernel launch.
 * TOO_LARGE if n >= 2^31. */
gist_status gist_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val,
                             int64_t capacity, int64_t *nnz, void *workspace,
                             size_t workspace_bytes, cudaStream_t stream);

/* ---------------------------------------------------------------- a5: SSDC decode
 * P:160 ("converts the data back into dense format only before it is actually required").
 * x[i] = +0.0f everywhere, then x[256 r + col[k]] = val[k] for k in row r's range.
 *   row_end/col/val as written by gist_ssdc_encode (complete encoding), x [n] fp32 written.
 * TOO_LARGE if n >= 2^31. */
gist_status gist_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n,
                             float *x, cudaStream_t stream);

/* ---------------------------------------------------------------- a6/a7: DPR
 * P:166-P:171 §IV-A.  bits = 16: IEEE binary16 (1-5-10) of x clamped to +-65504, round to
 * nearest even, subnormals kept, NaN -> 0x7E00|sign.  bits = 10: 1-5-4, bits = 8: 1-4-3,
 * bias 2^(E-1)-1, no Inf/NaN codes (max 126976 / 480), round to nearest even, results
 * below the minimum normal flush to +-0, larger magnitudes (and Inf/NaN) saturate to
 * +-max (R13-R18).  Packing (R19): value i -> word i/k, bits [b*(i%k), b*(i%k)+b), k = 2/3/4;
 * FP10 bits 30-31 and unused tail fields are 0.
 *   encode: x [n] fp32 read, packed [gist_dpr_words(n,bits)] uint32 written.
 *   decode: packed read, x [n] fp32 written (exact value of each code).
 * UNSUPPORTED if bits is not 8, 10 or 16.  Any n >= 0 (64-bit). */
gist_status gist_dpr_encode(const float *x, int64_t n, int32_t bits, uint32_t *packed, cudaStream_t stream);
gist_status gist_dpr_decode(const uint32_t *packed, int64_t n, int32_t bits, float *x, cudaStream_t stream);

/* ---------------------------------------------------------------- f1: DPR over SSDC values
 * P:169 §IV-A: "We also apply it [DPR] over SSDC encoding, compressing the non-zero values array
 * in the CSR format.  We do not touch the meta array in CSR format".  Same conversion and
 * packing as gist_dpr_encode/decode, applied to the first min(*nnz, capacity) entries of the
 * CSR value array; *nnz is the DEVICE count written by gist_ssdc_encode, read on the device
 * (no host synchronization).  Words past ceil(count/k) are left untouched.
 *   encode: val [capacity] fp32 read, packed [gist_dpr_words(capacity, bits)] uint32 written.
 *   decode: packed read, val [capacity] fp32 written (first count entries).
 * Encoded footprint: 4*ceil(nnz/k) + nnz + 4*rows bytes (vs 5*nnz + 4*rows). */
gist_status gist_ssdc_dpr_encode(const float *val, const int64_t *nnz, int64_t capacity, int32_t bits,
                                 uint32_t *packed, cudaStream_t stream);
gist_status gist_ssdc_dpr_decode(const uint32_t *packed, const int64_t *nnz, int64_t capacity, int32_t bits,
                                 float *val, cudaStream_t stream);

/* ---------------------------------------------------------------- many maps per call
 * P:171 ("these conversions can happen in parallel"): a network stashes many maps per minibatch;
 * these calls encode/decode several maps in ONE persistent launch (per up to 48 SSDC / 64 SSDC-
 * decode / 96 DPR maps), so the per-launch fill and drain is paid once instead of once per map.
 * Each job's results are exactly those of the single-map call on the same arguments; every job is
 * validated as the single-map call validates it (status of the first failing job, nothing
 * launched).  Jobs must not overlap each other's outputs.  count == 0 returns GIST_OK.
 *
 * offset (append mode, f2): NULL, or a DEVICE int64 holding the position where this map's CSR
 * entries start inside col/val (a stash arena shared by several maps).  Then entry k of the map is
 * written at col[*offset + k] / val[*offset + k] (only where *offset + k < capacity), row_end holds
 * ABSOLUTE inclusive ends (< 2^31), and *nnz receives the END offset *offset + count.  Decode jobs
 * take the same offset so that row 0 starts at *offset.  With offset == NULL a job is the plain
 * single-map encoding (*nnz = count).  Within one encode_many call a job's offset may be the nnz
 * of the PREVIOUS job (both n > 0): its entries then follow that job's in the same arena, computed
 * in the same launch (a chained stash arena: exact-size, no host synchronization).  Any other
 * aliasing of an offset with a job's nnz is INVALID_ARGUMENT. */
typedef struct {
    const float *x;
    int64_t n;
    int32_t *row_end;
    uint8_t *col;
    float *val;
    int64_t capacity;
    int64_t *nnz;
    const int64_t *offset;
} gist_ssdc_job;

typedef struct {
    const int32_t *row_end;
    const uint8_t *col;
    const float *val;
    const int64_t *offset;
    int64_t n;
    float *x;
} gist_ssdc_decode_job;

typedef struct {
    const float *x;    /* encode: read; decode: written */
    int64_t n;
    uint32_t *packed;  /* encode: written; decode: read */
} gist_dpr_job;

/* Workspace bytes for gist_ssdc_encode_many over these jobs: 128 + 8 * sum of their 32-row tiles. */
size_t gist_ssdc_workspace_bytes_many(const gist_ssdc_job *jobs, int32_t count);
gist_status gist_ssdc_encode_many(const gist_ssdc_job *jobs, int32_t count, void *workspace,
                                  size_t workspace_bytes, cudaStream_t stream);
gist_status gist_ssdc_decode_many(const gist_ssdc_decode_job *jobs, int32_t count, cudaStream_t stream);
gist_status gist_dpr_encode_many(const gist_dpr_job *jobs, int32_t count, int32_t bits, cudaStream_t stream);
gist_status gist_dpr_decode_many(const gist_dpr_job *jobs, int32_t count, int32_t bits, cudaStream_t stream);

/* ---------------------------------------------------------------- f4: decode inside the consumer GEMM
 * P:166 §IV-A ("the backward pass implementation can be modified to work directly on
 * precision-reduced values"), §V-H ("decode only the data that is required in near
 * future ... the near-future tile in a tiled matrix multiplication"), P:128 (the conv backward needs
 * its stashed input X for the weight gradient).  Weight gradient of a 3x3 / stride 1 / pad 1
 * convolution (every VGG16 conv) whose input X is held as its SSDC encoding:
 *     dW[co][ci][kh][kw] = sum_{n,oh,ow} dY[n][co][oh][ow] * X[n][ci][oh+kh-1][ow+kw-1]
 * (out-of-range X is 0).  X is decoded tile by tile into shared memory inside a tcgen05 (UMMA)
 * implicit GEMM; no dense X exists in device memory.
 *   dy      [N,Co,H,W] fp32, read.   row_end/col/val: gist_ssdc_encode of X [N,Ci,H,W] (complete).
 *   dw      [Co,Ci,3,3] fp32, written.
 *   passes  3: "3xTF32" (each operand split into TF32 hi + lo; hi*hi + hi*lo + lo*hi accumulated in
 *           fp32: every product within ~2^-19 relative of the fp32 product); 1: TF32 products (inputs
 *           truncated to 10-bit mantissas), fp32 accumulation.  Deterministic (fixed split-K order).
 *   workspace [>= gist_conv3x3_wgrad_workspace_bytes(...)] device bytes (split-K partials).
 * UNSUPPORTED unless Co % 128 == 0, Ci % 16 == 0, H*W % 4 == 0 (dY rows are TMA rows), W <= 252 and
 * the two decode slabs (16 x (R+2) x (W+2) floats each, R ~ 256/W rows) fit shared memory (W <= ~190),
 * passes in {1, 3};
 * TOO_LARGE if N*Ci*H*W or N*Co*H*W >= 2^31.  N, H or W == 0: dW is set to 0 (an empty sum) with
 * cudaMemsetAsync; Ci or Co == 0: nothing to write. */
size_t gist_conv3x3_wgrad_workspace_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W);
gist_status gist_conv3x3_wgrad_ssdc(const float *dy, const int32_t *row_end, const uint8_t *col, const float *val,
                                    int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes,
                                    float *dw, void *workspace, size_t workspace_bytes, cudaStream_t stream);

/* Number of SMs the launch heuristics use (cached on first call; for diagnostics). */
int32_t gist_num_sms(void);

/* Total kernels this library has enqueued since load (process-wide, atomic).  Lets a
 * caller count the library's launches inside a timed region. */
uint64_t gist_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* GIST_H_ */
