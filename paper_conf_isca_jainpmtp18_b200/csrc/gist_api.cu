// gist_api.cu — the C ABI (include/gist.h): host-side validation, size helpers, dispatch
// to the sm_100a kernels.  Stateless apart from per-device caches (SM count, shared-memory opt-ins).
#include <cuda_runtime.h>

#include <atomic>
#include <climits>
#include <vector>

#include "../../include/gist.h"
#include "kernels.h"

namespace gist {

static std::atomic<uint64_t> g_launches{0};
void count_launches(int k) { g_launches.fetch_add((uint64_t)k, std::memory_order_relaxed); }

int current_device() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0) dev = 0;
    return dev;
}

// SM count of the CURRENT device, cached per device (a process may drive several GPUs).
int num_sms() {
    constexpr int kMaxDev = 64;
    static std::atomic<int> cache[kMaxDev];
    const int dev = current_device();
    if (dev >= kMaxDev) {
        int v = 0;
        return cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0 ? v : 148;
    }
    int v = cache[dev].load(std::memory_order_relaxed);
    if (v <= 0) {
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
        cache[dev].store(v, std::memory_order_relaxed);
    }
    return v;
}

cudaError_t PerDeviceAttr::ensure(const void *func, int smem_bytes) {
    const int dev = current_device();
    if (dev < kMaxDevices && set[dev].load(std::memory_order_acquire) >= smem_bytes) return cudaSuccess;
    const cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
    if (e == cudaSuccess && dev < kMaxDevices) {
        int cur = set[dev].load(std::memory_order_relaxed);
        while (cur < smem_bytes && !set[dev].compare_exchange_weak(cur, smem_bytes, std::memory_order_acq_rel)) {
        }
    }
    return e;
}

}  // namespace gist

namespace {

constexpr int64_t kI32Limit = (int64_t)1 << 31;

bool misaligned(const void *p) { return p != nullptr && (reinterpret_cast<uintptr_t>(p) & 15u) != 0; }

struct Range {
    const void *p;
    int64_t bytes;
};

bool overlap(Range a, Range b) {
    if (!a.p || !b.p || a.bytes <= 0 || b.bytes <= 0) return false;
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(a.p), b0 = reinterpret_cast<uintptr_t>(b.p);
    return a0 < b0 + (uintptr_t)b.bytes && b0 < a0 + (uintptr_t)a.bytes;
}

bool any_overlap(std::initializer_list<Range> ins, std::initializer_list<Range> outs) {
    for (const Range &o : outs) {
        for (const Range &i : ins)
            if (overlap(i, o)) return true;
    }
    for (auto o1 = outs.begin(); o1 != outs.end(); ++o1)
        for (auto o2 = o1 + 1; o2 != outs.end(); ++o2)
            if (overlap(*o1, *o2)) return true;
    return false;
}

gist_status launched(cudaError_t e, int kernels) {
    if (e != cudaSuccess) return GIST_ERR_CUDA;
    gist::count_launches(kernels);
    return GIST_OK;
}

int32_t pool_dim(int32_t in, int32_t k, int32_t s, int32_t p, int32_t ceil_mode) {
    const int64_t span = (int64_t)in + 2 * (int64_t)p - k;  // int64: no wrap for any int32 inputs
    if (span < 0) return 0;
    int64_t out = ceil_mode ? (span + s - 1) / s + 1 : span / s + 1;
    if (ceil_mode && (out - 1) * s >= (int64_t)in + p) out -= 1;
    return out > INT32_MAX ? -1 : (int32_t)out;
}

gist_status check_pool(int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d *p, int32_t *Ho, int32_t *Wo) {
    if (!p || N < 0 || C < 0 || H < 0 || W < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (p->kh < 1 || p->kw < 1 || p->sh < 1 || p->sw < 1 || p->ph < 0 || p->pw < 0 || p->ph > p->kh / 2 ||
        p->pw > p->kw / 2)
        return GIST_ERR_INVALID_ARGUMENT;
    // argmax must fit 4 bits; each side is bounded first so the product cannot wrap
    if (p->kh > 16 || p->kw > 16 || (int64_t)p->kh * p->kw > 16) return GIST_ERR_UNSUPPORTED;
    *Ho = pool_dim(H, p->kh, p->sh, p->ph, p->ceil_mode);
    *Wo = pool_dim(W, p->kw, p->sw, p->pw, p->ceil_mode);
    if ((H > 0 && *Ho < 1) || (W > 0 && *Wo < 1)) return GIST_ERR_INVALID_ARGUMENT;
    return GIST_OK;
}

}  // namespace

extern "C" {

const char *gist_status_string(gist_status s) {
    switch (s) {
        case GIST_OK: return "GIST_OK";
        case GIST_ERR_INVALID_ARGUMENT: return "GIST_ERR_INVALID_ARGUMENT";
        case GIST_ERR_MISALIGNED: return "GIST_ERR_MISALIGNED";
        case GIST_ERR_UNSUPPORTED: return "GIST_ERR_UNSUPPORTED";
        case GIST_ERR_TOO_LARGE: return "GIST_ERR_TOO_LARGE";
        case GIST_ERR_CUDA: return "GIST_ERR_CUDA";
    }
    return "GIST_ERR_UNKNOWN";
}

int64_t gist_binarize_words(int64_t n) { return n < 0 ? -1 : (n + 31) / 32; }
int64_t gist_argmax_words(int64_t n_out) { return n_out < 0 ? -1 : (n_out + 7) / 8; }
int64_t gist_ssdc_rows(int64_t n) { return n < 0 ? -1 : (n + 255) / 256; }
int64_t gist_ssdc_bytes(int64_t n, int64_t nnz) { return n < 0 || nnz < 0 ? -1 : 5 * nnz + 4 * gist_ssdc_rows(n); }
size_t gist_ssdc_workspace_bytes(int64_t n) { return gist::ssdc_workspace_bytes(n < 0 ? 0 : n); }
int64_t gist_dpr_words(int64_t n, int32_t bits) {
    const int k = bits == 16 ? 2 : bits == 10 ? 3 : bits == 8 ? 4 : 0;
    if (!k || n < 0) return -1;
    return (n + k - 1) / k;
}
int32_t gist_num_sms(void) { return gist::num_sms(); }
uint64_t gist_launch_count(void) { return gist::g_launches.load(std::memory_order_relaxed); }

gist_status gist_pool2d_out_dims(int32_t H, int32_t W, const gist_pool2d *p, int32_t *Ho, int32_t *Wo) {
    if (!Ho || !Wo) return GIST_ERR_INVALID_ARGUMENT;
    return check_pool(1, 1, H, W, p, Ho, Wo);
}

gist_status gist_binarize_encode(const float *y, int64_t n, uint32_t *mask, cudaStream_t stream) {
    if (n < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (n == 0) return GIST_OK;
    if (!y || !mask) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(y) || misaligned(mask)) return GIST_ERR_MISALIGNED;
    if (any_overlap({{y, 4 * n}}, {{mask, 4 * gist_binarize_words(n)}})) return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_binarize(y, n, mask, stream), 1);
}

gist_status gist_maxpool_fwd_argmax(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d *p,
                                    float *out, uint32_t *argmax, uint32_t *mask, cudaStream_t stream) {
    int32_t Ho = 0, Wo = 0;
    const gist_status st = check_pool(N, C, H, W, p, &Ho, &Wo);
    if (st != GIST_OK) return st;
    const int64_t n = (int64_t)N * C * H * W, n_out = (int64_t)N * C * Ho * Wo;
    if (n == 0) return GIST_OK;
    if (!y || !out || !argmax) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(y) || misaligned(out) || misaligned(argmax) || misaligned(mask)) return GIST_ERR_MISALIGNED;
    if (n >= kI32Limit || n_out >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (any_overlap({{y, 4 * n}},
                    {{out, 4 * n_out}, {argmax, 4 * gist_argmax_words(n_out)}, {mask, mask ? 4 * gist_binarize_words(n) : 0}}))
        return GIST_ERR_INVALID_ARGUMENT;
    bool fused = false;
    cudaError_t e = gist::launch_maxpool_fwd(y, N, C, H, W, *p, Ho, Wo, out, argmax, stream, mask, &fused);
    const bool separate = mask && !fused;  // geometry the fused kernel does not cover
    if (e == cudaSuccess && separate) e = gist::launch_binarize(y, n, mask, stream);
    return launched(e, separate ? 2 : 1);
}

gist_status gist_relu_maxpool_fwd_argmax(const float *x, int32_t N, int32_t C, int32_t H, int32_t W,
                                         const gist_pool2d *p, float *out, uint32_t *argmax, uint32_t *mask,
                                         cudaStream_t stream) {
    int32_t Ho = 0, Wo = 0;
    const gist_status st = check_pool(N, C, H, W, p, &Ho, &Wo);
    if (st != GIST_OK) return st;
    const int64_t n = (int64_t)N * C * H * W, n_out = (int64_t)N * C * Ho * Wo;
    if (n == 0) return GIST_OK;
    if (!x || !out || !argmax || !mask) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(x) || misaligned(out) || misaligned(argmax) || misaligned(mask)) return GIST_ERR_MISALIGNED;
    if (n >= kI32Limit || n_out >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (any_overlap({{x, 4 * n}},
                    {{out, 4 * n_out}, {argmax, 4 * gist_argmax_words(n_out)}, {mask, 4 * gist_binarize_words(n)}}))
        return GIST_ERR_INVALID_ARGUMENT;
    bool fused = false;
    cudaError_t e = gist::launch_relu_maxpool_fwd(x, N, C, H, W, *p, Ho, Wo, out, argmax, mask, &fused, stream);
    // relu(x) > 0 iff x > 0: the mask of the pre-activation map is the mask of the ReLU output
    if (e == cudaSuccess && !fused) e = gist::launch_binarize(x, n, mask, stream);
    return launched(e, fused ? 1 : 2);
}

gist_status gist_pool_relu_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                               int32_t H, int32_t W, const gist_pool2d *p, float *dx, cudaStream_t stream) {
    int32_t Ho = 0, Wo = 0;
    const gist_status st = check_pool(N, C, H, W, p, &Ho, &Wo);
    if (st != GIST_OK) return st;
    const int64_t n = (int64_t)N * C * H * W, n_out = (int64_t)N * C * Ho * Wo;
    if (n == 0) return GIST_OK;
    if (!dout || !argmax || !dx) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(dout) || misaligned(argmax) || misaligned(mask) || misaligned(dx)) return GIST_ERR_MISALIGNED;
    if (n >= kI32Limit || n_out >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (any_overlap({{dout, 4 * n_out}, {argmax, 4 * gist_argmax_words(n_out)}, {mask, mask ? 4 * gist_binarize_words(n) : 0}},
                    {{dx, 4 * n}}))
        return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_pool_bwd(dout, argmax, mask, N, C, H, W, *p, Ho, Wo, dx, stream), 1);
}

// Host-side checks of one SSDC encode job (shared by the single- and many-map calls).
static gist_status check_ssdc_job(const gist_ssdc_job &j, const void *workspace, size_t workspace_bytes) {
    const int64_t n = j.n, capacity = j.capacity;
    if (n < 0 || capacity < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (n >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (!j.nnz) return GIST_ERR_INVALID_ARGUMENT;
    if (n > 0 && (!j.x || !j.row_end || !workspace)) return GIST_ERR_INVALID_ARGUMENT;
    if (capacity > 0 && (!j.col || !j.val)) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(j.x) || misaligned(j.row_end) || misaligned(j.col) || misaligned(j.val) || misaligned(workspace) ||
        (reinterpret_cast<uintptr_t>(j.nnz) & 7u) || (reinterpret_cast<uintptr_t>(j.offset) & 7u))
        return GIST_ERR_MISALIGNED;
    // plain mode writes at most n entries; append mode anywhere in the capacity-sized arena
    const int64_t cap = j.offset ? capacity : (capacity < n ? capacity : n);
    if (any_overlap({{j.x, 4 * n}, {j.offset, j.offset ? 8 : 0}},
                    {{j.row_end, 4 * gist_ssdc_rows(n)}, {j.col, cap}, {j.val, 4 * cap}, {j.nnz, 8},
                     {workspace, (int64_t)workspace_bytes}}))
        return GIST_ERR_INVALID_ARGUMENT;
    return GIST_OK;
}

// n == 0: publish *nnz (= 0, or the start offset in append mode) in stream order, no kernel
static gist_status publish_empty(const gist_ssdc_job &j, cudaStream_t stream) {
    const cudaError_t e = j.offset ? cudaMemcpyAsync(j.nnz, j.offset, sizeof(int64_t), cudaMemcpyDeviceToDevice, stream)
                                   : cudaMemsetAsync(j.nnz, 0, sizeof(int64_t), stream);
    return e == cudaSuccess ? GIST_OK : GIST_ERR_CUDA;
}

gist_status gist_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val, int64_t capacity,
                             int64_t *nnz, void *workspace, size_t workspace_bytes, cudaStream_t stream) {
    const gist_ssdc_job j{x, n, row_end, col, val, capacity, nnz, nullptr};
    gist_status st = check_ssdc_job(j, workspace, workspace_bytes);
    if (st != GIST_OK) return st;
    if (n > 0 && workspace_bytes < gist_ssdc_workspace_bytes(n)) return GIST_ERR_INVALID_ARGUMENT;
    if (n == 0) return publish_empty(j, stream);
    return launched(gist::launch_ssdc_encode(x, n, row_end, col, val, capacity, nnz, workspace, stream), 1);
}

size_t gist_ssdc_workspace_bytes_many(const gist_ssdc_job *jobs, int32_t count) {
    if (!jobs || count <= 0) return gist_ssdc_workspace_bytes(0);
    return gist::ssdc_workspace_bytes_many(jobs, count);
}

gist_status gist_ssdc_encode_many(const gist_ssdc_job *jobs, int32_t count, void *workspace, size_t workspace_bytes,
                                  cudaStream_t stream) {
    if (count < 0 || (count > 0 && !jobs)) return GIST_ERR_INVALID_ARGUMENT;
    if (count == 0) return GIST_OK;
    std::vector<gist_ssdc_job> live;
    live.reserve(count);
    for (int32_t k = 0; k < count; ++k) {
        const gist_status st = check_ssdc_job(jobs[k], workspace, workspace_bytes);
        if (st != GIST_OK) return st;
        if (jobs[k].n > 0) live.push_back(jobs[k]);
    }
    if (!live.empty() && workspace_bytes < gist::ssdc_workspace_bytes_many(live.data(), (int32_t)live.size()))
        return GIST_ERR_INVALID_ARGUMENT;
    // an offset may be the nnz (end offset) of the PREVIOUS job only (a chained arena); any other job's
    // nnz, or its own, is written during the launch
    for (int32_t k = 0; k < count; ++k) {
        if (!jobs[k].offset) continue;
        for (int32_t i = 0; i < count; ++i)
            if (jobs[i].nnz == jobs[k].offset && i != k - 1) return GIST_ERR_INVALID_ARGUMENT;
        if (k > 0 && jobs[k].offset == jobs[k - 1].nnz && (jobs[k].n == 0 || jobs[k - 1].n == 0))
            return GIST_ERR_INVALID_ARGUMENT;  // chaining links launched maps (n > 0) only
    }
    for (int32_t k = 0; k < count; ++k)
        if (jobs[k].n == 0) {
            const gist_status st = publish_empty(jobs[k], stream);
            if (st != GIST_OK) return st;
        }
    if (live.empty()) return GIST_OK;
    int launches = 0;
    const cudaError_t e = gist::launch_ssdc_encode_many(live.data(), (int32_t)live.size(), workspace, stream, &launches);
    return launched(e, launches);
}

gist_status gist_ssdc_workspace_init(void *workspace, size_t bytes, cudaStream_t stream) {
    if (bytes == 0) return GIST_OK;
    if (!workspace) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(workspace)) return GIST_ERR_MISALIGNED;
    if (bytes < gist_ssdc_workspace_bytes(1)) return GIST_ERR_INVALID_ARGUMENT;  // the counter line
    return launched(gist::launch_ssdc_workspace_init(workspace, bytes, stream), 1);
}

static gist_status check_ssdc_decode_job(const gist_ssdc_decode_job &j) {
    const int64_t n = j.n;
    if (n < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (n >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (n == 0) return GIST_OK;
    if (!j.row_end || !j.x) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(j.row_end) || misaligned(j.col) || misaligned(j.val) || misaligned(j.x) ||
        (reinterpret_cast<uintptr_t>(j.offset) & 7u))
        return GIST_ERR_MISALIGNED;
    if (any_overlap({{j.row_end, 4 * gist_ssdc_rows(n)}, {j.offset, j.offset ? 8 : 0}}, {{j.x, 4 * n}}))
        return GIST_ERR_INVALID_ARGUMENT;
    return GIST_OK;
}

gist_status gist_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n, float *x,
                             cudaStream_t stream) {
    const gist_ssdc_decode_job j{row_end, col, val, nullptr, n, x};
    const gist_status st = check_ssdc_decode_job(j);
    if (st != GIST_OK || n == 0) return st;
    // col/val extents are only known on the device (row_end[rows-1]); they may be NULL only
    // for an all-zero map, which the kernel then never dereferences.
    return launched(gist::launch_ssdc_decode(row_end, col, val, n, x, stream), 1);
}

gist_status gist_ssdc_decode_many(const gist_ssdc_decode_job *jobs, int32_t count, cudaStream_t stream) {
    if (count < 0 || (count > 0 && !jobs)) return GIST_ERR_INVALID_ARGUMENT;
    std::vector<gist_ssdc_decode_job> live;
    for (int32_t k = 0; k < count; ++k) {
        const gist_status st = check_ssdc_decode_job(jobs[k]);
        if (st != GIST_OK) return st;
        if (jobs[k].n > 0) live.push_back(jobs[k]);
    }
    if (live.empty()) return GIST_OK;
    int launches = 0;
    const cudaError_t e = gist::launch_ssdc_decode_many(live.data(), (int32_t)live.size(), stream, &launches);
    return launched(e, launches);
}

gist_status gist_dpr_encode(const float *x, int64_t n, int32_t bits, uint32_t *packed, cudaStream_t stream) {
    if (bits != 8 && bits != 10 && bits != 16) return GIST_ERR_UNSUPPORTED;
    if (n < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (n == 0) return GIST_OK;
    if (!x || !packed) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(x) || misaligned(packed)) return GIST_ERR_MISALIGNED;
    if (any_overlap({{x, 4 * n}}, {{packed, 4 * gist_dpr_words(n, bits)}})) return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_dpr_encode(x, n, bits, packed, stream), 1);
}

gist_status gist_dpr_decode(const uint32_t *packed, int64_t n, int32_t bits, float *x, cudaStream_t stream) {
    if (bits != 8 && bits != 10 && bits != 16) return GIST_ERR_UNSUPPORTED;
    if (n < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (n == 0) return GIST_OK;
    if (!x || !packed) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(x) || misaligned(packed)) return GIST_ERR_MISALIGNED;
    if (any_overlap({{packed, 4 * gist_dpr_words(n, bits)}}, {{x, 4 * n}})) return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_dpr_decode(packed, n, bits, x, stream), 1);
}

static gist_status dpr_many(const gist_dpr_job *jobs, int32_t count, int32_t bits, bool encode, cudaStream_t stream) {
    if (bits != 8 && bits != 10 && bits != 16) return GIST_ERR_UNSUPPORTED;
    if (count < 0 || (count > 0 && !jobs)) return GIST_ERR_INVALID_ARGUMENT;
    std::vector<gist_dpr_job> live;
    for (int32_t k = 0; k < count; ++k) {
        const gist_dpr_job &j = jobs[k];
        if (j.n < 0) return GIST_ERR_INVALID_ARGUMENT;
        if (j.n == 0) continue;
        if (!j.x || !j.packed) return GIST_ERR_INVALID_ARGUMENT;
        if (misaligned(j.x) || misaligned(j.packed)) return GIST_ERR_MISALIGNED;
        if (overlap({j.x, 4 * j.n}, {j.packed, 4 * gist_dpr_words(j.n, bits)})) return GIST_ERR_INVALID_ARGUMENT;
        live.push_back(j);
    }
    if (live.empty()) return GIST_OK;
    int launches = 0;
    const cudaError_t e = gist::launch_dpr_many(live.data(), (int32_t)live.size(), bits, encode, stream, &launches);
    return launched(e, launches);
}

gist_status gist_ssdc_dpr_encode(const float *val, const int64_t *nnz, int64_t capacity, int32_t bits,
                                 uint32_t *packed, cudaStream_t stream) {
    if (bits != 8 && bits != 10 && bits != 16) return GIST_ERR_UNSUPPORTED;
    if (capacity < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (capacity == 0) return GIST_OK;
    if (!val || !nnz || !packed) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(val) || misaligned(packed) || (reinterpret_cast<uintptr_t>(nnz) & 7u)) return GIST_ERR_MISALIGNED;
    if (any_overlap({{val, 4 * capacity}, {nnz, 8}}, {{packed, 4 * gist_dpr_words(capacity, bits)}}))
        return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_dpr_encode(val, capacity, bits, packed, stream, nnz), 1);
}

gist_status gist_ssdc_dpr_decode(const uint32_t *packed, const int64_t *nnz, int64_t capacity, int32_t bits,
                                 float *val, cudaStream_t stream) {
    if (bits != 8 && bits != 10 && bits != 16) return GIST_ERR_UNSUPPORTED;
    if (capacity < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (capacity == 0) return GIST_OK;
    if (!val || !nnz || !packed) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(val) || misaligned(packed) || (reinterpret_cast<uintptr_t>(nnz) & 7u)) return GIST_ERR_MISALIGNED;
    if (any_overlap({{packed, 4 * gist_dpr_words(capacity, bits)}, {nnz, 8}}, {{val, 4 * capacity}}))
        return GIST_ERR_INVALID_ARGUMENT;
    return launched(gist::launch_dpr_decode(packed, capacity, bits, val, stream, nnz), 1);
}

gist_status gist_dpr_encode_many(const gist_dpr_job *jobs, int32_t count, int32_t bits, cudaStream_t stream) {
    return dpr_many(jobs, count, bits, true, stream);
}

gist_status gist_dpr_decode_many(const gist_dpr_job *jobs, int32_t count, int32_t bits, cudaStream_t stream) {
    return dpr_many(jobs, count, bits, false, stream);
}

size_t gist_conv3x3_wgrad_workspace_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W) {
    if (!gist::wgrad_shape_ok(N, Ci, Co, H, W)) return 0;
    return gist::wgrad_workspace_bytes(N, Ci, Co, H, W);
}

gist_status gist_conv3x3_wgrad_ssdc(const float *dy, const int32_t *row_end, const uint8_t *col, const float *val,
                                    int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes,
                                    float *dw, void *workspace, size_t workspace_bytes, cudaStream_t stream) {
    if (N < 0 || Ci < 0 || Co < 0 || H < 0 || W < 0) return GIST_ERR_INVALID_ARGUMENT;
    if (passes != 1 && passes != 3) return GIST_ERR_UNSUPPORTED;
    if (Ci == 0 || Co == 0) return GIST_OK;  // empty dW
    if (Co % 128 || Ci % 16) return GIST_ERR_UNSUPPORTED;
    if (N == 0 || H == 0 || W == 0) {  // no positions: dW = 0 (an empty sum)
        if (!dw) return GIST_ERR_INVALID_ARGUMENT;
        if (misaligned(dw)) return GIST_ERR_MISALIGNED;
        return cudaMemsetAsync(dw, 0, (size_t)Co * Ci * 9 * sizeof(float), stream) == cudaSuccess ? GIST_OK
                                                                                                  : GIST_ERR_CUDA;
    }
    if (!gist::wgrad_shape_ok(N, Ci, Co, H, W)) return GIST_ERR_UNSUPPORTED;
    const int64_t nx = (int64_t)N * Ci * H * W, ny = (int64_t)N * Co * H * W;
    if (nx >= kI32Limit || ny >= kI32Limit) return GIST_ERR_TOO_LARGE;
    if (!dy || !row_end || !dw || !workspace) return GIST_ERR_INVALID_ARGUMENT;
    if (misaligned(dy) || misaligned(row_end) || misaligned(col) || misaligned(val) || misaligned(dw) ||
        misaligned(workspace))
        return GIST_ERR_MISALIGNED;
    if (workspace_bytes < gist::wgrad_workspace_bytes(N, Ci, Co, H, W)) return GIST_ERR_INVALID_ARGUMENT;
    const int64_t ndw = (int64_t)Co * Ci * 9;
    if (any_overlap({{dy, 4 * ny}, {row_end, 4 * gist_ssdc_rows(nx)}}, {{dw, 4 * ndw}, {workspace, (int64_t)workspace_bytes}}))
        return GIST_ERR_INVALID_ARGUMENT;
    int launches = 0;
    const cudaError_t e =
        gist::launch_wgrad_ssdc(dy, row_end, col, val, N, Ci, Co, H, W, passes, dw, workspace, stream, &launches);
    if (e == cudaErrorNotSupported) return GIST_ERR_UNSUPPORTED;
    return launched(e, launches);
}

}  // extern "C"
