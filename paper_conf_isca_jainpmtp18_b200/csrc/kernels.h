// kernels.h — internal launchers behind the C ABI (include/gist.h).  Each returns the
// launch status; argument validation happens in gist_api.cu before these are called.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/gist.h"

namespace gist {

int current_device();
int num_sms();  // of the current device (cached per device)
// Dynamic shared-memory opt-in (cudaFuncAttributeMaxDynamicSharedMemorySize) of one kernel, applied
// once per DEVICE: the attribute is per device, so a process that launches on a second GPU sets it
// there too.
// The attribute only ever grows (a kernel whose shared memory depends on the call's shape keeps the
// largest size set so far).
struct PerDeviceAttr {
    static constexpr int kMaxDevices = 64;  // devices beyond: set on every launch
    std::atomic<int> set[kMaxDevices] = {};  // bytes already allowed on device d
    cudaError_t ensure(const void *func, int smem_bytes);
};
void count_launches(int k);  // bookkeeping for gist_launch_count()

cudaError_t launch_binarize(const float *y, int64_t n, uint32_t *mask, cudaStream_t s);
// mask != nullptr: write the a1 mask in the same pass when the geometry allows it
// (*mask_fused = true); otherwise the caller launches binarize separately.
cudaError_t launch_maxpool_fwd(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                               int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, cudaStream_t s,
                               uint32_t *mask = nullptr, bool *mask_fused = nullptr);
// f3: relu(x) on load (in-place ReLU); *mask_fused = false -> the caller adds binarize(x)
cudaError_t launch_relu_maxpool_fwd(const float *x, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                                    int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, uint32_t *mask, bool *mask_fused,
                                    cudaStream_t s);
cudaError_t launch_pool_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                            int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo, float *dx,
                            cudaStream_t s);
// 3x3 / stride 1 / pad <= 1 backward (pool_planes.cu): groups of whole planes staged by TMA
bool pool_planes_ok(const gist_pool2d &p, int32_t H, int32_t W, int32_t Ho, int32_t Wo);
cudaError_t launch_pool3s1_planes_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N,
                                      int32_t C, int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo,
                                      float *dx, cudaStream_t s);
size_t ssdc_workspace_bytes(int64_t n);
cudaError_t launch_ssdc_workspace_init(void *workspace, size_t bytes, cudaStream_t s);
cudaError_t launch_ssdc_encode(const float *x, int64_t n, int32_t *row_end, uint8_t *col, float *val,
                               int64_t capacity, int64_t *nnz, void *workspace, cudaStream_t s);
int64_t ssdc_tiles(int64_t n);
size_t ssdc_workspace_bytes_many(const gist_ssdc_job *jobs, int32_t count);
// every job has n > 0; *launches = kernels enqueued
cudaError_t launch_ssdc_encode_many(const gist_ssdc_job *jobs, int32_t count, void *workspace, cudaStream_t s,
                                    int *launches);
cudaError_t launch_ssdc_decode_many(const gist_ssdc_decode_job *jobs, int32_t count, cudaStream_t s, int *launches);
cudaError_t launch_ssdc_decode(const int32_t *row_end, const uint8_t *col, const float *val, int64_t n, float *x,
                               cudaStream_t s);
// n_dev != nullptr: the element count is min(n, *n_dev), read on the device.
cudaError_t launch_dpr_encode(const float *x, int64_t n, int bits, uint32_t *packed, cudaStream_t s,
                              const int64_t *n_dev = nullptr);
// every job has n > 0
cudaError_t launch_dpr_many(const gist_dpr_job *jobs, int32_t count, int bits, bool encode, cudaStream_t s,
                            int *launches);
cudaError_t launch_dpr_decode(const uint32_t *packed, int64_t n, int bits, float *x, cudaStream_t s,
                              const int64_t *n_dev = nullptr);

// pool3.cu: 3x3 windows (stride 1/2, pad 0/1, floor/ceil) through plane tiles in shared memory;
// cudaErrorNotSupported when a plane does not fit (the caller falls back)
bool pool3_ok(const gist_pool2d &p, bool fwd);
cudaError_t launch_pool3_fwd(const float *y, int32_t N, int32_t C, int32_t H, int32_t W, const gist_pool2d &p,
                             int32_t Ho, int32_t Wo, float *out, uint32_t *argmax, uint32_t *mask, bool relu,
                             cudaStream_t s);
cudaError_t launch_pool3_bwd(const float *dout, const uint32_t *argmax, const uint32_t *mask, int32_t N, int32_t C,
                             int32_t H, int32_t W, const gist_pool2d &p, int32_t Ho, int32_t Wo, float *dx,
                             cudaStream_t s);

// f4 (wgrad.cu): 3x3/s1/p1 conv weight gradient, X decoded from SSDC inside the tcgen05 GEMM
bool wgrad_shape_ok(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W);
size_t wgrad_workspace_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W);
size_t wgrad_smem_bytes(int32_t N, int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes);
cudaError_t launch_wgrad_ssdc(const float *dy, const int32_t *row_end, const uint8_t *col, const float *val, int32_t N,
                              int32_t Ci, int32_t Co, int32_t H, int32_t W, int32_t passes, float *dw, void *workspace,
                              cudaStream_t s, int *launches);

}  // namespace gist
