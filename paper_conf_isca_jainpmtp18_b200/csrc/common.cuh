// common.cuh — device helpers shared by the sm_100a kernels of libgist.
// (Product side only; the CPU oracle under oracle/ shares nothing with this file.)
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <utility>

namespace gist {

constexpr int kWarp = 32;
constexpr unsigned kFull = 0xffffffffu;

// Streaming 128-bit load: the input feature map is read exactly once per call, so ask
// L2 to evict it first (ld.global.cs) and keep the encodings resident instead.
__device__ __forceinline__ float4 ld_stream_f4(const float4 *p) { return __ldcs(p); }
__device__ __forceinline__ uint4 ld_stream_u4(const uint4 *p) { return __ldcs(p); }
__device__ __forceinline__ uint2 ld_stream_u2(const uint2 *p) { return __ldcs(p); }
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t *p) { return __ldcs(p); }
__device__ __forceinline__ float ld_stream_f32(const float *p) { return __ldcs(p); }
__device__ __forceinline__ float2 ld_stream_f2(const float2 *p) { return __ldcs(p); }

// Read-only path through L1 for data re-read by neighbouring threads (pool windows).
template <typename T>
__device__ __forceinline__ T ld_ro(const T *p) { return __ldg(p); }

// Division by a runtime constant d (< 2^31) for numerators < 2^31: q = umulhi(n, mul) >> shr
// (round-up reciprocal, Granlund-Montgomery).  Host builds it once per launch.
struct FastDiv {
    uint32_t d, mul, shr;
    __host__ static FastDiv make(uint32_t d_) {
        FastDiv f{d_, 0u, 0u};
        if (d_ > 1) {
            uint32_t l = 0;
            while ((1ull << l) < d_) ++l;  // ceil(log2 d)
            uint32_t p = 31 + l;
            f.mul = (uint32_t)(((1ull << p) + d_ - 1) / d_);
            f.shr = p - 32;
        }
        return f;
    }
    __device__ __forceinline__ uint32_t div(uint32_t n) const {
        return d == 1 ? n : (__umulhi(n, mul) >> shr);
    }
    __device__ __forceinline__ void divmod(uint32_t n, uint32_t &q, uint32_t &r) const {
        q = div(n);
        r = n - q * d;
    }
};

// Programmatic dependent launch (PDL): every libgist kernel is launched with programmatic
// stream serialization and starts with pdl_enter(), which waits until the previous kernel has
// completed and its memory is visible (griddepcontrol.wait) before touching global memory.  No
// kernel triggers its dependents early (GIST_PDL_EARLY=0): the next grid is launched as this
// one's CTAs exit, so its launch overlaps only this kernel's drain.  An early trigger (at kernel
// start) let the next grid's CTAs take SM slots from this grid's later waves and cost 5-16% per
// step (C3 2.100 -> 1.815 ms, C5o 0.646 -> 0.547 ms, C4 1.997 -> 1.945 ms when removed; plain
// launches, GIST_PDL=0: C3 1.849, C4 2.020).  Stream order of the results is unchanged.
#ifndef GIST_PDL
#define GIST_PDL 1
#endif
#ifndef GIST_PDL_EARLY
#define GIST_PDL_EARLY 0
#endif
__device__ __forceinline__ void pdl_enter() {
#if GIST_PDL
#if GIST_PDL_EARLY
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}

template <typename... K, typename... A>
inline cudaError_t launch_k(void (*kern)(K...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, A &&...args) {
#if GIST_PDL
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<A>(args)...);
#else
    kern<<<grid, block, smem, s>>>(std::forward<A>(args)...);
    return cudaPeekAtLastError();
#endif
}

__host__ __device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace gist
