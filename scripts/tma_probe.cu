// tma_probe.cu — standalone probe: read bandwidth of 1-D TMA bulk loads (cp.async.bulk) into a
// shared-memory ring vs plain LDG.128 streaming, for the SSDC encode design.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_probe scripts/tma_probe.cu && /tmp/tma_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int STAGES, int TILE_BYTES, bool HINT>
__global__ void tma_stream(const char *src, int64_t tiles, unsigned *sink) {
    extern __shared__ __align__(128) char sm[];
    uint64_t *full = reinterpret_cast<uint64_t *>(sm + STAGES * TILE_BYTES);
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    unsigned acc = 0;
    int64_t t = blockIdx.x;
    const int64_t stride = gridDim.x;
    auto issue = [&](int s, int64_t tile) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[s])), "r"(TILE_BYTES));
        const char *g = src + tile * TILE_BYTES;
        if (HINT)
            asm volatile(
                "{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], pol;\n\t}" ::"r"(
                    smem_u32(sm + s * TILE_BYTES)),
                "l"(g), "r"(TILE_BYTES), "r"(smem_u32(&full[s])));
        else
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(sm + s * TILE_BYTES)),
                         "l"(g), "r"(TILE_BYTES), "r"(smem_u32(&full[s])));
    };
    int issued = 0;
    for (int s = 0; s < STAGES && t + (int64_t)s * stride < tiles; ++s, ++issued) issue(s, t + (int64_t)s * stride);
    for (int j = 0; j < issued; ++j) {
        const int s = j % STAGES;
        asm volatile(
            "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(
                smem_u32(&full[s])),
            "r"((j / STAGES) & 1));
        acc += *reinterpret_cast<volatile unsigned *>(sm + s * TILE_BYTES);
        const int64_t nt = t + (int64_t)(j + STAGES) * stride;
        if (nt < tiles) {
            issue(s, nt);
            ++issued;
        }
    }
    sink[blockIdx.x] = acc;
}

__global__ void ldg_stream(const float4 *src, int64_t n4, unsigned *sink) {
    unsigned acc = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride * 8) {
        float4 v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = (i + u * stride < n4) ? __ldcs(src + i + u * stride) : make_float4(0, 0, 0, 0);
#pragma unroll
        for (int u = 0; u < 8; ++u) acc += __float_as_uint(v[u].x) ^ __float_as_uint(v[u].w);
    }
    if (acc == 0x12345678) sink[0] = acc;
}

template <int STAGES, int TILE_BYTES, bool HINT>
void run(const char *src, int64_t bytes, unsigned *sink, int sms, int ctas_per_sm) {
    const int smem = STAGES * TILE_BYTES + 8 * STAGES;
    cudaFuncSetAttribute(tma_stream<STAGES, TILE_BYTES, HINT>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int64_t tiles = bytes / TILE_BYTES;
    const int grid = sms * ctas_per_sm;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int w = 0; w < 3; ++w) tma_stream<STAGES, TILE_BYTES, HINT><<<grid, 32, smem>>>(src, tiles, sink);
    cudaEventRecord(a);
    const int reps = 10;
    for (int r = 0; r < reps; ++r) tma_stream<STAGES, TILE_BYTES, HINT><<<grid, 32, smem>>>(src, tiles, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    cudaError_t e = cudaGetLastError();
    printf("TMA stages=%d tile=%6d B ctas/SM=%d hint=%d in-flight/SM=%4d KB : %7.1f GB/s %s\n", STAGES, TILE_BYTES,
           ctas_per_sm, (int)HINT, STAGES * TILE_BYTES * ctas_per_sm / 1024, (double)tiles * TILE_BYTES * reps / (ms * 1e-3) / 1e9,
           e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t bytes = 1ll << 30;
    char *src;
    unsigned *sink;
    cudaMalloc(&src, bytes);
    cudaMalloc(&sink, 1 << 20);
    cudaMemset(src, 1, bytes);
    {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int w = 0; w < 3; ++w) ldg_stream<<<sms * 8, 256>>>((const float4 *)src, bytes / 16, sink);
        cudaEventRecord(a);
        for (int r = 0; r < 10; ++r) ldg_stream<<<sms * 8, 256>>>((const float4 *)src, bytes / 16, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("LDG.128 streaming                                           : %7.1f GB/s\n", 10.0 * bytes / (ms * 1e-3) / 1e9);
    }
    run<4, 16384, true>(src, bytes, sink, sms, 2);
    run<4, 16384, false>(src, bytes, sink, sms, 2);
    run<4, 16384, true>(src, bytes, sink, sms, 3);
    run<6, 16384, true>(src, bytes, sink, sms, 2);
    run<8, 16384, true>(src, bytes, sink, sms, 1);
    run<12, 16384, true>(src, bytes, sink, sms, 1);
    run<8, 8192, true>(src, bytes, sink, sms, 2);
    run<8, 8192, true>(src, bytes, sink, sms, 3);
    run<16, 8192, true>(src, bytes, sink, sms, 1);
    run<4, 32768, true>(src, bytes, sink, sms, 1);
    run<6, 32768, true>(src, bytes, sink, sms, 1);
    run<3, 32768, true>(src, bytes, sink, sms, 2);
    run<16, 4096, true>(src, bytes, sink, sms, 2);
    run<32, 4096, true>(src, bytes, sink, sms, 1);
    return 0;
}
