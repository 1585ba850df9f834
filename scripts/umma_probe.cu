// umma_probe.cu — microbenchmark: cycles per tcgen05.mma (cta_group::1, M = 128, SS operands with the
// 128-byte swizzle, K = 32 bytes per instruction) for kind::tf32 and kind::f16 (bf16) at several N,
// issued back to back by one thread from the same shared-memory tiles.  Used to read the f4
// kernel's MMA rate.  Not part of libgist.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_isca_jainpmtp18_b200/csrc \
//        scripts/umma_probe.cu -o scripts/umma_probe && scripts/umma_probe
#include <cstdio>
#include <cuda_runtime.h>

#include "tcgen05.cuh"

using namespace gist;

// MODE 0: back-to-back MMAs; 1: a tcgen05.commit after every 4 MMAs (a K = 32-float stage);
// 2: as 1, and before each stage wait for the commit of the stage D = 4 stages earlier (the
// operand-ring back-pressure of a pipelined kernel); 3: D = 8; 4: D = 1 (wait for the previous
// stage's commit: the commit round-trip latency is exposed); 5: as 2 with a test_wait polling loop
template <int N, bool BF16, int MODE>
__global__ void probe(long long *cycles, int iters) {
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ uint32_t tmem_base;
    __shared__ __align__(8) uint64_t bar, sbar[8];
    const uint32_t base = (smem_u32(smem) + 1023) & ~1023u;
    const uint32_t a_addr = base, b_addr = base + 128 * 128;  // A: 128 rows x 128 B, B: N rows x 128 B
    for (int i = threadIdx.x; i < (128 + N) * 128 / 4; i += blockDim.x)
        reinterpret_cast<uint32_t *>(smem + (base - smem_u32(smem)))[i] = 0x3c003c00u;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        for (int k = 0; k < 8; ++k) mbar_init(&sbar[k], 1);
        fence_mbar_init();
    }
    if (threadIdx.x < 32) tmem_alloc<256>(&tmem_base);
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (threadIdx.x == 0) {
        constexpr uint32_t idesc = BF16 ? ((1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) |
                                           ((uint32_t)(128 >> 4) << 24))
                                        : idesc_tf32<128, N>();
        const long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            const uint32_t kk = (uint32_t)(i & 3);
            const int stage = i >> 2;
            constexpr int D = MODE == 3 ? 8 : MODE == 4 ? 1 : 4;
            if (MODE >= 2 && MODE != 5 && kk == 0 && stage >= D) mbar_wait(&sbar[stage % D], (uint32_t)((stage / D) - 1) & 1u);
            if (MODE == 5 && kk == 0 && stage >= D)  // the same wait with non-blocking test_wait polling
                while (!mbar_test(&sbar[stage % D], (uint32_t)((stage / D) - 1) & 1u)) {
                }
            const uint64_t da = umma_desc_sw128(a_addr + 32 * kk), db = umma_desc_sw128(b_addr + 32 * kk);
            if (BF16)
                asm volatile(
                    "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                    "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_base),
                    "l"(da), "l"(db), "r"(idesc), "r"(i > 0 ? 1 : 0)
                    : "memory");
            else
                umma_tf32(tmem_base, da, db, idesc, i > 0 ? 1u : 0u);
            if (MODE >= 1 && kk == 3) umma_commit(&sbar[stage % (MODE == 3 ? 8 : MODE == 4 ? 1 : 4)]);
            if (MODE == 6 && kk == 3) asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        }
        umma_commit(&bar);
        mbar_wait(&bar, 0);
        const long long t1 = clock64();
        cycles[blockIdx.x] = t1 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tc_fence_after();
        tmem_dealloc<256>(tmem_base);
    }
}

template <int N, bool BF16, int MODE = 0>
void run(const char *name) {
    const int iters = 8192;
    long long *d, h[148];
    cudaMalloc(&d, sizeof(h));
    const int smem = (128 + N) * 128 + 1024;
    cudaFuncSetAttribute(probe<N, BF16, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int grid : {1, 148}) {
        probe<N, BF16, MODE><<<grid, 128, smem>>>(d, iters);
        probe<N, BF16, MODE><<<grid, 128, smem>>>(d, iters);
        cudaMemcpy(h, d, grid * sizeof(long long), cudaMemcpyDeviceToHost);
        long long mx = 0;
        for (int i = 0; i < grid; ++i) mx = h[i] > mx ? h[i] : mx;
        const double per = (double)mx / iters;
        const double flop = 2.0 * 128 * N * (BF16 ? 16 : 8);
        printf("%-5s N=%3d mode=%d grid=%3d: %6.1f cycles/MMA, %7.0f flop/cycle/SM (%s)\n", name, N, MODE, grid, per, flop / per,
               cudaGetErrorString(cudaGetLastError()));
    }
    cudaFree(d);
}

int main() {
    run<64, false>("tf32");
    run<128, false>("tf32");
    run<144, false>("tf32");
    run<256, false>("tf32");
    run<128, true>("bf16");
    run<144, true>("bf16");
    run<256, true>("bf16");
    run<144, false, 1>("tf32");
    run<144, false, 2>("tf32");
    run<144, false, 3>("tf32");
    run<144, false, 4>("tf32");
    run<144, false, 5>("tf32");
    return 0;
}
