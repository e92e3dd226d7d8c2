// int_peak.cu -- measured INT32 lane-op throughput of this GPU (the roofline
// denominator of the counting kernel).  Independent chains of
// IADD3/LOP3 (ALU pipe) interleaved with IMAD (FMA pipe), all SMs, several
// warps per scheduler; result = lane-ops / second.  Exposed as
// sel_int_peak() in libsel.so (diagnostic, not part of the hot path).
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/sel.h"

namespace sel {

template <int MODE>
__global__ void __launch_bounds__(512) k_int_peak(uint32_t iters, uint32_t seed, uint32_t* sink) {
    uint32_t a0 = threadIdx.x ^ seed, a1 = a0 * 3u, a2 = a0 * 5u, a3 = a0 * 7u;
    uint32_t b0 = a0 + 11u, b1 = a0 + 13u, b2 = a0 + 17u, b3 = a0 + 19u;
    const uint32_t k = seed | 1u;
    for (uint32_t i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 8; u++) {
            if (MODE == 0 || MODE == 2) {      // ALU pipe: IADD3 / LOP3, mutually dependent (not foldable)
                asm volatile("add.u32 %0, %0, %1;" : "+r"(a0) : "r"(a1));
                asm volatile("xor.b32 %0, %0, %1;" : "+r"(a1) : "r"(a2));
                asm volatile("add.u32 %0, %0, %1;" : "+r"(a2) : "r"(a3));
                asm volatile("xor.b32 %0, %0, %1;" : "+r"(a3) : "r"(a0));
            }
            if (MODE == 1 || MODE == 2) {      // FMA pipe: IMAD
                asm volatile("mad.lo.u32 %0, %0, %1, %1;" : "+r"(b0) : "r"(k));
                asm volatile("mad.lo.u32 %0, %0, %1, %1;" : "+r"(b1) : "r"(k));
                asm volatile("mad.lo.u32 %0, %0, %1, %1;" : "+r"(b2) : "r"(k));
                asm volatile("mad.lo.u32 %0, %0, %1, %1;" : "+r"(b3) : "r"(k));
            }
        }
    }
    const uint32_t r = a0 ^ a1 ^ a2 ^ a3 ^ b0 ^ b1 ^ b2 ^ b3;
    if (r == 0x9E3779B9u) sink[0] = r;
}

}  // namespace sel

extern "C" int sel_int_peak(int mode, double* lane_ops_per_s) {
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return SEL_ENODEV;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t* sink = nullptr;
    if (cudaMalloc(&sink, 4) != cudaSuccess) return SEL_ECUDA;
    const uint32_t iters = 4096;
    const int blocks = sms * 4, threads = 512;     // 64 warps / SM
    auto launch = [&]() {
        if (mode == 0) sel::k_int_peak<0><<<blocks, threads>>>(iters, 0x1234u, sink);
        else if (mode == 1) sel::k_int_peak<1><<<blocks, threads>>>(iters, 0x1234u, sink);
        else sel::k_int_peak<2><<<blocks, threads>>>(iters, 0x1234u, sink);
    };
    launch();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 5; rep++) {
        cudaEventRecord(e0);
        launch();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    if (cudaGetLastError() != cudaSuccess) return SEL_ECUDA;
    const double per_thread = double(iters) * 8.0 * (mode == 2 ? 8.0 : 4.0);
    *lane_ops_per_s = per_thread * double(blocks) * threads / (double(best) * 1e-3);
    return SEL_OK;
}
