// sel_next.cu -- SURVEY §8(f) NEXT rows built on top of the hot path.
//
// f3  Launch-configuration selection ("the maximum grid-geometry
//     selected by the runtime"; P:L331 ML grid-geometry predictors whose
//     inference is slower than the kernel): for each group of candidates
//     (one nest on one device under several launch configurations) pick the
//     valid candidate with the smallest predicted T_gpu -- a segmented argmin
//     over the batch the hot path just evaluated.  Ties and +inf go to the
//     lowest candidate index, so the result is unique and deterministic.
//     Two passes of 64-bit atomicMin: first on the value's bit pattern
//     (non-negative doubles order like their bits), then on the index among
//     candidates that reach the minimum.
#include "sel_device.cuh"
#include "sel_internal.h"

namespace sel {

__global__ void k_sl_init(uint64_t n_groups, uint32_t* best, unsigned long long* bits) {
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= n_groups) return;
    best[g] = kNoProblem;
    bits[g] = ~0ull;                        // above +inf: "no valid candidate yet"
}

__global__ void k_sl_min(const uint32_t* __restrict__ group_of, uint64_t n, const double* __restrict__ t_gpu,
                         const uint8_t* __restrict__ status, uint64_t n_groups, unsigned long long* bits) {
    const uint64_t c = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (c >= n) return;
    const uint32_t g = group_of[c];
    if (g >= n_groups || status[c]) return;
    atomicMin(&bits[g], (unsigned long long)__double_as_longlong(t_gpu[c]));
}

__global__ void k_sl_arg(const uint32_t* __restrict__ group_of, uint64_t n, const double* __restrict__ t_gpu,
                         const uint8_t* __restrict__ status, uint64_t n_groups, const unsigned long long* bits,
                         uint32_t* best) {
    const uint64_t c = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (c >= n) return;
    const uint32_t g = group_of[c];
    if (g >= n_groups || status[c]) return;
    if ((unsigned long long)__double_as_longlong(t_gpu[c]) == bits[g]) atomicMin(&best[g], uint32_t(c));
}

__global__ void k_sl_fin(uint64_t n_groups, unsigned long long* bits) {
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= n_groups) return;
    if (bits[g] == ~0ull) bits[g] = 0x7ff0000000000000ull;    // +inf
}

cudaError_t launch_select_launch(const uint32_t* group_of, uint64_t n, const double* t_gpu, const uint8_t* status,
                                 uint64_t n_groups, uint32_t* best, double* best_t, cudaStream_t s) {
    unsigned long long* bits = reinterpret_cast<unsigned long long*>(best_t);
    const unsigned gg = unsigned((n_groups + 255) / 256), gc = unsigned((n + 255) / 256);
    k_sl_init<<<gg, 256, 0, s>>>(n_groups, best, bits);
    if (n) {
        k_sl_min<<<gc, 256, 0, s>>>(group_of, n, t_gpu, status, n_groups, bits);
        k_sl_arg<<<gc, 256, 0, s>>>(group_of, n, t_gpu, status, n_groups, bits, best);
    }
    k_sl_fin<<<gg, 256, 0, s>>>(n_groups, bits);
    note_launch(n ? 4 : 2);
    return cudaGetLastError();
}

}  // namespace sel
