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
#include "sel_model.cuh"

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

// f1  Liao-Chapman CPU cost model (Fig. 3; Table II)
//     on the device, so the CPU side of the decision is modelled rather than
//     supplied: one thread per candidate evaluates the Fig. 3 sequence for a
//     statically scheduled parallel for and writes the result into the
//     candidate's cpu_cycles / cpu_hz (readings F1a-F1d in DESIGN.md).
//     fp64 with explicit round-to-nearest intrinsics, same order as the oracle.
namespace sel {

__global__ void __launch_bounds__(256) k_cpu_model(sel_candidate* __restrict__ cands, uint64_t n, sel_tables t,
                                                   const sel_cpu_input* __restrict__ in, sel_cpu_params p,
                                                   uint8_t* __restrict__ status) {
    const uint64_t c = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (c >= n) return;
    const sel_cpu_input x = in[c];
    const uint32_t nid = cands[c].nest_id;
    if (nid >= t.n_nests || x.threads == 0 || !(x.mca_cycles_per_iter >= 0.0) || !isfinite(x.mca_cycles_per_iter)) {
        status[c] = SEL_EINVAL;
        return;
    }
    const sel_nest nt = t.nests[nid];
    bool bad = false;
    cands[c].cpu_cycles = cpu_cycles_fig3(nt.P0 * nt.P1, __ull2double_rn(nt.bytes_h2d + nt.bytes_d2h), x, p, &bad);
    cands[c].cpu_hz = p.cpu_hz;
    status[c] = SEL_OK;
}

cudaError_t launch_cpu_model(sel_candidate* cands, uint64_t n, const sel_tables& t, const sel_cpu_input* in,
                             const sel_cpu_params& p, uint8_t* status, cudaStream_t s) {
    k_cpu_model<<<unsigned((n + 255) / 256), 256, 0, s>>>(cands, n, t, in, p, status);
    note_launch();
    return cudaGetLastError();
}

// f2  Runtime binding of symbolic IPDA expressions: one
//     thread per access evaluates the six byte coefficients as sums of terms
//     k * v[frame+s0] * v[frame+s1] * v[frame+s2] over the access's symbol
//     frame, with exact 128-bit products; |value| >= 2^62 -> SEL_ERANGE, a bad
//     index or element size -> SEL_EINVAL (output zeroed).  The result is a
//     concrete sel_access table the counting kernel consumes unchanged.
__global__ void __launch_bounds__(256) k_bind(const sel_sym_access* __restrict__ sym, uint64_t n_sym,
                                              const sel_sym_term* __restrict__ terms, uint64_t n_terms,
                                              const int64_t* __restrict__ values, uint64_t n_values,
                                              const sel_bind_item* __restrict__ items, uint64_t n,
                                              sel_access* __restrict__ out, uint8_t* __restrict__ status) {
    const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const __int128 lim = (__int128)1 << 62;
    const sel_bind_item it = items[i];
    uint8_t st = SEL_OK;
    int64_t coef[6] = {0, 0, 0, 0, 0, 0};
    int64_t e = 0;
    sel_access o{};
    if (it.sym_access >= n_sym) {
        st = SEL_EINVAL;
    } else {
        const sel_sym_access a = sym[it.sym_access];
        const uint64_t fr = it.frame;
        for (int slot = 0; slot < 6 && !st; slot++) {
            if (uint64_t(a.term_off[slot]) + a.n_terms[slot] > n_terms) { st = SEL_EINVAL; break; }
            __int128 acc = 0;
            for (int t = 0; t < a.n_terms[slot] && !st; t++) {
                const sel_sym_term tm = terms[a.term_off[slot] + t];
                __int128 p = tm.k;
                for (int f = 0; f < 3; f++) {
                    if (tm.sym[f] == SEL_SYM_ONE) continue;
                    if (fr + tm.sym[f] >= n_values) { st = SEL_EINVAL; break; }
                    p *= values[fr + tm.sym[f]];
                    if (p >= lim || p <= -lim) { st = SEL_ERANGE; break; }
                }
                if (st) break;
                acc += p;
                if (acc >= lim || acc <= -lim) st = SEL_ERANGE;
            }
            coef[slot] = int64_t(acc);
        }
        e = a.elem_bytes;
        if (!st && a.elem_sym != SEL_SYM_ONE) {
            if (fr + a.elem_sym >= n_values) st = SEL_EINVAL;
            else e = values[fr + a.elem_sym];
        }
        if (!st && !(e == 1 || e == 2 || e == 4 || e == 8 || e == 16)) st = SEL_EINVAL;
        if (!st) {
            o.base = coef[0];
            o.c_par[0] = coef[1];
            o.c_par[1] = coef[2];
            o.c_inner[0] = coef[3];
            o.c_inner[1] = coef[4];
            o.c_inner[2] = coef[5];
            o.elem_bytes = uint8_t(e);
            o.depth = a.depth;
            o.is_store = a.is_store;
        }
    }
    out[i] = o;
    status[i] = st;
}

cudaError_t launch_bind(const sel_sym_access* sym, uint64_t n_sym, const sel_sym_term* terms, uint64_t n_terms,
                        const int64_t* values, uint64_t n_values, const sel_bind_item* items, uint64_t n,
                        sel_access* out, uint8_t* status, cudaStream_t s) {
    k_bind<<<unsigned((n + 255) / 256), 256, 0, s>>>(sym, n_sym, terms, n_terms, values, n_values, items, n, out,
                                                     status);
    note_launch();
    return cudaGetLastError();
}

}  // namespace sel
