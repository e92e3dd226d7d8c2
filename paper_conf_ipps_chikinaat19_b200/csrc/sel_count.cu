// sel_count.cu -- the hot kernel: exact per-warp coalescing counts (a1-a3).
//
// For every counting problem (a nest and a block size class) and every
// memory access, every active warp of every OpenMP repetition and
// every inner-loop iteration is one warp-access (WA).  For each WA the kernel
// counts the distinct 128 B lines and 32 B sectors touched by the active
// lanes' byte addresses (the IPDA inter-thread stride evaluated with runtime
// values), classifies it as coalesced or not (R11) and
// accumulates W, L, S, C, U per problem.
//
// Mapping: ONE WARP PER ANALYSED WARP-ACCESS -- lane l of the CUDA warp plays
// lane l of the simulated warp.  A persistent grid pulls chunks of the
// flattened WA index space (problem, access, warp-rep, inner tuple) from an
// atomic counter, so a 16-WA nest and a 10^9-WA nest are balanced alike; a
// warp decodes its chunk start once (32-ary search over the problem prefix,
// one div/mod) and then walks with odometer steps.
//
// Two exact counting primitives:
//  * RESIDUE (default).  Per warp-rep the lane addresses A_l are fixed and
//    every inner iteration adds the same offset D to all of them, so their
//    sorted order and the gaps d_l between sorted neighbours are fixed.  Then
//    line(l) != line(pred(l))  <=>  (s_l + D) mod 128 < d_l  (d_l < 128), or
//    always (d_l >= 128); the same with 32 for sectors.  The hot loop keeps
//    y_l = (s_l + D) << 25 (the residue in the top 7 bits of a 32-bit
//    register) and tests y < d_l << 25: one ISETP per flag, no cross-lane
//    traffic.  1-D parallel accesses are monotone across lanes (no sort);
//    collapse(2) accesses are sorted once per warp-rep with a shuffle
//    bitonic network.  lines = 1 + #flags; coalesced (tmin = 1) <=> no flag
//    (__any_sync); tmin > 1 uses __ballot_sync/__popc.
//  * MATCH (SEL_F_MATCH_ANY).  The north star's literal primitive: full
//    64-bit lane addresses, __match_any_sync on (addr >> 7) and (addr >> 5),
//    first-occurrence flags, __ballot_sync/__popc.
#include "sel_device.cuh"
#include "sel_internal.h"

namespace sel {

struct CountArgs {
    const sel_nest* nests;
    const sel_access* acc;
    const uint32_t* prob_nest;
    const uint32_t* prob_B;
    const unsigned long long* prefix;   // exclusive prefix of W per problem, [n_problems] = total
    const unsigned long long* prob_WR;
    unsigned long long* prob_cnt;       // W, L, S, C, U per problem
    WsHeader* hdr;
};

// per-warp accumulators for the problem being counted
struct Acc {
    uint32_t LfA;        // per lane: line flags of tmin = 1 accesses
    uint32_t Sf;         // per lane: sector flags of all accesses (RESIDUE)
    uint64_t W1, C1;     // uniform: WAs / coalesced WAs of tmin = 1 accesses
    uint64_t W2, C2, L2, U2;   // uniform: tmin > 1 accesses (lines counted exactly)
    uint64_t Lm, Sm;     // uniform: MATCH path totals
};

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// q with prefix[q] <= x < prefix[q+1]; warp-cooperative 32-ary search
__device__ __forceinline__ uint64_t find_problem(const unsigned long long* prefix, uint64_t nq, uint64_t x,
                                                 int lane) {
    uint64_t lo = 0, hi = nq;
    while (hi - lo > 1) {
        const uint64_t span = hi - lo;
        const uint64_t pos = lo + (span * uint64_t(lane + 1)) / 33;
        const bool le = (pos == lo) ? true : (prefix[pos] <= x);
        const unsigned m = __ballot_sync(kFull, le);
        const int k = __popc(m);                      // le holds for lanes [0, k)
        const uint64_t nlo = __shfl_sync(kFull, pos, (k + 31) & 31);
        const uint64_t nhi = __shfl_sync(kFull, pos, k & 31);
        if (k > 0) lo = nlo;
        if (k < 32) hi = nhi;
    }
    return lo;
}

__device__ __forceinline__ int64_t bitonic_sort_warp(int64_t key, int lane) {
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const int64_t other = __shfl_xor_sync(kFull, key, j);
            const bool up = (lane & k) == 0;
            const bool lower = (lane & j) == 0;
            const int64_t mn = key < other ? key : other;
            const int64_t mx = key < other ? other : key;
            key = (lower == up) ? mn : mx;
        }
    }
    return key;
}

// lane address of warp-rep m, without the inner-loop part; sets n (active lanes)
__device__ __forceinline__ int64_t lane_address(const sel_nest& nest, const sel_access& a, uint64_t P, uint32_t B,
                                                uint64_t m, int lane, int* n_out) {
    uint64_t p0;
    uint32_t n;
    if ((B & 31u) == 0) {
        p0 = m * 32;
        n = uint32_t(umin64(32, P - p0));
    } else {
        const uint32_t wpb = (B + 31) >> 5;
        const uint64_t kb = m / wpb;
        const uint32_t w = uint32_t(m - kb * wpb);
        p0 = kb * B + 32ull * w;
        n = uint32_t(umin64(umin64(32, B - 32 * w), P - p0));
    }
    *n_out = int(n);
    const uint64_t p = p0 + uint64_t(lane < int(n) ? lane : 0);
    if (nest.par_dims == 1) return a.base + a.c_par[0] * int64_t(p);
    return a.base + a.c_par[0] * int64_t(p / nest.P1) + a.c_par[1] * int64_t(p % nest.P1);
}

// ----------------------------------------------------------- RESIDUE loops
template <bool T1>
__device__ __forceinline__ void hot_residue(uint32_t y, uint32_t step, uint32_t dl, uint32_t ds, uint64_t len,
                                            int tmin, Acc& acc) {
    uint32_t lf = 0, sf = 0, c = 0;
    uint64_t l2 = 0, u2 = 0;
#pragma unroll 4
    for (uint64_t i = 0; i < len; i++) {
        const bool fl = y < dl;
        const bool fs = (y << 2) < ds;
        sf += fs;
        if (T1) {
            lf += fl;
            c += !__any_sync(kFull, fl);
        } else {
            const int lines = __popc(__ballot_sync(kFull, fl)) + 1;
            const bool coal = lines <= tmin;
            c += coal;
            l2 += lines;
            u2 += coal ? 0 : lines;
        }
        y += step;
    }
    acc.Sf += sf;
    if (T1) {
        acc.LfA += lf;
        acc.W1 += len;
        acc.C1 += c;
    } else {
        acc.W2 += len;
        acc.C2 += c;
        acc.L2 += l2;
        acc.U2 += u2;
    }
}

template <bool T1>
__device__ __forceinline__ void hot_match(int64_t addr, int64_t step, uint64_t len, int tmin, Acc& acc) {
    const unsigned lt = lanemask_lt();
    uint64_t L = 0, S = 0, C = 0, U = 0;
    for (uint64_t i = 0; i < len; i++) {
        const unsigned ml = __match_any_sync(kFull, (unsigned long long)(addr >> 7));
        const unsigned ms = __match_any_sync(kFull, (unsigned long long)(addr >> 5));
        const int lines = __popc(__ballot_sync(kFull, (ml & lt) == 0));
        const int sectors = __popc(__ballot_sync(kFull, (ms & lt) == 0));
        const bool coal = lines <= tmin;
        L += lines;
        S += sectors;
        C += coal;
        U += coal ? 0 : lines;
        addr += step;
    }
    acc.Lm += L;
    acc.Sm += S;
    acc.W1 += len;
    acc.C1 += C;
    acc.U2 += U;
}

// Count WAs [off, off + cnt) of access `a` of a problem (instance order:
// warp-rep m, then inner tuple with the last inner loop fastest).
template <bool MATCH>
__device__ void count_access(const sel_nest& nest, const sel_access& a, uint64_t P, uint32_t B,
                             const uint64_t* T, uint64_t Mk, uint64_t off, uint64_t cnt, int lane, Acc& acc) {
    const int depth = a.depth;
    const int tmin = (32 * int(a.elem_bytes) + 127) / 128;        // R11
    uint64_t m = off / Mk;
    uint64_t tt = off - m * Mk;
    uint64_t idx[3] = {0, 0, 0};
    {
        uint64_t r = tt;
        for (int j = depth - 1; j >= 0; j--) {
            idx[j] = r % T[j];
            r /= T[j];
        }
    }
    const int64_t c_last = depth ? a.c_inner[depth - 1] : 0;
    const uint64_t T_last = depth ? T[depth - 1] : 1;
    while (cnt > 0) {
        int n;
        const int64_t A = lane_address(nest, a, P, B, m, lane, &n);
        // per-warp-rep setup
        uint32_t u_low = 0, dl = 0, ds = 0;
        int64_t Am = A;
        if (!MATCH) {
            int64_t upper;
            uint64_t gap;
            bool has;
            if (nest.par_dims == 1) {
                const int64_t c0 = a.c_par[0];
                upper = A + (c0 < 0 ? -c0 : 0);     // larger address of the pair (l-1, l)
                gap = uabs(c0);
                has = lane >= 1 && lane < n;
            } else {
                const int64_t key = bitonic_sort_warp(lane < n ? A : INT64_MAX, lane);
                const int64_t prev = __shfl_up_sync(kFull, key, 1);
                upper = key;
                gap = uint64_t(key - prev);
                has = lane >= 1 && lane < n;
            }
            u_low = uint32_t(upper);
            dl = has ? (gap >= 128 ? 0xffffffffu : uint32_t(gap) << 25) : 0u;
            ds = has ? (gap >= 32 ? 0xffffffffu : uint32_t(gap) << 27) : 0u;
        } else {
            const int64_t a0 = __shfl_sync(kFull, A, 0);
            Am = lane < n ? A : a0;                 // inactive lanes duplicate lane 0
        }
        const uint64_t here = umin64(Mk - tt, cnt);
        uint64_t left = here;
        while (left > 0) {
            int64_t D = 0;
            for (int j = 0; j < depth; j++) D += a.c_inner[j] * int64_t(idx[j]);
            const uint64_t i_last = depth ? idx[depth - 1] : 0;
            const uint64_t len = umin64(T_last - i_last, left);
            if (MATCH) {
                if (tmin == 1) hot_match<true>(Am + D, c_last, len, tmin, acc);
                else hot_match<false>(Am + D, c_last, len, tmin, acc);
            } else {
                const uint32_t y = (u_low + uint32_t(uint64_t(D))) << 25;
                const uint32_t step = uint32_t(uint64_t(c_last)) << 25;
                if (tmin == 1) hot_residue<true>(y, step, dl, ds, len, tmin, acc);
                else hot_residue<false>(y, step, dl, ds, len, tmin, acc);
            }
            left -= len;
            // odometer carry
            if (depth) {
                idx[depth - 1] += len;
                int j = depth - 1;
                while (j >= 0 && idx[j] >= T[j]) {
                    idx[j] = 0;
                    if (j > 0) idx[j - 1] += 1;
                    j--;
                }
            }
        }
        cnt -= here;
        m += 1;
        tt = 0;
    }
}

template <bool MATCH>
__device__ void flush(const CountArgs& a, uint64_t q, Acc& acc, int lane) {
    const uint32_t sumLfA = __reduce_add_sync(kFull, acc.LfA);
    const uint32_t sumSf = __reduce_add_sync(kFull, acc.Sf);
    const uint64_t W = acc.W1 + acc.W2;
    uint64_t L, S, C, U;
    if (MATCH) {
        L = acc.Lm;
        S = acc.Sm;
        C = acc.C1;
        U = acc.U2;
    } else {
        L = acc.W1 + sumLfA + acc.L2;
        S = W + sumSf;
        C = acc.C1 + acc.C2;
        U = (acc.W1 - acc.C1) + sumLfA + acc.U2;
    }
    if (W && lane < 5) {
        const uint64_t v = lane == 0 ? W : lane == 1 ? L : lane == 2 ? S : lane == 3 ? C : U;
        atomicAdd(&a.prob_cnt[q * 5 + lane], (unsigned long long)v);
    }
    acc = Acc{};
}

template <bool MATCH>
__device__ void count_problem(const CountArgs& a, uint64_t q, uint64_t off, uint64_t take, int lane) {
    const sel_nest nest = a.nests[a.prob_nest[q]];
    const uint32_t B = a.prob_B[q];
    const uint64_t WR = a.prob_WR[q];
    const uint64_t P = nest.P0 * nest.P1;
    uint64_t T[3];
    for (int j = 0; j < 3; j++) T[j] = eff_trip(nest.trip[j]);
    Acc acc{};
    for (uint32_t k = 0; k < nest.n_access && take > 0; k++) {
        const sel_access ac = a.acc[nest.access_off + k];
        uint64_t Mk = 1;
        for (int j = 0; j < ac.depth; j++) Mk *= T[j];
        const uint64_t Wk = WR * Mk;
        if (off >= Wk) {
            off -= Wk;
            continue;
        }
        const uint64_t t = umin64(Wk - off, take);
        count_access<MATCH>(nest, ac, P, B, T, Mk, off, t, lane, acc);
        take -= t;
        off = 0;
    }
    flush<MATCH>(a, q, acc, lane);
}

template <bool MATCH>
__global__ void __launch_bounds__(256, 4) k_count(CountArgs a) {
    const int lane = threadIdx.x & 31;
    const uint64_t nq = a.hdr->n_problems;
    if (nq == 0) return;
    const uint64_t total = a.prefix[nq];
    if (total == 0) return;
    const uint64_t nwarps = uint64_t(gridDim.x) * (blockDim.x >> 5);
    uint64_t ch = total / (nwarps * 16);
    ch = ch < 256 ? 256 : (ch > (1ull << 20) ? (1ull << 20) : ch);
    for (;;) {
        unsigned long long chunk = 0;
        if (lane == 0) chunk = atomicAdd(&a.hdr->chunk_ctr, 1ull);
        chunk = __shfl_sync(kFull, chunk, 0);
        const uint64_t start = chunk * ch;
        if (start >= total) break;
        uint64_t len = umin64(ch, total - start);
        uint64_t q = find_problem(a.prefix, nq, start, lane);
        uint64_t off = start - a.prefix[q];
        while (len > 0) {
            const uint64_t Wq = a.prefix[q + 1] - a.prefix[q];
            if (off >= Wq) {
                off -= Wq;
                q++;
                continue;
            }
            const uint64_t take = umin64(Wq - off, len);
            count_problem<MATCH>(a, q, off, take, lane);
            len -= take;
            off = 0;
            q++;
        }
    }
}

cudaError_t launch_count(const sel_tables& t, const WsPtrs& w, uint64_t max_problems, uint32_t flags,
                         cudaStream_t s) {
    (void)max_problems;
    static int grid[2] = {0, 0};
    const bool match = (flags & SEL_F_MATCH_ANY) != 0;
    int& g = grid[match ? 1 : 0];
    if (g == 0) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (match) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_count<true>, 256, 0);
        else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_count<false>, 256, 0);
        g = sms * (per > 0 ? per : 1);
    }
    CountArgs a{t.nests, t.accesses, w.prob_nest, w.prob_B, w.prob_W, w.prob_WR, w.prob_cnt, w.hdr};
    prof_before_count(s);
    if (match) k_count<true><<<g, 256, 0, s>>>(a);
    else k_count<false><<<g, 256, 0, s>>>(a);
    prof_after_count(s);
    note_launch();
    return cudaGetLastError();
}

}  // namespace sel
