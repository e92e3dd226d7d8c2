// sel_device.cuh -- device-side helpers shared by the libsel kernels:
// validation rules V1-V7, launch geometry (a1,
// P:L225; readings R6-R9, R27) and the workspace layout.  No host code.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/sel.h"

namespace sel {

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint64_t kLim62 = 1ull << 62;
constexpr uint64_t kLim48 = 1ull << 48;
constexpr uint64_t kLim40 = 1ull << 40;
constexpr uint32_t kNoProblem = 0xffffffffu;
constexpr int kSlots = 8;              // distinct B classes shared per nest before overflow
constexpr uint32_t kClsMax = 1024;     // launch tables up to this size use direct problem ids
#ifndef SEL_CNT_STRIDE
#define SEL_CNT_STRIDE 6
#endif
constexpr int kCntStride = SEL_CNT_STRIDE;   // per problem: W, L, S, C, U (atomic), M_it (closed form)[, pad]
constexpr size_t kProbModelBytes = 112; // per problem: the candidate-independent part of a4 (sel_model.cu)

// ------------------------------------------------------------------ workspace
// All offsets are 256-byte aligned.  Sized for the worst case of one counting
// problem per candidate.
struct WsHeader {
    sel_stats stats;                   // 64 B, read by sel_read_stats
    unsigned long long n_problems;     // device-side problem count
    unsigned long long chunk_ctr;      // dynamic work counter of the count kernel
    unsigned int n_overflow;           // problems allocated past the slot table
    unsigned int _pad0;
    unsigned long long w_begin, w_end; // this call's slice of the problem work space (prefix units)
    unsigned int part, n_parts;        // sel_count_transactions_part: slice index / count
    unsigned long long small_begin, small_end;   // this call's range of lane-parallel (small) problems
    unsigned long long queue_len;      // problems handed from the lane kernel to the warp kernel
    unsigned long long queue_ctr;      // dynamic work counter of the warp (queue) kernel
    unsigned int direct;               // 1: problem id = nest * n_cls + class of the launch (k_classes)
    unsigned int n_cls;                // distinct B classes of the launch table (direct mode)
    unsigned long long n_nests_scan;   // nests scanned by the slot-table path (0 in direct mode)
    unsigned long long n_big;          // direct mode: problems counted through the WA prefix (k_count)
    unsigned int skip_scan;            // direct mode without big problems: the W prefix is all zero
    unsigned int _pad1;
    unsigned long long _pad[2];
};
static_assert(sizeof(WsHeader) == 256, "header size");

struct WsLayout {
    size_t hdr, slots, nest_base, cand_pid, prob_nest, prob_B, prob_W, prob_WR, prob_cnt,
        prob_status, cand_status, queue, prob_used, prob_md, cls, nest_key, lane_info, scan_tmp, total;
};

__host__ __device__ inline size_t ws_align(size_t x) { return (x + 255) & ~size_t(255); }

// Number of scan partial sums for n items (kScanItems per block).
constexpr int kScanThreads = 256;
constexpr int kScanPer = 8;
constexpr uint64_t kScanItems = uint64_t(kScanThreads) * kScanPer;
__host__ __device__ inline uint64_t scan_blocks(uint64_t n) { return (n + kScanItems) / kScanItems + 1; }

__host__ __device__ inline WsLayout ws_layout(uint64_t n, uint64_t n_nests, uint32_t flags) {
    WsLayout L{};
    bool dedup = !(flags & SEL_F_NO_DEDUP);
    size_t o = 0;
    L.hdr = o;        o = ws_align(o + sizeof(WsHeader));
    L.slots = o;      o = ws_align(o + (dedup ? n_nests * kSlots * sizeof(uint32_t) : 0));
    L.nest_base = o;  o = ws_align(o + (dedup ? (n_nests + 1) * sizeof(uint64_t) : 0));
    L.cand_pid = o;   o = ws_align(o + n * sizeof(uint32_t));
    L.prob_nest = o;  o = ws_align(o + n * sizeof(uint32_t));
    L.prob_B = o;     o = ws_align(o + n * sizeof(uint32_t));
    L.prob_W = o;     o = ws_align(o + (n + 1) * sizeof(uint64_t));
    L.prob_WR = o;    o = ws_align(o + n * sizeof(uint64_t));
    L.prob_cnt = o;   o = ws_align(o + n * kCntStride * sizeof(uint64_t));
    L.prob_status = o; o = ws_align(o + n);
    L.cand_status = o; o = ws_align(o + n);
    L.queue = o;      o = ws_align(o + n * sizeof(uint64_t));
    L.prob_used = o;  o = ws_align(o + n);
    L.prob_md = o;    o = ws_align(o + n * kProbModelBytes);
    L.cls = o;        o = ws_align(o + 2 * kClsMax * sizeof(uint32_t));
    L.nest_key = o;   o = ws_align(o + n);
    L.lane_info = o;  o = ws_align(o + (dedup ? n_nests * 8 : 0));
    uint64_t big = n > n_nests ? n : n_nests;
    L.scan_tmp = o;   o = ws_align(o + scan_blocks(big) * sizeof(uint64_t) * 2);
    L.total = o;
    return L;
}

// ------------------------------------------------------------------- basics
__device__ __forceinline__ uint64_t eff_trip(uint32_t t) {
    return t == SEL_TRIP_UNKNOWN ? 128ull : uint64_t(t);
}
// a / b with a 32-bit fast path (the common case: both operands below 2^32;
// the 64-bit division is a long software sequence)
__device__ __forceinline__ uint64_t udiv(uint64_t a, uint64_t b) {
    if (((a | b) >> 32) == 0) return uint32_t(a) / uint32_t(b);
    return a / b;
}
__device__ __forceinline__ uint64_t cdiv(uint64_t a, uint64_t b) {
    const uint64_t q = udiv(a, b);
    return q + (a - q * b != 0);
}
__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint64_t smul(uint64_t a, uint64_t b) {
    if (((a | b) >> 32) == 0) return a * b;               // both below 2^32: no overflow (the common case)
    if (a == 0 || b == 0) return 0;
    return __umul64hi(a, b) ? ~0ull : a * b;               // saturate on overflow
}
__device__ __forceinline__ uint64_t sadd(uint64_t a, uint64_t b) { return (a > ~0ull - b) ? ~0ull : a + b; }
__device__ __forceinline__ uint64_t uabs(int64_t v) { return v < 0 ? 0ull - uint64_t(v) : uint64_t(v); }

// B class for count sharing: counts depend on B only when 32 does not divide
// it (every warp is then an aligned 32-iteration chunk of p-space), and never
// on G_max or the device.
__device__ __forceinline__ uint32_t b_class(uint32_t B) { return (B & 31u) == 0 ? 32u : B; }

// Candidate-level checks V1, V2 (ids, host clock, launch bounds).
__device__ __forceinline__ uint8_t validate_candidate(const sel_candidate& c, const sel_tables& t,
                                                      int n_sets) {
    if (c.nest_id >= t.n_nests || c.launch_id >= t.n_launches || c.device_id >= uint32_t(n_sets) ||
        !(c.cpu_hz > 0.0))
        return SEL_EINVAL;
    const sel_launch l = t.launches[c.launch_id];
    if (l.block < 1 || l.block > 1024 || l.grid_max < 1) return SEL_EINVAL;
    return SEL_OK;
}

// Shape key of a nest for the lane kernel's tile sort: accesses, loop depth,
// collapse, how many accesses take each counting path (uniform / residue
// classes depth <= 1 / depth 2 / warp kernel; 8-bit counts in `paths`) and
// which element sizes occur (`emask`), hashed to 8 bits -- threads of a warp
// then run nests whose loops and branches match.  A hint only: collisions mix
// shapes, nothing else.
__device__ __forceinline__ uint8_t nest_shape_key(const sel_nest& n, uint32_t paths, uint32_t emask) {
    const uint32_t na = n.n_access < 31u ? n.n_access : 31u;
    uint32_t h = (na << 3) | (uint32_t(n.depth & 3u) << 1) | (n.par_dims == 2 ? 1u : 0u);
    h = h * 0x9E3779B1u + paths;
    h = h * 0x9E3779B1u + emask;
    return uint8_t((h * 0x9E3779B1u) >> 24);
}
__device__ __forceinline__ uint8_t nest_shape_key(const sel_nest& n) {
    const uint32_t na = n.n_access < 31u ? n.n_access : 31u;
    return uint8_t((na << 3) | (uint32_t(n.depth & 3u) << 1) | (n.par_dims == 2 ? 1u : 0u));
}

// Nest-level checks V3-V6, split so that the accesses can be checked by
// different threads: nest_precheck (structure, P range), access_check (one
// access: element size, depth, divisibility -> kAccInval; address bound ->
// kAccRange; its Mk), nest_status (combines them in validate_nest's order:
// a structural error of any access wins over a range error).
constexpr uint32_t kAccInval = 1u, kAccRange = 2u;
__device__ __forceinline__ uint8_t nest_precheck(const sel_nest& n, uint64_t n_acc_total) {
    if ((n.par_dims != 1 && n.par_dims != 2) || n.depth > 3 || (n.par_dims == 1 && n.P1 != 1) ||
        uint64_t(n.access_off) + uint64_t(n.n_access) > n_acc_total)
        return SEL_EINVAL;
    const uint64_t P = smul(n.P0, n.P1);
    if (n.P0 >= kLim40 || P >= kLim40) return SEL_ERANGE;
    return SEL_OK;
}
// P = P0 P1, T = effective trips of the nest
__device__ __forceinline__ uint32_t access_check(const sel_access& a, uint32_t par_dims, uint32_t depth, uint64_t P,
                                                 uint64_t P0, uint64_t P1, const uint64_t T[3], uint64_t* Mk_out) {
    const int64_t e = a.elem_bytes;
    if (!(e == 1 || e == 2 || e == 4 || e == 8 || e == 16) || a.depth > depth) return kAccInval;
    // power-of-two element size: divisibility by masking
    const int64_t m = e - 1;
    bool bad = (a.base & m) || (a.c_par[0] & m) || (par_dims == 2 && (a.c_par[1] & m));
#pragma unroll
    for (int j = 0; j < 3; j++) bad |= (j < a.depth) && (a.c_inner[j] & m) != 0;   // static indices: no local memory
    if (bad) return kAccInval;
    const uint64_t e0 = (par_dims == 1) ? P : P0;
    {
        // |base| < 2^60, every coefficient below 2^28 and every extent below
        // 2^20: each of the <= 5 product terms is below 2^48, so the bound stays
        // below 2^61 < 2^62 and M_k (<= 3 trips) below 2^60 -- no saturating
        // arithmetic needed (the common case: array bases are large, strides
        // and trip counts small)
        uint64_t coef = uabs(a.c_par[0]), ext = e0;
        if (par_dims == 2) {
            coef |= uabs(a.c_par[1]);
            ext |= P1;
        }
        uint64_t Mk = 1;
#pragma unroll
        for (int j = 0; j < 3; j++)
            if (j < a.depth) {
                coef |= uabs(a.c_inner[j]);
                ext |= T[j];
                Mk *= T[j];
            }
        if (((uabs(a.base) >> 60) | (coef >> 28) | (ext >> 20)) == 0) {
            *Mk_out = Mk;
            return 0u;
        }
    }
    uint64_t bound = uabs(a.base);
    bound = sadd(bound, smul(uabs(a.c_par[0]), e0 ? e0 - 1 : 0));
    if (par_dims == 2) bound = sadd(bound, smul(uabs(a.c_par[1]), P1 ? P1 - 1 : 0));
    uint64_t Mk = 1;
#pragma unroll
    for (int j = 0; j < 3; j++) {
        if (j < a.depth) {
            bound = sadd(bound, smul(uabs(a.c_inner[j]), T[j] ? T[j] - 1 : 0));
            Mk = smul(Mk, T[j]);
        }
    }
    *Mk_out = Mk;
    return bound >= kLim62 ? kAccRange : 0u;
}
__device__ __forceinline__ uint8_t nest_status(uint8_t pre, uint32_t acc_flags, uint64_t P, uint64_t M_it) {
    if (pre) return pre;
    if (acc_flags & kAccInval) return SEL_EINVAL;
    if (acc_flags & kAccRange) return SEL_ERANGE;
    if (smul(P, M_it) >= kLim48) return SEL_ERANGE;
    return SEL_OK;
}

// Nest-level checks V3-V6; on success *M_it = sum_k prod_{j<depth_k} T_j.
__device__ inline uint8_t validate_nest(const sel_nest& n, const sel_access* acc_all, uint64_t n_acc_total,
                                        uint64_t* M_it_out) {
    const uint8_t pre = nest_precheck(n, n_acc_total);
    if (pre) return pre;
    const uint64_t P = smul(n.P0, n.P1);
    uint64_t T[3];
    for (int j = 0; j < 3; j++) T[j] = eff_trip(n.trip[j]);
    const sel_access* acc = acc_all + n.access_off;
    uint32_t flags = 0;
    uint64_t M_it = 0;
    for (uint32_t k = 0; k < n.n_access; k++) {
        uint64_t Mk = 0;
        flags |= access_check(acc[k], n.par_dims, n.depth, P, n.P0, n.P1, T, &Mk);
        if (flags & kAccInval) break;
        M_it = sadd(M_it, Mk);
    }
    const uint8_t st = nest_status(SEL_OK, flags, P, M_it);
    if (st == SEL_OK) *M_it_out = M_it;
    return st;
}


// Problems counted one per lane (k_lane_problems) rather than through the WA
// prefix: 1-D, small enough for 32-bit lane sums and a short warp-rep walk.
constexpr uint64_t kSmallMaxW = 1ull << 24;
constexpr uint64_t kSmallMaxWR = 1024;

// Warps with at least one active lane (R8, R9), summed over the R*G blocks of
// the launch.  Block k covers iterations [kB, kB + B); block-to-grid mapping
// (R7) does not change which iterations share a warp, so WR depends only on
// P and B.
__device__ __forceinline__ uint64_t warp_reps(uint64_t P, uint32_t B) {
    if (P == 0) return 0;
    if ((B & 31u) == 0) return cdiv(P, 32);
    const uint64_t wpb = cdiv(B, 32);
    const uint64_t nb = cdiv(P, B);
    return (nb - 1) * wpb + cdiv(P - (nb - 1) * B, 32);
}

}  // namespace sel
