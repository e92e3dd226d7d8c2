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
// one div/mod) and then walks with odometer steps.  A chunk holds at most
// 2^20 WAs, so every accumulator is 32-bit until the per-chunk flush.
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
//    bitonic network.  lines = 1 + #flags.  Line flags of 32 consecutive
//    WAs are collected as per-lane bitmasks and classified with one warp
//    reduction per group (see "hot loops" below).
//  * MATCH (SEL_F_MATCH_ANY).  The north star's literal primitive: full
//    64-bit lane addresses, __match_any_sync on (addr >> 7) and (addr >> 5),
//    first-occurrence flags, __ballot_sync/__popc.
#include "sel_device.cuh"
#include "sel_internal.h"

namespace sel {

constexpr uint64_t kMaxChunk = 1ull << 20;   // WAs per chunk: keeps all accumulators 32-bit
#ifndef SEL_COUNT_MIN_BLOCKS
#define SEL_COUNT_MIN_BLOCKS 3
#endif
#ifndef SEL_COUNT_THREADS
#define SEL_COUNT_THREADS 256
#endif
#ifndef SEL_HIST_MIN_MK
#define SEL_HIST_MIN_MK 32
#endif
constexpr uint64_t kHistMinMk = SEL_HIST_MIN_MK;
// Nominal algorithmic integer lane-ops of each counting path,
// summed by the kernels into sel_stats.alg_lane_ops (the roofline numerator):
constexpr uint32_t kOpsExpandWA = 224;   // lane-by-lane expansion, per WA (7 ops x 32 lanes)
constexpr uint32_t kOpsArithWA = 12;     // arithmetic lanes, per WA: residue 2, lines 2, sectors 3, class 2, sums 3
constexpr uint32_t kOpsClass = 6;        // uniform flags, per (access, lane-count class): lines, class, 4 sums
constexpr uint32_t kOpsHistEntry = 6;    // residue histogram of one loop, per entry: residue 3, count 3
constexpr uint32_t kOpsConvTerm = 5;     // histogram convolution, per (iteration, residue): index 4, MAC 1
constexpr uint32_t kOpsPrefixEntry = 3;  // prefix sums of a residue histogram, per entry
constexpr uint32_t kOpsEvalClass = 24;   // one residue class from the prefix sums: 2 cyclic range sums + sums
// per-warp shared words of a residue histogram: h / its exclusive prefix pf[0..R]
// at [0, 129), the prefix of h folded mod 32 bytes p32[0..R/4] at [kP32Off, +33)
constexpr uint32_t kP32Off = 132;
constexpr uint32_t kHistWords = 168;

struct CountArgs {
    const sel_nest* nests;
    const sel_access* acc;
    const uint32_t* prob_nest;
    const uint32_t* prob_B;
    const unsigned long long* prefix;   // exclusive prefix of W per problem, [n_problems] = total
    const unsigned long long* prob_WR;
    unsigned long long* prob_cnt;       // W, L, S, C, U per problem
    WsHeader* hdr;
    uint32_t one;                       // 1 at run time: keeps adds as IMAD on the FMA pipe
    uint32_t closed_form;               // resolve warp-reps with uniform lane flags in closed form
    uint32_t residue_classes;           // whole arithmetic-lane warp-reps by residue classes (count_hist)
    unsigned long long* queue;          // small problems handed from k_lane_problems to k_queue
    const uint8_t* nest_key;            // direct mode: shape key per nest (k_problem_w)
    const uint2* lane_info;             // direct mode: per nest (M_it, mask of classes < 32 counted here)
    const uint32_t* cls_B;              // direct mode: B class of each class index
};

// nest and block size of problem q: derived from the id in direct mode
// (q = nest * n_cls + class; k_problem_w does not materialise them there),
// the plan's tables otherwise
__device__ __forceinline__ void problem_nest_B(const CountArgs& a, uint64_t q, uint32_t& nid, uint32_t& B) {
    if (a.hdr->direct) {
        const uint32_t nc = a.hdr->n_cls;
        nid = uint32_t(q / nc);
        B = a.cls_B[q - uint64_t(nid) * nc];
    } else {
        nid = a.prob_nest[q];
        B = a.prob_B[q];
    }
}

// Accumulators of one warp for the problem being counted (<= kMaxChunk WAs).
//   L = W + sum_lanes(lf) + lk      S = W + sum_lanes(sf) + sk
//   C = C                           U = (W - C) + sum_lanes(uf) + uk
// lf / sf: per-lane line / sector flags (a lane whose line or sector differs
// from its sorted predecessor's); uf: line flags of uncoalesced WAs.
// lk, sk, uk: the same quantities accumulated warp-uniformly (tmin = 4 and
// MATCH paths).
struct Acc {
    uint32_t lf, sf, uf;             // per lane
    uint32_t cc;                     // per lane: coalesced WAs (arithmetic-lane path)
    uint32_t W, C, lk, sk, uk;       // uniform
    uint32_t K, Q, H;                // uniform statistics: WAs in closed form / arithmetic lanes / residue classes
    uint32_t ops;                    // per lane: nominal algorithmic lane-ops (summed at the flush)
};
// Per-lane partial sums returned by the out-of-line 1-D paths (by value, so
// the caller's accumulators stay in registers): line flags, sector flags,
// coalesced WAs, line flags of uncoalesced WAs, WAs done lane by lane.
struct Part {
    uint32_t lf, sf, cc, uf, q, ops;
};
__device__ __forceinline__ void add_part(Acc& acc, const Part& p) {
    acc.lf += p.lf;
    acc.sf += p.sf;
    acc.cc += p.cc;
    acc.uf += p.uf;
    acc.ops += p.ops;
}

__device__ __forceinline__ uint32_t lane0(int lane, uint32_t x) { return lane == 0 ? x : 0u; }

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

// ------------------------------------------------------------- hot loops
// RESIDUE.  Per lane and WA: line flag  y < dl,  sector flag  (y << 2) < ds.
// WAs are processed in groups of up to 32 consecutive inner iterations: each
// lane sets bit i of m when it has a line flag in WA i of the group, so the
// class of the 32 WAs needs one warp reduction per group instead of a vote
// per WA (coalesced <=> lines <= tmin <=> #flags <= tmin - 1, R11):
//   tmin = 1: uncoalesced WAs = OR over lanes of m
//   tmin = 2: uncoalesced WAs = OR over lanes of (m & exclusive-prefix-OR of m)
//             (bit i set <=> at least two lanes flag WA i)
// tmin = 4 (16-byte elements) keeps a per-WA ballot + popc.

// one WA of a group: bit `bit` of m, sector flag count
__device__ __forceinline__ void wa_step(uint32_t& m, uint32_t& sf, uint32_t y, uint32_t dl, uint32_t ds,
                                        uint32_t bit) {
    const uint32_t z = y << 2;
    asm("{\n\t.reg .pred pl, ps;\n\t"
        "setp.lt.u32 pl, %2, %4;\n\t"
        "setp.lt.u32 ps, %3, %5;\n\t"
        "@pl or.b32 %0, %0, %6;\n\t"
        "@ps add.u32 %1, %1, 1;\n\t}"
        : "+r"(m), "+r"(sf)
        : "r"(y), "r"(z), "r"(dl), "r"(ds), "r"(bit));
}

template <int TC>
__device__ __forceinline__ void group_end(uint32_t m, uint32_t g, Acc& a) {
    uint32_t unc;
    if (TC == 1) {
        unc = __reduce_or_sync(kFull, m);
    } else {
        uint32_t x = m;                                   // inclusive prefix OR over lanes
        const int lane = threadIdx.x & 31;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(kFull, x, o);
            if (lane >= o) x |= t;
        }
        uint32_t ex = __shfl_up_sync(kFull, x, 1);
        if (lane == 0) ex = 0;
        unc = __reduce_or_sync(kFull, m & ex);
    }
    a.lf += __popc(m);
    a.uf += __popc(m & unc);
    a.C += g - __popc(unc);
    a.W += g;
}

template <int TC>
__device__ __forceinline__ void hot_row(uint32_t y, uint32_t step, uint32_t dl, uint32_t ds, uint32_t len,
                                        Acc& a) {
    // four independent accumulator chains (ILP): WA i of a group uses chain i & 3
    uint32_t s0 = 0, s1 = 0, s2 = 0, s3 = 0;
    while (len >= 32) {                                   // full groups: bits are immediates
        uint32_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
#pragma unroll
        for (int i = 0; i < 32; i += 4) {
            wa_step(m0, s0, y + uint32_t(i) * step, dl, ds, 1u << i);
            wa_step(m1, s1, y + uint32_t(i + 1) * step, dl, ds, 2u << i);
            wa_step(m2, s2, y + uint32_t(i + 2) * step, dl, ds, 4u << i);
            wa_step(m3, s3, y + uint32_t(i + 3) * step, dl, ds, 8u << i);
        }
        y += 32u * step;
        group_end<TC>((m0 | m1) | (m2 | m3), 32, a);
        len -= 32;
    }
    if (len) {                                            // partial group
        uint32_t m0 = 0, m1 = 0, bit = 1;
        uint32_t i = 0;
        for (; i + 2 <= len; i += 2) {
            wa_step(m0, s0, y, dl, ds, bit);
            wa_step(m1, s1, y + step, dl, ds, bit << 1);
            bit <<= 2;
            y += 2u * step;
        }
        if (i < len) wa_step(m0, s2, y, dl, ds, bit);
        group_end<TC>(m0 | m1, len, a);
    }
    a.sf += (s0 + s1) + (s2 + s3);
}

// tmin = 4: per-WA ballot + popc
__device__ __forceinline__ void hot_row_t4(uint32_t y, uint32_t step, uint32_t dl, uint32_t ds, uint32_t len,
                                           Acc& a) {
    uint32_t sf = a.sf, c = 0, lk = 0, uk = 0;
    for (uint32_t i = 0; i < len; i++) {
        const uint32_t z = y << 2;
        const uint32_t k = __popc(__ballot_sync(kFull, y < dl));
        sf += z < ds;
        lk += k;
        const bool coal = k <= 3;
        c += coal;
        uk += coal ? 0 : k;
        y += step;
    }
    a.sf = sf;
    a.C += c;
    a.lk += lk;
    a.uk += uk;
    a.W += len;
}

// RESIDUE, byte-sliced (SWAR, default).  The line residue r = (s_l + D) mod
// 128 of four consecutive WAs sits in the four bytes of one register (bit 7
// of each byte clear).  For a per-lane threshold d <= 128 (gap, capped),
//   T = R + (0x80808080 - d * 0x01010101)
// never borrows across bytes (r + 128 - d >= 0) and bit 7 of byte j is set
// iff r_j >= d, i.e. iff WA j has NO line flag; the same with r mod 32 and
// d_s <= 32 for sectors.  Byte j of quad q of a group is WA 4q + j; its flag
// is moved to bit 8j + q of the group mask (shift by 7 - q, mask
// 0x01010101 << q), so the per-group classification of hot_row applies
// unchanged.  9 lane ops per quad: 2.25 per WA and lane.
// Pipe balance: the adds and the right shifts run on the FMA pipe (IMAD with
// a runtime `one`, IMAD.HI by 2^(25+q)), the masks on the ALU pipe (LOP3):
// 5 FMA + 4 ALU ops per quad instead of 9 ALU ops.
__device__ __forceinline__ uint32_t add_fma(uint32_t a, uint32_t b, uint32_t one) {
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
    return d;
}

#ifndef SEL_SWAR_FMA_ADD
#define SEL_SWAR_FMA_ADD 0
#endif
#ifndef SEL_SWAR_FMA_SHIFT
#define SEL_SWAR_FMA_SHIFT 0
#endif
__device__ __forceinline__ uint32_t swar_add(uint32_t a, uint32_t b, uint32_t one) {
    if (SEL_SWAR_FMA_ADD) return add_fma(a, b, one);
    (void)one;
    return a + b;
}

__device__ __forceinline__ void swar_quad(uint32_t R, uint32_t KL, uint32_t KS, uint32_t q, uint32_t valid,
                                          uint32_t one, uint32_t& m, uint32_t& ms) {
    const uint32_t T = swar_add(R, KL, one);                 // bit 7 of byte j: no line flag
    const uint32_t Ts = swar_add(R & 0x1F1F1F1Fu, KS, one);  // bit 7 of byte j: no sector flag
    const uint32_t sel = (0x01010101u << q) & valid;
    uint32_t x, xs;                                          // T >> (7 - q)
    if (SEL_SWAR_FMA_SHIFT && q != 7) {
        x = __umulhi(T, 1u << (25 + q));
        xs = __umulhi(Ts, 1u << (25 + q));
    } else {
        x = T >> (7 - q);
        xs = Ts >> (7 - q);
    }
    m |= ~x & sel;
    ms |= ~xs & sel;
}

template <int TC>
__device__ __forceinline__ void hot_row_swar(uint32_t r0, uint32_t cr, uint32_t KL, uint32_t KS, uint32_t len,
                                             uint32_t one, Acc& a) {
    const uint32_t S4 = ((4u * cr) & 127u) * 0x01010101u;  // per-byte residue step of 4 WAs
    // bytes r0 + j*cr (mod 128), j = 0..3
    uint32_t R = (r0 & 127u) | (((r0 + cr) & 127u) << 8) | (((r0 + 2u * cr) & 127u) << 16) |
                 (((r0 + 3u * cr) & 127u) << 24);
    uint32_t sf = 0;
#ifndef SEL_SWAR_CHAINS
#define SEL_SWAR_CHAINS 1
#endif
    const uint32_t S8 = ((8u * cr) & 127u) * 0x01010101u;
    while (len >= 32) {                                     // full groups: shifts are immediates
        uint32_t m = 0, ms = 0;
        if (SEL_SWAR_CHAINS == 2) {                         // two independent residue chains (ILP)
            uint32_t Rb = swar_add(R, S4, one) & 0x7F7F7F7Fu;
#pragma unroll
            for (int q = 0; q < 8; q += 2) {
                swar_quad(R, KL, KS, uint32_t(q), 0xffffffffu, one, m, ms);
                swar_quad(Rb, KL, KS, uint32_t(q + 1), 0xffffffffu, one, m, ms);
                R = swar_add(R, S8, one) & 0x7F7F7F7Fu;
                Rb = swar_add(Rb, S8, one) & 0x7F7F7F7Fu;
            }
        } else {
#pragma unroll
            for (int q = 0; q < 8; q++) {
                swar_quad(R, KL, KS, uint32_t(q), 0xffffffffu, one, m, ms);
                R = swar_add(R, S4, one) & 0x7F7F7F7Fu;
            }
        }
        group_end<TC>(m, 32, a);
        sf += __popc(ms);
        len -= 32;
    }
    if (len) {                                              // partial group
        uint32_t m = 0, ms = 0, q = 0;
        for (uint32_t i = 0; i < len; i += 4, q++) {
            const uint32_t k = len - i;                     // WAs left; bytes >= k are past the row
            const uint32_t valid = k >= 4 ? 0xffffffffu : (1u << (8 * k)) - 1u;
            swar_quad(R, KL, KS, q, valid, one, m, ms);
            R = swar_add(R, S4, one) & 0x7F7F7F7Fu;
        }
        group_end<TC>(m, len, a);
        sf += __popc(ms);
    }
    a.sf += sf;
}

// MATCH: literal __match_any_sync expansion over 64-bit lane addresses.
__device__ __forceinline__ void hot_match(int64_t addr, int64_t step, uint32_t len, uint32_t tmin, Acc& a) {
    const unsigned lt = lanemask_lt();
    uint32_t L = 0, S = 0, C = 0, U = 0;
    for (uint32_t i = 0; i < len; i++) {
        const unsigned ml = __match_any_sync(kFull, (unsigned long long)(addr >> 7));
        const unsigned ms = __match_any_sync(kFull, (unsigned long long)(addr >> 5));
        const uint32_t lines = __popc(__ballot_sync(kFull, (ml & lt) == 0));
        const uint32_t sectors = __popc(__ballot_sync(kFull, (ms & lt) == 0));
        const bool coal = lines <= tmin;
        L += lines - 1;
        S += sectors - 1;
        C += coal;
        U += coal ? 0 : lines - 1;
        addr += step;
    }
    a.lk += L;
    a.sk += S;
    a.uk += U;
    a.C += C;
    a.W += len;
}

// --------------------------------------------------------- warp iterator
// Enumerates the active warps of a problem (R8, R9): block k covers
// iterations [kB, kB + B) and holds ceil(B/32) warps, the last one partial
// when 32 does not divide B; warps past P are skipped (WR counts the rest).
struct WarpIter {
    uint64_t p0;        // first iteration of the warp
    uint64_t blk_end;   // end of the current block's iterations
    uint32_t n;         // active lanes
};

__device__ __forceinline__ void warp_seek(WarpIter& it, uint64_t m, uint64_t P, uint32_t B) {
    if ((B & 31u) == 0) {
        it.p0 = m * 32;
        it.blk_end = ~0ull;
    } else {
        const uint32_t wpb = (B + 31) >> 5;
        const uint64_t kb = udiv(m, wpb);
        const uint32_t w = uint32_t(m - kb * wpb);
        it.p0 = kb * B + 32ull * w;
        it.blk_end = (kb + 1) * B;
    }
    uint64_t e = it.p0 + 32;
    if (e > it.blk_end) e = it.blk_end;
    if (e > P) e = P;
    it.n = uint32_t(e - it.p0);
}

__device__ __forceinline__ void warp_next(WarpIter& it, uint64_t P, uint32_t B) {
    uint64_t p = it.p0 + 32;
    if (p >= it.blk_end) {               // next block (only when 32 does not divide B)
        p = it.blk_end;
        it.blk_end += B;
    }
    it.p0 = p;
    uint64_t e = p + 32;
    if (e > it.blk_end) e = it.blk_end;
    if (e > P) e = P;
    it.n = uint32_t(e - p);
}

// lane address of the current warp without the inner-loop part (a2, R25)
__device__ __forceinline__ int64_t lane_address(const sel_nest& nest, const sel_access& a, const WarpIter& it,
                                                int lane) {
    const uint64_t p = it.p0 + uint64_t(lane < int(it.n) ? lane : 0);
    if (nest.par_dims == 1) return a.base + a.c_par[0] * int64_t(p);
    return a.base + a.c_par[0] * int64_t(p / nest.P1) + a.c_par[1] * int64_t(p % nest.P1);
}


// ------------------------------------------------------------- uniform flags
// A 1-D parallel stride g of 0 or >= 128 bytes gives every active lane after
// the first a line and a sector flag (g >= 128) or none (g = 0) in every
// warp-access, independently of the inner offset: a warp-rep with n active
// lanes has lines = sectors = 1 + (g ? n - 1 : 0) in all of its warp-accesses.
// Lane l adds up warp-reps m0 + l, m0 + l + 32, ... of the chunk (closed form,
// no expansion).
__device__ __noinline__ Part count_uniform(uint64_t P, uint32_t B, uint64_t Mk, uint64_t m0, uint64_t tt,
                                           uint32_t cnt, bool flags, uint32_t tmin, int lane) {
    const uint64_t start = tt, end = tt + cnt;           // instances relative to warp-rep m0
    const uint64_t nw = udiv(end - 1, Mk) + 1;           // warp-reps touched
    const bool blocked = (B & 31u) != 0;
    const uint32_t wpb = (B + 31u) >> 5;
    uint64_t kb = 0;
    uint32_t w = 0;
    if (blocked) {
        const uint64_t mm = m0 + uint64_t(lane);
        kb = udiv(mm, wpb);
        w = uint32_t(mm - kb * wpb);
    }
    const uint32_t qb = 32u / wpb, rw = 32u % wpb;       // 32 warps = qb blocks + rw warps
    uint32_t lf = 0, cc = 0, uf = 0, ops = 0;
    for (uint64_t j = uint64_t(lane); j < nw; j += 32) {
        const uint64_t lo = j * Mk > start ? j * Mk : start;
        const uint64_t hi = (j + 1) * Mk < end ? (j + 1) * Mk : end;
        const uint32_t k = uint32_t(hi - lo);
        uint64_t p0, e;
        if (blocked) {
            p0 = kb * B + 32ull * w;
            e = umin64(p0 + 32, (kb + 1) * uint64_t(B));
            kb += qb;
            w += rw;
            if (w >= wpb) { w -= wpb; kb++; }
        } else {
            p0 = (m0 + j) * 32;
            e = p0 + 32;
        }
        e = umin64(e, P);
        const uint32_t nl = flags ? uint32_t(e - p0) - 1u : 0u;
        lf += k * nl;
        if (nl + 1u <= tmin) cc += k;                     // R11
        else uf += k * nl;
        ops += kOpsClass;
    }
    return Part{lf, lf, cc, uf, 0u, ops};
}

// ------------------------------------------------------------- arithmetic lanes
// A 1-D parallel access with lane stride 0 < g < 128 places the n active lanes
// of a warp-access at lo, lo + g, ..., lo + (n-1) g (lo = the lowest lane
// address; lanes descend when c_par < 0).  Consecutive lanes are < 128 bytes
// apart, so no line between the first and the last is skipped:
//   lines   = 1 + ((r + span) >> 7),  r = (lo + D) mod 128,  span = (n-1) g
//   sectors = 1 + (((r mod 32) + span) >> 5)   if g < 32   (none skipped)
//           = n                                  if g >= 32 (one per lane)
// -- the same integers as the lane-by-lane definition, from one residue.  Each
// lane therefore evaluates its OWN warp-accesses (lane l takes instances l,
// l + 32, ... of the chunk, walking (warp-rep, inner tuple) as a mixed-radix
// counter), 32 warp-accesses per warp instruction instead of one.
template <int DEPTH>
__device__ __noinline__ Part count_arith(const sel_access& a, uint64_t P, uint32_t B, uint64_t T0, uint64_t T1,
                                         uint64_t T2, uint64_t Mk, uint64_t m0, uint64_t tt, uint32_t cnt, int lane,
                                         uint32_t tmin) {
    const int64_t c0 = a.c_par[0];
    const uint32_t g = uint32_t(uabs(c0));
    const bool neg = c0 < 0;
    const uint32_t base32 = uint32_t(uint64_t(a.base)), c032 = uint32_t(uint64_t(c0));
    const uint32_t k0 = uint32_t(uint64_t(a.c_inner[0])), k1 = uint32_t(uint64_t(a.c_inner[1])),
                   k2 = uint32_t(uint64_t(a.c_inner[2]));
    const uint32_t t0 = uint32_t(T0), t1 = uint32_t(T1), t2 = uint32_t(T2);
    // this lane's first instance: offset tt + lane from warp-rep m0
    const uint64_t u = tt + uint64_t(lane);
    const uint64_t um = udiv(u, Mk);
    uint64_t m = m0 + um;
    const uint64_t rm = u - um * Mk;
    uint32_t i0 = 0, i1 = 0, i2 = 0;
    if (DEPTH == 1) { i0 = uint32_t(rm); }
    if (DEPTH == 2) { const uint64_t q = udiv(rm, T1); i0 = uint32_t(q); i1 = uint32_t(rm - q * T1); }
    if (DEPTH == 3) {
        const uint64_t q = udiv(rm, T2), q2 = udiv(q, T1);
        i2 = uint32_t(rm - q * T2); i1 = uint32_t(q - q2 * T1); i0 = uint32_t(q2);
    }
    // the step of 32 instances as mixed-radix digits (warp-rep, i0, i1, i2)
    const uint32_t sm = Mk > 32 ? 0u : 32u / uint32_t(Mk);      // 0 unless Mk <= 32
    const uint32_t sr = Mk > 32 ? 32u : 32u % uint32_t(Mk);
    uint32_t d0 = 0, d1 = 0, d2 = 0;
    if (DEPTH == 1) { d0 = sr; }
    if (DEPTH == 2) { d1 = sr < t1 ? sr : sr % t1; d0 = sr < t1 ? 0u : sr / t1; }
    if (DEPTH == 3) {
        const uint32_t q = sr < t2 ? 0u : sr / t2;
        d2 = sr - q * t2; d1 = q < t1 ? q : q % t1; d0 = q < t1 ? 0u : q / t1;
    }
    // warp-rep m = (block kb, warp w) when 32 does not divide B (R8, R9)
    const bool blocked = (B & 31u) != 0;
    const uint32_t wpb = (B + 31u) >> 5;
    uint64_t kb = blocked ? udiv(m, wpb) : 0;
    uint32_t w = blocked ? uint32_t(m - kb * wpb) : 0u;
    uint32_t lo32 = 0, nm1 = 0, span = 0;
    auto warp_props = [&]() {
        uint64_t p0, e;
        if (blocked) {
            p0 = kb * B + 32ull * w;
            e = umin64(p0 + 32, (kb + 1) * uint64_t(B));
        } else {
            p0 = m * 32;
            e = p0 + 32;
        }
        e = umin64(e, P);
        nm1 = uint32_t(e - p0) - 1u;                   // active lanes - 1 (unused past the chunk)
        lo32 = base32 + c032 * uint32_t(p0) + (neg ? c032 * nm1 : 0u);
        span = nm1 * g;
    };
    warp_props();
    uint32_t lf = 0, sf = 0, uf = 0, cc = 0;
    for (uint32_t t = uint32_t(lane); t < cnt; t += 32) {
        uint32_t D = 0;
        if (DEPTH >= 1) D += k0 * i0;
        if (DEPTH >= 2) D += k1 * i1;
        if (DEPTH >= 3) D += k2 * i2;
        const uint32_t r = (lo32 + D) & 127u;
        const uint32_t nl = (r + span) >> 7;           // lines - 1
        const uint32_t ns = g < 32u ? ((r & 31u) + span) >> 5 : nm1;
        lf += nl;
        sf += ns;
        if (nl + 1u <= tmin) cc++;                      // R11
        else uf += nl;
        uint32_t carry = 0;
        if (DEPTH >= 3) { i2 += d2; carry = i2 >= t2; if (carry) i2 -= t2; }
        if (DEPTH >= 2) {
            i1 += (DEPTH == 2 ? d1 : d1 + carry);
            carry = i1 >= t1;
            if (carry) i1 -= t1;
        }
        if (DEPTH >= 1) {
            i0 += (DEPTH == 1 ? d0 : d0 + carry);
            carry = i0 >= t0;
            if (carry) i0 -= t0;
        }
        const uint32_t dm = sm + carry;
        if (dm) {
            m += dm;
            if (blocked) {
                w += dm;
                while (w >= wpb) { w -= wpb; kb++; }
            }
            warp_props();
        }
    }
    return Part{lf, sf, cc, uf, cnt, lane0(lane, kOpsArithWA * cnt)};
}

// ------------------------------------------------------------- residue classes
// Within one full warp-rep of an arithmetic-lane access (above) every
// warp-access is fixed by r = (lo + D) mod 128, and D = sum_j k_j i_j.  So the
// warp-rep's sums over its Mk inner tuples are  sum_rho h[rho] * f(lo + rho),
// h[rho] = #{tuples : D = rho (mod 128)} -- the same integers as the tuple
// by tuple sum, grouped by residue.  Addresses are multiples of the element
// size E (V5), so h lives on the R = 128/E residues rho = s*E (slot s).
//
// h of one loop (k, T): k*i mod 128 has period pi = 128 / gcd(k mod 128, 128),
// distinct over i < pi; residue k*i (i < min(T, pi)) occurs ceil((T - i)/pi)
// times.  Nested loops convolve (cyclically, mod 128) the one-loop histograms.
__device__ __forceinline__ uint32_t loop_period_log2(uint32_t k) {   // log2 pi
    const uint32_t km = k & 127u;
    return km == 0 ? 0u : 7u - uint32_t(__ffs(km) - 1);
}

// h <- histogram of one loop (k, T), T >= 1; smem, R slots of 2^sh bytes
__device__ __forceinline__ void hist_one(uint32_t* h, uint32_t R, uint32_t sh, uint32_t k, uint32_t T, int lane,
                                         uint32_t& ops) {
#pragma unroll
    for (uint32_t j = 0; j < 4; j++)
        if (lane + 32u * j < R) h[lane + 32u * j] = 0;
    __syncwarp();
    const uint32_t lp = loop_period_log2(k), pi = 1u << lp;
    const uint32_t n = T < pi ? T : pi;                         // <= 128
    ops += lane0(lane, kOpsHistEntry * n);
#pragma unroll
    for (uint32_t j = 0; j < 4; j++) {
        const uint32_t i = lane + 32u * j;
        if (i < n) h[((k * i) & 127u) >> sh] = (T - i + pi - 1u) >> lp;
    }
    __syncwarp();
}

// h <- h (*) histogram of loop (k, T): out[rho] = sum_i cnt(i) h[rho - k i]
__device__ __forceinline__ void hist_conv(uint32_t* h, uint32_t R, uint32_t sh, uint32_t k, uint32_t T, int lane,
                                          uint32_t& ops) {
    const uint32_t lp = loop_period_log2(k), pi = 1u << lp;
    const uint32_t n = T < pi ? T : pi;
    ops += lane0(lane, kOpsConvTerm * n * R);
    uint32_t o[4] = {0u, 0u, 0u, 0u};
    for (uint32_t i = 0; i < n; i++) {
        const uint32_t c = (T - i + pi - 1u) >> lp;
        const uint32_t off = k * i;
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const uint32_t s = uint32_t(lane) + 32u * j;
            if (s < R) o[j] += c * h[(((s << sh) - off) & 127u) >> sh];
        }
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 4; j++) {
        const uint32_t s = uint32_t(lane) + 32u * j;
        if (s < R) h[s] = o[j];
    }
    __syncwarp();
}

// h[0..R) -> its exclusive prefix pf[0..R] (in place, pf[R] = the total) and
// the exclusive prefix p32[0..R/4] of h folded mod 32 bytes (slot u of the
// fold = slots u, u + R/4, u + R/2, u + 3R/4: the same residue mod 32).
__device__ __forceinline__ void hist_prefix(uint32_t* h, uint32_t R, int lane, uint32_t& ops) {
    const uint32_t R32 = R >> 2;
    uint32_t v[4];
#pragma unroll
    for (uint32_t j = 0; j < 4; j++) v[j] = lane + 32u * j < R ? h[lane + 32u * j] : 0u;
    const uint32_t f = uint32_t(lane) < R32 ? h[lane] + h[lane + R32] + h[lane + 2u * R32] + h[lane + 3u * R32] : 0u;
    __syncwarp();
    ops += lane0(lane, kOpsPrefixEntry * (R + R32));
    uint32_t carry = 0;
#pragma unroll
    for (uint32_t j = 0; j < 4; j++) {
        if (32u * j >= R) break;
        uint32_t x = v[j];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(kFull, x, o);
            if (lane >= o) x += t;
        }
        if (lane + 32u * j < R) h[1u + lane + 32u * j] = carry + x;
        carry += __shfl_sync(kFull, x, 31);
    }
    uint32_t y = f;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, y, o);
        if (lane >= o) y += t;
    }
    if (uint32_t(lane) < R32) h[kP32Off + 1u + lane] = y;
    if (lane == 0) {
        h[0] = 0u;
        h[kP32Off] = 0u;
    }
    __syncwarp();
}

// sum of h over the cyclic slot range start, start + 1, ..., start + len - 1
// (mod R), len < R, from the exclusive prefix pf (any indexable view)
template <class A>
__device__ __forceinline__ uint32_t crange(const A& pf, uint32_t R, uint32_t start, uint32_t len) {
    const uint32_t e = start + len;
    return e <= R ? pf[e] - pf[start] : pf[R] - pf[start] + pf[e - R];
}

// `mult` warp-reps whose lowest lane address is lo (mod 128) with nm1 + 1
// active lanes, summed over the residues of h in closed form from its prefix
// sums (the same integers as the residue-by-residue sum of count_arith):
// with span = (n - 1) g = 128 a + b, a WA at residue r has lines - 1 =
// a + [r >= 128 - b], so  sum_r h(r) (lines - 1) = a H + X,  X = the h-mass of
// the residues (lo + rho) mod 128 in [128 - b, 128): ONE cyclic range of
// slots.  Sectors likewise mod 32 (g < 32), or n per WA (g >= 32).  Coalesced
// <=> lines - 1 < tmin (R11): all, none, or the H - X WAs without the extra
// line.  Everything in slot units (addresses, strides and spans are multiples
// of the element size, V5).  pf: exclusive prefix of h over R slots (pf[R] =
// H); p32: the same of h folded mod 32 bytes (R / 4 slots).
struct ClassSums {
    uint32_t lf, sf, cc, uf;
};
template <class A>
__device__ __forceinline__ ClassSums class_sums(const A& pf, const A& p32, uint32_t R, uint32_t sh, uint32_t lo,
                                                uint32_t nm1, uint32_t g, uint32_t tmin, uint32_t mult) {
    const uint32_t Ht = pf[R];
    const uint32_t span = nm1 * g;
    const uint32_t a = span >> 7, bs = (span & 127u) >> sh, los = (lo & 127u) >> sh;
    const uint32_t X = bs ? crange(pf, R, (2u * R - bs - los) & (R - 1u), bs) : 0u;
    ClassSums o;
    o.lf = a * Ht + X;
    if (a + 1u < tmin) {
        o.cc = Ht;
        o.uf = 0u;
    } else if (a < tmin) {
        o.cc = Ht - X;
        o.uf = (a + 1u) * X;
    } else {
        o.cc = 0u;
        o.uf = o.lf;
    }
    if (g >= 32u) {
        o.sf = nm1 * Ht;
    } else {
        const uint32_t R32 = R >> 2;
        const uint32_t b2s = (span & 31u) >> sh, l32 = (lo & 31u) >> sh;
        const uint32_t Y = b2s ? crange(p32, R32, (2u * R32 - b2s - l32) & (R32 - 1u), b2s) : 0u;
        o.sf = (span >> 5) * Ht + Y;
    }
    o.lf *= mult;
    o.sf *= mult;
    o.cc *= mult;
    o.uf *= mult;
    return o;
}
__device__ __forceinline__ ClassSums hist_eval_pf(const uint32_t* h, uint32_t R, uint32_t sh, uint32_t lo,
                                                  uint32_t nm1, uint32_t g, uint32_t tmin, uint32_t mult) {
    const uint32_t* p32 = h + kP32Off;
    return class_sums(h, p32, R, sh, lo, nm1, g, tmin, mult);
}

// lane-uniform class sums, added once (lane 0)
__device__ __forceinline__ void hist_eval(const uint32_t* h, uint32_t R, uint32_t sh, uint32_t lo, uint32_t nm1,
                                          uint32_t g, uint32_t tmin, uint32_t mult, int lane, uint32_t& lf,
                                          uint32_t& sf, uint32_t& cc, uint32_t& uf, uint32_t& ops) {
    const ClassSums c = hist_eval_pf(h, R, sh, lo, nm1, g, tmin, mult);
    ops += lane0(lane, kOpsEvalClass);
    if (lane == 0) {
        lf += c.lf;
        sf += c.sf;
        cc += c.cc;
        uf += c.uf;
    }
}

// WAs [tt, tt + cnt) from warp-rep m0 of a 1-D access with lane stride
// 0 < g < 128: head and tail fragments of a warp-rep lane by lane
// (count_arith), whole warp-reps by residue classes.
template <int DEPTH>
__device__ __noinline__ Part count_hist(const sel_access& a, uint64_t P, uint32_t B, uint64_t T0, uint64_t T1,
                                        uint64_t T2, uint64_t Mk, uint64_t m0, uint64_t tt, uint32_t cnt, int lane,
                                        uint32_t tmin, uint32_t* h) {
    uint64_t m = m0;
    Part out{0u, 0u, 0u, 0u, 0u, 0u};
    auto add = [&](const Part& p) {
        out.lf += p.lf; out.sf += p.sf; out.cc += p.cc; out.uf += p.uf; out.q += p.q; out.ops += p.ops;
    };
    if (tt > 0) {                                               // head: rest of warp-rep m0
        const uint32_t k = uint32_t(umin64(Mk - tt, cnt));
        add(count_arith<DEPTH>(a, P, B, T0, T1, T2, Mk, m, tt, k, lane, tmin));
        cnt -= k;
        m++;
        if (cnt == 0) return out;
    }
    const uint32_t Mk32 = uint32_t(Mk);                         // Mk <= cnt <= kMaxChunk here
    const uint32_t nfull = cnt / Mk32;
    const uint32_t rest = cnt - nfull * Mk32;
    if (nfull) {
        const uint32_t sh = uint32_t(__ffs(a.elem_bytes) - 1), R = 128u >> sh;
        const uint32_t k0 = uint32_t(uint64_t(a.c_inner[0])), k1 = uint32_t(uint64_t(a.c_inner[1])),
                       k2 = uint32_t(uint64_t(a.c_inner[2]));
        uint32_t ops = 0;
        if (DEPTH == 1) hist_one(h, R, sh, k0, uint32_t(T0), lane, ops);
        if (DEPTH == 2) {
            hist_one(h, R, sh, k1, uint32_t(T1), lane, ops);
            hist_conv(h, R, sh, k0, uint32_t(T0), lane, ops);
        }
        if (DEPTH == 3) {
            hist_one(h, R, sh, k2, uint32_t(T2), lane, ops);
            hist_conv(h, R, sh, k1, uint32_t(T1), lane, ops);
            hist_conv(h, R, sh, k0, uint32_t(T0), lane, ops);
        }
        hist_prefix(h, R, lane, ops);
        const int64_t c0 = a.c_par[0];
        const uint32_t g = uint32_t(uabs(c0));
        const bool neg = c0 < 0;
        const uint32_t base32 = uint32_t(uint64_t(a.base)), c032 = uint32_t(uint64_t(c0));
        uint32_t lf = 0, sf = 0, cc = 0, uf = 0;
        if ((B & 31u) == 0) {
            // warp-rep j: p0 = 32 j, all 32 lanes active except the last one of P;
            // lo mod 128 of a full warp-rep depends on j mod 4 only
            const uint64_t nfl = P >> 5;                        // warp-reps with 32 active lanes
            const uint64_t e = m + nfull;
            const uint64_t ef = e < nfl ? e : (nfl > m ? nfl : m);
            const uint64_t nf = ef - m;                         // full-lane warp-reps in [m, e)
            for (uint32_t j = 0; j < 4; j++) {
                // #{x in [m, m + nf) : x = j (mod 4)}
                const uint64_t first = m + ((j - uint32_t(m)) & 3u);
                const uint32_t cntj = first < m + nf ? uint32_t((m + nf - 1 - first) / 4 + 1) : 0u;
                if (cntj == 0) continue;
                const uint32_t lo = base32 + c032 * (32u * uint32_t(first)) + (neg ? c032 * 31u : 0u);
                hist_eval(h, R, sh, lo, 31u, g, tmin, cntj, lane, lf, sf, cc, uf, ops);
            }
            if (ef < e) {                                       // the partial last warp-rep of P
                const uint32_t nm1 = uint32_t(P - 32ull * ef) - 1u;
                const uint32_t lo = base32 + c032 * (32u * uint32_t(ef)) + (neg ? c032 * nm1 : 0u);
                hist_eval(h, R, sh, lo, nm1, g, tmin, 1u, lane, lf, sf, cc, uf, ops);
            }
        } else {
            const uint32_t wpb = (B + 31u) >> 5;
            uint64_t kb = udiv(m, wpb);
            uint32_t w = uint32_t(m - kb * wpb);
            for (uint32_t x = 0; x < nfull; x++) {
                const uint64_t p0 = kb * B + 32ull * w;
                const uint64_t pe = umin64(umin64(p0 + 32, (kb + 1) * uint64_t(B)), P);
                const uint32_t nm1 = uint32_t(pe - p0) - 1u;
                const uint32_t lo = base32 + c032 * uint32_t(p0) + (neg ? c032 * nm1 : 0u);
                hist_eval(h, R, sh, lo, nm1, g, tmin, 1u, lane, lf, sf, cc, uf, ops);
                if (++w == wpb) { w = 0; kb++; }
            }
        }
        add(Part{lf, sf, cc, uf, 0u, ops});
        __syncwarp();                                           // h is reused by the next access
    }
    if (rest) add(count_arith<DEPTH>(a, P, B, T0, T1, T2, Mk, m + nfull, 0, rest, lane, tmin));
    return out;
}

// ------------------------------------------------------------- whole accesses
// When a chunk holds all WR * Mk warp-accesses of an access (the common case:
// a chunk spans many small problems) the warp-reps need not be walked: by R8
// and R9 they fall into at most three lane-count classes, computed once per
// problem -- n32 warp-reps with 32 active lanes, nA with B mod 32 lanes (the
// last warp of every complete block when 32 does not divide B) and at most
// one with the last lanes of P.
struct RepClasses {
    uint64_t n32, nA;
    uint32_t lanesA, lanesR;        // 0: class empty
};
__device__ __forceinline__ RepClasses rep_classes(uint64_t P, uint32_t B) {
    RepClasses c;
    if ((B & 31u) == 0) {
        c.n32 = P >> 5;
        c.nA = 0;
        c.lanesA = 0;
        c.lanesR = uint32_t(P & 31u);
    } else {
        const uint64_t nbf = udiv(P, B);                    // complete blocks
        const uint32_t rem = uint32_t(P - nbf * B);         // iterations of the last, incomplete block
        c.n32 = nbf * ((B - 1u) >> 5) + (rem >> 5);
        c.nA = nbf;
        c.lanesA = B & 31u;
        c.lanesR = rem & 31u;
    }
    return c;
}

// Uniform lane flags over a whole access: a warp-rep with n active lanes has
// lines = sectors = 1 + (flags ? n - 1 : 0) in each of its Mk warp-accesses
// (count_uniform); warp-uniform accumulators.
__device__ __forceinline__ void uniform_whole(const RepClasses& rc, uint32_t Mk, bool flags, uint32_t tmin,
                                              Acc& acc, int lane) {
    auto cls = [&](uint32_t lanes, uint32_t reps) {
        acc.ops += lane0(lane, kOpsClass);
        const uint32_t w = reps * Mk;                       // <= WR * Mk <= kMaxChunk
        const uint32_t nl = flags ? lanes - 1u : 0u;
        acc.lk += w * nl;
        acc.sk += w * nl;
        if (nl + 1u <= tmin) acc.C += w;                    // R11
        else acc.uk += w * nl;
    };
    if (rc.n32) cls(32u, uint32_t(rc.n32));
    if (rc.nA) cls(rc.lanesA, uint32_t(rc.nA));
    if (rc.lanesR) cls(rc.lanesR, 1u);
}

// h <- residue histogram of the access's inner offsets (runtime depth 0..3)
__device__ __forceinline__ void hist_build(uint32_t* h, const sel_access& a, int depth, uint32_t T0, uint32_t T1,
                                           uint32_t T2, uint32_t R, uint32_t sh, int lane, uint32_t& ops) {
    const uint32_t k0 = uint32_t(uint64_t(a.c_inner[0])), k1 = uint32_t(uint64_t(a.c_inner[1])),
                   k2 = uint32_t(uint64_t(a.c_inner[2]));
    if (depth == 0) hist_one(h, R, sh, 0u, 1u, lane, ops);
    else if (depth == 1) hist_one(h, R, sh, k0, T0, lane, ops);
    else if (depth == 2) { hist_one(h, R, sh, k1, T1, lane, ops); hist_conv(h, R, sh, k0, T0, lane, ops); }
    else {
        hist_one(h, R, sh, k2, T2, lane, ops);
        hist_conv(h, R, sh, k1, T1, lane, ops);
        hist_conv(h, R, sh, k0, T0, lane, ops);
    }
}

// Residue classes over a whole access when the warp-reps' lowest lane
// addresses fall into many classes (32 does not divide B and B c != 0 mod
// 128): one warp-rep PER LANE (p0, active lanes and lo from the block
// geometry, R8/R9), each lane summing its warp-rep over the R residues of h.
// Same integers as hist_eval per warp-rep.  WR <= kSmallMaxWR.
__device__ __noinline__ Part count_hist_reps(const sel_access* ap, int depth, uint32_t T0, uint32_t T1, uint32_t T2,
                                             uint32_t P, uint32_t B, uint32_t WR, uint32_t tmin, uint32_t* h,
                                             int lane) {
    const sel_access a = *ap;
    const uint32_t sh = uint32_t(__ffs(a.elem_bytes) - 1), R = 128u >> sh;
    uint32_t ops = 0;
    hist_build(h, a, depth, T0, T1, T2, R, sh, lane, ops);
    hist_prefix(h, R, lane, ops);
    ops += lane0(lane, kOpsEvalClass * WR);
    const int64_t c0 = a.c_par[0];
    const uint32_t g = uint32_t(uabs(c0));
    const bool neg = c0 < 0;
    const uint32_t base32 = uint32_t(uint64_t(a.base)), c032 = uint32_t(uint64_t(c0));
    const uint32_t wpb = (B + 31u) >> 5;
    Part o{0u, 0u, 0u, 0u, 0u, ops};
    for (uint32_t m0 = 0; m0 < WR; m0 += 32) {
        const uint32_t m = m0 + uint32_t(lane);
        if (m < WR) {
            const uint32_t kb = m / wpb, w = m - kb * wpb;
            const uint32_t p0 = kb * B + 32u * w;
            uint32_t pe = p0 + 32u;
            pe = pe < (kb + 1u) * B ? pe : (kb + 1u) * B;
            pe = pe < P ? pe : P;
            const uint32_t nm1 = pe - p0 - 1u;
            const uint32_t lo = base32 + c032 * p0 + (neg ? c032 * nm1 : 0u);
            const ClassSums c = hist_eval_pf(h, R, sh, lo, nm1, g, tmin, 1u);
            o.lf += c.lf;
            o.sf += c.sf;
            o.cc += c.cc;
            o.uf += c.uf;
        }
    }
    __syncwarp();                                           // h is reused by the next access
    return o;
}

// Residue classes over a whole access (count_hist) when the lowest lane
// address mod 128 of a warp-rep depends only on its lane count (32 | B with
// 32 c = 0 mod 128, or B c = 32 c = 0 mod 128), or, for 32 | B, on the
// warp-rep index mod 4: the histogram is built once and evaluated once per
// class.  Runtime depth (0..3).
__device__ __forceinline__ Part count_hist_whole(const sel_access& a, int depth, uint32_t T0, uint32_t T1,
                                                 uint32_t T2, RepClasses rc, uint32_t tmin, uint32_t* h, int lane) {
    const uint32_t sh = uint32_t(__ffs(a.elem_bytes) - 1), R = 128u >> sh;
    Part o{0u, 0u, 0u, 0u, 0u, 0u};
    hist_build(h, a, depth, T0, T1, T2, R, sh, lane, o.ops);
    hist_prefix(h, R, lane, o.ops);
    const int64_t c0 = a.c_par[0];
    const uint32_t g = uint32_t(uabs(c0));
    const bool neg = c0 < 0;
    const uint32_t base32 = uint32_t(uint64_t(a.base)), c032 = uint32_t(uint64_t(c0));
    // lowest lane address of a warp-rep starting at iteration p0 with n lanes
    auto lo_of = [&](uint32_t p0, uint32_t n) { return base32 + c032 * p0 + (neg ? c032 * (n - 1u) : 0u); };
    if (rc.n32) {
        if (((32u * c032) & 127u) == 0) {
            hist_eval(h, R, sh, lo_of(0u, 32u), 31u, g, tmin, uint32_t(rc.n32), lane, o.lf, o.sf, o.cc, o.uf, o.ops);
        } else {                                            // 32 | B here: warp-rep j starts at 32 j
            for (uint32_t j = 0; j < 4; j++) {
                const uint32_t cj = uint32_t((rc.n32 + 3u - j) >> 2);   // #{x < n32 : x = j mod 4}
                if (cj) hist_eval(h, R, sh, lo_of(32u * j, 32u), 31u, g, tmin, cj, lane, o.lf, o.sf, o.cc, o.uf, o.ops);
            }
        }
    }
    if (rc.nA) hist_eval(h, R, sh, lo_of(0u, rc.lanesA), rc.lanesA - 1u, g, tmin, uint32_t(rc.nA), lane, o.lf, o.sf,
                         o.cc, o.uf, o.ops);
    if (rc.lanesR) {                                        // the last warp-rep of P starts at 32 n32 (32 | B)
        const uint32_t p0 = rc.nA ? 0u : uint32_t(32u * rc.n32);
        hist_eval(h, R, sh, lo_of(p0, rc.lanesR), rc.lanesR - 1u, g, tmin, 1u, lane, o.lf, o.sf, o.cc, o.uf, o.ops);
    }
    __syncwarp();                                           // h is reused by the next access
    return o;
}

// ------------------------------------------------------------- per access
// Count WAs [off, off + cnt) of access `a` (instance order: warp-rep, then
// inner tuple with the last inner loop fastest).  DEPTH = a.depth.
// MODE: 0 = MATCH (__match_any_sync), 1 = scalar residue, 2 = byte-sliced residue.
template <int MODE, int DEPTH, int TC>
__device__ void count_access(const sel_nest& nest, const sel_access& a, uint64_t P, uint32_t B, uint64_t T0,
                             uint64_t T1, uint64_t T2, uint64_t Mk, uint64_t off, uint32_t cnt, int lane, uint32_t one,
                             uint32_t closed_form, Acc& acc) {
    const uint32_t tmin = (32u * a.elem_bytes + 127u) / 128u;       // R11
    const uint64_t Tl = DEPTH == 1 ? T0 : DEPTH == 2 ? T1 : DEPTH == 3 ? T2 : 1;
    const int64_t cl = DEPTH == 1 ? a.c_inner[0] : DEPTH == 2 ? a.c_inner[1] : DEPTH == 3 ? a.c_inner[2] : 0;
    uint64_t m = udiv(off, Mk);
    uint64_t tt = off - m * Mk;
    // inner indices, last fastest
    uint64_t i0 = 0, i1 = 0, i2 = 0;
    if (DEPTH == 1) { i0 = tt; }
    if (DEPTH == 2) { i0 = udiv(tt, T1); i1 = tt - i0 * T1; }
    if (DEPTH == 3) { const uint64_t r = udiv(tt, T2); i2 = tt - r * T2; i0 = udiv(r, T1); i1 = r - i0 * T1; }
    WarpIter it;
    warp_seek(it, m, P, B);
    while (cnt > 0) {
        const int64_t A = lane_address(nest, a, it, lane);
        uint32_t u_low = 0, dl = 0, ds = 0, KL = 0, KS = 0, dlb_u = 0, dsb_u = 0;
        int64_t Am = A;
        if (MODE != 0) {
            int64_t upper;
            uint64_t gap;
            if (nest.par_dims == 1) {
                const int64_t c0 = a.c_par[0];
                upper = A + (c0 < 0 ? -c0 : 0);     // larger address of the lane pair (l-1, l)
                gap = uabs(c0);
            } else {
                const int64_t key = bitonic_sort_warp(lane < int(it.n) ? A : INT64_MAX, lane);
                const int64_t prev = __shfl_up_sync(kFull, key, 1);
                upper = key;
                gap = uint64_t(key - prev);
            }
            const bool has = lane >= 1 && lane < int(it.n);
            u_low = uint32_t(upper);
            dl = has ? (gap >= 128 ? 0xffffffffu : uint32_t(gap) << 25) : 0u;
            ds = has ? (gap >= 32 ? 0xffffffffu : uint32_t(gap) << 27) : 0u;
            // byte-sliced thresholds: d capped at 128 (lines) / 32 (sectors); 0 = never a flag
            const uint32_t dlb = has ? uint32_t(umin64(gap, 128)) : 0u;
            const uint32_t dsb = has ? uint32_t(umin64(gap, 32)) : 0u;
            dlb_u = dlb;
            dsb_u = dsb;
            KL = 0x80808080u - dlb * 0x01010101u;
            KS = 0x80808080u - dsb * 0x01010101u;
        } else {
            const int64_t a0 = __shfl_sync(kFull, A, 0);
            Am = lane < int(it.n) ? A : a0;         // inactive lanes duplicate lane 0
        }
        // rows of the last inner loop within this warp-rep
        const uint64_t here64 = umin64(Mk - tt, cnt);
        uint32_t left = uint32_t(here64);
        if (MODE != 0 && closed_form) {
            // UNIFORM FLAGS.  A lane's line flag  (s_l + D) mod 128 < gap_l  does
            // not depend on the inner offset D when gap_l is 0 (never) or >= 128
            // (always); likewise sectors with 0 or >= 32.  When that holds on every
            // lane, all WAs of this warp-rep are identical: lines = 1 + #line
            // flags, sectors = 1 + #sector flags, coalesced <=> lines <= tmin
            // (R11) -- added for all `left` WAs at once (exact, no expansion).
            const bool uni = (dlb_u == 0u || dlb_u == 128u) && (dsb_u == 0u || dsb_u == 32u);
            if (__all_sync(kFull, uni)) {
                const uint32_t nl = __popc(__ballot_sync(kFull, dlb_u == 128u));
                const uint32_t ns = __popc(__ballot_sync(kFull, dsb_u == 32u));
                acc.W += left;
                acc.K += left;
                acc.ops += lane0(lane, kOpsClass);
                acc.lk += left * nl;
                acc.sk += left * ns;
                if (nl + 1u <= tmin) acc.C += left;
                else acc.uk += left * nl;
                left = 0;
                i0 = i1 = i2 = 0;          // the warp-rep is finished (or cnt is exhausted)
            }
        }
        while (left > 0) {
            int64_t D = 0;
            if (DEPTH >= 1) D += a.c_inner[0] * int64_t(i0);
            if (DEPTH >= 2) D += a.c_inner[1] * int64_t(i1);
            if (DEPTH >= 3) D += a.c_inner[2] * int64_t(i2);
            const uint64_t il = DEPTH == 1 ? i0 : DEPTH == 2 ? i1 : DEPTH == 3 ? i2 : 0;
            const uint32_t len = uint32_t(umin64(Tl - il, left));
            if (MODE == 0) {
                hot_match(Am + D, cl, len, tmin, acc);
            } else if (TC == 4 || MODE == 1) {
                const uint32_t y = (u_low + uint32_t(uint64_t(D))) << 25;
                const uint32_t step = uint32_t(uint64_t(cl)) << 25;
                if (TC == 4) hot_row_t4(y, step, dl, ds, len, acc);
                else hot_row<TC == 4 ? 1 : TC>(y, step, dl, ds, len, acc);
            } else {
                hot_row_swar<TC == 4 ? 1 : TC>(u_low + uint32_t(uint64_t(D)), uint32_t(uint64_t(cl)) & 127u, KL,
                                               KS, len, one, acc);
            }
            acc.ops += lane0(lane, kOpsExpandWA * len);
            left -= len;
            // odometer carry (registers only)
            if (DEPTH == 1) { i0 += len; if (i0 >= T0) i0 = 0; }
            if (DEPTH == 2) { i1 += len; if (i1 >= T1) { i1 = 0; if (++i0 >= T0) i0 = 0; } }
            if (DEPTH == 3) {
                i2 += len;
                if (i2 >= T2) { i2 = 0; if (++i1 >= T1) { i1 = 0; if (++i0 >= T0) i0 = 0; } }
            }
        }
        cnt -= uint32_t(here64);
        tt = 0;
        if (cnt > 0) warp_next(it, P, B);
    }
}

// Path statistics of one warp, summed over everything it counted and added to
// the workspace header once per warp at kernel exit (one address line shared
// by every warp: per-problem atomics there serialise in one L2 slice).
struct WarpStats {
    unsigned long long K, Q, H, ops;
};
__device__ __forceinline__ void stats_flush(const CountArgs& a, const WarpStats& st, int lane) {
    if (st.K && lane == 0) atomicAdd((unsigned long long*)&a.hdr->stats.wa_closed_form, st.K);
    if (st.Q && lane == 1) atomicAdd((unsigned long long*)&a.hdr->stats.wa_arith_lanes, st.Q);
    if (st.H && lane == 2) atomicAdd((unsigned long long*)&a.hdr->stats.wa_residue_classes, st.H);
    if (st.ops && lane == 3) atomicAdd((unsigned long long*)&a.hdr->stats.alg_lane_ops, st.ops);
}

// counts of problem q += this warp's accumulators; statistics move to st
__device__ void flush(const CountArgs& a, uint64_t q, Acc& acc, int lane, WarpStats& st) {
    const uint64_t slf = __reduce_add_sync(kFull, acc.lf);
    const uint64_t ssf = __reduce_add_sync(kFull, acc.sf);
    const uint64_t suf = __reduce_add_sync(kFull, acc.uf);
    const uint64_t W = acc.W;
    const uint64_t L = W + slf + acc.lk;
    const uint64_t S = W + ssf + acc.sk;
    const uint64_t C = acc.C + __reduce_add_sync(kFull, acc.cc);
    const uint64_t U = (W - C) + suf + acc.uk;
    if (W && lane < 5) {
        const uint64_t v = lane == 0 ? W : lane == 1 ? L : lane == 2 ? S : lane == 3 ? C : U;
        atomicAdd(&a.prob_cnt[q * kCntStride + lane], (unsigned long long)v);
    }
    st.K += acc.K;
    st.Q += acc.Q;
    st.H += acc.H;
    st.ops += __reduce_add_sync(kFull, acc.ops);
    acc = Acc{};
}

// Cold and warm paths, out of line so the hot per-problem loop stays compact
// in the instruction cache.  General 1-D access slice (chunk boundaries,
// blocks that break the residue classes): uniform flags, residue classes
// with head/tail fragments, or arithmetic lanes.
struct Part1 {
    Part p;
    uint32_t uniform;                                       // 1: the WAs were uniform-flag closed form
};
__device__ __noinline__ Part1 count_1d_general(const sel_access* ap, uint64_t P, uint32_t B, uint64_t T0,
                                               uint64_t T1, uint64_t T2, uint64_t Mk, uint64_t off, uint32_t t,
                                               uint32_t tc, int lane, uint32_t* hist) {
    const sel_access ac = *ap;
    const int d = ac.depth;
    const uint64_t g = uabs(ac.c_par[0]);
    const uint64_t m = off ? udiv(off, Mk) : 0, tt = off - m * Mk;
    if (g == 0 || g >= 128) return Part1{count_uniform(P, B, Mk, m, tt, t, g != 0, tc, lane), 1u};
    const bool hs = d >= 1 && hist && Mk >= kHistMinMk;
    Part p;
    switch (d) {
    case 0: p = count_arith<0>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc); break;
    case 1: p = hs ? count_hist<1>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc, hist)
                   : count_arith<1>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc); break;
    case 2: p = hs ? count_hist<2>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc, hist)
                   : count_arith<2>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc); break;
    default: p = hs ? count_hist<3>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc, hist)
                    : count_arith<3>(ac, P, B, T0, T1, T2, Mk, m, tt, t, lane, tc); break;
    }
    return Part1{p, 0u};
}

// Lane-by-lane expansion (collapse(2) accesses, SEL_F_EXPAND_ALL, MATCH).
template <int MODE>
__device__ __noinline__ Acc expand_access(const sel_nest* np, const sel_access* ap, uint64_t P, uint32_t B,
                                          uint64_t T0, uint64_t T1, uint64_t T2, uint64_t Mk, uint64_t off, uint32_t t,
                                          int lane, uint32_t one, uint32_t closed_form, Acc acc) {
    const sel_nest nest = *np;
    const sel_access ac = *ap;
    const int d = ac.depth;
    const int tc = (32 * int(ac.elem_bytes) + 127) / 128;       // tmin (R11): 1, 2 or 4
#define SEL_DISPATCH(M, TCV)                                                                                  \
    switch (d) {                                                                                              \
    case 0: count_access<M, 0, TCV>(nest, ac, P, B, T0, T1, T2, Mk, off, t, lane, one, closed_form, acc); break;  \
    case 1: count_access<M, 1, TCV>(nest, ac, P, B, T0, T1, T2, Mk, off, t, lane, one, closed_form, acc); break;  \
    case 2: count_access<M, 2, TCV>(nest, ac, P, B, T0, T1, T2, Mk, off, t, lane, one, closed_form, acc); break;  \
    default: count_access<M, 3, TCV>(nest, ac, P, B, T0, T1, T2, Mk, off, t, lane, one, closed_form, acc); break; \
    }
    if (MODE == 0) {
        SEL_DISPATCH(0, 1)
    } else if (tc == 1) {
        SEL_DISPATCH(MODE, 1)
    } else if (tc == 2) {
        SEL_DISPATCH(MODE, 2)
    } else {
        SEL_DISPATCH(MODE, 4)
    }
#undef SEL_DISPATCH
    return acc;
}

// WAs [off, off + take) of problem q, access by access.
template <int MODE>
__device__ __noinline__ void count_problem(const CountArgs& a, uint64_t q, uint64_t off, uint32_t take, int lane,
                                           uint32_t* hist, WarpStats& st) {
    uint32_t nid, B;
    problem_nest_B(a, q, nid, B);
    const sel_nest* np = a.nests + nid;
    const sel_nest nest = *np;
    const uint64_t WR = a.prob_WR[q];
    const uint64_t P = nest.P0 * nest.P1;
    const uint64_t T0 = eff_trip(nest.trip[0]), T1 = eff_trip(nest.trip[1]), T2 = eff_trip(nest.trip[2]);
    const uint64_t Mks[4] = {1, T0, T0 * T1, T0 * T1 * T2};
    const bool one_d = MODE != 0 && a.closed_form && nest.par_dims == 1;
    RepClasses rc{0, 0, 0u, 0u};
    if (one_d) rc = rep_classes(P, B);
    Acc acc{};
    const sel_access* ap = a.acc + nest.access_off;
    for (uint32_t k = 0; k < nest.n_access && take > 0; k++, ap++) {
        const sel_access ac = *ap;
        const int d = ac.depth;
        const uint64_t Mk = d == 0 ? Mks[0] : d == 1 ? Mks[1] : d == 2 ? Mks[2] : Mks[3];
        const uint64_t Wk = WR * Mk;
        if (off >= Wk) {
            off -= Wk;
            continue;
        }
        const uint32_t t = uint32_t(umin64(Wk - off, take));
        acc.W += t;
        take -= t;
        if (!one_d) {
            acc.W -= t;                                         // expand_access accumulates W itself
            acc = expand_access<MODE>(np, ap, P, B, T0, T1, T2, Mk, off, t, lane, a.one, a.closed_form, acc);
            off = 0;
            continue;
        }
        // 1-D parallel access: lane addresses an arithmetic progression
        const uint32_t tc = ac.elem_bytes <= 4 ? 1u : ac.elem_bytes == 8 ? 2u : 4u;   // tmin (R11)
        const uint32_t g = uint32_t(umin64(uabs(ac.c_par[0]), 128));
        const bool whole = off == 0 && t == Wk;
        const uint64_t off0 = off;
        off = 0;
        if (whole && (g == 0 || g == 128)) {
            uniform_whole(rc, uint32_t(Mk), g != 0, tc, acc, lane);
            acc.K += t;
            continue;
        }
        const uint32_t cB = uint32_t(uint64_t(ac.c_par[0])) * B;
        if (whole && hist && ((B & 31u) == 0 || (((cB | (32u * g)) & 127u) == 0))) {
            add_part(acc, count_hist_whole(ac, d, uint32_t(T0), uint32_t(T1), uint32_t(T2), rc, tc, hist, lane));
            acc.H += t;
            continue;
        }
        const Part1 r = count_1d_general(ap, P, B, T0, T1, T2, Mk, off0, t, tc, lane, hist);
        add_part(acc, r.p);
        if (r.uniform) acc.K += t;
        else {
            acc.Q += r.p.q;
            acc.H += t - r.p.q;
        }
    }
    flush(a, q, acc, lane, st);
}

// ------------------------------------------------------------- lane-parallel problems
// Whole 1-D problems inside a chunk, ONE PER LANE: the closed forms above are
// scalar work per (problem, access) -- a warp doing them in lockstep issues
// 32 copies of the same scalar instructions.  Lane l takes problem qa + l and
// handles its uniform-flag accesses (lane-count classes) and its depth <= 1
// residue-class accesses (<= 128 residues of one loop, evaluated per class in
// the lane); at the first access that needs the warp (deeper loop nests, block
// sizes whose warp-reps fall into many residue classes, collapse(2)) it hands
// the rest of its problem to the warp (queue of <= 32 entries).
#ifndef SEL_LANE_DYN
#define SEL_LANE_DYN 1      // warps take 32-nest chunks of a tile dynamically
#endif
#ifndef SEL_LANE_PF
#define SEL_LANE_PF 1       // L1 prefetch of the nest's next access descriptors (2: + the next nest into L2)
#endif
#ifndef SEL_LANE_OPS
#define SEL_LANE_OPS 1      // nominal lane-op accounting (count_nominal_ops); 0 drops it from the lane kernel
#endif
#if SEL_LANE_OPS
#define LANE_OPS(x) x
#else
#define LANE_OPS(x) ((void)0)
#endif
struct LaneSums {
    uint32_t W, L, S, C, U;
    unsigned long long ops;          // nominal algorithmic lane-ops of this thread
};

// uniform flags over a whole access, one lane (uniform_whole)
__device__ __forceinline__ void lane_uniform(const RepClasses& rc, uint32_t Mk, bool flags, uint32_t tmin,
                                             LaneSums& z) {
    auto cls = [&](uint32_t lanes, uint32_t reps) {
        LANE_OPS(z.ops += kOpsClass);
        const uint32_t w = reps * Mk;
        const uint32_t nl = flags ? lanes : 1u;             // lines = sectors per WA
        z.L += w * nl;
        z.S += w * nl;
        if (nl <= tmin) z.C += w;                           // R11
        else z.U += w * nl;
    };
    if (rc.n32) cls(32u, uint32_t(rc.n32));
    if (rc.nA) cls(rc.lanesA, uint32_t(rc.nA));
    if (rc.lanesR) cls(rc.lanesR, 1u);
}

// Residue classes of one access over a whole problem, ONE THREAD: the
// thread's own residue histogram lives in a shared-memory column (row-major
// over slots, one column per thread: bank = thread, conflict-free whatever
// the slot), built from its loops (depth <= 2), turned into prefix sums in
// place, and every warp-rep class is then evaluated in O(1) (class_sums).
// Element size >= 4 bytes: R = 128 / E <= 32 slots.
constexpr uint32_t kLaneThreads = 256;
constexpr uint32_t kLaneSlots = 32;
constexpr uint32_t kLaneP32 = kLaneSlots + 1;              // p32 rows after pf[0..R]
constexpr uint32_t kLaneRows = kLaneP32 + kLaneSlots / 4 + 1;
struct Col {
    uint32_t* p;
    __device__ __forceinline__ uint32_t& operator[](uint32_t s) const { return p[s * kLaneThreads]; }
};

__device__ __forceinline__ void lane_hist_build(Col h, uint32_t R, uint32_t sh, const sel_access& a, uint32_t T0,
                                                uint32_t T1, unsigned long long& ops) {
    for (uint32_t s = 0; s < R; s++) h[s] = 0u;
    const uint32_t d = a.depth;
    if (d == 0) {
        h[0] = 1u;
        return;
    }
    const uint32_t kA = uint32_t(uint64_t(a.c_inner[0]));
    const uint32_t lA = loop_period_log2(kA), pA = 1u << lA, nA = T0 < pA ? T0 : pA;
    if (d == 1) {
        LANE_OPS(ops += kOpsHistEntry * nA);
        for (uint32_t i = 0; i < nA; i++) h[((kA * i) & 127u) >> sh] = (T0 - i + pA - 1u) >> lA;
        return;
    }
    // depth 2: every (i, j) residue pair of the two loops' one-loop histograms
    const uint32_t kB = uint32_t(uint64_t(a.c_inner[1]));
    const uint32_t lB = loop_period_log2(kB), pB = 1u << lB, nB = T1 < pB ? T1 : pB;
    LANE_OPS(ops += kOpsHistEntry * (nA + nB) + kOpsConvTerm * nA * nB);
    for (uint32_t i = 0; i < nA; i++) {
        const uint32_t ci = (T0 - i + pA - 1u) >> lA, oi = kA * i;
        for (uint32_t j = 0; j < nB; j++) {
            const uint32_t cj = (T1 - j + pB - 1u) >> lB;
            h[((oi + kB * j) & 127u) >> sh] += ci * cj;
        }
    }
}

// h[0..R) -> exclusive prefix pf[0..R] in place; p32 rows: the prefix of h
// folded mod 32 bytes (R / 4 slots)
__device__ __forceinline__ void lane_hist_prefix(Col h, uint32_t R, unsigned long long& ops) {
    const uint32_t R32 = R >> 2;
    LANE_OPS(ops += kOpsPrefixEntry * (R + R32));
    uint32_t run = 0;
    for (uint32_t u = 0; u < R32; u++) {
        run += h[u] + h[u + R32] + h[u + 2u * R32] + h[u + 3u * R32];
        h[kLaneP32 + 1u + u] = run;
    }
    h[kLaneP32] = 0u;
    run = 0;
    for (uint32_t s = 0; s < R; s++) {
        const uint32_t v = h[s];
        h[s] = run;
        run += v;
    }
    h[R] = run;
}

__device__ __forceinline__ void lane_add(LaneSums& z, const ClassSums& c, uint32_t w) {
    z.L += w + c.lf;
    z.S += w + c.sf;
    z.C += c.cc;
    z.U += (w - c.cc) + c.uf;
}

// one access (depth <= 2, E >= 4, 0 < |c_par| < 128): its residue histogram
// and prefix sums in the thread's column (shared by every block size class
// of the nest), then the warp-rep classes of one problem (B, WR, rc)
__device__ __forceinline__ void lane_hist_prepare(Col h, const sel_access& a, uint32_t T0, uint32_t T1,
                                                  unsigned long long& ops) {
    const uint32_t sh = uint32_t(__ffs(a.elem_bytes) - 1), R = 128u >> sh;
    lane_hist_build(h, R, sh, a, T0, T1, ops);
    lane_hist_prefix(h, R, ops);
}
#ifndef SEL_LANE_BLOCK_PERIOD
#define SEL_LANE_BLOCK_PERIOD 1
#endif
#ifndef SEL_LANE_ONE_EVAL
#define SEL_LANE_ONE_EVAL 1
#endif
__device__ __forceinline__ void lane_hist_eval(Col h, const sel_access& a, uint32_t P, uint32_t B, uint32_t WR,
                                               const RepClasses& rc, uint32_t tmin, LaneSums& z) {
    const uint32_t sh = uint32_t(__ffs(a.elem_bytes) - 1), R = 128u >> sh;
    const Col p32{h.p + kLaneP32 * kLaneThreads};
    const uint32_t Ht = h[R];                               // = Mk
    const int64_t c0 = a.c_par[0];
    const uint32_t g = uint32_t(uabs(c0));
    const bool neg = c0 < 0;
    const uint32_t base32 = uint32_t(uint64_t(a.base)), c032 = uint32_t(uint64_t(c0));
    auto cls = [&](uint32_t lo, uint32_t nm1, uint32_t mult) {
        LANE_OPS(z.ops += kOpsEvalClass);
        lane_add(z, class_sums(h, p32, R, sh, lo, nm1, g, tmin, mult), Ht * mult);
    };
    auto lo_of = [&](uint32_t p0, uint32_t n) { return base32 + c032 * p0 + (neg ? c032 * (n - 1u) : 0u); };
#if SEL_LANE_BLOCK_PERIOD
    // Element sizes >= 4 (the only ones the lane kernel sends here) make 32 c
    // = 0 (mod 128): every full warp of a block has the lowest lane address of
    // the block's first warp (mod 128 -- all class_sums looks at).  When 32 | B
    // or c B = 0 (mod 128) the warp-reps fall into the lane-count classes of
    // rep_classes (count_hist_whole); otherwise block kb's offset c kb B (mod
    // 128) repeats with period pi = 128 / gcd(c B, 128), so the complete
    // blocks' warp-reps fall into <= 2 min(pi, #blocks) classes (full warps,
    // the B mod 32 tail warp) with multiplicities, plus the last block's full
    // warps and tail (R8, R9) -- the same integers as walking every warp-rep.
    // The classes are enumerated as items through ONE call site of class_sums
    // (its copies were the kernel's code size).
    const bool whole = (B & 31u) == 0 || ((c032 * B) & 127u) == 0;
    const uint32_t nfull = (B - 1u) >> 5, lt = B & 31u;
    const uint32_t nbf = uint32_t(rc.nA), rem_full = whole ? 0u : uint32_t(rc.n32) - nbf * nfull;
    const uint32_t lp = whole ? 0u : 7u - uint32_t(__ffs((c032 * B) & 127u) - 1);   // log2 pi
    const uint32_t nr = whole ? 0u : (nbf < (1u << lp) ? nbf : (1u << lp));
    const uint32_t items = whole ? 3u : 2u * nr + 2u;
    for (uint32_t x = 0; x < items; x++) {
        uint32_t p0, n, mult;
        if (whole) {
            if (x == 0) { p0 = 0u; n = 32u; mult = uint32_t(rc.n32); }
            else if (x == 1) { p0 = 0u; n = rc.lanesA; mult = uint32_t(rc.nA); }
            else { p0 = rc.nA ? 0u : uint32_t(32u * rc.n32); n = rc.lanesR; mult = rc.lanesR ? 1u : 0u; }
        } else if (x < 2u * nr) {
            const uint32_t r = x >> 1, m = ((nbf - 1u - r) >> lp) + 1u;   // complete blocks kb = r (mod pi)
            const bool tail = x & 1u;
            p0 = r * B + (tail ? 32u * nfull : 0u);
            n = tail ? lt : 32u;
            mult = tail ? m : m * nfull;
        } else if (x == 2u * nr) {
            p0 = nbf * B; n = 32u; mult = rem_full;
        } else {
            p0 = nbf * B + 32u * rem_full; n = rc.lanesR; mult = rc.lanesR ? 1u : 0u;
        }
        if (mult) cls(lo_of(p0, n), n - 1u, mult);
    }
    (void)WR;
    (void)P;
#else
    if ((B & 31u) == 0 || (((c032 * B) | (32u * g)) & 127u) == 0) {
        // the lowest lane address mod 128 of a warp-rep depends on its lane count only
        // (or, for 32 | B, on the warp-rep index mod 4): count_hist_whole's classes
        if (rc.n32) {
            if (((32u * c032) & 127u) == 0) cls(lo_of(0u, 32u), 31u, uint32_t(rc.n32));
            else
                for (uint32_t j = 0; j < 4; j++) {
                    const uint32_t cj = uint32_t((rc.n32 + 3u - j) >> 2);
                    if (cj) cls(lo_of(32u * j, 32u), 31u, cj);
                }
        }
        if (rc.nA) cls(lo_of(0u, rc.lanesA), rc.lanesA - 1u, uint32_t(rc.nA));
        if (rc.lanesR) cls(lo_of(rc.nA ? 0u : uint32_t(32u * rc.n32), rc.lanesR), rc.lanesR - 1u, 1u);
    } else {
        // every warp-rep from the block geometry (R8, R9), as count_hist_reps
        const uint32_t wpb = (B + 31u) >> 5;
        uint32_t kb = 0, w = 0;
        for (uint32_t m = 0; m < WR; m++) {
            const uint32_t p0 = kb * B + 32u * w;
            uint32_t pe = p0 + 32u;
            pe = pe < (kb + 1u) * B ? pe : (kb + 1u) * B;
            pe = pe < P ? pe : P;
            const uint32_t nm1 = pe - p0 - 1u;
            cls(base32 + c032 * p0 + (neg ? c032 * nm1 : 0u), nm1, 1u);
            if (++w == wpb) { w = 0; kb++; }
        }
    }
#endif
}

// Small problems (k_problem_w: 1-D, W <= kSmallMaxW, WR <= kSmallMaxWR), one
// UNIT per thread: a nest with all of its block size classes in direct mode
// (problems u * n_cls + c; the classes share the nest's residue histograms),
// one problem otherwise.  A block takes a tile of kLaneTile units and sorts
// them by a shape key (accesses, loop depth, collapse) in shared memory, so a
// warp's lanes run nests of one shape side by side instead of 32 different
// loop structures.  A thread hands the accesses it cannot count to the warp
// kernel (k_queue): entry = problem << 32 | mask of handed accesses.
#ifndef SEL_LANE_NEST_KEY
#define SEL_LANE_NEST_KEY 1
#endif
#ifndef SEL_LANE_MIN_BLOCKS
#define SEL_LANE_MIN_BLOCKS 2
#endif
#ifndef SEL_LANE_GRP
#define SEL_LANE_GRP 3
#endif
constexpr uint32_t kLaneGrp = SEL_LANE_GRP;   // problems of a unit counted together
#ifndef SEL_LANE_TILE
#define SEL_LANE_TILE 4096
#endif
constexpr uint32_t kLaneTile = SEL_LANE_TILE;   // units sorted per block tile
constexpr uint32_t kLaneKeyBits = 8;
constexpr uint32_t kLaneKeys = 1u << kLaneKeyBits;
constexpr size_t kLaneSmem = (size_t(kLaneRows) * kLaneThreads + kLaneTile + kLaneKeys) * sizeof(uint32_t);

// shape key of a unit: direct mode, the nest's key from k_problem_w (one
// coalesced byte; it also hashes the accesses' counting paths and element
// sizes, which k_problem_w sees anyway -- loading descriptors here for that
// cost more than it gained, profiles/r01_variants_v8/); otherwise accesses,
// loop depth and collapse of the problem's nest.
__device__ __forceinline__ uint32_t lane_unit_key(const CountArgs& a, uint64_t u, bool direct) {
#if SEL_LANE_NEST_KEY
    if (direct) return a.nest_key[u];
#endif
    const uint32_t nid = direct ? uint32_t(u) : a.prob_nest[u];
    if (nid == kNoProblem) return 0u;
    return nest_shape_key(a.nests[nid]);
}

template <int MODE>
__global__ void __launch_bounds__(kLaneThreads, SEL_LANE_MIN_BLOCKS) k_lane_problems(const __grid_constant__ CountArgs a) {
    extern __shared__ uint32_t s_lane[];                    // hist columns | tile order | key counts
#if SEL_LANE_DYN
    __shared__ uint32_t s_next;                             // next 32-nest chunk of the tile
#endif
    uint32_t* s_order = s_lane + kLaneRows * kLaneThreads;
    uint32_t* s_cnt = s_order + kLaneTile;
    const Col hcol{s_lane + threadIdx.x};
    const int lane = threadIdx.x & 31;
    const bool direct = a.hdr->direct != 0;
    const uint32_t ncls = direct ? a.hdr->n_cls : 1u;
    const uint64_t qb = a.hdr->small_begin, qe = a.hdr->small_end;

    const uint64_t ub = qb / ncls, ue = (qe + ncls - 1) / ncls;
    unsigned long long sK = 0, sH = 0;                      // statistics: WAs by path (64-bit: ADVICE r01)
    unsigned long long sW = 0, sOps = 0;
    // tile size: kLaneTile units when there are enough to keep every block busy
    // (c5: 3.1 M nests), else the units spread over the grid in tiles of at
    // least 512 (small batches no longer run on a few blocks)
    const uint64_t per_block = (ue - ub + gridDim.x - 1) / gridDim.x;
#ifndef SEL_LANE_BALANCE
#define SEL_LANE_BALANCE 1
#endif
#if SEL_LANE_BALANCE
    // the fewest waves of tiles of <= kLaneTile units, and the tile size that
    // fills the last wave (c5: 3.1 M nests on 296 blocks -> 3 waves of 3584,
    // not 2.58 waves of 4096 whose last wave leaves 42 % of the blocks idle)
    const uint64_t waves = (per_block + kLaneTile - 1) / kLaneTile;
    const uint64_t per_wave = waves ? (per_block + waves - 1) / waves : 0;
    const uint32_t tile = uint32_t(per_wave <= 512 ? 512u
                                   : umin64(((per_wave + kLaneThreads - 1) / kLaneThreads) * kLaneThreads, kLaneTile));
#else
    const uint32_t tile = uint32_t(per_block >= kLaneTile ? kLaneTile
                                   : per_block <= 512 ? 512u : ((per_block + kLaneThreads - 1) / kLaneThreads) * kLaneThreads);
#endif
    for (uint64_t t0 = ub + uint64_t(blockIdx.x) * tile; t0 < ue; t0 += uint64_t(gridDim.x) * tile) {
        const uint32_t nt = uint32_t(umin64(tile, ue - t0));
        // ---- sort the tile's units by shape key (counting sort in shared memory)
        for (uint32_t i = threadIdx.x; i < kLaneKeys; i += blockDim.x) s_cnt[i] = 0u;
#if SEL_LANE_DYN
        if (threadIdx.x == 0) s_next = 0u;
#endif
        __syncthreads();
        uint32_t key[kLaneTile / kLaneThreads];
#pragma unroll
        for (uint32_t r = 0; r < kLaneTile / kLaneThreads; r++) {
            const uint32_t i = r * kLaneThreads + threadIdx.x;
            key[r] = i < nt ? lane_unit_key(a, t0 + i, direct) : 0u;
            if (i < nt) atomicAdd(&s_cnt[key[r]], 1u);
        }
        __syncthreads();
        if (threadIdx.x < 32) {                             // exclusive scan of the 256 key counts
            uint32_t v[kLaneKeys / 32], sum = 0;
#pragma unroll
            for (uint32_t j = 0; j < kLaneKeys / 32; j++) { v[j] = s_cnt[threadIdx.x * (kLaneKeys / 32) + j]; sum += v[j]; }
            uint32_t x = sum;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, x, o);
                if (lane >= o) x += y;
            }
            uint32_t run = x - sum;
#pragma unroll
            for (uint32_t j = 0; j < kLaneKeys / 32; j++) { s_cnt[threadIdx.x * (kLaneKeys / 32) + j] = run; run += v[j]; }
        }
        __syncthreads();
#pragma unroll
        for (uint32_t r = 0; r < kLaneTile / kLaneThreads; r++) {
            const uint32_t i = r * kLaneThreads + threadIdx.x;
            if (i < nt) s_order[atomicAdd(&s_cnt[key[r]], 1u)] = i;
        }
        __syncthreads();
        // ---- count: round r, thread t takes the unit at sorted position r * threads + t
#if SEL_LANE_DYN
        // warps take 32-nest chunks of the sorted tile from a shared counter:
        // chunks of different shapes cost different times, and a static round
        // assignment left warps idle at the end-of-tile barrier
        for (;;) {
            uint32_t chunk = 0;
            if (lane == 0) chunk = atomicAdd(&s_next, 1u);
            chunk = __shfl_sync(kFull, chunk, 0);
            if (chunk * 32u >= nt) break;
            const uint32_t i = chunk * 32u + uint32_t(lane);
#else
        for (uint32_t r = 0; r * kLaneThreads < nt; r++) {
            const uint32_t i = r * kLaneThreads + threadIdx.x;
#endif
            const bool has = i < nt;
            const uint64_t u = has ? t0 + s_order[i] : 0ull;
#if SEL_LANE_PF >= 2
            // the next round's nest into L2 while this one is counted
            if (i + kLaneThreads < nt && direct)
                asm volatile("prefetch.global.L2 [%0];" ::"l"(a.nests + (t0 + s_order[i + kLaneThreads])));
#endif

            for (uint32_t g0 = 0; g0 < ncls; g0 += kLaneGrp) {
                // problems q = u * ncls + g0 + c of this group that are small and in this call's range
                uint32_t B[kLaneGrp], WR[kLaneGrp], hm[kLaneGrp];
                RepClasses rc[kLaneGrp];
                LaneSums z[kLaneGrp];
                uint32_t vmask = 0, rc_wr = 0;          // rc_wr: WR of these classes still to take from rc
                uint64_t Mit = 0;
                sel_nest nest{};
                if (has) {
                    // direct ids: one 8-byte per-nest record (k_problem_w) says which classes are
                    // small, valid and non-empty, and gives M_it; WR follows from the warp-rep classes
                    const uint2 li = direct ? a.lane_info[u] : make_uint2(0u, 0u);
                    Mit = li.x;
#pragma unroll
                    for (uint32_t c = 0; c < kLaneGrp; c++) {
                        hm[c] = 0u;
                        z[c] = LaneSums{0u, 0u, 0u, 0u, 0u, 0ull};
                        B[c] = 0u;
                        WR[c] = 0u;
                        rc[c] = RepClasses{0ull, 0ull, 0u, 0u};
                        const uint32_t ci = g0 + c;
                        const uint64_t q = u * ncls + ci;
                        if (ci >= ncls || q < qb || q >= qe) continue;
                        if (direct && ci < 32) {
                            if ((li.y >> ci) & 1u) {
                                vmask |= 1u << c;
                                rc_wr |= 1u << c;
                                B[c] = a.cls_B[ci];
                            }
                        } else if (a.prefix[q + 1] == a.prefix[q]) {
                            const uint64_t WR64 = a.prob_WR[q];
                            const uint64_t M = a.prob_cnt[q * kCntStride + 5];
                            if (WR64 * M) {                                   // small, valid, W > 0
                                vmask |= 1u << c;
                                WR[c] = uint32_t(WR64);
                                B[c] = a.prob_B[q];
                                Mit = M;
                            }
                        }
                    }
                }
                if (vmask) {
                    nest = a.nests[direct ? uint32_t(u) : a.prob_nest[u]];
#pragma unroll
                    for (uint32_t c = 0; c < kLaneGrp; c++)
                        if ((vmask >> c) & 1u) {
                            rc[c] = rep_classes(nest.P0, B[c]);
                            if ((rc_wr >> c) & 1u)
                                WR[c] = uint32_t(rc[c].n32 + rc[c].nA) + (rc[c].lanesR ? 1u : 0u);
                        }
                    const uint32_t T0 = uint32_t(eff_trip(nest.trip[0])), T1 = uint32_t(eff_trip(nest.trip[1])),
                                   T2 = uint32_t(eff_trip(nest.trip[2]));
                    const sel_access* ap = a.acc + nest.access_off;
#if SEL_LANE_PF >= 1
                    // the nest's access descriptors are read one after another, each
                    // load on the critical path: touch the next line ahead of time
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(ap + 2));
#endif
                    for (uint32_t k = 0; k < nest.n_access; k++, ap++) {
#if SEL_LANE_PF >= 1
                        if ((k & 1u) == 0u && k + 4u < nest.n_access)
                            asm volatile("prefetch.global.L1 [%0];" ::"l"(ap + 4));
#endif
                        if (k == 31) {                      // accesses 31, 32, ...: all to the warp kernel
#pragma unroll
                            for (uint32_t c = 0; c < kLaneGrp; c++) hm[c] |= ((vmask >> c) & 1u) << 31;
                            break;
                        }
                        const sel_access ac = *ap;
                        const uint32_t d = ac.depth;
                        const uint32_t Mk = d == 0 ? 1u : d == 1 ? T0 : d == 2 ? T0 * T1 : T0 * T1 * T2;
                        if (Mk == 0) continue;
                        const uint32_t tc = ac.elem_bytes <= 4 ? 1u : ac.elem_bytes == 8 ? 2u : 4u;   // R11
                        const uint32_t g = uint32_t(umin64(uabs(ac.c_par[0]), 128));
                        if (g == 0 || g == 128) {
#pragma unroll
                            for (uint32_t c = 0; c < kLaneGrp; c++)
                                if ((vmask >> c) & 1u) {
                                    lane_uniform(rc[c], Mk, g != 0, tc, z[c]);
                                    sK += uint64_t(WR[c]) * Mk;
                                    z[c].W += WR[c] * Mk;
                                }
                        } else if (d <= 2 && ac.elem_bytes >= 4 && a.residue_classes) {
                            lane_hist_prepare(hcol, ac, T0, T1, z[0].ops);
#if SEL_LANE_ONE_EVAL
                            // the block-size classes through ONE inlined copy of lane_hist_eval (its
                            // class_sums evaluations dominate the kernel; code size showed in the
                            // stalls): the class's inputs and sums picked with constant indices
#pragma unroll 1
                            for (uint32_t c = 0; c < kLaneGrp; c++) {
                                if (!((vmask >> c) & 1u)) continue;
                                uint32_t Bc = B[0], WRc = WR[0];
                                RepClasses rcc = rc[0];
#pragma unroll
                                for (uint32_t i = 1; i < kLaneGrp; i++)
                                    if (c == i) { Bc = B[i]; WRc = WR[i]; rcc = rc[i]; }
                                LaneSums dz{0u, 0u, 0u, 0u, 0u, 0ull};
                                lane_hist_eval(hcol, ac, uint32_t(nest.P0), Bc, WRc, rcc, tc, dz);
                                dz.W = WRc * Mk;
#pragma unroll
                                for (uint32_t i = 0; i < kLaneGrp; i++)
                                    if (c == i) {
                                        z[i].W += dz.W; z[i].L += dz.L; z[i].S += dz.S; z[i].C += dz.C; z[i].U += dz.U;
                                        LANE_OPS(z[i].ops += dz.ops);
                                    }
                                sH += uint64_t(WRc) * Mk;
                            }
#else
#pragma unroll
                            for (uint32_t c = 0; c < kLaneGrp; c++)
                                if ((vmask >> c) & 1u) {
                                    lane_hist_eval(hcol, ac, uint32_t(nest.P0), B[c], WR[c], rc[c], tc, z[c]);
                                    sH += uint64_t(WR[c]) * Mk;
                                    z[c].W += WR[c] * Mk;
                                }
#endif
                        } else {
#pragma unroll
                            for (uint32_t c = 0; c < kLaneGrp; c++) hm[c] |= ((vmask >> c) & 1u) << k;   // to k_queue
                        }
                    }
#pragma unroll
                    for (uint32_t c = 0; c < kLaneGrp; c++) {
                        if (!((vmask >> c) & 1u)) continue;
                        const uint64_t q = u * ncls + g0 + c;
                        sW += uint64_t(WR[c]) * Mit;
                        LANE_OPS(sOps += z[c].ops);
                        {   // the only writer so far (k_problem_w leaves these counters unzeroed): store
                            unsigned long long* pc = a.prob_cnt + q * kCntStride;
                            if (a.hdr->n_parts == 1) {         // the whole 48-byte record, M_it included
                                ulonglong2* p2 = reinterpret_cast<ulonglong2*>(pc);
                                p2[0] = make_ulonglong2(z[c].W, z[c].L);
                                p2[1] = make_ulonglong2(z[c].S, z[c].C);
                                p2[2] = make_ulonglong2(z[c].U, Mit);
                            } else if (z[c].W) {
                                atomicAdd(pc + 0, (unsigned long long)z[c].W);
                                atomicAdd(pc + 1, (unsigned long long)z[c].L);
                                atomicAdd(pc + 2, (unsigned long long)z[c].S);
                                atomicAdd(pc + 3, (unsigned long long)z[c].C);
                                atomicAdd(pc + 4, (unsigned long long)z[c].U);
                            }
                        }

                    }
                }
                // warp-aggregated append of the handed problems to the queue (converged)
#pragma unroll
                for (uint32_t c = 0; c < kLaneGrp; c++) {
                    const bool enq = ((vmask >> c) & 1u) && hm[c] != 0u;
                    const unsigned m = __ballot_sync(kFull, enq);
                    if (m) {
                        unsigned long long base = 0;
                        if (lane == __ffs(m) - 1) base = atomicAdd(&a.hdr->queue_len, (unsigned long long)__popc(m));
                        base = __shfl_sync(kFull, base, __ffs(m) - 1);
                        if (enq) a.queue[base + __popc(m & lanemask_lt())] = ((u * ncls + g0 + c) << 32) | hm[c];
                    }
                }
            }

        }
        __syncthreads();                                    // s_order / s_cnt are rewritten by the next tile
    }
    unsigned long long K = sK, H = sH, Wt = sW;
    for (int o = 16; o; o >>= 1) {
        K += __shfl_xor_sync(kFull, K, o);
        H += __shfl_xor_sync(kFull, H, o);
        Wt += __shfl_xor_sync(kFull, Wt, o);
    }
    if (K && lane == 0) atomicAdd((unsigned long long*)&a.hdr->stats.wa_closed_form, K);
    if (H && lane == 1) atomicAdd((unsigned long long*)&a.hdr->stats.wa_residue_classes, H);
    if (Wt && lane == 2) atomicAdd((unsigned long long*)&a.hdr->stats.wa_resolved, Wt);
    for (int o = 16; o; o >>= 1) sOps += __shfl_xor_sync(kFull, sOps, o);
    if (sOps && lane == 3) atomicAdd((unsigned long long*)&a.hdr->stats.alg_lane_ops, sOps);
}

// The handed-over accesses of small problems, one warp per queue entry.
// Entries are taken 32 at a time: lane j loads entry j's problem metadata
// (independent loads, one latency for the batch), then the warp walks the
// batch with the metadata broadcast by shuffles.  The descriptors of the
// handed accesses of entry j+1 are copied to shared memory (cp.async, 16 B per
// request, lane = access) while entry j is counted, so an entry waits for no
// global load of its own (up to kPrefetch accesses; more read global memory).
constexpr uint32_t kPrefetch = 8;

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const uint32_t sa = uint32_t(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// lane k (< 31) with bit k of the handed mask and rank r < kPrefetch among the
// set bits copies descriptor k (64 B) to buf[r]
__device__ __forceinline__ void prefetch_accesses(sel_access* buf, const sel_access* acc_nest, uint32_t hm, int lane) {
    if (lane < 31 && ((hm >> lane) & 1u)) {
        const uint32_t r = uint32_t(__popc(hm & ((1u << lane) - 1u)));
        if (r < kPrefetch) {
            const char* src = reinterpret_cast<const char*>(acc_nest + lane);
            char* dst = reinterpret_cast<char*>(buf + r);
#pragma unroll
            for (int c = 0; c < 4; c++) cp_async16(dst + 16 * c, src + 16 * c);
        }
    }
    cp_async_commit();
}

template <int MODE>
__global__ void __launch_bounds__(SEL_COUNT_THREADS, SEL_COUNT_MIN_BLOCKS) k_queue(const __grid_constant__ CountArgs a) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    __shared__ uint32_t s_hist[SEL_COUNT_THREADS / 32][kHistWords];
    __shared__ __align__(16) sel_access s_acc[SEL_COUNT_THREADS / 32][2][kPrefetch];
    uint32_t* hist = a.residue_classes ? s_hist[wid] : nullptr;
    const uint64_t n = a.hdr->queue_len;
    WarpStats st{0ull, 0ull, 0ull, 0ull};
    unsigned long long e0 = 0;
    if (lane == 0) e0 = atomicAdd(&a.hdr->queue_ctr, 32ull);
    e0 = __shfl_sync(kFull, e0, 0);
    while (e0 < n) {
        const uint32_t nb = uint32_t(umin64(32, n - e0));
        // lane j: metadata of entry e0 + j
        uint32_t q_l = 0, hm_l = 0, B_l = 0, WR_l = 0, P_l = 0, T0_l = 0, T1_l = 0, T2_l = 0, ao_l = 0;
        if (uint32_t(lane) < nb) {
            const unsigned long long v = a.queue[e0 + lane];
            q_l = uint32_t(v >> 32);
            hm_l = uint32_t(v);
            uint32_t nid_l;
            problem_nest_B(a, q_l, nid_l, B_l);
            const sel_nest* np = a.nests + nid_l;
            WR_l = uint32_t(a.prob_WR[q_l]);
            P_l = uint32_t(np->P0);
            T0_l = uint32_t(eff_trip(np->trip[0]));
            T1_l = uint32_t(eff_trip(np->trip[1]));
            T2_l = uint32_t(eff_trip(np->trip[2]));
            ao_l = np->access_off;
        }
        // the next batch's start, fetched while this one is counted
        unsigned long long e_next = 0;
        if (lane == 0) e_next = atomicAdd(&a.hdr->queue_ctr, 32ull);
        prefetch_accesses(s_acc[wid][0], a.acc + __shfl_sync(kFull, ao_l, 0), __shfl_sync(kFull, hm_l, 0) & 0x7fffffffu,
                          lane);
        for (uint32_t j = 0; j < nb; j++) {
            const uint32_t q = __shfl_sync(kFull, q_l, j), hmask = __shfl_sync(kFull, hm_l, j);
            const uint32_t B = __shfl_sync(kFull, B_l, j), WR = __shfl_sync(kFull, WR_l, j);
            const uint32_t P = __shfl_sync(kFull, P_l, j);
            const uint32_t T0 = __shfl_sync(kFull, T0_l, j), T1 = __shfl_sync(kFull, T1_l, j),
                           T2 = __shfl_sync(kFull, T2_l, j);
            const uint32_t aoff = __shfl_sync(kFull, ao_l, j);
            const uint32_t jn = j + 1 < nb ? j + 1 : j;             // (a dummy copy of j itself at the end)
            const uint32_t hm_n = __shfl_sync(kFull, hm_l, jn), ao_n = __shfl_sync(kFull, ao_l, jn);
            prefetch_accesses(s_acc[wid][(j + 1) & 1], a.acc + ao_n, j + 1 < nb ? hm_n & 0x7fffffffu : 0u, lane);
            cp_async_wait<1>();                                     // entry j's copies have landed
            __syncwarp();
            const sel_access* buf = s_acc[wid][j & 1];
            Acc acc{};
            uint32_t rank = 0;
            for (uint32_t mk = hmask & 0x7fffffffu; mk; mk &= mk - 1u, rank++) {
                const uint32_t k = uint32_t(__ffs(mk) - 1);
                const sel_access* ap = rank < kPrefetch ? buf + rank : a.acc + aoff + k;
                const sel_access ac = *ap;
                const uint32_t d = ac.depth;
                const uint32_t Mk = d == 0 ? 1u : d == 1 ? T0 : d == 2 ? T0 * T1 : T0 * T1 * T2;
                const uint32_t Wk = WR * Mk;
                const uint32_t tc = ac.elem_bytes <= 4 ? 1u : ac.elem_bytes == 8 ? 2u : 4u;   // R11
                const uint32_t g = uint32_t(uabs(ac.c_par[0]));
                const uint32_t cB = uint32_t(uint64_t(ac.c_par[0])) * B;
                Part p;
                if (!hist) {
                    p = count_1d_general(ap, P, B, T0, T1, T2, Mk, 0, Wk, tc, lane, hist).p;
                    acc.Q += p.q;
                    acc.H += Wk - p.q;
                } else if ((B & 31u) == 0 || ((cB | (32u * g)) & 127u) == 0) {
                    p = count_hist_whole(ac, int(d), T0, T1, T2, rep_classes(P, B), tc, hist, lane);
                    acc.H += Wk;
                } else {
                    p = count_hist_reps(ap, int(d), T0, T1, T2, P, B, WR, tc, hist, lane);
                    acc.H += Wk;
                }
                add_part(acc, p);
                acc.W += Wk;
            }
            flush(a, q, acc, lane, st);
            if (hmask >> 31) {                              // accesses 31, 32, ...: the general path
                uint32_t woff = 0;
                for (uint32_t k = 0; k < 31; k++) {
                    const uint32_t d = a.acc[aoff + k].depth;
                    woff += WR * (d == 0 ? 1u : d == 1 ? T0 : d == 2 ? T0 * T1 : T0 * T1 * T2);
                }
                const uint64_t Wq = uint64_t(WR) * a.prob_cnt[uint64_t(q) * kCntStride + 5];
                count_problem<MODE>(a, q, woff, uint32_t(Wq - woff), lane, hist, st);
            }
            __syncwarp();                                   // buffer j & 1 is refilled for entry j + 2
        }
        cp_async_wait<0>();
        __syncwarp();
        e0 = __shfl_sync(kFull, e_next, 0);
    }
    stats_flush(a, st, lane);
}

template <int MODE>
__global__ void __launch_bounds__(SEL_COUNT_THREADS, SEL_COUNT_MIN_BLOCKS) k_count(const __grid_constant__ CountArgs a) {
    const int lane = threadIdx.x & 31;
    __shared__ uint32_t s_hist[SEL_COUNT_THREADS / 32][kHistWords];
    uint32_t* hist = a.residue_classes ? s_hist[threadIdx.x >> 5] : nullptr;
    const uint64_t nq = a.hdr->n_problems;
    if (nq == 0) return;
    const uint64_t base = a.hdr->w_begin, end = a.hdr->w_end;   // this call's slice of [0, prefix[nq])
    if (end <= base) return;
    const uint64_t total = end - base;
    const uint64_t nwarps = uint64_t(gridDim.x) * (blockDim.x >> 5);
    uint64_t ch = total / (nwarps * 16);
    ch = ch < 256 ? 256 : (ch > kMaxChunk ? kMaxChunk : ch);
    WarpStats st{0ull, 0ull, 0ull, 0ull};
    for (;;) {
        unsigned long long chunk = 0;
        if (lane == 0) chunk = atomicAdd(&a.hdr->chunk_ctr, 1ull);
        chunk = __shfl_sync(kFull, chunk, 0);
        if (chunk * ch >= total) break;
        const uint64_t start = base + chunk * ch;
        uint32_t len = uint32_t(umin64(ch, end - start));
        uint64_t q = find_problem(a.prefix, nq, start, lane);
        uint64_t off = start - a.prefix[q];
        while (len > 0) {
            const uint64_t Wq = a.prefix[q + 1] - a.prefix[q];
            if (off >= Wq) {
                off -= Wq;
                q++;
                continue;
            }
            const uint32_t take = uint32_t(umin64(Wq - off, len));
            count_problem<MODE>(a, q, off, take, lane, hist, st);
            len -= take;
            off = 0;
            q++;
        }
    }
    stats_flush(a, st, lane);
}

// persistent grid: #SMs x resident blocks of kernel k
template <typename K>
static int persistent_grid(K k, int threads, size_t smem = 0) {
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, threads, smem);
    return sms * (per > 0 ? per : 1);
}

template <int MODE>
static void launch_mode(const CountArgs& a, cudaStream_t s) {
    static int g_count = 0, g_queue = 0, g_lane = 0;
    const size_t lane_smem = kLaneSmem;
    if (g_count == 0) {
        g_count = persistent_grid(k_count<MODE>, SEL_COUNT_THREADS);
        g_queue = persistent_grid(k_queue<MODE>, SEL_COUNT_THREADS);
        g_lane = persistent_grid(k_lane_problems<MODE>, kLaneThreads, kLaneSmem);
    }
    if (MODE != 0) {
        prof_begin(SEL_PROF_K_LANE, s);
        k_lane_problems<MODE><<<g_lane, kLaneThreads, lane_smem, s>>>(a);
        prof_end(SEL_PROF_K_LANE, s);
        k_queue<MODE><<<g_queue, SEL_COUNT_THREADS, 0, s>>>(a);
        note_launch(2);
    }
    k_count<MODE><<<g_count, SEL_COUNT_THREADS, 0, s>>>(a);
    note_launch();
}

cudaError_t launch_count(const sel_tables& t, const WsPtrs& w, uint64_t max_problems, uint32_t flags,
                         cudaStream_t s) {
    (void)max_problems;
    const int mode = (flags & SEL_F_MATCH_ANY) ? 0 : (flags & SEL_F_SCALAR) ? 1 : 2;
    CountArgs a{t.nests, t.accesses, w.prob_nest, w.prob_B, w.prob_W, w.prob_WR, w.prob_cnt, w.hdr, 1u,
                (flags & SEL_F_EXPAND_ALL) ? 0u : 1u, (flags & SEL_F_NO_RESIDUE_CLASSES) ? 0u : 1u,
                w.queue, w.nest_key, w.lane_info, w.cls + kClsMax};
    prof_before_count(s);
    if (mode == 0) launch_mode<0>(a, s);
    else if (mode == 1) launch_mode<1>(a, s);
    else launch_mode<2>(a, s);
    prof_after_count(s);
    return cudaGetLastError();
}

}  // namespace sel
