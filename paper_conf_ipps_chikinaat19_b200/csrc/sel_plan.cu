// sel_plan.cu -- turns a batch of candidates into counting problems.
//
// Counts (a1-a3) of a candidate depend only on its nest and on B when
// 32 does not divide B (every warp is then an aligned 32-iteration chunk of
// the parallel iteration space), never on G_max or the device set
// (DESIGN.md "Count sharing").  Candidates that share (nest, B class) are
// therefore counted once: a per-nest slot table collects the distinct B
// classes (warp-aggregated with __match_any_sync), the classes are sorted
// so problem ids are deterministic, and a device-wide scan assigns ids.
// Each problem then gets its closed-form number of warp-accesses
// W = WR * M_it, and a second scan turns those into the prefix the counting
// kernel partitions.  Everything stays on the device (no host sync).
#include "sel_device.cuh"
#include "sel_internal.h"

namespace sel {

// ------------------------------------------------------------------- scan
// Exclusive scan of unsigned 64-bit values in place: x[0..n) -> prefix,
// x[n] = total.  n is read from *n_dev when given (device-side count).
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(const unsigned long long* x, uint64_t n_host,
                                                              const unsigned long long* n_dev,
                                                              unsigned long long* partial, const unsigned* skip) {
    if (skip && *skip) return;
    const uint64_t n = n_dev ? *n_dev : n_host;
    __shared__ unsigned long long red[kScanThreads / 32];
    // grid-stride over chunks (the grid is sized for the host's upper bound of n)
    for (uint64_t b = blockIdx.x; b * kScanItems <= n; b += gridDim.x) {
        const uint64_t begin = b * kScanItems;
        unsigned long long s = 0;
        for (int i = 0; i < kScanPer; i++) {
            uint64_t idx = begin + uint64_t(i) * kScanThreads + threadIdx.x;
            if (idx < n) s += x[idx];
        }
        for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long t = 0;
            for (int w = 0; w < kScanThreads / 32; w++) t += red[w];
            partial[b] = t;
        }
        __syncthreads();
    }
}

// single block: exclusive scan of the per-block partial sums
__global__ void __launch_bounds__(1024) k_scan_partials(unsigned long long* partial, uint64_t nb_host,
                                                        uint64_t n_host, const unsigned long long* n_dev,
                                                        const unsigned* skip) {
    if (skip && *skip) return;
    const uint64_t n = n_dev ? *n_dev : n_host;
    uint64_t nb = (n + kScanItems - 1) / kScanItems;
    if (nb > nb_host) nb = nb_host;
    __shared__ unsigned long long wsum[32];
    __shared__ unsigned long long carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (uint64_t base = 0; base < nb; base += 1024) {
        uint64_t i = base + threadIdx.x;
        unsigned long long v = i < nb ? partial[i] : 0, inc = v;
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long y = __shfl_up_sync(kFull, inc, o);
            if ((threadIdx.x & 31) >= o) inc += y;
        }
        if ((threadIdx.x & 31) == 31) wsum[threadIdx.x >> 5] = inc;
        __syncthreads();
        if (threadIdx.x < 32) {
            unsigned long long w = wsum[threadIdx.x], wi = w;
            for (int o = 1; o < 32; o <<= 1) {
                unsigned long long y = __shfl_up_sync(kFull, wi, o);
                if (threadIdx.x >= o) wi += y;
            }
            wsum[threadIdx.x] = wi - w;
        }
        __syncthreads();
        unsigned long long excl = carry + wsum[threadIdx.x >> 5] + inc - v;
        if (i < nb) partial[i] = excl;
        __syncthreads();
        if (threadIdx.x == 1023) carry = excl + v;
        __syncthreads();
    }
    if (threadIdx.x == 0) partial[nb] = carry;
}

__global__ void __launch_bounds__(kScanThreads) k_scan_down(unsigned long long* x, uint64_t n_host,
                                                            const unsigned long long* n_dev,
                                                            const unsigned long long* partial, const unsigned* skip) {
    if (skip && *skip) return;
    const uint64_t n = n_dev ? *n_dev : n_host;
    __shared__ unsigned long long wsum[kScanThreads / 32];
    for (uint64_t b = blockIdx.x; b * kScanItems <= n; b += gridDim.x) {
        const uint64_t begin = b * kScanItems;
        if (begin == n) {                       // the chunk that owns x[n] = total
            if (threadIdx.x == 0) x[n] = partial[b];
            continue;
        }
        // each thread scans kScanPer consecutive items
        const uint64_t my = begin + uint64_t(threadIdx.x) * kScanPer;
        unsigned long long v[kScanPer], s = 0;
        for (int i = 0; i < kScanPer; i++) {
            v[i] = (my + i < n) ? x[my + i] : 0;
            s += v[i];
        }
        unsigned long long inc = s;
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long y = __shfl_up_sync(kFull, inc, o);
            if ((threadIdx.x & 31) >= o) inc += y;
        }
        if ((threadIdx.x & 31) == 31) wsum[threadIdx.x >> 5] = inc;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long c = 0;
            for (int w = 0; w < kScanThreads / 32; w++) { unsigned long long t = wsum[w]; wsum[w] = c; c += t; }
        }
        __syncthreads();
        unsigned long long run = partial[b] + wsum[threadIdx.x >> 5] + inc - s;
        for (int i = 0; i < kScanPer; i++) {
            if (my + i < n) x[my + i] = run;
            run += v[i];
        }
        const uint64_t last = begin + kScanItems;
        if (last >= n && threadIdx.x == 0 && n < last) x[n] = partial[b + 1];
        __syncthreads();                        // wsum is rewritten by the next chunk
    }
}

// skip (device flag, optional): set by the plan when every x[i] is zero -- the
// prefix is then all zero and only x[n] = 0 must be written (k_drop_unused)
static cudaError_t scan_u64(unsigned long long* x, uint64_t n_max, const unsigned long long* n_dev,
                            unsigned long long* partial, cudaStream_t s, const unsigned* skip = nullptr) {
    const uint64_t nb = (n_max + kScanItems) / kScanItems;     // covers index n_max as well
    const unsigned g = unsigned(nb < 148u * 8 ? nb : 148u * 8);  // grid-stride over the chunks
    k_scan_reduce<<<g, kScanThreads, 0, s>>>(x, n_max, n_dev, partial, skip);
    k_scan_partials<<<1, 1024, 0, s>>>(partial, nb, n_max, n_dev, skip);
    k_scan_down<<<g, kScanThreads, 0, s>>>(x, n_max, n_dev, partial, skip);
    note_launch(3);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ plan
// Direct problem ids (launch tables of <= kClsMax entries whose nests x
// classes fit the workspace): the distinct B classes of the launch table,
// sorted, give every launch a class index, and problem = nest * n_cls +
// class index -- deterministic, no slot table, no pass over the candidates
// (k_problem_w sets up every nest x class problem; k_model_tile derives the
// id of each candidate).  One block; O(n_launches^2) comparisons.
__global__ void __launch_bounds__(1024) k_classes(sel_tables t, uint64_t n, uint64_t n_nests, int dedup,
                                                  WsHeader* hdr, uint32_t* cls) {
    __shared__ uint32_t s_bc[kClsMax];
    __shared__ uint8_t s_first[kClsMax];
    __shared__ uint32_t s_ncls;
    const uint64_t nl = t.n_launches;
    if (!dedup || nl == 0 || nl > kClsMax) {
        if (threadIdx.x == 0) {
            hdr->direct = 0;
            hdr->n_nests_scan = n_nests;
        }
        return;
    }
    if (threadIdx.x == 0) s_ncls = 0;
    for (uint32_t i = threadIdx.x; i < nl; i += blockDim.x) s_bc[i] = b_class(t.launches[i].block);
    __syncthreads();
    uint32_t nf = 0;
    for (uint32_t i = threadIdx.x; i < nl; i += blockDim.x) {
        uint8_t first = 1;
        for (uint32_t j = 0; j < i; j++)
            if (s_bc[j] == s_bc[i]) { first = 0; break; }
        s_first[i] = first;
        nf += first;
    }
    atomicAdd(&s_ncls, nf);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < nl; i += blockDim.x) {
        uint32_t rank = 0;
        for (uint32_t j = 0; j < nl; j++) rank += (s_first[j] && s_bc[j] < s_bc[i]) ? 1u : 0u;
        cls[i] = rank;
        if (s_first[i]) cls[kClsMax + rank] = s_bc[i];
    }
    if (threadIdx.x == 0) {
        const uint64_t ncls = s_ncls;
        const bool direct = n_nests * ncls <= n;
        hdr->direct = direct ? 1u : 0u;
        hdr->n_cls = uint32_t(ncls);
        hdr->n_nests_scan = direct ? 0ull : n_nests;
    }
}

// V1-V2 per candidate; dedup: the candidate's problem id directly (direct
// mode), or insert its B class into its nest's slot table (one CAS per
// distinct key per warp).
__global__ void __launch_bounds__(256) k_insert(const sel_candidate* __restrict__ cands, uint64_t n,
                                                sel_tables t, int n_sets, uint32_t* slots,
                                                uint8_t* cand_status, int dedup, uint32_t* prob_nest,
                                                uint32_t* prob_B, uint32_t* cand_pid, const WsHeader* hdr,
                                                const uint32_t* cls) {
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    // direct mode: the model kernel derives problem ids and validates V1-V2
    // itself, and every (nest, class) pair is a problem -- no pass over the
    // candidates here
    if (dedup && hdr->direct) return;
    for (uint64_t base = uint64_t(blockIdx.x) * blockDim.x; base < n; base += stride) {
        const uint64_t c = base + threadIdx.x;
        const bool in = c < n;
        const unsigned inmask = __ballot_sync(kFull, in);
        if (!in) continue;
        const sel_candidate cd = cands[c];
        const uint8_t st = validate_candidate(cd, t, n_sets);
        cand_status[c] = st;
        if (!dedup) {
            cand_pid[c] = st ? kNoProblem : uint32_t(c);          // kNoProblem <=> candidate invalid (all modes)
            prob_nest[c] = st ? kNoProblem : cd.nest_id;
            prob_B[c] = st ? 0u : t.launches[cd.launch_id].block;
            continue;
        }
        const uint32_t bc = st ? 0u : b_class(t.launches[cd.launch_id].block);
        const unsigned long long key = st ? ~0ull : ((unsigned long long)cd.nest_id << 32) | bc;
        const unsigned peers = __match_any_sync(inmask, key);
        const int leader = __ffs(peers) - 1;
        if (st == 0 && (threadIdx.x & 31) == leader) {
            // open addressing from a hashed start slot (k_rank_slots sorts the slots
            // afterwards, so positions do not matter): usually one CAS, not a chain
            uint32_t* s = slots + uint64_t(cd.nest_id) * kSlots;
            const uint32_t h0 = (bc * 0x9E3779B1u) >> 29;
            for (int j = 0; j < kSlots; j++) {
                const uint32_t old = atomicCAS(s + ((h0 + j) & (kSlots - 1)), 0u, bc);
                if (old == 0u || old == bc) break;
            }
        }
    }
}

// sort each nest's B classes (deterministic ids) and count them
__global__ void __launch_bounds__(256) k_rank_slots(uint32_t* slots, uint64_t n_nests,
                                                    unsigned long long* nest_cnt, const WsHeader* hdr) {
    const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i >= n_nests || hdr->direct) return;
    uint32_t v[kSlots];
    int m = 0;
    for (int j = 0; j < kSlots; j++) {
        uint32_t x = slots[i * kSlots + j];
        if (x) v[m++] = x;
    }
    for (int a = 1; a < m; a++) {
        uint32_t x = v[a];
        int b = a - 1;
        while (b >= 0 && v[b] > x) { v[b + 1] = v[b]; b--; }
        v[b + 1] = x;
    }
    for (int j = 0; j < kSlots; j++) slots[i * kSlots + j] = j < m ? v[j] : 0u;
    nest_cnt[i] = (unsigned long long)m;
}

__device__ __forceinline__ void assign_one(const sel_candidate* __restrict__ cands, uint64_t c, const sel_tables& t,
                                           const uint32_t* slots, const unsigned long long* nest_base,
                                           uint64_t n_nests, const uint8_t* cand_status, uint32_t* cand_pid,
                                           uint32_t* prob_nest, uint32_t* prob_B, WsHeader* hdr) {
    if (cand_status[c]) { cand_pid[c] = kNoProblem; return; }
    const sel_candidate cd = cands[c];
    const uint32_t bc = b_class(t.launches[cd.launch_id].block);
    const uint32_t* s = slots + uint64_t(cd.nest_id) * kSlots;
    uint64_t pid = ~0ull;
    for (int j = 0; j < kSlots; j++) {
        if (s[j] == bc) { pid = nest_base[cd.nest_id] + j; break; }
    }
    if (pid == ~0ull) pid = nest_base[n_nests] + atomicAdd(&hdr->n_overflow, 1u);   // slot table full
    cand_pid[c] = uint32_t(pid);
    // identical values from every sharer: one write per distinct problem of the warp
    const unsigned peers = __match_any_sync(__activemask(), pid);
    if ((threadIdx.x & 31) == __ffs(peers) - 1) {
        prob_nest[pid] = cd.nest_id;
        prob_B[pid] = bc;
    }
}

__global__ void __launch_bounds__(256) k_assign(const sel_candidate* __restrict__ cands, uint64_t n,
                                                sel_tables t, const uint32_t* slots,
                                                const unsigned long long* nest_base, uint64_t n_nests,
                                                const uint8_t* cand_status, uint32_t* cand_pid,
                                                uint32_t* prob_nest, uint32_t* prob_B, WsHeader* hdr) {
    if (hdr->direct) return;
    for (uint64_t c = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; c < n; c += uint64_t(gridDim.x) * blockDim.x)
        assign_one(cands, c, t, slots, nest_base, n_nests, cand_status, cand_pid, prob_nest, prob_B, hdr);
}
__global__ void k_finalize_plan(WsHeader* hdr, const unsigned long long* nest_base, uint64_t n_nests,
                                uint64_t n, int dedup, uint32_t part, uint32_t n_parts) {
    const bool direct = dedup && hdr->direct;
    unsigned long long np = !dedup ? n : direct ? n_nests * hdr->n_cls : nest_base[n_nests] + hdr->n_overflow;
    hdr->n_problems = np;
    hdr->part = part;
    hdr->n_parts = n_parts;
    hdr->chunk_ctr = 0;
    hdr->stats.n_candidates = n;
    hdr->stats.n_problems = direct ? 0ull : np;        // direct mode: k_problem_w counts the used ids
}

// closed-form W = WR * M_it per problem (+ nest validation V3-V6)
// The counters of a small problem with W > 0 are not zeroed here: in a
// single-part call the lane kernel thread that counts it STORES its sums
// (k_queue adds the handed-over accesses afterwards).
// returns bit 0: counted through the WA prefix (big), bit 1: counted by the lane kernel (small, W > 0)
__device__ __forceinline__ uint32_t problem_w_one(uint64_t q, const sel_nest& nest, uint8_t st, uint64_t M_it,
                                              uint32_t B, unsigned long long* prob_W,
                                              unsigned long long* prob_WR, uint8_t* prob_status,
                                              unsigned long long* prob_cnt, int lane_ok, bool one_part,
                                              bool lane_mit = false) {
    prob_status[q] = st;
    if (st) {
        for (int f = 0; f < kCntStride; f++) prob_cnt[q * kCntStride + f] = 0;
        prob_W[q] = 0;
        prob_WR[q] = 0;
        return 0u;
    }
    const uint64_t WR = warp_reps(nest.P0 * nest.P1, B);
    prob_WR[q] = WR;
    // small problems are counted one per lane (k_lane_problems), outside the prefix
    const uint64_t W = WR * M_it;
    const bool small = lane_ok && nest.par_dims == 1 && W <= kSmallMaxW && WR <= kSmallMaxWR;
    prob_W[q] = small ? 0ull : W;
    // lane_mit: the lane kernel writes this problem's whole counter record,
    // M_it included (one full 48-byte record instead of an 8-byte store here)
    if (!(lane_mit && small && W != 0 && one_part)) prob_cnt[q * kCntStride + 5] = M_it;
    if (!(small && W != 0 && one_part))
        for (int f = 0; f < 5; f++) prob_cnt[q * kCntStride + f] = 0;     // W, L, S, C, U
    return (!small && W != 0 ? 1u : 0u) | (small && W != 0 ? 2u : 0u);
}

#ifndef SEL_PW_MIN_BLOCKS
#define SEL_PW_MIN_BLOCKS 4      // 64 registers, 4 blocks per SM: 0.386 -> 0.349 ms (3 blocks at 78 registers before)
#endif
__global__ void __launch_bounds__(256, SEL_PW_MIN_BLOCKS) k_problem_w(sel_tables t, WsHeader* hdr, const uint32_t* prob_nest,
                                                   const uint32_t* prob_B, unsigned long long* prob_W,
                                                   unsigned long long* prob_WR, uint8_t* prob_status,
                                                   unsigned long long* prob_cnt, int lane_ok, uint8_t* nest_key,
                                                   uint32_t* prob_nest_w, uint32_t* prob_B_w, const uint32_t* cls,
                                                   uint8_t* prob_used, uint2* lane_info) {
    const uint64_t nq = hdr->n_problems;
    const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
    (void)prob_nest_w;                                      // direct mode no longer materialises nest / B per
    (void)prob_B_w;                                         // problem (problem_nest_B derives them)
    if (hdr->direct) {
        // direct ids: the problems of nest i are i * n_cls + [0, n_cls), every
        // one of them counted (direct mode requires n_nests * n_cls <= n, so
        // at most one problem per candidate; a big problem no candidate refers
        // to is dropped again by k_mark_big / k_drop_unused).  A warp
        // takes 32 nests (lane = nest), checks the concatenation of their access
        // lists 32 accesses at a time (lane = access: the descriptor loads are
        // independent and, for consecutive nests, contiguous), reduces each
        // nest's flags and M_it (saturating) over its lanes, and the nest's lane
        // writes its n_cls problems.
        __shared__ uint32_t s_flags[8][32];
        __shared__ unsigned long long s_mit[8][32];
        __shared__ uint32_t s_paths[8][32], s_emask[8][32];
        const uint32_t ncls = hdr->n_cls;
        const uint64_t nn = ncls ? nq / ncls : 0;
        const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
        const uint64_t nwarps = uint64_t(gridDim.x) * (blockDim.x >> 5);
        uint32_t used = 0, big = 0;
        for (uint64_t i0 = (uint64_t(blockIdx.x) * (blockDim.x >> 5) + wib) * 32; i0 < nn; i0 += nwarps * 32) {
            const uint64_t i = i0 + lane;
            sel_nest nest{};
            uint8_t pre = SEL_EINVAL;
            if (i < nn) {
                nest = t.nests[i];
                pre = nest_precheck(nest, t.n_accesses);
            }
            const uint32_t na = pre == SEL_OK ? nest.n_access : 0u;
            uint32_t incl = na;                                 // inclusive prefix of the access counts
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            const uint32_t tot = __shfl_sync(kFull, incl, 31);
            const uint64_t P = smul(nest.P0, nest.P1);
            s_flags[wib][lane] = 0u;
            s_paths[wib][lane] = 0u;
            s_emask[wib][lane] = 0u;
            s_mit[wib][lane] = 0ull;
            __syncwarp();
            for (uint32_t j0 = 0; j0 < tot; j0 += 32) {
                const uint32_t j = j0 + uint32_t(lane);
                // owner: the first lane whose inclusive prefix exceeds j
                int own = 0;
#pragma unroll
                for (int step = 16; step; step >>= 1) {
                    const uint32_t v = __shfl_sync(kFull, incl, own + step - 1);
                    if (v <= j) own += step;
                }
                own = own > 31 ? 31 : own;
                const uint32_t ex = __shfl_sync(kFull, incl - na, own);
                const uint32_t aoff = __shfl_sync(kFull, nest.access_off, own);
                const uint32_t pd = __shfl_sync(kFull, uint32_t(nest.par_dims), own);
                const uint32_t dp = __shfl_sync(kFull, uint32_t(nest.depth), own);
                const uint64_t Po = __shfl_sync(kFull, P, own), P0o = __shfl_sync(kFull, nest.P0, own),
                               P1o = __shfl_sync(kFull, nest.P1, own);
                const uint64_t T[3] = {eff_trip(__shfl_sync(kFull, nest.trip[0], own)),
                                       eff_trip(__shfl_sync(kFull, nest.trip[1], own)),
                                       eff_trip(__shfl_sync(kFull, nest.trip[2], own))};
                uint32_t fl = 0, paths = 0, em = 0;
                uint64_t Mk = 0;
                if (j < tot) {
                    const sel_access ac = t.accesses[aoff + (j - ex)];
                    fl = access_check(ac, pd, dp, Po, P0o, P1o, T, &Mk);
                    // the counting path the lane kernel will take (for its shape sort), 8-bit counts
                    const uint64_t g = uabs(ac.c_par[0]);
                    const uint32_t path = (g == 0 || g >= 128) ? 0u : ac.elem_bytes < 4 ? 3u : ac.depth <= 1 ? 1u :
                                          ac.depth == 2 ? 2u : 3u;
                    paths = 1u << (8u * path);
                    em = 1u << (__ffs(ac.elem_bytes) & 31);
                }
                // segmented (by owner) sum over the lanes of this round: the owner's
                // lanes are contiguous from seg_lo (its first access in this round),
                // so lane l takes lane l - o's values iff l - o >= seg_lo; the flags
                // and the element-size mask travel in one word (both OR-combined),
                // and M_k in 32 bits when every lane's is below 2^26 (no overflow in
                // 32 terms), else 64-bit saturating
                const bool in = j < tot;
                const int seg_lo = int(ex) - int(j0) > 0 ? int(ex) - int(j0) : 0;
                uint32_t flem = fl | (em << 8);
                if (__all_sync(kFull, Mk < (1ull << 26))) {
                    uint32_t m32 = uint32_t(Mk);
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(kFull, m32, o);
                        const uint32_t yf = __shfl_up_sync(kFull, flem, o), yp = __shfl_up_sync(kFull, paths, o);
                        if (lane - o >= seg_lo) {
                            m32 += y;
                            flem |= yf;
                            paths += yp;
                        }
                    }
                    Mk = m32;
                } else {
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint64_t y = __shfl_up_sync(kFull, Mk, o);
                        const uint32_t yf = __shfl_up_sync(kFull, flem, o), yp = __shfl_up_sync(kFull, paths, o);
                        if (lane - o >= seg_lo) {
                            Mk = sadd(Mk, y);
                            flem |= yf;
                            paths += yp;
                        }
                    }
                }
                fl = flem & 0xffu;
                em = flem >> 8;
                const int nxt = __shfl_down_sync(kFull, own, 1);
                const bool tail = in && (lane == 31 || j + 1 >= tot || nxt != own);
                if (tail) {                                     // one lane per owner per round
                    s_mit[wib][own] = sadd(s_mit[wib][own], Mk);
                    s_flags[wib][own] |= fl;
                    s_paths[wib][own] += paths;
                    s_emask[wib][own] |= em;
                }
                __syncwarp();
            }
            if (i < nn) {
                nest_key[i] = nest_shape_key(nest, s_paths[wib][lane], s_emask[wib][lane]);
                const uint64_t M_it = s_mit[wib][lane];
                const uint8_t st = nest_status(pre, s_flags[wib][lane], P, M_it);
                uint32_t lane_mask = 0;
                for (uint32_t c = 0; c < ncls; c++) {
                    const uint64_t q = i * ncls + c;
                    used++;
                    // (nest and B of a direct id are derived where needed: problem_nest_B)
                    const uint32_t r = problem_w_one(q, nest, st, st == SEL_OK ? M_it : 0ull, cls[kClsMax + c],
                                                     prob_W, prob_WR, prob_status, prob_cnt, lane_ok,
                                                     hdr->n_parts == 1, c < 32);
                    if (r & 1u) prob_used[q] = 0;              // k_mark_big / k_drop_unused look at big ones only
                    big += r & 1u;
                    if (c < 32) lane_mask |= ((r >> 1) & 1u) << c;
                }
                // the lane kernel's per-nest view: one 8-byte load instead of per-class prefix / WR / M_it
                lane_info[i] = make_uint2(uint32_t(M_it < 0xffffffffull ? M_it : 0xffffffffull), lane_mask);
            }
            __syncwarp();
        }
        used = __reduce_add_sync(kFull, used);
        big = __reduce_add_sync(kFull, big);
        if ((threadIdx.x & 31) == 0 && used) atomicAdd((unsigned long long*)&hdr->stats.n_problems, (unsigned long long)used);
        if ((threadIdx.x & 31) == 0 && big) atomicAdd((unsigned long long*)&hdr->n_big, (unsigned long long)big);
        return;
    }
    // grid-stride: the grid is sized for the candidates, the problems (known on
    // the device only) are usually an order of magnitude fewer
    for (uint64_t q = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; q < nq; q += stride) {
        const uint32_t nid = prob_nest[q];
        sel_nest nest{};
        uint64_t M_it = 0;
        uint8_t st = SEL_EINVAL;
        if (nid != kNoProblem) {
            nest = t.nests[nid];
            st = validate_nest(nest, t.accesses, t.n_accesses, &M_it);
        }
        problem_w_one(q, nest, st, M_it, prob_B[q], prob_W, prob_WR, prob_status, prob_cnt, lane_ok,
                      hdr->n_parts == 1);
    }
}

// Direct mode with big problems (counted warp-access by warp-access through
// the prefix): mark the ones some valid candidate refers to, then drop the
// others from the prefix (unreferenced small problems are left in: their
// closed-form counting costs O(accesses) per nest).  Both return at once when
// the batch has no big problem (c5) -- a launch each, no pass over the data.
__global__ void __launch_bounds__(256) k_mark_big(const sel_candidate* __restrict__ cands, uint64_t n, sel_tables t,
                                                  int n_sets, WsHeader* hdr, const uint32_t* cls,
                                                  const unsigned long long* prob_W, uint8_t* prob_used) {
    if (!hdr->direct || hdr->n_big == 0) return;
    const uint32_t ncls = hdr->n_cls;
    for (uint64_t c = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; c < n; c += uint64_t(gridDim.x) * blockDim.x) {
        const sel_candidate cd = cands[c];
        if (validate_candidate(cd, t, n_sets)) continue;
        const uint64_t q = uint64_t(cd.nest_id) * ncls + cls[cd.launch_id];
        if (prob_W[q] != 0 && !prob_used[q]) prob_used[q] = 1;
    }
}
__global__ void __launch_bounds__(256) k_drop_unused(WsHeader* hdr, unsigned long long* prob_W,
                                                     unsigned long long* prob_WR, unsigned long long* prob_cnt,
                                                     uint8_t* prob_status, const uint8_t* prob_used) {
    if (!hdr->direct) return;
    const uint64_t nq = hdr->n_problems;
    if (hdr->n_big == 0) {                        // no W in the prefix: all-zero, skip the scan
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            hdr->skip_scan = 1;
            prob_W[nq] = 0;
        }
        return;
    }
    uint32_t dropped = 0;
    for (uint64_t q = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; q < nq; q += uint64_t(gridDim.x) * blockDim.x) {
        if (prob_W[q] != 0 && !prob_used[q]) {
            prob_W[q] = 0;
            prob_WR[q] = 0;
            prob_cnt[q * kCntStride + 5] = 0;
            prob_status[q] = SEL_EINVAL;             // not counted; no candidate refers to it
            dropped++;
        }
    }
    dropped = __reduce_add_sync(kFull, dropped);
    if ((threadIdx.x & 31) == 0 && dropped)
        atomicAdd((unsigned long long*)&hdr->stats.n_problems, 0ull - (unsigned long long)dropped);
}

// slice [total*part/n_parts, total*(part+1)/n_parts) of the problem work space
// (one huge candidate's warp-accesses split R ways)
__global__ void k_plan_stats(WsHeader* hdr, const unsigned long long* prefix) {
    const unsigned __int128 total = prefix[hdr->n_problems];
    const uint64_t b = uint64_t(total * hdr->part / hdr->n_parts);
    const uint64_t e = uint64_t(total * (hdr->part + 1) / hdr->n_parts);
    hdr->w_begin = b;
    hdr->w_end = e;
    hdr->stats.wa_resolved = e - b;               // + the small problems' W (k_lane_problems)
    const unsigned __int128 nq = hdr->n_problems;
    hdr->small_begin = uint64_t(nq * hdr->part / hdr->n_parts);
    hdr->small_end = uint64_t(nq * (hdr->part + 1) / hdr->n_parts);
    hdr->queue_len = 0;
    hdr->queue_ctr = 0;
}

cudaError_t launch_plan(const sel_candidate* cands, uint64_t n, const sel_tables& t, int n_sets,
                        const WsPtrs& w, uint64_t n_nests, uint32_t flags, uint32_t part, uint32_t n_parts,
                        cudaStream_t s) {
    const bool dedup = !(flags & SEL_F_NO_DEDUP);
    prof_begin(SEL_PROF_PLAN, s);
    cudaError_t e = cudaMemsetAsync(w.hdr, 0, sizeof(WsHeader), s);
    if (e != cudaSuccess) return e;
    if (dedup && n_nests) {
        e = cudaMemsetAsync(w.slots, 0, n_nests * kSlots * sizeof(uint32_t), s);
        if (e != cudaSuccess) return e;
    }
    k_classes<<<1, 1024, 0, s>>>(t, n, n_nests, dedup ? 1 : 0, w.hdr, w.cls);
    const unsigned gb = unsigned((n + 255) / 256 < 148u * 64 ? (n + 255) / 256 : 148u * 64);
    k_insert<<<gb, 256, 0, s>>>(cands, n, t, n_sets, w.slots, w.cand_status, dedup ? 1 : 0, w.prob_nest,
                                w.prob_B, w.cand_pid, w.hdr, w.cls);
    note_launch(2);
    if (dedup) {
        if (n_nests) {
            k_rank_slots<<<unsigned((n_nests + 255) / 256), 256, 0, s>>>(w.slots, n_nests, w.nest_base, w.hdr);
            note_launch();
        }
        if ((e = scan_u64(w.nest_base, n_nests, &w.hdr->n_nests_scan, w.scan_tmp, s)) != cudaSuccess) return e;
        k_assign<<<gb, 256, 0, s>>>(cands, n, t, w.slots, w.nest_base, n_nests, w.cand_status, w.cand_pid,
                                    w.prob_nest, w.prob_B, w.hdr);
        note_launch();
    }
    k_finalize_plan<<<1, 1, 0, s>>>(w.hdr, w.nest_base, n_nests, n, dedup ? 1 : 0, part, n_parts);
    prof_begin(SEL_PROF_K_PROBLEM_W, s);
    k_problem_w<<<gb, 256, 0, s>>>(t, w.hdr, w.prob_nest, w.prob_B, w.prob_W, w.prob_WR,
                                                          w.prob_status, w.prob_cnt,
                                                          (flags & (SEL_F_MATCH_ANY | SEL_F_EXPAND_ALL |
                                                                    SEL_F_WARP_PROBLEMS)) ? 0 : 1,
                                                          w.nest_key, w.prob_nest, w.prob_B, w.cls, w.prob_used,
                                                          w.lane_info);
    prof_end(SEL_PROF_K_PROBLEM_W, s);
    note_launch(2);
    if (dedup) {
        k_mark_big<<<148u * 8, 256, 0, s>>>(cands, n, t, n_sets, w.hdr, w.cls, w.prob_W, w.prob_used);
        k_drop_unused<<<148u * 8, 256, 0, s>>>(w.hdr, w.prob_W, w.prob_WR, w.prob_cnt, w.prob_status, w.prob_used);
        note_launch(2);
    }
    if ((e = scan_u64(w.prob_W, n, &w.hdr->n_problems, w.scan_tmp, s, &w.hdr->skip_scan)) != cudaSuccess) return e;
    k_plan_stats<<<1, 1, 0, s>>>(w.hdr, w.prob_W);
    note_launch();
    prof_end(SEL_PROF_PLAN, s);
    return cudaGetLastError();
}

}  // namespace sel
