/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).  Not used by the
 * product path; only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load liboracle.so.
 *
 * A plain, slow, obviously correct CPU implementation of the hot path of
 * Chikin, Amaral, Ali, Tiotto, "Toward an Analytical Performance Model to
 * Select between GPU and CPU Execution" (IPDPSW 2019), PAPER.md cited as
 * P:L<line>.  Per candidate it
 *   (a1)   derives the runtime grid geometry and #OMP_Rep,
 *   (a2-3) enumerates every thread of every warp for every OpenMP repetition
 *          and every inner-loop iteration, computes each access's exact
 *          int64 byte address (the IPDA stride with runtime values bound,
 *          P:L231-256, L301) and counts the distinct 128 B lines and 32 B
 *          sectors per warp-access by sorting the lane values,
 *   (a4-6) evaluates Hong & Kim's MWP/CWP model with the #OMP_Rep factor
 *          (Figs. 4-5) literally, in fp64, in the order listed
 *          in DESIGN.md "Model sequence" (compile with -ffp-contract=off),
 *   (a7)   picks the target with the lower predicted time.
 * Readings R1-R31 resolve what the paper leaves open.
 *
 * Parity pins: tests/test_oracle_*.py (closed forms, brute force in pure
 * Python, the paper's worked examples, invariants) and, for the model half,
 * tests/test_oracle_hand.py: hand-computed candidates for every case of
 * Fig. 4, the bandwidth branch of Fig. 5, mixed coalesced / uncoalesced
 * weights, a non-integer #Rep, #OMP_Rep, an exact T_gpu and the NEXT row f4
 * extensions; scripts/mutate_oracle.py shows that 29 single-term mutations
 * of this file each fail one of them.  What stays unverifiable from PAPER.md
 * is the FORM of the Hong & Kim equations it does not print (Mem_L,
 * Departure_delay, MWP_Without_BW, #Rep, Comp/Mem cycles; readings R2, R5):
 * the pins fix this code to those equations as DESIGN.md restates them.
 */
#include "oracle.h"
#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#define LIM62 (1ULL << 62)
#define LIM48 (1ULL << 48)
#define LIM40 (1ULL << 40)

/* "all loops are assumed to execute 128 iterations" when unknown. */
static uint64_t eff_trip(uint32_t t) { return t == 0xFFFFFFFFu ? 128u : (uint64_t)t; }

static uint64_t ceil_div(uint64_t a, uint64_t b) { return a / b + (a % b != 0); }

static uint64_t umin(uint64_t a, uint64_t b) { return a < b ? a : b; }

/* min(x, y) as "x < y ? x : y" (DESIGN.md model sequence). */
static double dmin(double x, double y) { return x < y ? x : y; }

/* saturating helpers for the range checks */
static uint64_t sat_mul(uint64_t a, uint64_t b) {
    if (a == 0 || b == 0) return 0;
    if (a > UINT64_MAX / b) return UINT64_MAX;
    return a * b;
}
static uint64_t sat_add(uint64_t a, uint64_t b) { return (a > UINT64_MAX - b) ? UINT64_MAX : a + b; }
static uint64_t uabs64(int64_t v) { return v < 0 ? (uint64_t)0 - (uint64_t)v : (uint64_t)v; }

/* floor division by a power of two for signed addresses (R10). */
static int64_t floor_div(int64_t a, int64_t d) {
    int64_t q = a / d;
    if ((a % d != 0) && (a < 0)) q -= 1;
    return q;
}

/* number of distinct values among v[0..n) -- sort, then count changes */
static uint32_t count_distinct(int64_t* v, int n) {
    for (int i = 1; i < n; i++) {                 /* insertion sort */
        int64_t x = v[i];
        int j = i - 1;
        while (j >= 0 && v[j] > x) { v[j + 1] = v[j]; j--; }
        v[j + 1] = x;
    }
    uint32_t d = n > 0 ? 1 : 0;
    for (int i = 1; i < n; i++) if (v[i] != v[i - 1]) d++;
    return d;
}

/* tmin(e) = ceil(32 e / 128): the fewest lines a warp of 32 elements of e
 * bytes can touch; coalesced <=> lines <= tmin (reading R11). */
static uint64_t tmin_lines(uint64_t elem) { return ceil_div(32 * elem, 128); }

void oracle_geometry(uint64_t P, uint32_t B, uint32_t grid_max, uint64_t out[4]) {
    /* R6: the runtime launches ceil(P/B) blocks, capped at the maximum grid
     * geometry; each thread then runs #OMP_Rep = ceil(P / (G*B))
     * iterations (R27). */
    uint64_t G = umin(ceil_div(P, B), grid_max);
    uint64_t T = G * B;
    out[0] = G;
    out[1] = T;
    out[2] = T ? ceil_div(P, T) : 0;
    out[3] = ceil_div(B, 32);
}

static int valid_device(const or_device* d) {
    return d->num_sms >= 1 && d->max_warps_per_sm >= 1 && d->max_threads_per_sm >= 1 &&
           d->max_blocks_per_sm >= 1 && d->regs_per_sm >= 0 && d->smem_per_sm >= 0 &&
           d->sm_clock_hz > 0 && d->mem_bw_Bps > 0 && d->link_bw_Bps > 0 &&
           d->launch_overhead_s >= 0 && d->mem_ld_cycles > 0 && d->dep_del_coal > 0 &&
           d->dep_del_uncoal > 0 && d->issue_cycles > 0 && d->reg_alloc_unit >= 0 && d->warp_alloc_gran >= 0 &&
           d->smem_alloc_unit >= 0 && (d->txn_sectors == 0 || d->txn_sectors == 1);
}

/* ------------------------------------------------------------------ model */
void oracle_model(const or_device* dev, const or_nest* nest, const or_access* acc,
                  const or_launch* launch, const or_candidate* cand, or_result* r) {
    const uint64_t B = launch->block;
    const uint64_t P = nest->P0 * nest->P1;
    uint64_t T[3];
    for (int j = 0; j < 3; j++) T[j] = eff_trip(nest->trip[j]);

    uint64_t geo[4];
    oracle_geometry(P, launch->block, launch->grid_max, geo);
    r->G = geo[0]; r->T = geo[1]; r->R = geo[2]; r->wpb = geo[3];

    /* a4: #Mem_insts per thread per parallel iteration, M_it = sum_k prod_{j<depth_k} T_j (R14) */
    r->M_it = 0;
    for (uint32_t k = 0; k < nest->n_access; k++) {
        uint64_t m = 1;
        for (int j = 0; j < acc[k].depth; j++) m *= T[j];
        r->M_it += m;
    }

    /* a4: #Comp_insts per thread per parallel iteration (R14) */
    double comp = 0.0, prod = 1.0;
    for (int d = 0; d <= nest->depth; d++) {
        comp = comp + nest->comp_insts[d] * prod;
        if (d < nest->depth) prod = prod * (double)T[d];
    }
    r->comp = comp;

    /* a5: occupancy (R17) */
    uint64_t abps = (uint64_t)dev->max_blocks_per_sm;
    abps = umin(abps, (uint64_t)dev->max_warps_per_sm / r->wpb);
    abps = umin(abps, (uint64_t)dev->max_threads_per_sm / B);
    if (launch->regs_per_thread > 0) {
        if (dev->reg_alloc_unit > 0) {
            /* NEXT row f4, allocation granularity (reading F4c): registers are
             * allocated per warp in units of reg_alloc_unit, and the warps the
             * register file holds are rounded down to warp_alloc_gran */
            const uint64_t unit = (uint64_t)dev->reg_alloc_unit;
            const uint64_t regs_per_warp = ceil_div((uint64_t)launch->regs_per_thread * 32, unit) * unit;
            uint64_t warps = (uint64_t)dev->regs_per_sm / regs_per_warp;
            if (dev->warp_alloc_gran > 1) warps = (warps / (uint64_t)dev->warp_alloc_gran) * (uint64_t)dev->warp_alloc_gran;
            abps = umin(abps, warps / r->wpb);
        } else {
            abps = umin(abps, (uint64_t)dev->regs_per_sm / ((uint64_t)launch->regs_per_thread * B));
        }
    }
    if (launch->smem_per_block > 0) {
        /* F4c: shared memory is allocated per block in units of smem_alloc_unit */
        uint64_t smem_b = (uint64_t)launch->smem_per_block;
        if (dev->smem_alloc_unit > 0)
            smem_b = ceil_div(smem_b, (uint64_t)dev->smem_alloc_unit) * (uint64_t)dev->smem_alloc_unit;
        abps = umin(abps, (uint64_t)dev->smem_per_sm / smem_b);
    }
    abps = umin(abps, ceil_div(r->G, (uint64_t)dev->num_sms));
    r->abps = abps;
    r->active_sms = umin(r->G, (uint64_t)dev->num_sms);
    if (abps == 0) {
        r->status = OR_ELAUNCH;
        return;
    }
    const double N = (double)(abps * r->wpb);
    const double Rep = (double)r->G / ((double)abps * (double)r->active_sms);   /* R5 [H&K] */
    r->N = N;
    r->Rep = Rep;

    const double f_sm = dev->sm_clock_hz, issue = dev->issue_cycles;
    const double Mem_LD = dev->mem_ld_cycles, dd_c = dev->dep_del_coal, dd_u = dev->dep_del_uncoal;
    double Exec;
    if (r->W == 0) {
        /* R22: no memory instruction -- compute-bound case with Mem_L = 0 */
        r->hk_case = 0;
        Exec = (((issue * comp) * N) * Rep) * (double)r->R;
    } else {
        const uint64_t W = r->W, S = r->S, WR = r->WR;
        /* NEXT row f4, 32 B-sector transactions (reading F4d): every
         * warp-access is one class whose memory transactions are its distinct
         * sectors -- H&K's inputs with #Coal = 0 and uncoalesced transactions
         * U = S.  Otherwise 128 B lines with the R11 classes. */
        const uint64_t C = dev->txn_sectors ? 0 : r->C;
        const uint64_t U = dev->txn_sectors ? S : r->U;
        const double n_coal = (double)C / (double)WR;            /* #Coal_Mem_insts per warp */
        const double n_unc = (double)(W - C) / (double)WR;       /* #Uncoal_Mem_insts per warp */
        const double mem = (double)r->M_it;                      /* #Mem_insts (R4, R14) */
        const double w_unc = (double)(W - C) / (double)W;
        const double w_coal = (double)C / (double)W;
        const double upmw = (W > C) ? (double)U / (double)(W - C) : 0.0;   /* R12 */
        const double LB = (32.0 * (double)S) / (double)W;                   /* R13 */
        r->mem = mem;
        /* [H&K]: memory latency of coalesced / uncoalesced warps */
        r->MemL_u = Mem_LD + (upmw - 1.0) * dd_u;
        r->MemL_c = Mem_LD;
        r->MemL = r->MemL_u * w_unc + r->MemL_c * w_coal;
        r->Dep = (dd_u * upmw) * w_unc + dd_c * w_coal;
        /* Fig. 5 */
        const double MWPnbf = r->MemL / r->Dep;
        r->MWPnb = dmin(MWPnbf, N);
        r->BWpw = (f_sm * LB) / r->MemL;
        r->MWPbw = dev->mem_bw_Bps / (r->BWpw * (double)r->active_sms);
        r->MWP = dmin(dmin(r->MWPnb, r->MWPbw), N);
        r->Comp = issue * (comp + mem);                           /* [H&K] */
        r->Mem = r->MemL_u * n_unc + r->MemL_c * n_coal;          /* [H&K] */
        r->CWP = dmin((r->Mem + r->Comp) / r->Comp, N);
        const double Cp = r->Comp / mem;
        /* Fig. 4, conditions per readings R1-R3 */
        double E;
        if (r->MWP == N && r->CWP == N) {
            r->hk_case = 1;
            E = (r->Mem + r->Comp) + Cp * (r->MWP - 1.0);
        } else if (r->CWP >= r->MWP || r->Comp > r->Mem) {
            r->hk_case = 2;
            E = (r->Mem * N) / r->MWP + Cp * (r->MWP - 1.0);
        } else {
            r->hk_case = 3;
            E = r->MemL + r->Comp * N;
        }
        r->E = E;
        Exec = (E * Rep) * (double)r->R;                          /* x #Rep x #OMP_Rep */
        if (nest->n_sync > 0) {
            /* NEXT row f4, [H&K] synchronisation cost (readings F4a, F4b):
             * Departure_delay x (MWP - 1) x #synch x #Active_blocks_per_SM
             * x #Rep, once per OpenMP repetition. */
            const double Sync = ((((r->Dep * (r->MWP - 1.0)) * (double)nest->n_sync) * (double)abps) * Rep)
                                * (double)r->R;
            Exec = Exec + Sync;
        }
    }
    r->cycles = Exec;
    /* a7 (R20, R21) */
    r->t_gpu = (Exec / f_sm + (double)(nest->bytes_h2d + nest->bytes_d2h) / dev->link_bw_Bps)
               + dev->launch_overhead_s;
    r->t_cpu = cand->cpu_cycles / cand->cpu_hz;
    r->decision = (r->t_gpu < r->t_cpu) ? 1 : 0;
    r->status = OR_OK;
}

/* --------------------------------------------------------------- counting */
/* exact int64 byte address of access a for parallel iteration p and inner
 * indices i[] (a2; R25 for collapse(2)) */
static int64_t address(const or_access* a, const or_nest* n, uint64_t p, const uint64_t* i) {
    int64_t addr = a->base;
    if (n->par_dims == 1) {
        addr += a->c_par[0] * (int64_t)p;
    } else {
        addr += a->c_par[0] * (int64_t)(p / n->P1) + a->c_par[1] * (int64_t)(p % n->P1);
    }
    for (int j = 0; j < a->depth; j++) addr += a->c_inner[j] * (int64_t)i[j];
    return addr;
}

static void evaluate_one(const or_device* devs, int n_devs, const or_candidate* c,
                         const or_nest* nests, uint64_t n_nests, const or_access* acc_all,
                         uint64_t n_acc, const or_launch* launches, uint64_t n_launches,
                         or_result* r) {
    memset(r, 0, sizeof *r);
    r->decision = 0xFF;
    /* -------- validation (DESIGN.md "Validation" V1-V7, in order) */
    if (c->nest_id >= n_nests || c->launch_id >= n_launches || c->device_id >= (uint64_t)n_devs ||
        !(c->cpu_hz > 0.0)) { r->status = OR_EINVAL; return; }
    const or_nest* n = &nests[c->nest_id];
    const or_launch* l = &launches[c->launch_id];
    const or_device* dev = &devs[c->device_id];
    if (l->block < 1 || l->block > 1024 || l->grid_max < 1) { r->status = OR_EINVAL; return; }
    if ((n->par_dims != 1 && n->par_dims != 2) || n->depth > 3 || (n->par_dims == 1 && n->P1 != 1) ||
        (uint64_t)n->access_off + (uint64_t)n->n_access > n_acc) { r->status = OR_EINVAL; return; }
    const uint64_t P = sat_mul(n->P0, n->P1);
    if (n->P0 >= LIM40 || P >= LIM40) { r->status = OR_ERANGE; return; }
    uint64_t T[3];
    for (int j = 0; j < 3; j++) T[j] = eff_trip(n->trip[j]);
    const or_access* acc = acc_all + n->access_off;
    for (uint32_t k = 0; k < n->n_access; k++) {
        const or_access* a = &acc[k];
        const int64_t e = a->elem_bytes;
        if (!(e == 1 || e == 2 || e == 4 || e == 8 || e == 16) || a->depth > n->depth) {
            r->status = OR_EINVAL; return;
        }
        int bad = (a->base % e) != 0 || (a->c_par[0] % e) != 0 ||
                  (n->par_dims == 2 && (a->c_par[1] % e) != 0);
        for (int j = 0; j < a->depth; j++) bad |= (a->c_inner[j] % e) != 0;
        if (bad) { r->status = OR_EINVAL; return; }
    }
    for (uint32_t k = 0; k < n->n_access; k++) {
        const or_access* a = &acc[k];
        uint64_t e0 = (n->par_dims == 1) ? P : n->P0;
        uint64_t bound = uabs64(a->base);
        bound = sat_add(bound, sat_mul(uabs64(a->c_par[0]), e0 ? e0 - 1 : 0));
        if (n->par_dims == 2) bound = sat_add(bound, sat_mul(uabs64(a->c_par[1]), n->P1 ? n->P1 - 1 : 0));
        for (int j = 0; j < a->depth; j++) bound = sat_add(bound, sat_mul(uabs64(a->c_inner[j]), T[j] ? T[j] - 1 : 0));
        if (bound >= LIM62) { r->status = OR_ERANGE; return; }
    }
    uint64_t M_it = 0;                                  /* a4: sum_k prod_{j<depth_k} T_j */
    for (uint32_t k = 0; k < n->n_access; k++) {
        uint64_t m = 1;
        for (int j = 0; j < acc[k].depth; j++) m = sat_mul(m, T[j]);
        M_it = sat_add(M_it, m);
    }
    if (sat_mul(P, M_it) >= LIM48) { r->status = OR_ERANGE; return; }
    if (P == 0) {
        /* empty iteration space: nothing to offload (V8) */
        r->status = OR_OK; r->decision = 0; r->cycles = 0.0; r->t_gpu = INFINITY;
        r->t_cpu = c->cpu_cycles / c->cpu_hz;
        return;
    }

    /* -------- a1-a3: brute-force expansion of every warp-access */
    uint64_t geo[4];
    oracle_geometry(P, l->block, l->grid_max, geo);
    const uint64_t G = geo[0], Tt = geo[1], R = geo[2], wpb = geo[3], B = l->block;
    int64_t lanes_p[32], linev[32], secv[32];
    for (uint64_t rr = 0; rr < R; rr++) {
        for (uint64_t b = 0; b < G; b++) {
            for (uint64_t w = 0; w < wpb; w++) {
                int nl = 0;
                for (uint64_t ln = 0; ln < 32; ln++) {
                    uint64_t t = 32 * w + ln;                   /* threadIdx.x (R8) */
                    if (t >= B) break;
                    uint64_t p = rr * Tt + b * B + t;            /* cyclic, chunk 1 (R7) */
                    if (p < P) lanes_p[nl++] = (int64_t)p;        /* R9 */
                }
                if (nl == 0) continue;
                r->WR += 1;
                for (uint32_t k = 0; k < n->n_access; k++) {
                    const or_access* a = &acc[k];
                    const uint64_t tmin = tmin_lines(a->elem_bytes);
                    uint64_t i[3] = {0, 0, 0};
                    int done = 0;
                    for (int j = 0; j < a->depth; j++) if (T[j] == 0) done = 1;
                    while (!done) {
                        for (int q = 0; q < nl; q++) {
                            int64_t ad = address(a, n, (uint64_t)lanes_p[q], i);
                            linev[q] = floor_div(ad, 128);      /* 128 B line (R10) */
                            secv[q] = floor_div(ad, 32);        /* 32 B sector */
                        }
                        uint64_t lines = count_distinct(linev, nl);
                        uint64_t sectors = count_distinct(secv, nl);
                        r->W += 1;
                        r->L += lines;
                        r->S += sectors;
                        if (lines <= tmin) r->C += 1; else r->U += lines;   /* R11 */
                        /* next inner tuple, last loop fastest */
                        int j = (int)a->depth - 1;
                        while (j >= 0) {
                            if (++i[j] < T[j]) break;
                            i[j] = 0;
                            j--;
                        }
                        if (j < 0) done = 1;
                    }
                }
            }
        }
    }
    /* -------- a4-a7 */
    oracle_model(dev, n, acc, l, c, r);
    if (r->status != OR_OK) {
        uint8_t st = r->status;
        memset(r, 0, sizeof *r);
        r->status = st;
        r->decision = 0xFF;
    }
}

/* ------------------------------------------------------------- threading */
typedef struct {
    const or_device* devs; int n_devs;
    const or_candidate* cands; uint64_t n;
    const or_nest* nests; uint64_t n_nests;
    const or_access* acc; uint64_t n_acc;
    const or_launch* launches; uint64_t n_launches;
    or_result* out;
    uint64_t next;
} job;

static void* worker(void* arg) {
    job* J = (job*)arg;
    for (;;) {
        uint64_t i = __atomic_fetch_add(&J->next, 1, __ATOMIC_RELAXED);
        if (i >= J->n) break;
        evaluate_one(J->devs, J->n_devs, &J->cands[i], J->nests, J->n_nests, J->acc, J->n_acc,
                     J->launches, J->n_launches, &J->out[i]);
    }
    return NULL;
}

int oracle_evaluate(const or_device* devs, int n_devs, const or_candidate* cands, uint64_t n,
                    const or_nest* nests, uint64_t n_nests, const or_access* acc, uint64_t n_acc,
                    const or_launch* launches, uint64_t n_launches, or_result* out, int threads) {
    if (n == 0) return 0;
    if (!devs || n_devs < 1 || !cands || !nests || !launches || !out) return -1;
    for (int d = 0; d < n_devs; d++) if (!valid_device(&devs[d])) return -1;
    if (threads <= 0) threads = (int)sysconf(_SC_NPROCESSORS_ONLN);
    if (threads < 1) threads = 1;
    if ((uint64_t)threads > n) threads = (int)n;
    job J = {devs, n_devs, cands, n, nests, n_nests, acc, n_acc, launches, n_launches, out, 0};
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)threads);
    for (int t = 0; t < threads; t++) pthread_create(&th[t], NULL, worker, &J);
    for (int t = 0; t < threads; t++) pthread_join(th[t], NULL);
    free(th);
    return 0;
}

/* ---------------------------------------------------------------- layout */
size_t oracle_sizeof(int which) {
    switch (which) {
    case 0: return sizeof(or_device);
    case 1: return sizeof(or_access);
    case 2: return sizeof(or_nest);
    case 3: return sizeof(or_launch);
    case 4: return sizeof(or_candidate);
    case 5: return sizeof(or_result);
    default: return 0;
    }
}

#define OFF(T, f) ((size_t)offsetof(T, f))
size_t oracle_offsetof(int which, int field) {
    static const size_t dev[] = {OFF(or_device, num_sms), OFF(or_device, max_warps_per_sm),
        OFF(or_device, max_threads_per_sm), OFF(or_device, max_blocks_per_sm), OFF(or_device, regs_per_sm),
        OFF(or_device, smem_per_sm), OFF(or_device, sm_clock_hz), OFF(or_device, mem_bw_Bps),
        OFF(or_device, link_bw_Bps), OFF(or_device, launch_overhead_s), OFF(or_device, mem_ld_cycles),
        OFF(or_device, dep_del_coal), OFF(or_device, dep_del_uncoal), OFF(or_device, issue_cycles),
        OFF(or_device, reg_alloc_unit), OFF(or_device, warp_alloc_gran), OFF(or_device, smem_alloc_unit),
        OFF(or_device, txn_sectors)};
    static const size_t acc[] = {OFF(or_access, base), OFF(or_access, c_par), OFF(or_access, c_inner),
        OFF(or_access, elem_bytes), OFF(or_access, depth), OFF(or_access, is_store)};
    static const size_t nest[] = {OFF(or_nest, P0), OFF(or_nest, P1), OFF(or_nest, trip), OFF(or_nest, par_dims),
        OFF(or_nest, depth), OFF(or_nest, n_sync), OFF(or_nest, comp_insts), OFF(or_nest, bytes_h2d), OFF(or_nest, bytes_d2h),
        OFF(or_nest, access_off), OFF(or_nest, n_access)};
    static const size_t lau[] = {OFF(or_launch, block), OFF(or_launch, grid_max), OFF(or_launch, regs_per_thread),
        OFF(or_launch, smem_per_block)};
    static const size_t cand[] = {OFF(or_candidate, nest_id), OFF(or_candidate, launch_id),
        OFF(or_candidate, device_id), OFF(or_candidate, cpu_cycles), OFF(or_candidate, cpu_hz)};
    const size_t* t; size_t nf;
    switch (which) {
    case 0: t = dev; nf = sizeof dev / sizeof *dev; break;
    case 1: t = acc; nf = sizeof acc / sizeof *acc; break;
    case 2: t = nest; nf = sizeof nest / sizeof *nest; break;
    case 3: t = lau; nf = sizeof lau / sizeof *lau; break;
    case 4: t = cand; nf = sizeof cand / sizeof *cand; break;
    default: return (size_t)-1;
    }
    return (field >= 0 && (size_t)field < nf) ? t[field] : (size_t)-1;
}

/* -------------------------------------------------- NEXT row f3 (launch) */
/* Launch-configuration selection ("the maximum
 * grid-geometry selected by the runtime", P:L331 ML grid-geometry
 * predictors whose inference is too slow): for every group g of candidates
 * (the same nest and device under different launch configurations), the
 * valid candidate with the smallest predicted GPU time; ties and +inf go to
 * the lowest candidate index.  Plain definition: one ascending pass. */
void oracle_select_launch(const uint32_t* group_of, uint64_t n, const double* t_gpu, const uint8_t* status,
                          uint64_t n_groups, uint32_t* best, double* best_val) {
    for (uint64_t g = 0; g < n_groups; g++) { best[g] = 0xFFFFFFFFu; best_val[g] = INFINITY; }
    for (uint64_t c = 0; c < n; c++) {
        uint64_t g = group_of[c];
        if (g >= n_groups || status[c] != 0) continue;
        if (best[g] == 0xFFFFFFFFu || t_gpu[c] < best_val[g]) { best[g] = (uint32_t)c; best_val[g] = t_gpu[c]; }
    }
}

/* -------------------------------------------------- NEXT row f1 (CPU) */
/* Liao-Chapman OpenMP cost model (Fig. 3) with the Table II
 * parameters, for a target region holding one statically
 * scheduled parallel for (the paper's kernels are "strictly parallel loop
 * code").  Written out in the order of Fig. 3:
 *   Chunk_size     = ceil(P / threads)               static schedule (F1a)
 *   Cache_c        = TLB misses x TLB miss penalty   (F1c: misses = pages of
 *                    the thread's share of the data beyond the TLB entries)
 *   Loop_chunk_c   = Machine_c x per_iter x Chunk_size + Cache_c + Loop_overhead_c
 *                    with Loop_overhead_c = Loop_overhead_per_iter x Chunk_size
 *   Parallel_for_c = Schedule_times x (Schedule_c + Loop_chunk_c + Ordered_c + Reduction_c)
 *                    Schedule_times = 1, Ordered = Reduction = 0        (F1b)
 *   Thread_exe     = Parallel_for_c + Synchronization_c (implicit barrier)
 *   Parallel_Region = Fork_c + max_threads(Thread_exe) + Join_c
 *                    Fork = Par_Startup, Join folded into the barrier    (F1d)
 * Machine_c x per_iter is the LLVM-MCA cost of one parallel iteration
 * (P:L107-109), an input.  Status: EINVAL for a bad nest id, threads = 0 or a
 * negative / non-finite MCA cost. */
void oracle_cpu_model(const or_cpu_params* p, const or_nest* nests, uint64_t n_nests, const or_candidate* cands,
                      const or_cpu_input* in, uint64_t n, double* cpu_cycles, uint8_t* status) {
    for (uint64_t c = 0; c < n; c++) {
        cpu_cycles[c] = 0.0;
        status[c] = OR_OK;
        const double mca = in[c].mca_cycles_per_iter;
        if (cands[c].nest_id >= n_nests || in[c].threads == 0 || !(mca >= 0.0) || !isfinite(mca)) {
            status[c] = OR_EINVAL;
            continue;
        }
        const or_nest* nt = &nests[cands[c].nest_id];
        const uint64_t P = nt->P0 * nt->P1;
        const uint64_t chunk = ceil_div(P, in[c].threads);
        const double footprint = (double)(nt->bytes_h2d + nt->bytes_d2h) / (double)in[c].threads;
        const double pages = ceil(footprint / p->page_bytes);
        const double misses = pages > p->tlb_entries ? pages - p->tlb_entries : 0.0;
        const double cache = misses * p->tlb_miss_cycles;
        const double loop_overhead = p->loop_overhead_cycles * (double)chunk;
        const double loop_chunk = (mca * (double)chunk + cache) + loop_overhead;
        const double parallel_for = 1.0 * (((p->schedule_static_cycles + loop_chunk) + 0.0) + 0.0);
        const double thread_exe = parallel_for + p->sync_cycles;
        cpu_cycles[c] = (p->startup_cycles + thread_exe) + 0.0;
    }
}

/* -------------------------------------------------- NEXT row f2 (IPDA) */
/* Runtime binding of symbolic IPDA expressions (the symbolic
 * inter-thread stride of A[max*a] is [max]; "at the program point
 * when the target region is encountered, the unknown values are extracted and
 * used in the symbolic expression to compute the actual stride").  Every byte
 * coefficient of an access (base, c_par[0..1], c_inner[0..2]) is the sum of
 * its terms k * v[frame+s0] * v[frame+s1] * v[frame+s2] (a symbol index of
 * 0xFFFF is the factor 1).  Plain definition with exact 128-bit arithmetic:
 * any product or partial sum reaching 2^62 in magnitude -> ERANGE; a bad
 * index or an element size outside {1,2,4,8,16} -> EINVAL; invalid outputs
 * are all-zero. */
void oracle_bind(const or_sym_access* sym, uint64_t n_sym, const or_sym_term* terms, uint64_t n_terms,
                 const int64_t* values, uint64_t n_values, const or_bind_item* items, uint64_t n,
                 or_access* out, uint8_t* status) {
    const __int128 LIM = (__int128)1 << 62;
    for (uint64_t i = 0; i < n; i++) {
        or_access* o = &out[i];
        memset(o, 0, sizeof *o);
        status[i] = OR_OK;
        if (items[i].sym_access >= n_sym) { status[i] = OR_EINVAL; continue; }
        const or_sym_access* a = &sym[items[i].sym_access];
        const uint64_t fr = items[i].frame;
        int64_t coef[6];
        int bad = 0;
        for (int slot = 0; slot < 6 && !bad; slot++) {
            __int128 acc = 0;
            if ((uint64_t)a->term_off[slot] + a->n_terms[slot] > n_terms) { bad = OR_EINVAL; break; }
            for (int t = 0; t < a->n_terms[slot] && !bad; t++) {
                const or_sym_term* tm = &terms[a->term_off[slot] + t];
                __int128 p = tm->k;
                for (int f = 0; f < 3; f++) {
                    if (tm->sym[f] == 0xFFFFu) continue;
                    if (fr + tm->sym[f] >= n_values) { bad = OR_EINVAL; break; }
                    p *= values[fr + tm->sym[f]];
                    if (p >= LIM || p <= -LIM) { bad = OR_ERANGE; break; }
                }
                if (bad) break;
                acc += p;
                if (acc >= LIM || acc <= -LIM) bad = OR_ERANGE;
            }
            coef[slot] = (int64_t)acc;
        }
        int64_t e = a->elem_bytes;
        if (!bad && a->elem_sym != 0xFFFFu) {
            if (fr + a->elem_sym >= n_values) bad = OR_EINVAL;
            else e = values[fr + a->elem_sym];
        }
        if (!bad && !(e == 1 || e == 2 || e == 4 || e == 8 || e == 16)) bad = OR_EINVAL;
        if (bad) { status[i] = (uint8_t)bad; continue; }
        o->base = coef[0];
        o->c_par[0] = coef[1]; o->c_par[1] = coef[2];
        o->c_inner[0] = coef[3]; o->c_inner[1] = coef[4]; o->c_inner[2] = coef[5];
        o->elem_bytes = (uint8_t)e;
        o->depth = a->depth;
        o->is_store = a->is_store;
    }
}
