/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.  Plain, slow CPU oracle for the
 * batched GPU-side offload-model evaluation (Chikin et al., IPDPSW 2019).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code (no header, no
 * helper, no constant) with the CUDA path in paper_conf_ipps_chikinaat19_b200/;
 * the record layouts below are declared here independently and checked
 * against the generator's and the product's by tests/test_layout.py.
 */
#ifndef SEL_ORACLE_H
#define SEL_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int32_t num_sms, max_warps_per_sm, max_threads_per_sm, max_blocks_per_sm, regs_per_sm, smem_per_sm;
    double sm_clock_hz, mem_bw_Bps, link_bw_Bps, launch_overhead_s,
           mem_ld_cycles, dep_del_coal, dep_del_uncoal, issue_cycles;
    /* NEXT row f4: allocation granularity (F4c) and the transaction unit (F4d) */
    int32_t reg_alloc_unit, warp_alloc_gran, smem_alloc_unit, txn_sectors;
} or_device;

typedef struct {
    int64_t base, c_par[2], c_inner[3];
    uint8_t elem_bytes, depth, is_store, _pad[13];
} or_access;

typedef struct {
    uint64_t P0, P1;
    uint32_t trip[3];
    uint8_t par_dims, depth;
    uint16_t n_sync;
    double comp_insts[4];
    uint64_t bytes_h2d, bytes_d2h;
    uint32_t access_off, n_access;
} or_nest;

typedef struct { uint32_t block, grid_max, regs_per_thread, smem_per_block; } or_launch;

typedef struct {
    uint32_t nest_id;
    uint16_t launch_id, device_id;
    double cpu_cycles, cpu_hz;
} or_candidate;

/* NEXT row f1 inputs (same layouts as gen/selgen.h, declared independently) */
typedef struct {
    double cpu_hz, tlb_entries, tlb_miss_cycles, loop_overhead_cycles,
           schedule_static_cycles, sync_cycles, startup_cycles, page_bytes;
} or_cpu_params;
typedef struct { double mca_cycles_per_iter; uint32_t threads, _pad; } or_cpu_input;

/* NEXT row f2 inputs (layouts as gen/selgen.h, declared independently) */
typedef struct { int64_t k; uint16_t sym[3], _pad; } or_sym_term;
typedef struct {
    uint32_t term_off[6];
    uint8_t n_terms[6];
    uint16_t elem_sym;
    uint8_t elem_bytes, depth, is_store, _pad[5];
} or_sym_access;
typedef struct { uint32_t sym_access, frame; } or_bind_item;

/* Everything the oracle computes for one candidate: the hot path's outputs
 * (counts, cycles, t_gpu, decision, status) plus the model's intermediate
 * values, exposed so that tests can pin them against closed forms. */
typedef struct {
    /* a1-a4 counts */
    uint64_t W, L, S, C, U, WR;
    /* a1 geometry, a5 occupancy */
    uint64_t G, T, R, wpb, abps, active_sms, M_it;
    double N, Rep;
    /* a4 / a6 intermediates */
    double comp, mem, MemL_u, MemL_c, MemL, Dep, MWPnb, BWpw, MWPbw, MWP, Comp, Mem, CWP, E;
    int32_t hk_case;                     /* 0: W == 0 (R22), 1, 2, 3 as in Fig. 4 */
    /* outputs */
    double cycles, t_gpu, t_cpu;
    uint8_t decision, status, _pad[6];
} or_result;

enum { OR_OK = 0, OR_EINVAL = 1, OR_ERANGE = 2, OR_ELAUNCH = 3 };

/* a1 geometry of a launch (reading R6/R27): out = {G, T, R, wpb}. */
void oracle_geometry(uint64_t P, uint32_t B, uint32_t grid_max, uint64_t out[4]);

/* Full evaluation of n candidates (brute-force counting + literal model).
 * threads <= 0 means "all host cores".  Returns 0, or -1 on bad arguments
 * (null pointers, invalid device parameter set). */
int oracle_evaluate(const or_device* devs, int n_devs,
                    const or_candidate* cands, uint64_t n,
                    const or_nest* nests, uint64_t n_nests,
                    const or_access* acc, uint64_t n_acc,
                    const or_launch* launches, uint64_t n_launches,
                    or_result* out, int threads);

/* The model part only (a4-a7) for given counts r->{W,L,S,C,U,WR}: fills the
 * rest of *r.  Used by tests to pin the Hong & Kim arithmetic on hand-made
 * counts. */
void oracle_model(const or_device* dev, const or_nest* nest, const or_access* acc,
                  const or_launch* launch, const or_candidate* cand, or_result* r);

/* NEXT row f3: per-group argmin of t_gpu over valid candidates (ties and
 * +inf: lowest index; no valid candidate: best = 0xFFFFFFFF, +inf). */
void oracle_select_launch(const uint32_t* group_of, uint64_t n, const double* t_gpu, const uint8_t* status,
                          uint64_t n_groups, uint32_t* best, double* best_val);

/* NEXT row f1: Liao-Chapman CPU cycles (Fig. 3 + Table II) per candidate. */
void oracle_cpu_model(const or_cpu_params* p, const or_nest* nests, uint64_t n_nests, const or_candidate* cands,
                      const or_cpu_input* in, uint64_t n, double* cpu_cycles, uint8_t* status);

/* NEXT row f2: bind symbolic accesses to concrete ones (see oracle.c). */
void oracle_bind(const or_sym_access* sym, uint64_t n_sym, const or_sym_term* terms, uint64_t n_terms,
                 const int64_t* values, uint64_t n_values, const or_bind_item* items, uint64_t n,
                 or_access* out, uint8_t* status);

/* Layout self-description for tests/test_layout.py. */
size_t oracle_sizeof(int which);
size_t oracle_offsetof(int which, int field);

#ifdef __cplusplus
}
#endif
#endif
