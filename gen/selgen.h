/*
 * selgen.h -- seeded, counter-based synthetic input generator.
 *
 * This module produces INPUT BYTES ONLY: loop-nest descriptors, access
 * descriptors, launch configurations, device parameter sets and candidates
 * for the five BASELINE.json configs.  It contains none of the hot path's
 * arithmetic (no coalescing counts, no Hong & Kim model, no decision).  Both
 * the CPU oracle (oracle/) and the CUDA path consume its output; neither
 * includes the other.  The record layouts below are this module's own
 * definition of the data format; include/sel.h (product) and oracle/oracle.h
 * (test oracle) declare the same layouts independently and a CPU test checks
 * that all three agree byte for byte.
 *
 * Recipe: DESIGN.md "Input recipe".  Every candidate is a
 * pure function of (config, candidate index); any rank can generate any
 * index range without communication.
 */
#ifndef SELGEN_H
#define SELGEN_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {                       /* 104 bytes */
    int32_t num_sms, max_warps_per_sm, max_threads_per_sm, max_blocks_per_sm, regs_per_sm, smem_per_sm;
    double sm_clock_hz, mem_bw_Bps, link_bw_Bps, launch_overhead_s,
           mem_ld_cycles, dep_del_coal, dep_del_uncoal, issue_cycles;
    int32_t reg_alloc_unit, warp_alloc_gran, smem_alloc_unit, txn_sectors;   /* NEXT row f4 */
} gen_device_params;

typedef struct {                       /* 64 bytes; all quantities in bytes */
    int64_t base, c_par[2], c_inner[3];
    uint8_t elem_bytes, depth, is_store, _pad[13];
} gen_access;

typedef struct {                       /* 88 bytes */
    uint64_t P0, P1;
    uint32_t trip[3];
    uint8_t par_dims, depth;
    uint16_t n_sync;                   /* barriers per parallel iteration (NEXT row f4) */
    double comp_insts[4];
    uint64_t bytes_h2d, bytes_d2h;
    uint32_t access_off, n_access;
} gen_nest;

typedef struct {                       /* 16 bytes */
    uint32_t block, grid_max, regs_per_thread, smem_per_block;
} gen_launch;

typedef struct {                       /* 24 bytes */
    uint32_t nest_id;
    uint16_t launch_id, device_id;
    double cpu_cycles, cpu_hz;
} gen_candidate;

/* NEXT row f1 (Liao-Chapman CPU model) inputs: Table II constants and the
 * per-candidate LLVM-MCA stand-in cost per parallel iteration + threads. */
typedef struct {                       /* 64 bytes */
    double cpu_hz, tlb_entries, tlb_miss_cycles, loop_overhead_cycles,
           schedule_static_cycles, sync_cycles, startup_cycles, page_bytes;
} gen_cpu_params;

typedef struct {                       /* 16 bytes */
    double mca_cycles_per_iter;
    uint32_t threads, _pad;
} gen_cpu_input;

/* NEXT row f2 (symbolic IPDA binding) inputs. */
typedef struct { int64_t k; uint16_t sym[3], _pad; } gen_sym_term;          /* 16 bytes */
typedef struct {                                                             /* 40 bytes */
    uint32_t term_off[6];
    uint8_t n_terms[6];
    uint16_t elem_sym;
    uint8_t elem_bytes, depth, is_store, _pad[5];
} gen_sym_access;
typedef struct { uint32_t sym_access, frame; } gen_bind_item;               /* 8 bytes */

/* Config ids follow BASELINE.json "configs" order, 1-based. */
enum { SELGEN_C1 = 1, SELGEN_C2 = 2, SELGEN_C3 = 3, SELGEN_C4 = 4, SELGEN_C5 = 5 };

/* Number of candidates in the full config (c5: 10^8). */
uint64_t selgen_num_candidates(int cfg);
/* The four device parameter sets (K80 one GK210, P100, V100, B200). Returns 4. */
int selgen_device_sets(gen_device_params* out);
/* Launch table of a config (c1..c3: 1 entry, c4/c5: 8). Returns the count. */
int selgen_launches(int cfg, gen_launch* out);
/* Sizes of the nest/access tables needed for candidates [c0, c1). */
int selgen_count(int cfg, uint64_t c0, uint64_t c1, uint64_t* n_nests, uint64_t* n_access);
/* Fill candidates [c0, c1) and the nest/access tables they reference
 * (nest ids are local to the slice).  Returns 0 or -1 on bad arguments. */
int selgen_fill(int cfg, uint64_t c0, uint64_t c1,
                gen_candidate* cands, gen_nest* nests, gen_access* acc);
/* Arbitrary candidate indices of an index-addressable config (c3, c5); each
 * candidate gets its own nest copy (nest_id = position in idx). */
int selgen_count_indices(int cfg, const uint64_t* idx, uint64_t m, uint64_t* n_access);
int selgen_fill_indices(int cfg, const uint64_t* idx, uint64_t m, gen_candidate* cands, gen_nest* nests,
                        gen_access* acc);
/* f1 inputs of candidates [c0, c1) and the Table II parameter set. */
int selgen_cpu_inputs(int cfg, uint64_t c0, uint64_t c1, gen_cpu_input* out);
void selgen_cpu_params(gen_cpu_params* p);
/* f2: the static symbolic table (24 shapes x {1-D, collapse} x 12 slots;
 * pass NULL arrays to size it), and the frames / bind items of [c0, c1)
 * for configs 2 and 5, aligned with selgen_fill's access order. */
int selgen_sym_tables(gen_sym_access* sym, gen_sym_term* terms, uint32_t* n_sym, uint32_t* n_terms);
int selgen_sym_count(int cfg, uint64_t c0, uint64_t c1, uint64_t* n_values, uint64_t* n_items);
int selgen_sym_fill(int cfg, uint64_t c0, uint64_t c1, int64_t* values, gen_bind_item* items);
/* Shape catalogue (24 Polybench-style sub-kernels). */
int selgen_num_shapes(void);
const char* selgen_shape_name(int s);
/* Counter-based generator: splitmix64(seed ^ (i * golden)). */
uint64_t selgen_rng(uint64_t seed, uint64_t i);

#ifdef __cplusplus
}
#endif
#endif
