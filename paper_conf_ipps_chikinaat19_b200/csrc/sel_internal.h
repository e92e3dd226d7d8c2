// sel_internal.h -- host-side declarations shared by the libsel translation
// units (launchers implemented in sel_plan.cu, sel_count.cu, sel_model.cu).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/sel.h"

namespace sel {

struct Ws;   // device workspace pointers (defined below)

struct WsPtrs {
    struct WsHeader* hdr;
    uint32_t* slots;
    unsigned long long* nest_base;
    uint32_t* cand_pid;
    uint32_t* prob_nest;
    uint32_t* prob_B;
    unsigned long long* prob_W;      // closed-form W, scanned in place to the prefix
    unsigned long long* prob_WR;
    unsigned long long* prob_cnt;    // 5 x u64 per problem: W, L, S, C, U
    uint8_t* prob_status;
    uint8_t* cand_status;
    unsigned long long* queue;       // (problem << 32 | first WA) handed from the lane to the warp kernel
    uint8_t* prob_used;              // direct mode: big problem referenced by a candidate (k_mark_big)
    void* prob_md;                   // per problem: ProbModel (sel_model.cu)
    uint32_t* cls;                   // [kClsMax] class index per launch, [kClsMax..) B class per index
    uint8_t* nest_key;               // direct mode: shape key per nest (k_problem_w -> k_lane_problems)
    uint2* lane_info;                // direct mode, per nest: (M_it, mask of classes < 32 the lane kernel counts)
    unsigned long long* scan_tmp;
};

WsPtrs ws_ptrs(void* ws, uint64_t n, uint64_t n_nests, uint32_t flags);

// number of kernels launched by the library (profiling / gpu_launches claim)
void note_launch(int k = 1);
// records the profiling events around the counting kernel, when enabled
void prof_before_count(cudaStream_t s);
void prof_after_count(cudaStream_t s);
void prof_begin(int region, cudaStream_t s);
void prof_end(int region, cudaStream_t s);

// sel_plan.cu: candidates -> counting problems, closed-form W per problem, prefix
cudaError_t launch_plan(const sel_candidate* cands, uint64_t n, const sel_tables& t, int n_sets,
                        const WsPtrs& w, uint64_t n_nests, uint32_t flags, uint32_t part, uint32_t n_parts,
                        cudaStream_t s);
// sel_count.cu: the hot kernel
cudaError_t launch_count(const sel_tables& t, const WsPtrs& w, uint64_t max_problems, uint32_t flags,
                         cudaStream_t s);
// sel_model.cu
int n_device_sets();
cudaError_t load_device_params(const sel_device_params* host, int n);
cudaError_t launch_gather_counts(const sel_candidate* cands, uint64_t n, const sel_tables& t, const WsPtrs& w,
                                 sel_counts* out, uint8_t* status,
                                 cudaStream_t s);
cudaError_t launch_model_fused(const sel_candidate* cands, uint64_t n, const sel_tables& t, const WsPtrs& w,
                               uint8_t* decision, double* cycles, double* t_gpu, sel_counts* counts,
                               uint8_t* status, cudaStream_t s, const sel_cpu_input* cin = nullptr,
                               const sel_cpu_params* cp = nullptr);
cudaError_t launch_model_from_counts(const sel_candidate* cands, uint64_t n, const sel_tables& t,
                                     const sel_counts* counts, double* cycles, double* t_gpu, uint8_t* status,
                                     cudaStream_t s);
cudaError_t launch_selftest_ddiv(const double* a, const double* b, uint64_t n, double* q_fast, uint8_t* ok,
                                 double* q_ref, cudaStream_t s);
cudaError_t launch_select(const sel_candidate* cands, uint64_t n, const double* t_gpu, const uint8_t* status,
                          uint8_t* decision, cudaStream_t s);

// sel_next.cu (NEXT rows)
cudaError_t launch_select_launch(const uint32_t* group_of, uint64_t n, const double* t_gpu, const uint8_t* status,
                                 uint64_t n_groups, uint32_t* best, double* best_t, cudaStream_t s);

cudaError_t launch_bind(const sel_sym_access* sym, uint64_t n_sym, const sel_sym_term* terms, uint64_t n_terms,
                        const int64_t* values, uint64_t n_values, const sel_bind_item* items, uint64_t n,
                        sel_access* out, uint8_t* status, cudaStream_t s);
cudaError_t launch_cpu_model(sel_candidate* cands, uint64_t n, const sel_tables& t, const sel_cpu_input* in,
                             const sel_cpu_params& p, uint8_t* status, cudaStream_t s);

}  // namespace sel
