// sel_api.cu -- the extern "C" boundary of libsel.so (include/sel.h):
// argument checking, workspace carving, stream-ordered launch sequencing,
// error strings and the profiling hooks.  All compute runs in the kernels of
// sel_plan.cu, sel_count.cu and sel_model.cu; there is no CPU fallback.
#include <atomic>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <vector>
#include <nvtx3/nvToolsExt.h>
#include "sel_device.cuh"
#include "sel_internal.h"

namespace sel {

static thread_local char t_err[512] = "";
static std::atomic<uint64_t> g_launches{0};

void note_launch(int k) { g_launches.fetch_add(uint64_t(k), std::memory_order_relaxed); }

static int fail(int code, const char* fmt, const char* detail = "") {
    std::snprintf(t_err, sizeof t_err, fmt, detail);
    return code;
}
static int cuda_fail(cudaError_t e, const char* where) {
    std::snprintf(t_err, sizeof t_err, "%s: %s", where, cudaGetErrorString(e));
    return SEL_ECUDA;
}

// ------------------------------------------------------------- profiling
// Regions (sel.h SEL_PROF_*): CUDA events recorded on the launching stream
// around the plan, counting and model kernels of every call.
static std::mutex g_prof_mu;
static bool g_prof_on = false;
static std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_prof_pending[SEL_PROF_REGIONS];
static std::vector<cudaEvent_t> g_prof_free;
static cudaEvent_t g_prof_cur_begin[SEL_PROF_REGIONS] = {};

static cudaEvent_t prof_event() {
    if (!g_prof_free.empty()) {
        cudaEvent_t e = g_prof_free.back();
        g_prof_free.pop_back();
        return e;
    }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
}

// NVTX ranges (tracing) around the same regions, on the host
// timeline of the enqueueing thread: a no-op unless a tool is attached.
static const char* const kProfNames[SEL_PROF_REGIONS] = {"sel:plan", "sel:count", "sel:model",
                                                         "sel:k_model_fused", "sel:k_lane_problems",
                                                         "sel:k_problem_w"};
static nvtxRangeId_t g_nvtx[SEL_PROF_REGIONS] = {};

void prof_begin(int region, cudaStream_t s) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    if (g_nvtx[region]) nvtxRangeEnd(g_nvtx[region]);
    g_nvtx[region] = nvtxRangeStartA(kProfNames[region]);
    if (!g_prof_on) return;
    g_prof_cur_begin[region] = prof_event();
    cudaEventRecord(g_prof_cur_begin[region], s);
}
void prof_end(int region, cudaStream_t s) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    if (g_nvtx[region]) {
        nvtxRangeEnd(g_nvtx[region]);
        g_nvtx[region] = 0;
    }
    if (!g_prof_on || !g_prof_cur_begin[region]) return;
    cudaEvent_t e = prof_event();
    cudaEventRecord(e, s);
    g_prof_pending[region].emplace_back(g_prof_cur_begin[region], e);
    g_prof_cur_begin[region] = nullptr;
}
void prof_before_count(cudaStream_t s) { prof_begin(SEL_PROF_COUNT, s); }
void prof_after_count(cudaStream_t s) { prof_end(SEL_PROF_COUNT, s); }

WsPtrs ws_ptrs(void* ws, uint64_t n, uint64_t n_nests, uint32_t flags) {
    const WsLayout L = ws_layout(n, n_nests, flags);
    char* b = static_cast<char*>(ws);
    WsPtrs p;
    p.hdr = reinterpret_cast<WsHeader*>(b + L.hdr);
    p.slots = reinterpret_cast<uint32_t*>(b + L.slots);
    p.nest_base = reinterpret_cast<unsigned long long*>(b + L.nest_base);
    p.cand_pid = reinterpret_cast<uint32_t*>(b + L.cand_pid);
    p.prob_nest = reinterpret_cast<uint32_t*>(b + L.prob_nest);
    p.prob_B = reinterpret_cast<uint32_t*>(b + L.prob_B);
    p.prob_W = reinterpret_cast<unsigned long long*>(b + L.prob_W);
    p.prob_WR = reinterpret_cast<unsigned long long*>(b + L.prob_WR);
    p.prob_cnt = reinterpret_cast<unsigned long long*>(b + L.prob_cnt);
    p.prob_status = reinterpret_cast<uint8_t*>(b + L.prob_status);
    p.cand_status = reinterpret_cast<uint8_t*>(b + L.cand_status);
    p.queue = reinterpret_cast<unsigned long long*>(b + L.queue);
    p.prob_used = reinterpret_cast<uint8_t*>(b + L.prob_used);
    p.prob_md = b + L.prob_md;
    p.cls = reinterpret_cast<uint32_t*>(b + L.cls);
    p.nest_key = reinterpret_cast<uint8_t*>(b + L.nest_key);
    p.lane_info = reinterpret_cast<uint2*>(b + L.lane_info);
    p.scan_tmp = reinterpret_cast<unsigned long long*>(b + L.scan_tmp);
    return p;
}

static int check_tables(const sel_tables* t) {
    if (!t) return fail(SEL_EINVAL, "tables is NULL%s");
    if ((t->n_nests && !t->nests) || (t->n_accesses && !t->accesses) || (t->n_launches && !t->launches))
        return fail(SEL_EINVAL, "a table pointer is NULL while its count is non-zero%s");
    if (t->n_nests >= (1ull << 32)) return fail(SEL_EINVAL, "n_nests must be < 2^32%s");
    return SEL_OK;
}

static int check_common(const sel_candidate* c, uint64_t n, const sel_tables* t) {
    if (n && !c) return fail(SEL_EINVAL, "candidates is NULL%s");
    if (n >= 0xffffffffull) return fail(SEL_EINVAL, "n must be < 2^32 - 1%s");
    if (int r = check_tables(t)) return r;
    if (n_device_sets() == 0) return fail(SEL_ENODEV, "no device parameters loaded (sel_load_device_params)%s");
    return SEL_OK;
}

static int check_ws(void* ws, size_t bytes, uint64_t n, uint64_t n_nests, uint32_t flags) {
    if (!ws) return fail(SEL_EINVAL, "workspace is NULL%s");
    if (reinterpret_cast<uintptr_t>(ws) & 255) return fail(SEL_EINVAL, "workspace must be 256-byte aligned%s");
    if (bytes < ws_layout(n, n_nests, flags).total) return fail(SEL_EINVAL, "workspace too small%s");
    return SEL_OK;
}

static int plan_and_count(const sel_candidate* c, uint64_t n, const sel_tables* t, const WsPtrs& w, uint32_t flags,
                          cudaStream_t s, uint32_t part = 0, uint32_t n_parts = 1) {
    cudaError_t e = launch_plan(c, n, *t, n_device_sets(), w, t->n_nests, flags, part, n_parts, s);
    if (e != cudaSuccess) return cuda_fail(e, "plan");
    e = launch_count(*t, w, n, flags, s);
    if (e != cudaSuccess) return cuda_fail(e, "count");
    return SEL_OK;
}

}  // namespace sel

using namespace sel;

extern "C" {

int sel_load_device_params(const sel_device_params* h, int n_sets) {
    if (!h || n_sets < 1 || n_sets > SEL_MAX_DEVICE_SETS) return fail(SEL_EINVAL, "n_sets must be 1..16%s");
    for (int i = 0; i < n_sets; i++) {
        const sel_device_params& d = h[i];
        const bool ok = d.num_sms >= 1 && d.max_warps_per_sm >= 1 && d.max_threads_per_sm >= 1 &&
                        d.max_blocks_per_sm >= 1 && d.regs_per_sm >= 0 && d.smem_per_sm >= 0 &&
                        d.sm_clock_hz > 0 && d.mem_bw_Bps > 0 && d.link_bw_Bps > 0 && d.launch_overhead_s >= 0 &&
                        d.mem_ld_cycles > 0 && d.dep_del_coal > 0 && d.dep_del_uncoal > 0 && d.issue_cycles > 0 &&
                        d.reg_alloc_unit >= 0 && d.warp_alloc_gran >= 0 && d.smem_alloc_unit >= 0 &&
                        (d.txn_sectors == 0 || d.txn_sectors == 1);
        if (!ok) return fail(SEL_EINVAL, "invalid device parameter set%s");
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(SEL_ENODEV, "no CUDA device%s");
    cudaError_t e = load_device_params(h, n_sets);
    if (e != cudaSuccess) return cuda_fail(e, "sel_load_device_params");
    return SEL_OK;
}

size_t sel_workspace_size(uint64_t n, uint64_t n_nests, uint32_t flags) {
    return ws_layout(n, n_nests, flags).total;
}

int sel_count_transactions(const sel_candidate* c, uint64_t n, const sel_tables* t, sel_counts* out,
                           uint8_t* status, void* ws, size_t ws_bytes, uint32_t flags, sel_stream_t stream) {
    return sel_count_transactions_part(c, n, t, 0, 1, out, status, ws, ws_bytes, flags, stream);
}

int sel_count_transactions_part(const sel_candidate* c, uint64_t n, const sel_tables* t, uint32_t part,
                                uint32_t n_parts, sel_counts* out, uint8_t* status, void* ws, size_t ws_bytes,
                                uint32_t flags, sel_stream_t stream) {
    if (n_parts < 1 || part >= n_parts) return fail(SEL_EINVAL, "need 0 <= part < n_parts%s");
    if (int r = check_common(c, n, t)) return r;
    if (n == 0) return SEL_OK;
    if (!out || !status) return fail(SEL_EINVAL, "out/status is NULL%s");
    if (int r = check_ws(ws, ws_bytes, n, t->n_nests, flags)) return r;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const WsPtrs w = ws_ptrs(ws, n, t->n_nests, flags);
    if (int r = plan_and_count(c, n, t, w, flags, s, part, n_parts)) return r;
    cudaError_t e = launch_gather_counts(c, n, *t, w, out, status, s);
    if (e != cudaSuccess) return cuda_fail(e, "gather");
    return SEL_OK;
}

int sel_predict_gpu_cycles(const sel_candidate* c, uint64_t n, const sel_tables* t, const sel_counts* counts,
                           double* cycles, double* t_gpu, uint8_t* status, sel_stream_t stream) {
    if (int r = check_common(c, n, t)) return r;
    if (n == 0) return SEL_OK;
    if (!counts || !cycles || !status) return fail(SEL_EINVAL, "counts/cycles/status is NULL%s");
    cudaError_t e = launch_model_from_counts(c, n, *t, counts, cycles, t_gpu, status,
                                             reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "predict");
    return SEL_OK;
}

int sel_select(const sel_candidate* c, uint64_t n, const double* t_gpu, const uint8_t* status, uint8_t* decision,
               sel_stream_t stream) {
    if (n == 0) return SEL_OK;
    if (!c || !t_gpu || !status || !decision) return fail(SEL_EINVAL, "NULL argument%s");
    cudaError_t e = launch_select(c, n, t_gpu, status, decision, reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "select");
    return SEL_OK;
}

int sel_evaluate(const sel_candidate* c, uint64_t n, const sel_tables* t, uint8_t* decision, double* cycles,
                 double* t_gpu, sel_counts* counts, uint8_t* status, void* ws, size_t ws_bytes, uint32_t flags,
                 sel_stream_t stream) {
    if (int r = check_common(c, n, t)) return r;
    if (n == 0) return SEL_OK;
    if (!decision || !cycles || !status) return fail(SEL_EINVAL, "decision/cycles/status is NULL%s");
    if (int r = check_ws(ws, ws_bytes, n, t->n_nests, flags)) return r;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const WsPtrs w = ws_ptrs(ws, n, t->n_nests, flags);
    if (int r = plan_and_count(c, n, t, w, flags, s)) return r;
    cudaError_t e = launch_model_fused(c, n, *t, w, decision, cycles, t_gpu, counts, status, s);
    if (e != cudaSuccess) return cuda_fail(e, "model");
    return SEL_OK;
}

int sel_evaluate_cpu_model(const sel_candidate* c, uint64_t n, const sel_tables* t, const sel_cpu_input* cin,
                           const sel_cpu_params* p, uint8_t* decision, double* cycles, double* t_gpu,
                           sel_counts* counts, uint8_t* status, void* ws, size_t ws_bytes, uint32_t flags,
                           sel_stream_t stream) {
    if (int r = check_common(c, n, t)) return r;
    if (n == 0) return SEL_OK;
    if (!decision || !cycles || !status || !cin || !p) return fail(SEL_EINVAL, "NULL argument%s");
    if (!(p->cpu_hz > 0) || !(p->page_bytes > 0) || p->tlb_entries < 0 || p->tlb_miss_cycles < 0 ||
        p->loop_overhead_cycles < 0 || p->schedule_static_cycles < 0 || p->sync_cycles < 0 || p->startup_cycles < 0)
        return fail(SEL_EINVAL, "invalid CPU parameter set%s");
    if (int r = check_ws(ws, ws_bytes, n, t->n_nests, flags)) return r;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const WsPtrs w = ws_ptrs(ws, n, t->n_nests, flags);
    if (int r = plan_and_count(c, n, t, w, flags, s)) return r;
    cudaError_t e = launch_model_fused(c, n, *t, w, decision, cycles, t_gpu, counts, status, s, cin, p);
    if (e != cudaSuccess) return cuda_fail(e, "model");
    return SEL_OK;
}

int sel_select_launch(const uint32_t* group_of, uint64_t n, const double* t_gpu, const uint8_t* status,
                      uint64_t n_groups, uint32_t* best, double* best_t, sel_stream_t stream) {
    if (n_groups == 0) return SEL_OK;
    if (!best || !best_t || (n && (!group_of || !t_gpu || !status))) return fail(SEL_EINVAL, "NULL argument%s");
    if (n >= 0xffffffffull) return fail(SEL_EINVAL, "n must be < 2^32 - 1%s");
    cudaError_t e = launch_select_launch(group_of, n, t_gpu, status, n_groups, best, best_t,
                                         reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "select_launch");
    return SEL_OK;
}

int sel_bind_accesses(const sel_sym_access* sym, uint64_t n_sym, const sel_sym_term* terms, uint64_t n_terms,
                      const int64_t* values, uint64_t n_values, const sel_bind_item* items, uint64_t n,
                      sel_access* out, uint8_t* status, sel_stream_t stream) {
    if (n == 0) return SEL_OK;
    if (!items || !out || !status || (n_sym && !sym) || (n_terms && !terms) || (n_values && !values))
        return fail(SEL_EINVAL, "NULL argument%s");
    cudaError_t e = launch_bind(sym, n_sym, terms, n_terms, values, n_values, items, n, out, status,
                                reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "bind_accesses");
    return SEL_OK;
}

int sel_model_cpu_cost(sel_candidate* c, uint64_t n, const sel_tables* t, const sel_cpu_input* in,
                       const sel_cpu_params* p, uint8_t* status, sel_stream_t stream) {
    if (int r = check_tables(t)) return r;
    if (n == 0) return SEL_OK;
    if (!c || !in || !p || !status) return fail(SEL_EINVAL, "NULL argument%s");
    if (!(p->cpu_hz > 0) || !(p->page_bytes > 0) || p->tlb_entries < 0 || p->tlb_miss_cycles < 0 ||
        p->loop_overhead_cycles < 0 || p->schedule_static_cycles < 0 || p->sync_cycles < 0 || p->startup_cycles < 0)
        return fail(SEL_EINVAL, "invalid CPU parameter set%s");
    cudaError_t e = launch_cpu_model(c, n, *t, in, *p, status, reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "model_cpu_cost");
    return SEL_OK;
}

int sel_read_stats(const void* ws, sel_stats* out, sel_stream_t stream) {
    if (!ws || !out) return fail(SEL_EINVAL, "NULL argument%s");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t e = cudaMemcpyAsync(out, ws, sizeof(sel_stats), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "sel_read_stats");
    out->wa_expanded = out->wa_resolved - out->wa_closed_form - out->wa_arith_lanes - out->wa_residue_classes;
    return SEL_OK;
}

int sel_profile_enable(int on) {
    std::lock_guard<std::mutex> g(g_prof_mu);
    g_prof_on = on != 0;
    return SEL_OK;
}

int sel_profile_read_region(int region, double* ms_out, uint64_t* launches_out) {
    if (region < 0 || region >= SEL_PROF_REGIONS) return fail(SEL_EINVAL, "unknown profiling region%s");
    std::lock_guard<std::mutex> g(g_prof_mu);
    double ms = 0.0;
    uint64_t k = 0;
    for (auto& pr : g_prof_pending[region]) {
        cudaError_t e = cudaEventSynchronize(pr.second);
        if (e != cudaSuccess) return cuda_fail(e, "sel_profile_read");
        float x = 0.f;
        cudaEventElapsedTime(&x, pr.first, pr.second);
        ms += x;
        k++;
        g_prof_free.push_back(pr.first);
        g_prof_free.push_back(pr.second);
    }
    g_prof_pending[region].clear();
    if (ms_out) *ms_out = ms;
    if (launches_out) *launches_out = k;
    return SEL_OK;
}

int sel_profile_read(double* count_ms, uint64_t* count_launches) {
    return sel_profile_read_region(SEL_PROF_COUNT, count_ms, count_launches);
}

uint64_t sel_kernel_launches(void) { return g_launches.load(); }

int sel_selftest_ddiv(const double* a, const double* b, uint64_t n, double* q_fast, uint8_t* ok, double* q_ref,
                      sel_stream_t stream) {
    if (n && (!a || !b || !q_fast || !ok || !q_ref)) return fail(SEL_EINVAL, "NULL argument%s");
    cudaError_t e = launch_selftest_ddiv(a, b, n, q_fast, ok, q_ref, reinterpret_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "sel_selftest_ddiv");
    return SEL_OK;
}

const char* sel_last_error(void) { return t_err; }
const char* sel_version(void) { return "libsel 0.1 sm_100a"; }

size_t sel_sizeof(int which) {
    switch (which) {
    case 0: return sizeof(sel_device_params);
    case 1: return sizeof(sel_access);
    case 2: return sizeof(sel_nest);
    case 3: return sizeof(sel_launch);
    case 4: return sizeof(sel_candidate);
    case 5: return sizeof(sel_counts);
    default: return 0;
    }
}

#define OFF(T, f) (size_t)offsetof(T, f)
size_t sel_offsetof(int which, int field) {
    static const size_t dev[] = {OFF(sel_device_params, num_sms), OFF(sel_device_params, max_warps_per_sm),
        OFF(sel_device_params, max_threads_per_sm), OFF(sel_device_params, max_blocks_per_sm),
        OFF(sel_device_params, regs_per_sm), OFF(sel_device_params, smem_per_sm), OFF(sel_device_params, sm_clock_hz),
        OFF(sel_device_params, mem_bw_Bps), OFF(sel_device_params, link_bw_Bps),
        OFF(sel_device_params, launch_overhead_s), OFF(sel_device_params, mem_ld_cycles),
        OFF(sel_device_params, dep_del_coal), OFF(sel_device_params, dep_del_uncoal),
        OFF(sel_device_params, issue_cycles), OFF(sel_device_params, reg_alloc_unit),
        OFF(sel_device_params, warp_alloc_gran), OFF(sel_device_params, smem_alloc_unit),
        OFF(sel_device_params, txn_sectors)};
    static const size_t acc[] = {OFF(sel_access, base), OFF(sel_access, c_par), OFF(sel_access, c_inner),
        OFF(sel_access, elem_bytes), OFF(sel_access, depth), OFF(sel_access, is_store)};
    static const size_t nest[] = {OFF(sel_nest, P0), OFF(sel_nest, P1), OFF(sel_nest, trip), OFF(sel_nest, par_dims),
        OFF(sel_nest, depth), OFF(sel_nest, n_sync), OFF(sel_nest, comp_insts), OFF(sel_nest, bytes_h2d), OFF(sel_nest, bytes_d2h),
        OFF(sel_nest, access_off), OFF(sel_nest, n_access)};
    static const size_t lau[] = {OFF(sel_launch, block), OFF(sel_launch, grid_max), OFF(sel_launch, regs_per_thread),
        OFF(sel_launch, smem_per_block)};
    static const size_t cand[] = {OFF(sel_candidate, nest_id), OFF(sel_candidate, launch_id),
        OFF(sel_candidate, device_id), OFF(sel_candidate, cpu_cycles), OFF(sel_candidate, cpu_hz)};
    static const size_t cnt[] = {OFF(sel_counts, warp_accesses), OFF(sel_counts, lines), OFF(sel_counts, sectors),
        OFF(sel_counts, coalesced), OFF(sel_counts, uncoal_lines), OFF(sel_counts, warp_reps)};
    const size_t* tb;
    size_t nf;
    switch (which) {
    case 0: tb = dev; nf = sizeof dev / sizeof *dev; break;
    case 1: tb = acc; nf = sizeof acc / sizeof *acc; break;
    case 2: tb = nest; nf = sizeof nest / sizeof *nest; break;
    case 3: tb = lau; nf = sizeof lau / sizeof *lau; break;
    case 4: tb = cand; nf = sizeof cand / sizeof *cand; break;
    case 5: tb = cnt; nf = sizeof cnt / sizeof *cnt; break;
    default: return size_t(-1);
    }
    return (field >= 0 && size_t(field) < nf) ? tb[field] : size_t(-1);
}

}  // extern "C"

static_assert(sizeof(sel_device_params) == 104, "sel_device_params layout");
static_assert(sizeof(sel_access) == 64, "sel_access layout");
static_assert(sizeof(sel_nest) == 88, "sel_nest layout");
static_assert(sizeof(sel_launch) == 16, "sel_launch layout");
static_assert(sizeof(sel_candidate) == 24, "sel_candidate layout");
static_assert(sizeof(sel_counts) == 48, "sel_counts layout");
static_assert(sizeof(sel_stats) == 128, "sel_stats layout");
static_assert(sizeof(sel_cpu_params) == 64, "sel_cpu_params layout");
static_assert(sizeof(sel_cpu_input) == 16, "sel_cpu_input layout");
static_assert(sizeof(sel_sym_term) == 16, "sel_sym_term layout");
static_assert(sizeof(sel_sym_access) == 40, "sel_sym_access layout");
static_assert(sizeof(sel_bind_item) == 8, "sel_bind_item layout");
