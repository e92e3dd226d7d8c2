#!/usr/bin/env python
"""Benchmark of the batched GPU-side offload-model evaluation (one JSON line).

Workload (BASELINE.json configs[4], the configuration the metric is quoted
on): the c5 sweep of 10^8 candidates (24 Polybench-shaped loop nests x
index-derived trip counts x 8 launch configurations x 4 device parameter
sets), synthetic and seeded (gen/).  A step is one
pass of the whole hot path over the batch: per-warp coalescing counts, Hong &
Kim cycles and the CPU-or-GPU decision for every candidate, plus the NCCL
all-gather of the decisions when N > 1.  The batch is fixed and sharded
across ranks by candidate index ("scaling": "strong").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "model evaluations/sec and warp-accesses analysed/sec at 1/2/4/8 B200 (% roofline)"
UNIT = "evals/s"
WORKLOAD = ("c5: 10^8-candidate selection sweep (24 Polybench-shaped nests x trip counts x "
            "8 launch configs x 4 device sets)")
OPS_PER_WA = 224           # 7 integer lane-ops x 32 lanes per warp-access (lane expansion)
CAND_BYTES = 24 + 1 + 8    # per candidate: sel_candidate read, decision + cycles written
MODEL_BYTES = 24 + 1 + 8 + 1   # model kernels: record in, decision + cycles + status out
PLAN_BYTES = 24 + 4 + 1    # plan: record in, problem id + candidate status out


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", type=int, default=5,
                   help="BASELINE config 1..5 (5 = the metric's workload; 4 = warp-range split across ranks)")
    p.add_argument("--candidates", type=int, default=0, help="override the batch size (testing)")
    p.add_argument("--flags", type=int, default=0, help="libsel flags (1 no count sharing, 2 match_any)")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-next", action="store_true", help="skip timing the NEXT rows f1-f3")
    p.add_argument("--cpu-seconds", type=float, default=15.0)
    return p.parse_args()


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock and throttle reasons sampled DURING the timed region: an NVML
    polling thread (every ~2 ms, so a region of a few tens of ms still gets
    samples), falling back to `nvidia-smi -lms`."""
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []
        self.samples = []               # (sm_mhz, max_mhz, reason bits) from NVML
        self.nvml = None
        self.stop = threading.Event()

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        try:
            import torch
            bus = torch.cuda.get_device_properties(self.idx).pci_bus_id
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId_v2(
                "%08x:%02x:%02x.0" % (torch.cuda.get_device_properties(self.idx).pci_domain_id, bus,
                                      torch.cuda.get_device_properties(self.idx).pci_device_id))
        except Exception:
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            idx = int(vis.split(",")[self.idx]) if vis and vis.split(",")[self.idx].isdigit() else self.idx
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(idx)

    def __enter__(self):
        try:
            self.nvml = self._nvml_handle()
            pm, h = self.nvml
            self.max_mhz = float(pm.nvmlDeviceGetMaxClockInfo(h, pm.NVML_CLOCK_SM))
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return self
        except Exception:
            self.nvml = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _poll(self):
        pm, h = self.nvml
        while not self.stop.is_set():
            try:
                self.samples.append((float(pm.nvmlDeviceGetClockInfo(h, pm.NVML_CLOCK_SM)), self.max_mhz,
                                     int(pm.nvmlDeviceGetCurrentClocksEventReasons(h))))
            except Exception:
                pass
            self.stop.wait(0.002)

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        self.stop.set()
        if self.nvml:
            self.t.join(timeout=2)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        sm, smax, reasons = [], 0.0, set()
        for mhz, mx, bits in self.samples:
            sm.append(mhz)
            smax = max(smax, mx)
            for name, bit in self.REASONS:
                if bits & bit:
                    reasons.add(name)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                smax = max(smax, float(f[1]))
            except ValueError:
                continue
            for name, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": smax, "reasons": sorted(reasons),
                "samples": len(sm), "source": "nvml" if self.samples else "nvidia-smi"}


# ---------------------------------------------------------------- helpers
def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


NCU_REGION_KERNELS = {
    "plan": ("k_classes", "k_insert", "k_rank_slots", "k_scan_reduce", "k_scan_partials", "k_scan_down", "k_assign",
             "k_finalize_plan", "k_problem_w", "k_mark_big", "k_drop_unused", "k_plan_stats"),
    "count": ("k_lane_problems", "k_queue", "k_count"),
    "model": ("k_problem_model", "k_model_fused"),
}


def ncu_kernels():
    """Per-kernel counters of the committed ncu --set full capture of one bench
    step (profiles/ncu_kernels.json, written by scripts/ncu_kernels.py)."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_kernels.json")) as f:
            return json.load(f)
    except (OSError, ValueError):
        return {}


def ncu_region_traffic(ncu, region):
    """dram read + write bytes per launch of a region's kernels (committed capture), or None."""
    ks = [ncu["kernels"][k] for k in NCU_REGION_KERNELS[region] if k in ncu.get("kernels", {})]
    return sum(k["dram_bytes"] for k in ks) if ks else None


def ncu_region(ncu, region):
    """The committed capture's counters of the region's kernels (source: profiles/ncu_kernels.json)."""
    ks = {k: v for k, v in ncu.get("kernels", {}).items() if k in NCU_REGION_KERNELS[region]}
    return {"source": ncu.get("source"), "kernels": ks} if ks else {}


def cpu_oracle_sample(batch, seconds: float, total_candidates: int, keep=None):
    """The oracle (as it stands) on a bounded, deterministic sample of the
    workload, on all host cores.  ``keep`` (a dict) receives the sample's
    indices and oracle records for the per-run parity check."""
    import oracle
    cores = os.cpu_count() or 1
    n = len(batch)
    cal = max(32, min(256, n))
    idx = np.linspace(0, n - 1, cal).astype(np.int64)
    t0 = time.perf_counter()
    oracle.evaluate(batch.select(idx), threads=cores)
    t_cal = time.perf_counter() - t0
    m = int(min(n, max(cal, seconds / max(t_cal / cal, 1e-9))))
    idx = np.linspace(0, n - 1, m).astype(np.int64)
    sub = batch.select(idx)
    t0 = time.perf_counter()
    r = oracle.evaluate(sub, threads=cores)
    dt = time.perf_counter() - t0
    if keep is not None:
        keep["idx"], keep["ref"] = idx, r
    return {"value": m / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{m} candidates evenly spaced over the {total_candidates}-candidate sweep "
                      f"({int(r['W'].sum())} warp-accesses, {dt:.1f} s)",
            "wa_per_s": float(r["W"].sum()) / dt}


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    """--impl reference: the CPU oracle timed as it stands on the same workload,
    each step a bounded sample (rank 0 only)."""
    import gen
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    total = gen.num_candidates(args.config) if not args.candidates else args.candidates
    cores = os.cpu_count() or 1
    # size a step to ~6 s of host time, calibrated on a strided probe
    probe_idx = np.linspace(0, total - 1, 96).astype(np.int64)
    t0 = time.perf_counter()
    oracle.evaluate(gen.generate_indices(args.config, probe_idx), threads=cores)
    per_cand = (time.perf_counter() - t0) / len(probe_idx)
    step_s = float(os.environ.get("REF_STEP_SECONDS", "6.0"))
    per_step = int(max(32, min(total, step_s / max(per_cand, 1e-9))))
    stride = max(1, total // per_step)
    times, evals, was = [], 0, 0
    for step in range(args.warmup + args.steps):
        off = (step * 7919) % stride
        cidx = np.arange(off, total, stride)[:per_step]
        b = gen.generate_indices(args.config, cidx)
        t0 = time.perf_counter()
        r = oracle.evaluate(b, threads=cores)
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            times.append(dt)
            evals += len(b)
            was += int(r["W"].sum())
    T = sum(times)
    value = evals / T
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * T / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64+f64",
            "data": "synthetic", "config": {"workload": WORKLOAD, "candidates": total},
            "wa_expanded_per_s": was / T,
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"each step {per_step} candidates strided over the {total}-candidate sweep"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- our arm
def run_ours(args):
    import torch

    import gen
    import paper_conf_ipps_chikinaat19_b200 as sel
    from paper_conf_ipps_chikinaat19_b200 import dist as D

    rank, world, local = D.init()
    dev = torch.device("cuda", local)
    total = gen.num_candidates(args.config) if not args.candidates else args.candidates
    # config 4 (192 huge candidates) splits every candidate's warp-accesses across ranks
    # (SURVEY §8(e)); the others shard candidates by index range
    split = args.config == 4 and world > 1
    # N > 1: rank r evaluates chunks r and N + r of 2N (D.TwoPhaseGather) so the all-gather of the
    # first half of every rank's decisions runs while the second half is evaluated; the decisions
    # land directly in the preallocated gather buffer (in-place collectives, no copies)
    gatherer = D.TwoPhaseGather(total, world, rank, dev) if world > 1 and not split else None
    ranges = [(0, total)] if split or world == 1 else gatherer.ranges
    t_gen = time.perf_counter()
    shards = []
    for i, (a, b) in enumerate(ranges):
        bt = gen.generate(args.config, a, b)
        e = sel.Evaluator((bt.nests, bt.accesses, bt.launches, bt.devices), max(len(bt), 1), args.flags, device=dev)
        ch = torch.from_numpy(bt.cands.view(np.uint8).reshape(-1)).pin_memory()
        n_i = len(bt)
        o = {"decision": gatherer.slots[i] if gatherer else torch.empty(n_i, dtype=torch.uint8, device=dev),
             "cycles": torch.empty(n_i, dtype=torch.float64, device=dev),
             "status": torch.empty(n_i, dtype=torch.uint8, device=dev)}
        shards.append({"batch": bt, "ev": e, "cands_host": ch, "cands": ch.to(dev), "out": o, "range": (a, b)})
    t_gen = time.perf_counter() - t_gen
    batch, ev, cands, cands_host = shards[0]["batch"], shards[0]["ev"], shards[0]["cands"], shards[0]["cands_host"]
    c0, c1 = shards[0]["range"]
    out = shards[0]["out"]
    stream = torch.cuda.current_stream(dev)

    def step():
        nonlocal out
        if split:
            out = D.evaluate_split(cands, ev.tables, ev.workspace, rank, world, args.flags)
            return
        for i, sh in enumerate(shards):
            if len(sh["batch"]):
                sh["ev"].evaluate(sh["cands"], out=sh["out"])
            if gatherer:
                gatherer.gather(i)              # NCCL stream: overlaps the next shard's kernels
        if gatherer:
            gatherer.wait()

    int_peak = {"alu": sel.int_peak(0), "fma": sel.int_peak(1), "both": sel.int_peak(2)}
    nvtx = torch.cuda.nvtx                      # host-timeline ranges (the library adds sel:plan/count/model)
    nvtx.range_push("bench:warmup")
    for _ in range(args.warmup):
        step()
    nvtx.range_pop()
    torch.cuda.synchronize(dev)
    stats = {}
    for sh in shards:
        if not len(sh["batch"]):
            continue
        for k, v in sh["ev"].stats().items():
            stats[k] = stats.get(k, 0) + v
    sel.profile_enable(True)
    PROF = {"plan": sel.PROF_PLAN, "count": sel.PROF_COUNT, "model": sel.PROF_MODEL,
            "k_model_fused": sel.PROF_K_MODEL, "k_lane_problems": sel.PROF_K_LANE, "k_problem_w": sel.PROF_K_PROBLEM_W}
    for r in PROF.values():
        sel.profile_read_region(r)
    launches0 = sel.kernel_launches()
    D.barrier(world)
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        e0.record(stream)
        for k in range(args.steps):
            nvtx.range_push(f"bench:step {k}")
            step()
            nvtx.range_pop()
        e1.record(stream)
        torch.cuda.synchronize(dev)
    D.barrier(world)
    ms_local = e0.elapsed_time(e1)
    launches = sel.kernel_launches() - launches0
    prof = {k: sel.profile_read_region(r) for k, r in PROF.items()}       # name -> (ms, launches)
    sel.profile_enable(False)
    ms = D.max_over_ranks(ms_local, world, dev)
    wa_resolved = D.sum_over_ranks(stats["wa_resolved"], world, dev)
    wa_covered = D.sum_over_ranks(stats["wa_covered"], world, dev)
    n_invalid = D.sum_over_ranks(stats["n_invalid"], world, dev)
    wa_closed = D.sum_over_ranks(stats["wa_closed_form"], world, dev)
    wa_expanded = D.sum_over_ranks(stats["wa_expanded"], world, dev)
    t_step = ms / 1e3 / args.steps
    clocks = clk.summary()

    # ---- end to end through the public API: pinned host inputs -> decisions + cycles on the host
    e2e = None
    if not args.no_e2e and not split:
        # every step uploads its inputs (candidates + nest and access tables) from pinned host
        # memory and downloads decision + cycles to pinned host memory; sel.HostPipeline overlaps
        # step k+1's upload and step k-1's download with step k's kernels (two device slots)
        pipes, h2d, d2h = [], 0, 0
        for sh in shards:
            if not len(sh["batch"]):
                continue
            bt = sh["batch"]
            nests_h = torch.from_numpy(bt.nests.view(np.uint8).reshape(-1)).pin_memory()
            acc_h = torch.from_numpy(bt.accesses.view(np.uint8).reshape(-1)).pin_memory()
            hb, db = sel.HostPipeline.bytes_per_step(sh["cands_host"], nests_h, acc_h, len(bt))
            h2d, d2h = h2d + hb, d2h + db
            pipes.append((sel.HostPipeline(sh["ev"], sh["cands_host"], nests_h, acc_h), sh["cands_host"], nests_h,
                          acc_h))
        for k in range(max(1, args.warmup)):
            for p, ch, nh, ah in pipes:
                p.step(k, ch, nh, ah)
        torch.cuda.synchronize(dev)
        D.barrier(world)
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        join = torch.cuda.Stream(dev)
        if pipes:
            f0.record(pipes[0][0].h2d)
            for p, _, _, _ in pipes[1:]:
                p.h2d.wait_event(f0)             # no pipeline starts before the clock does
        else:
            f0.record(join)
        for k in range(args.steps):
            nvtx.range_push(f"bench:e2e step {k}")
            for p, ch, nh, ah in pipes:
                p.step(k, ch, nh, ah)
            nvtx.range_pop()
        for p, _, _, _ in pipes:
            join.wait_stream(p.d2h)
        f1.record(join)
        torch.cuda.synchronize(dev)
        ms_e2e = D.max_over_ranks(f0.elapsed_time(f1), world, dev)
        e2e = {"value": total / (ms_e2e / 1e3 / args.steps), "unit": UNIT,
               "h2d_bytes_per_step": D.sum_over_ranks(h2d, world, dev),
               "d2h_bytes_per_step": D.sum_over_ranks(d2h, world, dev),
               "ms_per_step": ms_e2e / args.steps, "overlap": "double-buffered H2D / kernels / D2H streams"}
        del pipes

    if rank != 0:
        return
    # ---- per-region device time (CUDA events the library records on the launching stream around the
    # plan, counting and model kernels of every call) and the roofline of each
    f_mhz = clocks["sm_mhz"] or measured_peaks().get("clocks_under_load", {}).get("sm_mhz_median", 1965.0)
    hbm_peak = measured_peaks().get("hbm_gbs")
    ncu = ncu_kernels()
    per_launch = {k: ms / max(k_n, 1) for k, (ms, k_n) in prof.items()}
    # counting kernels: INT bound.  peak = measured INT32 lane-op rate with the ALU and FMA pipes both
    # issuing (sel_int_peak mode 2), all SMs.  achieved = the nominal algorithmic lane-ops of the paths
    # the counting kernels took (sel_stats.alg_lane_ops) / their measured time
    peak_ops = int_peak["both"]
    wa_arith, wa_res, wa_cf = stats["wa_arith_lanes"], stats["wa_residue_classes"], stats["wa_closed_form"]
    wa_lane = stats["wa_resolved"] - wa_cf - wa_arith - wa_res
    avg_count_ms = per_launch["count"]
    achieved = stats["alg_lane_ops"] / (avg_count_ms / 1e3)
    survey_eq = stats["wa_resolved"] * OPS_PER_WA / (avg_count_ms / 1e3)
    roof_count = {"bound": "alu", "builder_weighted": True, "achieved": achieved / 1e12, "peak": peak_ops / 1e12,
                  "unit": "Tops/s",
                  "frac": achieved / peak_ops, "traffic": ncu_region_traffic(ncu, "count"),
                  "kernel": "counting kernels (k_lane_problems + k_queue + k_count)",
                  "ms_per_launch": avg_count_ms, "share_of_step": avg_count_ms / (t_step * 1e3),
                  "alg_lane_ops_per_step": stats["alg_lane_ops"],
                  "peak_source": "measured: sel_int_peak (independent IADD3/LOP3 + IMAD chains, all SMs, ALU and "
                                 "FMA pipes both issuing) at the run's clocks",
                  "peak_alu_pipe_only": int_peak["alu"] / 1e12, "peak_fma_pipe_only": int_peak["fma"] / 1e12,
                  "peak_nominal_issue": 148 * 128 * f_mhz * 1e6 / 1e12,
                  "wa_per_path": {"lane_expansion": wa_lane, "arith_lanes": wa_arith, "residue_classes": wa_res,
                                  "uniform_closed_form": wa_cf},
                  "survey_equivalent": {"ops_per_wa": OPS_PER_WA, "achieved": survey_eq / 1e12,
                                        "ratio_to_peak": survey_eq / peak_ops,
                                        "note": "SURVEY §8(d)'s 224 lane-ops x every analysed warp-access / "
                                                "counting time: the brute-force expansion rate the exact closed "
                                                "forms stand in for (> 1 = faster than expanding at the INT peak)"},
                  "note": ("NOT a measured counter: achieved = builder-weighted nominal lane-ops of the paths the "
                           "counting kernels took (sel_stats.alg_lane_ops) / their time; the measured INT-pipe "
                           "utilisation is int_pipe_ncu"),
                  "ncu": ncu_region(ncu, "count")}
    # model kernels (k_problem_model + k_model_fused): per candidate the 24 B record in, decision (1) +
    # cycles (8) + status (1) out -- HBM is the roofline of a streaming per-candidate kernel
    def hbm_roof(name, kernel, bytes_per_launch, detail):
        ms = per_launch[name]
        a = bytes_per_launch / (ms / 1e3) / 1e9 if ms > 0 else 0.0
        r = {"bound": "hbm", "achieved": a, "peak": hbm_peak, "unit": "GB/s",
             "frac": a / hbm_peak if hbm_peak else None, "traffic": ncu_region_traffic(ncu, name),
             "kernel": kernel, "ms_per_launch": ms, "share_of_step": ms / (t_step * 1e3),
             "algorithmic_bytes_per_launch": bytes_per_launch, "bytes": detail,
             "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy bandwidth, burst)", "ncu": ncu_region(ncu, name)}
        return r
    # per launch: a step evaluates every shard once, so each kernel launch processes on average
    # 1/len(shards) of this rank's candidates, nests and accesses
    ns = len(shards)
    n_cand_launch = sum(len(sh["batch"]) for sh in shards) // ns
    n_nests = sum(len(sh["batch"].nests) for sh in shards) // ns
    n_acc = sum(len(sh["batch"].accesses) for sh in shards) // ns
    roof_model = hbm_roof("model", "model kernels (k_problem_model + k_model_fused)", MODEL_BYTES * n_cand_launch,
                          f"{MODEL_BYTES} B per candidate (record in, decision + cycles + status out)")
    roof_plan = hbm_roof("plan", "plan kernels (k_classes, k_insert, k_problem_w, scans, ...)",
                         PLAN_BYTES * n_cand_launch + 88 * n_nests + 64 * n_acc,
                         f"{PLAN_BYTES} B per candidate (record in, problem id + status out) + every nest (88 B) "
                         f"and access (64 B) record once")
    regions = {"plan": roof_plan, "count": roof_count, "model": roof_model}
    # the dominant KERNEL (CUDA events around it alone, on the launching stream): k_model_fused against
    # HBM on its algorithmic 34 B per candidate, or k_lane_problems / k_problem_w, whichever is longest
    kern = {k: per_launch[k] for k in ("k_model_fused", "k_lane_problems", "k_problem_w")}
    dominant = max(kern, key=kern.get)
    kbytes = {"k_model_fused": (MODEL_BYTES * n_cand_launch,
                                f"{MODEL_BYTES} B per candidate (24 B record in; decision, cycles, status out)"),
              "k_problem_w": (88 * n_nests + 64 * n_acc + 34 * n_cand_launch // 10,
                              "every nest (88 B) and access (64 B) in, ~34 B per problem out"),
              "k_lane_problems": (88 * n_nests + 64 * n_acc + 40 * (n_cand_launch * 3 // 32),
                                  "every nest (88 B) and access (64 B) in, 40 B of counts per problem out")}
    kb, kdesc = kbytes[dominant]
    kms = kern[dominant]
    ka = kb / (kms / 1e3) / 1e9
    knc = ncu.get("kernels", {}).get(dominant, {})
    roofline = {"bound": "hbm", "achieved": ka, "peak": hbm_peak, "unit": "GB/s",
                "frac": ka / hbm_peak if hbm_peak else None,
                "traffic": knc.get("dram_bytes"), "kernel": dominant, "ms_per_launch": kms,
                "share_of_step": kms / (t_step * 1e3), "algorithmic_bytes_per_launch": kb, "bytes": kdesc,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy bandwidth, burst)",
                "traffic_source": ncu.get("source"),
                "ncu": {k: knc.get(k) for k in ("issue_active_pct", "warps_active_pct", "warp_instructions",
                                                "fp64_cycles_pct", "alu_cycles_pct", "fma_cycles_pct")}}
    # the north star's INT-pipe criterion: ncu sm__pipe_alu/fma_cycles_active of the counting kernel
    lane_nc = ncu.get("kernels", {}).get("k_lane_problems", {})
    int_pipe = {"kernel": "k_lane_problems", "source": ncu.get("source"),
                "alu_cycles_pct": lane_nc.get("alu_cycles_pct"), "fma_cycles_pct": lane_nc.get("fma_cycles_pct"),
                "alu_inst_pct": lane_nc.get("alu_pipe_pct"), "fma_inst_pct": lane_nc.get("fma_pipe_pct"),
                "issue_active_pct": lane_nc.get("issue_active_pct"),
                "ms_per_launch": per_launch["k_lane_problems"]}
    # the whole step against HBM: per candidate the 24 B record in, decision + cycles out
    step_hbm = {"bound": "hbm", "bytes_per_candidate": CAND_BYTES,
                "achieved": CAND_BYTES * total / t_step / 1e9, "peak": hbm_peak, "unit": "GB/s"}
    if step_hbm["peak"]:
        step_hbm["frac"] = step_hbm["achieved"] / step_hbm["peak"]
    hbm_bytes = (24 + 9) * total                     # candidate read + decision/cycles write per step
    workload = WORKLOAD if args.config == 5 else f"c{args.config}: BASELINE.json configs[{args.config - 1}]"
    parallelism = (f"dp{world} (warp-range split of every candidate) + all_reduce(SUM) of u64 counters" if split
                   else f"dp{world} (candidate shards) + NCCL all-gather of decisions")
    line = {"metric": METRIC, "value": total / t_step, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_step * 1e3, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int64+f64", "data": "synthetic",
            "config": {"workload": workload, "candidates": total, "count_sharing": not (args.flags & 1),
                       "lane_pattern_paths": not (args.flags & 8),
                       "residue_classes": not (args.flags & (8 | 16)),
                       "problems_per_lane": not (args.flags & (2 | 8 | 32)),
                       "counting_primitive": ("match_any" if args.flags & 2 else
                                              "residue (scalar)" if args.flags & 4 else "residue (byte-sliced)"),
                       "l2": (f"inputs larger than L2 ({24 * total / 1e9:.1f} GB of candidates per pass)"
                              if 24 * total > 126e6 else "inputs fit in L2 (not the metric workload)"),
                       "parallelism": parallelism},
            "wa_resolved_per_s": wa_resolved / t_step, "wa_expanded_per_s": wa_expanded / t_step,
            "wa_covered_per_s": wa_covered / t_step,
            "wa_resolved_per_step": wa_resolved, "wa_expanded_per_step": wa_expanded,
            "wa_covered_per_step": wa_covered, "invalid": n_invalid,
            "wa_closed_form_per_step": wa_closed,
            "wa_note": ("resolved = counted exactly on the GPU (closed forms included), expanded = of those, "
                        "expanded lane by lane, covered = sum over candidates (count sharing)"),
            "hbm_gbs": hbm_bytes / t_step / 1e9, "roofline": roofline,
            "roofline_by_region": {k: {kk: v[kk] for kk in ("bound", "achieved", "peak", "unit", "frac", "traffic",
                                                            "ms_per_launch", "share_of_step")}
                                   for k, v in regions.items()},
            "kernel_ms": {k: per_launch[k] for k in ("k_problem_w", "k_lane_problems", "k_model_fused")},
            "int_pipe_ncu": int_pipe, "count_nominal_ops": roof_count, "step_hbm_roofline": step_hbm,
            "gpu_launches": launches,
            "clocks": clocks, "e2e": e2e, "gen_s": t_gen}
    if not args.no_next and args.config == 5:
        line["next_rows"] = time_next_rows(sel, gen, ev, batch, cands, args, c0, c1, dev)
    if not args.no_cpu_baseline and world == 1:
        keep = {}
        line["cpu_baseline"] = cpu_oracle_sample(batch, args.cpu_seconds, total, keep)
        if not split:
            line["parity"] = parity_check(sel, batch, out, keep, dev, args.flags)
    print(json.dumps(line), flush=True)
    if line.get("parity", {}).get("mismatches"):
        sys.exit(3)


def parity_check(sel, batch, out, keep, dev, flags):
    """Per-run parity ("parity is checked on that subset every
    run"): the oracle records of the cpu_baseline sample against the timed
    step's decision, status and cycles at the same candidate indices (bit for
    bit), and the sample's counts (W, L, S, C, U, WR) from a second, small
    sel_evaluate on the sub-batch (slot-table problem ids).  Any mismatch
    makes bench.py exit with status 3 after printing its line."""
    import torch
    idx, ref = keep["idx"], keep["ref"]
    it = torch.from_numpy(idx).to(dev)
    got = {k: out[k][it].cpu().numpy() for k in ("decision", "status", "cycles")}
    sub = batch.select(idx)
    ev2 = sel.Evaluator((sub.nests, sub.accesses, sub.launches, sub.devices), len(sub), flags, device=dev)
    r2 = ev2.evaluate(sel._as_bytes_tensor(sub.cands, "candidate", dev), want_counts=True)
    cnt = r2["counts"].cpu().numpy().astype(np.uint64)
    bad = {"decision": int((got["decision"] != ref["decision"]).sum()),
           "status": int((got["status"] != ref["status"]).sum()),
           "cycles": int((got["cycles"].view(np.uint64) != ref["cycles"].view(np.uint64)).sum()),
           "subset_call_decision": int((r2["decision"].cpu().numpy() != ref["decision"]).sum()),
           "subset_call_cycles": int((r2["cycles"].cpu().numpy().view(np.uint64)
                                      != ref["cycles"].view(np.uint64)).sum())}
    for j, f in enumerate(("W", "L", "S", "C", "U", "WR")):
        bad[f] = int((cnt[:, j] != ref[f]).sum())
    del ev2
    return {"checked": int(len(idx)), "mismatches": int(sum(bad.values())), "by_field": bad,
            "how": ("oracle (cpu_baseline sample) vs the timed step's outputs at the same indices, bit for bit; "
                    "counts via a second sel_evaluate on the sample")}


def time_next_rows(sel, gen, ev, batch, cands, args, c0, c1, dev):
    """NEXT rows on this rank's c5 batch: f2 symbolic IPDA
    binding of every access, f1 Liao-Chapman CPU model of every candidate, f3
    launch selection per (nest, device) group.  Device time with CUDA events
    (best of 3 after a warm-up); results checked against the generator's
    concrete accesses (f2) and the supplied CPU cost (f1, no TLB misses in c5)."""
    import torch
    import numpy as np

    def timed(fn, reps=3):
        fn()
        torch.cuda.synchronize(dev)
        best = 1e30
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize(dev)
            best = min(best, a.elapsed_time(b))
        return best

    res = {}
    sym, terms = gen.sym_tables()
    vals, items = gen.sym_instances(args.config, c0, c1)
    sym_d, terms_d = sel._dev_bytes(sym, dev), sel._dev_bytes(terms, dev)
    vals_d, items_d = sel._dev_bytes(vals, dev), sel._dev_bytes(items, dev)
    bound = torch.empty(len(items) * 64, dtype=torch.uint8, device=dev)
    st = torch.empty(len(items), dtype=torch.uint8, device=dev)
    L = sel._lib.lib()

    def f2():
        sel._lib.check(L.sel_bind_accesses(sel._ptr(sym_d), len(sym), sel._ptr(terms_d), len(terms),
                                           sel._ptr(vals_d), len(vals), sel._ptr(items_d), len(items),
                                           sel._ptr(bound), sel._ptr(st), sel._stream()))
    ms = timed(f2)
    ok = bool(torch.equal(bound, ev.tables.accesses[: len(items) * 64])) and int(st.max().item()) == 0
    nbytes = len(items) * (8 + 64 + 1) + 9 * 8 * len(batch.nests)
    res["f2_bind"] = {"items": len(items), "ms": ms, "items_per_s": len(items) / (ms / 1e3),
                      "hbm_gbs": nbytes / (ms / 1e3) / 1e9, "matches_generator": ok}

    cin = sel._dev_bytes(gen.cpu_inputs(args.config, c0, c1), dev)
    params = gen.cpu_params()
    cc = cands.clone()

    def f1():
        sel.model_cpu_cost(cc, ev.tables, cin, params)
    ms = timed(f1)
    same = bool(torch.equal(cc, cands))
    n = len(batch)
    res["f1_cpu_model"] = {"candidates": n, "ms": ms, "candidates_per_s": n / (ms / 1e3),
                           "hbm_gbs": n * (24 + 16 + 24 + 1) / (ms / 1e3) / 1e9, "equals_supplied_cost": same}

    r = ev.evaluate(cands, want_t_gpu=True)
    group = torch.from_numpy((batch.cands["nest_id"].astype(np.int64) * 4 + batch.cands["device_id"]).astype(
        np.int32)).to(dev)
    n_groups = len(batch.nests) * 4

    def f3():
        sel.select_launch(group, r["t_gpu"], r["status"], n_groups)
    ms = timed(f3)
    res["f3_select_launch"] = {"candidates": n, "groups": n_groups, "ms": ms, "candidates_per_s": n / (ms / 1e3)}
    return res


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)
    try:
        import torch.distributed as dist
        if dist.is_initialized():
            dist.destroy_process_group()
    except Exception:
        pass


if __name__ == "__main__":
    main()
