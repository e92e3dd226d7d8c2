"""B200-native batched GPU-side offload-model evaluation (Chikin et al., IPDPSW 2019).

Thin Python layer over the C ABI of libsel.so (include/sel.h).  Torch is
used for device memory and streams only; every step of the hot path -- the
per-warp coalescing counts, the Hong & Kim MWP/CWP cycle prediction with
#OMP_Rep and the CPU-or-GPU decision -- runs in the sm_100a kernels behind
the ABI.  There is no CPU fallback: without libsel.so or a GPU these calls
raise.

Records are passed as raw bytes: numpy structured arrays or torch uint8
tensors whose layout is the one declared in include/sel.h (the generator in
gen/ produces exactly that layout).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _lib
from ._lib import (DECISION_CPU, DECISION_GPU, DECISION_INVALID, SEL_EINTERNAL, SEL_EINVAL, SEL_ELAUNCH,
                   SEL_ERANGE, SEL_F_MATCH_ANY, SEL_F_NO_DEDUP, SEL_OK, SelError)

__all__ = ["load_device_params", "workspace_size", "DeviceTables", "count_transactions", "predict_gpu_cycles",
           "select", "evaluate", "evaluate_cpu_model", "read_stats", "profile_enable", "profile_read", "profile_read_region", "PROF_PLAN", "PROF_COUNT", "PROF_MODEL",
           "PROF_K_MODEL", "PROF_K_LANE", "PROF_K_PROBLEM_W", "kernel_launches",
           "Evaluator", "SelError", "SEL_F_NO_DEDUP", "SEL_F_MATCH_ANY", "DECISION_CPU", "DECISION_GPU",
           "DECISION_INVALID", "SEL_OK", "SEL_EINVAL", "SEL_ERANGE", "SEL_ELAUNCH", "SEL_EINTERNAL"]

_REC_SIZE = {"device": ctypes.sizeof(_lib.DeviceParams), "access": ctypes.sizeof(_lib.Access),
             "nest": ctypes.sizeof(_lib.Nest), "launch": ctypes.sizeof(_lib.Launch),
             "candidate": ctypes.sizeof(_lib.Candidate), "counts": ctypes.sizeof(_lib.Counts)}


def _as_bytes_tensor(x, rec: str, device="cuda") -> torch.Tensor:
    """numpy structured array / bytes tensor -> contiguous uint8 tensor on ``device``."""
    if isinstance(x, torch.Tensor):
        t = x.view(torch.uint8) if x.dtype != torch.uint8 else x
        t = t.reshape(-1)
    else:
        a = np.ascontiguousarray(x)
        if a.dtype.itemsize != _REC_SIZE[rec]:
            raise ValueError(f"{rec} records must be {_REC_SIZE[rec]} bytes, got {a.dtype.itemsize}")
        t = torch.from_numpy(a.view(np.uint8).reshape(-1))
    if t.numel() % _REC_SIZE[rec]:
        raise ValueError(f"{rec} buffer is not a whole number of records")
    if device is not None and (t.device.type != torch.device(device).type):
        t = t.to(device, non_blocking=True)
    return t.contiguous()


def _n(t: torch.Tensor, rec: str) -> int:
    return t.numel() // _REC_SIZE[rec]


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _require_cuda(*ts):
    for t in ts:
        if t is not None and t.device.type != "cuda":
            raise ValueError("libsel arguments must be CUDA tensors")


# ------------------------------------------------------------------ API
def load_device_params(sets) -> None:
    """sel_load_device_params: copy 1..16 device parameter sets (host)."""
    a = np.ascontiguousarray(sets)
    if a.dtype.itemsize != _REC_SIZE["device"]:
        raise ValueError(f"device parameter records must be {_REC_SIZE['device']} bytes")
    _lib.check(_lib.lib().sel_load_device_params(a.ctypes.data, len(a)))


def workspace_size(n: int, n_nests: int, flags: int = 0) -> int:
    return int(_lib.lib().sel_workspace_size(n, n_nests, flags))


def alloc_workspace(n: int, n_nests: int, flags: int = 0, device="cuda") -> torch.Tensor:
    nbytes = workspace_size(n, n_nests, flags)
    return torch.empty(nbytes + 256, dtype=torch.uint8, device=device)


def _ws_ptr(ws: torch.Tensor):
    p = ws.data_ptr()
    return ctypes.c_void_p((p + 255) & ~255), ws.numel() - (((p + 255) & ~255) - p)


class DeviceTables:
    """Device copies of the shared descriptor tables (nests, accesses, launches)."""

    def __init__(self, nests, accesses, launches, device="cuda"):
        self.nests = _as_bytes_tensor(nests, "nest", device)
        self.accesses = _as_bytes_tensor(accesses, "access", device)
        self.launches = _as_bytes_tensor(launches, "launch", device)
        self.n_nests = _n(self.nests, "nest")
        self.c = _lib.Tables(self.nests.data_ptr(), self.n_nests, self.accesses.data_ptr(),
                             _n(self.accesses, "access"), self.launches.data_ptr(), _n(self.launches, "launch"))

    def ref(self):
        return ctypes.byref(self.c)


def count_transactions(cands: torch.Tensor, tables: DeviceTables, workspace: torch.Tensor, flags: int = 0,
                       out=None, status=None, stream=None, part: int = 0, n_parts: int = 1):
    """sel_count_transactions (or sel_count_transactions_part when n_parts > 1)
    -> (counts int64[n, 6], status uint8[n])."""
    _require_cuda(cands, workspace)
    n = _n(cands, "candidate")
    dev = cands.device
    out = torch.empty((n, 6), dtype=torch.int64, device=dev) if out is None else out
    status = torch.empty(n, dtype=torch.uint8, device=dev) if status is None else status
    wp, wb = _ws_ptr(workspace)
    if n_parts == 1 and part == 0:
        _lib.check(_lib.lib().sel_count_transactions(_ptr(cands), n, tables.ref(), _ptr(out), _ptr(status), wp, wb,
                                                     flags, _stream(stream)))
    else:
        _lib.check(_lib.lib().sel_count_transactions_part(_ptr(cands), n, tables.ref(), part, n_parts, _ptr(out),
                                                          _ptr(status), wp, wb, flags, _stream(stream)))
    return out, status


def predict_gpu_cycles(cands: torch.Tensor, tables: DeviceTables, counts: torch.Tensor, status: torch.Tensor,
                       want_t_gpu: bool = True, stream=None):
    """sel_predict_gpu_cycles -> (cycles f64[n], t_gpu f64[n] | None); status is updated in place."""
    _require_cuda(cands, counts, status)
    n = _n(cands, "candidate")
    cycles = torch.empty(n, dtype=torch.float64, device=cands.device)
    t_gpu = torch.empty(n, dtype=torch.float64, device=cands.device) if want_t_gpu else None
    _lib.check(_lib.lib().sel_predict_gpu_cycles(_ptr(cands), n, tables.ref(), _ptr(counts), _ptr(cycles),
                                                 _ptr(t_gpu), _ptr(status), _stream(stream)))
    return cycles, t_gpu


def select(cands: torch.Tensor, t_gpu: torch.Tensor, status: torch.Tensor, stream=None) -> torch.Tensor:
    """sel_select -> decision uint8[n] (1 GPU, 0 CPU, 0xFF invalid)."""
    _require_cuda(cands, t_gpu, status)
    n = _n(cands, "candidate")
    decision = torch.empty(n, dtype=torch.uint8, device=cands.device)
    _lib.check(_lib.lib().sel_select(_ptr(cands), n, _ptr(t_gpu), _ptr(status), _ptr(decision), _stream(stream)))
    return decision


def evaluate(cands: torch.Tensor, tables: DeviceTables, workspace: torch.Tensor, flags: int = 0,
             want_counts: bool = False, want_t_gpu: bool = False, out: dict | None = None, stream=None) -> dict:
    """sel_evaluate (fused a1-a7) -> dict of decision, cycles, status [, t_gpu, counts]."""
    _require_cuda(cands, workspace)
    n = _n(cands, "candidate")
    dev = cands.device
    if out is None:
        out = {"decision": torch.empty(n, dtype=torch.uint8, device=dev),
               "cycles": torch.empty(n, dtype=torch.float64, device=dev),
               "status": torch.empty(n, dtype=torch.uint8, device=dev)}
        if want_t_gpu:
            out["t_gpu"] = torch.empty(n, dtype=torch.float64, device=dev)
        if want_counts:
            out["counts"] = torch.empty((n, 6), dtype=torch.int64, device=dev)
    wp, wb = _ws_ptr(workspace)
    _lib.check(_lib.lib().sel_evaluate(_ptr(cands), n, tables.ref(), _ptr(out["decision"]), _ptr(out["cycles"]),
                                       _ptr(out.get("t_gpu")), _ptr(out.get("counts")), _ptr(out["status"]), wp, wb,
                                       flags, _stream(stream)))
    return out


def evaluate_cpu_model(cands: torch.Tensor, tables: DeviceTables, workspace: torch.Tensor, cpu_in, params,
                       flags: int = 0, want_counts: bool = False, want_t_gpu: bool = False, stream=None) -> dict:
    """sel_evaluate_cpu_model (NEXT row f1 fused into a7): sel_evaluate with the
    Liao-Chapman CPU cost computed in the same pass -> dict of decision,
    cycles, status [, t_gpu, counts]."""
    _require_cuda(cands, workspace)
    n = _n(cands, "candidate")
    dev = cands.device
    cin = cpu_in if isinstance(cpu_in, torch.Tensor) else torch.from_numpy(
        np.ascontiguousarray(cpu_in).view(np.uint8).reshape(-1)).to(dev)
    p = np.ascontiguousarray(params)
    if p.dtype.itemsize != 64:
        raise ValueError("CPU parameter record must be 64 bytes")
    out = {"decision": torch.empty(n, dtype=torch.uint8, device=dev),
           "cycles": torch.empty(n, dtype=torch.float64, device=dev),
           "status": torch.empty(n, dtype=torch.uint8, device=dev)}
    if want_t_gpu:
        out["t_gpu"] = torch.empty(n, dtype=torch.float64, device=dev)
    if want_counts:
        out["counts"] = torch.empty((n, 6), dtype=torch.int64, device=dev)
    wp, wb = _ws_ptr(workspace)
    _lib.check(_lib.lib().sel_evaluate_cpu_model(_ptr(cands), n, tables.ref(), _ptr(cin), p.ctypes.data,
                                                 _ptr(out["decision"]), _ptr(out["cycles"]), _ptr(out.get("t_gpu")),
                                                 _ptr(out.get("counts")), _ptr(out["status"]), wp, wb, flags,
                                                 _stream(stream)))
    return out


def select_launch(group_of: torch.Tensor, t_gpu: torch.Tensor, status: torch.Tensor, n_groups: int, stream=None):
    """sel_select_launch (NEXT row f3) -> (best uint32-as-int32[n_groups], best_t_gpu f64[n_groups])."""
    _require_cuda(group_of, t_gpu, status)
    n = t_gpu.numel()
    best = torch.empty(n_groups, dtype=torch.int32, device=t_gpu.device)
    best_t = torch.empty(n_groups, dtype=torch.float64, device=t_gpu.device)
    _lib.check(_lib.lib().sel_select_launch(_ptr(group_of), n, _ptr(t_gpu), _ptr(status), n_groups, _ptr(best),
                                            _ptr(best_t), _stream(stream)))
    return best, best_t


def model_cpu_cost(cands: torch.Tensor, tables: DeviceTables, cpu_in, params, stream=None) -> torch.Tensor:
    """sel_model_cpu_cost (NEXT row f1): overwrite the candidates' cpu_cycles /
    cpu_hz with the Liao-Chapman model; returns status uint8[n]."""
    _require_cuda(cands)
    n = _n(cands, "candidate")
    cin = cpu_in if isinstance(cpu_in, torch.Tensor) else torch.from_numpy(
        np.ascontiguousarray(cpu_in).view(np.uint8).reshape(-1)).to(cands.device)
    p = np.ascontiguousarray(params)
    if p.dtype.itemsize != 64:
        raise ValueError("CPU parameter record must be 64 bytes")
    status = torch.empty(n, dtype=torch.uint8, device=cands.device)
    _lib.check(_lib.lib().sel_model_cpu_cost(_ptr(cands), n, tables.ref(), _ptr(cin), p.ctypes.data,
                                             _ptr(status), _stream(stream)))
    return status


def _dev_bytes(x, device):
    if isinstance(x, torch.Tensor):
        return x.view(torch.uint8).reshape(-1).to(device)
    a = np.ascontiguousarray(x)
    return torch.from_numpy(a.view(np.uint8).reshape(-1)).to(device)


def bind_accesses(sym, terms, values, items, device="cuda", out: torch.Tensor | None = None, stream=None):
    """sel_bind_accesses (NEXT row f2): symbolic IPDA accesses + symbol frames
    -> (concrete access records as uint8[n*64] on the device, status uint8[n])."""
    sym_d, terms_d = _dev_bytes(sym, device), _dev_bytes(terms, device)
    val_d, items_d = _dev_bytes(values, device), _dev_bytes(items, device)
    n = items_d.numel() // 8
    out = torch.empty(n * 64, dtype=torch.uint8, device=device) if out is None else out
    status = torch.empty(n, dtype=torch.uint8, device=device)
    _lib.check(_lib.lib().sel_bind_accesses(_ptr(sym_d), sym_d.numel() // 40, _ptr(terms_d), terms_d.numel() // 16,
                                            _ptr(val_d), val_d.numel() // 8, _ptr(items_d), n, _ptr(out),
                                            _ptr(status), _stream(stream)))
    return out, status


def read_stats(workspace: torch.Tensor, stream=None) -> dict:
    st = _lib.Stats()
    wp, _ = _ws_ptr(workspace)
    _lib.check(_lib.lib().sel_read_stats(wp, ctypes.byref(st), _stream(stream)))
    return {k: int(getattr(st, k)) for k in ("n_candidates", "n_problems", "wa_resolved", "wa_covered",
                                             "n_invalid", "wa_closed_form", "wa_arith_lanes", "wa_residue_classes",
                                             "alg_lane_ops", "wa_expanded")}


def profile_enable(on: bool = True) -> None:
    _lib.check(_lib.lib().sel_profile_enable(1 if on else 0))


def profile_read():
    """-> (counting-kernel milliseconds, counting launches) since the last read."""
    ms, k = ctypes.c_double(), ctypes.c_uint64()
    _lib.check(_lib.lib().sel_profile_read(ctypes.byref(ms), ctypes.byref(k)))
    return ms.value, k.value


PROF_PLAN, PROF_COUNT, PROF_MODEL = 0, 1, 2        # sel.h SEL_PROF_*: regions
PROF_K_MODEL, PROF_K_LANE, PROF_K_PROBLEM_W = 3, 4, 5   # single kernels


def profile_read_region(region: int):
    """-> (milliseconds, launches) of one profiling region (PROF_PLAN,
    PROF_COUNT, PROF_MODEL) or kernel (PROF_K_*) since its last read."""
    ms, k = ctypes.c_double(), ctypes.c_uint64()
    _lib.check(_lib.lib().sel_profile_read_region(int(region), ctypes.byref(ms), ctypes.byref(k)))
    return ms.value, k.value


def int_peak(mode: int = 2) -> float:
    """Measured INT32 lane-ops/s (mode 0 ALU pipe, 1 FMA pipe, 2 both)."""
    v = ctypes.c_double()
    _lib.check(_lib.lib().sel_int_peak(mode, ctypes.byref(v)))
    return v.value


def kernel_launches() -> int:
    return int(_lib.lib().sel_kernel_launches())


# same names as the C ABI
sel_load_device_params = load_device_params
sel_workspace_size = workspace_size
sel_count_transactions = count_transactions
sel_predict_gpu_cycles = predict_gpu_cycles
sel_select = select
sel_evaluate = evaluate
sel_evaluate_cpu_model = evaluate_cpu_model
sel_read_stats = read_stats
sel_select_launch = select_launch
sel_model_cpu_cost = model_cpu_cost
sel_bind_accesses = bind_accesses


class Evaluator:
    """Convenience holder: device tables + a workspace sized for up to
    ``max_n`` candidates.  ``evaluate`` takes device candidates;
    ``evaluate_host`` takes host (ideally pinned) candidates and copies them
    in and the decisions/cycles out on the same stream (end-to-end path)."""

    def __init__(self, batch_tables, max_n: int, flags: int = 0, device="cuda"):
        nests, accesses, launches, devices = batch_tables
        load_device_params(devices)
        self.tables = DeviceTables(nests, accesses, launches, device)
        self.flags = flags
        self.max_n = max_n
        self.workspace = alloc_workspace(max_n, self.tables.n_nests, flags, device)
        self.device = device

    def evaluate(self, cands: torch.Tensor, **kw) -> dict:
        if _n(cands, "candidate") > self.max_n:
            raise ValueError("batch larger than the workspace")
        return evaluate(cands, self.tables, self.workspace, self.flags, **kw)

    def evaluate_host(self, cands_host: torch.Tensor, out_host: dict | None = None, stream=None) -> dict:
        """H2D copy of the candidates, sel_evaluate, D2H copy of decision and cycles."""
        n = _n(cands_host, "candidate")
        d = cands_host.to(self.device, non_blocking=True)
        res = self.evaluate(d)
        if out_host is None:
            out_host = {"decision": torch.empty(n, dtype=torch.uint8, pin_memory=True),
                        "cycles": torch.empty(n, dtype=torch.float64, pin_memory=True)}
        out_host["decision"].copy_(res["decision"], non_blocking=True)
        out_host["cycles"].copy_(res["cycles"], non_blocking=True)
        return out_host

    def stats(self) -> dict:
        return read_stats(self.workspace)


class HostPipeline:
    """End-to-end evaluation from pinned host memory with copy/compute overlap.

    Each ``step`` uploads that step's inputs (candidates, nest and access
    tables) from pinned host buffers into one of two device slots on an H2D
    stream, runs ``sel_evaluate`` on a compute stream once that upload is done,
    and downloads decision and cycles into pinned host buffers on a D2H stream,
    so the uploads of step k+1 and the downloads of step k-1 overlap the
    kernels of step k.  Results of step k are valid after ``wait(k)``."""

    def __init__(self, ev: Evaluator, cands_host: torch.Tensor, nests_host: torch.Tensor, acc_host: torch.Tensor):
        dev = ev.device
        self.ev = ev
        self.n = _n(cands_host, "candidate")
        self.h2d, self.comp, self.d2h = (torch.cuda.Stream(dev) for _ in range(3))
        self.slots = []
        for _ in range(2):
            s = {"cands": torch.empty(cands_host.numel(), dtype=torch.uint8, device=dev),
                 "nests": torch.empty(nests_host.numel(), dtype=torch.uint8, device=dev),
                 "acc": torch.empty(acc_host.numel(), dtype=torch.uint8, device=dev),
                 "out": {"decision": torch.empty(self.n, dtype=torch.uint8, device=dev),
                         "cycles": torch.empty(self.n, dtype=torch.float64, device=dev),
                         "status": torch.empty(self.n, dtype=torch.uint8, device=dev)},
                 "host": {"decision": torch.empty(self.n, dtype=torch.uint8, pin_memory=True),
                          "cycles": torch.empty(self.n, dtype=torch.float64, pin_memory=True)},
                 "up": torch.cuda.Event(), "done": torch.cuda.Event(), "down": torch.cuda.Event(),
                 "used": False}
            s["tables"] = DeviceTables(s["nests"], s["acc"], ev.tables.launches, dev)
            self.slots.append(s)

    def step(self, k: int, cands_host: torch.Tensor, nests_host: torch.Tensor, acc_host: torch.Tensor) -> dict:
        s = self.slots[k % 2]
        if s["used"]:
            self.h2d.wait_event(s["done"])        # inputs of step k-2 consumed
            self.comp.wait_event(s["down"])       # outputs of step k-2 downloaded
        with torch.cuda.stream(self.h2d):
            s["cands"].copy_(cands_host, non_blocking=True)
            s["nests"].copy_(nests_host, non_blocking=True)
            s["acc"].copy_(acc_host, non_blocking=True)
            s["up"].record(self.h2d)
        self.comp.wait_event(s["up"])
        evaluate(s["cands"], s["tables"], self.ev.workspace, self.ev.flags, out=s["out"], stream=self.comp)
        s["done"].record(self.comp)
        self.d2h.wait_event(s["done"])
        with torch.cuda.stream(self.d2h):
            s["host"]["decision"].copy_(s["out"]["decision"], non_blocking=True)
            s["host"]["cycles"].copy_(s["out"]["cycles"], non_blocking=True)
            s["down"].record(self.d2h)
        s["used"] = True
        return s["host"]

    def wait(self, k: int) -> dict:
        s = self.slots[k % 2]
        s["down"].synchronize()
        return s["host"]

    @staticmethod
    def bytes_per_step(cands_host, nests_host, acc_host, n):
        return cands_host.numel() + nests_host.numel() + acc_host.numel(), n * 9
