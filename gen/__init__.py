"""Seeded synthetic inputs (ctypes binding to gen/libselgen.so).

Input data only -- none of the hot path's arithmetic lives here (see
selgen.h).  Both ``oracle/`` and the CUDA path consume these arrays.  The
numpy dtypes below are this module's own copy of the record layouts; the
CPU test ``tests/test_layout.py`` checks them against include/sel.h (via the
product binding) and oracle/oracle.h (via the oracle library).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libselgen.so")

DEVICE_DTYPE = np.dtype([
    ("num_sms", "<i4"), ("max_warps_per_sm", "<i4"), ("max_threads_per_sm", "<i4"),
    ("max_blocks_per_sm", "<i4"), ("regs_per_sm", "<i4"), ("smem_per_sm", "<i4"),
    ("sm_clock_hz", "<f8"), ("mem_bw_Bps", "<f8"), ("link_bw_Bps", "<f8"),
    ("launch_overhead_s", "<f8"), ("mem_ld_cycles", "<f8"), ("dep_del_coal", "<f8"),
    ("dep_del_uncoal", "<f8"), ("issue_cycles", "<f8"),
    ("reg_alloc_unit", "<i4"), ("warp_alloc_gran", "<i4"), ("smem_alloc_unit", "<i4"), ("txn_sectors", "<i4"),
])
ACCESS_DTYPE = np.dtype([
    ("base", "<i8"), ("c_par", "<i8", (2,)), ("c_inner", "<i8", (3,)),
    ("elem_bytes", "u1"), ("depth", "u1"), ("is_store", "u1"), ("_pad", "u1", (13,)),
])
NEST_DTYPE = np.dtype([
    ("P0", "<u8"), ("P1", "<u8"), ("trip", "<u4", (3,)), ("par_dims", "u1"), ("depth", "u1"),
    ("n_sync", "<u2"), ("comp_insts", "<f8", (4,)), ("bytes_h2d", "<u8"), ("bytes_d2h", "<u8"),
    ("access_off", "<u4"), ("n_access", "<u4"),
])
LAUNCH_DTYPE = np.dtype([
    ("block", "<u4"), ("grid_max", "<u4"), ("regs_per_thread", "<u4"), ("smem_per_block", "<u4"),
])
CANDIDATE_DTYPE = np.dtype([
    ("nest_id", "<u4"), ("launch_id", "<u2"), ("device_id", "<u2"),
    ("cpu_cycles", "<f8"), ("cpu_hz", "<f8"),
])
COUNTS_DTYPE = np.dtype([
    ("warp_accesses", "<u8"), ("lines", "<u8"), ("sectors", "<u8"),
    ("coalesced", "<u8"), ("uncoal_lines", "<u8"), ("warp_reps", "<u8"),
])

CPU_PARAMS_DTYPE = np.dtype([
    ("cpu_hz", "<f8"), ("tlb_entries", "<f8"), ("tlb_miss_cycles", "<f8"), ("loop_overhead_cycles", "<f8"),
    ("schedule_static_cycles", "<f8"), ("sync_cycles", "<f8"), ("startup_cycles", "<f8"), ("page_bytes", "<f8"),
])
CPU_INPUT_DTYPE = np.dtype([("mca_cycles_per_iter", "<f8"), ("threads", "<u4"), ("_pad", "<u4")])

SYM_TERM_DTYPE = np.dtype([("k", "<i8"), ("sym", "<u2", (3,)), ("_pad", "<u2")])
SYM_ACCESS_DTYPE = np.dtype([("term_off", "<u4", (6,)), ("n_terms", "u1", (6,)), ("elem_sym", "<u2"),
                             ("elem_bytes", "u1"), ("depth", "u1"), ("is_store", "u1"), ("_pad", "u1", (5,))])
BIND_ITEM_DTYPE = np.dtype([("sym_access", "<u4"), ("frame", "<u4")])
SYM_ONE = 0xFFFF

TRIP_UNKNOWN = 0xFFFFFFFF  # unknown trip counts are assumed to be 128
DEVICE_NAMES = ("K80", "P100", "V100", "B200")
V100 = 2

_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "selgen.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "selgen.h"))):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared",
                               "-o", _LIB_PATH, src])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        u64, vp = ctypes.c_uint64, ctypes.c_void_p
        L.selgen_num_candidates.restype = u64
        L.selgen_num_candidates.argtypes = [ctypes.c_int]
        L.selgen_device_sets.argtypes = [vp]
        L.selgen_launches.argtypes = [ctypes.c_int, vp]
        L.selgen_count.argtypes = [ctypes.c_int, u64, u64, ctypes.POINTER(u64), ctypes.POINTER(u64)]
        L.selgen_fill.argtypes = [ctypes.c_int, u64, u64, vp, vp, vp]
        L.selgen_shape_name.restype = ctypes.c_char_p
        L.selgen_shape_name.argtypes = [ctypes.c_int]
        L.selgen_count_indices.argtypes = [ctypes.c_int, vp, u64, ctypes.POINTER(u64)]
        L.selgen_fill_indices.argtypes = [ctypes.c_int, vp, u64, vp, vp, vp]
        L.selgen_cpu_inputs.argtypes = [ctypes.c_int, u64, u64, vp]
        L.selgen_cpu_params.argtypes = [vp]
        L.selgen_sym_tables.argtypes = [vp, vp, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
        L.selgen_sym_count.argtypes = [ctypes.c_int, u64, u64, ctypes.POINTER(u64), ctypes.POINTER(u64)]
        L.selgen_sym_fill.argtypes = [ctypes.c_int, u64, u64, vp, vp]
        L.selgen_rng.restype = u64
        L.selgen_rng.argtypes = [u64, u64]
        _lib = L
    return _lib


def num_candidates(cfg: int) -> int:
    return int(lib().selgen_num_candidates(cfg))


def device_sets() -> np.ndarray:
    out = np.zeros(4, DEVICE_DTYPE)
    lib().selgen_device_sets(out.ctypes.data)
    return out


def launches(cfg: int) -> np.ndarray:
    out = np.zeros(8, LAUNCH_DTYPE)
    n = lib().selgen_launches(cfg, out.ctypes.data)
    if n < 0:
        raise ValueError(f"unknown config {cfg}")
    return out[:n].copy()


def shape_names() -> list[str]:
    return [lib().selgen_shape_name(i).decode() for i in range(24)]


class Batch:
    """One batch of candidates plus the tables they reference (host numpy)."""

    def __init__(self, cands, nests, accesses, launches_, devices):
        self.cands = cands
        self.nests = nests
        self.accesses = accesses
        self.launches = launches_
        self.devices = devices

    def __len__(self):
        return len(self.cands)

    def select(self, idx) -> "Batch":
        """Sub-batch of candidates ``idx`` (tables are shared, not copied)."""
        return Batch(self.cands[np.asarray(idx)], self.nests, self.accesses, self.launches, self.devices)


def generate(cfg: int, c0: int = 0, c1: int | None = None) -> Batch:
    """Candidates [c0, c1) of config ``cfg`` (1..5) and their tables."""
    L = lib()
    if c1 is None:
        c1 = num_candidates(cfg)
    nn, na = ctypes.c_uint64(), ctypes.c_uint64()
    if L.selgen_count(cfg, c0, c1, ctypes.byref(nn), ctypes.byref(na)) != 0:
        raise ValueError(f"bad range [{c0}, {c1}) for config {cfg}")
    cands = np.zeros(c1 - c0, CANDIDATE_DTYPE)
    nests = np.zeros(max(nn.value, 1), NEST_DTYPE)
    acc = np.zeros(max(na.value, 1), ACCESS_DTYPE)
    if L.selgen_fill(cfg, c0, c1, cands.ctypes.data, nests.ctypes.data, acc.ctypes.data) != 0:
        raise ValueError("selgen_fill failed")
    return Batch(cands, nests, acc, launches(cfg), device_sets())


def generate_indices(cfg: int, idx) -> Batch:
    """Candidates ``idx`` of config 3 or 5 (index-addressable sweeps), each
    with its own nest copy; for configs 1, 2, 4 the full config is generated
    and sub-selected."""
    idx = np.ascontiguousarray(np.asarray(idx, dtype=np.uint64))
    if cfg not in (3, 5):
        return generate(cfg).select(idx.astype(np.int64))
    L = lib()
    na = ctypes.c_uint64()
    if L.selgen_count_indices(cfg, idx.ctypes.data, len(idx), ctypes.byref(na)) != 0:
        raise ValueError("bad candidate index")
    cands = np.zeros(len(idx), CANDIDATE_DTYPE)
    nests = np.zeros(max(len(idx), 1), NEST_DTYPE)
    acc = np.zeros(max(na.value, 1), ACCESS_DTYPE)
    if L.selgen_fill_indices(cfg, idx.ctypes.data, len(idx), cands.ctypes.data, nests.ctypes.data,
                             acc.ctypes.data) != 0:
        raise ValueError("selgen_fill_indices failed")
    return Batch(cands, nests, acc, launches(cfg), device_sets())


def cpu_inputs(cfg: int, c0: int = 0, c1: int | None = None) -> np.ndarray:
    """NEXT row f1 inputs (MCA stand-in cycles per parallel iteration, threads)."""
    if c1 is None:
        c1 = num_candidates(cfg)
    out = np.zeros(c1 - c0, CPU_INPUT_DTYPE)
    if lib().selgen_cpu_inputs(cfg, c0, c1, out.ctypes.data) != 0:
        raise ValueError("bad range")
    return out


def cpu_params() -> np.ndarray:
    """Table II constants + page size, one record."""
    out = np.zeros(1, CPU_PARAMS_DTYPE)
    lib().selgen_cpu_params(out.ctypes.data)
    return out


def sym_tables():
    """NEXT row f2: (symbolic accesses, term pool) of the 24 shapes x {1-D, collapse}."""
    L = lib()
    ns, nt = ctypes.c_uint32(), ctypes.c_uint32()
    L.selgen_sym_tables(None, None, ctypes.byref(ns), ctypes.byref(nt))
    sym = np.zeros(ns.value, SYM_ACCESS_DTYPE)
    terms = np.zeros(nt.value, SYM_TERM_DTYPE)
    L.selgen_sym_tables(sym.ctypes.data, terms.ctypes.data, ctypes.byref(ns), ctypes.byref(nt))
    return sym, terms


def sym_instances(cfg: int, c0: int = 0, c1: int | None = None):
    """NEXT row f2: (symbol frames int64, bind items) for the accesses that
    ``generate(cfg, c0, c1)`` produces, in the same order (configs 2, 5)."""
    L = lib()
    if c1 is None:
        c1 = num_candidates(cfg)
    nv, ni = ctypes.c_uint64(), ctypes.c_uint64()
    if L.selgen_sym_count(cfg, c0, c1, ctypes.byref(nv), ctypes.byref(ni)) != 0:
        raise ValueError("symbolic instances exist for configs 2 and 5 only")
    values = np.zeros(max(nv.value, 1), np.int64)
    items = np.zeros(max(ni.value, 1), BIND_ITEM_DTYPE)
    if L.selgen_sym_fill(cfg, c0, c1, values.ctypes.data, items.ctypes.data) != 0:
        raise ValueError("selgen_sym_fill failed")
    return values, items[:ni.value]


def rng(seed: int, i: int) -> int:
    return int(lib().selgen_rng(seed, i))


# ---------------------------------------------------------------- builders
def make_access(base=0, c_par=(0, 0), c_inner=(0, 0, 0), elem_bytes=4, depth=0, is_store=0):
    a = np.zeros(1, ACCESS_DTYPE)[0]
    a["base"] = base
    a["c_par"] = list(c_par) + [0] * (2 - len(c_par))
    a["c_inner"] = list(c_inner) + [0] * (3 - len(c_inner))
    a["elem_bytes"], a["depth"], a["is_store"] = elem_bytes, depth, is_store
    return a


def custom_batch(items, devices=None, launches_=None) -> Batch:
    """Build a batch from hand-written candidates (tests).

    ``items`` is a list of dicts with keys: P0, P1 (default 1), par_dims
    (default 1), trip (list), depth, comp (list), accesses (list of
    make_access records), bytes_h2d, bytes_d2h, launch (index), device
    (index), cpu_cycles, cpu_hz.
    """
    if devices is None:
        devices = device_sets()
    if launches_ is None:
        launches_ = np.zeros(1, LAUNCH_DTYPE)
        launches_[0] = (256, 65535, 32, 0)
    nests = np.zeros(max(len(items), 1), NEST_DTYPE)
    accs = []
    cands = np.zeros(len(items), CANDIDATE_DTYPE)
    for i, it in enumerate(items):
        n = nests[i]
        n["P0"], n["P1"] = it["P0"], it.get("P1", 1)
        n["par_dims"] = it.get("par_dims", 1)
        trip = list(it.get("trip", [])) + [0] * (3 - len(it.get("trip", [])))
        n["trip"] = trip
        n["depth"] = it.get("depth", len(it.get("trip", [])))
        comp = list(it.get("comp", [])) + [0.0] * (4 - len(it.get("comp", [])))
        n["comp_insts"] = comp
        n["bytes_h2d"], n["bytes_d2h"] = it.get("bytes_h2d", 0), it.get("bytes_d2h", 0)
        n["access_off"] = len(accs)
        n["n_access"] = len(it["accesses"])
        accs.extend(it["accesses"])
        cands[i] = (i, it.get("launch", 0), it.get("device", V100),
                    it.get("cpu_cycles", 1e6), it.get("cpu_hz", 3e9))
    acc = np.zeros(max(len(accs), 1), ACCESS_DTYPE)
    for k, a in enumerate(accs):
        acc[k] = a
    return Batch(cands, nests, acc, launches_, devices)
