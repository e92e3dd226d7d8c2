"""ctypes binding to libsel.so (include/sel.h) -- argument marshalling only.

Every step of the hot path runs in the CUDA kernels behind the C ABI; this
module only converts torch tensors / numpy arrays into pointers, sizes and
the caller's CUDA stream.  It never imports the CPU oracle and has no
fallback: if libsel.so is missing or no GPU is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SEL_LIBSEL", os.path.join(_HERE, "libsel.so"))   # override: build variants

SEL_OK, SEL_EINVAL, SEL_ERANGE, SEL_ELAUNCH, SEL_ENODEV, SEL_ECUDA, SEL_EINTERNAL = range(7)
SEL_F_NO_DEDUP = 1
SEL_F_MATCH_ANY = 2
SEL_F_SCALAR = 4
SEL_F_EXPAND_ALL = 8
SEL_F_NO_RESIDUE_CLASSES = 16
SEL_F_WARP_PROBLEMS = 32
DECISION_CPU, DECISION_GPU, DECISION_INVALID = 0, 1, 0xFF


class SelError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"libsel error {code}: {msg}")
        self.code = code


# ---------------------------------------------------------------- records
class DeviceParams(ctypes.Structure):
    _fields_ = [("num_sms", ctypes.c_int32), ("max_warps_per_sm", ctypes.c_int32),
                ("max_threads_per_sm", ctypes.c_int32), ("max_blocks_per_sm", ctypes.c_int32),
                ("regs_per_sm", ctypes.c_int32), ("smem_per_sm", ctypes.c_int32),
                ("sm_clock_hz", ctypes.c_double), ("mem_bw_Bps", ctypes.c_double),
                ("link_bw_Bps", ctypes.c_double), ("launch_overhead_s", ctypes.c_double),
                ("mem_ld_cycles", ctypes.c_double), ("dep_del_coal", ctypes.c_double),
                ("dep_del_uncoal", ctypes.c_double), ("issue_cycles", ctypes.c_double),
                ("reg_alloc_unit", ctypes.c_int32), ("warp_alloc_gran", ctypes.c_int32),
                ("smem_alloc_unit", ctypes.c_int32), ("txn_sectors", ctypes.c_int32)]


class Access(ctypes.Structure):
    _fields_ = [("base", ctypes.c_int64), ("c_par", ctypes.c_int64 * 2), ("c_inner", ctypes.c_int64 * 3),
                ("elem_bytes", ctypes.c_uint8), ("depth", ctypes.c_uint8), ("is_store", ctypes.c_uint8),
                ("_pad", ctypes.c_uint8 * 13)]


class Nest(ctypes.Structure):
    _fields_ = [("P0", ctypes.c_uint64), ("P1", ctypes.c_uint64), ("trip", ctypes.c_uint32 * 3),
                ("par_dims", ctypes.c_uint8), ("depth", ctypes.c_uint8), ("n_sync", ctypes.c_uint16),
                ("comp_insts", ctypes.c_double * 4), ("bytes_h2d", ctypes.c_uint64),
                ("bytes_d2h", ctypes.c_uint64), ("access_off", ctypes.c_uint32), ("n_access", ctypes.c_uint32)]


class Launch(ctypes.Structure):
    _fields_ = [("block", ctypes.c_uint32), ("grid_max", ctypes.c_uint32),
                ("regs_per_thread", ctypes.c_uint32), ("smem_per_block", ctypes.c_uint32)]


class Candidate(ctypes.Structure):
    _fields_ = [("nest_id", ctypes.c_uint32), ("launch_id", ctypes.c_uint16), ("device_id", ctypes.c_uint16),
                ("cpu_cycles", ctypes.c_double), ("cpu_hz", ctypes.c_double)]


class Counts(ctypes.Structure):
    _fields_ = [("warp_accesses", ctypes.c_uint64), ("lines", ctypes.c_uint64), ("sectors", ctypes.c_uint64),
                ("coalesced", ctypes.c_uint64), ("uncoal_lines", ctypes.c_uint64), ("warp_reps", ctypes.c_uint64)]


class Tables(ctypes.Structure):
    _fields_ = [("nests", ctypes.c_void_p), ("n_nests", ctypes.c_uint64),
                ("accesses", ctypes.c_void_p), ("n_accesses", ctypes.c_uint64),
                ("launches", ctypes.c_void_p), ("n_launches", ctypes.c_uint64)]


class Stats(ctypes.Structure):
    _fields_ = [("n_candidates", ctypes.c_uint64), ("n_problems", ctypes.c_uint64),
                ("wa_resolved", ctypes.c_uint64), ("wa_covered", ctypes.c_uint64),
                ("n_invalid", ctypes.c_uint64), ("wa_closed_form", ctypes.c_uint64),
                ("wa_arith_lanes", ctypes.c_uint64), ("wa_residue_classes", ctypes.c_uint64),
                ("alg_lane_ops", ctypes.c_uint64), ("wa_expanded", ctypes.c_uint64),
                ("_reserved", ctypes.c_uint64 * 6)]


RECORDS = (DeviceParams, Access, Nest, Launch, Candidate, Counts)

_lib = None


def lib():
    """Load libsel.so (built by __graft_entry__.build()); raises if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        vp, u64, u32, sz = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_size_t
        T = ctypes.POINTER(Tables)
        L.sel_load_device_params.argtypes = [vp, ctypes.c_int]
        L.sel_workspace_size.restype = sz
        L.sel_workspace_size.argtypes = [u64, u64, u32]
        L.sel_count_transactions.argtypes = [vp, u64, T, vp, vp, vp, sz, u32, vp]
        L.sel_count_transactions_part.argtypes = [vp, u64, T, u32, u32, vp, vp, vp, sz, u32, vp]
        L.sel_predict_gpu_cycles.argtypes = [vp, u64, T, vp, vp, vp, vp, vp]
        L.sel_select.argtypes = [vp, u64, vp, vp, vp, vp]
        L.sel_evaluate.argtypes = [vp, u64, T, vp, vp, vp, vp, vp, vp, sz, u32, vp]
        L.sel_evaluate_cpu_model.argtypes = [vp, u64, T, vp, vp, vp, vp, vp, vp, vp, vp, sz, u32, vp]
        L.sel_read_stats.argtypes = [vp, ctypes.POINTER(Stats), vp]
        L.sel_select_launch.argtypes = [vp, u64, vp, vp, u64, vp, vp, vp]
        L.sel_model_cpu_cost.argtypes = [vp, u64, T, vp, vp, vp, vp]
        L.sel_bind_accesses.argtypes = [vp, u64, vp, u64, vp, u64, vp, u64, vp, vp, vp]
        L.sel_profile_enable.argtypes = [ctypes.c_int]
        L.sel_profile_read.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_uint64)]
        L.sel_profile_read_region.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                              ctypes.POINTER(ctypes.c_uint64)]
        L.sel_kernel_launches.restype = u64
        L.sel_int_peak.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_double)]
        L.sel_selftest_ddiv.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        L.sel_last_error.restype = ctypes.c_char_p
        L.sel_version.restype = ctypes.c_char_p
        L.sel_sizeof.restype = sz
        L.sel_sizeof.argtypes = [ctypes.c_int]
        L.sel_offsetof.restype = sz
        L.sel_offsetof.argtypes = [ctypes.c_int, ctypes.c_int]
        for i, R in enumerate(RECORDS):
            if L.sel_sizeof(i) != ctypes.sizeof(R):
                raise ImportError(f"record {R.__name__}: libsel sizeof {L.sel_sizeof(i)} != {ctypes.sizeof(R)}")
        _lib = L
    return _lib


def check(rc: int):
    if rc != SEL_OK:
        raise SelError(rc, lib().sel_last_error().decode(errors="replace"))


EXPORTED = ("sel_load_device_params", "sel_workspace_size", "sel_count_transactions", "sel_count_transactions_part",
            "sel_predict_gpu_cycles", "sel_select", "sel_evaluate", "sel_evaluate_cpu_model", "sel_select_launch", "sel_model_cpu_cost", "sel_bind_accesses", "sel_read_stats",
            "sel_profile_enable", "sel_profile_read", "sel_profile_read_region", "sel_kernel_launches", "sel_int_peak", "sel_selftest_ddiv", "sel_last_error",
            "sel_version", "sel_sizeof", "sel_offsetof")
