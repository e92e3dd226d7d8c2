"""CPU oracle binding -- TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_ipps_chikinaat19_b200`` never imports it and has no CPU
fallback.  See oracle.c for what is computed and which passages it follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SEL_ORACLE_LIB: load a prebuilt variant instead (scripts/mutate_oracle.py runs
# the pins against deliberately broken copies of oracle.c)
_LIB_PATH = os.environ.get("SEL_ORACLE_LIB") or os.path.join(_HERE, "liboracle.so")

RESULT_DTYPE = np.dtype([
    ("W", "<u8"), ("L", "<u8"), ("S", "<u8"), ("C", "<u8"), ("U", "<u8"), ("WR", "<u8"),
    ("G", "<u8"), ("T", "<u8"), ("R", "<u8"), ("wpb", "<u8"), ("abps", "<u8"),
    ("active_sms", "<u8"), ("M_it", "<u8"),
    ("N", "<f8"), ("Rep", "<f8"),
    ("comp", "<f8"), ("mem", "<f8"), ("MemL_u", "<f8"), ("MemL_c", "<f8"), ("MemL", "<f8"),
    ("Dep", "<f8"), ("MWPnb", "<f8"), ("BWpw", "<f8"), ("MWPbw", "<f8"), ("MWP", "<f8"),
    ("Comp", "<f8"), ("Mem", "<f8"), ("CWP", "<f8"), ("E", "<f8"),
    ("hk_case", "<i4"),
    ("cycles", "<f8"), ("t_gpu", "<f8"), ("t_cpu", "<f8"),
    ("decision", "u1"), ("status", "u1"), ("_pad", "u1", (6,)),
], align=True)

OK, EINVAL, ERANGE, ELAUNCH = 0, 1, 2, 3
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    hdr = os.path.join(_HERE, "oracle.h")
    if os.environ.get("SEL_ORACLE_LIB"):
        return _LIB_PATH
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
            os.path.getmtime(src), os.path.getmtime(hdr)):
        # -ffp-contract=off: no FMA contraction, so the fp64 model sequence
        # is evaluated exactly in the order written (R30).
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-ffp-contract=off",
                               "-fno-fast-math", "-fPIC", "-shared", "-pthread",
                               "-o", _LIB_PATH, src, "-lm"])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        vp, u64 = ctypes.c_void_p, ctypes.c_uint64
        L.oracle_geometry.argtypes = [u64, ctypes.c_uint32, ctypes.c_uint32, vp]
        L.oracle_evaluate.restype = ctypes.c_int
        L.oracle_evaluate.argtypes = [vp, ctypes.c_int, vp, u64, vp, u64, vp, u64, vp, u64, vp,
                                      ctypes.c_int]
        L.oracle_model.argtypes = [vp, vp, vp, vp, vp, vp]
        L.oracle_select_launch.argtypes = [vp, u64, vp, vp, u64, vp, vp]
        L.oracle_cpu_model.argtypes = [vp, vp, u64, vp, vp, u64, vp, vp]
        L.oracle_bind.argtypes = [vp, u64, vp, u64, vp, u64, vp, u64, vp, vp]
        L.oracle_sizeof.restype = ctypes.c_size_t
        L.oracle_sizeof.argtypes = [ctypes.c_int]
        L.oracle_offsetof.restype = ctypes.c_size_t
        L.oracle_offsetof.argtypes = [ctypes.c_int, ctypes.c_int]
        assert L.oracle_sizeof(5) == RESULT_DTYPE.itemsize, "or_result layout mismatch"
        _lib = L
    return _lib


def geometry(P: int, B: int, grid_max: int):
    """(G, T, #OMP_Rep, warps per block) -- P:L225, readings R6/R27."""
    out = np.zeros(4, np.uint64)
    lib().oracle_geometry(P, B, grid_max, out.ctypes.data)
    return tuple(int(x) for x in out)


def evaluate(batch, threads: int = 0) -> np.ndarray:
    """Evaluate every candidate of a ``gen.Batch``; returns RESULT_DTYPE records."""
    n = len(batch.cands)
    out = np.zeros(n, RESULT_DTYPE)
    if n == 0:
        return out
    c = np.ascontiguousarray(batch.cands)
    ne = np.ascontiguousarray(batch.nests)
    ac = np.ascontiguousarray(batch.accesses)
    la = np.ascontiguousarray(batch.launches)
    dv = np.ascontiguousarray(batch.devices)
    rc = lib().oracle_evaluate(dv.ctypes.data, len(dv), c.ctypes.data, n, ne.ctypes.data, len(ne),
                               ac.ctypes.data, len(ac), la.ctypes.data, len(la), out.ctypes.data,
                               threads)
    if rc != 0:
        raise ValueError("oracle_evaluate rejected its arguments")
    return out


def model(device, nest, accesses, launch, cand, W, L, S, C, U, WR) -> np.void:
    """a4-a7 only, for hand-made counts (pins of the Hong & Kim arithmetic)."""
    r = np.zeros(1, RESULT_DTYPE)
    r["W"], r["L"], r["S"], r["C"], r["U"], r["WR"] = W, L, S, C, U, WR
    dv = np.array([device]).copy()
    ne = np.array([nest]).copy()
    ac = np.ascontiguousarray(np.asarray(accesses)).copy() if len(accesses) else np.zeros(1, accesses.dtype)
    la = np.array([launch]).copy()
    cd = np.array([cand]).copy()
    lib().oracle_model(dv.ctypes.data, ne.ctypes.data, ac.ctypes.data, la.ctypes.data,
                       cd.ctypes.data, r.ctypes.data)
    return r[0]


def select_launch(group_of, t_gpu, status, n_groups):
    """NEXT row f3: per-group argmin of t_gpu (see oracle.c)."""
    g = np.ascontiguousarray(group_of, dtype=np.uint32)
    t = np.ascontiguousarray(t_gpu, dtype=np.float64)
    s = np.ascontiguousarray(status, dtype=np.uint8)
    best = np.zeros(n_groups, np.uint32)
    val = np.zeros(n_groups, np.float64)
    lib().oracle_select_launch(g.ctypes.data, len(g), t.ctypes.data, s.ctypes.data, n_groups, best.ctypes.data,
                               val.ctypes.data)
    return best, val


def cpu_model(params, batch, cpu_in):
    """NEXT row f1: (cpu_cycles f64[n], status u8[n]) -- Liao-Chapman Fig. 3 with Table II."""
    n = len(batch.cands)
    cyc = np.zeros(n, np.float64)
    st = np.zeros(n, np.uint8)
    p = np.ascontiguousarray(params)
    ne = np.ascontiguousarray(batch.nests)
    c = np.ascontiguousarray(batch.cands)
    ci = np.ascontiguousarray(cpu_in)
    lib().oracle_cpu_model(p.ctypes.data, ne.ctypes.data, len(ne), c.ctypes.data, ci.ctypes.data, n,
                           cyc.ctypes.data, st.ctypes.data)
    return cyc, st


def bind(sym, terms, values, items):
    """NEXT row f2: (concrete accesses as raw 64-byte records, status u8[n])."""
    n = len(items)
    out = np.zeros(max(n, 1) * 64, np.uint8)
    st = np.zeros(max(n, 1), np.uint8)
    s = np.ascontiguousarray(sym)
    t = np.ascontiguousarray(terms)
    v = np.ascontiguousarray(values, dtype=np.int64)
    it = np.ascontiguousarray(items)
    lib().oracle_bind(s.ctypes.data, len(s), t.ctypes.data, len(t), v.ctypes.data, len(v), it.ctypes.data, n,
                      out.ctypes.data, st.ctypes.data)
    return out[: n * 64], st[:n]


def layout(which: int):
    """(sizeof, [field offsets]) of oracle record ``which`` (0 device .. 4 candidate)."""
    L = lib()
    offs = []
    f = 0
    while True:
        o = L.oracle_offsetof(which, f)
        if o == ctypes.c_size_t(-1).value:
            break
        offs.append(int(o))
        f += 1
    return int(L.oracle_sizeof(which)), offs
