"""CPU: the C-ABI library loads, exports every symbol include/sel.h declares,
and the three independent declarations of the record layouts (generator,
oracle, product) agree byte for byte.  No compute calls (no GPU here)."""
import ctypes
import os
import re

import numpy as np

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _sel():
    import __graft_entry__
    __graft_entry__.build_libsel()
    from paper_conf_ipps_chikinaat19_b200 import _lib
    return _lib


def test_header_symbols_exported():
    _lib = _sel()
    hdr = open(os.path.join(ROOT, "include", "sel.h")).read()
    declared = set(re.findall(r"^\s*(?:int|size_t|uint64_t|const char\*)\s+(sel_\w+)\s*\(", hdr, re.M))
    assert len(declared) >= 14
    L = ctypes.CDLL(_lib.LIB_PATH)
    for name in declared:
        assert hasattr(L, name), f"libsel.so does not export {name}"
    assert declared == set(_lib.EXPORTED)
    assert b"sm_100a" in _lib.lib().sel_version()


def _numpy_layout(dt):
    return dt.itemsize, [dt.fields[f][1] for f in dt.names if not f.startswith("_")]


def test_record_layouts_agree():
    _lib = _sel()
    L = _lib.lib()
    gen_dtypes = [gen.DEVICE_DTYPE, gen.ACCESS_DTYPE, gen.NEST_DTYPE, gen.LAUNCH_DTYPE, gen.CANDIDATE_DTYPE,
                  gen.COUNTS_DTYPE]
    for which, dt in enumerate(gen_dtypes):
        size, offs = _numpy_layout(dt)
        sel_offs = []
        f = 0
        while True:
            o = L.sel_offsetof(which, f)
            if o == ctypes.c_size_t(-1).value:
                break
            sel_offs.append(o)
            f += 1
        assert L.sel_sizeof(which) == size, which
        assert sel_offs == offs, (which, sel_offs, offs)
        R = _lib.RECORDS[which]
        assert ctypes.sizeof(R) == size
        assert [getattr(R, n).offset for n, _ in R._fields_ if not n.startswith("_")] == offs
        if which < 5:
            osize, ooffs = oracle.layout(which)
            assert osize == size and ooffs == offs, which


def test_workspace_size_monotone():
    _lib = _sel()
    L = _lib.lib()
    a = L.sel_workspace_size(1000, 10, 0)
    b = L.sel_workspace_size(2000, 10, 0)
    c = L.sel_workspace_size(1000, 10, 1)
    assert 0 < a < b and c < a
    # the c5 sweep (10^8 candidates) plans in an eighth of the 180 GB of HBM:
    # ~217 B per candidate, sized for the worst case of one problem per candidate
    # (per problem: counts 48 B, model inputs 128 B, W / WR / nest / B / status / used 26 B)
    assert L.sel_workspace_size(10 ** 8, 3125000, 0) < 23 * 10 ** 9


def test_product_does_not_import_oracle():
    """The product package never imports or links the oracle (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_chikinaat19_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", src, re.M), f
                assert "liboracle" not in src and "oracle_" not in src, f


def test_calls_fail_loudly_without_gpu():
    """No CUDA device here: loading params must report ENODEV, not fall back."""
    import torch
    if torch.cuda.is_available():
        return
    _lib = _sel()
    dev = gen.device_sets()
    rc = _lib.lib().sel_load_device_params(np.ascontiguousarray(dev).ctypes.data, 4)
    assert rc == _lib.SEL_ENODEV
