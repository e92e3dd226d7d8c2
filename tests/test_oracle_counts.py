"""Pins of the oracle's counting part (a1-a4) against things other than itself:
closed forms, the paper's worked examples, an independent pure-Python brute
force, and invariants.  CPU only."""
import json
import os
import random

import numpy as np
import pytest

import gen
import oracle
import bruteforce

HERE = os.path.dirname(os.path.abspath(__file__))
BASE = 1 << 28


def one_access_batch(specs):
    """specs: list of (P, B, grid_max, access-kwargs, trip) -> Batch with one
    candidate per spec, each on its own launch."""
    launches = np.zeros(len(specs), gen.LAUNCH_DTYPE)
    items = []
    for i, (P, B, gmax, akw, trip) in enumerate(specs):
        launches[i] = (B, gmax, 0, 0)
        items.append(dict(P0=P, trip=trip, depth=len(trip), comp=[1.0] * (len(trip) + 1),
                          accesses=[gen.make_access(**akw)], launch=i))
    return gen.custom_batch(items, launches_=launches)


# ----------------------------------------------------------- closed forms
def lines_closed(o, sb, n, gran):
    """distinct gran-byte blocks touched by n lanes at o, o+sb, ... (sb >= 0)."""
    if sb >= gran:
        return n
    return (o + (n - 1) * sb) // gran - o // gran + 1


@pytest.mark.parametrize("b", [1, 2, 4, 8, 16])
def test_full_warp_stride_offset_closed_form(b):
    """One full warp (P = 32), stride s elements of b bytes, base offset o:
    lines = 32 if s*b >= 128 else floor((o+31sb)/128) - floor(o/128) + 1,
    and the same with 32 for sectors (SURVEY §8(c) pins)."""
    specs, expect = [], []
    for s in range(1, 65):
        for o in range(0, 128, b):
            specs.append((32, 256, 65535, dict(base=BASE + o, c_par=(s * b,), elem_bytes=b), []))
            expect.append((lines_closed(o, s * b, 32, 128), lines_closed(o, s * b, 32, 32)))
    r = oracle.evaluate(one_access_batch(specs))
    assert (r["status"] == 0).all()
    assert (r["W"] == 1).all() and (r["WR"] == 1).all()
    np.testing.assert_array_equal(r["L"], [e[0] for e in expect])
    np.testing.assert_array_equal(r["S"], [e[1] for e in expect])
    tmin = -(-32 * b // 128)
    coal = np.array([e[0] <= tmin for e in expect])
    np.testing.assert_array_equal(r["C"], coal.astype(np.uint64))
    np.testing.assert_array_equal(r["U"], np.where(coal, 0, [e[0] for e in expect]))


@pytest.mark.parametrize("b", [4, 8])
def test_north_star_stride_formula_aligned(b):
    """North star / IPDA example (A[max*a] has inter-thread stride
    [max]): aligned base, stride s elements -> min(32, ceil(32*s*b/128))
    lines per full warp.  Exact for b in {4, 8}; a unit-stride 4 B access
    touches exactly one 128 B line."""
    specs = [(32, 256, 65535, dict(base=BASE, c_par=(s * b,), elem_bytes=b), []) for s in range(1, 65)]
    r = oracle.evaluate(one_access_batch(specs))
    expect = [min(32, -(-32 * s * b // 128)) for s in range(1, 65)]
    np.testing.assert_array_equal(r["L"], expect)
    if b == 4:
        assert r["L"][0] == 1 and r["S"][0] == 4 and r["C"][0] == 1


def test_partial_warps_and_negative_stride_closed_form():
    """Partial warps (n < 32 active lanes) and negative strides: the lane
    address set of stride -s starting at o + (n-1)sb equals that of +s
    starting at o, so the counts agree with the closed form."""
    rnd = random.Random(7)
    specs, expect = [], []
    for _ in range(600):
        b = rnd.choice([1, 2, 4, 8, 16])
        s = rnd.randint(0, 70)
        n = rnd.randint(1, 32)
        o = b * rnd.randrange(128 // b)
        neg = rnd.random() < 0.5
        sb = s * b
        if neg:
            akw = dict(base=BASE + o + (n - 1) * sb, c_par=(-sb,), elem_bytes=b)
        else:
            akw = dict(base=BASE + o, c_par=(sb,), elem_bytes=b)
        specs.append((n, 256, 65535, akw, []))
        expect.append((lines_closed(o, sb, n, 128), lines_closed(o, sb, n, 32)))
    r = oracle.evaluate(one_access_batch(specs))
    np.testing.assert_array_equal(r["L"], [e[0] for e in expect])
    np.testing.assert_array_equal(r["S"], [e[1] for e in expect])


def test_omp_rep_worked_example():
    """1024 iterations on 1 block of 128 threads -> #OMP_Rep = 8."""
    G, T, R, wpb = oracle.geometry(1024, 128, 1)
    assert (G, T, R, wpb) == (1, 128, 8, 4)
    # R6 cap by the maximum grid and the ceil of R27
    assert oracle.geometry(2 ** 24, 64, 65535) == (65535, 65535 * 64, 5, 2)
    assert oracle.geometry(1025, 128, 1)[2] == 9


def test_c1_gemm_worked_counts():
    """Worked config c1 (tests/golden/c1_gemm64.json, hand-derived)."""
    with open(os.path.join(HERE, "golden", "c1_gemm64.json")) as f:
        gold = json.load(f)
    r = oracle.evaluate(gen.generate(1))
    for i, key in enumerate(["gemm64_1d", "gemm64_collapse2"]):
        for f_ in ["W", "L", "S", "C", "U", "WR"]:
            assert int(r[f_][i]) == gold[key][f_], (key, f_)


def test_unknown_trip_defaults_to_128():
    """loops with unknown trip count are assumed to run 128 times."""
    a = gen.make_access(base=BASE, c_par=(4,), c_inner=(4,), elem_bytes=4, depth=1)
    b1 = gen.custom_batch([dict(P0=32, trip=[gen.TRIP_UNKNOWN], accesses=[a], comp=[1, 1])])
    b2 = gen.custom_batch([dict(P0=32, trip=[128], accesses=[a], comp=[1, 1])])
    r1, r2 = oracle.evaluate(b1), oracle.evaluate(b2)
    assert r1["W"][0] == 128
    for f in ["W", "L", "S", "C", "U", "WR", "cycles"]:
        assert r1[f][0] == r2[f][0]


# ----------------------------------------------------------- brute force
def random_nest(rnd):
    par_dims = rnd.choice([1, 1, 2])
    if par_dims == 1:
        P0, P1 = rnd.randint(0, 96), 1
    else:
        P0, P1 = rnd.randint(0, 9), rnd.randint(1, 11)
    depth = rnd.randint(0, 2)
    trip = [rnd.randint(0, 4) for _ in range(depth)]
    acc = []
    for _ in range(rnd.randint(0, 3)):
        e = rnd.choice([1, 2, 4, 8, 16])
        d = rnd.randint(0, depth)

        def coef():
            return e * rnd.choice([0, 1, -1, 2, 3, -5, 8, 16, 31, 33, 64, -64, 130, 1000])
        acc.append(dict(base=BASE + e * rnd.randint(-64, 64), c_par=[coef(), coef() if par_dims == 2 else 0],
                        c_inner=[coef() for _ in range(d)] + [0] * (3 - d), elem=e, depth=d))
    B = rnd.choice([1, 7, 32, 33, 48, 64, 96, 128])
    gmax = rnd.choice([1, 2, 3, 65535])
    return dict(P0=P0, P1=P1, par_dims=par_dims, trip=trip, acc=acc, B=B, gmax=gmax)


def test_oracle_matches_python_bruteforce():
    rnd = random.Random(2019)
    nests = [random_nest(rnd) for _ in range(250)]
    launches = np.zeros(len(nests), gen.LAUNCH_DTYPE)
    items = []
    for i, n in enumerate(nests):
        launches[i] = (n["B"], n["gmax"], 0, 0)
        items.append(dict(P0=n["P0"], P1=n["P1"], par_dims=n["par_dims"], trip=n["trip"], depth=len(n["trip"]),
                          comp=[1.0] * 4, launch=i,
                          accesses=[gen.make_access(base=a["base"], c_par=a["c_par"], c_inner=a["c_inner"],
                                                    elem_bytes=a["elem"], depth=a["depth"]) for a in n["acc"]]))
    r = oracle.evaluate(gen.custom_batch(items, launches_=launches))
    for i, n in enumerate(nests):
        exp = bruteforce.counts(n["P0"], n["P1"], n["par_dims"], n["trip"], n["acc"], n["B"], n["gmax"])
        got = tuple(int(r[f][i]) for f in ["W", "L", "S", "C", "U", "WR"])
        assert r["status"][i] == 0
        assert got == exp, (i, n, got, exp)


# ----------------------------------------------------------- invariants
def test_count_invariants_on_c3_slice():
    """Aggregated per-WA invariants: 1 <= lines <= 32, lines <= sectors <=
    4 lines, W = WR * M_it, U >= 2 (W - C) when tmin = 1."""
    b = gen.generate(3, 0, 4000)
    r = oracle.evaluate(b)
    assert (r["status"] == 0).all()
    W, L, S, C, U, WR = (r[f].astype(np.int64) for f in ["W", "L", "S", "C", "U", "WR"])
    assert (L >= W).all() and (L <= 32 * W).all()
    assert (S >= L).all() and (S <= 4 * L).all()
    assert (W == WR * r["M_it"].astype(np.int64)).all()
    elem = b.accesses["elem_bytes"][b.nests["access_off"][b.cands["nest_id"]]]
    t1 = elem <= 4
    assert (U[t1] >= 2 * (W - C)[t1]).all()
    assert (U <= 32 * (W - C)).all()


def test_lines_monotone_in_stride_and_base_shift():
    specs = []
    for o in (0, 4, 60, 124):
        for s in range(1, 40):
            specs.append((32, 256, 65535, dict(base=BASE + o, c_par=(4 * s,), elem_bytes=4), []))
            specs.append((32, 256, 65535, dict(base=BASE + o + 128 * 1000, c_par=(4 * s,), elem_bytes=4), []))
    r = oracle.evaluate(one_access_batch(specs))
    L = r["L"].reshape(4, 39, 2)
    np.testing.assert_array_equal(L[:, :, 0], L[:, :, 1])      # base += 128k invariance
    assert (np.diff(L[:, :, 0].astype(int), axis=1) >= 0).all()  # non-decreasing in s


def test_counts_independent_of_device_and_gridmax():
    """Counts do not depend on the device set or G_max, nor on B when 32 | B
    (SURVEY §8(d) dedup note) -- the property the GPU path's count sharing
    relies on, checked here on the oracle (c2 nests, several launches)."""
    c2 = gen.generate(2)
    launches = np.zeros(9, gen.LAUNCH_DTYPE)
    for i, (B, g) in enumerate([(32, 65535), (64, 1), (128, 3), (256, 65535), (1024, 2),
                                (96, 7), (48, 65535), (48, 1), (48, 5)]):
        launches[i] = (B, g, 0, 0)
    rows = []
    for nest in range(0, 27, 3):
        for li in range(9):
            for dev in range(4):
                rows.append((nest, li, dev))
    cands = np.zeros(len(rows), gen.CANDIDATE_DTYPE)
    for i, (nest, li, dev) in enumerate(rows):
        cands[i] = (nest, li, dev, 1e6, 3e9)
    r = oracle.evaluate(gen.Batch(cands, c2.nests, c2.accesses, launches, c2.devices))
    assert (r["status"] == 0).all()
    key = np.array([f"{n}-{'x' if launches[li]['block'] % 32 == 0 else launches[li]['block']}" for n, li, _ in rows])
    for k in np.unique(key):
        sel = key == k
        for f in ["W", "L", "S", "C", "U", "WR"]:
            assert len(np.unique(r[f][sel])) == 1, (k, f)
