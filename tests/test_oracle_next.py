"""Pins of the oracle's NEXT rows against independent
numpy formulations.  CPU only."""
import numpy as np

import oracle


def test_select_launch_matches_numpy_argmin():
    rng = np.random.default_rng(3)
    n, G = 5000, 700
    group = rng.integers(0, G + 20, n).astype(np.uint32)          # some out-of-range groups
    t = rng.choice([0.5, 1.0, 2.0, np.inf], n) * rng.integers(1, 4, n)
    st = (rng.random(n) < 0.1).astype(np.uint8)
    best, val = oracle.select_launch(group, t, st, G)
    for g in range(G):
        idx = np.nonzero((group == g) & (st == 0))[0]
        if len(idx) == 0:
            assert best[g] == 0xFFFFFFFF and np.isinf(val[g])
            continue
        m = t[idx].min()
        first = idx[np.nonzero(t[idx] == m)[0][0]]                # ties: lowest index
        assert best[g] == first and val[g] == m


# ---------------------------------------------------------------- f1 (CPU model)
import gen  # noqa: E402


def _one_nest(P, bytes_total=0):
    n = np.zeros(1, gen.NEST_DTYPE)
    n["P0"], n["P1"], n["par_dims"] = P, 1, 1
    n["bytes_h2d"] = bytes_total
    c = np.zeros(1, gen.CANDIDATE_DTYPE)
    return gen.Batch(c, n, np.zeros(1, gen.ACCESS_DTYPE), gen.launches(1), gen.device_sets())


def _cin(mca, threads):
    x = np.zeros(1, gen.CPU_INPUT_DTYPE)
    x["mca_cycles_per_iter"], x["threads"] = mca, threads
    return x


def test_cpu_model_hand_values():
    """Fig. 3 with Table II: Par_Startup 3000 + static schedule
    10154 + Chunk x (Machine x per_iter + loop overhead 4) + sync 4000."""
    p = gen.cpu_params()
    cyc, st = oracle.cpu_model(p, _one_nest(1000), _cin(10.0, 160))
    assert st[0] == 0 and cyc[0] == 3000 + 10154 + 7 * (10 + 4) + 4000
    cyc, _ = oracle.cpu_model(p, _one_nest(1000), _cin(10.0, 1))            # one thread: chunk = P
    assert cyc[0] == 17154 + 1000 * 14
    cyc, _ = oracle.cpu_model(p, _one_nest(50), _cin(10.0, 160))            # more threads than iterations
    assert cyc[0] == 17154 + 1 * 14


def test_cpu_model_tlb_term():
    """TLB term (F1c): misses = pages of the thread's share beyond the 1024
    entries, 14 cycles each (Table II)."""
    p = gen.cpu_params()
    page = 65536
    for extra in (0, 1, 10, 1000):
        cyc, _ = oracle.cpu_model(p, _one_nest(160, (1024 + extra) * page * 4), _cin(1.0, 4))
        assert cyc[0] == 17154 + 40 * (1 + 4) + 14 * extra
    cyc, _ = oracle.cpu_model(p, _one_nest(160, 1024 * page * 4 - 1), _cin(1.0, 4))
    assert cyc[0] == 17154 + 40 * 5


def test_cpu_model_matches_supplied_synthetic_cost():
    """Without TLB misses the modelled cost equals the synthetic cost the
    generator supplies (same Fig. 3 form, written independently in gen/)."""
    p = gen.cpu_params()
    for cfg, rng in ((1, (0, 2)), (2, (0, 108)), (3, (0, 20000)), (5, (1234567, 1334567))):
        b = gen.generate(cfg, *rng)
        cyc, st = oracle.cpu_model(p, b, gen.cpu_inputs(cfg, *rng))
        assert (st == 0).all()
        np.testing.assert_array_equal(cyc, b.cands["cpu_cycles"])


def test_cpu_model_monotone_and_invalid():
    p = gen.cpu_params()
    prev = 0
    for mca in (0.0, 0.5, 1.0, 7.0, 100.0):
        cyc, _ = oracle.cpu_model(p, _one_nest(777), _cin(mca, 8))
        assert cyc[0] > prev
        prev = cyc[0]
    for bad in (_cin(1.0, 0), _cin(-1.0, 4), _cin(float("nan"), 4), _cin(float("inf"), 4)):
        _, st = oracle.cpu_model(p, _one_nest(10), bad)
        assert st[0] == oracle.EINVAL


# ---------------------------------------------------------------- f4 (H&K synchronisation)
def _with_sync(b, k):
    n = b.nests.copy()
    n["n_sync"] = k
    return gen.Batch(b.cands, n, b.accesses, b.launches, b.devices)


def test_sync_term_linear_and_zero_cases():
    """[H&K] synchronisation cost Departure_delay x (MWP-1) x #synch x
    #Active_blocks x #Rep (x #OMP_Rep, F4a): zero without barriers, linear in
    the barrier count, zero when a single warp runs (MWP = 1)."""
    b = gen.generate(2)
    r0 = oracle.evaluate(b)
    r1 = oracle.evaluate(_with_sync(b, 1))
    r2 = oracle.evaluate(_with_sync(b, 2))
    s1, s2 = r1["cycles"] - r0["cycles"], r2["cycles"] - r0["cycles"]
    assert (s1 >= 0).all() and (s1 > 0).any()
    np.testing.assert_allclose(s2, 2 * s1, rtol=1e-9)
    m = r0["W"] > 0
    expect = r0["Dep"] * (r0["MWP"] - 1.0) * r0["abps"].astype(float) * r0["Rep"] * r0["R"].astype(float)
    np.testing.assert_allclose(s1[m], expect[m], rtol=1e-9)
    np.testing.assert_array_equal(r1["hk_case"], r0["hk_case"])
    # lone warp: MWP = N = 1 -> no synchronisation cost
    a = gen.make_access(base=1 << 28, c_par=(4,), c_inner=(0,), elem_bytes=4, depth=1)
    lau = np.zeros(1, gen.LAUNCH_DTYPE)
    lau[0] = (32, 1, 0, 0)
    one = gen.custom_batch([dict(P0=64, trip=[5], comp=[1.0, 2.0], accesses=[a])], launches_=lau)
    assert oracle.evaluate(_with_sync(one, 3))["cycles"][0] == oracle.evaluate(one)["cycles"][0]


# ---------------------------------------------------------------- f2 (symbolic IPDA binding)
def _sym_one(terms_per_slot, elem_sym=0, elem_bytes=0, depth=0):
    """one symbolic access; terms_per_slot: 6 lists of (k, syms)."""
    sym = np.zeros(1, gen.SYM_ACCESS_DTYPE)
    terms = []
    for slot, tl in enumerate(terms_per_slot):
        sym["term_off"][0][slot] = len(terms)
        sym["n_terms"][0][slot] = len(tl)
        for k, ss in tl:
            ss = list(ss) + [gen.SYM_ONE] * (3 - len(ss))
            terms.append((k, ss, 0))
    sym["elem_sym"], sym["elem_bytes"], sym["depth"] = elem_sym, elem_bytes, depth
    t = np.zeros(max(len(terms), 1), gen.SYM_TERM_DTYPE)
    for i, (k, ss, _) in enumerate(terms):
        t[i]["k"], t[i]["sym"] = k, ss
    return sym, t


def test_bind_ipda_worked_example():
    """A[max*a] in a parallel loop over a has inter-thread stride
    [max] (x 4-byte elements); binding max at runtime gives the concrete
    access, whose full warp touches min(32, ceil(32*max*4/128)) lines."""
    sym, terms = _sym_one([[(1 << 28, [])], [(1, [0, 1])], [], [], [], []])   # frame: v0 = elem, v1 = max
    items = np.zeros(6, gen.BIND_ITEM_DTYPE)
    vals = []
    for i, mx in enumerate([1, 2, 7, 31, 32, 100]):
        items[i]["frame"] = len(vals)
        vals += [4, mx]
    out, st = oracle.bind(sym, terms, np.array(vals), items)
    acc = out.view(gen.ACCESS_DTYPE)
    assert (st == 0).all()
    assert list(acc["c_par"][:, 0]) == [4, 8, 28, 124, 128, 400]
    lau = np.zeros(1, gen.LAUNCH_DTYPE)
    lau[0] = (256, 65535, 0, 0)
    b = gen.custom_batch([dict(P0=32, trip=[], accesses=[a]) for a in acc], launches_=lau)
    r = oracle.evaluate(b)
    assert list(r["L"]) == [min(32, -(-32 * m * 4 // 128)) for m in [1, 2, 7, 31, 32, 100]]


def test_bind_reproduces_generator_accesses():
    """The symbolic table bound with each nest's frame gives back, byte for
    byte, the concrete accesses the generator writes directly (c2, c5)."""
    sym, terms = gen.sym_tables()
    for cfg, rng in ((2, (0, 108)), (5, (0, 200000)), (5, (77000000, 77200000))):
        b = gen.generate(cfg, *rng)
        vals, items = gen.sym_instances(cfg, *rng)
        out, st = oracle.bind(sym, terms, vals, items)
        assert (st == 0).all()
        assert np.array_equal(out, np.ascontiguousarray(b.accesses[:len(items)]).view(np.uint8).reshape(-1))


def test_bind_errors():
    sym, terms = _sym_one([[(1 << 40, [0])], [(1, [1])], [], [], [], []])
    items = np.zeros(5, gen.BIND_ITEM_DTYPE)
    items[0]["frame"] = 0      # ok
    items[1]["frame"] = 2      # v[2] * 2^40 overflows 2^62
    items[2]["frame"] = 4      # elem 3 -> EINVAL
    items[3]["frame"] = 100    # frame out of range -> EINVAL
    items[4]["sym_access"] = 9  # bad symbolic access
    vals = np.array([4, 8, 1 << 23, 8, 3, 8])
    out, st = oracle.bind(sym, terms, vals, items)
    assert list(st) == [0, 2, 1, 1, 1]
    acc = out.view(gen.ACCESS_DTYPE)
    assert acc["base"][0] == 4 << 40 and acc["c_par"][0, 0] == 8 and acc["elem_bytes"][0] == 4
    assert (out.reshape(5, 64)[1:] == 0).all()
