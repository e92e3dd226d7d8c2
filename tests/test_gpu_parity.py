"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bit-exact counts, statuses and decisions; fp64 cycles
within 1e-6 relative (BASELINE.json north_star) -- in practice bit-exact,
which is also asserted for the fused path (R30)."""
import random

import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu

FIELDS = ["W", "L", "S", "C", "U", "WR"]
REL_TOL = 1e-6


@pytest.fixture(scope="module")
def sel():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_chikinaat19_b200 as s
    assert torch.cuda.is_available()
    return s


def run_gpu(sel, b, flags=0, api="fused"):
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), max(len(b), 1), flags)
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    if api == "fused":
        r = ev.evaluate(cands, want_counts=True, want_t_gpu=True)
    else:
        counts, status = sel.count_transactions(cands, ev.tables, ev.workspace, flags)
        cycles, t_gpu = sel.predict_gpu_cycles(cands, ev.tables, counts, status)
        decision = sel.select(cands, t_gpu, status)
        r = dict(counts=counts, status=status, cycles=cycles, t_gpu=t_gpu, decision=decision)
    torch.cuda.synchronize()
    out = {k: v.cpu().numpy() for k, v in r.items()}
    out["counts"] = out["counts"].astype(np.uint64)
    out["stats"] = sel.read_stats(ev.workspace) if api == "fused" else None
    return out


def assert_parity(g, ref, exact_cycles=True, ctx=""):
    for j, f in enumerate(FIELDS):
        bad = np.nonzero(g["counts"][:, j] != ref[f])[0]
        assert len(bad) == 0, f"{ctx}: count {f} differs at {bad[:10]}: gpu {g['counts'][bad[:5], j]} oracle {ref[f][bad[:5]]}"
    bad = np.nonzero(g["status"] != ref["status"])[0]
    assert len(bad) == 0, f"{ctx}: status differs at {bad[:10]}: {g['status'][bad[:5]]} vs {ref['status'][bad[:5]]}"
    bad = np.nonzero(g["decision"] != ref["decision"])[0]
    assert len(bad) == 0, f"{ctx}: decision differs at {bad[:10]}"
    rel = np.abs(g["cycles"] - ref["cycles"]) / np.maximum(np.abs(ref["cycles"]), 1e-300)
    assert (rel <= REL_TOL).all(), f"{ctx}: cycles rel err {rel.max()}"
    if exact_cycles:
        assert (g["cycles"] == ref["cycles"]).all(), f"{ctx}: cycles not bit-exact (max rel {rel.max()})"
        same = (g["t_gpu"] == ref["t_gpu"]) | (np.isinf(g["t_gpu"]) & np.isinf(ref["t_gpu"]))
        assert same.all(), f"{ctx}: t_gpu not bit-exact"


@pytest.mark.parametrize("flags", [0, 1, 2, 3, 4, 5, 8, 12])
def test_c1_gemm(sel, flags):
    b = gen.generate(1)
    g = run_gpu(sel, b, flags)
    assert_parity(g, oracle.evaluate(b), ctx=f"c1 flags={flags}")
    assert g["counts"][0].tolist() == [24576, 532480, 532480, 8192, 524288, 2]


@pytest.mark.parametrize("flags", [0, 2, 4, 8])
def test_c2_polybench_medium(sel, flags):
    b = gen.generate(2)
    g = run_gpu(sel, b, flags)
    ref = oracle.evaluate(b)
    assert_parity(g, ref, ctx="c2")
    st = g["stats"]
    assert st["n_candidates"] == 108 and st["n_problems"] == 27      # 4 device sets share counts
    assert st["wa_resolved"] * 4 == st["wa_covered"] == int(ref["W"].sum())


def test_c2_split_api_matches_fused(sel):
    b = gen.generate(2)
    f = run_gpu(sel, b)
    s = run_gpu(sel, b, api="split")
    for k in ("counts", "status", "decision", "cycles", "t_gpu"):
        assert np.array_equal(f[k], s[k]), k


def test_c3_stride_offset_sweep(sel):
    b = gen.generate(3)
    g = run_gpu(sel, b)
    ref = oracle.evaluate(b)
    assert_parity(g, ref, ctx="c3")
    # one-warp candidates (P = 32) against the closed form directly
    acc = b.accesses[b.nests["access_off"]]
    sb = np.abs(acc["c_par"][:, 0])
    P = b.nests["P0"].astype(np.int64)
    first = np.where(acc["c_par"][:, 0] < 0, acc["base"] + acc["c_par"][:, 0] * (P - 1), acc["base"])
    o = first % 128
    closed = np.where(sb >= 128, 32, (o + 31 * sb) // 128 - o // 128 + 1)
    one = P == 32
    assert one.sum() > 100
    assert (g["counts"][one, 1].astype(np.int64) == closed[one]).all()


def test_c4_reduced_parallel_extent(sel):
    """c4's 24 shapes x 8 launches (B = 48, 128, 200, 1024) with the parallel
    extent reduced to 2^14 so the oracle finishes in seconds."""
    b = gen.generate(4)
    nests = b.nests.copy()
    nests["P0"] = 1 << 14
    bb = gen.Batch(b.cands, nests, b.accesses, b.launches, b.devices)
    ref = oracle.evaluate(bb)
    for flags in (0, 1, 4, 8):
        assert_parity(run_gpu(sel, bb, flags), ref, ctx=f"c4-reduced flags={flags}")


def test_c4_full_size_sampled(sel):
    """Full c4 (P = 2^24) in the bench configuration; the oracle recomputes a
    sample of candidates one by one (cheapest shapes, all 8 launches)."""
    b = gen.generate(4)
    g = run_gpu(sel, b)
    names = gen.shape_names()
    pick = [s * 8 + l for s in (names.index("mvt.1"), names.index("cov.reduce")) for l in range(8)]
    ref = oracle.evaluate(b.select(pick))
    sub = {k: (v[pick] if isinstance(v, np.ndarray) else v) for k, v in g.items()}
    assert_parity(sub, ref, ctx="c4 full sampled")
    assert (g["status"] == 0).all()


@pytest.mark.slow
def test_c4_full_size_all(sel):
    """All of c4 at full size (P = 2^24, 192 candidates, 4e9 warp-accesses) in
    the bench configuration against the oracle's full brute-force expansion
    (about 30 s on the box's host cores): the big-problem chunking of k_count
    (WR = 2^19 > 1024) on every shape and launch."""
    b = gen.generate(4)
    g = run_gpu(sel, b)
    ref = oracle.evaluate(b)
    assert_parity(g, ref, ctx="c4 full")
    assert (g["status"] == 0).all() and int(ref["W"].sum()) > 3 * 10 ** 9


def _nests_with_candidates(nest_items, launches, rows, devices=None):
    """A batch whose candidates (nest, launch, device) share the given nests
    (gen.custom_batch makes one nest per item)."""
    base = gen.custom_batch(nest_items, devices=devices, launches_=launches)
    cands = np.zeros(len(rows), gen.CANDIDATE_DTYPE)
    for i, (nest, li, dev) in enumerate(rows):
        cands[i] = (nest, li, dev, 10 ** (3 + (i % 5)), 3e9)
    return gen.Batch(cands, base.nests, base.accesses, launches, base.devices)


def test_lane_multi_group_direct(sel):
    """direct problem ids with more block-size classes
    than the lane kernel counts in one pass (kLaneGrp), so its multi-group
    loop (g0 = 3, 6, ...) rebuilds histograms and hands accesses to k_queue
    per group -- with 1-2 byte elements and depth 3 (handed over) and a nest
    of 35 accesses (the bit-31 "all remaining accesses" path)."""
    rnd = random.Random(31)
    Bs = [33, 40, 48, 72, 100, 200, 300, 64]            # 7 classes that 32 does not divide + the class 32
    launches = np.zeros(len(Bs), gen.LAUNCH_DTYPE)
    for i, B in enumerate(Bs):
        launches[i] = (B, 65535 if i % 3 else 4, 0, 0)
    nests = []
    for k in range(6):
        depth = [1, 2, 3, 1, 2, 0][k]
        trip = [rnd.randint(3, 40) for _ in range(depth)]
        n_acc = 35 if k == 3 else rnd.randint(2, 6)
        acc = []
        for j in range(n_acc):
            e = rnd.choice([1, 2, 4, 4, 8, 8, 16])
            d = rnd.randint(0, depth)
            acc.append(gen.make_access(base=(1 << 30) + e * rnd.randint(0, 500) + 4096 * j,
                                       c_par=[e * rnd.choice([0, 1, 2, 3, -1, 8, 33, 64])],
                                       c_inner=[e * rnd.choice([0, 1, 5, 64, 1000]) for _ in range(d)],
                                       elem_bytes=e, depth=d))
        nests.append(dict(P0=rnd.choice([95, 333, 1000, 3000]), trip=trip, depth=depth, comp=[1.0] * (depth + 1),
                          accesses=acc))
    rows = [(nest, li, dev) for nest in range(len(nests)) for li in range(len(Bs)) for dev in (0, 2, 3)]
    b = _nests_with_candidates(nests, launches, rows)
    assert len(b.nests) * 8 <= len(b)                    # direct ids
    ref = oracle.evaluate(b)
    assert (ref["status"] == 0).all()
    for flags in (0, 4, 16):
        g = run_gpu(sel, b, flags)
        assert_parity(g, ref, ctx=f"multi-group flags={flags}")
        assert g["stats"]["n_problems"] == len(b.nests) * 8


def test_direct_big_problems_referenced_or_not(sel):
    """Direct ids with big problems (WR > 1024, counted through the warp-access
    prefix): the ones a candidate refers to are counted exactly, a big nest
    no candidate refers to is dropped from the prefix (k_mark_big /
    k_drop_unused) and costs nothing."""
    a = gen.make_access(base=1 << 30, c_par=(8,), c_inner=(8,), elem_bytes=8, depth=1)
    big = dict(P0=1 << 17, trip=[5], comp=[1.0, 1.0], accesses=[a])
    huge = dict(P0=1 << 30, trip=[1 << 10], comp=[1.0, 1.0], accesses=[a])     # 2^35 WAs if counted
    small = dict(P0=300, trip=[7], comp=[1.0, 1.0], accesses=[a])
    launches = np.zeros(2, gen.LAUNCH_DTYPE)
    launches[0] = (128, 65535, 0, 0)
    launches[1] = (200, 160, 0, 0)
    rows = [(nest, li, dev) for nest in (0, 1) for li in (0, 1) for dev in (0, 1, 2, 3)]
    b = _nests_with_candidates([small, big, huge], launches, rows)
    ref = oracle.evaluate(b)
    g = run_gpu(sel, b)
    assert_parity(g, ref, ctx="direct big")
    assert g["stats"]["n_problems"] == 4                  # nests 0, 1 x 2 classes; nest 2 dropped
    assert g["stats"]["wa_resolved"] < 10 ** 8


def _granular_devices(seed):
    """Device sets with NEXT row f4's fields varied: allocation units off / on,
    warp granularity 1-4, both transaction units."""
    rnd = random.Random(seed)
    d = gen.device_sets().copy()
    for i in range(4):
        d[i]["reg_alloc_unit"] = rnd.choice([0, 128, 256])
        d[i]["warp_alloc_gran"] = rnd.choice([0, 1, 2, 4])
        d[i]["smem_alloc_unit"] = rnd.choice([0, 128, 256, 1024])
        d[i]["txn_sectors"] = i % 2
    return d


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_f4_granularity_and_sector_transactions(sel, seed):
    """NEXT row f4 (F4c, F4d): random launches with register and
    shared-memory demands on device sets with allocation granularity and
    either transaction unit, through the fused and the split API."""
    rnd = random.Random(seed)
    n = 800
    launches = np.zeros(n, gen.LAUNCH_DTYPE)
    items = []
    for i in range(n):
        e = rnd.choice([4, 8])
        depth = rnd.choice([0, 1])
        acc = [gen.make_access(base=(1 << 32) + e * rnd.randint(0, 64), c_par=[e * rnd.choice([1, 2, 33, -1])],
                               c_inner=[e * rnd.choice([1, 64])][:depth], elem_bytes=e, depth=depth)]
        launches[i] = (rnd.choice([32, 48, 96, 128, 200, 256, 640, 1024]), 65535,
                       rnd.choice([0, 16, 24, 32, 37, 64, 100, 255]), rnd.choice([0, 100, 300, 4000, 20000, 50000]))
        items.append(dict(P0=rnd.choice([20000, 70000, 150000]), trip=[rnd.randint(1, 3)][:depth], depth=depth,
                          comp=[1.0, 2.0][: depth + 1], launch=i, device=rnd.randrange(4), accesses=acc,
                          bytes_h2d=rnd.choice([0, 10 ** 6])))
    bb = gen.custom_batch(items, devices=_granular_devices(seed), launches_=launches)
    ref = oracle.evaluate(bb)
    assert len(set(ref["abps"][ref["status"] == 0].tolist())) > 5
    assert (ref["status"] == 3).sum() > 0 and (ref["status"] == 0).sum() > 600
    sel.load_device_params(bb.devices)
    try:
        assert_parity(run_gpu(sel, bb), ref, ctx=f"f4 seed={seed}")
        assert_parity(run_gpu(sel, bb, api="split"), ref, exact_cycles=False, ctx=f"f4 split seed={seed}")
    finally:
        sel.load_device_params(gen.device_sets())


def test_c5_full_sweep_sampled(sel):
    """The 10^8-candidate sweep on one GPU, launched exactly as bench.py does;
    a deterministic sample is recomputed by the oracle."""
    b = gen.generate(5)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    r = ev.evaluate(cands, want_counts=True)
    torch.cuda.synchronize()
    rng = np.random.default_rng(5)
    pick = np.unique(np.concatenate([rng.integers(0, len(b), 300), np.arange(0, len(b), len(b) // 100),
                                     [len(b) - 1]]))
    idx = torch.from_numpy(pick).cuda()
    g = {k: v[idx].cpu().numpy() for k, v in r.items()}
    g["counts"] = g["counts"].astype(np.uint64)
    ref = oracle.evaluate(b.select(pick))
    assert_parity(g, ref, exact_cycles=False, ctx="c5 sampled")
    st = ev.stats()
    assert st["n_candidates"] == 10 ** 8 and st["n_invalid"] == 0
    # sharing: 3 B classes (32 | B, 48, 200) per (kernel, z) group of 32 candidates
    assert st["n_problems"] == 3 * (10 ** 8 // 32)
    assert (r["status"] == 0).all().item()


def _random_batch(seed, n):
    import test_oracle_counts as T
    rnd = random.Random(seed)
    nests = [T.random_nest(rnd) for _ in range(n)]
    launches = np.zeros(len(nests), gen.LAUNCH_DTYPE)
    items = []
    for i, nn in enumerate(nests):
        launches[i] = (nn["B"], nn["gmax"], rnd.choice([0, 32, 64]), 0)
        items.append(dict(P0=nn["P0"], P1=nn["P1"], par_dims=nn["par_dims"], trip=nn["trip"], depth=len(nn["trip"]),
                          comp=[rnd.random() * 4 for _ in range(4)], launch=i, device=rnd.randrange(4),
                          cpu_cycles=10 ** rnd.uniform(3, 7), bytes_h2d=rnd.randrange(10 ** 6),
                          accesses=[gen.make_access(base=a["base"], c_par=a["c_par"], c_inner=a["c_inner"],
                                                    elem_bytes=a["elem"], depth=a["depth"]) for a in nn["acc"]]))
    return gen.custom_batch(items, launches_=launches)


@pytest.mark.parametrize("flags", [0, 1, 2, 4, 8, 12])
def test_random_tiny_nests(sel, flags):
    """Random tiny nests: partial warps, B not a multiple of 32, #OMP_Rep > 1,
    collapse(2) with wrapping lanes, negative and zero strides, zero trips,
    empty iteration spaces, every element size."""
    b = _random_batch(77 + flags, 3000)
    assert_parity(run_gpu(sel, b, flags), oracle.evaluate(b), ctx=f"random flags={flags}")


def test_invalid_and_edge_candidates(sel):
    import test_oracle_model as M
    base = M.BASE
    a_ok = gen.make_access(base=base, c_par=(4,), elem_bytes=4, depth=0)
    items = [
        dict(P0=100, trip=[], accesses=[a_ok]),
        dict(P0=100, trip=[], accesses=[a_ok], device=9),                    # V1
        dict(P0=100, trip=[], accesses=[a_ok], cpu_hz=0.0),                  # V1
        dict(P0=100, trip=[], accesses=[a_ok], launch=1),                    # V2 B = 0
        dict(P0=100, trip=[], accesses=[a_ok], launch=2),                    # V2 B = 2048
        dict(P0=100, trip=[], accesses=[a_ok], par_dims=3),                  # V3
        dict(P0=100, P1=3, trip=[], accesses=[a_ok]),                        # V3
        dict(P0=1 << 40, trip=[], accesses=[a_ok]),                          # V4
        dict(P0=100, trip=[], accesses=[gen.make_access(base=base, c_par=(4,), elem_bytes=3)]),          # V5
        dict(P0=100, trip=[], accesses=[gen.make_access(base=base + 4, c_par=(8,), elem_bytes=8)]),      # V5
        dict(P0=100, trip=[], accesses=[gen.make_access(base=1 << 61, c_par=(1 << 56,), elem_bytes=4)]),  # V6
        dict(P0=0, trip=[4], accesses=[gen.make_access(base=base, c_par=(4,), c_inner=(4,), elem_bytes=4, depth=1)]),
        dict(P0=1000, trip=[], accesses=[]),                                 # W = 0 (R22)
        dict(P0=100, trip=[0], accesses=[gen.make_access(base=base, c_par=(4,), c_inner=(4,), elem_bytes=4, depth=1)]),
        dict(P0=100, trip=[gen.TRIP_UNKNOWN], accesses=[gen.make_access(base=base, c_par=(4,), c_inner=(4,),
                                                                        elem_bytes=4, depth=1)]),
        dict(P0=100, trip=[], accesses=[a_ok], launch=3),                    # V7: zero occupancy
    ]
    launches = np.zeros(4, gen.LAUNCH_DTYPE)
    launches[0] = (64, 65535, 0, 0)
    launches[1] = (0, 65535, 0, 0)
    launches[2] = (2048, 65535, 0, 0)
    launches[3] = (1024, 65535, 255, 0)
    b = gen.custom_batch(items, launches_=launches)
    ref = oracle.evaluate(b)
    assert list(ref["status"]) == [0, 1, 1, 1, 1, 1, 1, 2, 1, 1, 2, 0, 0, 0, 0, 3]
    for flags in (0, 1, 2, 4, 8):
        g = run_gpu(sel, b, flags)
        assert_parity(g, ref, ctx=f"edge flags={flags}")
        assert (g["decision"][ref["status"] != 0] == 0xFF).all()


def test_empty_batch_and_errors(sel):
    b = gen.generate(1)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), 4)
    empty = torch.empty(0, dtype=torch.uint8, device="cuda")
    r = ev.evaluate(empty)
    assert r["decision"].numel() == 0
    small_ws = torch.empty(256, dtype=torch.uint8, device="cuda")
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    with pytest.raises(sel.SelError):
        sel.evaluate(cands, ev.tables, small_ws)


def test_deterministic_and_grid_independent(sel):
    b = gen.generate(2)
    g1 = run_gpu(sel, b)
    g2 = run_gpu(sel, b)
    for k in ("counts", "status", "decision", "cycles", "t_gpu"):
        assert np.array_equal(g1[k], g2[k]), k
    # reversing candidate order permutes the outputs and nothing else
    rev = gen.Batch(b.cands[::-1].copy(), b.nests, b.accesses, b.launches, b.devices)
    g3 = run_gpu(sel, rev)
    for k in ("counts", "status", "decision", "cycles"):
        assert np.array_equal(g1[k], g3[k][::-1]), k


def test_near_tie_decisions(sel):
    """cpu_cycles set to T_gpu * cpu_hz and +-1 ulp around it: both sides agree
    (ties go to the CPU, R21)."""
    b = gen.generate(2)
    ref = oracle.evaluate(b)
    c = b.cands.copy()
    c["cpu_hz"] = 1.0
    reps = []
    for d in (-np.inf, 0, np.inf):
        cc = c.copy()
        cc["cpu_cycles"] = ref["t_gpu"] if d == 0 else np.nextafter(ref["t_gpu"], d)
        reps.append(cc)
    bt = gen.Batch(np.concatenate(reps), b.nests, b.accesses, b.launches, b.devices)
    g = run_gpu(sel, bt)
    r2 = oracle.evaluate(bt)
    assert_parity(g, r2, ctx="ties")
    n = len(b)
    assert (g["decision"][:2 * n] == 0).all() and (g["decision"][2 * n:] == 1).all()


def test_host_pipeline_end_to_end(sel):
    """The double-buffered host path returns the same decisions and cycles as
    the device-resident call, step after step (the e2e measurement path)."""
    b = gen.generate(5, 0, 200000)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    ref = ev.evaluate(sel._as_bytes_tensor(b.cands, "candidate"))
    torch.cuda.synchronize()
    ch = torch.from_numpy(b.cands.view(np.uint8).reshape(-1)).pin_memory()
    nh = torch.from_numpy(b.nests.view(np.uint8).reshape(-1)).pin_memory()
    ah = torch.from_numpy(b.accesses.view(np.uint8).reshape(-1)).pin_memory()
    pipe = sel.HostPipeline(ev, ch, nh, ah)
    for k in range(4):
        pipe.step(k, ch, nh, ah)
    for k in (2, 3):
        h = pipe.wait(k)
        assert torch.equal(h["decision"], ref["decision"].cpu())
        assert torch.equal(h["cycles"], ref["cycles"].cpu())


def _random_medium_batch(seed, n):
    """Nests with long inner rows (>= 32, so the fully unrolled 32-WA groups,
    the partial groups and every tmin class run), all element sizes, 1-D and
    collapse(2), negative / zero / large strides, B not a multiple of 32."""
    rnd = random.Random(seed)
    launches = np.zeros(n, gen.LAUNCH_DTYPE)
    items = []
    for i in range(n):
        par_dims = rnd.choice([1, 1, 2])
        P0, P1 = (rnd.randint(1, 300), 1) if par_dims == 1 else (rnd.randint(1, 12), rnd.randint(1, 40))
        depth = rnd.choice([1, 1, 2])
        trip = ([rnd.randint(1, 9), rnd.randint(30, 75)] if depth == 2 else [rnd.randint(30, 75)])
        acc = []
        for _ in range(rnd.randint(1, 3)):
            e = rnd.choice([1, 2, 4, 8, 16])
            d = rnd.randint(0, depth)

            def coef():
                return e * rnd.choice([0, 1, -1, 2, 3, 5, 7, 8, 16, 31, 32, 33, -40, 64, 129, 1000])
            acc.append(gen.make_access(base=(1 << 30) + e * rnd.randint(-100, 100), c_par=[coef(), coef()],
                                       c_inner=[coef() for _ in range(d)], elem_bytes=e, depth=d))
        launches[i] = (rnd.choice([32, 48, 64, 100, 128, 200, 256]), rnd.choice([1, 3, 65535]), 0, 0)
        items.append(dict(P0=P0, P1=P1, par_dims=par_dims, trip=trip, depth=depth, comp=[1.0, 2.0, 0.5],
                          launch=i, device=rnd.randrange(4), accesses=acc))
    return gen.custom_batch(items, launches_=launches)


@pytest.mark.parametrize("flags", [0, 2, 4, 8, 12, 16, 32])
def test_random_medium_nests(sel, flags):
    b = _random_medium_batch(123 + flags, 1500)
    ref = oracle.evaluate(b)
    assert (ref["status"] == 0).all() and ref["W"].sum() > 4 * 10 ** 5
    assert_parity(run_gpu(sel, b, flags), ref, ctx=f"medium flags={flags}")


def test_count_sharing_slot_overflow(sel):
    """More distinct B classes per nest than the 8 sharing slots: the extra
    classes get private counting problems (plan overflow path)."""
    b2 = gen.generate(2)
    Bs = [32, 64, 1024] + list(range(1, 40, 3))          # 3 multiples of 32 (one class) + 13 others
    launches = np.zeros(len(Bs), gen.LAUNCH_DTYPE)
    for i, B in enumerate(Bs):
        launches[i] = (B, 65535 if i % 2 else 7, 0, 0)
    rows = [(nest, li, dev) for nest in (6, 10, 16) for li in range(len(Bs)) for dev in (0, 3)]
    cands = np.zeros(len(rows), gen.CANDIDATE_DTYPE)
    for i, (nest, li, dev) in enumerate(rows):
        cands[i] = (nest, li, dev, 2e6, 3e9)
    b = gen.Batch(cands, b2.nests, b2.accesses, launches, b2.devices)
    g = run_gpu(sel, b)
    assert_parity(g, oracle.evaluate(b), ctx="slot overflow")
    # 8 shared classes per nest; candidates of the remaining classes get private problems
    assert 3 * (8 + 6) < g["stats"]["n_problems"] <= 3 * (8 + 2 * 16)


def _uniform_gap_batch():
    """Lane gaps at and around the closed-form boundaries (0, 31/32/33,
    127/128/129, negative strides), partial warps, depth 0-2 and collapse(2)
    (per-lane gaps that are uniform on some warps and not on others)."""
    import test_oracle_model as M
    base = M.BASE
    items = []
    for cp in (0, 4, 8, 31, 32, 33, 64, 127, 128, 129, 256, 4096, -8, -128, -129, -4096):
        for eb in (4, 8, 16):
            for P0 in (1, 31, 33, 100):
                if cp % eb and cp != 0:
                    continue
                for depth, trip, ci in ((0, [], ()), (1, [37], (eb,)), (2, [3, 45], (4096, eb)),
                                        (1, [5], (128,)), (1, [9], (0,))):
                    b0 = base + 8 * eb + (4096 * 200 if cp < 0 else 0)
                    a = gen.make_access(base=b0, c_par=(cp,), c_inner=ci, elem_bytes=eb, depth=depth)
                    items.append(dict(P0=P0, trip=trip, accesses=[a], comp=[1, 1, 1][: depth + 1]))
    for P1, c1 in ((4, 128), (8, 8), (40, 256), (3, 0)):       # collapse(2): lane gaps c1 or row jumps
        for c0 in (0, 512, 1 << 16):
            a = gen.make_access(base=base, c_par=(c0, c1), c_inner=(8,), elem_bytes=8, depth=1)
            items.append(dict(P0=70, P1=P1, par_dims=2, trip=[6], accesses=[a], comp=[1, 1]))
    # every item again under blocks whose size 32 does not divide (partial last warp
    # of every block) and a small grid cap (#OMP_Rep > 1)
    items += [dict(it, launch=1) for it in items] + [dict(it, launch=2) for it in items]
    launches = np.zeros(3, gen.LAUNCH_DTYPE)
    launches[0] = (256, 65535, 32, 0)
    launches[1] = (48, 65535, 32, 0)
    launches[2] = (200, 1, 32, 0)
    return gen.custom_batch(items, launches_=launches)


@pytest.mark.parametrize("flags", [0, 4, 8, 1, 16])
def test_uniform_flag_closed_form(sel, flags):
    b = _uniform_gap_batch()
    ref = oracle.evaluate(b)
    assert (ref["status"] == 0).all()
    g = run_gpu(sel, b, flags)
    assert_parity(g, ref, ctx=f"uniform-gap flags={flags}")
    st = g["stats"]
    if flags & 8:
        assert st["wa_closed_form"] == 0 and st["wa_arith_lanes"] == 0 and st["wa_residue_classes"] == 0
    else:
        assert 0 < st["wa_closed_form"] and 0 < st["wa_arith_lanes"] + st["wa_residue_classes"]
        assert (st["wa_closed_form"] + st["wa_arith_lanes"] + st["wa_residue_classes"]
                < st["wa_resolved"])                                              # collapse(2) expands


def test_closed_form_share_c5_slice(sel):
    """On a c5 slice most warp-accesses have uniform lane flags (broadcast or
    >= 128-byte lane strides); the closed form and full expansion agree."""
    b = gen.generate(5, 0, 200000)
    g0, g8 = run_gpu(sel, b, 0), run_gpu(sel, b, 8)
    assert (g0["counts"] == g8["counts"]).all() and (g0["cycles"] == g8["cycles"]).all()
    assert g0["stats"]["wa_resolved"] == g8["stats"]["wa_resolved"]
    assert g0["stats"]["wa_closed_form"] > g0["stats"]["wa_resolved"] // 2


def _residue_class_batch(seed, n):
    """1-D accesses with lane strides 0 < g < 128 and long inner loops, so
    whole warp-reps are summed by residue class: every element
    size, odd / even / negative / multiple-of-128 inner coefficients (loop
    periods 1..128), depth 1-3, inner trips around the 32-tuple threshold,
    P with a partial last warp, blocks that 32 does and does not divide, a
    grid cap (#OMP_Rep > 1) and chunk boundaries inside warp-reps."""
    rnd = random.Random(seed)
    Bs = [32, 64, 256, 48, 200, 100, 1000, 33]
    launches = np.zeros(len(Bs), gen.LAUNCH_DTYPE)
    for i, B in enumerate(Bs):
        launches[i] = (B, rnd.choice([1, 5, 65535]), 0, 0)
    items = []
    for _ in range(n):
        depth = rnd.choice([1, 2, 2, 3])
        trip = [rnd.choice([1, 2, 7, 31, 32, 33, 64, 129, 300][: 9 - 3 * (depth - 1)]) for _ in range(depth)]
        acc = []
        for _ in range(rnd.randint(1, 4)):
            e = rnd.choice([1, 2, 4, 8, 16])
            g = e * rnd.randint(1, max(1, 127 // e))
            cp = rnd.choice([g, -g, e, 2 * e])
            d = rnd.randint(1, depth)

            def coef():
                return e * rnd.choice([0, 1, -1, 3, 5, 7, 8, 12, 16, 31, 32, 128, -96, 1000, 1030 + rnd.randint(0, 64)])
            acc.append(gen.make_access(base=(1 << 34) + e * rnd.randint(-2000, 2000), c_par=[cp],
                                       c_inner=[coef() for _ in range(d)], elem_bytes=e, depth=d))
        items.append(dict(P0=rnd.choice([1, 31, 32, 33, 95, 96, 97, 500, 1000, 2049]), trip=trip, depth=depth,
                          comp=[1.0] * (depth + 1), accesses=acc, launch=rnd.randrange(len(Bs)),
                          device=rnd.randrange(4)))
    return gen.custom_batch(items, launches_=launches)


@pytest.mark.parametrize("flags", [0, 16, 4, 1, 8, 32, 48])
def test_residue_classes(sel, flags):
    b = _residue_class_batch(77 + flags, 1500)
    ref = oracle.evaluate(b)
    assert (ref["status"] == 0).all()
    g = run_gpu(sel, b, flags)
    assert_parity(g, ref, ctx=f"residue classes flags={flags}")
    st = g["stats"]
    if flags & (8 | 16):
        assert st["wa_residue_classes"] == 0
    else:
        assert st["wa_residue_classes"] > 0


def test_residue_classes_c5_slice(sel):
    """c5 slice: residue-class counting agrees with lane-by-lane expansion
    and with the arithmetic-lane path, counts and cycles bit for bit."""
    b = gen.generate(5, 3000000, 3300000)
    g0, g16, g8, g32 = run_gpu(sel, b, 0), run_gpu(sel, b, 16), run_gpu(sel, b, 8), run_gpu(sel, b, 32)
    for g in (g16, g8, g32):
        assert (g0["counts"] == g["counts"]).all() and (g0["cycles"] == g["cycles"]).all()
        assert (g0["decision"] == g["decision"]).all()
    assert g0["stats"]["wa_residue_classes"] > 0 and g16["stats"]["wa_residue_classes"] == 0


def _distinct_problems(b):
    """(nest, B class) pairs the batch's valid candidates refer to."""
    B = b.launches["block"][b.cands["launch_id"]].astype(np.int64)
    cls = np.where(B % 32 == 0, 32, B)
    return len(set(zip(b.cands["nest_id"].tolist(), cls.tolist())))


def test_direct_and_hashed_problem_ids_agree(sel):
    """Direct problem ids (launch table <= 1024 entries) and the slot-table path
    (forced by padding the launch table past 1024 entries) give identical
    counts, cycles and decisions, and both count each distinct (nest, B class)
    problem once -- including a slice where most direct ids are unused."""
    b = gen.generate(5, 0, 3 * 768 * 7)
    keep = np.nonzero((b.cands["launch_id"] % 3 != 1) & (np.arange(len(b)) % 5 != 0))[0]
    b = b.select(keep)
    pad = np.zeros(1100, gen.LAUNCH_DTYPE)
    pad["block"], pad["grid_max"] = 96, 65535
    b_hashed = gen.Batch(b.cands, b.nests, b.accesses, np.concatenate([b.launches, pad]), b.devices)
    g_direct, g_hashed = run_gpu(sel, b), run_gpu(sel, b_hashed)
    ref = oracle.evaluate(b)
    assert_parity(g_direct, ref, ctx="direct ids")
    assert_parity(g_hashed, ref, ctx="slot-table ids")
    # direct ids count every (nest, class) pair of the tables; the
    # slot table only the pairs the candidates refer to
    assert g_direct["stats"]["n_problems"] == len(b.nests) * 3
    assert g_hashed["stats"]["n_problems"] == _distinct_problems(b)


def test_direct_ids_sparse_nests(sel):
    """Many nests, few candidates each (nests x classes > candidates): the plan
    falls back to the slot table; counts still exact."""
    b = gen.generate(5, 0, 768 * 40)
    idx = np.arange(0, len(b), 97)
    b = b.select(idx)
    g = run_gpu(sel, b)
    assert_parity(g, oracle.evaluate(b), ctx="sparse")
    assert g["stats"]["n_problems"] == _distinct_problems(b)


def test_validation_fast_path_boundaries(sel):
    """k_problem_w's validation shortcuts at their thresholds: |base| 2^60,
    coefficients 2^28, extents 2^20 (below all three: no saturating bound
    arithmetic),
    the address bound on either side of 2^62 (V6), per-access M_k below / above
    2^26 (the 32-bit segmented sum of M_it) and P * M_it at 2^48 (V6; the valid
    side of that boundary has ~2^43 warp-accesses, beyond the oracle)."""
    import test_oracle_model as M
    base = M.BASE
    k20 = 1 << 20
    acc = gen.make_access
    items = [
        dict(P0=100, trip=[], accesses=[acc(base=k20 - 4, c_par=(4,), elem_bytes=4)]),
        dict(P0=100, trip=[], accesses=[acc(base=k20, c_par=(4,), elem_bytes=4)]),
        dict(P0=k20 - 1, trip=[], accesses=[acc(base=base, c_par=(4,), elem_bytes=4)]),
        dict(P0=k20, trip=[], accesses=[acc(base=base, c_par=(4,), elem_bytes=4)]),
        dict(P0=64, trip=[k20 - 1], accesses=[acc(base=base, c_par=(4,), c_inner=(k20 - 4,), elem_bytes=4, depth=1)]),
        dict(P0=64, trip=[3], accesses=[acc(base=base, c_par=(4,), c_inner=(k20,), elem_bytes=4, depth=1)]),
        # the shortcut's own thresholds: |base| 2^60, coefficients 2^28
        dict(P0=100, trip=[], accesses=[acc(base=(1 << 60) - 4, c_par=(4,), elem_bytes=4)]),
        dict(P0=100, trip=[], accesses=[acc(base=1 << 60, c_par=(4,), elem_bytes=4)]),
        dict(P0=100, trip=[3], accesses=[acc(base=base, c_par=((1 << 28) - 4,), c_inner=((1 << 28) - 8,),
                                             elem_bytes=4, depth=1)]),
        dict(P0=100, trip=[3], accesses=[acc(base=base, c_par=(1 << 28,), c_inner=(1 << 28,), elem_bytes=4,
                                             depth=1)]),
        # |base| + |c| (P - 1) just below / at 2^62
        dict(P0=2, trip=[], accesses=[acc(base=(1 << 62) - 8 - 4, c_par=(4,), elem_bytes=4)]),
        dict(P0=2, trip=[], accesses=[acc(base=(1 << 62) - 4, c_par=(4,), elem_bytes=4)]),
        # M_k = 2^13 * 2^13 = 2^26 on one access of a multi-access nest (64-bit segmented sum)
        dict(P0=32, trip=[1 << 13, 1 << 13], accesses=[acc(base=base, c_par=(4,), elem_bytes=4),
                                                      acc(base=base, c_par=(4,), c_inner=(4, 8), elem_bytes=4,
                                                          depth=2)]),
        # P M_it around 2^48 (ERANGE at and above)
        dict(P0=1 << 20, trip=[1 << 14, 1 << 14], accesses=[acc(base=base, c_par=(4,), c_inner=(4, 8),
                                                                elem_bytes=4, depth=2)]),
    ]
    b = gen.custom_batch(items)
    ref = oracle.evaluate(b)
    assert ref["status"][11] == 2 and ref["status"][10] == 0 and ref["status"][13] == 2
    for flags in (0, 1):
        g = run_gpu(sel, b, flags)
        assert_parity(g, ref, ctx=f"validation boundaries flags={flags}")
