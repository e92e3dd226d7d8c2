"""Pins of the oracle's model part (a4-a7): special cases that reduce to a
closed form, the #OMP_Rep factor, invariants, the tie-break and validation.
The Hong & Kim equations that PAPER.md does not print (readings R2, R5,
Mem_L, Departure_delay) are parity-unpinned beyond these."""
import numpy as np
import pytest

import gen
import oracle

BASE = 1 << 28
DEV = gen.device_sets()
V = DEV[gen.V100]


def unit_stride_nest(P, trip, comp, B=32, gmax=65535, device=gen.V100, regs=0, bytes_=(0, 0), cpu=1e6):
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (B, gmax, regs, 0)
    a = gen.make_access(base=BASE, c_par=(4,), c_inner=(0,), elem_bytes=4, depth=1)
    return gen.custom_batch([dict(P0=P, trip=[trip], comp=comp, accesses=[a], device=device,
                                  bytes_h2d=bytes_[0], bytes_d2h=bytes_[1], cpu_cycles=cpu)],
                            launches_=launches)


@pytest.mark.parametrize("trip,comp0,comp1,P,gmax", [(1, 0.0, 0.0, 32, 1), (7, 3.0, 2.0, 32, 65535),
                                                     (100, 4.0, 6.5, 64, 1), (128, 0.0, 1.0, 96, 1)])
def test_single_warp_serial_closed_form(trip, comp0, comp1, P, gmax):
    """One warp per SM (B = 32, one block resident, G <= #SMs): N = 1 so
    MWP = CWP = N = 1 (Fig. 4 first case).  A lone warp executes
    serially: every (coalesced) memory instruction costs Mem_LD and every
    instruction costs issue cycles, so per OpenMP repetition
    Exec = Mem_LD * mem + issue * (comp + mem)."""
    r = oracle.evaluate(unit_stride_nest(P, trip, [comp0, comp1], B=32, gmax=gmax))[0]
    assert r["status"] == 0 and r["hk_case"] == 1 and r["N"] == 1.0
    R = -(-P // 32) if gmax == 1 else 1
    mem = trip
    comp = comp0 + comp1 * trip
    expect = (V["mem_ld_cycles"] * mem + V["issue_cycles"] * (comp + mem)) * R
    assert r["cycles"] == pytest.approx(expect, rel=1e-15)


def test_no_memory_instructions_compute_only():
    """R22: no memory instruction (W = 0, P > 0): all N warps are
    compute-bound, Exec = issue * comp * N * #Rep * #OMP_Rep."""
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (256, 65535, 0, 0)
    b = gen.custom_batch([dict(P0=10000, trip=[5], comp=[3.0, 2.0], accesses=[])], launches_=launches)
    r = oracle.evaluate(b)[0]
    assert r["status"] == 0 and r["W"] == 0 and r["hk_case"] == 0
    G = -(-10000 // 256)
    abps = min(32, 64 // 8, 2048 // 256, -(-G // 80))
    N, Rep = abps * 8, G / (abps * min(G, 80))
    assert r["cycles"] == pytest.approx(2.0 * (3.0 + 2.0 * 5) * N * Rep * 1, rel=1e-15)


def test_omp_rep_multiplies_exec():
    """P:L225 / Fig. 4: with the grid capped at one block, doubling the
    iteration count doubles #OMP_Rep and leaves the per-warp averages
    unchanged, so Exec_Cycles doubles exactly."""
    r1 = oracle.evaluate(unit_stride_nest(1024, 9, [1.0, 3.0], B=128, gmax=1))[0]
    r2 = oracle.evaluate(unit_stride_nest(2048, 9, [1.0, 3.0], B=128, gmax=1))[0]
    assert r1["R"] == 8 and r2["R"] == 16
    assert r2["cycles"] == 2.0 * r1["cycles"]


def test_occupancy_and_rep():
    """R17 / R5 on concrete numbers: V100, B = 1024, 32 regs/thread,
    G = 800 blocks -> 2 resident blocks per SM (warp, thread and register
    limits), N = 64 warps, #Rep = 800 / (2 * 80) = 5."""
    r = oracle.evaluate(unit_stride_nest(800 * 1024, 2, [1.0, 1.0], B=1024, regs=32))[0]
    assert (r["G"], r["abps"], r["active_sms"]) == (800, 2, 80)
    assert r["N"] == 64.0 and r["Rep"] == 5.0
    r = oracle.evaluate(unit_stride_nest(800 * 1024, 2, [1.0, 1.0], B=1024, regs=33))[0]
    assert r["abps"] == 1
    r = oracle.evaluate(unit_stride_nest(800 * 1024, 2, [1.0, 1.0], B=1024, regs=65))[0]
    assert r["status"] == oracle.ELAUNCH and r["decision"] == 0xFF


def test_latency_homogeneity():
    """Every cycle term is linear in the latency parameters: with ample
    bandwidth, scaling Mem_LD, both departure delays and the issue cost by 2
    (exact in binary) scales the predicted cycles by exactly 2 in every
    case of Fig. 4."""
    b = gen.generate(2)
    dev = b.devices.copy()
    dev["mem_bw_Bps"] = 1e30
    b1 = gen.Batch(b.cands, b.nests, b.accesses, b.launches, dev)
    dev2 = dev.copy()
    for f in ["mem_ld_cycles", "dep_del_coal", "dep_del_uncoal", "issue_cycles"]:
        dev2[f] *= 2
    b2 = gen.Batch(b.cands, b.nests, b.accesses, b.launches, dev2)
    r1, r2 = oracle.evaluate(b1), oracle.evaluate(b2)
    np.testing.assert_array_equal(r2["hk_case"], r1["hk_case"])
    np.testing.assert_array_equal(r2["cycles"], 2.0 * r1["cycles"])


def test_model_invariants_c2():
    b = gen.generate(2)
    r = oracle.evaluate(b)
    assert (r["status"] == 0).all()
    m = r["W"] > 0
    assert (r["CWP"][m] >= 1.0).all() and (r["CWP"][m] <= r["N"][m]).all()
    assert (r["MWP"][m] > 0).all() and (r["MWP"][m] <= r["N"][m]).all()
    assert (r["cycles"] >= 0).all()
    # case selection as read in R1-R3
    c1 = (r["MWP"] == r["N"]) & (r["CWP"] == r["N"])
    c2 = ~c1 & ((r["CWP"] >= r["MWP"]) | (r["Comp"] > r["Mem"]))
    np.testing.assert_array_equal(r["hk_case"][m], np.where(c1, 1, np.where(c2, 2, 3))[m])
    assert set(np.unique(r["hk_case"])) >= {1, 2}
    # T_gpu = cycles / f + bytes / link + launch (R20), decision = T_gpu < T_cpu
    f = b.devices["sm_clock_hz"][b.cands["device_id"]]
    assert (r["t_gpu"] > r["cycles"] / f).all()
    np.testing.assert_array_equal(r["decision"], (r["t_gpu"] < r["t_cpu"]).astype(np.uint8))


def test_tgpu_monotone_in_bytes_and_decision_monotone_in_cpu_cost():
    b = gen.generate(2)
    r0 = oracle.evaluate(b)
    nests = b.nests.copy()
    nests["bytes_h2d"] += 10 ** 9
    r1 = oracle.evaluate(gen.Batch(b.cands, nests, b.accesses, b.launches, b.devices))
    assert (r1["t_gpu"] >= r0["t_gpu"]).all() and (r1["cycles"] == r0["cycles"]).all()
    prev = None
    for scale in [1e-6, 1e-3, 1.0, 1e3, 1e6, 1e9]:
        c = b.cands.copy()
        c["cpu_cycles"] *= scale
        d = oracle.evaluate(gen.Batch(c, b.nests, b.accesses, b.launches, b.devices))["decision"]
        if prev is not None:
            assert (d >= prev).all()    # never GPU -> CPU as the CPU cost grows
        prev = d


def test_tie_goes_to_cpu():
    """R21: strict '<' -- an exact tie keeps the loop on the host."""
    b = gen.generate(1)
    r = oracle.evaluate(b)
    c = b.cands.copy()
    c["cpu_hz"] = 1.0
    c["cpu_cycles"] = r["t_gpu"]
    assert (oracle.evaluate(gen.Batch(c, b.nests, b.accesses, b.launches, b.devices))["decision"] == 0).all()
    c["cpu_cycles"] = np.nextafter(r["t_gpu"], np.inf)
    assert (oracle.evaluate(gen.Batch(c, b.nests, b.accesses, b.launches, b.devices))["decision"] == 1).all()


def test_empty_iteration_space():
    r = oracle.evaluate(unit_stride_nest(0, 4, [1.0, 1.0]))[0]
    assert r["status"] == 0 and r["decision"] == 0 and r["cycles"] == 0.0 and np.isinf(r["t_gpu"])
    assert r["W"] == 0 and r["WR"] == 0


def _one(access=None, **kw):
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (kw.pop("B", 64), kw.pop("gmax", 65535), 0, 0)
    a = access if access is not None else gen.make_access(base=BASE, c_par=(4,), elem_bytes=4, depth=0)
    item = dict(P0=100, trip=[], accesses=[a], comp=[1.0])
    item.update(kw)
    return oracle.evaluate(gen.custom_batch([item], launches_=launches))[0]


def test_validation_statuses():
    assert _one()["status"] == 0
    assert _one(device=7)["status"] == oracle.EINVAL
    assert _one(cpu_hz=0.0)["status"] == oracle.EINVAL
    assert _one(B=0)["status"] == oracle.EINVAL
    assert _one(B=1025)["status"] == oracle.EINVAL
    assert _one(gmax=0)["status"] == oracle.EINVAL
    assert _one(par_dims=3)["status"] == oracle.EINVAL
    assert _one(P1=2)["status"] == oracle.EINVAL                       # par_dims 1 needs P1 = 1
    assert _one(access=gen.make_access(base=BASE, c_par=(4,), elem_bytes=3))["status"] == oracle.EINVAL
    assert _one(access=gen.make_access(base=BASE + 2, c_par=(4,), elem_bytes=4))["status"] == oracle.EINVAL
    assert _one(access=gen.make_access(base=BASE, c_par=(6,), elem_bytes=4))["status"] == oracle.EINVAL
    assert _one(access=gen.make_access(base=BASE, c_par=(4,), elem_bytes=4, depth=1))["status"] == oracle.EINVAL
    assert _one(access=gen.make_access(base=1 << 61, c_par=(1 << 56,), elem_bytes=4))["status"] == oracle.ERANGE
    assert _one(P0=1 << 40)["status"] == oracle.ERANGE
    a = gen.make_access(base=BASE, c_par=(4,), c_inner=(4, 4), elem_bytes=4, depth=2)
    assert _one(access=a, trip=[1 << 24, 1 << 24], depth=2, comp=[1, 1, 1])["status"] == oracle.ERANGE
    r = _one(device=7)
    assert r["decision"] == 0xFF and r["W"] == 0 and r["cycles"] == 0.0
