"""GPU parity at the boundaries of the model kernel's lazy fast path
(csrc/sel_model.cu:hk_eval_lazy): the comparisons it takes from
certified estimates -- MWP_peak_BW against N (Fig. 5), CWP against
N and T_gpu < T_cpu (R21) -- are driven to within a few
ulps and a few multiples of the 2^-20 margin of their threshold, where the
kernel must fall back to the exact quotients.  Everything is compared bit for
bit with the oracle, with t_gpu stored and not stored (the decision estimate
is used only in the second case's exact-path-free route)."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu

DELTAS = [-2.0 ** -10, -2.0 ** -19, -2.0 ** -20, -2.0 ** -21, -2.0 ** -28, -2.0 ** -40, -2.0 ** -52, 0.0,
          2.0 ** -52, 2.0 ** -40, 2.0 ** -28, 2.0 ** -21, 2.0 ** -20, 2.0 ** -19, 2.0 ** -10]


@pytest.fixture(scope="module")
def sel():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_chikinaat19_b200 as s
    assert torch.cuda.is_available()
    return s


def base_device():
    d = gen.device_sets()[gen.V100].copy()
    d["issue_cycles"] = 1.0
    d["dep_del_uncoal"] = 1.0
    d["dep_del_coal"] = 1.0
    d["mem_ld_cycles"] = 27.0
    d["txn_sectors"] = 1
    d["mem_bw_Bps"] = 1e30
    d["sm_clock_hz"] = 1e9
    return d


def one_warp_batch(devices, cpu_cycles=1e6, cpu_hz=3e9):
    """One candidate per device set: 32 iterations of a stride-1 fp32 access
    (4 sectors per warp-access, M_it = 1), comp = 9, B = 128: G = 1, abps = 1,
    N = 4, Comp = 10, Mem = MemL_u = mem_ld + 3 (sector transactions, F4d)."""
    launches = np.zeros(1, gen.LAUNCH_DTYPE)
    launches[0] = (128, 65535, 32, 0)
    a = gen.make_access(base=0, c_par=(4,), elem_bytes=4, depth=0)
    items = [dict(P0=32, trip=[], depth=0, comp=[9.0], accesses=[a], launch=0, device=i,
                  bytes_h2d=4096, cpu_cycles=(cpu_cycles[i] if np.ndim(cpu_cycles) else cpu_cycles),
                  cpu_hz=cpu_hz) for i in range(len(devices))]
    return gen.custom_batch(items, devices=np.array(devices), launches_=launches)


def check(sel, b):
    ref = oracle.evaluate(b)
    assert (ref["status"] == 0).all()
    for want_t in (True, False):
        ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
        cands = sel._as_bytes_tensor(b.cands, "candidate")
        r = ev.evaluate(cands, want_counts=want_t, want_t_gpu=want_t)   # neither: the bench's loop instance
        torch.cuda.synchronize()
        g = {k: v.cpu().numpy() for k, v in r.items()}
        assert (g["status"] == ref["status"]).all()
        assert (g["decision"] == ref["decision"]).all(), (want_t, g["decision"], ref["decision"])
        assert (g["cycles"] == ref["cycles"]).all(), (want_t, g["cycles"] - ref["cycles"])
        if want_t:
            assert (g["t_gpu"] == ref["t_gpu"]).all()
    return ref


def test_cwp_against_n(sel):
    """CWP_raw = 1 + Mem/Comp = 1 + (mem_ld + 3)/10 crosses N = 4 at mem_ld = 27."""
    devs = []
    for dl in DELTAS:
        d = base_device()
        d["mem_ld_cycles"] = 27.0 * (1.0 + dl)
        devs.append(d)
    ref = check(sel, one_warp_batch(devs))
    assert (ref["N"] == 4.0).all()
    assert (ref["CWP"] == 4.0).any() and (ref["CWP"] < 4.0).any()


def test_mwp_peak_bw_against_n(sel):
    """MWP_peak_BW = Mem_BW / (BW_per_warp #Active_SMs) set to N (1 + delta)
    in exact fp64 (Python floats round like the kernel)."""
    d0 = base_device()
    d0["mem_ld_cycles"] = 60.0           # CWP = 1 + 63/10 > N: case 1 / 2 decided by MWP
    MemL = 60.0 + (4.0 - 1.0) * 1.0      # sectors: upmw = S/W = 4, w_unc = 1
    LB = 32.0 * 4                        # Load_bytes_per_warp = 32 S / W
    X = (1e9 * LB) / MemL * 1.0          # BW_per_warp * #Active_SMs (act = G = 1)
    devs = []
    for dl in DELTAS:
        d = d0.copy()
        d["mem_bw_Bps"] = 4.0 * X * (1.0 + dl)
        devs.append(d)
    for k in (-1, 1):                    # the quotient one ulp either side of N
        d = d0.copy()
        d["mem_bw_Bps"] = np.nextafter(4.0 * X, k * np.inf)
        devs.append(d)
    ref = np.concatenate([check(sel, one_warp_batch(devs[:15])), check(sel, one_warp_batch(devs[15:]))])
    assert (ref["MWPbw"] >= 4.0).any() and (ref["MWPbw"] < 4.0).any()


def test_decision_against_t_cpu(sel):
    """cpu_cycles = T_gpu cpu_hz (1 + delta), around the 2^-20 decision margin
    and at the exact tie (ties: CPU, R21)."""
    devs = [base_device() for _ in DELTAS]
    b = one_warp_batch(devs)
    ref = oracle.evaluate(b)
    hz = 3e9
    cyc = np.array([ref["t_gpu"][i] * hz * (1.0 + dl) for i, dl in enumerate(DELTAS)])
    ref2 = check(sel, one_warp_batch(devs, cpu_cycles=cyc, cpu_hz=hz))
    assert (ref2["decision"] == 1).any() and (ref2["decision"] == 0).any()
    # ulp neighbours of the tie with cpu_hz = 1
    t = ref["t_gpu"][:3]
    cyc = np.concatenate([np.nextafter(t, -np.inf), t, np.nextafter(t, np.inf)])
    devs = [base_device() for _ in range(len(cyc))]
    ref3 = check(sel, one_warp_batch(devs, cpu_cycles=cyc, cpu_hz=1.0))
    assert list(ref3["decision"]) == [0] * 6 + [1] * 3


def test_zero_cpu_cost_and_rep(sel):
    """cpu_cycles = 0 (T_cpu = +0: CPU) and a grid larger than the SM count
    (#Rep through the division) next to G <= #SMs (#Rep = 1 exactly)."""
    devs = [base_device() for _ in range(4)]
    b = one_warp_batch(devs, cpu_cycles=np.array([0.0, 1e3, 1e12, 0.0]))
    check(sel, b)
    launches = np.zeros(2, gen.LAUNCH_DTYPE)
    launches[0] = (128, 65535, 32, 0)
    launches[1] = (32, 65535, 32, 0)
    a = gen.make_access(base=0, c_par=(4,), elem_bytes=4, depth=0)
    items = [dict(P0=p, trip=[], depth=0, comp=[9.0], accesses=[a], launch=li, device=gen.V100)
             for p in (32, 80 * 32, 81 * 32, 300 * 128, 10 ** 6 + 7) for li in (0, 1)]
    check(sel, gen.custom_batch(items, launches_=launches))


def _plain(sel, b):
    """decision / cycles / status only (the loop instance the bench times)."""
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), max(len(b), 1))
    r = ev.evaluate(sel._as_bytes_tensor(b.cands, "candidate"))
    torch.cuda.synchronize()
    return {k: v.cpu().numpy() for k, v in r.items()}


@pytest.mark.parametrize("order", ["sweep", "shuffled", "reversed"])
def test_plain_loop_any_order(sel, order):
    """The candidate loop for direct ids with no t_gpu / counts stored (the
    bench's instance) on c5's sweep order, a random permutation and the
    reverse, with a batch that is not a multiple of any tile: the oracle's
    bits."""
    idx = np.arange(0, 5 * 768 + 77)
    b = gen.generate_indices(5, 1000 * 768 + idx)
    if order == "shuffled":
        b = b.select(np.random.default_rng(3).permutation(len(b)))
    elif order == "reversed":
        b = b.select(np.arange(len(b))[::-1])
    ref = oracle.evaluate(b)
    g = _plain(sel, b)
    assert (g["status"] == ref["status"]).all()
    assert (g["decision"] == ref["decision"]).all()
    assert (g["cycles"] == ref["cycles"]).all()


def test_plain_loop_edges_and_device_counts(sel):
    """Invalid and off-fast-path candidates in the bench's loop instance
    (deferred to the exact path), with 4 and 3 device sets."""
    b = gen.generate(2)
    c = b.cands.copy()
    c["cpu_hz"][5] = 0.0                          # V1 inside a run
    c["launch_id"][9] = 200                       # V1: launch id out of range
    c["cpu_cycles"][11] = 0.0                     # T_cpu = +0
    b2 = gen.Batch(c, b.nests, b.accesses, b.launches, b.devices)
    for bb in (b2, gen.Batch(c[c["device_id"] < 3], b.nests, b.accesses, b.launches, b.devices[:3])):
        ref = oracle.evaluate(bb)
        g = _plain(sel, bb)
        assert (g["status"] == ref["status"]).all()
        assert (g["decision"] == ref["decision"]).all()
        assert (g["cycles"] == ref["cycles"]).all()
