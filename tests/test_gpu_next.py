"""GPU parity of the NEXT rows against the oracle."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sel():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_chikinaat19_b200 as s
    return s


def test_select_launch_random(sel):
    rng = np.random.default_rng(11)
    n, G = 200000, 30000
    group = rng.integers(0, G + 50, n).astype(np.uint32)
    t = rng.choice([0.25, 1.0, 3.0, np.inf], n) * rng.integers(1, 5, n)
    st = (rng.random(n) < 0.05).astype(np.uint8)
    b_ref, v_ref = oracle.select_launch(group, t, st, G)
    g_d = torch.from_numpy(group.view(np.int32)).cuda()
    best, val = sel.select_launch(g_d, torch.from_numpy(t).cuda(), torch.from_numpy(st).cuda(), G)
    torch.cuda.synchronize()
    assert (best.cpu().numpy().view(np.uint32) == b_ref).all()
    v = val.cpu().numpy()
    assert ((v == v_ref) | (np.isinf(v) & np.isinf(v_ref))).all()


def test_select_launch_on_c4(sel):
    """c4: each of the 24 nests under 8 launch configurations -> the launch
    with the lowest predicted T_gpu per nest, from the fused evaluation."""
    b = gen.generate(4)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    c = sel._as_bytes_tensor(b.cands, "candidate")
    r = ev.evaluate(c, want_t_gpu=True)
    group = torch.from_numpy(b.cands["nest_id"].astype(np.int32)).cuda()
    best, val = sel.select_launch(group, r["t_gpu"], r["status"], 24)
    torch.cuda.synchronize()
    b_ref, v_ref = oracle.select_launch(b.cands["nest_id"], r["t_gpu"].cpu().numpy(), r["status"].cpu().numpy(), 24)
    assert (best.cpu().numpy().view(np.uint32) == b_ref).all()
    assert (val.cpu().numpy() == v_ref).all()


@pytest.mark.parametrize("cfg,rng", [(1, (0, 2)), (2, (0, 108)), (4, (0, 192)), (5, (0, 2000000))])
def test_cpu_model_parity(sel, cfg, rng):
    """NEXT row f1: the device Liao-Chapman model writes the same cpu_cycles
    (bit-exact) and statuses as the oracle; c4 exercises the TLB term."""
    b = gen.generate(cfg, *rng)
    cin = gen.cpu_inputs(cfg, *rng)
    cin["threads"][::97] = 0                                  # some invalid inputs
    ref, st_ref = oracle.cpu_model(gen.cpu_params(), b, cin)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    c = sel._as_bytes_tensor(b.cands.copy(), "candidate")
    st = sel.model_cpu_cost(c, ev.tables, cin, gen.cpu_params())
    torch.cuda.synchronize()
    out = c.cpu().numpy().view(gen.CANDIDATE_DTYPE)
    st = st.cpu().numpy()
    assert (st == st_ref).all()
    ok = st == 0
    assert (out["cpu_cycles"][ok] == ref[ok]).all()
    assert (out["cpu_hz"][ok] == 3e9).all()
    assert (out["cpu_cycles"][~ok] == b.cands["cpu_cycles"][~ok]).all()    # invalid: untouched
    # the modelled cost then drives the decision exactly like a supplied one
    if cfg in (1, 2):
        r = ev.evaluate(c, want_t_gpu=True)
        bb = gen.Batch(out.copy(), b.nests, b.accesses, b.launches, b.devices)
        ref_eval = oracle.evaluate(bb)
        assert (r["decision"].cpu().numpy() == ref_eval["decision"]).all()


def test_sync_term_parity(sel):
    """NEXT row f4: nests with barriers (n_sync > 0) -> bit-exact cycles."""
    import test_gpu_parity as P
    b = P._random_batch(5, 2000)
    nests = b.nests.copy()
    nests["n_sync"] = np.arange(len(nests)) % 4
    bb = gen.Batch(b.cands, nests, b.accesses, b.launches, b.devices)
    P.assert_parity(P.run_gpu(sel, bb), oracle.evaluate(bb), ctx="f4 sync")


@pytest.mark.parametrize("cfg,rng", [(2, (0, 108)), (5, (0, 10000000))])
def test_bind_parity(sel, cfg, rng):
    """NEXT row f2: device binding == oracle binding == the generator's
    concrete accesses; bound tables evaluate identically."""
    sym, terms = gen.sym_tables()
    vals, items = gen.sym_instances(cfg, *rng)
    vals[9 * 5 + 2] = 1 << 61                            # one overflowing frame (ERANGE)
    ref, st_ref = oracle.bind(sym, terms, vals, items)
    out, st = sel.bind_accesses(sym, terms, vals, items)
    torch.cuda.synchronize()
    assert (st.cpu().numpy() == st_ref).all()
    assert np.array_equal(out.cpu().numpy(), ref)
    assert (st_ref != 0).sum() >= 1


@pytest.mark.parametrize("cfg,rng", [(2, (0, 108)), (4, (0, 192)), (5, (0, 300000))])
def test_evaluate_cpu_model_fused(sel, cfg, rng):
    """NEXT row f1 fused into a7 (sel_evaluate_cpu_model): one pass with the
    Liao-Chapman CPU cost gives the oracle's decisions and cycles computed on
    candidates whose cpu_cycles / cpu_hz the oracle's own f1 model replaced;
    invalid CPU inputs -> SEL_EINVAL.  The candidate records stay untouched."""
    b = gen.generate(cfg, *rng)
    cin = gen.cpu_inputs(cfg, *rng)
    cin["threads"][::53] = 0
    cin["mca_cycles_per_iter"][7::61] = -1.0
    params = gen.cpu_params()
    cyc, st_f1 = oracle.cpu_model(params, b, cin)
    cm = b.cands.copy()
    ok = st_f1 == 0
    cm["cpu_cycles"][ok] = cyc[ok]
    cm["cpu_hz"][ok] = params["cpu_hz"][0]
    ref = oracle.evaluate(gen.Batch(cm, b.nests, b.accesses, b.launches, b.devices))
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    c = sel._as_bytes_tensor(b.cands.copy(), "candidate")
    before = c.clone()
    r = sel.evaluate_cpu_model(c, ev.tables, ev.workspace, cin, params, want_t_gpu=True)
    torch.cuda.synchronize()
    assert torch.equal(c, before)
    status = r["status"].cpu().numpy()
    exp_status = np.where(ok, ref["status"], 1)
    assert (status == exp_status).all()
    v = ok & (ref["status"] == 0)
    assert (r["decision"].cpu().numpy()[v] == ref["decision"][v]).all()
    assert (r["cycles"].cpu().numpy()[v] == ref["cycles"][v]).all()
    assert (r["t_gpu"].cpu().numpy()[v] == ref["t_gpu"][v]).all()
    assert (r["decision"].cpu().numpy()[~ok] == 0xFF).all()
    assert v.sum() > 0.9 * len(b) - 2 * len(b) // 50
