"""GPU: config-4 multi-GPU partitioning -- each rank counts a
1/R slice of the deduplicated warp-access space (sel_count_transactions_part)
and one all_reduce(SUM) of the u64 counters restores the exact counts.

Checks: the parts sum to sel_count_transactions exactly for several R (and to
the oracle's brute-force counts); warp_reps appears in part 0 only; statuses
are identical across parts; the part sizes add up to the whole; the 2-rank
path (evaluate_split over gloo, both ranks on the box's single GPU) matches
the oracle end to end."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FIELDS = ["W", "L", "S", "C", "U", "WR"]


@pytest.fixture(scope="module")
def sel():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_chikinaat19_b200 as s
    assert torch.cuda.is_available()
    return s


def c4_reduced():
    b = gen.generate(4)
    nests = b.nests.copy()
    nests["P0"] = 1 << 14
    return gen.Batch(b.cands, nests, b.accesses, b.launches, b.devices)


def _parts(sel, b, n_parts, flags=0):
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), max(len(b), 1), flags)
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    full, st_full = sel.count_transactions(cands, ev.tables, ev.workspace, flags)
    full = full.cpu().numpy().astype(np.uint64)
    st_full = st_full.cpu().numpy()
    total = sel.read_stats(ev.workspace)["wa_resolved"]
    acc = np.zeros_like(full)
    sizes = []
    for p in range(n_parts):
        c, st = sel.count_transactions(cands, ev.tables, ev.workspace, flags, part=p, n_parts=n_parts)
        c = c.cpu().numpy().astype(np.uint64)
        assert (st.cpu().numpy() == st_full).all(), f"part {p}: status differs"
        if p > 0:
            assert (c[:, 5] == 0).all(), "warp_reps must come from part 0 only"
        acc += c
        sizes.append(sel.read_stats(ev.workspace)["wa_resolved"])
    # the parts tile the work: big problems by equal slices of the WA prefix, small
    # problems (counted one per lane) by problem-index ranges
    assert sum(sizes) == total
    return full, acc, st_full


@pytest.mark.parametrize("n_parts", [2, 3, 8])
def test_parts_sum_exactly_c4(sel, n_parts):
    b = c4_reduced()
    full, acc, _ = _parts(sel, b, n_parts)
    assert (acc == full).all()
    ref = oracle.evaluate(b)
    for j, f in enumerate(FIELDS):
        assert (acc[:, j] == ref[f]).all(), f"field {f}"


@pytest.mark.parametrize("flags", [0, 1, 4])
def test_parts_sum_exactly_c2_c5(sel, flags):
    for b in (gen.generate(2), gen.generate(5, 0, 20000)):
        full, acc, st = _parts(sel, b, 5, flags)
        assert (acc == full).all()
        assert (st == 0).all()


def test_more_parts_than_work(sel):
    b = gen.generate(1)          # 24 576 WAs split 10 ^ 5 ways: most parts are empty
    full, acc, _ = _parts(sel, b, 100000)
    assert (acc == full).all()


def test_part_out_of_range(sel):
    b = gen.generate(1)
    ev = sel.Evaluator((b.nests, b.accesses, b.launches, b.devices), len(b))
    cands = sel._as_bytes_tensor(b.cands, "candidate")
    for part, n_parts in ((1, 1), (3, 2), (0, 0)):
        with pytest.raises(sel.SelError) as e:
            sel.count_transactions(cands, ev.tables, ev.workspace, part=part, n_parts=n_parts)
        assert e.value.code == sel.SEL_EINVAL


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_evaluate_split_two_ranks(tmp_path):
    import __graft_entry__
    __graft_entry__.build()
    env = dict(os.environ, SEL_DIST_BACKEND="gloo", SPLIT_OUT=str(tmp_path))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()),
           os.path.join(ROOT, "tests", "split_worker.py")]
    p = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert p.returncode == 0, p.stderr[-3000:]
    b = c4_reduced()
    ref = oracle.evaluate(b)
    for r in range(2):
        d = json.load(open(tmp_path / f"rank{r}.json"))
        counts = np.array(d["counts"], dtype=np.uint64)
        for j, f in enumerate(FIELDS):
            assert (counts[:, j] == ref[f]).all(), f"rank {r}: field {f}"
        assert (np.array(d["decision"], dtype=np.uint8) == ref["decision"]).all()
        assert (np.array(d["cycles"]) == ref["cycles"]).all()
