"""CPU: the multi-rank host logic (shard ranges, padded all-gather of
decisions, max-over-ranks timing) with world_size 2 on the gloo backend."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_chikinaat19_b200 import dist as D


def test_shard_ranges_cover_exactly():
    for total in (0, 1, 7, 100, 10 ** 8 + 3):
        for world in (1, 2, 3, 4, 8):
            ranges = [D.shard_range(total, r, world) for r in range(world)]
            assert ranges[0][0] == 0 and ranges[-1][1] == total
            for (a0, a1), (b0, b1) in zip(ranges, ranges[1:]):
                assert a1 == b0
            sizes = [b - a for a, b in ranges]
            n_pad = D.padded_len(total, world)
            assert max(sizes) <= n_pad
            # rank r's range starts at r * n_pad (its slot of the gather buffer) unless past the end
            assert all(a == min(total, r * n_pad) for r, (a, _) in enumerate(ranges))


def test_weighted_ranges_balance_work():
    rng = np.random.default_rng(3)
    for n, world in ((1, 1), (10, 3), (1000, 8), (12345, 4)):
        w = rng.integers(0, 1000, n) * (rng.random(n) < 0.7)
        w[: n // 10] *= 50                                   # a heavy head
        p = np.cumsum(w)
        r = D.weighted_ranges(p, world)
        assert r[0][0] == 0 and r[-1][1] == n and all(a[1] == b[0] for a, b in zip(r, r[1:]))
        total = int(p[-1]) if n else 0
        share = [int(w[a:b].sum()) for a, b in r]
        assert sum(share) == total
        # every rank's work is within one candidate's work of the ideal share
        assert max(share) <= total / world + w.max() + 1
    assert D.weighted_ranges(np.zeros(5, np.int64), 2) == [(0, 2), (2, 5)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, total, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    r, w, _ = D.init("gloo")
    assert (r, w) == (rank, world)
    import gen
    c0, c1 = D.shard_range(total, r, w)
    b = gen.generate(5, c0, c1)
    # stand-in for the GPU decisions: a deterministic function of the candidate
    local = torch.from_numpy(((b.cands["nest_id"] + b.cands["device_id"]) % 3).astype(np.uint8))
    full = D.gather_decisions(local, total, w)
    # the hot-loop form: write into the preallocated slot, gather in place (twice: reusable)
    g = D.DecisionGather(total, w, r, torch.device("cpu"))
    for _ in range(2):
        g.slot.copy_(local)
        assert torch.equal(g.gather(), full)
    # two-phase (overlapped) gather: chunks r and w + r of 2w, evaluated and gathered half by half
    g2 = D.TwoPhaseGather(total, w, r, torch.device("cpu"))
    dec = ((np.arange(total) * 7 + 3) % 3).astype(np.uint8)     # stand-in decisions, a function of the index
    for half, (a, b) in enumerate(g2.ranges):
        g2.slots[half].copy_(torch.from_numpy(dec[a:b]))
        g2.gather(half)
    assert g2.wait().numpy().tolist() == dec.tolist()
    st = torch.tensor([0, 6 * rank, 0, rank], dtype=torch.uint8)
    assert D.all_reduce_max_(st, w).tolist() == [0, 6, 0, 1]
    t = D.max_over_ranks(float(rank + 1), w, torch.device("cpu"))
    s = D.sum_over_ranks(c1 - c0, w, torch.device("cpu"))
    # config-4 partial counters: parts near 2^62 sum exactly (int64, no float staging)
    part = torch.tensor([[(1 << 62) - 7 + rank, rank, 3 * rank + 1]], dtype=torch.int64)
    red = D.all_reduce_sum_(part, w).tolist()
    q.put((rank, full.numpy().tobytes(), t, s, red))
    dist.destroy_process_group()


@pytest.mark.parametrize("total", [1001, 4096])
def test_gather_decisions_two_ranks_gloo(total):
    import gen
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, total, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    b = gen.generate(5, 0, total)
    # every rank sees the same full vector, in candidate order, equal to a 1-rank run
    nests_global = np.concatenate([gen.generate(5, *D.shard_range(total, r, 2)).cands["nest_id"] for r in range(2)])
    devs = b.cands["device_id"]
    expect = ((nests_global + devs) % 3).astype(np.uint8)
    for rank, full, t, s, red in res:
        assert np.frombuffer(full, np.uint8).tolist() == expect.tolist()
        assert t == 2.0 and s == total
        assert red == [[2 * ((1 << 62) - 7) + 1, 1, 5]]
