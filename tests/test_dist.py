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
            assert max(sizes) - min(sizes) <= 1
            assert max(sizes) <= D.padded_len(total, world)


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
