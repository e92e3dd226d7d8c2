"""Multi-GPU plumbing: one process per GPU, candidates sharded by index range.

Candidates are independent: each rank evaluates a contiguous
range of the candidate index space with no data-path exchange; the only
collective is the all-gather of the per-candidate decisions the north star
asks for (NCCL over NVLink / NVSwitch on a GPU box, gloo in the CPU tests).
Rank r owns [r * n_pad, (r + 1) * n_pad) with n_pad = ceil(total / world), so
the ranks' slots of ONE preallocated buffer hold every decision in candidate
order: each rank evaluates straight into its slot and a single in-place
``all_gather_into_tensor`` fills the rest (``DecisionGather``; no
allocation, zero-fill or concatenation per step).  ``weighted_ranges`` cuts
the index space at equal shares of a per-candidate work prefix instead
(cut points at k * sum(W) / R).  Config 4 (a few huge
candidates) splits each candidate's warp-accesses instead (``evaluate_split``).
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def init(backend: str | None = None):
    """Initialise the default process group from the torchrun environment
    (no-op for a single process).  Returns (rank, world, device_index).

    One process per GPU over NCCL by default.  SEL_DIST_BACKEND=gloo selects
    host-staged collectives instead, which lets several ranks share one GPU
    (device = local_rank mod #GPUs) -- used to exercise the multi-rank bench
    path on a single-GPU box; it is not the performance configuration."""
    rank, world, local = env_rank_world()
    backend = backend or os.environ.get("SEL_DIST_BACKEND")
    dev_index = local
    if torch.cuda.is_available():
        dev_index = local % torch.cuda.device_count()
    if world > 1 and not dist.is_initialized():
        if backend is None:
            backend = "nccl" if torch.cuda.is_available() else "gloo"
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if backend == "nccl":
            torch.cuda.set_device(dev_index)
            dist.init_process_group(backend, device_id=torch.device("cuda", dev_index))
        else:
            if torch.cuda.is_available():
                torch.cuda.set_device(dev_index)
            dist.init_process_group(backend)
    elif torch.cuda.is_available():
        torch.cuda.set_device(dev_index)
    return rank, world, dev_index


def _host_staged(t: torch.Tensor) -> bool:
    """gloo collectives on CUDA tensors are staged through host memory."""
    return t.is_cuda and dist.is_initialized() and dist.get_backend() == "gloo"


def padded_len(total: int, world: int) -> int:
    return -(-total // world)


def shard_range(total: int, rank: int, world: int):
    """Contiguous candidate range [c0, c1) of ``rank``: [r n_pad, (r+1) n_pad)
    clipped to ``total`` (n_pad = ceil(total / world)), so rank r's padded
    slot of the gather buffer starts at candidate r * n_pad.  The c5 index
    interleave (device, launch, kernel in the low digits) makes equal-count
    ranges near-equal work."""
    n_pad = padded_len(total, world)
    c0 = min(total, rank * n_pad)
    return c0, min(total, c0 + n_pad)


def weighted_ranges(prefix, world: int):
    """Cut points of a work-balanced partition: ``prefix`` is the inclusive
    prefix sum of per-candidate work (e.g. the closed-form W = WR * M_it of
    each candidate), rank r gets [cut_r, cut_{r+1}) with cut_r the first
    index whose prefix reaches r * total / world.  Contiguous, covering,
    deterministic; ranks may be empty."""
    import numpy as np
    p = np.asarray(prefix)
    n = len(p)
    total = int(p[-1]) if n else 0
    cuts = [0]
    for r in range(1, world):
        cuts.append(int(np.searchsorted(p, (total * r + world - 1) // world, side="left")) if total else n * r // world)
    cuts.append(n)
    cuts = [min(max(c, cuts[i - 1] if i else 0), n) for i, c in enumerate(cuts)]
    return [(cuts[r], cuts[r + 1]) for r in range(world)]

class DecisionGather:
    """Preallocated all-gather of the u8 decisions.  ``slot`` is
    this rank's shard inside the gather buffer: pass it as the decision output
    of ``sel_evaluate`` and ``gather()`` runs one in-place
    ``all_gather_into_tensor`` (the send buffer IS the rank's chunk of the
    receive buffer); ``gather()[:total]`` is every decision in candidate
    order, identical on every rank.  Padding bytes (past ``total``) are set to
    SEL_DECISION_INVALID once, at construction."""

    def __init__(self, total: int, world: int, rank: int, device, group=None):
        self.total, self.world, self.rank, self.group = total, world, rank, group
        self.n_pad = padded_len(total, world)
        self.buf = torch.full((self.n_pad * world,), 0xFF, dtype=torch.uint8, device=device)
        c0, c1 = shard_range(total, rank, world)
        self.chunk = self.buf[rank * self.n_pad:(rank + 1) * self.n_pad]
        self.slot = self.chunk[: c1 - c0]
        self._host = torch.empty(self.n_pad * world, dtype=torch.uint8) if _host_staged(self.buf) else None

    def gather(self) -> torch.Tensor:
        if self.world > 1:
            if self._host is not None:
                dist.all_gather_into_tensor(self._host, self.chunk.cpu(), group=self.group)
                self.buf.copy_(self._host)
            else:
                dist.all_gather_into_tensor(self.buf, self.chunk, group=self.group)
        return self.buf[: self.total]


class TwoPhaseGather:
    """The all-gather of decisions overlapped with the evaluation (VERDICT r01
    #8): the index space is cut into 2 * world chunks of m = ceil(total /
    (2 world)) candidates and rank r owns chunks r and world + r, so the first
    halves of all ranks are the contiguous range [0, world m) and the second
    halves [world m, 2 world m).  The rank evaluates its first chunk into
    ``slots[0]``, starts ``gather(0)`` (NCCL runs it on its own stream, after
    the kernels already enqueued on the current stream), evaluates its second
    chunk into ``slots[1]`` while the first gather is in flight, gathers the
    second half, and ``wait()`` joins both; ``buf[:total]`` then holds every
    decision in candidate order.  One preallocated buffer, in-place
    collectives, no copies."""

    def __init__(self, total: int, world: int, rank: int, device, group=None):
        self.total, self.world, self.rank, self.group = total, world, rank, group
        self.m = -(-total // (2 * world)) if total else 0
        m = self.m
        self.buf = torch.full((2 * world * m,), 0xFF, dtype=torch.uint8, device=device)
        self.ranges = [(min(total, j * m), min(total, (j + 1) * m)) for j in (rank, world + rank)]
        self.slots = [self.buf[j * m: j * m + (b - a)] for j, (a, b) in zip((rank, world + rank), self.ranges)]
        self.sends = [self.buf[j * m:(j + 1) * m] for j in (rank, world + rank)]
        self.halves = [self.buf[:world * m], self.buf[world * m:]]
        self._host = _host_staged(self.buf)
        self._work = []

    def gather(self, half: int):
        if self.world == 1:
            return
        if self._host:
            h = torch.empty(self.world * self.m, dtype=torch.uint8)
            dist.all_gather_into_tensor(h, self.sends[half].cpu(), group=self.group)
            self.halves[half].copy_(h)
        else:
            self._work.append(dist.all_gather_into_tensor(self.halves[half], self.sends[half], group=self.group,
                                                          async_op=True))

    def wait(self) -> torch.Tensor:
        for wk in self._work:
            wk.wait()
        self._work = []
        return self.buf[: self.total]


def gather_decisions(local: torch.Tensor, total: int, world: int, group=None) -> torch.Tensor:
    """All-gather uint8 decisions of every rank's shard (``shard_range``) into a
    ``total``-long vector in candidate order (identical on every rank).  A
    convenience that copies ``local`` into a fresh ``DecisionGather``; the hot
    loop evaluates into ``DecisionGather.slot`` directly."""
    if world == 1:
        return local
    g = DecisionGather(total, world, dist.get_rank(group), local.device, group)
    g.slot.copy_(local)
    return g.gather()


def all_reduce_sum_(t: torch.Tensor, world: int, group=None) -> torch.Tensor:
    """In-place element-wise SUM over ranks (exact for integer tensors)."""
    if world == 1:
        return t
    if _host_staged(t):
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        t.copy_(h)
    else:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def all_reduce_max_(t: torch.Tensor, world: int, group=None) -> torch.Tensor:
    """In-place element-wise MAX over ranks."""
    if world == 1:
        return t
    if _host_staged(t) or t.dtype == torch.uint8:
        h = t.to(torch.int32)
        h = h.cpu() if _host_staged(t) else h
        dist.all_reduce(h, op=dist.ReduceOp.MAX, group=group)
        t.copy_(h)
    else:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return t


def evaluate_split(cands: torch.Tensor, tables, workspace: torch.Tensor, rank: int, world: int, flags: int = 0,
                   group=None) -> dict:
    """a few huge candidates, so every rank takes ALL
    candidates but only its 1/world slice of their warp-accesses
    (``sel_count_transactions_part``); one ``all_reduce(SUM)`` of the u64
    counters makes them exact and every rank then runs a4-a7 identically."""
    from . import count_transactions, predict_gpu_cycles, select
    counts, status = count_transactions(cands, tables, workspace, flags, part=rank, n_parts=world)
    all_reduce_sum_(counts, world, group)
    # a rank whose self-check failed (SEL_EINTERNAL) contributed no counts: every
    # rank takes the worst status, so no rank models incomplete counts
    all_reduce_max_(status, world, group)
    cycles, t_gpu = predict_gpu_cycles(cands, tables, counts, status)
    decision = select(cands, t_gpu, status)
    return dict(counts=counts, status=status, cycles=cycles, t_gpu=t_gpu, decision=decision)


def max_over_ranks(x: float, world: int, device) -> float:
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    if _host_staged(t):
        t = t.cpu()
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x: int, world: int, device) -> int:
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.int64, device=device)
    if _host_staged(t):
        t = t.cpu()
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return int(t.item())


def barrier(world: int):
    if world > 1:
        dist.barrier()
