"""Multi-GPU plumbing: one process per GPU, candidates sharded by index range.

Candidates are independent: each rank evaluates a contiguous
range of the candidate index space with no data-path exchange; the only
collective is the all-gather of the per-candidate decisions the north star
asks for (NCCL over NVLink / NVSwitch on a GPU box, gloo in the CPU tests).
Ranges are padded to a common length so a single ``all_gather_into_tensor``
suffices; padding bytes are dropped after the gather.  Config 4 (a few huge
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


def shard_range(total: int, rank: int, world: int):
    """Contiguous candidate range [c0, c1) of ``rank``; sizes differ by <= 1.
    The c5 index interleave (device, launch, kernel in the low digits) makes
    equal-count ranges near-equal work."""
    base, rem = divmod(total, world)
    c0 = rank * base + min(rank, rem)
    return c0, c0 + base + (1 if rank < rem else 0)


def padded_len(total: int, world: int) -> int:
    return -(-total // world)


def gather_decisions(local: torch.Tensor, total: int, world: int, out: torch.Tensor | None = None,
                     group=None) -> torch.Tensor:
    """All-gather uint8 decisions of every rank's shard into a ``total``-long
    vector in candidate order (identical on every rank)."""
    if world == 1:
        return local
    n_pad = padded_len(total, world)
    buf = torch.zeros(n_pad, dtype=torch.uint8, device=local.device)
    buf[: local.numel()].copy_(local)
    full = torch.empty(n_pad * world, dtype=torch.uint8, device=local.device) if out is None else out
    if _host_staged(buf):
        hfull = torch.empty(n_pad * world, dtype=torch.uint8)
        dist.all_gather_into_tensor(hfull, buf.cpu(), group=group)
        full.copy_(hfull)
    else:
        dist.all_gather_into_tensor(full, buf, group=group)
    parts = []
    for r in range(world):
        c0, c1 = shard_range(total, r, world)
        parts.append(full[r * n_pad: r * n_pad + (c1 - c0)])
    return torch.cat(parts)


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


def evaluate_split(cands: torch.Tensor, tables, workspace: torch.Tensor, rank: int, world: int, flags: int = 0,
                   group=None) -> dict:
    """a few huge candidates, so every rank takes ALL
    candidates but only its 1/world slice of their warp-accesses
    (``sel_count_transactions_part``); one ``all_reduce(SUM)`` of the u64
    counters makes them exact and every rank then runs a4-a7 identically."""
    from . import count_transactions, predict_gpu_cycles, select
    counts, status = count_transactions(cands, tables, workspace, flags, part=rank, n_parts=world)
    all_reduce_sum_(counts, world, group)
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
