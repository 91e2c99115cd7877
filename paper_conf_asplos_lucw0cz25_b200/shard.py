"""Proof sharding across GPUs -- host logic only.

Proofs are independent, so a batch shards by proof with no data-path collective: rank r proves
the contiguous global indices [r*B/W, (r+1)*B/W) (or, for weak scaling, [r*B, (r+1)*B)).  The
global index enters the transcript (``first_index``), so every proof's bytes are identical for
any world size.  torch.distributed (NCCL on GPUs, gloo in the CPU tests) is used only after the
timed region: to take the max of the per-rank device times and to gather outputs/digests.
"""
from __future__ import annotations

import hashlib


def shard_range(global_batch: int, world: int, rank: int) -> tuple[int, int]:
    """[first, first + count) for a strong-scaling split (balanced, contiguous)."""
    base, rem = divmod(global_batch, world)
    first = rank * base + min(rank, rem)
    return first, base + (1 if rank < rem else 0)


def weak_range(per_rank: int, rank: int) -> tuple[int, int]:
    """[first, first + per_rank) for weak scaling (fixed work per GPU)."""
    return rank * per_rank, per_rank


def output_digest(arrays) -> str:
    """SHA-256 over the raw bytes of the output arrays (numpy or torch CPU tensors), in order."""
    h = hashlib.sha256()
    for a in arrays:
        h.update(a.numpy().tobytes() if hasattr(a, "numpy") else a.tobytes())
    return h.hexdigest()


def _dev(dist, device):
    """NCCL needs CUDA tensors; gloo (CPU tests, single-GPU smoke runs) takes CPU tensors."""
    return device if dist.get_backend() == "nccl" else None


def max_over_ranks(value: float, dist, device=None) -> float:
    """Max of a per-rank scalar (the device time of the timed region)."""
    import torch
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=_dev(dist, device))
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_bytes(blob: bytes, dist, device=None) -> list[bytes]:
    """All-gather one fixed-size byte string per rank."""
    import torch
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return [blob]
    t = torch.tensor(list(blob), dtype=torch.uint8, device=_dev(dist, device))
    out = [torch.zeros_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(out, t)
    return [bytes(x.cpu().tolist()) for x in out]


def gather_outputs(tensors: dict, dist, dst: int = 0):
    """Gather each rank's output tensors to rank ``dst`` (torch.distributed.gather: only ``dst``
    receives), concatenated along the proof dimension in rank order.  Ranks may hold different proof
    counts (strong scaling with a remainder): every rank pads to the largest count and ``dst`` trims.
    Returns the dict on ``dst``, None elsewhere."""
    import torch
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return tensors
    world, rank = dist.get_world_size(), dist.get_rank()
    nccl = dist.get_backend() == "nccl"
    any_t = next(iter(tensors.values()))
    dev = any_t.device if (nccl and any_t.is_cuda) else torch.device("cpu")
    cnt = torch.tensor([any_t.shape[0]], dtype=torch.int64, device=dev)
    counts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(counts, cnt)
    counts = [int(c.item()) for c in counts]
    top = max(counts)
    out = {}
    for key in sorted(tensors):
        t = tensors[key].to(dev).contiguous()
        if t.shape[0] < top:
            t = torch.cat([t, t.new_zeros((top - t.shape[0],) + tuple(t.shape[1:]))])
        parts = [torch.empty_like(t) for _ in range(world)] if rank == dst else None
        dist.gather(t, parts, dst=dst)
        if rank == dst:
            out[key] = torch.cat([p[:c] for p, c in zip(parts, counts)], dim=0)
    return out if rank == dst else None
