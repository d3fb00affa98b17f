"""Multi-GPU plumbing (one process per GPU, torch.distributed over NCCL).

The paper runs on a single GPU (§IV).  The path shards
naturally: outer tuples are independent (Fig. 2), so R is split
into contiguous row blocks, one per rank; the inner relation is needed whole
on every rank.  The one real exchange step is therefore

  * a broadcast of the invariant inner side (the built index, or S's
    columns for the nested-loop path) from rank 0 -- over NVLink/NVSwitch
    via NCCL, directly into tensor views of each rank's engine arena;
  * a gather of the variable-length survivor lists to rank 0 (NCCL has no
    gatherv: counts are all-gathered first, payloads padded to the max).

These helpers only move tensors; they work with any backend (NCCL on the
GPU box, gloo on CPU tensors in the tests).
"""
import torch
import torch.distributed as dist


def shard_range(n, rank, world):
    """Contiguous block [lo, hi) of n rows owned by `rank` (sizes differ by <= 1)."""
    base, extra = divmod(int(n), int(world))
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def broadcast_tensors(tensors, src=0, group=None):
    """Broadcast each tensor in place from `src` (tensor views of the arena on
    the receiving ranks, so the bytes land where the engine reads them)."""
    for t in tensors:
        if t.numel():
            dist.broadcast(t, src=src, group=group)


def broadcast_int(value, src=0, device="cpu", group=None):
    t = torch.tensor([int(value)], dtype=torch.int64, device=device)
    dist.broadcast(t, src=src, group=group)
    return int(t.item())


def gather_rows(parts, dst=0, group=None):
    """Gather variable-length 1-D tensors (same dtype per position in `parts`)
    from every rank to `dst`.  Returns the per-field concatenation in rank
    order on dst, None elsewhere.  Collective: every rank must call it."""
    world = dist.get_world_size(group)
    dev = parts[0].device
    n = torch.tensor([parts[0].numel()], dtype=torch.int64, device=dev)
    counts = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(counts, n, group=group)
    counts = [int(c.item()) for c in counts]
    mx = max(counts) if counts else 0
    out = []
    for p in parts:
        pad = torch.zeros(mx, dtype=p.dtype, device=dev)
        pad[:p.numel()] = p
        bufs = [torch.zeros_like(pad) for _ in range(world)]
        dist.all_gather(bufs, pad, group=group)
        out.append(torch.cat([b[:c] for b, c in zip(bufs, counts)]) if dist.get_rank(group) == dst else None)
    return out if dist.get_rank(group) == dst else None


def max_over_ranks(x, device="cpu", group=None):
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
