"""Multi-GPU plumbing (one process per GPU, torch.distributed over NCCL).

The paper runs on a single GPU (§IV).  The path shards
naturally: outer tuples are independent (Fig. 2), so R is split
into contiguous row blocks, one per rank; the inner relation is needed whole
on every rank.  The one real exchange step is therefore

  * a broadcast of the invariant inner side (S's columns, and the built index
    so only rank 0 sorts) from rank 0 -- over NVLink/NVSwitch via NCCL,
    directly into tensor views of each rank's engine arena;
  * a gather of the variable-length survivor lists to rank 0 (NCCL has no
    gatherv: counts are all-gathered first, payloads padded to the max).

The helpers move tensors only; they work with NCCL (GPU box) and gloo (CPU
tests, or several ranks sharing one GPU: gloo collectives that do not take
CUDA tensors are staged through host memory).
"""
import os

import torch
import torch.distributed as dist


def backend_name():
    return os.environ.get("NESTGPU_DIST_BACKEND", "nccl")


def _is_gloo(group=None):
    return dist.get_backend(group) == "gloo"


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


def broadcast_ints(values, src=0, device="cpu", group=None):
    dev = "cpu" if _is_gloo(group) else device
    t = torch.tensor([int(v) for v in values], dtype=torch.int64, device=dev)
    dist.broadcast(t, src=src, group=group)
    return [int(v) for v in t.tolist()]


def broadcast_int(value, src=0, device="cpu", group=None):
    return broadcast_ints([value], src=src, device=device, group=group)[0]


def gather_rows(parts, dst=0, group=None):
    """Gather variable-length 1-D tensors (same dtype per position in `parts`)
    from every rank to `dst`.  Returns the per-field concatenation in rank
    order on dst, None elsewhere.  Collective: every rank must call it."""
    world = dist.get_world_size(group)
    dev = parts[0].device
    stage = _is_gloo(group) and dev.type != "cpu"     # gloo all_gather takes CPU tensors
    cdev = torch.device("cpu") if stage else dev
    n = torch.tensor([parts[0].numel()], dtype=torch.int64, device=cdev)
    counts = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(counts, n, group=group)
    counts = [int(c.item()) for c in counts]
    mx = max(counts) if counts else 0
    out = []
    for p in parts:
        pad = torch.zeros(mx, dtype=p.dtype, device=cdev)
        pad[:p.numel()] = p.to(cdev)
        bufs = [torch.zeros_like(pad) for _ in range(world)]
        dist.all_gather(bufs, pad, group=group)
        out.append(torch.cat([b[:c] for b, c in zip(bufs, counts)]).to(dev) if dist.get_rank(group) == dst else None)
    return out if dist.get_rank(group) == dst else None


def max_over_ranks(x, device="cpu", group=None):
    dev = "cpu" if (dist.is_available() and dist.is_initialized() and _is_gloo(group)) else device
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


# ------------------------------------------------------------------ engine-level
def share_table(eng, host_cols, names, n, dtypes=None, device=None, group=None):
    """Rank 0 loads `host_cols` ({name: array}); every other rank reserves
    the same columns in its arena and receives their bytes by broadcast.
    Returns {name: column id} on every rank.  NOT NULL columns only."""
    dtypes = dtypes or {}
    rank = dist.get_rank(group)
    if rank == 0:
        cols = {k: eng.load_column(host_cols[k], dtype=dtypes.get(k)) for k in names}
    else:
        cols = {k: eng.alloc_column(n, dtypes.get(k) or "int32") for k in names}
    views = []
    for k in names:
        info = eng.column_info(cols[k])
        w = 4 if info["dtype"] in (0, 3, 4) else 8
        views.append(eng.arena_view(info["d_values"], n * w))
    broadcast_tensors(views, group=group)
    return cols


def share_index(eng, S, key, payload, inner_preds=(), device=None, group=None):
    """Rank 0 builds the correlated-column index (filter + radix sort);
    the sorted keys and payload are broadcast into an index of the same shape
    reserved on every other rank.  Returns the index id on every rank."""
    rank = dist.get_rank(group)
    if rank == 0:
        idx = eng.build_index(S, key, payload, inner_preds)
        info = eng.index_info(idx)
        shape = [info["n"], info["key_bytes"], info["payload_bytes"]]
    else:
        shape = [0, 0, 0]
    n, kb, vb = broadcast_ints(shape, device=device, group=group)
    if rank != 0:
        idx, info = eng.index_create_empty(S, key, payload, inner_preds, n, kb, vb)
    views = [eng.arena_view(info["d_keys"], n * kb)]
    if vb:
        views.append(eng.arena_view(info["d_payload"], n * vb))
    broadcast_tensors(views, group=group)
    return idx


def gather_result(eng, res, group=None):
    """Gather one exec result's (row id, value, valid, passed) to rank 0 (row
    ids are global when the shard passed row_id_base)."""
    t = eng.result_tensors(res)
    return gather_rows([t["row"].clone(), t["value"].clone(), t["valid"].clone(), t["passed"].clone()], group=group)
