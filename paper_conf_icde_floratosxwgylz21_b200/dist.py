"""Multi-GPU plumbing (one process per GPU, torch.distributed over NCCL).

The paper runs on a single GPU (§IV).  The path shards
naturally: outer tuples are evaluated independently (Fig. 2), so
ONE R is split into contiguous row blocks, one per rank (strong scaling; the
global row id of a shard's first row is passed to the engine as
``row_id_base``); the inner relation is needed whole on every rank.  The
exchange steps are therefore

  * a broadcast of the invariant inner side (S's columns, and the built index
    so only rank 0 sorts) from rank 0 -- over NVLink/NVSwitch via NCCL,
    directly into tensor views of each rank's engine arena;
  * a gather of the variable-length survivor lists to rank 0 only: the
    counts are exchanged (8 B per rank), then either every rank STORES its
    rows into a window on rank 0 from its own kernel (PeerGather: CUDA IPC
    peer memory, over NVLink/NVSwitch between GPUs -- the default of
    bench.py) or sends them with point-to-point NCCL sends (gather_rows: one
    grouped batch) -- rank 0 receives each survivor once, no padding and no
    copy on the other ranks.

The helpers move tensors only; they work with NCCL (GPU box) and gloo (CPU
tests, or several ranks sharing one GPU: gloo collectives that do not take
CUDA tensors are staged through host memory).

``launch_ranks`` starts the N-rank job (torchrun, 127.0.0.1 rendezvous) when
a script is started without a torch.distributed environment.
"""
import glob
import os
import socket
import subprocess
import sys

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


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def in_distributed_env():
    return "WORLD_SIZE" in os.environ and "RANK" in os.environ


def launch_ranks(script, argv, n, env=None, timeout=None):
    """Run `script argv` as an n-rank job, one process per rank (torchrun
    --standalone-style rendezvous on 127.0.0.1), inheriting stdout/stderr.
    Returns the job's exit code.  Used by bench.py when it is started with
    --gpus N > 1 outside torchrun."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(int(n)),
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), script] + list(argv)
    e = dict(os.environ if env is None else env)
    e.setdefault("OMP_NUM_THREADS", "1")
    return subprocess.call(cmd, env=e, timeout=timeout)


def nccl_debug_setup(tag="nestgpu"):
    """Ask NCCL (before the communicator exists) to log its INIT subsystem to
    a per-process file, so the run can report what NCCL built (ranks,
    transports, NVLS) without NCCL writing into stdout.  Returns the pattern."""
    d = os.environ.get("TMPDIR", "/tmp")
    pat = os.path.join(d, "%s_nccl.%d" % (tag, os.getpid()))
    os.environ.setdefault("NCCL_DEBUG", "INFO")
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT,NVLS")
    os.environ.setdefault("NCCL_DEBUG_FILE", pat + ".%h.%p.log")
    return pat


def nccl_init_summary(pattern):
    """The lines of this process's NCCL INIT log that show the communicator
    (rank count, NVLS / channel setup, version)."""
    out = []
    for f in sorted(glob.glob(pattern + "*")):
        try:
            for ln in open(f, errors="replace"):
                if ("Init COMPLETE" in ln or "NCCL version" in ln or "NVLS" in ln or "nRanks" in ln
                        or "Connected all" in ln):
                    out.append(ln.strip()[-240:])
        except OSError:
            pass
    return out[:12]


def broadcast_tensors(tensors, src=0, group=None):
    """Broadcast each tensor in place from `src` (tensor views of the arena on
    the receiving ranks, so the bytes land where the engine reads them)."""
    for t in tensors:
        if t.numel():
            if _is_gloo(group) and t.is_cuda:
                h = t.cpu()
                dist.broadcast(h, src=src, group=group)
                t.copy_(h)
            else:
                dist.broadcast(t, src=src, group=group)


def broadcast_ints(values, src=0, device="cpu", group=None):
    dev = "cpu" if _is_gloo(group) else device
    t = torch.tensor([int(v) for v in values], dtype=torch.int64, device=dev)
    dist.broadcast(t, src=src, group=group)
    return [int(v) for v in t.tolist()]


def broadcast_int(value, src=0, device="cpu", group=None):
    return broadcast_ints([value], src=src, device=device, group=group)[0]


def all_counts(n, device="cpu", group=None):
    """Every rank's n (one int64 per rank, all-gathered)."""
    world = dist.get_world_size(group)
    dev = "cpu" if _is_gloo(group) else device
    t = torch.tensor([int(n)], dtype=torch.int64, device=dev)
    bufs = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(bufs, t, group=group)
    return [int(b.item()) for b in bufs]


def gather_rows(parts, dst=0, group=None):
    """Gather variable-length 1-D tensors (same length within a rank, same
    dtype per position in `parts`) from every rank to `dst` only.  Returns the
    per-field concatenation in rank order on dst, None elsewhere.
    Collective: every rank must call it.

    Counts first (8 B per rank), then one grouped batch of point-to-point
    transfers into exactly-sized buffers on dst: dst receives sum(counts)
    rows once per field; no rank pads or receives anything else."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    dev = parts[0].device
    gloo = _is_gloo(group)
    cdev = torch.device("cpu") if (gloo and dev.type != "cpu") else dev
    counts = all_counts(parts[0].numel(), device=dev, group=group)
    if world == 1:
        return list(parts)
    ops, recv = [], {}
    peer = (lambda r: dist.get_global_rank(group, r)) if group is not None else (lambda r: r)
    if rank == dst:
        for r in range(world):
            if r == dst or counts[r] == 0:
                continue
            for i, p in enumerate(parts):
                buf = torch.empty(counts[r], dtype=p.dtype, device=cdev)
                recv[(r, i)] = buf
                ops.append(dist.P2POp(dist.irecv, buf, peer(r), group))
    elif counts[rank]:
        for p in parts:
            ops.append(dist.P2POp(dist.isend, p.contiguous().to(cdev), peer(dst), group))
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()
    if rank != dst:
        return None
    out = []
    for i, p in enumerate(parts):
        pieces = [p if r == dst else recv[(r, i)].to(dev) for r in range(world) if counts[r] and (r == dst or (r, i) in recv)]
        out.append(torch.cat(pieces) if pieces else p[:0])
    return out


def max_over_ranks(x, device="cpu", group=None):
    dev = "cpu" if (dist.is_available() and dist.is_initialized() and _is_gloo(group)) else device
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def sum_over_ranks(x, device="cpu", group=None):
    dev = "cpu" if (dist.is_available() and dist.is_initialized() and _is_gloo(group)) else device
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
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


class PeerGather:
    """Survivor gather by peer stores (nestgpu_window_* / nestgpu_result_put):
    rank 0 owns a window of `cap` rows; every rank maps it once (CUDA IPC: an
    NVLink/NVSwitch peer mapping across GPUs, the same memory for ranks that
    share a device) and, per gather, stores its survivors into it at its row
    offset from its own kernel.  The control path is two tiny host
    collectives -- the survivor counts (8 B per rank) and a barrier that
    orders the puts before rank 0 reads; no NCCL send/recv carries rows.
    Collective: every rank constructs it and calls gather()."""

    def __init__(self, eng, cap, device=None, group=None):
        self.eng, self.cap, self.group = eng, int(cap), group
        self.device = device if device is not None else eng.device
        self.rank = dist.get_rank(group)
        self.own = None
        if self.rank == 0:
            self.own, handle = eng.window_create(self.cap)
            h = torch.tensor(list(handle), dtype=torch.uint8)
        else:
            h = torch.zeros(64, dtype=torch.uint8)
        hd = h if _is_gloo(group) else h.to(self.device)
        dist.broadcast(hd, src=0, group=group)
        self.handle = bytes(hd.cpu().tolist())
        self.peer, self.error = self.own, None
        if self.rank != 0:
            try:
                self.peer = eng.window_open(self.handle)
            except Exception as e:   # no peer access between these devices
                self.peer, self.error = None, str(e)
        # every rank must agree: if any rank cannot map the window, nobody uses it
        ok = torch.tensor([0.0 if self.error else 1.0], dtype=torch.float64,
                          device="cpu" if _is_gloo(group) else self.device)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
        self.ok = bool(ok.item() > 0.5)
        if not self.ok:
            self.close()

    def gather(self, res):
        """Rank 0: (row ids, values) torch views of the gathered rows in rank
        order (valid until the next gather); other ranks: None."""
        counts = all_counts(res.n_rows, device=self.device, group=self.group)
        off = sum(counts[:self.rank])
        if sum(counts) > self.cap:
            raise ValueError("PeerGather: %d rows exceed the window's %d" % (sum(counts), self.cap))
        self.eng.result_put(res, self.peer, self.cap, off)   # synchronous: stores complete + visible
        dist.barrier(group=self.group)
        if self.rank != 0:
            return None
        return self.eng.window_tensors(self.own, self.cap, sum(counts))

    def close(self):
        if getattr(self, "_closed", False):
            return
        self._closed = True
        if self.rank == 0:
            dist.barrier(group=self.group)   # every peer has unmapped
            if self.own:
                self.eng.window_free(self.own)
                self.own = None
        else:
            if self.peer:
                self.eng.window_close(self.peer)
                self.peer = None
            dist.barrier(group=self.group)


def gather_result(eng, res, group=None):
    """Gather one exec result's (row id, value, valid, passed) to rank 0 (row
    ids are global when the shard passed row_id_base)."""
    t = eng.result_tensors(res)
    return gather_rows([t["row"], t["value"], t["valid"], t["passed"]], group=group)
