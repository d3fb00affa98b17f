"""Multi-process (world_size 2, gloo, CPU) tests of the sharding / broadcast /
gather host logic the multi-GPU bench uses (paper_conf_icde_floratosxwgylz21_b200.dist),
including an end-to-end check that sharded oracle evaluation + gather equals
the single-process result (outer tuples are independent)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icde_floratosxwgylz21_b200 import dist as ngd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from datagen import make_plan, query1
        t = query1.config("C1")
        n = len(t["R"]["col1"])
        lo, hi = ngd.shard_range(n, rank, world)
        # broadcast of the inner side: rank 0 owns S, others receive it
        s1 = torch.from_numpy(t["S"]["col1"].copy()) if rank == 0 else torch.zeros(len(t["S"]["col1"]), dtype=torch.int32)
        s2 = torch.from_numpy(t["S"]["col2"].copy()) if rank == 0 else torch.zeros(len(t["S"]["col2"]), dtype=torch.int32)
        nS = ngd.broadcast_int(len(s1) if rank == 0 else -1)
        assert ngd.broadcast_ints([7, rank]) == [7, 0]
        assert nS == len(s1)
        ngd.broadcast_tensors([s1, s2])
        shard = {"R": {k: v[lo:hi] for k, v in t["R"].items()}, "S": {"col1": s1.numpy(), "col2": s2.numpy()}}
        plan = make_plan(">", "min", "=")
        res = oracle.evaluate(shard, plan)
        rows, vals = oracle.survivors(res)
        got = ngd.gather_rows([torch.from_numpy(rows + lo), torch.from_numpy(vals)])
        mx = ngd.max_over_ranks(float(rank + 1))
        if rank == 0:
            full = oracle.evaluate(t, plan)
            er, ev = oracle.survivors(full)
            q.put(("ok", np.array_equal(got[0].numpy(), er) and np.array_equal(got[1].numpy(), ev), mx))
        else:
            assert got is None
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e), None))
        raise
    finally:
        dist.destroy_process_group()


def test_shard_range_partitions():
    for n in (0, 1, 7, 1000, 1000003):
        for w in (1, 2, 3, 8):
            parts = [ngd.shard_range(n, r, w) for r in range(w)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(parts, parts[1:]))
            sizes = [h - l for l, h in parts]
            assert max(sizes) - min(sizes) <= 1


def test_gloo_world2_broadcast_shard_gather():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs)
    status, ok, mx = q.get(timeout=10)
    assert status == "ok" and ok
    assert mx == 2.0


def test_launch_ranks_world4(tmp_path):
    """The spawn path of `bench.py --gpus N` outside torchrun
    (dist.launch_ranks -> torchrun on 127.0.0.1) at world 4 with gloo: shard
    one R, gather the survivors to rank 0 only (point-to-point, one rank with
    an empty shard), compare with the whole-R result."""
    out = tmp_path / "verdict.json"
    env = dict(os.environ, NESTGPU_DIST_BACKEND="gloo")
    rc = ngd.launch_ranks(os.path.join(os.path.dirname(__file__), "dist_worker.py"), [str(out)], 4, env=env,
                          timeout=300)
    assert rc == 0
    import json
    v = json.loads(out.read_text())
    assert v["world"] == 4 and v["ok"] and v["plans"] == 4
    assert v["counts_ok"] and v["max"] == 3.0 and v["sum"] == 4.0
